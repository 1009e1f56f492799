#!/bin/bash
# Dev: copy the outputs of tools/gpu_evidence.sh (gpurun_out/) into profiles/ with headers.
set -e
TAG=${TAG:-r2}
NOTE=${NOTE:-"round 2 final"}
python - "$TAG" <<'PY'
import json, sys
tag = sys.argv[1]
line = open("gpurun_out/bench.json").read().strip().splitlines()[-1]
json.dump(json.loads(line), open(f"profiles/{tag}_bench_full.json", "w"), indent=1)
PY
(echo "# fused [Dice,Shade] RTC kernel alone over 64 frames' leaves (tools/ncu_targets.py rtc_leaf --frames 64), $NOTE"; cat gpurun_out/${TAG}_rtc_leaf.txt) > profiles/${TAG}_rtc_leaf.txt
(echo "# [Bound,Split] depth-first kernel alone (tools/ncu_targets.py bs_online --frames 32), $NOTE"; cat gpurun_out/${TAG}_bs_ncu_dfs.txt) > profiles/${TAG}_bs_ncu_dfs.txt
cp gpurun_out/${TAG}_rtc_leaf_traffic.json gpurun_out/${TAG}_reyes_kernels.json profiles/
cp gpurun_out/${TAG}_launches_bench.csv profiles/${TAG}_launches_bench.csv
mkdir -p /tmp/ll_$$ && cp gpurun_out/${TAG}_launches_bench.csv /tmp/ll_$$/bench_tuned.csv
python tools/ncu_launch_summary.py /tmp/ll_$$ > /tmp/ll_$$/sum.txt
SHARE=$(python -c "import json; print(round(100*json.load(open('profiles/${TAG}_bench_full.json'))['roofline']['kernel_share_of_step'],1))")
(echo "ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 600 --csv python bench.py --steps 2 --warmup 3 --no-suite --no-baselines --no-e2e --no-qbench --tune-seconds 10"
 echo "(ncu serialises kernels: the tuned hybrid's two persistent groups cannot co-run, so under ncu the"
 echo "auto-tuner's hybrid candidates abort as not co-resident and fall back, and the tuner keeps the megakernel;"
 echo "the 600 captured launches are mostly tuner candidates (KBK waves). Shares are cold-cache and serialised."
 echo "In the timed bench step (no profiler) the fused [Dice,Shade] RTC kernel co-runs with the [Bound,Split]"
 echo "kernel and takes ${SHARE}% of the step's event time (profiles/${TAG}_bench_full.json"
 echo "roofline.kernel_share_of_step); single-kernel captures of both kernels: ${TAG}_rtc_leaf.txt, ${TAG}_bs_ncu_dfs.txt.)"
 cat /tmp/ll_$$/sum.txt) > profiles/${TAG}_launches_bench.txt
rm -rf /tmp/ll_$$
echo saved
