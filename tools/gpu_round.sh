#!/bin/bash
# Dev: one gpurun call = GPU tests + smoke + bench + ncu launch list + full captures of the top kernels.
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
if [ "$VP_TESTS" != "0" ]; then
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
fi
date +%s > gpurun_out/bench_t0; timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$? secs=$(( $(date +%s) - $(cat gpurun_out/bench_t0) ))" >> gpurun_out/bench.err
if [ "$VP_NCU" = "1" ]; then
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --no-suite --no-baselines --no-e2e --tune-seconds 10 > gpurun_out/b_ncu.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:vp_kernel -c 1 -o gpurun_out/rtc_leaf python tools/ncu_targets.py rtc_leaf --frames 64 --runs 1 > gpurun_out/ncu_full.log 2>&1
fi
if [ "$VP_NCU_WL" = "1" ]; then
bash tools/prof_cfd_pyr.sh > gpurun_out/prof_cfd_pyr.log 2>&1
fi
