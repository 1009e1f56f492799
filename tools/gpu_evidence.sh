# Dev: one gpurun call = bench line + launch list of the bench command + full captures of both
# Reyes kernels (+ the JSONs bench.py reads).  TAG names the files under gpurun_out/.
mkdir -p gpurun_out
TAG=${TAG:-r2}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 600 --csv --log-file gpurun_out/${TAG}_launches_bench.csv python bench.py --steps 2 --warmup 3 --no-suite --no-baselines --no-e2e --no-qbench --tune-seconds 10 > gpurun_out/b_ncu.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:vp_kernel -c 1 -o gpurun_out/rtc_leaf python tools/ncu_targets.py rtc_leaf --frames 64 --runs 1 > gpurun_out/ncu_rtc.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:vp_kernel -c 1 -o gpurun_out/bs python tools/ncu_targets.py bs_online --frames 32 --runs 1 > gpurun_out/ncu_bs.log 2>&1
python tools/ncu_summary.py gpurun_out/rtc_leaf.ncu-rep 40 > gpurun_out/${TAG}_rtc_leaf.txt 2>&1
python tools/ncu_summary.py gpurun_out/bs.ncu-rep 40 > gpurun_out/${TAG}_bs_ncu_dfs.txt 2>&1
mkdir -p profiles && python tools/reyes_kernel_json.py $TAG gpurun_out/rtc_leaf.ncu-rep gpurun_out/ncu_rtc.log gpurun_out/bs.ncu-rep gpurun_out/ncu_bs.log > gpurun_out/kjson.log 2>&1
cp profiles/${TAG}_rtc_leaf_traffic.json profiles/${TAG}_reyes_kernels.json gpurun_out/ 2>/dev/null
date +%s > gpurun_out/bench_t0; timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$? secs=$(( $(date +%s) - $(cat gpurun_out/bench_t0) ))" >> gpurun_out/bench.err
