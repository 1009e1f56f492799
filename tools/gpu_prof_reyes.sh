mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:vp_kernel -c 1 -o gpurun_out/rtc_leaf python tools/ncu_targets.py rtc_leaf --frames 64 --runs 1 > gpurun_out/ncu_full.log 2>&1
ncu -i gpurun_out/rtc_leaf.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/rtc_leaf_src.csv 2>&1
python tools/ncu_summary.py gpurun_out/rtc_leaf.ncu-rep 60 > gpurun_out/rtc_leaf_sum.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:vp_kernel -c 1 -o gpurun_out/bs python tools/ncu_targets.py bs_online --frames 32 --runs 1 > gpurun_out/ncu_bs.log 2>&1
ncu -i gpurun_out/bs.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/bs_src.csv 2>&1
python tools/ncu_summary.py gpurun_out/bs.ncu-rep 60 > gpurun_out/bs_sum.txt 2>&1
