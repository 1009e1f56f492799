# Dev: ncu --set full of the fused [Dice,Shade] kernel alone (source view summarised)
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:vp_kernel -c 1 -o gpurun_out/rtc_leaf${VP_TAG} python tools/ncu_targets.py rtc_leaf --frames 64 --runs 1 > gpurun_out/ncu_full${VP_TAG}.log 2>&1
ncu -i gpurun_out/rtc_leaf${VP_TAG}.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/rtc_leaf_src${VP_TAG}.csv 2>&1
python tools/ncu_summary.py gpurun_out/rtc_leaf${VP_TAG}.ncu-rep 40 > gpurun_out/rtc_leaf_sum${VP_TAG}.txt 2>&1
