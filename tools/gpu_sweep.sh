mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_reyes.py -x -q > gpurun_out/pytest_reyes.log 2>&1
timeout 900 python tools/reyes_sweep.py --reps 2 --no-timers --configs mega,h60b16_16_64_4 > gpurun_out/sweep6.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:vp_kernel -c 1 -o gpurun_out/mega_local python tools/ncu_targets.py mega --frames 32 --runs 1 > gpurun_out/ncu_mega.log 2>&1
