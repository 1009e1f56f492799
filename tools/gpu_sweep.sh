mkdir -p gpurun_out
timeout 300 ./tools/div_check > gpurun_out/div_check.log 2>&1
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_reyes.py tests/test_gpu_edge.py tests/test_gpu_online.py -q > gpurun_out/pr.log 2>&1
timeout 900 python tools/reyes_sweep.py --reps 3 --no-timers --configs h58b16_16_64_4,h60b16_16_64_4,h62b16_16_64_4 > gpurun_out/sweep17.log 2>&1
