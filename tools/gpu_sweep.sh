mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_online.py -x -q > gpurun_out/pytest_online.log 2>&1
timeout 900 python tools/reyes_sweep.py --reps 2 --no-timers --online --configs h56b16_16_64_4,h60b16_16_64_4,h64b16_16_64_4 > gpurun_out/sweep7.log 2>&1
