mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_reyes.py -x -q > gpurun_out/pytest_reyes.log 2>&1
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
timeout 900 python tools/reyes_sweep.py --no-timers --reps 2 --configs h28b16_16_64_4,h36b16_16_64_4,h44b16_16_64_4,h52b16_16_64_4,h60b16_16_64_4,h68b16_16_64_4 > gpurun_out/sweep3.log 2>&1
