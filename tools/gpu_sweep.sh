mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python tools/reyes_sweep.py --reps 3 --no-timers --configs h56b16_16_64_4,h57b16_16_64_4,h58b16_16_64_4,h59b16_16_64_4,h60b16_16_64_4,h58b16_16_48_4,h58b16_16_32_4,h58b8_16_64_4,h58b16_8_64_4 > gpurun_out/sweep13.log 2>&1
