mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python tools/diag_r1x.py 256 > gpurun_out/dr1x.log 2>&1
timeout 600 python tools/reyes_sweep.py --reps 3 --no-timers --configs h56b16_16_64_4,h60b16_16_64_4,mega > gpurun_out/sweep8.log 2>&1
