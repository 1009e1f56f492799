mkdir -p gpurun_out
for lib in libvp.so libvp_r2.so; do echo "== $lib"; VP_LIB_NAME=$lib timeout 600 python tools/reyes_sweep.py --reps 3 --no-timers --configs h50b16_16_64_4,h54b16_16_64_4,h58b16_16_64_4,h62b16_16_64_4; done > gpurun_out/sweep14.log 2>&1
