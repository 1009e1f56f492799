mkdir -p gpurun_out
for lib in libvp.so libvp_p4.so libvp_p5.so; do echo "== $lib"; VP_LIB_NAME=$lib timeout 300 python tools/pyr_time.py; done > gpurun_out/pyr_time3.log 2>&1
