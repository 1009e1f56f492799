mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_basic.py -q > gpurun_out/pb.log 2>&1
for lib in libvp.so libvp_p4.so libvp_p5.so; do echo "== $lib"; VP_LIB_NAME=$lib timeout 300 python tools/pyr_time.py; done > gpurun_out/pyr_time3.log 2>&1
timeout 1200 python tools/suite_only.py > gpurun_out/suite.json 2> gpurun_out/suite.err
