mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cfd.py -m gpu -x -q > gpurun_out/pytest_cfd.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_cfd.log
(cd ab_base && timeout 300 python tools/cfd_time.py) > gpurun_out/cfd_base.txt 2>&1
timeout 300 python tools/cfd_time.py > gpurun_out/cfd_new.txt 2>&1
