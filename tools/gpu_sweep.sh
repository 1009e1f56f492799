mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_tuner.py tests/test_gpu_basic.py -q > gpurun_out/pt.log 2>&1
timeout 1200 python tools/suite_only.py > gpurun_out/suite.json 2> gpurun_out/suite.err
