mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ttm.py tests/test_gpu_cpals.py tests/test_gpu_multirank.py -x -q > gpurun_out/pytest_parity.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_parity.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
