mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_ttm.py tests/test_gpu_parity.py tests/test_gpu_multirank.py -x -q > gpurun_out/pytest_ttm.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_ttm.log
timeout 900 python bench.py --steps 30 > gpurun_out/bench4.log 2>&1
