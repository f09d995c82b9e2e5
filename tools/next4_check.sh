mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_next4.py tests/test_gpu_ghicoo.py -x -q > gpurun_out/pytest_next4.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_next4.log
timeout 900 python bench.py --steps 30 --warmup 3 > gpurun_out/bench2.log 2>&1; echo "rc=$?" >> gpurun_out/bench2.log
