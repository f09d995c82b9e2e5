mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_next4.py -x -q > gpurun_out/pytest_next4.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_next4.log
for V in 0 1 2 3 4; do PASTA_EW_VARIANT=$V timeout 300 python tools/ew_sweep.py; done > gpurun_out/ew_sweep.log 2>&1
bash tools/cache_sweep.sh h
