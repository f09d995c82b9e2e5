mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_ttm.py -x -q > gpurun_out/pytest_ttv.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_ttv.log
timeout 900 python bench.py --steps 10 --hicoo-steps 0 --cpals-iters 0 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench5.log 2>&1
PASTA_TTV_SEGSUM=0 timeout 900 python bench.py --steps 10 --hicoo-steps 0 --cpals-iters 0 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench5b.log 2>&1
