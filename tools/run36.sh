mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ttm.py tests/test_gpu_cpals.py -x -q > gpurun_out/pytest_parity.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_parity.log
timeout 900 python bench.py --no-cpu-baseline --hicoo-steps 0 --cpals-iters 2 --ew-steps 0 --e2e-steps 0 > gpurun_out/bench.json 2> gpurun_out/bench.err
PASTA_HOT_SMEM=0 timeout 900 python bench.py --no-cpu-baseline --hicoo-steps 0 --cpals-iters 0 --ew-steps 0 --e2e-steps 0 --steps 10 > gpurun_out/bench_nohs.json 2> gpurun_out/bench_nohs.err
