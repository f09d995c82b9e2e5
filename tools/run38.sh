mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_ttm.py -x -q > gpurun_out/pytest_ttm.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_ttm.log
timeout 900 python bench.py --no-cpu-baseline --hicoo-steps 0 --cpals-iters 0 --ew-steps 10 --e2e-steps 0 --steps 10 > gpurun_out/bench.json 2> gpurun_out/bench.err
