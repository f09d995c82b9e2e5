mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "allmodes or hot or random" > gpurun_out/pytest_parity.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_parity.log
timeout 900 python bench.py --no-cpu-baseline --hicoo-steps 0 --cpals-iters 0 --ew-steps 0 > gpurun_out/bench.json 2> gpurun_out/bench.err
