mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "shared_memory" > gpurun_out/pytest_hs.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_hs.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 python bench.py --config c2 --no-cpu-baseline > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
bash tools/profile_round3.sh r01d
