bash tools/gpu_evidence.sh r02b micro l2_home_bench
mkdir -p gpurun_out/r02b
timeout 900 python bench.py --steps 20 --warmup 5 --hicoo-steps 5 --cpals-iters 2 --ew-steps 5 --e2e-steps 3 > gpurun_out/r02b/bench_h.json 2> gpurun_out/r02b/bench_h.err
timeout 2400 python -m pytest tests/test_gpu_cpals.py tests/test_gpu_parity_full.py tests/test_gpu_multirank.py -q -x > gpurun_out/r02b/pytest_new.log 2>&1; echo rc=$? >> gpurun_out/r02b/pytest_new.log
tail -5 gpurun_out/r02b/pytest_new.log; head -12 gpurun_out/r02b/micro_l2_home_bench.txt; tail -c 1500 gpurun_out/r02b/bench_h.json
