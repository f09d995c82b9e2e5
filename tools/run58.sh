mkdir -p gpurun_out
timeout 900 python bench.py --config c3 --no-cpu-baseline --e2e-steps 3 --steps 20 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err
timeout 900 python bench.py --config c4 --no-cpu-baseline --e2e-steps 3 --steps 20 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err
timeout 1200 python bench.py --config c5 --no-cpu-baseline --e2e-steps 0 --hicoo-steps 0 --cpals-iters 0 --ew-steps 0 --steps 5 --warmup 3 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
