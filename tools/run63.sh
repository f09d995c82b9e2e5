mkdir -p gpurun_out
timeout 900 python bench.py --no-cpu-baseline --steps 10 > gpurun_out/bench_a.json 2> gpurun_out/bench_a.err
timeout 900 python bench.py --no-cpu-baseline --hicoo-steps 0 --ew-steps 0 --e2e-steps 0 --steps 10 > gpurun_out/bench_b.json 2> gpurun_out/bench_b.err
