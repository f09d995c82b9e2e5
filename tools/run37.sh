mkdir -p gpurun_out
timeout 900 python bench.py --no-cpu-baseline --hicoo-steps 0 --cpals-iters 0 --ew-steps 10 --e2e-steps 0 --steps 10 > gpurun_out/bench.json 2> gpurun_out/bench.err
PASTA_HOT_SMEM=0 timeout 900 python bench.py --no-cpu-baseline --hicoo-steps 0 --cpals-iters 0 --ew-steps 10 --e2e-steps 0 --steps 10 > gpurun_out/bench_nohs.json 2> gpurun_out/bench_nohs.err
