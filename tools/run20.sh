mkdir -p gpurun_out
rm -f gpurun_out/hs_sweep5.txt
echo "== c3" >> gpurun_out/hs_sweep5.txt
timeout 600 python tools/sweep.py --config c3 --variants 0 --runs 64 --formats coo --reps 10 >> gpurun_out/hs_sweep5.txt 2>&1
echo "== c3 rows 512 no L2 tier run 64" >> gpurun_out/hs_sweep5.txt
PASTA_HOT_MB=0 PASTA_HOT_SMEM_ROWS=512 timeout 600 python tools/sweep.py --config c3 --variants 0 --runs 64 --formats coo --reps 10 >> gpurun_out/hs_sweep5.txt 2>&1
timeout 900 python bench.py --steps 50 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 python bench.py --config c2 --steps 50 --no-cpu-baseline > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
