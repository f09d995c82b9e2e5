mkdir -p gpurun_out
for MB in 64 128 256 512; do
  PASTA_HOT_MB=$MB timeout 600 python tools/sweep.py --config h --variants 0 --runs 128 --formats coo --reps 5 --caches 0,4,12 | sed "s/^/mb=$MB /"
done > gpurun_out/hot_budget.log 2>&1
