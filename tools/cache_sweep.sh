# COO kernel L2-policy / hot-row-budget sweep on one workload (default h)
CFG=${1:-h}
mkdir -p gpurun_out
for MB in 32 48 64 80; do
  PASTA_HOT_MB=$MB timeout 600 python tools/sweep.py --config $CFG --variants 0 --runs 128 --formats coo --reps 5 --caches 0,8,16,24 > gpurun_out/cache_${CFG}_mb$MB.log 2>&1
done
