mkdir -p gpurun_out
rm -f gpurun_out/hs_sweep2.txt
for CFG in c2 c4 h c3; do
  for ROWS in 64 256 512 1024 1584; do
    echo "== $CFG HOT_SMEM=1 ROWS=$ROWS" >> gpurun_out/hs_sweep2.txt
    PASTA_HOT_SMEM_ROWS=$ROWS PASTA_HOT_SMEM=1 timeout 600 python tools/sweep.py --config $CFG --variants 0 --runs 128 --formats coo --reps 10 >> gpurun_out/hs_sweep2.txt 2>&1
  done
  echo "== $CFG HOT_SMEM=0" >> gpurun_out/hs_sweep2.txt
  PASTA_HOT_SMEM=0 timeout 600 python tools/sweep.py --config $CFG --variants 0 --runs 128 --formats coo --reps 10 >> gpurun_out/hs_sweep2.txt 2>&1
done
