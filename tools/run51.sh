mkdir -p gpurun_out
rm -f gpurun_out/sweep24.txt
for CFG in c2 h; do for R in 8 64; do for ST in 1 0; do
  echo "== $CFG R=$R STAGED=$ST" >> gpurun_out/sweep24.txt
  PASTA_COO_STAGED=$ST timeout 900 python tools/sweep.py --config $CFG --R $R --variants 0 --runs 0 --formats coo --reps 5 >> gpurun_out/sweep24.txt 2>&1
done; done; done
