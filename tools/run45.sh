mkdir -p gpurun_out
rm -f gpurun_out/sweep20.txt
for P in 0 1; do for MB in 32 48 64; do
  echo "== h PERSIST=$P HOT_MB=$MB" >> gpurun_out/sweep20.txt
  PASTA_HOT_PERSIST=$P PASTA_HOT_MB=$MB timeout 900 python tools/sweep.py --config h --variants 0 --runs 0 --formats coo --reps 10 >> gpurun_out/sweep20.txt 2>&1
done; done
