mkdir -p gpurun_out
rm -f gpurun_out/sweep10.txt
for MB in 0 16 32 48 64 96; do
  echo "== h HOT_MB=$MB" >> gpurun_out/sweep10.txt
  PASTA_HOT_MB=$MB timeout 600 python tools/sweep.py --config h --variants 0 --runs 0 --formats coo --reps 10 >> gpurun_out/sweep10.txt 2>&1
done
for MB in 0 32 64; do
  echo "== c3 HOT_MB=$MB" >> gpurun_out/sweep10.txt
  PASTA_HOT_MB=$MB timeout 600 python tools/sweep.py --config c3 --variants 0 --runs 0 --formats coo --reps 10 >> gpurun_out/sweep10.txt 2>&1
done
