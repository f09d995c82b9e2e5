mkdir -p gpurun_out
rm -f gpurun_out/sweep11.txt
for CFG in h c3; do
  echo "== $CFG" >> gpurun_out/sweep11.txt
  timeout 600 python tools/sweep.py --config $CFG --variants 0 --runs 0 --caches 0,4,8,16,24,28 --formats coo --reps 10 >> gpurun_out/sweep11.txt 2>&1
done
for MB in 32 96; do
  echo "== h HOT_MB=$MB" >> gpurun_out/sweep11.txt
  PASTA_HOT_MB=$MB timeout 600 python tools/sweep.py --config h --variants 0 --runs 0 --caches 0,24 --formats coo --reps 10 >> gpurun_out/sweep11.txt 2>&1
done
