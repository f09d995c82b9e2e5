mkdir -p gpurun_out
rm -f gpurun_out/sweep27.txt
echo "== h runs" >> gpurun_out/sweep27.txt
timeout 900 python tools/sweep.py --config h --variants 0 --runs 32,64,96 --formats coo --reps 10 >> gpurun_out/sweep27.txt 2>&1
for ROWS in 256 1024; do
  echo "== h ROWS=$ROWS" >> gpurun_out/sweep27.txt
  PASTA_HOT_SMEM_ROWS=$ROWS timeout 900 python tools/sweep.py --config h --variants 0 --runs 0 --formats coo --reps 10 >> gpurun_out/sweep27.txt 2>&1
done
for MB in 48 80; do
  echo "== h HOT_MB=$MB" >> gpurun_out/sweep27.txt
  PASTA_HOT_MB=$MB timeout 900 python tools/sweep.py --config h --variants 0 --runs 0 --formats coo --reps 10 >> gpurun_out/sweep27.txt 2>&1
done
