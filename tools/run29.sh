mkdir -p gpurun_out
timeout 2700 python -m pytest tests -m gpu -x -q -rs > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
rm -f gpurun_out/sweep12.txt
for HC in 1 0; do
  echo "== c5 HS_CFG=$HC" >> gpurun_out/sweep12.txt
  PASTA_HS_CFG=$HC timeout 900 python tools/sweep.py --config c5 --variants 0 --runs 0 --formats coo --reps 3 >> gpurun_out/sweep12.txt 2>&1
done
