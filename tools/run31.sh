mkdir -p gpurun_out
rm -f gpurun_out/sweep14.txt
PASTA_HS_CFG=3 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "random or hot_row" > gpurun_out/pytest_parity.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_parity.log
for CFG in h c5; do
  for HC in 1 2 3; do
  echo "== $CFG HS_CFG=$HC" >> gpurun_out/sweep14.txt
  PASTA_HS_CFG=$HC timeout 900 python tools/sweep.py --config $CFG --variants 0 --runs 0,128 --formats coo --reps 5 >> gpurun_out/sweep14.txt 2>&1
  done
done
