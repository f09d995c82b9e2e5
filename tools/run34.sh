mkdir -p gpurun_out
rm -f gpurun_out/sweep15.txt
PASTA_HS_CFG=4 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "random or hot_row" > gpurun_out/pytest_parity.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_parity.log
for CFG in h c3 c2; do
  for HC in 2 4 5; do
  echo "== $CFG HS_CFG=$HC" >> gpurun_out/sweep15.txt
  PASTA_HS_CFG=$HC timeout 900 python tools/sweep.py --config $CFG --variants 0 --runs 0 --formats coo --reps 10 >> gpurun_out/sweep15.txt 2>&1
  done
done
