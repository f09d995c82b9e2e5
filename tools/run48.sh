mkdir -p gpurun_out
rm -f gpurun_out/sweep23.txt
PASTA_HS_CFG=3 timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "random or hot_row" > gpurun_out/pytest_parity.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_parity.log
for CFG in c4 h c2; do for HC in 0 2 3; do
  echo "== $CFG HS_CFG=$HC" >> gpurun_out/sweep23.txt
  PASTA_HS_CFG=$HC timeout 900 python tools/sweep.py --config $CFG --variants 0 --runs 0 --formats coo --reps 10 >> gpurun_out/sweep23.txt 2>&1
done; done
