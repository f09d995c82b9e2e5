mkdir -p gpurun_out
rm -f gpurun_out/sweep9.txt
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ttm.py tests/test_gpu_cpals.py -x -q > gpurun_out/pytest_parity.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_parity.log
for CFG in h c3; do
  for ROWS in 256 512 1024 1536; do
  echo "== $CFG ROWS=$ROWS" >> gpurun_out/sweep9.txt
  PASTA_HOT_SMEM_ROWS=$ROWS timeout 600 python tools/sweep.py --config $CFG --variants 0 --runs 0,32,128 --formats coo --reps 10 >> gpurun_out/sweep9.txt 2>&1
  done
done
for CFG in c2; do
  for ROWS in 512 1024 2096; do
  echo "== $CFG ROWS=$ROWS" >> gpurun_out/sweep9.txt
  PASTA_HOT_SMEM_ROWS=$ROWS timeout 600 python tools/sweep.py --config $CFG --variants 0 --runs 0,64,256 --formats coo --reps 10 >> gpurun_out/sweep9.txt 2>&1
  done
done
