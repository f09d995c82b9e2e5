mkdir -p gpurun_out
rm -f gpurun_out/sweep22.txt
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "hot" > gpurun_out/pytest_parity.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_parity.log
for P in 0 1; do for MB in 32 64; do
  echo "== h PERSIST=$P HOT_MB=$MB" >> gpurun_out/sweep22.txt
  PASTA_HOT_PERSIST=$P PASTA_HOT_MB=$MB timeout 900 python tools/sweep.py --config h --variants 0 --runs 0 --formats coo --reps 10 >> gpurun_out/sweep22.txt 2>&1
done; done
