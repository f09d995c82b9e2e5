mkdir -p gpurun_out
rm -f gpurun_out/sweep18.txt
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ttm.py -x -q > gpurun_out/pytest_parity.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_parity.log
for CFG in c2 c4 h; do
  echo "== $CFG" >> gpurun_out/sweep18.txt
  timeout 900 python tools/sweep.py --config $CFG --variants 0 --runs 0 --formats coo --reps 10 >> gpurun_out/sweep18.txt 2>&1
done
