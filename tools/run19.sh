mkdir -p gpurun_out
rm -f gpurun_out/hs_sweep4.txt
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ttm.py tests/test_gpu_cpals.py -x -q > gpurun_out/pytest_parity.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_parity.log
for CFG in h c2 c4 c3; do
  echo "== $CFG" >> gpurun_out/hs_sweep4.txt
  timeout 600 python tools/sweep.py --config $CFG --variants 0 --runs 32,64,128,256 --formats coo --reps 10 >> gpurun_out/hs_sweep4.txt 2>&1
done
