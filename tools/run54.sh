mkdir -p gpurun_out
rm -f gpurun_out/sweep26.txt
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ghicoo.py -x -q -k "hicoo or ghicoo or random or config1" > gpurun_out/pytest_parity.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_parity.log
for CFG in h c2 c3 c4; do
  echo "== $CFG" >> gpurun_out/sweep26.txt
  timeout 900 python tools/sweep.py --config $CFG --variants 0 --runs 0 --formats hicoo --reps 5 >> gpurun_out/sweep26.txt 2>&1
done
