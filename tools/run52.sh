mkdir -p gpurun_out
rm -f gpurun_out/sweep25.txt
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -k "random or shared" > gpurun_out/pytest_parity.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_parity.log
for CFG in c2 h; do for R in 8; do
  echo "== $CFG R=$R" >> gpurun_out/sweep25.txt
  timeout 900 python tools/sweep.py --config $CFG --R $R --variants 0 --runs 0 --formats coo --reps 5 >> gpurun_out/sweep25.txt 2>&1
done; done
