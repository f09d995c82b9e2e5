mkdir -p gpurun_out
rm -f gpurun_out/hs_sweep3.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/pytest_parity.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_parity.log
for MB in 32 64 96; do
  echo "== h HOT_MB=$MB" >> gpurun_out/hs_sweep3.txt
  PASTA_HOT_MB=$MB timeout 600 python tools/sweep.py --config h --variants 0 --runs 64,128,256 --formats coo --reps 10 >> gpurun_out/hs_sweep3.txt 2>&1
done
echo "== c2" >> gpurun_out/hs_sweep3.txt
timeout 600 python tools/sweep.py --config c2 --variants 0 --runs 64,128,256 --formats coo --reps 10 >> gpurun_out/hs_sweep3.txt 2>&1
echo "== c5" >> gpurun_out/hs_sweep3.txt
timeout 900 python tools/sweep.py --config c5 --variants 0 --runs 128 --formats coo --reps 3 >> gpurun_out/hs_sweep3.txt 2>&1
echo "== c5 HOT_SMEM=0" >> gpurun_out/hs_sweep3.txt
PASTA_HOT_SMEM=0 timeout 900 python tools/sweep.py --config c5 --variants 0 --runs 128 --formats coo --reps 3 >> gpurun_out/hs_sweep3.txt 2>&1
timeout 900 python bench.py --steps 50 > gpurun_out/bench.json 2> gpurun_out/bench.err
