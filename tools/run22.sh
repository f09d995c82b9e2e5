mkdir -p gpurun_out
rm -f gpurun_out/sweep6.txt
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ttm.py -x -q > gpurun_out/pytest_parity.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_parity.log
for CFG in h c2 c4 c3; do
  echo "== $CFG" >> gpurun_out/sweep6.txt
  timeout 600 python tools/sweep.py --config $CFG --variants 0 --runs 0,64,256 --formats coo --reps 10 >> gpurun_out/sweep6.txt 2>&1
done
timeout 900 ncu --set full --clock-control none -k regex:coo_staged_kernel -s 3 -c 1 -o /tmp/c2 python tools/sweep.py --config c2 --variants 0 --runs 0 --formats coo --reps 1 > /dev/null 2>&1
python tools/ncu_summary.py full /tmp/c2.ncu-rep c2 gpurun_out/ncu_c2_swz.md > /dev/null
