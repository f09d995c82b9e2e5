mkdir -p gpurun_out
rm -f gpurun_out/hs_sweep.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "hot" > gpurun_out/pytest_hot.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_hot.log
for CFG in c2 c4 h; do
  for HS in 0 1 1:64; do
    echo "== $CFG HOT_SMEM=$HS" >> gpurun_out/hs_sweep.txt
    PASTA_HOT_SMEM_ROWS=$([ "${HS#*:}" = "$HS" ] && echo 0 || echo ${HS#*:}) PASTA_HOT_SMEM=${HS%%:*} timeout 600 python tools/sweep.py --config $CFG --variants 0 --runs 128 --formats coo --reps 10 >> gpurun_out/hs_sweep.txt 2>&1
  done
done
