mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_ghicoo.py -x -q > gpurun_out/pytest_ghicoo.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_ghicoo.log
for C in c3 h c2 c4; do
  timeout 600 python tools/sweep.py --config $C --variants 0 --runs 128 --formats coo,hicoo,ghicoo --reps 5 > gpurun_out/sweep_g_$C.log 2>&1
done
for M in 1 2 4 5 6; do
  timeout 600 python tools/sweep.py --config c3 --variants 0 --runs 128 --formats ghicoo --cmask $M --reps 5 > gpurun_out/sweep_g_c3_m$M.log 2>&1
done
