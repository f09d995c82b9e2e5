mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q > gpurun_out/pytest_reuse.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_reuse.log
for C in h c2 c4 c3; do timeout 600 python tools/sweep.py --config $C --variants 0 --runs 128 --formats coo --reps 5; done > gpurun_out/sweep_reuse.log 2>&1
for WA in 6; do for C in h c2; do PASTA_STAGED_WA=$WA timeout 600 python tools/sweep.py --config $C --variants 0 --runs 128 --formats coo --reps 5; done; done > gpurun_out/sweep_wa6.log 2>&1
PASTA_EW_VARIANT=0 timeout 300 python tools/ew_sweep.py > gpurun_out/ew_default.log 2>&1
