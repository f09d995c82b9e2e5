mkdir -p gpurun_out
for F in 0 1 0 1; do PASTA_CPALS_FUSED=$F timeout 600 python tools/cpals_run.py h 10 | sed "s/^/fused=$F /"; done > gpurun_out/cpals_time2.log 2>&1
for WA in 1 6; do PASTA_STAGED_WA=$WA timeout 600 python tools/sweep.py --config h --variants 0 --runs 128 --formats coo --reps 5 | sed "s/^/wa=$WA /"; done > gpurun_out/sweep_wa.log 2>&1
