mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cpals.py tests/test_gpu_multirank.py -x -q > gpurun_out/pytest_cpals2.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_cpals2.log
for F in 0 1 0 1; do PASTA_CPALS_FUSED=$F timeout 600 python tools/cpals_run.py h 10 | sed "s/^/fused=$F /"; done > gpurun_out/cpals_time3.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/cpals_launches2.csv python tools/cpals_run.py h 1 > gpurun_out/cpals_ncu2.log 2>&1
