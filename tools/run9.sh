mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_multirank.py tests/test_gpu_cpals.py -x -q > gpurun_out/pytest_p2p.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_p2p.log
for C in 2 4 8 16; do PASTA_TILE_CTAS_PER_SM=$C timeout 600 python tools/cpals_run.py h 10 | sed "s/^/ctas=$C /"; done > gpurun_out/cpals_time4.log 2>&1
for C in 4 8; do PASTA_TILE_CTAS_PER_SM=$C timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/cpals_launches_c$C.csv python tools/cpals_run.py h 1 > /dev/null 2>&1; done
