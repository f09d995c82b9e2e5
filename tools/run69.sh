mkdir -p gpurun_out/v20
O=gpurun_out/v20
timeout 900 python -m pytest tests/test_gpu_cpals.py -x -q > $O/pytest_cpals.log 2>&1; echo "rc=$?" >> $O/pytest_cpals.log
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"gram_tile|apply_tile|cpals_prep" -c 12 --csv python tools/cpals_run.py h 1 > $O/cpals_ncu.csv 2>&1
timeout 900 python bench.py > $O/bench_h.json 2> $O/bench_h.err
