mkdir -p gpurun_out/v21
O=gpurun_out/v21
timeout 900 python -m pytest tests/test_gpu_cpals.py -x -q > $O/pytest_cpals.log 2>&1; echo "rc=$?" >> $O/pytest_cpals.log
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"gram_tile|apply_tile|cpals_prep" -c 12 --csv python tools/cpals_run.py h 1 > $O/cpals_ncu.csv 2>&1
timeout 600 compute-sanitizer --tool racecheck --error-exitcode 9 python tests/sanitize_cases.py > $O/sanitizer_racecheck.log 2>&1; echo "rc=$?" >> $O/sanitizer_racecheck.log
timeout 600 compute-sanitizer --tool memcheck --error-exitcode 9 python tests/sanitize_cases.py > $O/sanitizer_memcheck.log 2>&1; echo "rc=$?" >> $O/sanitizer_memcheck.log
timeout 900 python bench.py > $O/bench_h.json 2> $O/bench_h.err
