mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_cpals.py -x -q > gpurun_out/pytest_cpals.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_cpals.log
timeout 900 python bench.py --no-cpu-baseline --hicoo-steps 0 --ew-steps 0 --e2e-steps 0 --steps 10 > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"gram_tile|apply_tile|cpals_prep" -c 12 --csv python tools/cpals_run.py h 1 > gpurun_out/cpals_ncu.csv 2>&1
