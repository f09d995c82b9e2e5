bash tools/gpu_evidence.sh r02a micro l2_home_bench
timeout 1500 python -m pytest tests/test_gpu_cpals.py tests/test_gpu_parity_full.py -q -x -k "not every_row and not conversion_bit_exact" > gpurun_out/r02a/pytest_new.log 2>&1; echo rc=$? >> gpurun_out/r02a/pytest_new.log
tail -5 gpurun_out/r02a/pytest_new.log; tail -30 gpurun_out/r02a/micro_l2_home_bench.txt
