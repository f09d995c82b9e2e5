mkdir -p gpurun_out/v22
for i in 1 2 3; do timeout 300 python tools/cpals_run.py h 10 >> gpurun_out/v22/cpals_new.log 2>&1; done
