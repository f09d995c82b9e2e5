bash tools/gpu_evidence.sh r02j tests
tail -3 gpurun_out/r02j/pytest_gpu.log; tail -2 gpurun_out/r02j/smoke.log
bash tools/gpu_evidence.sh r02j bench --steps 20 --warmup 5
tail -c 600 gpurun_out/r02j/bench.json
