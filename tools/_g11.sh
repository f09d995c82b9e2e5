bash tools/gpu_evidence.sh r02k micro tma_gather4_bench
cat gpurun_out/r02k/micro_tma_gather4_bench.txt
bash tools/gpu_evidence.sh r02k sanitize
tail -3 gpurun_out/r02k/sanitizer_memcheck.log gpurun_out/r02k/sanitizer_racecheck.log
bash tools/gpu_evidence.sh r02k ncu c3 coo
bash tools/gpu_evidence.sh r02k ncu h coo
bash tools/gpu_evidence.sh r02k launches h
git checkout profiles/ncu_summary.json 2>/dev/null; ls gpurun_out/r02k
