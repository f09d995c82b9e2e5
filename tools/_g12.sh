O=gpurun_out/r02l; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "die_split or hot_tier or hot_row_cache or random_tensors or shards" > $O/pytest.log 2>&1; echo rc=$? >> $O/pytest.log; tail -2 $O/pytest.log
bash tools/gpu_evidence.sh r02l sanitize
tail -4 gpurun_out/r02l/sanitizer_memcheck.log gpurun_out/r02l/sanitizer_racecheck.log
for SPLIT in 0 1; do PASTA_DIE_SPLIT=$SPLIT timeout 300 python tools/sweep.py --config h --variants 0 --runs 0 --formats coo --reps 10 >> $O/sweep.txt 2>&1; done
cat $O/sweep.txt
