O=gpurun_out/r02d; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "die_split or hot_tier or hot_row_cache or staged_decode or random_tensors" > $O/pytest_a.log 2>&1; echo rc=$? >> $O/pytest_a.log
timeout 900 python -m pytest tests/test_gpu_parity_full.py -q -x -k "retag or hot_row_ten" > $O/pytest_b.log 2>&1; echo rc=$? >> $O/pytest_b.log
tail -3 $O/pytest_a.log $O/pytest_b.log
for SPLIT in 0 1; do for MB in 48 64 96 128; do
  echo "== h split=$SPLIT hot_mb=$MB" >> $O/sweep.txt
  PASTA_DIE_SPLIT=$SPLIT PASTA_HOT_MB=$MB timeout 300 python tools/sweep.py --config h --variants 0 --runs 0 --formats coo --reps 10 >> $O/sweep.txt 2>>$O/sweep.err
done; done
for CFG in c3 c5; do for SPLIT in 0 1; do
  echo "== $CFG split=$SPLIT" >> $O/sweep.txt
  PASTA_DIE_SPLIT=$SPLIT timeout 300 python tools/sweep.py --config $CFG --variants 0 --runs 0 --formats coo --reps 5 >> $O/sweep.txt 2>>$O/sweep.err
done; done
cat $O/sweep.txt
