O=gpurun_out/r02e; mkdir -p $O
for SPLIT in 0 1; do
PASTA_DIE_SPLIT=$SPLIT timeout 900 ncu --set full --clock-control none -k regex:coo_staged_kernel -s 3 -c 1 -o /tmp/split$SPLIT python tools/sweep.py --config h --variants 0 --runs 0 --formats coo --reps 1 > $O/ncu_split$SPLIT.log 2>&1
python tools/ncu_summary.py full /tmp/split$SPLIT.ncu-rep h $O/ncu_full_coo_h_split$SPLIT.md coo_split$SPLIT > /dev/null
ncu -i /tmp/split$SPLIT.ncu-rep --page raw --csv > $O/raw_split$SPLIT.csv 2>/dev/null
done
git checkout profiles/ncu_summary.json 2>/dev/null
head -40 $O/ncu_full_coo_h_split1.md
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_cpals.py tests/test_gpu_multirank.py -q -x -k "shards or generator or tns or cpals or row_partitioned" > $O/pytest.log 2>&1; echo rc=$? >> $O/pytest.log
tail -3 $O/pytest.log
