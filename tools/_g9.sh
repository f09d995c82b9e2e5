O=gpurun_out/r02i; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "die_split" > $O/pytest.log 2>&1; echo rc=$? >> $O/pytest.log; tail -2 $O/pytest.log
for SPLIT in 0 1; do for MB in 64 96 128; do
  echo "== h split=$SPLIT hot_mb=$MB" >> $O/sweep.txt
  PASTA_DIE_SPLIT=$SPLIT PASTA_HOT_MB=$MB timeout 300 python tools/sweep.py --config h --variants 0 --runs 0 --formats coo --reps 10 >> $O/sweep.txt 2>>$O/sweep.err
done; done
PASTA_DIE_SPLIT=1 PASTA_HOT_MB=96 timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,gpu__time_duration.sum --clock-control none -k regex:coo_staged_kernel -s 3 -c 3 python tools/sweep.py --config h --variants 0 --runs 0 --formats coo --reps 1 > $O/ncu_split1.txt 2>&1
for CFG in h c2; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:coo_staged_kernel -s 2 -c 1 -o /tmp/hic_$CFG python tools/sweep.py --config $CFG --variants 0 --runs 0 --formats hicoo --reps 1 > $O/ncu_hic_$CFG.log 2>&1
python tools/ncu_summary.py full /tmp/hic_$CFG.ncu-rep $CFG $O/ncu_full_hicoo_raw_$CFG.md hicoo_raw > /dev/null
ncu -i /tmp/hic_$CFG.ncu-rep --page source --csv > $O/source_hicoo_raw_$CFG.csv 2>/dev/null
done
git checkout profiles/ncu_summary.json
cat $O/sweep.txt; grep -E "dram__bytes|hit_rate|duration" $O/ncu_split1.txt
