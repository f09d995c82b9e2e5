O=gpurun_out/r02g; mkdir -p $O
for SPLIT in 0 1; do for C in 0 8 10; do for MB in 64 128; do
  echo "== h split=$SPLIT cache=$C hot_mb=$MB" >> $O/sweep.txt
  PASTA_DIE_SPLIT=$SPLIT PASTA_MTTKRP_CACHE=$C PASTA_HOT_MB=$MB timeout 300 python tools/sweep.py --config h --variants 0 --runs 0 --formats coo --reps 10 >> $O/sweep.txt 2>>$O/sweep.err
done; done; done
for SPLIT in 0 1; do
PASTA_DIE_SPLIT=$SPLIT PASTA_MTTKRP_CACHE=8 PASTA_HOT_MB=96 timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,gpu__time_duration.sum --clock-control none -k regex:coo_staged_kernel -s 3 -c 3 python tools/sweep.py --config h --variants 0 --runs 0 --formats coo --reps 1 > $O/ncu_split$SPLIT.txt 2>&1
done
cat $O/sweep.txt; grep -E "dram__bytes|hit_rate|duration" $O/ncu_split*.txt
