O=gpurun_out/r02h; mkdir -p $O
bash tools/gpu_evidence.sh r02h micro l2_home_bench
PASTA_DEBUG=1 python -c "
import paper_conf_iiswc_lilwlob20_b200 as p, torch
torch.cuda.init()
d, n = p.pasta_die_map(); print('lib die map', n, ''.join(str(int(v)) for v in d))
" > $O/libmap.txt 2>&1
head -3 $O/micro_l2_home_bench.txt; cat $O/libmap.txt | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "random_tensors or hicoo or staged_decode or shards or config1 or hot_row_spanning" > $O/pytest.log 2>&1; echo rc=$? >> $O/pytest.log
tail -3 $O/pytest.log
for CFG in h c2 c3; do
  echo "== $CFG raw" >> $O/sweep.txt
  timeout 300 python tools/sweep.py --config $CFG --variants 0 --runs 0 --formats hicoo --reps 10 >> $O/sweep.txt 2>>$O/sweep.err
  echo "== $CFG wa9" >> $O/sweep.txt
  PASTA_HICOO_RAW=0 timeout 300 python tools/sweep.py --config $CFG --variants 0 --runs 0 --formats hicoo --reps 10 >> $O/sweep.txt 2>>$O/sweep.err
done
cat $O/sweep.txt
