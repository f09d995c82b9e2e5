mkdir -p gpurun_out
rm -f gpurun_out/sweep17.txt
for CFG in h c2; do
  echo "== $CFG" >> gpurun_out/sweep17.txt
  timeout 900 python tools/sweep.py --config $CFG --variants 0,2,3,4,5,6,7 --runs 0,256 --formats hicoo --reps 5 >> gpurun_out/sweep17.txt 2>&1
done
