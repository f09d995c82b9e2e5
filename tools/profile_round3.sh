#!/bin/bash
# Evidence for the persistent COO kernel (run on the GPU box): launch list of the default bench
# command, ncu --set full of coo_staged_kernel on H and C2.
TAG=${1:-r01b}
OUT=gpurun_out/prof3
mkdir -p $OUT
NCU="ncu --set full --clock-control none --import-source on"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv \
  --log-file $OUT/${TAG}_launches_h.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 0 --hicoo-steps 1 --cpals-iters 1 --ew-steps 2 \
  > $OUT/${TAG}_launches_h.log 2>&1
python tools/ncu_summary.py launches $OUT/${TAG}_launches_h.csv $OUT/${TAG}_launches_h.md > /dev/null
for CFG in h c2; do
  timeout 900 $NCU -k regex:coo_staged_kernel -s 3 -c 1 -o /tmp/${TAG}_coo_$CFG \
    python tools/sweep.py --config $CFG --variants 0 --runs 0 --formats coo --reps 1 > $OUT/coo_$CFG.log 2>&1
  python tools/ncu_summary.py full /tmp/${TAG}_coo_$CFG.ncu-rep $CFG $OUT/${TAG}_ncu_full_coo_$CFG.md > /dev/null
  ncu -i /tmp/${TAG}_coo_$CFG.ncu-rep --page source --csv > $OUT/${TAG}_source_coo_$CFG.csv 2>/dev/null
  ncu -i /tmp/${TAG}_coo_$CFG.ncu-rep --page details --csv > $OUT/${TAG}_details_coo_$CFG.csv 2>/dev/null
done
cp profiles/ncu_summary.json $OUT/ncu_summary.json
ls -la $OUT
# HiCOO / gHiCOO row slices through the staged kernel (WA 9) on H
for FMT in hicoo ghicoo; do
  timeout 900 $NCU -k regex:coo_staged_kernel -s 3 -c 1 -o /tmp/${TAG}_${FMT}_h \
    python tools/sweep.py --config h --variants 0 --runs 0 --formats $FMT --reps 1 > $OUT/${FMT}_h.log 2>&1
  python tools/ncu_summary.py full /tmp/${TAG}_${FMT}_h.ncu-rep h $OUT/${TAG}_ncu_full_${FMT}_h.md ${FMT}_mttkrp > /dev/null
done
cp profiles/ncu_summary.json $OUT/ncu_summary.json
