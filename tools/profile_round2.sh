#!/bin/bash
# Round evidence (run on the GPU box via gpurun): launch list of the default bench command and
# ncu --set full captures of the hot kernels, summarised into gpurun_out/prof2/ (-> profiles/).
TAG=${1:-r01}
OUT=gpurun_out/prof2
mkdir -p $OUT
NCU="ncu --set full --clock-control none --import-source on"
# 1. launch list of the bench command (cold-cache, serialised: shares, not absolute times)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv \
  --log-file $OUT/${TAG}_launches_h.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 0 --hicoo-steps 1 --cpals-iters 1 --ew-steps 2 \
  > $OUT/${TAG}_launches_h.log 2>&1
python tools/ncu_summary.py launches $OUT/${TAG}_launches_h.csv $OUT/${TAG}_launches_h.md > /dev/null
# 2. the dominant kernel: COO MTTKRP on H
timeout 900 $NCU -k regex:coo_staged_kernel -s 3 -c 1 -o /tmp/${TAG}_coo_h \
  python tools/sweep.py --config h --variants 0 --runs 128 --formats coo --reps 1 > $OUT/coo_h.log 2>&1
python tools/ncu_summary.py full /tmp/${TAG}_coo_h.ncu-rep h $OUT/${TAG}_ncu_full_coo_h.md > /dev/null
ncu -i /tmp/${TAG}_coo_h.ncu-rep --page source --csv > $OUT/${TAG}_source_coo_h.csv 2>/dev/null
# 3. TEW / TS streaming kernels
timeout 900 $NCU -k regex:ew_kernel -s 6 -c 2 -o /tmp/${TAG}_ew \
  python tools/ew_sweep.py > $OUT/ew.log 2>&1
python tools/ncu_summary.py full /tmp/${TAG}_ew.ncu-rep ew $OUT/${TAG}_ncu_full_ew.md > /dev/null
# 4. HiCOO and gHiCOO row-slice MTTKRP on the hypersparse flickr-shaped C3
timeout 900 $NCU -k regex:mttkrp_kernel -s 3 -c 1 -o /tmp/${TAG}_ghicoo_c3 \
  python tools/sweep.py --config c3 --variants 0 --runs 128 --formats ghicoo --reps 1 > $OUT/ghicoo_c3.log 2>&1
python tools/ncu_summary.py full /tmp/${TAG}_ghicoo_c3.ncu-rep c3 $OUT/${TAG}_ncu_full_ghicoo_c3.md ghicoo_mttkrp > /dev/null
# 5. CP-ALS update kernels
timeout 900 $NCU -k regex:"gram_tile|apply_tile|cpals_prep" -s 3 -c 3 -o /tmp/${TAG}_cpals \
  python tools/cpals_run.py h 1 > $OUT/cpals.log 2>&1
python tools/ncu_summary.py full /tmp/${TAG}_cpals.ncu-rep h_cpals $OUT/${TAG}_ncu_full_cpals.md > /dev/null
cp profiles/ncu_summary.json $OUT/ncu_summary.json
cp /tmp/${TAG}_coo_h.ncu-rep $OUT/ 2>/dev/null
ls -la $OUT
