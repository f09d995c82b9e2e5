#!/bin/bash
# Capture the evidence committed under profiles/ (run on the GPU box via gpurun):
#   launch list of the bench command, ncu --set full of the COO and HiCOO MTTKRP kernels.
set -x
TAG=${1:-r01}
CFG=${2:-h}
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 500 --csv \
  --log-file gpurun_out/${TAG}_launches_${CFG}.csv \
  python bench.py --config $CFG --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 0 --hicoo-steps 1 \
  > gpurun_out/${TAG}_launches_${CFG}.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mttkrp_kernel \
  -s 3 -c 2 -o gpurun_out/${TAG}_prof_coo_${CFG} \
  python tools/sweep.py --config $CFG --variants 0 --runs 128 --formats coo --reps 1 \
  > gpurun_out/${TAG}_prof_coo_${CFG}.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mttkrp_kernel \
  -s 3 -c 2 -o gpurun_out/${TAG}_prof_hicoo_${CFG} \
  python tools/sweep.py --config $CFG --variants 0 --runs 128 --formats hicoo --reps 1 \
  > gpurun_out/${TAG}_prof_hicoo_${CFG}.log 2>&1
ls -la gpurun_out/ | grep $TAG
