# ncu --set full captures of the MTTKRP kernels, summarised on the box (reports are large)
mkdir -p gpurun_out/prof
for CFG in h c2; do
  for FMT in coo hicoo; do
    timeout 900 ncu --set full --clock-control none --import-source on -k regex:mttkrp_kernel -s 3 -c 1 \
      -o /tmp/r01_prof_${FMT}_${CFG} python tools/sweep.py --config $CFG --variants 0 --runs 128 \
      --formats $FMT --reps 1 > gpurun_out/prof/r01_prof_${FMT}_${CFG}.log 2>&1
    python tools/ncu_summary.py full /tmp/r01_prof_${FMT}_${CFG}.ncu-rep $CFG gpurun_out/prof/r01_ncu_full_${FMT}_${CFG}.md > /dev/null
    ncu -i /tmp/r01_prof_${FMT}_${CFG}.ncu-rep --page source --csv > gpurun_out/prof/r01_source_${FMT}_${CFG}.csv 2>/dev/null
  done
done
cp profiles/ncu_summary.json gpurun_out/prof/ncu_summary.json
cp /tmp/r01_prof_coo_h.ncu-rep gpurun_out/prof/
ls -la gpurun_out/prof
