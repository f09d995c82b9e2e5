#!/bin/bash
# One entry point for the GPU-box evidence committed under profiles/ (run through gpurun).
#   bash tools/gpu_evidence.sh TAG TASK [ARGS...]
# Tasks (outputs land in gpurun_out/TAG/):
#   tests                       pytest -m gpu (+ smoke)
#   bench  [bench.py args]      one bench line -> bench_<config>.json
#   launches CFG                ncu launch list (gpu__time_duration, --clock-control none) of a short bench run
#   ncu CFG FMT [KERNEL_REGEX]  ncu --set full of one MTTKRP launch (FMT coo|hicoo|ghicoo) + summary .md
#   sweep CFG [sweep.py args]   tools/sweep.py timing of kernel variants
#   sanitize                    compute-sanitizer memcheck / racecheck over tests/sanitize_cases.py
#   micro NAME                  build and run tools/micro/NAME.cu
set -u
TAG=$1; TASK=$2; shift 2
O=gpurun_out/$TAG
mkdir -p $O
NCU_FULL="ncu --set full --clock-control none --import-source on"
case $TASK in
  tests)
    timeout 2400 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
    timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log ;;
  bench)
    timeout 1200 python bench.py "$@" > $O/bench.json 2> $O/bench.err; echo "rc=$?" >> $O/bench.err ;;
  launches)
    CFG=$1
    timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv \
      --log-file $O/launches_$CFG.csv \
      python bench.py --config $CFG --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 0 --hicoo-steps 1 \
      --cpals-iters 1 --ew-steps 2 --no-dram-counters > $O/launches_$CFG.log 2>&1
    python tools/ncu_summary.py launches $O/launches_$CFG.csv $O/launches_$CFG.md > /dev/null ;;
  ncu)
    CFG=$1; FMT=$2; K=${3:-coo_staged_kernel}
    timeout 900 $NCU_FULL -k regex:$K -s 3 -c 1 -o /tmp/${TAG}_${FMT}_$CFG \
      python tools/sweep.py --config $CFG --variants 0 --runs 0 --formats $FMT --reps 1 > $O/ncu_${FMT}_$CFG.log 2>&1
    python tools/ncu_summary.py full /tmp/${TAG}_${FMT}_$CFG.ncu-rep $CFG $O/ncu_full_${FMT}_$CFG.md ${FMT}_mttkrp > /dev/null
    ncu -i /tmp/${TAG}_${FMT}_$CFG.ncu-rep --page source --csv > $O/source_${FMT}_$CFG.csv 2>/dev/null
    ncu -i /tmp/${TAG}_${FMT}_$CFG.ncu-rep --page raw --csv > $O/raw_${FMT}_$CFG.csv 2>/dev/null ;;
  sweep)
    CFG=$1; shift
    timeout 1200 python tools/sweep.py --config $CFG "$@" >> $O/sweep_$CFG.txt 2>&1 ;;
  sanitize)
    for T in memcheck racecheck; do
      timeout 900 compute-sanitizer --tool $T --error-exitcode 9 python tests/sanitize_cases.py > $O/sanitizer_$T.log 2>&1
      echo "rc=$?" >> $O/sanitizer_$T.log
    done ;;
  micro)
    NAME=$1
    nvcc -O3 -gencode arch=compute_100a,code=sm_100a -lineinfo -o /tmp/$NAME tools/micro/$NAME.cu && \
      timeout 600 /tmp/$NAME > $O/micro_$NAME.txt 2>&1; echo "rc=$?" >> $O/micro_$NAME.txt ;;
  *) echo "unknown task $TASK"; exit 2 ;;
esac
