mkdir -p gpurun_out/v15
O=gpurun_out/v15
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
timeout 900 python bench.py > $O/bench_h.json 2> $O/bench_h.err
timeout 600 python bench.py --impl reference > $O/bench_ref.json 2> $O/bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv \
  --log-file $O/launches_h.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-steps 0 --hicoo-steps 1 --cpals-iters 1 --ew-steps 2 \
  > $O/launches_h.log 2>&1
python tools/ncu_summary.py launches $O/launches_h.csv $O/launches_h.md > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:coo_staged_kernel -s 3 -c 1 -o /tmp/v15_coo_h \
  python tools/sweep.py --config h --variants 0 --runs 0 --formats coo --reps 1 > $O/coo_h.log 2>&1
python tools/ncu_summary.py full /tmp/v15_coo_h.ncu-rep h $O/ncu_full_coo_h.md > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"gram_tile|apply_tile" -c 2 -o /tmp/v15_cpals \
  python tools/cpals_run.py h 1 > $O/cpals_ncu.log 2>&1
python tools/ncu_summary.py full /tmp/v15_cpals.ncu-rep h $O/ncu_full_cpals.md cpals > /dev/null 2>&1
cp profiles/ncu_summary.json $O/ncu_summary.json
ls -la $O
