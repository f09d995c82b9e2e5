mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_all.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke2.log 2>&1
timeout 900 python bench.py > gpurun_out/bench3.log 2>&1
bash tools/profile_round2.sh r01 > gpurun_out/prof2.log 2>&1
