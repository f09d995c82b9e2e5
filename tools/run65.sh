mkdir -p gpurun_out/v16
O=gpurun_out/v16
timeout 300 python -m pytest tests/test_golden.py -q > $O/pytest_golden.log 2>&1; echo "rc=$?" >> $O/pytest_golden.log
timeout 600 python tests/sanitize_cases.py > $O/plain.log 2>&1; echo "rc=$?" >> $O/plain.log
for T in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $T --error-exitcode 9 --print-limit 20 python tests/sanitize_cases.py > $O/sanitizer_$T.log 2>&1; echo "rc=$?" >> $O/sanitizer_$T.log
done
