cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "central or device_inputs or models" > gpurun_out/ab_tests.log 2>&1; echo "pytest rc $?" >> gpurun_out/ab_tests.log
timeout 900 python scripts/perf_ab.py ablib/lib_head.so ablib/lib_b2.so - --reps 3 > gpurun_out/ab_perf.txt 2>&1
tail -3 gpurun_out/ab_tests.log; cat gpurun_out/ab_perf.txt
