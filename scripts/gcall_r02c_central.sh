cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "central or device_inputs" > gpurun_out/ab_tests.log 2>&1; echo "pytest rc $?" >> gpurun_out/ab_tests.log
timeout 900 python scripts/perf_ab.py ablib/lib_head.so - --reps 3 > gpurun_out/ab_perf.txt 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/central_launches_new.csv python scripts/prof_one.py 5 1048576 1 rws none 0 6 > /dev/null 2>&1
tail -3 gpurun_out/ab_tests.log; cat gpurun_out/ab_perf.txt
