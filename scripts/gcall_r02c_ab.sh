# A/B of the in-tree build against ablib/$1 (default lib_base.so) + parity subset + central launch list
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
A=${1:-lib_base.so}; K=${2:-resample or vose or trajectory or full_size or exchange or central}
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "$K" > gpurun_out/ab_tests.log 2>&1; echo "pytest rc $?" >> gpurun_out/ab_tests.log
timeout 900 python scripts/perf_ab.py ablib/$A - --reps 3 > gpurun_out/ab_perf.txt 2>&1
if [ -n "$CENTRAL" ]; then
  for res in rws vose; do
    timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
      --log-file gpurun_out/central_launches_$res.csv python scripts/prof_one.py 5 1048576 1 $res none 0 6 > /dev/null 2>&1
  done
  timeout 300 python scripts/sweeps.py central > gpurun_out/central_sweep.jsonl 2>/dev/null
fi
tail -3 gpurun_out/ab_tests.log; cat gpurun_out/ab_perf.txt
