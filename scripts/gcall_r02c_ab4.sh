cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
A=${1:-lib_head.so}
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "trajectory or full_size or exchange or resample or peer" > gpurun_out/ab_tests.log 2>&1; echo "pytest rc $?" >> gpurun_out/ab_tests.log
timeout 900 python scripts/perf_ab.py ablib/$A - --reps 3 > gpurun_out/ab_perf.txt 2>&1
export PF_LIB=$PWD/ablib/libtl.so
for cfg in "5 256 4096 rws" "5 256 4096 vose"; do
  echo "== $cfg"; timeout 120 python scripts/timeline.py $cfg 2>&1 | grep -v "busy sub\|TIMELINE" | tail -9
done > gpurun_out/ab_timeline.txt 2>&1
tail -3 gpurun_out/ab_tests.log; cat gpurun_out/ab_perf.txt gpurun_out/ab_timeline.txt
