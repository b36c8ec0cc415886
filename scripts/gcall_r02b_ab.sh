# A/B: ablib/$1 (A, the previous build) vs the in-tree build (B) + a pytest subset + the C2 timeline of the new build
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
A=${1:-lib_base.so}; K=${2:-trajectory or full_size or exchange}
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "$K" > gpurun_out/ab_tests.log 2>&1; echo "pytest rc $?" >> gpurun_out/ab_tests.log
timeout 900 python scripts/perf_ab.py ablib/$A - --reps 3 > gpurun_out/ab_perf.txt 2>&1
if [ -f ablib/libtl.so ]; then PF_LIB=$PWD/ablib/libtl.so timeout 120 python scripts/timeline.py 5 256 4096 rws 2>&1 | grep -v "busy sub" | tail -7 > gpurun_out/ab_timeline.txt; fi
tail -3 gpurun_out/ab_tests.log; cat gpurun_out/ab_perf.txt; cat gpurun_out/ab_timeline.txt
