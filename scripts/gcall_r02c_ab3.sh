# full GPU tests + A/B of the in-tree build against ablib/$1
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
A=${1:-lib_head.so}
timeout 1200 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/ab_tests.log 2>&1; echo "pytest rc $?" >> gpurun_out/ab_tests.log
timeout 900 python scripts/perf_ab.py ablib/$A - --reps 3 > gpurun_out/ab_perf.txt 2>&1
tail -3 gpurun_out/ab_tests.log; cat gpurun_out/ab_perf.txt
