# A/B: ablib/$1 (A) vs the in-tree build (B), after the GPU tests named in $2 (pytest -k expression)
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
A=${1:-lib_hook.so}; K=${2:-resample or vose or trajectory}
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "$K" > gpurun_out/ab_tests.log 2>&1; echo "pytest rc $?" >> gpurun_out/ab_tests.log
timeout 900 python scripts/perf_ab.py ablib/$A - --reps 3 > gpurun_out/ab_perf.txt 2>&1
tail -3 gpurun_out/ab_tests.log; cat gpurun_out/ab_perf.txt
