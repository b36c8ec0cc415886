# round-2: full GPU test suite + A/B of the round-1 library (ablib/lib_r1.so) against the in-tree build
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/r02_pytest_gpu.log 2>&1; echo "pytest rc $?" >> gpurun_out/r02_pytest_gpu.log
if [ -f ablib/lib_r1.so ]; then timeout 600 python scripts/perf_ab.py ablib/lib_r1.so - --reps 3 > gpurun_out/r02_ab_model_hook.txt 2>&1; fi
tail -5 gpurun_out/r02_pytest_gpu.log; cat gpurun_out/r02_ab_model_hook.txt
