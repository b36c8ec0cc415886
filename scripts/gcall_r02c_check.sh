# Re-entry check of the committed kernels: GPU tests, smoke, bench line, per-config device times.
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r02c_gpu_tests.txt 2>&1; echo "pytest rc $?" >> gpurun_out/r02c_gpu_tests.txt
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02c_smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/r02c_bench.json 2> gpurun_out/r02c_bench.err
timeout 600 python scripts/perf_ab.py - --reps 2 > gpurun_out/r02c_perf.txt 2>&1
tail -3 gpurun_out/r02c_gpu_tests.txt; cat gpurun_out/r02c_smoke.txt | tail -2; cat gpurun_out/r02c_perf.txt
