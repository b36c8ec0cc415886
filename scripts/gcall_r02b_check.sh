# round-2 re-entry: GPU tests + smoke + bench line on the current kernels
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/r02b_pytest_gpu.log 2>&1; echo "pytest rc $?" >> gpurun_out/r02b_pytest_gpu.log
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02b_smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/r02b_bench.json 2> gpurun_out/r02b_bench.err
tail -3 gpurun_out/r02b_pytest_gpu.log; cat gpurun_out/r02b_smoke.txt | tail -2; tail -c 2500 gpurun_out/r02b_bench.json
