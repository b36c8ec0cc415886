# usage: gcall_ab.sh LIB_A LIB_B [extra perf_ab args]; runs the GPU tests first
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc $?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
timeout 900 python scripts/perf_ab.py "$@" 2>&1 | tee gpurun_out/ab.txt
