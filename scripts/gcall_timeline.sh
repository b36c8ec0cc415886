cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
export PF_LIB=$PWD/variants/libtl.so
for cfg in "5 256 4096 rws" "5 256 65536 rws" "5 256 16 rws"; do
  echo "== $cfg"; timeout 120 python scripts/timeline.py $cfg 2>&1 | tail -40
done > gpurun_out/timeline.txt 2>&1
cat gpurun_out/timeline.txt
