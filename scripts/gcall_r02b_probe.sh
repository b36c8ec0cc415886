cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 120 python scripts/dev/flush_floor.py > gpurun_out/r02b_flush_floor.txt 2>&1
export PF_LIB=$PWD/ablib/libtl.so
for cfg in "5 256 4096 rws 1" "5 256 4096 rws 0" "5 256 4096 rws 1 host"; do
  echo "== $cfg"; timeout 120 python scripts/timeline.py $cfg 2>&1 | grep -v "busy sub" | tail -14
done > gpurun_out/r02b_timeline.txt 2>&1
cat gpurun_out/r02b_flush_floor.txt gpurun_out/r02b_timeline.txt
