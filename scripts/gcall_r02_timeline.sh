# per-phase timeline (PF_TIMELINE build) of the step kernel: C2 RWS / Vose, 16M d=9 RWS / Vose
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
export PF_LIB=$PWD/ablib/libtl.so
for cfg in "5 256 4096 rws" "5 256 4096 vose" "5 256 65536 rws" "5 256 65536 vose"; do
  echo "== $cfg"; timeout 120 python scripts/timeline.py $cfg 2>&1 | tail -12
done > gpurun_out/r02_timeline.txt 2>&1
grep TIMELINE gpurun_out/r02_timeline.txt | sed 's/^TIMELINE //' > gpurun_out/r02_timeline.jsonl
cat gpurun_out/r02_timeline.jsonl
