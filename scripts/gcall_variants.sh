cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
for v in 0 2 3 4 5 6 7 8 9 10 11 12 13 14 15 16 17; do
  echo "== PF_VARIANT=$v"
  PF_VARIANT=$v timeout 120 python scripts/perf_ab.py - --reps 1 --quick 2>&1 | tail -3
done | tee gpurun_out/variants.txt
