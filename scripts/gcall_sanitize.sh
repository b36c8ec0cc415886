cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  echo "== compute-sanitizer --tool $tool --kernel-name kns=pf_ python scripts/sanitize_run.py"
  timeout 900 compute-sanitizer --tool $tool --kernel-name kns=pf_ python scripts/sanitize_run.py 2>&1 | grep -v "^\s*$"
done > gpurun_out/sanitizer.txt 2>&1
tail -5 gpurun_out/sanitizer.txt
