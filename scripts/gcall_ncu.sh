# full ncu captures of the step kernel at C2 and 16M d=9 (current in-tree build)
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
for cfg in "c2 5 256 4096 rws" "c5 5 256 65536 rws"; do
  set -- $cfg
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:pf_step_kernel --launch-skip 3 \
    --launch-count 1 -f -o gpurun_out/prof_$1 python scripts/prof_one.py $2 $3 $4 $5 > gpurun_out/prof_$1.log 2>&1
done
ls -la gpurun_out
