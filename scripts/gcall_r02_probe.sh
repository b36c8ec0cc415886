# round-2 baseline probe: timings of the in-tree build + ncu full of Vose 16M d=9 and C2 (RWS/Vose)
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r02_probe_smi.txt
timeout 300 python scripts/perf_ab.py - --reps 3 > gpurun_out/r02_probe_ab.txt 2>&1
for cfg in "c5v 5 256 65536 vose" "c2v 5 256 4096 vose" "c2 5 256 4096 rws"; do
  set -- $cfg
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:pf_step_kernel --launch-skip 3 \
    --launch-count 1 -f -o gpurun_out/r02_prof_$1 python scripts/prof_one.py $2 $3 $4 $5 > gpurun_out/r02_prof_$1.log 2>&1
done
ls -la gpurun_out
