#!/bin/bash
# One GPU call: bench line, the ncu launch list of the bench command, full ncu
# captures of the step kernel at C2 / 16M d=9 / 16M d=32, sweeps.
# Outputs under gpurun_out/ (scratch); summarise into profiles/ afterwards.
set -x
cd "${GRAFT_REPO_ROOT:-.}"
timeout 400 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-extras --cpu-seconds 1 \
  > gpurun_out/bench_under_ncu.log 2>&1
for cfg in "c2 5 256 4096 rws" "c5 5 256 65536 rws" "c4 28 256 65536 vose" "c4rws 28 256 65536 rws"; do
  set -- $cfg
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:pf_step_kernel --launch-skip 3 \
    --launch-count 1 -f -o gpurun_out/prof_$1 python scripts/prof_one.py $2 $3 $4 $5 > gpurun_out/prof_$1.log 2>&1
done
timeout 600 python scripts/sweeps.py > gpurun_out/sweeps.jsonl 2> gpurun_out/sweeps.err
ls -la gpurun_out
