# Final round-2 refresh after the centralized-RWS change and the new mapping tests: GPU tests, smoke, bench
# line, centralized-filter sweep and ncu captures.
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r02_gpu_tests.txt 2>&1; echo "pytest rc $?" >> gpurun_out/r02_gpu_tests.txt
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02_smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/r02_bench.json 2> gpurun_out/r02_bench.err
timeout 300 python scripts/sweeps.py central > gpurun_out/r02_central_sweep.jsonl 2> gpurun_out/r02_sweeps.err
for res in rws vose; do
  timeout 300 ncu --set full --clock-control none -k regex:"cz_|vz_" --launch-skip 6 --launch-count 5 -f \
    -o gpurun_out/r02_prof_central_$res python scripts/prof_one.py 5 1048576 1 $res none 0 6 > gpurun_out/r02_prof_central_$res.log 2>&1
  timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    --log-file gpurun_out/r02_central_launches_$res.csv python scripts/prof_one.py 5 1048576 1 $res none 0 6 > /dev/null 2>&1
  ncu -i gpurun_out/r02_prof_central_$res.ncu-rep --page raw --csv \
    --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.per_cycle_active,launch__registers_per_thread,launch__grid_size,smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio \
    > gpurun_out/r02_ncu_central_$res.csv 2>&1
  rm -f gpurun_out/r02_prof_central_$res.ncu-rep
done
tail -3 gpurun_out/r02_gpu_tests.txt; cat gpurun_out/r02_smoke.txt; tail -2 gpurun_out/r02_central_sweep.jsonl | cut -c1-200
