cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "resample or vose or central or trajectory" > gpurun_out/ab_tests.log 2>&1; echo "pytest rc $?" >> gpurun_out/ab_tests.log
timeout 900 python scripts/perf_ab.py ablib/lib_base.so - --reps 3 > gpurun_out/ab_perf.txt 2>&1
timeout 600 python scripts/variants_one.py 5 256 65536 vose 2,5,6 > gpurun_out/ab_var16.txt 2>&1
timeout 600 python scripts/variants_one.py 5 256 4096 vose 0,5,6 > gpurun_out/ab_varc2.txt 2>&1
for res in rws vose; do
  timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none --clock-control none --csv \
    --log-file gpurun_out/central_nocc_$res.csv python scripts/prof_central.py 1048576 $res 6 > /dev/null 2>&1
done
tail -3 gpurun_out/ab_tests.log; cat gpurun_out/ab_perf.txt gpurun_out/ab_var16.txt gpurun_out/ab_varc2.txt
