# Round-2 final evidence in one GPU call (outputs under gpurun_out/, copied into profiles/ afterwards):
# GPU tests, smoke, bench line + reference arm, ncu launch list of the bench command, ncu --set full of the
# step kernel (C2 / 16M d=9 / 16M d=32, RWS and Vose) and of the centralized filter's kernels, sweeps,
# mapping variants, per-phase timeline, a 2-rank functional run of bench.py on one GPU.
set -x
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r02_gpu_tests.txt 2>&1; echo "pytest rc $?" >> gpurun_out/r02_gpu_tests.txt
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02_smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/r02_bench.json 2> gpurun_out/r02_bench.err
timeout 300 python bench.py --impl reference --steps 20 --warmup 3 > gpurun_out/r02_bench_reference.json 2> gpurun_out/r02_bench_reference.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/r02_launches.csv python bench.py --steps 5 --warmup 3 --no-extras --cpu-seconds 1 \
  > gpurun_out/r02_bench_under_ncu.log 2>&1
for cfg in "c2 5 256 4096 rws" "c2v 5 256 4096 vose" "c5 5 256 65536 rws" "c5v 5 256 65536 vose" "c4rws 28 256 65536 rws" "c4 28 256 65536 vose"; do
  set -- $cfg
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:pf_step_kernel --launch-skip 3 \
    --launch-count 1 -f -o gpurun_out/r02_prof_$1 python scripts/prof_one.py $2 $3 $4 $5 > gpurun_out/r02_prof_$1.log 2>&1
done
python scripts/ncu_summary.py C2=gpurun_out/r02_prof_c2.ncu-rep:1048576 C2_vose=gpurun_out/r02_prof_c2v.ncu-rep:1048576 \
  C5_nj5_16M=gpurun_out/r02_prof_c5.ncu-rep:16777216 C5_nj5_16M_vose=gpurun_out/r02_prof_c5v.ncu-rep:16777216 \
  C4_nj28_16M_rws=gpurun_out/r02_prof_c4rws.ncu-rep:16777216 C4_nj28_16M_vose=gpurun_out/r02_prof_c4.ncu-rep:16777216 \
  > gpurun_out/r02_ncu_full.txt 2>&1
cp profiles/ncu_summary.json gpurun_out/r02_ncu_summary.json
python scripts/ncu_opcodes.py gpurun_out/r02_prof_c2.ncu-rep 1048576 40 > gpurun_out/r02_sass_opcodes_c2.txt
python scripts/ncu_opcodes.py gpurun_out/r02_prof_c5.ncu-rep 16777216 40 > gpurun_out/r02_sass_opcodes_c5.txt
python scripts/ncu_opcodes.py gpurun_out/r02_prof_c5v.ncu-rep 16777216 40 > gpurun_out/r02_sass_opcodes_c5_vose.txt
python scripts/ncu_lines.py gpurun_out/r02_prof_c2.ncu-rep 50 > gpurun_out/r02_source_lines_c2.txt
python scripts/ncu_lines.py gpurun_out/r02_prof_c5.ncu-rep 60 > gpurun_out/r02_source_lines_c5.txt
python scripts/ncu_lines.py gpurun_out/r02_prof_c2.ncu-rep 100000 > gpurun_out/r02_lines_all_c2.txt
python scripts/ncu_lines.py gpurun_out/r02_prof_c5.ncu-rep 100000 > gpurun_out/r02_lines_all_c5.txt
rm -f gpurun_out/r02_prof_c2v.ncu-rep gpurun_out/r02_prof_c5.ncu-rep gpurun_out/r02_prof_c5v.ncu-rep gpurun_out/r02_prof_c4.ncu-rep gpurun_out/r02_prof_c4rws.ncu-rep
timeout 900 python scripts/sweeps.py > gpurun_out/r02_sweeps.jsonl 2> gpurun_out/r02_sweeps.err
timeout 600 python scripts/sweeps.py dim > gpurun_out/r02_dim_sweep.jsonl 2>> gpurun_out/r02_sweeps.err
timeout 300 python scripts/dev/n_sweep.py 1776 2000 2664 3552 3700 4096 4440 5328 7104 > gpurun_out/r02_rounds_sweep.txt 2>&1
# (compute-sanitizer is closed on this GPU pool)
(python scripts/variants_one.py 5 256 4096 rws 16; python scripts/variants_one.py 5 256 4096 vose 10; python scripts/variants_one.py 5 256 65536 vose 9) > gpurun_out/r02_variants_raw.txt 2>&1
bash scripts/gcall_r02_timeline.sh > /dev/null 2>&1
timeout 400 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29555 \
  bench.py --gpus 2 --steps 5 --warmup 3 --no-extras --cpu-seconds 1 > gpurun_out/r02_bench_2rank.json 2> gpurun_out/r02_bench_2rank.err
ls -la gpurun_out | grep r02
