# Round-end evidence: bench line, reference arm, ncu launch list of the bench command,
# full ncu captures (C2, 16M d=9, 16M d=32 RWS/Vose) summarised on the box (the
# reports themselves exceed gpurun's 64 MiB return limit; C2's is kept), sweeps,
# compute-sanitizer, a 2-rank functional run of bench.py on one GPU.
set -x
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
bash scripts/profile_round.sh
timeout 300 python bench.py --impl reference --steps 10 --warmup 3 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
bash scripts/gcall_sanitize.sh
timeout 400 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29555 \
  bench.py --gpus 2 --steps 5 --warmup 3 --no-extras --cpu-seconds 1 > gpurun_out/bench2.json 2> gpurun_out/bench2.err
python scripts/ncu_summary.py C2=gpurun_out/prof_c2.ncu-rep:1048576 C5_nj5_16M=gpurun_out/prof_c5.ncu-rep:16777216 \
  C4_nj28_16M_vose=gpurun_out/prof_c4.ncu-rep:16777216 C4_nj28_16M_rws=gpurun_out/prof_c4rws.ncu-rep:16777216 \
  > gpurun_out/ncu_full.txt 2>&1
cp profiles/ncu_summary.json gpurun_out/ncu_summary.json
python scripts/ncu_opcodes.py gpurun_out/prof_c2.ncu-rep 1048576 40 > gpurun_out/sass_opcodes_c2.txt
python scripts/ncu_opcodes.py gpurun_out/prof_c4rws.ncu-rep 16777216 40 > gpurun_out/sass_opcodes_c4_rws.txt
python scripts/ncu_lines.py gpurun_out/prof_c2.ncu-rep 50 > gpurun_out/source_lines_c2.txt
rm -f gpurun_out/prof_c5.ncu-rep gpurun_out/prof_c4.ncu-rep gpurun_out/prof_c4rws.ncu-rep
ls -la gpurun_out
