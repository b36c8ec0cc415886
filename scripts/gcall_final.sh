# Round-end evidence: bench line, reference arm, ncu launch list of the bench command,
# full ncu captures (C2, 16M d=9, 16M d=32 RWS/Vose), sweeps, compute-sanitizer.
set -x
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
bash scripts/profile_round.sh
timeout 300 python bench.py --impl reference --steps 10 --warmup 3 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
bash scripts/gcall_sanitize.sh
ls -la gpurun_out
