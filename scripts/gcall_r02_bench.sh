# round-2: bench line (N=1) + reference arm + a 2-rank functional run (ranks share the GPU)
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 600 python bench.py > gpurun_out/r02_bench.json 2> gpurun_out/r02_bench.err
timeout 300 python bench.py --impl reference --steps 20 --warmup 3 > gpurun_out/r02_bench_ref.json 2> gpurun_out/r02_bench_ref.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 > gpurun_out/r02_bench_2rank.json 2> gpurun_out/r02_bench_2rank.err
tail -c 3000 gpurun_out/r02_bench.json; tail -3 gpurun_out/r02_bench.err; tail -c 600 gpurun_out/r02_bench_ref.json; tail -c 300 gpurun_out/r02_bench_2rank.json; tail -3 gpurun_out/r02_bench_2rank.err
