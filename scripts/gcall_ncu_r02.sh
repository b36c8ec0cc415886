# ncu --set full captures of the step kernel (current in-tree build).
# usage: gcall_ncu_r02.sh TAG "name nj m N res" ["name nj m N res" ...]
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
TAG=$1; shift
for cfg in "$@"; do
  set -- $cfg
  timeout 400 ncu --set full --import-source on --clock-control none -k regex:pf_step_kernel --launch-skip 3 \
    --launch-count 1 -f -o gpurun_out/${TAG}_prof_$1 python scripts/prof_one.py $2 $3 $4 $5 > gpurun_out/${TAG}_prof_$1.log 2>&1
done
ls -la gpurun_out | grep ${TAG}_prof
