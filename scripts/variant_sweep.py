"""Dev tool: time every compiled mapping (PF_VARIANT=i) of one (nj, m, res) at given N.
usage: variant_sweep.py nj m res N1,N2,... nvariants | v1,v2,... (-1 = auto)"""
import os, subprocess, sys
nj, m, res, Ns = sys.argv[1], sys.argv[2], sys.argv[3], sys.argv[4].split(",")
vs = [int(v) for v in sys.argv[5].split(",")] if "," in sys.argv[5] else list(range(-1, int(sys.argv[5])))
code = r'''
import sys, os; sys.path.insert(0, os.getcwd())
import torch
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W
nj, m, N, res = %s, %s, %s, "%s"
T = 30
tr = W.make_trajectory(nj, T + 10, 0)
g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), m=m, n_filters=N, resampler=res)
zs = torch.tensor(tr["Z"][1:], device="cuda"); us = torch.tensor(tr["U"][:-1], device="cuda")
g.step_batch(zs[:5], us[:5]); torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(g.stream); g.step_batch(zs[5:5+T], us[5:5+T]); e1.record(g.stream); torch.cuda.synchronize()
print(f"{e0.elapsed_time(e1) / T * 1e3:.1f}")
'''
for v in vs:
    env = dict(os.environ)
    if v >= 0:
        env["PF_VARIANT"] = str(v)
    out = []
    for N in Ns:
        r = subprocess.run([sys.executable, "-c", code % (nj, m, N, res)], capture_output=True, text=True, env=env)
        out.append(r.stdout.strip() or ("ERR " + r.stderr.strip().splitlines()[-1][:80] if r.stderr.strip() else "ERR"))
    print(f"variant {'auto' if v < 0 else v}: " + "  ".join(f"N={N}: {o} us" for N, o in zip(Ns, out)), flush=True)
