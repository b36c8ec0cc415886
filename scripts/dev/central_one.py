"""Dev: a few steps of the centralized filter (for ncu). usage: central_one.py M res [steps] [nj]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W
M, res = int(sys.argv[1]), sys.argv[2]
steps = int(sys.argv[3]) if len(sys.argv) > 3 else 4
nj = int(sys.argv[4]) if len(sys.argv) > 4 else 5
tr = W.make_trajectory(nj, steps + 2, 0)
g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), m=M, n_filters=1, t=0, topo="none",
                     resampler=res, seed=7, device_inputs=True)
zs = torch.tensor(tr["Z"][1:], device="cuda"); us = torch.tensor(tr["U"][:-1], device="cuda")
for k in range(steps):
    g.step(zs[k], us[k])
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(g.stream)
for k in range(steps):
    g.step(zs[k % steps], us[k % steps])
e1.record(g.stream); torch.cuda.synchronize()
print("done", M, res, f"{e0.elapsed_time(e1) / steps * 1e3:.1f} us/step (back to back)")
