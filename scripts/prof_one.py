"""Dev tool: run a few steps of one configuration (for ncu capture of the step kernel).
usage: prof_one.py nj m N res [topo] [t] [steps]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W
nj, m, N, res = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
topo = sys.argv[5] if len(sys.argv) > 5 else "ring"
t = int(sys.argv[6]) if len(sys.argv) > 6 else 1
steps = int(sys.argv[7]) if len(sys.argv) > 7 else 4
tr = W.make_trajectory(nj, steps + 2, 0)
g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), m=m, n_filters=N, t=t, topo=topo,
                     resampler=res, seed=7, device_inputs=True)
zs = torch.tensor(tr["Z"][1:], device="cuda"); us = torch.tensor(tr["U"][:-1], device="cuda")
for k in range(steps):
    g.step(zs[k], us[k])
torch.cuda.synchronize()
print("done", nj, m, N, res, topo, t, steps)
