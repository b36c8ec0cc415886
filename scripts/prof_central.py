"""Dev tool: the centralized filter with the bench's L2 flush before every step, for an ncu launch list
with --cache-control none (per-kernel times as they run after the flush).  usage: prof_central.py M res [steps]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W
M, res = int(sys.argv[1]), sys.argv[2]
steps = int(sys.argv[3]) if len(sys.argv) > 3 else 6
tr = W.make_trajectory(5, steps + 2, 0)
g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=5), m=M, n_filters=1, t=0, topo="none",
                     resampler=res, seed=7, device_inputs=True)
zs = torch.tensor(tr["Z"][1:], device="cuda"); us = torch.tensor(tr["U"][:-1], device="cuda")
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for k in range(steps):
    flush.zero_()
    g.step(zs[k], us[k])
torch.cuda.synchronize()
print("done")
