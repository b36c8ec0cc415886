"""Device time of the step kernel for one config: usage NJ M N RES [T] (dev tool)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W
from paper_conf_ipps_chitchianasks13_b200 import binding as B
nj, m, N, res = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
T = int(sys.argv[5]) if len(sys.argv) > 5 else 30
tr = W.make_trajectory(nj, T + 10, 0)
g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), m=m, n_filters=N, resampler=res)
zs = torch.tensor(tr["Z"][1:], device="cuda"); us = torch.tensor(tr["U"][:-1], device="cuda")
g.step_batch(zs[:5], us[:5]); torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(g.stream); g.step_batch(zs[5:5 + T], us[5:5 + T]); e1.record(g.stream); torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / T
M = m * N; d = nj + 4
print(f"nj={nj} m={m} N={N} {res}: {ms*1e3:8.1f} us/step {M/(ms*1e-3)/1e9:6.2f} Gps/s {(8*d+8)*M/(ms*1e-3)/1e9:6.0f} GB/s")
