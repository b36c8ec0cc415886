"""Run a few steps of one config (for ncu). usage: profile_step.py NJ M N RES [steps]"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W
nj, m, N, res = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
T = int(sys.argv[5]) if len(sys.argv) > 5 else 4
tr = W.make_trajectory(nj, T + 2, 0)
g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), m=m, n_filters=N, resampler=res)
zs = torch.tensor(tr["Z"][1:T + 1], device="cuda"); us = torch.tensor(tr["U"][:T], device="cuda")
g.step_batch(zs, us); torch.cuda.synchronize(); print("done")
