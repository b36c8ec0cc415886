"""Quick device timing of the step kernel (dev tool; bench.py is the contract)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W

def run(nj, m, N, res, T=50, topo="ring"):
    tr = W.make_trajectory(nj, T + 10, 0)
    g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), m=m, n_filters=N, resampler=res, topo=topo)
    zs = torch.tensor(tr["Z"][1:], device="cuda"); us = torch.tensor(tr["U"][:-1], device="cuda")
    g.step_batch(zs[:5], us[:5]); torch.cuda.synchronize()
    s = g.stream
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s); g.step_batch(zs[5:5+T], us[5:5+T]); e1.record(s); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / T
    M = m * N; d = nj + 4
    gbs = (8 * d + 8) * M / (ms * 1e-3) / 1e9
    print(f"nj={nj} m={m} N={N} {res} {topo}: {ms*1e3:.1f} us/step  {M/(ms*1e-3)/1e9:.2f} Gpart-steps/s  {gbs:.0f} GB/s algorithmic", flush=True)
    g.close()

for args in [(5,256,4096,"rws"),(5,256,4096,"vose"),(2,64,16,"rws"),(5,256,65536,"rws"),(28,256,65536,"vose"),(28,256,65536,"rws"),
             (5,32,131072,"rws"),(5,64,65536,"rws"),(5,128,32768,"rws"),(5,512,8192,"rws"),(5,1024,4096,"rws")]:
    run(*args)
