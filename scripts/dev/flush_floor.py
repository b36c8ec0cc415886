"""Dev probe: what the flushed C2 step time is made of.  Times (CUDA events on
the filter's stream, median of 30) an empty torch kernel and the C2 step after:
no flush, the bench's 512 MiB write flush, and a write flush followed by a
512 MiB read (L2 then holds clean lines of another buffer)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W

nj, m, N = 5, 256, 4096
tr = W.make_trajectory(nj, 200, 0)
g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), m=m, n_filters=N, device_inputs=True)
zs = torch.tensor(tr["Z"][1:], device="cuda"); us = torch.tensor(tr["U"][:-1], device="cuda")
fl = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
rd = torch.ones(512 << 20, dtype=torch.uint8, device="cuda")
tiny = torch.zeros(32, device="cuda")
k = [0]
def step():
    g.step(zs[k[0] % 190], us[k[0] % 190]); k[0] += 1
def empty():
    with torch.cuda.stream(g.stream):
        tiny.add_(1.0)
for _ in range(10): step()
torch.cuda.synchronize()
for name, fn in (("empty", empty), ("step", step)):
    for fmode in ("none", "write", "write+read"):
        ts = []
        for r in range(30):
            if fmode != "none": fl.zero_()
            if fmode == "write+read": rd.sum()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(g.stream); fn(); e1.record(g.stream)
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e3)
        print(f"{name:6s} flush={fmode:10s} median {np.median(ts):7.2f} us  p10 {np.percentile(ts,10):7.2f}  p90 {np.percentile(ts,90):7.2f}")
