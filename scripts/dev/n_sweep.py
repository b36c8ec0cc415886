"""Dev: flushed step time vs number of sub-filters around C2 (tail / rounds effect)."""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for _ in range(200): flush.zero_()
for N in [int(a) for a in sys.argv[1:]]:
    tr = W.make_trajectory(5, 60, 0)
    g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=5), m=256, n_filters=N, device_inputs=True)
    zs = torch.tensor(tr["Z"][1:], device="cuda"); us = torch.tensor(tr["U"][:-1], device="cuda")
    for k in range(5): g.step(zs[k], us[k])
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(30)]
    for i in range(30):
        with torch.cuda.stream(g.stream): flush.zero_()
        ev[i][0].record(g.stream); g.step(zs[5 + i], us[5 + i]); ev[i][1].record(g.stream)
    torch.cuda.synchronize()
    t = statistics.median(a.elapsed_time(b) * 1e3 for a, b in ev)
    print(f"N={N:6d} ({N / 1776:.2f} rounds of 1776 groups): {t:6.1f} us  {t / N * 1000:6.2f} ns per sub-filter", flush=True)
    g.close()
