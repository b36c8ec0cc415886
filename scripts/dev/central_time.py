"""Dev: centralized filter step time under different timing regimes."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W
M = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 20
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for _ in range(300):   # ramp the clocks up before timing
    flush.zero_()
torch.cuda.synchronize()
for res in ("rws", "vose"):
    tr = W.make_trajectory(5, 40, 0)
    g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=5), m=M, n_filters=1, t=0, topo="none",
                         resampler=res, seed=7, device_inputs=True)
    zs = torch.tensor(tr["Z"][1:], device="cuda"); us = torch.tensor(tr["U"][:-1], device="cuda")
    for k in range(3):
        g.step(zs[k], us[k])
    torch.cuda.synchronize()
    out = {}
    for mode in ("flush", "flush_sync", "batch"):
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(10)]
        if mode == "batch":
            ev[0][0].record(g.stream)
            g.step_batch(zs[3:23], us[3:23])
            ev[0][1].record(g.stream)
            torch.cuda.synchronize()
            out[mode] = ev[0][0].elapsed_time(ev[0][1]) / 20 * 1e3
            continue
        for i in range(10):
            with torch.cuda.stream(g.stream):
                flush.zero_()
            if mode == "flush_sync":
                torch.cuda.synchronize()
            ev[i][0].record(g.stream)
            g.step(zs[3 + i], us[3 + i])
            ev[i][1].record(g.stream)
        torch.cuda.synchronize()
        out[mode] = sum(a.elapsed_time(b) for a, b in ev) / 10 * 1e3
    print(M, res, {k: round(v, 1) for k, v in out.items()}, flush=True)
    g.close()
