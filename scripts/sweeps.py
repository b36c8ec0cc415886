"""Throughput sweeps on one B200 (SURVEY.md §8 configs C3/C4 and the paper's
Fig.3/4/5 axes: particle count, sub-filter size m, exchange count t, state
dimension, RWS vs Vose).  Device-resident inputs, L2 flushed before every
timed step (CUDA events around each launch).  Writes JSON lines to stdout."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W

flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")


def run(tag, nj, m, N, res="rws", topo="ring", t=1, steps=20, warm=3, policy="always", value=1.0):
    tr = W.make_trajectory(nj, steps + warm + 4, 0)
    g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), m=m, n_filters=N, t=t, topo=topo,
                         resampler=res, seed=7, device_inputs=True, policy=policy, policy_value=value)
    zs = torch.tensor(tr["Z"][1:], device="cuda")
    us = torch.tensor(tr["U"][:-1], device="cuda")
    for k in range(warm):
        g.step(zs[k], us[k])
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    for i in range(steps):
        flush.zero_()
        ev[i][0].record(g.stream)
        g.step(zs[warm + i], us[warm + i])
        ev[i][1].record(g.stream)
    torch.cuda.synchronize()
    ms = sum(a.elapsed_time(b) for a, b in ev) / steps
    M, d = m * N, nj + 4
    bytes_ = M * 8 * (d + 1)
    out = {"sweep": tag, "n_joints": nj, "d": d, "m": m, "N": N, "particles": M, "resampler": res, "topo": topo,
           "t": t, "policy": policy, "policy_value": value, "us_per_step": ms * 1e3, "estimates_per_s": 1e3 / ms, "particle_steps_per_s": M / (ms * 1e-3),
           "hbm_gbs_algorithmic": bytes_ / (ms * 1e-3) / 1e9}
    print(json.dumps(out), flush=True)
    g.close()


if __name__ == "__main__":
    which = sys.argv[1:] or ["count", "m", "t", "dim", "res", "central", "policy"]
    if "count" in which:   # Fig.3 / Fig.4b analogue: particle count (m = 256, d = 9)
        for N in [4, 16, 64, 256, 1024, 4096, 16384, 65536, 262144, 390625]:
            run("count", 5, 256, N, steps=10 if N > 100000 else 20)
    if "m" in which:       # Fig.4a / C3: sub-filter size at 4M particles
        for m in [32, 64, 128, 256, 512, 1024]:
            run("m", 5, m, (1 << 22) // m)
    if "t" in which:       # Fig.7 / C3: exchange count at 4M (ring and torus)
        for topo in ["ring", "torus", "all2all"]:
            for t in [0, 1, 2, 4]:
                run("t", 5, 256, 16384, topo=topo, t=t)
    if "dim" in which:     # Fig.4c / C4: state dimension (n_j = 2, 5, 28 compiled; the others the generic arm)
        for nj in [2, 5, 28]:
            run("dim", nj, 256, 65536)
        for nj in [3, 7, 11, 16, 22]:
            run("dim-generic", nj, 256, 65536)
    if "res" in which:     # Fig.5: RWS vs Vose
        for nj, N in [(5, 4096), (5, 65536), (28, 65536)]:
            for res in ["rws", "vose"]:
                run("res", nj, 256, N, res=res)
    if "central" in which:  # Fig.5 centralized curves / Fig.9: one filter of M particles (NEXT-2)
        for M in [1 << 14, 1 << 16, 1 << 18, 1 << 20]:
            for res in ["rws", "vose"]:
                run("central", 5, M, 1, res=res, topo="none", t=0)
    if "policy" in which:   # §IV conditional resampling (NEXT-4) at C2
        for policy, value in [("always", 1.0), ("ess", 0.05), ("freq", 0.5), ("freq", 0.1)]:
            run("policy", 5, 256, 4096, policy=policy, value=value)
