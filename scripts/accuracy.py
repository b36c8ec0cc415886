"""Estimation accuracy of the B200 filter over many runs (the
axes of the paper's Fig. 6, 7 and 9, §VII-D, §VIII-B).

For every configuration: R seeds x T steps of the medium robotic arm (d = 9,
Table II defaults, readings R15/R16) tracking the lemniscate; RMSE of the
estimated object position (R17) averaged over the seeds.  Steps run batched on
the device (pf_step_batch, estimates written on device, one sync per run).
Writes JSON lines; `--quick` runs a reduced grid.
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W


_TRAJ = {}


def rmse_runs(nj, m, N, topo, t, res, seeds, T):
    out = []
    d = nj + 4
    for s in seeds:
        if (nj, T, s) not in _TRAJ:
            _TRAJ[(nj, T, s)] = W.make_trajectory(nj, T, s)
        tr = _TRAJ[(nj, T, s)]
        g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), m=m, n_filters=N, t=t, topo=topo,
                             resampler=res, seed=s)
        zs = torch.tensor(tr["Z"][1:T + 1], device="cuda")
        us = torch.tensor(tr["U"][0:T], device="cuda")
        est = torch.zeros(T, 4 + d, device="cuda")
        g.step_batch(zs, us, est)
        e = est[:, 4 + nj:4 + nj + 2].cpu().numpy()
        g.close()
        err = np.hypot(*(e - tr["X"][1:T + 1, nj:nj + 2]).T)
        out.append(float(np.sqrt(np.mean(err ** 2))))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--seeds", type=int, default=100)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--quick", action="store_true")
    a = ap.parse_args()
    seeds = list(range(a.seeds))
    grid = []
    # Fig.6: exchange scheme x number of sub-filters x sub-filter size (t = 1)
    for topo in ["ring", "torus", "all2all"]:
        for N in ([16, 256] if a.quick else [16, 64, 256, 1024]):
            for m in ([64] if a.quick else [32, 64, 128, 256]):
                grid.append(("fig6", 5, m, N, topo, 1, "rws"))
    # Fig.7: particles per exchange (t = 0, 1, 2, 4; 64 x 64 ring and torus)
    for topo in ["ring", "torus", "all2all"]:
        for t in [0, 1, 2, 4]:
            grid.append(("fig7", 5, 64, 64, topo, t, "rws"))
    # Fig.9: distributed vs centralized with equal particle count (a single
    # sub-filter of m <= 1024 is the centralized filter)
    for M in [256, 1024]:
        grid.append(("fig9-central", 5, M, 1, "none", 0, "vose"))
        grid.append(("fig9-distributed", 5, 64, M // 64, "ring", 1, "rws"))
        grid.append(("fig9-distributed", 5, 32, M // 32, "torus", 1, "rws"))
    # RWS vs Vose (same distribution, R9/R10)
    grid.append(("resampler", 5, 64, 64, "ring", 1, "vose"))
    for tag, nj, m, N, topo, t, res in grid:
        r = rmse_runs(nj, m, N, topo, t, res, seeds, a.steps)
        print(json.dumps({"fig": tag, "n_joints": nj, "m": m, "N": N, "particles": m * N, "topo": topo, "t": t,
                          "resampler": res, "seeds": len(seeds), "steps": a.steps, "rmse_mean": float(np.mean(r)),
                          "rmse_sem": float(np.std(r) / np.sqrt(len(r)))}), flush=True)


if __name__ == "__main__":
    main()
