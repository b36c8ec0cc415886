"""Accuracy against an exact reference (SURVEY NEXT-3 + the Kalman special
case of §8(c)): the 1-D linear-Gaussian model (pf.h PF_MODEL_LINEAR_GAUSS_1D)
has the Kalman filter as its exact posterior, so the particle filter's error
can be measured against the optimum instead of only against the ground truth.
For the paper's design axes (§VII-D: exchange scheme, number and
size of sub-filters, centralized vs distributed at equal particle count):
RMSE of the weighted-mean estimate (R22) against the Kalman mean, in units of
the posterior std (sqrt P_k), and the RMSE against the ground truth of the
weighted mean, the max-weight estimate (R6) and the Kalman filter itself.
Writes JSON lines (profiles/r02_accuracy_kalman.jsonl)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W

H_S, SQ, SR = 0.1, 0.1, 0.2


def kalman(tr, T):
    m, P = float(tr["mu0"][0]), float(tr["sigma0"][0]) ** 2
    ms, Ps = [], []
    for k in range(1, T + 1):
        m, P = m + H_S * float(tr["U"][k - 1][0]), P + SQ * SQ
        K = P / (P + SR * SR)
        m, P = m + K * (float(tr["Z"][k][0]) - m), (1 - K) * P
        ms.append(m)
        Ps.append(P)
    return np.array(ms), np.array(Ps)


def run(m, N, topo, t, res, seeds, T):
    rows = []
    for s in seeds:
        tr = W.make_lg_trajectory(T, s, sigma_theta=SQ, sigma_meas=SR)
        km, kP = kalman(tr, T)
        g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.LinearGaussModel(h_s=H_S, sigma_theta=SQ, sigma_theta_meas=SR),
                             m=m, n_filters=N, t=t, topo=topo, resampler=res, seed=s)
        mean, mx = [], []
        for k in range(1, T + 1):
            g.step(tr["Z"][k], tr["U"][k - 1])
            mean.append(float(g.estimate_mean()[0]))
            mx.append(float(g.estimate()[0][0]))
        g.close()
        truth = tr["X"][1:T + 1, 0].astype(np.float64)
        mean, mx = np.array(mean), np.array(mx)
        rows.append((np.sqrt(np.mean((mean - km) ** 2 / kP)), np.sqrt(np.mean((mean - truth) ** 2)),
                     np.sqrt(np.mean((mx - truth) ** 2)), np.sqrt(np.mean((km - truth) ** 2))))
    r = np.array(rows)
    return {"m": m, "N": N, "particles": m * N, "topo": topo, "t": t, "resampler": res, "seeds": len(seeds),
            "steps": T, "mean_vs_kalman_in_post_std": float(r[:, 0].mean()),
            "rmse_mean": float(r[:, 1].mean()), "rmse_maxweight": float(r[:, 2].mean()),
            "rmse_kalman": float(r[:, 3].mean()), "sem_mean_vs_kalman": float(r[:, 0].std() / np.sqrt(len(r)))}


def main():
    seeds, T = list(range(int(os.environ.get("SEEDS", "30")))), 50
    grid = [(16384, 1, "none", 0, "vose"), (16384, 1, "none", 0, "rws"), (4096, 1, "none", 0, "vose")]
    for m, N in [(64, 256), (256, 64), (1024, 16)]:
        for topo, t in [("none", 0), ("ring", 1), ("torus", 1), ("all2all", 1)]:
            grid.append((m, N, topo, t, "rws"))
    for m, N in [(64, 64), (32, 128)]:   # equal particle count to the 4096 centralized filter
        grid.append((m, N, "ring", 1, "rws"))
    for cfg in grid:
        print(json.dumps(run(*cfg, seeds, T)), flush=True)


if __name__ == "__main__":
    main()
