"""Small workload for compute-sanitizer (memcheck / racecheck / synccheck /
initcheck): a few steps of every mapping family and exchange scheme."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from paper_conf_ipps_chitchianasks13_b200 import filter as F, workload as W

cases = [(2, 64, 16, 1, "ring", "rws"), (5, 256, 8, 2, "torus", "vose"), (5, 32, 16, 1, "all2all", "rws"),
         (5, 256, 64, 1, "ring", "rws"), (28, 256, 4, 1, "ring", "vose"), (28, 256, 4, 1, "ring", "rws"), (5, 1024, 4, 3, "torus", "rws"),
         (5, 128, 16, 2, "all2all", "vose")]
for nj, m, N, t, topo, res in cases:
    tr = W.make_trajectory(nj, 6, 1)
    g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), m=m, n_filters=N, t=t, topo=topo,
                         resampler=res, seed=3)
    g.set_trace(True)
    for k in range(1, 5):
        g.step(tr["Z"][k], tr["U"][k - 1])
        g.estimate()
    g.trace()
    w = W.random_logw(N, m, 2).ravel()
    g.debug_exchange(w)
    q = W.random_q(N, m, 3)
    g.debug_resample(q, q, q)
    g.close()
    print("ok", nj, m, N, t, topo, res, flush=True)
# the generic arm (runtime dimensions), the linear-Gaussian model, the centralized filter (RWS / Vose)
for nj, m, N, t, topo, res in [(3, 64, 8, 1, "ring", "vose"), (11, 256, 4, 1, "torus", "rws")]:
    tr = W.make_trajectory(nj, 6, 1)
    g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=nj), m=m, n_filters=N, t=t, topo=topo,
                         resampler=res, seed=3)
    for k in range(1, 5):
        g.step(tr["Z"][k], tr["U"][k - 1])
        g.estimate()
    g.close()
    print("ok generic", nj, m, N, t, topo, res, flush=True)
tr = W.make_lg_trajectory(6, 0)
g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.LinearGaussModel(), m=128, n_filters=16, resampler="vose", seed=3)
for k in range(1, 5):
    g.step(tr["Z"][k], tr["U"][k - 1])
    g.estimate()
g.close()
print("ok lg1", flush=True)
for res in ("rws", "vose"):
    tr = W.make_trajectory(5, 6, 1)
    g = F.ParticleFilter(tr["mu0"], tr["sigma0"], F.ArmModel(n_joints=5), m=8192, n_filters=1, t=0, topo="none",
                         resampler=res, seed=3)
    for k in range(1, 5):
        g.step(tr["Z"][k], tr["U"][k - 1])
        g.estimate()
    q = W.random_q(1, 8192, 3)
    g.debug_resample(q, q, q)
    g.close()
    print("ok central", res, flush=True)
