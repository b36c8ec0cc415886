"""Weighted-average estimate on the GPU (§VI-D "a
weighted average"; reading R22) vs the oracle.  The integer weights are
bit-identical (F7 on both sides); the double numerators are summed in a
different order, so the bar is the rounding of the final fp32 quotient:
|gpu - oracle| <= 2 ulp-ish, asserted as 1e-6 relative (R18's 1e-5 bound
holds with margin)."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu
TOL = 1e-6


@pytest.fixture(scope="module")
def P():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_chitchianasks13_b200 import build, filter as F
    build.build()
    return F


def _close(a, b):
    a, b = np.asarray(a, np.float64), np.asarray(b, np.float64)
    assert np.all(np.abs(a - b) <= TOL * np.maximum(1.0, np.abs(b))), float(np.max(np.abs(a - b)))


@pytest.mark.parametrize("nj,m,N,topo,res", [(2, 64, 16, "ring", "rws"), (5, 256, 8, "torus", "vose"),
                                             (28, 32, 8, "ring", "rws"), (7, 64, 8, "ring", "rws"),
                                             (15, 128, 4, "ring", "vose")])   # (+ the generic arm: d = 11, 19)
def test_mean_estimate_trajectory(P, orc, W, nj, m, N, topo, res):
    T = 20
    tr = W.make_trajectory(nj, T, 0)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=m, n_filters=N, t=1, topo=topo,
                         resampler=res, seed=3)
    o = orc.Filter(orc.Config(m=m, n_filters=N, t=1, topo=topo, resampler=res, seed=3), orc.Model(n_joints=nj),
                   tr["mu0"], tr["sigma0"])
    for k in range(1, T + 1):
        g.step(tr["Z"][k], tr["U"][k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        _close(g.estimate_mean(), o.estimate_mean())
        assert g.estimate()[2] == o.estimate()[2]     # the max-weight record is untouched
    g.close()


@pytest.mark.parametrize("nj,m,N", [(5, 256, 4096), (28, 256, 1024)])
def test_mean_full_size(P, orc, W, nj, m, N):
    # C2 at full size (and a d = 32 set): the GPU mean of the GPU's own set vs
    # the oracle's weighted mean of that same set (read back)
    tr = W.make_trajectory(nj, 6, 1)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=m, n_filters=N, seed=17)
    for k in range(1, 4):
        g.step(tr["Z"][k], tr["U"][k - 1])
    s, w, _ = g.get_particles()
    _close(g.estimate_mean(), orc.weighted_mean(s, w))
    g.close()


@pytest.mark.parametrize("M,res", [(8192, "rws"), (12288, "vose")])
def test_mean_central(P, orc, W, M, res):
    tr = W.make_trajectory(5, 6, 1)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=5), m=M, n_filters=1, t=0, topo="none",
                         resampler=res, seed=5)
    for k in range(1, 5):
        g.step(tr["Z"][k], tr["U"][k - 1])
        s, w, _ = g.get_particles()
        _close(g.estimate_mean(), orc.weighted_mean(s, w))
    g.close()


@pytest.mark.parametrize("world", [2, 4])
def test_mean_sharded_loopback(P, orc, W, world):
    # world shards on one GPU: partial records with the global L after the
    # record reduce, gathered and reduced, vs the unsharded oracle filter
    import torch
    from paper_conf_ipps_chitchianasks13_b200 import distributed as Dd
    nj, m, N, T = 5, 64, 16, 5
    tr = W.make_trajectory(nj, T, 4)
    kw = dict(m=m, n_filters=N, t=1, topo="ring", resampler="rws", seed=11)
    shards = [P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), rank=r, world=world, **kw)
              for r in range(world)]
    o = orc.Filter(orc.Config(**kw), orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"])
    plan = Dd.halo_plan("ring", N, world)
    recs = torch.zeros(world, 4 + nj + 4, device="cuda")
    parts = torch.zeros(world, nj + 5, dtype=torch.float64, device="cuda")
    for k in range(1, T + 1):
        if k > 1:
            Dd.loopback_exchange([s.mailbox[(k - 1) & 1] for s in shards], plan)
        for s in shards:
            s.step(tr["Z"][k], tr["U"][k - 1])
        for r, s in enumerate(shards):
            recs[r] = s.record
        for s in shards:
            s.reduce_records(recs)
        for r, s in enumerate(shards):
            parts[r] = s.mean_partial()
        o.step(tr["Z"][k], tr["U"][k - 1])
        _close(shards[0].reduce_means(parts), o.estimate_mean())
    for s in shards:
        s.close()


def test_mean_errors(P, W):
    from paper_conf_ipps_chitchianasks13_b200 import binding as B
    tr = W.make_trajectory(5, 3, 0)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=5), m=64, n_filters=4)
    with pytest.raises(B.PFError):   # before the first step
        g.estimate_mean()
    g.close()


@pytest.mark.parametrize("res", ["rws", "vose"])
def test_mean_central_aos(P, orc, W, res):
    # the centralized filter's AoS records: the mean of the GPU's own set vs
    # the oracle's weighted mean of that set (read back through get_particles)
    tr = W.make_trajectory(5, 6, 2)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=5), m=16384, n_filters=1, t=0, topo="none",
                         resampler=res, seed=8)
    for k in range(1, 5):
        g.step(tr["Z"][k], tr["U"][k - 1])
    s, w, _ = g.get_particles()
    _close(g.estimate_mean(), orc.weighted_mean(s, w))
    g.close()
