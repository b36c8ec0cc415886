"""Conditional resampling on the GPU (§IV; reading
R21, carried log-weight F12) vs the oracle, element by element: the ESS rule
and the per-sub-filter resampling coin decide identically (exact integers /
the same Philox word), kept sub-filters carry l - l_max, and the trajectories
are bit-identical."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def P():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_chitchianasks13_b200 import build, filter as F
    build.build()
    return F


def _pair(P, orc, W, nj, m, N, t, topo, res, policy, value, seed, T):
    tr = W.make_trajectory(nj, T, 0)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=m, n_filters=N, t=t, topo=topo,
                         resampler=res, seed=seed, policy=policy, policy_value=value)
    o = orc.Filter(orc.Config(m=m, n_filters=N, t=t, topo=topo, resampler=res, seed=seed, policy=policy,
                              policy_param=orc.policy_param(policy, value)),
                   orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"])
    return tr, g, o


@pytest.mark.parametrize("nj,m,N,t,topo,res,policy,value", [
    (2, 64, 16, 1, "ring", "rws", "ess", 0.05),      # C1 shape
    (5, 256, 16, 1, "ring", "vose", "ess", 0.02),    # packed two-particle path (P = 4)
    (5, 32, 32, 0, "none", "rws", "freq", 0.4),      # one particle per thread
    (5, 128, 64, 2, "torus", "rws", "freq", 0.25),
    (28, 256, 4, 1, "ring", "vose", "ess", 0.005),   # high-DOF arm
    (5, 1024, 4, 2, "torus", "vose", "freq", 0.5),   # u64 scans, P = 8
    (2, 64, 16, 0, "none", "rws", "ess", 0.0),       # never resample
])
def test_policy_trajectory_bit_exact(P, orc, W, nj, m, N, t, topo, res, policy, value):
    T = 12
    tr, g, o = _pair(P, orc, W, nj, m, N, t, topo, res, policy, value, seed=nj * 31 + m, T=T)
    g.set_trace(True)
    kept_seen = resampled_seen = False
    for k in range(1, T + 1):
        g.step(tr["Z"][k], tr["U"][k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        xg, lg, ig = g.estimate()
        xo, lo, io = o.estimate()
        assert ig == io, f"estimate index differs at step {k}"
        np.testing.assert_array_equal(xg, xo)
        src_g, anc_g = g.trace()
        src_o, anc_o = o.trace()
        np.testing.assert_array_equal(anc_g, anc_o)
        if k > 1:
            ident = (anc_o.reshape(N, m) == np.arange(m)).all(axis=1)
            kept_seen |= bool(ident.any())
            resampled_seen |= bool((~ident).any())
    sg, wg, _ = g.get_particles()
    so, wo, _ = o.get()
    np.testing.assert_array_equal(sg, so)
    np.testing.assert_array_equal(wg, wo)
    assert kept_seen                    # some sub-filter kept its set (else the test would not test R21)
    if value > 0:
        assert resampled_seen
    g.close()


def test_policy_full_size_sampled(P, orc, W):
    # C2 at full size (4096 x 256, ring t = 1) with the ESS rule, the bench's
    # launch configuration: one step from a generator-made weighted set, the
    # oracle recomputes a sample of sub-filters one by one
    nj, m, N, t = 5, 256, 4096, 1
    tr = W.make_trajectory(nj, 10, 2)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=m, n_filters=N, t=t, topo="ring",
                         seed=99, policy="ess", policy_value=0.05)
    s0 = W.random_particles(tr, m * N, 5)
    w0 = W.random_logw(N, m, 5).ravel()
    g.set_particles(s0, w0, 4)
    g.set_trace(True)
    g.step(tr["Z"][5], tr["U"][4])
    sg, wg, _ = g.get_particles()
    _, anc = g.trace()
    kept = np.flatnonzero((anc.reshape(N, m) == np.arange(m)).all(axis=1))
    assert 0 < len(kept) < N
    rng = np.random.default_rng(7)
    subs = np.unique(np.concatenate([[0, N - 1, N // 2], rng.integers(0, N, 21), kept[:8]]))
    cfg = orc.Config(m=m, n_filters=N, t=t, topo="ring", seed=99, policy="ess",
                     policy_param=orc.policy_param("ess", 0.05))
    so, wo = orc.step_subset(cfg, orc.Model(n_joints=nj), s0, w0, 5, tr["Z"][5], tr["U"][4], subs)
    for i, n in enumerate(subs):
        np.testing.assert_array_equal(sg[:, n * m:(n + 1) * m], so[:, i * m:(i + 1) * m], err_msg=f"sf {n}")
        np.testing.assert_array_equal(wg[n * m:(n + 1) * m], wo[i * m:(i + 1) * m], err_msg=f"sf {n}")
    g.close()


def test_policy_errors(P, W):
    from paper_conf_ipps_chitchianasks13_b200 import binding as B
    tr = W.make_trajectory(5, 4, 0)
    with pytest.raises(B.PFError):   # the centralized filter always resamples
        P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=5), m=4096, n_filters=1, t=0, topo="none",
                         policy="ess", policy_value=0.5)
    with pytest.raises(B.PFError):   # ratio above 1
        P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=5), m=64, n_filters=4, policy="freq",
                         policy_value=1.5)
