"""Oracle pins for the whole filter (Algorithm 2, §IV) —
invariants, special cases and the paper's validation methodology
(convergence to a known ground truth, §VIII-A; fp32 vs fp64,
PAPER.md:18 §VI)."""
import numpy as np
import pytest


def _run(orc, W, cfg, nj, T, seed=0, fp64=False, traj_seed=0, traj_len=None):
    tr = W.make_trajectory(nj, traj_len or T, traj_seed)
    f = orc.Filter(cfg, orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"], fp64=fp64)
    est = []
    for k in range(1, T + 1):
        f.step(tr["Z"][k], tr["U"][k - 1])
        est.append(f.estimate())
    return f, tr, est


def _rmse(tr, est, nj):
    e = [np.hypot(*(x[nj:nj + 2] - tr["X"][k + 1][nj:nj + 2])) for k, (x, _, _) in enumerate(est)]
    return float(np.sqrt(np.mean(np.square(e))))


def test_estimate_is_global_argmax(orc, W):
    cfg = orc.Config(m=32, n_filters=8, t=1, topo="ring", seed=4)
    f, tr, est = _run(orc, W, cfg, 2, 5)
    s, w, k = f.get()
    assert k == 5
    x, lw, idx = est[-1]
    best = max(range(len(w)), key=lambda p: (w[p], -p))
    assert idx == best and lw == w[best]
    np.testing.assert_array_equal(x, s[:, best])


def test_t0_subfilters_independent_of_N(orc, W):
    # with no exchange each sub-filter is its own filter: its trajectory does
    # not depend on how many other sub-filters run (global Philox counters, R13)
    a, _, _ = _run(orc, W, orc.Config(m=32, n_filters=4, t=0, topo="none", seed=2), 2, 8)
    b, _, _ = _run(orc, W, orc.Config(m=32, n_filters=9, t=0, topo="ring", seed=2), 2, 8)
    sa, wa, _ = a.get()
    sb, wb, _ = b.get()
    np.testing.assert_array_equal(sa, sb[:, :4 * 32])
    np.testing.assert_array_equal(wa, wb[:4 * 32])


def test_resampled_states_come_from_post_exchange_set(orc, W):
    # one step from a set()-injected state: every new particle = sample of an
    # ancestor that is a post-exchange particle of its own sub-filter
    cfg = orc.Config(m=16, n_filters=4, t=1, topo="ring", seed=1)
    md = orc.Model(n_joints=2)
    tr = W.make_trajectory(2, 10, 0)
    f = orc.Filter(cfg, md, tr["mu0"], tr["sigma0"])
    s0 = W.random_particles(tr, 64, 3)
    w0 = W.random_logw(4, 16, 3).ravel()
    f.set(s0, w0, 3)
    f.step(tr["Z"][4], tr["U"][3])
    src, anc = f.trace()
    np.testing.assert_array_equal(src, orc.exchange(cfg, w0.reshape(4, 16)).ravel())
    # recompute: gather post-exchange ancestors, then sample_weight at k = 4
    pre = s0[:, src]
    gathered = np.stack([pre[:, (p // 16) * 16 + anc[p]] for p in range(64)], 1)
    out, lw = orc.sample_weight(md, 1, gathered, tr["Z"][4], tr["U"][3], 4)
    s1, w1, k = f.get()
    assert k == 4
    np.testing.assert_array_equal(s1, out)
    np.testing.assert_array_equal(w1, lw)
    ancq, _ = orc.resample_logw(cfg, w0[src].reshape(4, 16), 4)
    np.testing.assert_array_equal(anc.reshape(4, 16), ancq)


def test_get_set_roundtrip_is_bit_exact(orc, W):
    cfg = orc.Config(m=32, n_filters=4, t=1, topo="torus", resampler="vose", seed=3)
    a, tr, _ = _run(orc, W, cfg, 5, 6, traj_len=12)
    s, w, k = a.get()
    b = orc.Filter(cfg, orc.Model(n_joints=5), tr["mu0"], tr["sigma0"])
    b.set(s, w, k)
    for kk in range(k + 1, k + 4):
        a.step(tr["Z"][kk], tr["U"][kk - 1])
        b.step(tr["Z"][kk], tr["U"][kk - 1])
    np.testing.assert_array_equal(a.get()[0], b.get()[0])


def test_rejects_invalid_config(orc):
    md = orc.Model(n_joints=2)
    mu, sg = np.zeros(6), np.ones(6)
    with pytest.raises(ValueError):
        orc.Filter(orc.Config(m=4, n_filters=4, t=2, topo="ring"), md, mu, sg)   # deg*t >= m (R19)
    with pytest.raises(ValueError):
        orc.Filter(orc.Config(m=8, n_filters=6, t=1, topo="torus", torus_rows=4, torus_cols=2), md, mu, sg)


@pytest.mark.slow
def test_lemniscate_convergence(orc, W):
    # PAPER.md:28 §VIII-A, Fig.8: the filter tracks the known ground truth,
    # and more particles track better
    r_small = np.mean([_rmse(*_run(orc, W, orc.Config(m=8, n_filters=4, t=1, seed=s), 2, 100, traj_seed=s)[1:], 2)
                       for s in range(6)])
    r_big = np.mean([_rmse(*_run(orc, W, orc.Config(m=64, n_filters=64, t=1, seed=s), 2, 100, traj_seed=s)[1:], 2)
                     for s in range(6)])
    assert r_big < r_small
    assert r_big < 0.2      # object moves on a 2 m wide figure-eight; noise 0.1 m


@pytest.mark.slow
def test_fp32_matches_fp64_accuracy(orc, W):
    # PAPER.md:18 §VI: double precision "does not improve our estimation
    # accuracy by a meaningful amount" — mean RMSE over seeds within MC error
    r32, r64 = [], []
    for s in range(12):
        cfg = orc.Config(m=64, n_filters=16, t=1, seed=s)
        r32.append(_rmse(*_run(orc, W, cfg, 2, 60, traj_seed=s)[1:], 2))
        r64.append(_rmse(*_run(orc, W, cfg, 2, 60, traj_seed=s, fp64=True)[1:], 2))
    diff = np.array(r32) - np.array(r64)
    se = np.std(r32 + r64) / np.sqrt(len(r32))
    assert abs(np.mean(diff)) < 3 * se + 1e-3


def test_step_subset_equals_whole_filter(orc, W):
    # the one-sub-filter-at-a-time oracle used for full-size sampled checks
    # reproduces the whole-filter step exactly
    for topo, res, t in [("ring", "rws", 1), ("torus", "vose", 2), ("none", "rws", 0), ("all2all", "rws", 2)]:
        cfg = orc.Config(m=32, n_filters=16, t=t, topo=topo, resampler=res, seed=5)
        md = orc.Model(n_joints=5)
        tr = W.make_trajectory(5, 10, 0)
        f = orc.Filter(cfg, md, tr["mu0"], tr["sigma0"])
        s0 = W.random_particles(tr, 512, 1)
        w0 = W.random_logw(16, 32, 1).ravel()
        f.set(s0, w0, 3)
        f.step(tr["Z"][4], tr["U"][3])
        s1, w1, _ = f.get()
        subs = [0, 5, 15, 7]
        os_, ow = orc.step_subset(cfg, md, s0, w0, 4, tr["Z"][4], tr["U"][3], subs)
        for i, n in enumerate(subs):
            np.testing.assert_array_equal(os_[:, i * 32:(i + 1) * 32], s1[:, n * 32:(n + 1) * 32])
            np.testing.assert_array_equal(ow[i * 32:(i + 1) * 32], w1[n * 32:(n + 1) * 32])


def test_central_slots_equals_whole_filter(orc, W):
    # the slot-sampled centralized oracle reproduces the whole-filter step
    for res in ("rws", "vose"):
        cfg = orc.Config(m=2048, n_filters=1, t=0, topo="none", resampler=res, seed=21)
        md = orc.Model(n_joints=5)
        tr = W.make_trajectory(5, 10, 0)
        f = orc.Filter(cfg, md, tr["mu0"], tr["sigma0"])
        s0 = W.random_particles(tr, 2048, 4)
        w0 = W.random_logw(1, 2048, 4).ravel()
        f.set(s0, w0, 2)
        f.step(tr["Z"][3], tr["U"][2])
        s1, w1, _ = f.get()
        slots = [0, 1, 777, 2047]
        os_, ow = orc.central_slots(cfg, md, s0, w0, 3, tr["Z"][3], tr["U"][2], slots)
        np.testing.assert_array_equal(os_, s1[:, slots])
        np.testing.assert_array_equal(ow, w1[slots])


@pytest.mark.parametrize("nj,m,N,res", [(2, 64, 16, "rws"), (2, 64, 16, "vose"), (5, 256, 16, "rws")])
def test_fp32_trajectory_matches_fp64_elementwise(orc, W, nj, m, N, res):
    # the fp32 contract (F1-F11) against the independent float64 / libm
    # oracle, element by element over 10 steps (every particle, every step):
    # within the north_star's 1e-5 relative bar, and no integer decision
    # (order, exchange, q, ancestor, argmax) differs (§VI)
    tr = W.make_trajectory(nj, 10, 0)
    cfg = orc.Config(m=m, n_filters=N, t=1, topo="ring", resampler=res, seed=3)
    a = orc.Filter(cfg, orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"])
    b = orc.Filter(cfg, orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"], fp64=True)
    for k in range(1, 11):
        a.step(tr["Z"][k], tr["U"][k - 1])
        b.step(tr["Z"][k], tr["U"][k - 1])
        s32, w32, _ = a.get()
        s64, w64, _ = b.get()
        np.testing.assert_array_less(np.abs(s32 - s64), 1e-5 * np.maximum(1, np.abs(s64)))
        np.testing.assert_array_less(np.abs(w32 - w64), 1e-5 * np.maximum(1, np.abs(w64)))
        assert a.estimate()[2] == b.estimate()[2]
