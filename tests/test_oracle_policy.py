"""Oracle pins for conditional resampling (§IV:
"we have experimented with the suggested metric to compute the effective
sample size as well as a simpler resampling frequency parameter (each
sub-filter randomly decides to resample at a fixed ratio of the time)";
reading R21, carried log-weight F12)."""
from fractions import Fraction

import numpy as np
import pytest


def test_ess_hand_example(orc):
    # q = [4, 1, 0, 3]: Q = 8, sum q^2 = 26, ESS = 64 / 26 = 2.4615...  (m = 4)
    q = [4, 1, 0, 3]
    assert not orc.should_resample("ess", orc.policy_param("ess", 0.60), q, 0, 0, 2)   # 2.4615 >= 2.40
    assert orc.should_resample("ess", orc.policy_param("ess", 0.62), q, 0, 0, 2)       # 2.4615 <  2.48


def test_ess_rule_brute_force(orc):
    # the integer rule Q^2 2^16 < param m S2 is exactly ESS < (param / 2^16) m
    rng = np.random.default_rng(0)
    for _ in range(300):
        m = int(rng.integers(1, 64))
        q = rng.integers(0, 1 << 22, m)
        q[rng.random(m) < 0.4] = 0
        q[int(rng.integers(0, m))] = 1 << 22            # the maximum (R8: q_max = 2^22)
        param = int(rng.integers(0, 1 << 17))
        Q, S2 = int(q.sum()), int((q.astype(object) ** 2).sum())
        want = Fraction(Q * Q, S2) < Fraction(param, 1 << 16) * m
        assert orc.should_resample("ess", param, q, 0, 0, 1) == want


def test_ess_uniform_never_below_m(orc):
    # uniform weights: ESS = m exactly, so tau <= 1 keeps the set and tau > 1 resamples
    q = np.full(16, 1 << 22)
    assert not orc.should_resample("ess", 1 << 16, q, 0, 0, 1)
    assert orc.should_resample("ess", (1 << 16) + 1, q, 0, 0, 1)
    onehot = np.zeros(16, np.int64)
    onehot[3] = 1 << 22                                 # ESS = 1
    assert orc.should_resample("ess", orc.policy_param("ess", 0.07), onehot, 0, 0, 1)   # 1 < 1.12
    assert not orc.should_resample("ess", orc.policy_param("ess", 0.06), onehot, 0, 0, 1)


def test_freq_ratio_and_bounds(orc):
    q = [1, 1]
    assert not any(orc.should_resample("freq", 0, q, 3, n, 5) for n in range(200))
    assert all(orc.should_resample("freq", 1 << 32, q, 3, n, 5) for n in range(200))
    ratio, trials = 0.3, 20000
    hits = sum(orc.should_resample("freq", orc.policy_param("freq", ratio), q, 3, n % 400, 2 + n // 400)
               for n in range(trials))
    assert abs(hits - ratio * trials) < 5 * np.sqrt(trials * ratio * (1 - ratio))


def _run(orc, W, cfg, nj, T):
    tr = W.make_trajectory(nj, T, 0)
    f = orc.Filter(cfg, orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"])
    for k in range(1, T + 1):
        f.step(tr["Z"][k], tr["U"][k - 1])
    return f, tr


@pytest.mark.parametrize("res", ["rws", "vose"])
def test_always_equivalent_policies(orc, W, res):
    # tau > 1 (ESS <= m always below tau m) and ratio 1 both resample every step:
    # bit-identical to the default policy
    base = dict(m=32, n_filters=6, t=1, topo="ring", resampler=res, seed=8)
    a, _ = _run(orc, W, orc.Config(**base), 2, 6)
    b, _ = _run(orc, W, orc.Config(**base, policy="ess", policy_param=orc.policy_param("ess", 1.5)), 2, 6)
    c, _ = _run(orc, W, orc.Config(**base, policy="freq", policy_param=1 << 32), 2, 6)
    for o in (b, c):
        np.testing.assert_array_equal(a.get()[0], o.get()[0])
        np.testing.assert_array_equal(a.get()[1], o.get()[1])


def test_never_resample_is_importance_sampling(orc, W):
    # tau = 0: no sub-filter ever resamples.  With no exchange every particle
    # then follows its own proposal path (ancestor = own slot) and its weight
    # is the product of its likelihoods: exp(l_i - max l) equals the float64
    # normalisation of exp(sum_k loglik_ik), computed here from single
    # sample+weight steps of the same Philox stream.
    nj, m, N, T = 2, 16, 3, 6
    cfg = orc.Config(m=m, n_filters=N, t=0, topo="none", seed=21, policy="ess", policy_param=0)
    tr = W.make_trajectory(nj, T, 0)
    f = orc.Filter(cfg, orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"])
    x, _, _ = f.get()                                   # the prior X_0
    total = np.zeros(N * m)
    for k in range(1, T + 1):
        f.step(tr["Z"][k], tr["U"][k - 1])
        x, ll = orc.sample_weight(orc.Model(n_joints=nj), 21, x, tr["Z"][k], tr["U"][k - 1], k)
        total += ll.astype(np.float64)
        s, w, _ = f.get()
        np.testing.assert_array_equal(s, x)             # no resampling: the proposal path itself
        _, anc = f.trace()
        np.testing.assert_array_equal(anc, np.tile(np.arange(m), N))
        for n in range(N):
            sl = slice(n * m, (n + 1) * m)
            ref = np.exp(total[sl] - total[sl].max())
            got = np.exp(w[sl].astype(np.float64) - w[sl].max())
            np.testing.assert_allclose(got, ref, rtol=2e-4, atol=1e-30)


def test_freq_mixed_steps(orc, W):
    # ratio 0.5: some sub-filters resample, others carry (F12): the kept ones
    # hold ancestor = own slot, their weight = (l - l_max) + loglik
    cfg = orc.Config(m=16, n_filters=8, t=0, topo="none", seed=5, policy="freq",
                     policy_param=orc.policy_param("freq", 0.5))
    tr = W.make_trajectory(2, 6, 0)
    f = orc.Filter(cfg, orc.Model(n_joints=2), tr["mu0"], tr["sigma0"])
    f.step(tr["Z"][1], tr["U"][0])
    kinds = set()
    for k in range(2, 6):
        s0, w0, _ = f.get()
        f.step(tr["Z"][k], tr["U"][k - 1])
        s1, w1, _ = f.get()
        _, anc = f.trace()
        for n in range(8):
            sl = slice(n * 16, (n + 1) * 16)
            res = orc.should_resample("freq", cfg.policy_param, orc.normalise(w0[sl]), 5, n, k)
            kinds.add(res)
            x, ll = orc.sample_weight(orc.Model(n_joints=2), 5, s0[:, sl] if not res else s0[:, sl][:, anc[sl]],
                                      tr["Z"][k], tr["U"][k - 1], k, p_offset=n * 16)
            np.testing.assert_array_equal(s1[:, sl], x)
            if res:
                np.testing.assert_array_equal(w1[sl], ll)
            else:
                np.testing.assert_array_equal(anc[sl], np.arange(16))
                np.testing.assert_array_equal(w1[sl], (w0[sl] - w0[sl].max()).astype(np.float32) + ll)
    assert kinds == {True, False}


# ---- weighted-average estimate (R22; §VI-D "a weighted average") ----

def test_weighted_mean_equal_weights_is_the_mean(orc):
    rng = np.random.default_rng(3)
    x = rng.normal(0, 2, (6, 1000)).astype(np.float32)
    got = orc.weighted_mean(x, np.full(1000, -3.25, np.float32))
    np.testing.assert_allclose(got, x.astype(np.float64).mean(axis=1), rtol=1e-6, atol=1e-7)


def test_weighted_mean_dominant_particle(orc):
    # every other weight below e^-16 of the best is dropped (F7): exactly that particle
    rng = np.random.default_rng(4)
    x = rng.normal(0, 1, (5, 300)).astype(np.float32)
    lw = rng.uniform(-80, -20, 300).astype(np.float32)
    lw[123] = -1.0
    np.testing.assert_array_equal(orc.weighted_mean(x, lw), x[:, 123])


def test_weighted_mean_vs_exact_weights(orc):
    # against the plain definition sum w x / sum w with float64 weights exp(l - L):
    # the 2^-22 quantisation of the integer weights bounds the difference
    rng = np.random.default_rng(5)
    for M in (7, 256, 4096):
        x = rng.normal(0, 1, (9, M)).astype(np.float32)
        lw = (-rng.exponential(2.0, M)).astype(np.float32)
        w = np.exp(lw.astype(np.float64) - lw.max())
        ref = (x.astype(np.float64) * w).sum(axis=1) / w.sum()
        got = orc.weighted_mean(x, lw)
        np.testing.assert_allclose(got, ref, rtol=0, atol=4 * M * 2.0**-22 / w.sum() * np.abs(x).max() + 1e-6)
        got64 = orc.weighted_mean(x, lw, fp64=True)
        np.testing.assert_allclose(got64, ref, rtol=0, atol=4 * M * 2.0**-22 / w.sum() * np.abs(x).max() + 1e-9)


def test_filter_mean_estimate_tracks(orc, W):
    # the weighted average of the filter's own set, after it converged, lies
    # near its max-weight estimate and near the true object position
    nj, T = 2, 40
    tr = W.make_trajectory(nj, T, 0)
    f = orc.Filter(orc.Config(m=64, n_filters=16, t=1, topo="ring", seed=2), orc.Model(n_joints=nj),
                   tr["mu0"], tr["sigma0"])
    err = []
    for k in range(1, T + 1):
        f.step(tr["Z"][k], tr["U"][k - 1])
        xm = f.estimate_mean()
        s, w, _ = f.get()
        np.testing.assert_array_equal(xm, orc.weighted_mean(s, w))
        err.append(np.hypot(*(xm[nj:nj + 2] - tr["X"][k][nj:nj + 2])))
    assert np.sqrt(np.mean(np.square(err[10:]))) < 0.25
