"""Whole-filter pin (ii) of SURVEY §8(c): the Kalman special case.

The 1-D linear-Gaussian model (one joint of the arm with its angle sensor,
no camera: theta_k = theta_{k-1} + h_s u + w, z_k = theta_k + v; pf.h
PF_MODEL_LINEAR_GAUSS_1D) has the exact posterior N(m_k, P_k) of the Kalman
filter.  The oracle's particle filter (Algorithm 2, one
centralized filter, N = 1) must reproduce it within Monte-Carlo error: the
weighted mean (R22, §VI-D "a weighted average") within 5 standard
errors sqrt(P_k / ESS_k), the weighted variance within 5 sqrt(2 / ESS_k)
relative, at every step.  The Kalman recursion is written here in float64,
independently of the oracle."""
import math

import numpy as np
import pytest

H_S, SQ, SR = 0.1, 0.1, 0.2   # distinct process / measurement noise (a swapped sigma fails)


def kalman(tr, T):
    m, P = float(tr["mu0"][0]), float(tr["sigma0"][0]) ** 2
    out = []
    for k in range(1, T + 1):
        m, P = m + H_S * float(tr["U"][k - 1][0]), P + SQ * SQ          # predict
        K = P / (P + SR * SR)                                           # update
        m, P = m + K * (float(tr["Z"][k][0]) - m), (1 - K) * P
        out.append((m, P))
    return out


def _check(f, tr, T):
    for k, (mk, Pk) in enumerate(kalman(tr, T), 1):
        f.step(tr["Z"][k], tr["U"][k - 1])
        s, w, _ = f.get()
        ww = np.exp(w.astype(np.float64) - w.max())
        ess = ww.sum() ** 2 / (ww ** 2).sum()
        mean = float(f.estimate_mean()[0])
        x = s[0].astype(np.float64)
        mu = (ww * x).sum() / ww.sum()
        var = (ww * (x - mu) ** 2).sum() / ww.sum()
        assert abs(mean - mk) < 5 * math.sqrt(Pk / ess), (k, mean, mk, Pk, ess)
        assert abs(var / Pk - 1) < 5 * math.sqrt(2 / ess), (k, var, Pk, ess)


@pytest.mark.parametrize("res,m", [("vose", 102400), ("rws", 8192)])
def test_kalman_special_case(orc, W, res, m):
    # N = 1, m = 10^5 (Vose: O(1) draws); the oracle's RWS is the plain
    # linear scan (O(m^2) per step), so it is pinned at m = 8192
    T = 20
    for seed in (0, 1):
        tr = W.make_lg_trajectory(T, seed, sigma_theta=SQ, sigma_meas=SR)
        md = orc.Model(kind="lg1", h_s=H_S, sigma_theta=SQ, sigma_theta_meas=SR)
        cfg = orc.Config(m=m, n_filters=1, t=0, topo="none", resampler=res, seed=seed)
        _check(orc.Filter(cfg, md, tr["mu0"], tr["sigma0"]), tr, T)


def test_lg_model_hooks(orc):
    # F8 joint row and the F10 joint term in closed form
    md = orc.Model(kind="lg1", h_s=0.1, sigma_theta=0.0, sigma_theta_meas=0.5)
    s = np.array([[0.25, -1.0, 3.0]], np.float32)
    u = np.array([2.0], np.float32)
    z = np.array([0.75], np.float32)
    out, lw = orc.sample_weight(md, 1, s, z, u, 1)
    np.testing.assert_array_equal(out[0], s[0] + np.float32(0.1) * np.float32(2.0))   # sigma = 0: deterministic
    exp = -0.5 * ((0.75 - out[0].astype(np.float64)) / 0.5) ** 2
    np.testing.assert_allclose(lw, exp, rtol=1e-6)
    assert orc.loglik(md, [0.25], [0.75]) == -0.5      # residual = one sigma => -1/2 exactly


def test_lg_noise_is_first_normal(orc):
    # theta' - (theta + h_s u) = sigma * (first Box–Muller normal of Philox (p, k, 0, 0) words 2, 3)
    md = orc.Model(kind="lg1", h_s=0.1, sigma_theta=0.3, sigma_theta_meas=0.1)
    s = np.zeros((1, 8), np.float32)
    out, _ = orc.sample_weight(md, 11, s, [0.0], [0.0], 4, fp64=True)
    for p in range(8):
        w = orc.philox([p, 4, 0, 0], [11, 0])
        u1 = 1 - ((int(w[2]) >> 9) + 0.5) * 2.0 ** -23
        u2 = (int(w[3]) >> 9) * 2.0 ** -23
        xi = math.sqrt(-2 * math.log(u1)) * math.cos(2 * math.pi * u2)
        assert abs(out[0, p] - np.float64(np.float32(0.3)) * xi) < 1e-9
