"""Oracle pins for the prior draw a0 (F11, reading R13 stream 2): the
implicit input X_0 of Algorithm 2 ("Input: X, z, n particles, n filters,
n transfers", §IV) drawn as X_0 ~ N(mu0, diag sigma0^2) (the
filters "start in the center on the right off the ground truth", PAPER.md:28
Fig.8).  Pinned against the mathematics, not against the oracle itself:
(1) the per-component moments and the KS distance of >= 10^5 draws against
N(mu0_c, sigma0_c^2); (2) the Philox word layout of stream 2 recomputed here
(pair q of particle p = words 2(q&1), 2(q&1)+1 of counter (p, 0, 2, q>>1),
Box–Muller in float64 from the KAT-pinned Philox words); (3) the fp32 and
fp64 oracles agree to fp32 rounding."""
import math

import numpy as np
import pytest
from scipy import stats

MU = np.array([0.3, -0.2, 0.1, 0.0, -0.4, 0.9, 0.05, -0.3, 0.2], np.float32)
SIG = np.array([0.1, 0.2, 0.05, 0.3, 0.15, 0.25, 0.5, 0.01, 1.0], np.float32)


def _prior(orc, m, N, seed, fp64=False, nj=5):
    cfg = orc.Config(m=m, n_filters=N, t=0, topo="none", seed=seed)
    f = orc.Filter(cfg, orc.Model(n_joints=nj), MU[:nj + 4], SIG[:nj + 4], fp64=fp64)
    s, w, k = f.get()
    assert k == 0
    return s, w


def _bm64(x0, x1):
    # F2 in real arithmetic: u1 = the midpoint of the 23-bit cell of 1 - u(x0)
    u1 = 1.0 - ((x0 >> 9) + 0.5) * 2.0 ** -23
    u2 = (x1 >> 9) * 2.0 ** -23
    r = math.sqrt(-2.0 * math.log(u1))
    return r * math.cos(2 * math.pi * u2), r * math.sin(2 * math.pi * u2)


@pytest.mark.slow
def test_prior_moments_and_ks(orc):
    s, w = _prior(orc, 1024, 128, seed=(3 << 32) | 11)    # 131072 particles
    n = s.shape[1]
    assert np.all(w == 0.0)                               # unweighted prior
    x = s.astype(np.float64)
    for c in range(9):
        mu, sg = float(MU[c]), float(SIG[c])
        m1 = x[c].mean()
        v1 = x[c].var()
        assert abs(m1 - mu) < 5 * sg / math.sqrt(n), (c, m1, mu)            # mean, 5 sigma
        assert abs(v1 / sg ** 2 - 1) < 5 * math.sqrt(2.0 / n), (c, v1, sg)  # variance, 5 sigma
        p = stats.kstest((x[c] - mu) / sg, "norm").pvalue
        assert p > 1e-3, (c, p)
    # components are independent draws: a sigma on the wrong component or a
    # shared word would correlate them
    cc = np.corrcoef(x)
    assert np.max(np.abs(cc - np.eye(9))) < 5 / math.sqrt(n)


@pytest.mark.parametrize("fp64", [False, True])
def test_prior_philox_stream2_layout(orc, fp64):
    seed = (7 << 32) | 5
    s, _ = _prior(orc, 32, 4, seed, fp64=fp64)
    key = [seed & 0xFFFFFFFF, seed >> 32]
    for p in (0, 1, 31, 64, 127):
        ref = []
        for q in range(5):                                # (d + 1) / 2 pairs, d = 9
            wds = orc.philox([p, 0, 2, q >> 1], key)
            ref += list(_bm64(int(wds[2 * (q & 1)]), int(wds[2 * (q & 1) + 1])))
        xi = np.array(ref[:9])
        exp = MU.astype(np.float64) + SIG.astype(np.float64) * xi
        np.testing.assert_allclose(s[:, p], exp, rtol=0, atol=2e-6 if not fp64 else 1e-12)


def test_prior_draw_differs_from_step_stream(orc):
    # stream 2 (init) is not stream 0 (step): X_0 of particle p must not be
    # built from the words of counter (p, 0, 0, j)
    seed = 9
    s, _ = _prior(orc, 32, 1, seed, nj=2)
    key = [seed, 0]
    wds = orc.philox([0, 0, 0, 0], key)
    z0, _ = _bm64(int(wds[0]), int(wds[1]))
    assert abs(s[0, 0] - (MU[0] + SIG[0] * z0)) > 1e-4


def test_prior_fp32_vs_fp64(orc):
    s32, _ = _prior(orc, 256, 8, seed=123)
    s64, _ = _prior(orc, 256, 8, seed=123, fp64=True)
    np.testing.assert_allclose(s32, s64, rtol=0, atol=3e-6)
