"""Oracle pins: integer RWS and Vose resampling (§IV,
:20–22 §VI-F; readings R7–R11 of DESIGN.md §3)."""
import json
import os

import numpy as np
import pytest
from scipy import stats

from conftest import GOLDEN

G = json.load(open(os.path.join(GOLDEN, "resample_golden.json")))


def test_rws_golden(orc):
    for case in G["rws"]:
        assert orc.rws_draw(G["q"], case["U"]) == case["a"]


def test_vose_golden(orc):
    prob, alias = orc.vose_build(G["q"])
    assert list(prob) == G["vose_table"]["prob"]
    assert list(alias) == G["vose_table"]["alias"]
    for case in G["vose"]:
        assert orc.vose_draw(prob, alias, G["Q"], case["Ua"], case["Ub"]) == case["a"]


def _alias_mass(q, prob, alias):
    m, Q = len(q), int(np.sum(q, dtype=np.uint64))
    mass = np.zeros(m, np.int64)
    for b in range(m):
        mass[b] += int(prob[b])
        mass[int(alias[b])] += Q - int(prob[b])
    return mass


@pytest.mark.parametrize("kind", ["mixed", "uniform", "onehot"])
def test_vose_exact_mass(orc, W, kind):
    # every slot j receives exactly m*q_j of the m*Q table mass (alias invariant:
    # the table reproduces the distribution q/Q exactly, and the mass sums to 1)
    for m in (1, 2, 3, 4, 7, 32, 64, 100, 256, 1024):
        q = W.random_q(3, m, m, kind)
        for row in q:
            prob, alias = orc.vose_build(row)
            assert np.all(prob <= int(row.sum(dtype=np.uint64)))
            np.testing.assert_array_equal(_alias_mass(row, prob, alias), m * row.astype(np.int64))


def _closed_form_alias(q):
    """Independent derivation of the sweep's table (R10): with D the
    inclusive deficits over small slots L and E the inclusive excesses over
    large slots H, small L[i] takes alias H[#{h: E_h < D_{i-1}}] and large H[h]
    with E_h < D_last ends at Q + E_h - D[first i: D_i > E_h], alias H[h+1]."""
    q = np.asarray(q, np.int64)
    m, Q = len(q), int(q.sum())
    a = m * q
    L = [j for j in range(m) if a[j] < Q]
    H = [j for j in range(m) if a[j] >= Q]
    D = np.cumsum([Q - a[j] for j in L]) if L else np.zeros(0, np.int64)
    E = np.cumsum([a[j] - Q for j in H]) if H else np.zeros(0, np.int64)
    prob = np.full(m, Q, np.int64)
    alias = np.arange(m)
    for i, s in enumerate(L):
        prev = D[i - 1] if i > 0 else 0
        prob[s] = a[s]
        alias[s] = H[int(np.searchsorted(E, prev, side="left"))]
    Dl = D[-1] if len(D) else 0
    for h, j in enumerate(H):
        if E[h] < Dl:
            prob[j] = Q + E[h] - D[int(np.searchsorted(D, E[h], side="right"))]
            alias[j] = H[h + 1]
    return prob, alias


def test_vose_sweep_equals_closed_form(orc, W):
    rng = np.random.default_rng(5)
    for trial in range(300):
        m = int(rng.integers(1, 300))
        kind = ["mixed", "uniform", "onehot"][trial % 3]
        row = W.random_q(1, m, trial, kind)[0]
        if trial % 7 == 0:
            row[rng.random(m) < 0.5] = 0
            row[rng.integers(0, m)] = 1 << 22
        prob, alias = orc.vose_build(row)
        p2, a2 = _closed_form_alias(row)
        np.testing.assert_array_equal(prob.astype(np.int64), p2)
        np.testing.assert_array_equal(alias, a2)


def test_rws_is_papers_highest_index_rule(orc, W):
    # "highest index with a [cumulative] weight not larger than the drawn
    # number" over the exclusive sums, restricted to slots with weight > 0
    # (R9) == first inclusive sum exceeding the draw; zero slots never drawn
    rng = np.random.default_rng(6)
    q = W.random_q(1, 64, 0)[0]
    q[rng.random(64) < 0.3] = 0
    q[5] = 1 << 22
    excl = np.concatenate([[0], np.cumsum(q.astype(np.int64))[:-1]])
    Q = int(q.sum(dtype=np.uint64))
    for U in rng.integers(0, 2**32, 3000):
        c = (int(U) * Q) >> 32
        cand = [j for j in range(64) if q[j] > 0 and excl[j] <= c]
        a = orc.rws_draw(q, int(U))
        assert a == max(cand) and q[a] > 0


def test_uniform_weights_identical_indices(orc, W):
    # uniform weights: RWS and Vose both give a = floor(U_a m / 2^32)
    N, m = 8, 64
    q = W.random_q(N, m, 0, "uniform")
    rng = np.random.default_rng(7)
    ua = rng.integers(0, 2**32, (N, m), dtype=np.uint64).astype(np.uint32)
    ub = rng.integers(0, 2**32, (N, m), dtype=np.uint64).astype(np.uint32)
    expect = ((ua.astype(np.uint64) * m) >> 32).astype(np.int32)
    np.testing.assert_array_equal(orc.resample_q(q, "rws", ua, ub), expect)
    np.testing.assert_array_equal(orc.resample_q(q, "vose", ua, ub), expect)


def test_onehot_draws_that_slot(orc, W):
    N, m = 16, 32
    q = W.random_q(N, m, 1, "onehot")
    rng = np.random.default_rng(8)
    ua = rng.integers(0, 2**32, (N, m), dtype=np.uint64).astype(np.uint32)
    ub = rng.integers(0, 2**32, (N, m), dtype=np.uint64).astype(np.uint32)
    hot = np.argmax(q, 1)
    for r in ("rws", "vose"):
        anc = orc.resample_q(q, r, ua, ub)
        assert np.all(anc == hot[:, None])


@pytest.mark.slow
def test_rws_vose_same_multinomial(orc, W):
    # 10^6 draws each: chi-square vs q/Q, and RWS-vs-Vose two-sample (alpha 1e-3)
    m = 64
    rng = np.random.default_rng(9)
    ell = -rng.chisquare(7, m) / 2
    row = np.floor(np.exp(ell - ell.max()) * 2**22).astype(np.uint32)
    n_rows = 1_000_000 // m
    q = np.tile(row, (n_rows, 1))
    ua = rng.integers(0, 2**32, q.shape, dtype=np.uint64).astype(np.uint32)
    ub = rng.integers(0, 2**32, q.shape, dtype=np.uint64).astype(np.uint32)
    p = row / row.sum()
    counts = {}
    for r in ("rws", "vose"):
        anc = orc.resample_q(q, r, ua, ub).ravel()
        counts[r] = np.bincount(anc, minlength=m)
        keep = p > 0
        assert counts[r][~keep].sum() == 0
        chi = stats.chisquare(counts[r][keep], p[keep] * len(anc))
        assert chi.pvalue > 1e-3, (r, chi)
    keep = (counts["rws"] + counts["vose"]) > 0
    tab = np.stack([counts["rws"][keep], counts["vose"][keep]])
    assert stats.chi2_contingency(tab).pvalue > 1e-3


def test_normalise(orc, W):
    # q = floor(2^22 exp(l - lmax)) (R7, R8): the best slot gets exactly 2^22,
    # order is preserved, and shifting all log-weights changes nothing
    w = W.random_logw(1, 256, 0)[0]
    q = orc.normalise(w)
    assert q.max() == 1 << 22 and q[np.argmax(w)] == 1 << 22
    order = np.argsort(-w, kind="stable")
    assert np.all(np.diff(q[order].astype(np.int64)) <= 0)
    np.testing.assert_array_equal(orc.normalise(w - np.float32(64.0)), q)


def test_resample_logw_matches_components(orc, W):
    # normalise + Philox (p, k, 0, 0) words 0-1 + resample_q compose exactly
    cfg = orc.Config(m=64, n_filters=4, resampler="vose", seed=(3 << 32) | 11)
    w = W.random_logw(4, 64, 1)
    anc, q = orc.resample_logw(cfg, w, 5)
    ua = np.zeros((4, 64), np.uint32)
    ub = np.zeros((4, 64), np.uint32)
    for p in range(256):
        b = orc.philox([p, 5, 0, 0], [11, 3])
        ua.flat[p], ub.flat[p] = b[0], b[1]
    for n in range(4):
        np.testing.assert_array_equal(q[n], orc.normalise(w[n]))
    np.testing.assert_array_equal(anc, orc.resample_q(q, "vose", ua, ub))
