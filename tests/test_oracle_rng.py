"""Oracle pins: Philox4x32-10 and Box–Muller (reading R12, DESIGN.md §3;
the paper's MTGP + Box–Muller kernel is PAPER.md:20 §VI-A)."""
import math
import os

import numpy as np
import pytest
from scipy import stats

from conftest import GOLDEN


def _kat():
    rows = []
    for line in open(os.path.join(GOLDEN, "philox_kat.txt")):
        if line.strip() and not line.startswith("#"):
            rows.append([int(v, 16) for v in line.split()])
    return rows


def test_philox_known_answers(orc):
    rows = _kat()
    assert len(rows) == 3
    for r in rows:
        out = orc.philox(r[0:4], r[4:6])
        assert [int(v) for v in out] == r[6:10]


def test_philox_counter_sensitivity(orc):
    # every counter/key word changes the block (no ignored input word)
    base = orc.philox([5, 3, 0, 0], [42, 0])
    for i in range(4):
        c = [5, 3, 0, 0]
        c[i] ^= 1
        assert not np.array_equal(orc.philox(c, [42, 0]), base)
    assert not np.array_equal(orc.philox([5, 3, 0, 0], [42, 1]), base)


def test_normal_pair_golden(orc):
    gold = [float(v) for v in open(os.path.join(GOLDEN, "normals_golden.txt")).read().split("\n")[-2].split()]
    words = list(orc.philox([0, 1, 0, 0], [42, 0])) + list(orc.philox([0, 1, 0, 1], [42, 0]))
    z = []
    for q in range(3):
        z += list(orc.s_normal_pair(int(words[2 + 2 * q]), int(words[3 + 2 * q])))
    np.testing.assert_allclose(z, gold, atol=1e-5, rtol=0)


def _words(n, seed):
    rng = np.random.default_rng(seed)
    return rng.integers(0, 2**32, size=(n, 2), dtype=np.uint64)


def test_normal_pair_fp32_vs_fp64(orc):
    # the fp32 contract (F2) agrees with libm double Box–Muller within 1e-5
    w = _words(20000, 1)
    # include the extremes u1 = 2^-24 (r = 5.77) and u1 = 1 - 2^-24 (r = 3.5e-4)
    w[0] = [0xFFFFFFFF, 0x12345678]
    w[1] = [0x000001FF, 0x9ABCDEF0]
    err = 0.0
    for x0, x1 in w:
        a = orc.s_normal_pair(int(x0), int(x1))
        b = orc.d_normal_pair(int(x0), int(x1))
        err = max(err, float(np.max(np.abs(a - b))))
    assert err < 1e-5


@pytest.mark.slow
def test_box_muller_moments_and_ks(orc):
    # 10^6 normals from Philox blocks (p, 1, 0, j): mean, variance, KS
    n_pairs = 500_000
    z = np.empty(2 * n_pairs)
    for p in range(n_pairs // 2):
        w = orc.philox([p, 1, 0, 0], [7, 0])
        z[4 * p:4 * p + 2] = orc.s_normal_pair(int(w[0]), int(w[1]))
        z[4 * p + 2:4 * p + 4] = orc.s_normal_pair(int(w[2]), int(w[3]))
    n = len(z)
    assert abs(z.mean()) < 5 / math.sqrt(n)
    assert abs(z.var() - 1) < 5 * math.sqrt(2 / n)
    assert stats.kstest(z, "norm").pvalue > 1e-3
