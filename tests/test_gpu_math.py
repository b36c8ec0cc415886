"""The device fp32 contract against the oracle's, bit for bit,
through the pf_debug_math test hook; and the kernels' branch-free sqrt
against IEEE sqrt.rn over the whole Box–Muller domain (F2)."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def B():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_chitchianasks13_b200 import binding, build
    build.build()
    return binding


def _f32bits(x):
    return np.ascontiguousarray(x, np.float32).view(np.uint32)


def test_sqrt_exhaustive_on_box_muller_domain(B):
    # -2 ln u1 for u1 in [2^-24, 1 - 2^-24] lies in [1.19e-7, 33.3]: check every float in [1e-7, 40]
    lo, hi = int(_f32bits([1e-7])[0]), int(_f32bits([40.0])[0])
    assert B.pf_debug_check_sqrt(lo, hi) == 0


@pytest.mark.parametrize("x2", [False, True], ids=["scalar", "packed"])
@pytest.mark.parametrize("fn", ["sin", "cos"])
def test_sincos_bit_exact(B, orc, fn, x2):
    rng = np.random.default_rng(1)
    # F5 domain |x| < 2^22 pi/2 (the quadrant index fits the 1.5 2^23 rounding add)
    x = np.concatenate([rng.uniform(-4, 4, 3000), rng.uniform(-60, 60, 3000), rng.uniform(-6.5e6, 6.5e6, 1000),
                        [0.0, -0.0, 0.7853981, 1e-30, 2.3561945, -2.3561945, 3.926991, -5.497787]])
    x = x.astype(np.float32)
    got = B.pf_debug_math(fn, _f32bits(x), len(x), x2).view(np.float32)
    ref = np.array([orc.s_sin(float(v)) if fn == "sin" else orc.s_cos(float(v)) for v in x], np.float32)
    np.testing.assert_array_equal(got.view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("x2", [False, True], ids=["scalar", "packed"])
def test_log_bit_exact(B, orc, x2):
    rng = np.random.default_rng(2)
    n1 = np.concatenate([rng.integers(1, 1 << 24, 5000) | 1, [1, (1 << 24) - 1]])
    u = (n1.astype(np.float64) * 2.0**-24).astype(np.float32)
    got = B.pf_debug_math("log", _f32bits(u), len(u), x2).view(np.float32)
    ref = np.array([orc.s_log(float(v)) for v in u], np.float32)
    np.testing.assert_array_equal(got.view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("x2", [False, True], ids=["scalar", "packed"])
def test_expq_bit_exact(B, orc, x2):
    rng = np.random.default_rng(3)
    d = np.concatenate([-rng.exponential(3.0, 5000), [0.0, -16.0, -16.0001, -15.25, -1e-8, -0.34657359, -1000.0,
                                                      -0.0]]).astype(np.float32)
    got = B.pf_debug_math("expq", _f32bits(d), len(d), x2)
    ref = np.array([orc.s_expq(float(v)) for v in d], np.uint32)
    np.testing.assert_array_equal(got, ref)


@pytest.mark.parametrize("x2", [False, True], ids=["scalar", "packed"])
def test_normal_pair_and_sincos2pi_bit_exact(B, orc, x2):
    rng = np.random.default_rng(4)
    n = 4000
    x0 = rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32)
    x1 = rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32)
    x0[:4] = [0, 0xFFFFFFFF, 0x1FF, 0x200]
    x1[4:8] = [0, 1 << 29, 2 << 29, 3 << 29]   # exact quadrant multiples: f = 0, signed zeros
    got = B.pf_debug_math("normal_pair", np.concatenate([x0, x1]), n, x2).view(np.float32).reshape(n, 2)
    ref = np.array([orc.s_normal_pair(int(a), int(b)) for a, b in zip(x0, x1)], np.float32)
    np.testing.assert_array_equal(got.view(np.uint32), ref.view(np.uint32))
    m = (x1 >> 9).astype(np.uint32)
    got2 = B.pf_debug_math("sincos2pi", m, n, x2).view(np.float32).reshape(n, 2)
    ref2 = np.array([orc.s_sincos2pi(int(v)) for v in m], np.float32)
    np.testing.assert_array_equal(got2.view(np.uint32), ref2.view(np.uint32))


def test_philox_kat_on_device(B, orc):
    import os
    from conftest import GOLDEN
    rows = [[int(v, 16) for v in l.split()] for l in open(os.path.join(GOLDEN, "philox_kat.txt"))
            if l.strip() and not l.startswith("#")]
    for r in rows:
        words = np.array([r[0], r[1], r[2], r[3], r[4], r[5]], np.uint32)
        out = B.pf_debug_math("philox", words, 1)
        assert list(map(int, out)) == r[6:10]


def test_sqrt_packed_matches_scalar(B):
    rng = np.random.default_rng(5)
    x = np.concatenate([rng.uniform(1.2e-7, 33.3, 4000), [1.1920929e-07, 33.27]]).astype(np.float32)
    a = B.pf_debug_math("sqrt", _f32bits(x), len(x))
    b = B.pf_debug_math("sqrt", _f32bits(x), len(x), True)
    np.testing.assert_array_equal(a, b)
    np.testing.assert_array_equal(a.view(np.float32), np.sqrt(x))
