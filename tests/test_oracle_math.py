"""Oracle pins: the fp32 arithmetic contract F3–F7 against
float64 libm.  The paper computes in fp32 (§VI) and compares
against a double-precision reference; these bounds show the specified
evaluations are accurate fp32 functions, so fixing them changes no result
beyond fp32 rounding."""
import numpy as np


def test_sin_cos_accuracy(orc):
    rng = np.random.default_rng(0)
    xs = np.concatenate([rng.uniform(-4, 4, 4000), rng.uniform(-100, 100, 4000),
                         [0.0, np.pi / 4, -np.pi / 4, np.pi / 2, np.pi, 3.0]]).astype(np.float32)
    es = max(abs(orc.s_sin(float(x)) - np.sin(np.float64(x))) for x in xs)
    ec = max(abs(orc.s_cos(float(x)) - np.cos(np.float64(x))) for x in xs)
    assert es < 2.5e-7 and ec < 2.5e-7   # ~2 ulp(1)
    assert orc.s_sin(0.0) == 0.0 and orc.s_cos(0.0) == 1.0


def test_sincos2pi_accuracy_and_quadrants(orc):
    rng = np.random.default_rng(1)
    ms = np.concatenate([rng.integers(0, 2**23, 4000), [0, 1 << 21, 1 << 22, 3 << 21, (1 << 23) - 1]])
    for m in ms:
        s, c = orc.s_sincos2pi(int(m))
        a = 2 * np.pi * int(m) / 2**23
        assert abs(s - np.sin(a)) < 2.5e-7 and abs(c - np.cos(a)) < 2.5e-7
    # exact quadrant points
    assert orc.s_sincos2pi(0) == (0.0, 1.0)
    assert orc.s_sincos2pi(1 << 21) == (1.0, -0.0) or orc.s_sincos2pi(1 << 21) == (1.0, 0.0)


def test_log_accuracy(orc):
    # the whole Box–Muller domain u1 = n 2^-23, n = 1..2^23 (strided) + random
    rng = np.random.default_rng(2)
    us = np.concatenate([np.arange(1, 2**23 + 1, 4093) * 2.0**-23, rng.uniform(0.5, 1, 4000), [1.0]])
    us = us.astype(np.float32)
    for u in us:
        ref = np.log(np.float64(u))
        assert abs(orc.s_log(float(u)) - ref) <= 1.5e-7 * max(1.0, abs(ref))
    assert orc.s_log(1.0) == 0.0


def test_expq_floor_exp(orc):
    # q = floor(2^22 exp(delta)) up to one unit (F7, R8); exact ends
    rng = np.random.default_rng(3)
    ds = np.concatenate([-rng.uniform(0, 16, 6000), -rng.uniform(0, 1e-4, 500)]).astype(np.float32)
    for d in ds:
        ref = int(np.floor(np.exp(np.float64(d)) * 2**22))
        assert 0 <= orc.s_expq(float(d)) - ref <= 1
    assert orc.s_expq(0.0) == 1 << 22
    assert orc.s_expq(-16.0001) == 0 and orc.s_expq(-1000.0) == 0
    # monotone non-increasing in |delta|
    grid = -np.linspace(0, 16, 20001).astype(np.float32)
    q = [orc.s_expq(float(d)) for d in grid]
    assert all(a >= b for a, b in zip(q, q[1:]))
