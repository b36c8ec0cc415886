"""Model hooks (§I: "Our application separates generic particle
filtering from model-specific routines"): the step kernels are templates over
a model policy (csrc/pf_model.cuh); the 1-D linear-Gaussian model runs
through the same kernels as the arm and is checked against the oracle (bit
for bit) and against the Kalman filter (SURVEY §8(c) whole-filter pin (ii))."""
import math

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

H_S, SQ, SR = 0.1, 0.1, 0.2


@pytest.fixture(scope="module")
def P():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_chitchianasks13_b200 import build, filter as F
    build.build()
    return F


def _models(P, orc):
    return (P.LinearGaussModel(h_s=H_S, sigma_theta=SQ, sigma_theta_meas=SR),
            orc.Model(kind="lg1", h_s=H_S, sigma_theta=SQ, sigma_theta_meas=SR))


@pytest.mark.parametrize("m,N,topo,t,res", [
    (256, 64, "ring", 1, "rws"), (256, 64, "ring", 1, "vose"), (64, 16, "torus", 2, "rws"),
    (1024, 4, "all2all", 2, "vose"), (32, 8, "none", 0, "rws"), (128, 32, "ring", 3, "vose")])
def test_lg_trajectory_bit_exact(P, orc, W, m, N, topo, t, res):
    tr = W.make_lg_trajectory(20, 1, sigma_theta=SQ, sigma_meas=SR)
    gm, om = _models(P, orc)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], gm, m=m, n_filters=N, t=t, topo=topo, resampler=res, seed=9)
    o = orc.Filter(orc.Config(m=m, n_filters=N, t=t, topo=topo, resampler=res, seed=9), om, tr["mu0"], tr["sigma0"])
    for k in range(1, 21):
        g.step(tr["Z"][k], tr["U"][k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        xg, lg, ig = g.estimate()
        xo, lo, io = o.estimate()
        assert ig == io, (k, ig, io)
        np.testing.assert_array_equal(xg, xo)
        assert lg == lo
    sg, wg, _ = g.get_particles()
    so, wo, _ = o.get()
    np.testing.assert_array_equal(sg, so)
    np.testing.assert_array_equal(wg, wo)
    g.close()


def test_lg_sample_weight_bit_exact(P, orc, W):
    tr = W.make_lg_trajectory(10, 2, sigma_theta=SQ, sigma_meas=SR)
    gm, om = _models(P, orc)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], gm, m=256, n_filters=16, seed=5)
    s_in = (np.random.default_rng(3).standard_normal((1, 4096)) * 0.3).astype(np.float32)
    for k in (1, 6):
        sg, wg = g.debug_sample_weight(s_in, tr["Z"][k], tr["U"][k - 1], k)
        so, wo = orc.sample_weight(om, 5, s_in, tr["Z"][k], tr["U"][k - 1], k)
        np.testing.assert_array_equal(sg, so)
        np.testing.assert_array_equal(wg, wo)
    g.close()


def _kalman(tr, T):
    m, Pk = float(tr["mu0"][0]), float(tr["sigma0"][0]) ** 2
    out = []
    for k in range(1, T + 1):
        m, Pk = m + H_S * float(tr["U"][k - 1][0]), Pk + SQ * SQ
        K = Pk / (Pk + SR * SR)
        m, Pk = m + K * (float(tr["Z"][k][0]) - m), (1 - K) * Pk
        out.append((m, Pk))
    return out


@pytest.mark.parametrize("res", ["rws", "vose"])
def test_lg_central_kalman_and_oracle(P, orc, W, res):
    # centralized filter (N = 1, m = 102400 = 25 x 4096): the weighted mean and
    # variance of every step against the Kalman posterior within MC error, and
    # step 5 slot by slot against the oracle (from the GPU's step-4 set)
    T, m = 20, 102400
    tr = W.make_lg_trajectory(T, 0, sigma_theta=SQ, sigma_meas=SR)
    gm, om = _models(P, orc)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], gm, m=m, n_filters=1, t=0, topo="none", resampler=res, seed=4)
    cfg = orc.Config(m=m, n_filters=1, t=0, topo="none", resampler=res, seed=4)
    prev = None
    for k, (mk, Pk) in enumerate(_kalman(tr, T), 1):
        g.step(tr["Z"][k], tr["U"][k - 1])
        s, w, _ = g.get_particles()
        if k == 5:
            slots = np.r_[0:64, m - 64:m, np.random.default_rng(1).integers(0, m, 256)]
            os_, ow = orc.central_slots(cfg, om, prev[0], prev[1], 5, tr["Z"][5], tr["U"][4], slots)
            np.testing.assert_array_equal(s[:, slots], os_)
            np.testing.assert_array_equal(w[slots], ow)
        prev = (s, w)
        ww = np.exp(w.astype(np.float64) - w.max())
        ess = ww.sum() ** 2 / (ww ** 2).sum()
        mean = float(g.estimate_mean()[0])
        x = s[0].astype(np.float64)
        mu = (ww * x).sum() / ww.sum()
        var = (ww * (x - mu) ** 2).sum() / ww.sum()
        assert abs(mean - mk) < 5 * math.sqrt(Pk / ess), (k, mean, mk)
        assert abs(var / Pk - 1) < 5 * math.sqrt(2 / ess), (k, var, Pk)
    g.close()


def test_lg_streamed_batched_same(P, W):
    import torch
    tr = W.make_lg_trajectory(12, 3, sigma_theta=SQ, sigma_meas=SR)
    gm = P.LinearGaussModel(h_s=H_S, sigma_theta=SQ, sigma_theta_meas=SR)
    a = P.ParticleFilter(tr["mu0"], tr["sigma0"], gm, m=128, n_filters=64, seed=2)
    b = P.ParticleFilter(tr["mu0"], tr["sigma0"], gm, m=128, n_filters=64, seed=2)
    for k in range(1, 13):
        a.step(tr["Z"][k], tr["U"][k - 1])
    b.step_batch(torch.tensor(tr["Z"][1:13], device="cuda"), torch.tensor(tr["U"][0:12], device="cuda"))
    np.testing.assert_array_equal(a.get_particles()[0], b.get_particles()[0])
    a.close()
    b.close()


@pytest.mark.parametrize("nj,m,N,topo,res", [(3, 64, 16, "ring", "rws"), (7, 128, 8, "torus", "vose"),
                                             (12, 256, 4, "ring", "rws"), (1, 32, 8, "all2all", "rws"),
                                             (20, 1024, 2, "ring", "vose")])
def test_generic_arm_bit_exact(P, orc, W, nj, m, N, topo, res):
    # any n_joints: the generic arm (runtime dimensions, pf_model.cuh ArmDyn)
    # against the oracle, every step and the final set bit for bit
    tr = W.make_trajectory(nj, 12, 2)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=m, n_filters=N, t=1, topo=topo,
                         resampler=res, seed=11)
    o = orc.Filter(orc.Config(m=m, n_filters=N, t=1, topo=topo, resampler=res, seed=11), orc.Model(n_joints=nj),
                   tr["mu0"], tr["sigma0"])
    for k in range(1, 13):
        g.step(tr["Z"][k], tr["U"][k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        xg, lg, ig = g.estimate()
        xo, lo, io = o.estimate()
        assert ig == io, (k, ig, io)
        np.testing.assert_array_equal(xg, xo)
    sg, wg, _ = g.get_particles()
    so, wo, _ = o.get()
    np.testing.assert_array_equal(sg, so)
    np.testing.assert_array_equal(wg, wo)
    g.close()


def test_generic_arm_sample_weight(P, orc, W):
    nj = 9
    tr = W.make_trajectory(nj, 6, 3)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=256, n_filters=8, seed=21)
    s_in = W.random_particles(tr, 2048, 4)
    sg, wg = g.debug_sample_weight(s_in, tr["Z"][2], tr["U"][1], 2)
    so, wo = orc.sample_weight(orc.Model(n_joints=nj), 21, s_in, tr["Z"][2], tr["U"][1], 2)
    np.testing.assert_array_equal(sg, so)
    np.testing.assert_array_equal(wg, wo)
    g.close()
