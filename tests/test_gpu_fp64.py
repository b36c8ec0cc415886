"""The CUDA path against the INDEPENDENT float64 / libm oracle (orc_d_*,
PAPER.md:18 §VI "double precision reference"), element by element at the
north_star's 1e-5 relative bar — not only transitively through the fp32
oracle that shares the kernels' arithmetic contract."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

TOL = 1e-5


def _close(a, b):
    a, b = np.asarray(a, np.float64), np.asarray(b, np.float64)
    err = np.abs(a - b) / np.maximum(1.0, np.abs(b))
    assert np.all(err <= TOL), float(err.max())


@pytest.fixture(scope="module")
def P():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_chitchianasks13_b200 import build, filter as F
    build.build()
    return F


def test_sample_weight_c2_vs_fp64(P, orc, W):
    # config C2 (medium arm, 4096 x 256 = 2^20 particles): a1-a3 of every particle
    nj, m, N = 5, 256, 4096
    tr = W.make_trajectory(nj, 10, 1)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=m, n_filters=N, seed=77)
    s_in = W.random_particles(tr, m * N, 3)
    sg, wg = g.debug_sample_weight(s_in, tr["Z"][3], tr["U"][2], 3)
    so, wo = orc.sample_weight(orc.Model(n_joints=nj), 77, s_in, tr["Z"][3], tr["U"][2], 3, fp64=True)
    _close(sg, so)
    _close(wg, wo)
    g.close()


@pytest.mark.parametrize("nj,m,N,res", [(2, 64, 16, "rws"), (2, 64, 16, "vose"), (5, 256, 16, "rws")])
def test_trajectory_vs_fp64(P, orc, W, nj, m, N, res):
    # C1 (2-link arm, 16 x 64, ring t = 1), 10 steps: every particle and the
    # estimate of every step within 1e-5 of the float64 oracle, same argmax
    tr = W.make_trajectory(nj, 10, 0)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=m, n_filters=N, t=1, topo="ring",
                         resampler=res, seed=3)
    o = orc.Filter(orc.Config(m=m, n_filters=N, t=1, topo="ring", resampler=res, seed=3), orc.Model(n_joints=nj),
                   tr["mu0"], tr["sigma0"], fp64=True)
    for k in range(1, 11):
        g.step(tr["Z"][k], tr["U"][k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        xg, lg, ig = g.estimate()
        xo, lo, io = o.estimate()
        assert ig == io, (k, ig, io)
        _close(xg, xo)
        _close([lg], [lo])
        sg, wg, _ = g.get_particles()
        so, wo, _ = o.get()
        _close(sg, so)
        _close(wg, wo)
    g.close()
