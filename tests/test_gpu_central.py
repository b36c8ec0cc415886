"""Centralized filter on the GPU (§VI "a
sequential, centralized particle filter", Fig. 5/9 PAPER.md:26–30): one filter
of M > 1024 particles resampled globally (RWS over all M, R9), no exchange.
Parity with the oracle's n_filters = 1 filter, element by element; the fp32
contract makes the trajectories bit-identical."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def P():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_chitchianasks13_b200 import build, filter as F
    build.build()
    return F


def _pair(P, orc, W, nj, M, seed, T=12, traj_seed=0, res="rws"):
    tr = W.make_trajectory(nj, T, traj_seed)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=M, n_filters=1, t=0, topo="none",
                         resampler=res, seed=seed)
    o = orc.Filter(orc.Config(m=M, n_filters=1, t=0, topo="none", resampler=res, seed=seed),
                   orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"])
    return tr, g, o


@pytest.mark.parametrize("nj,M,res", [(2, 4096, "rws"), (5, 8192, "rws"), (28, 4096, "rws"), (5, 12288, "rws"),
                                      (5, 8192, "vose"), (2, 12288, "vose"), (28, 4096, "vose")])
def test_central_trajectory_bit_exact(P, orc, W, nj, M, res):
    # several scan tiles (4096) and, for 12288, a non-power-of-two tile count
    tr, g, o = _pair(P, orc, W, nj, M, seed=nj * 7 + M, res=res)
    for k in range(1, 9):
        g.step(tr["Z"][k], tr["U"][k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        xg, lg, ig = g.estimate()
        xo, lo, io = o.estimate()
        assert ig == io, f"estimate index differs at step {k}"
        np.testing.assert_array_equal(xg, xo)
        assert lg == lo
        if k in (1, 2, 8):
            sg, wg, kg = g.get_particles()
            so, wo, ko = o.get()
            assert kg == ko == k
            np.testing.assert_array_equal(sg, so)
            np.testing.assert_array_equal(wg, wo)
    g.close()


def test_central_sample_weight_hook(P, orc, W):
    # a1-a3 alone (no resampling) through the debug hook vs the oracle
    nj, M = 5, 8192
    tr = W.make_trajectory(nj, 5, 1)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=M, n_filters=1, t=0, topo="none",
                         seed=99)
    s0 = W.random_particles(tr, M, 3)
    sg, wg = g.debug_sample_weight(s0, tr["Z"][3], tr["U"][2], 3)
    so, wo = orc.sample_weight(orc.Model(n_joints=nj), 99, s0, tr["Z"][3], tr["U"][2], 3)
    np.testing.assert_array_equal(sg, so)
    np.testing.assert_array_equal(wg, wo)
    g.close()


def test_central_resume_and_batch(P, orc, W):
    # checkpoint restore (publish of a loaded set) then batched device steps
    import torch
    nj, M, seed = 5, 8192, 5
    tr, g, o = _pair(P, orc, W, nj, M, seed, T=20)
    s0 = W.random_particles(tr, M, 11)
    w0 = W.random_logw(1, M, 11).ravel()
    g.set_particles(s0, w0, 6)
    o.set(s0, w0, 6)
    xg, lg, ig = g.estimate()
    assert ig == int(np.argmax(w0)) and lg == w0.max()
    zs = torch.tensor(tr["Z"][7:12], device="cuda")
    us = torch.tensor(tr["U"][6:11], device="cuda")
    est = torch.zeros(5, 4 + nj + 4, device="cuda")
    g.step_batch(zs, us, est)
    for k in range(7, 12):
        o.step(tr["Z"][k], tr["U"][k - 1])
        xo, lo, io = o.estimate()
        np.testing.assert_array_equal(est[k - 7, 4:].cpu().numpy(), xo)
    np.testing.assert_array_equal(g.get_particles()[0], o.get()[0])
    np.testing.assert_array_equal(g.particles[:, :nj + 4].T.cpu().numpy(), o.get()[0])   # AoS records
    np.testing.assert_array_equal(g.central_logw.cpu().numpy(), o.get()[1])
    g.close()


@pytest.mark.parametrize("nj,M,res", [(5, 1 << 20, "rws"), (5, 1 << 22, "rws"), (28, 1 << 20, "rws"),
                                      (5, 1 << 20, "vose")])
def test_central_full_size_sampled(P, orc, W, nj, M, res):
    # full size (the paper's centralized curves reach 2^20 particles, Fig. 5):
    # one step from a generator-made weighted set; the oracle recomputes a
    # sample of slots one by one (normalise over all M, RWS, sample, weight)
    tr = W.make_trajectory(nj, 10, 2)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=M, n_filters=1, t=0, topo="none",
                         seed=4242, resampler=res)
    s0 = W.random_particles(tr, M, 5)
    w0 = W.random_logw(1, M, 5).ravel()
    g.set_particles(s0, w0, 4)
    g.step(tr["Z"][5], tr["U"][4])
    sg, wg, k = g.get_particles()
    assert k == 5
    rng = np.random.default_rng(M + nj)
    slots = np.unique(np.concatenate([[0, 1, 4095, 4096, M // 2, M - 1], rng.integers(0, M, 58)]))
    cfg = orc.Config(m=M, n_filters=1, t=0, topo="none", resampler=res, seed=4242)
    so, wo = orc.central_slots(cfg, orc.Model(n_joints=nj), s0, w0, 5, tr["Z"][5], tr["U"][4], slots)
    np.testing.assert_array_equal(sg[:, slots], so)
    np.testing.assert_array_equal(wg[slots], wo)
    x, lw, idx = g.estimate()
    assert lw == wg.max() and idx == int(np.flatnonzero(wg == wg.max())[0])
    np.testing.assert_array_equal(x, sg[:, idx])
    g.close()


def test_central_errors(P, W):
    from paper_conf_ipps_chitchianasks13_b200 import binding as B
    tr = W.make_trajectory(5, 4, 0)
    mk = lambda **kw: P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=5), n_filters=1, t=0,
                                       topo="none", **kw)
    with pytest.raises(B.PFError):
        mk(m=5000)                       # not a multiple of the 4096-particle scan tile
    with pytest.raises(B.PFError):
        mk(m=1 << 21, resampler="vose")  # centralized Vose: u64 alias sums need m <= 2^20
    g = mk(m=4096)
    assert B.lib().pf_set_trace(g.h, 1) == B.PF_ESTATE
    g.close()


@pytest.mark.parametrize("M", [8192, 12288])
@pytest.mark.parametrize("kind", ["mixed", "uniform", "onehot", "sparse"])
def test_central_resample_tables_bit_exact(P, orc, W, M, kind):
    # the device-wide RWS search and Vose table (closed form over all M slots,
    # R10) against the oracle's sequential sum / sequential sweep, slot by slot
    from paper_conf_ipps_chitchianasks13_b200 import binding as B
    rng = np.random.default_rng(M + len(kind))
    if kind == "mixed":
        q = rng.integers(0, 1 << 22, M).astype(np.uint32)
        q[rng.random(M) < 0.3] = 0
    elif kind == "uniform":
        q = np.full(M, 1 << 22, np.uint32)
    elif kind == "onehot":
        q = np.zeros(M, np.uint32)
        q[M // 3] = 1 << 22
    else:
        q = np.zeros(M, np.uint32)
        q[rng.integers(0, M, 17)] = rng.integers(1, 1 << 22, 17).astype(np.uint32)
    ua = rng.integers(0, 2**32, M, dtype=np.uint64).astype(np.uint32)
    ub = rng.integers(0, 2**32, M, dtype=np.uint64).astype(np.uint32)
    ua[:3] = [0, 0xFFFFFFFF, 0x80000000]
    ub[:3] = [0, 0xFFFFFFFF, 0x7FFFFFFF]
    tr = W.make_trajectory(5, 3, 0)
    for res in ("rws", "vose"):
        g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=5), m=M, n_filters=1, t=0, topo="none",
                             resampler=res)
        anc = np.zeros(M, np.int32)
        prob = np.zeros(M, np.uint64)
        alias = np.zeros(M, np.int32)
        B.pf_debug_resample(g.h, q, ua, ub, anc, prob if res == "vose" else None, alias if res == "vose" else None)
        g.close()
        if res == "vose":
            pr, al = orc.vose_build(q)
            np.testing.assert_array_equal(prob, pr)
            np.testing.assert_array_equal(alias, al)
            Q = int(q.astype(np.uint64).sum())
            mass = prob.copy()   # alias mass of slot j = prob_j + sum over columns aliasing j of (Q - prob)
            np.add.at(mass, alias, np.uint64(Q) - prob)
            np.testing.assert_array_equal(mass, np.uint64(M) * q.astype(np.uint64))
            ref = np.array([orc.vose_draw(pr, al, Q, int(a), int(b)) for a, b in zip(ua, ub)], np.int32)
        else:
            ref = np.array([orc.rws_draw(q, int(a)) for a in ua], np.int32)
        np.testing.assert_array_equal(anc, ref)
        assert np.all(q[anc] > 0)   # never a zero-weight slot


@pytest.mark.parametrize("nj,res", [(3, "rws"), (9, "vose")])
def test_central_generic_arm(P, orc, W, nj, res):
    # the centralized filter with the generic arm (n_j not compiled): a few
    # steps bit for bit against the oracle, estimate every step
    M = 8192
    tr = W.make_trajectory(nj, 6, 4)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=M, n_filters=1, t=0, topo="none",
                         resampler=res, seed=9)
    o = orc.Filter(orc.Config(m=M, n_filters=1, t=0, topo="none", resampler=res, seed=9), orc.Model(n_joints=nj),
                   tr["mu0"], tr["sigma0"])
    for k in range(1, 6):
        g.step(tr["Z"][k], tr["U"][k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        assert g.estimate()[2] == o.estimate()[2]
    sg, wg, _ = g.get_particles()
    so, wo, _ = o.get()
    np.testing.assert_array_equal(sg, so)
    np.testing.assert_array_equal(wg, wo)
    g.close()
