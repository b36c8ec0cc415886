"""CUDA path (libpf_b200.so through the C ABI) vs the CPU oracle, element by
element on the same seeded inputs.  Bar (north_star, R18): indices and
exchange permutations bit-exact; states / log-weights / estimates within
1e-5 relative — and, because both sides follow the fp32 contract F1–F11,
the whole trajectory is expected to be bit-identical (asserted separately)."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

TOL = 1e-5


def _close(a, b):
    a, b = np.asarray(a, np.float64), np.asarray(b, np.float64)
    assert np.all(np.abs(a - b) <= TOL * np.maximum(1.0, np.abs(b))), float(np.max(np.abs(a - b)))


@pytest.fixture(scope="module")
def P():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_chitchianasks13_b200 import build, filter as F
    build.build()
    return F


def _pair(P, orc, W, nj, m, N, t=1, topo="ring", res="rws", seed=1, T=100, traj_seed=0):
    tr = W.make_trajectory(nj, T, traj_seed)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=m, n_filters=N, t=t, topo=topo,
                         resampler=res, seed=seed)
    o = orc.Filter(orc.Config(m=m, n_filters=N, t=t, topo=topo, resampler=res, seed=seed),
                   orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"])
    return tr, g, o


def test_init_prior_bit_exact(P, orc, W):
    tr, g, o = _pair(P, orc, W, 5, 64, 8, seed=(5 << 32) | 3)
    sg, _, kg = g.get_particles()
    so, _, ko = o.get()
    assert kg == ko == 0
    np.testing.assert_array_equal(sg, so)


@pytest.mark.parametrize("nj,m,N", [(2, 64, 16), (5, 256, 4), (28, 32, 8), (5, 1024, 2), (28, 256, 2)])
def test_sample_weight(P, orc, W, nj, m, N):
    tr = W.make_trajectory(nj, 10, 1)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=m, n_filters=N, seed=77)
    s_in = W.random_particles(tr, m * N, nj)
    for k in (1, 7):
        sg, wg = g.debug_sample_weight(s_in, tr["Z"][k], tr["U"][k - 1], k)
        so, wo = orc.sample_weight(orc.Model(n_joints=nj), 77, s_in, tr["Z"][k], tr["U"][k - 1], k)
        _close(sg, so)
        _close(wg, wo)
        np.testing.assert_array_equal(sg, so)     # fp32 contract: bit-identical
        np.testing.assert_array_equal(wg, wo)


@pytest.mark.parametrize("res", ["rws", "vose"])
@pytest.mark.parametrize("m", [32, 64, 256, 1024])
@pytest.mark.parametrize("kind", ["mixed", "uniform", "onehot"])
def test_resample_bit_exact(P, orc, W, res, m, kind):
    N = 24
    tr = W.make_trajectory(2, 4, 0)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=2), m=m, n_filters=N, resampler=res)
    q = W.random_q(N, m, m + len(kind), kind)
    if kind == "mixed":
        q[::3, ::2] = 0          # zero-weight slots (never drawn)
    rng = np.random.default_rng(m)
    ua = rng.integers(0, 2**32, (N, m), dtype=np.uint64).astype(np.uint32)
    ub = rng.integers(0, 2**32, (N, m), dtype=np.uint64).astype(np.uint32)
    ua[0, :4] = [0, 0xFFFFFFFF, 0x80000000, 1]
    anc, prob, alias = g.debug_resample(q, ua, ub)
    np.testing.assert_array_equal(anc, orc.resample_q(q, res, ua, ub))
    if res == "vose":
        for n in range(N):
            p_o, a_o = orc.vose_build(q[n])
            np.testing.assert_array_equal(prob[n], p_o)
            np.testing.assert_array_equal(alias[n], a_o)


@pytest.mark.parametrize("topo,N,m,t", [("ring", 16, 64, 1), ("ring", 8, 32, 3), ("torus", 16, 64, 2),
                                         ("torus", 8, 128, 1), ("ring", 2, 32, 1), ("torus", 4, 32, 1),
                                         ("ring", 1, 32, 2), ("all2all", 8, 32, 3), ("all2all", 64, 64, 1)])
def test_exchange_bit_exact(P, orc, W, topo, N, m, t):
    tr = W.make_trajectory(2, 4, 0)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=2), m=m, n_filters=N, t=t, topo=topo)
    for s in range(3):
        w = W.random_logw(N, m, 100 + s, ties=(s != 1))
        src = g.debug_exchange(w.ravel())
        np.testing.assert_array_equal(src.reshape(N, m),
                                      orc.exchange(orc.Config(m=m, n_filters=N, t=t, topo=topo), w))


def _run_compare(P, orc, W, nj, m, N, T, **kw):
    tr, g, o = _pair(P, orc, W, nj, m, N, T=T, **kw)
    g.set_trace(True)
    for k in range(1, T + 1):
        g.step(tr["Z"][k], tr["U"][k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        xg, lg, ig = g.estimate()
        xo, lo, io = o.estimate()
        assert ig == io, f"estimate index differs at step {k}"
        _close(xg, xo)
        _close(lg, lo)
        if k in (1, 2, T):
            src_g, anc_g = g.trace()
            src_o, anc_o = o.trace()
            np.testing.assert_array_equal(src_g, src_o)
            np.testing.assert_array_equal(anc_g, anc_o)
            sg, wg, kg = g.get_particles()
            so, wo, ko = o.get()
            assert kg == ko == k
            _close(sg, so)
            _close(wg, wo)
            np.testing.assert_array_equal(sg, so)
            np.testing.assert_array_equal(wg, wo)
    return g, o


def test_full_filter_c1(P, orc, W):
    # BASELINE config 1: 2-link arm, 16 sub-filters x 64, RWS, ring t = 1, 100 steps
    _run_compare(P, orc, W, 2, 64, 16, 100)


@pytest.mark.parametrize("nj,m,N,t,topo,res", [
    (2, 64, 16, 1, "torus", "vose"),
    (5, 256, 16, 2, "ring", "vose"),
    (5, 128, 64, 1, "torus", "rws"),
    (5, 32, 32, 0, "none", "rws"),
    (28, 64, 8, 1, "ring", "vose"),
    (28, 256, 8, 1, "ring", "rws"),     # high-DOF arm, packed pairs + chunked joint loop
    (28, 256, 16, 1, "torus", "vose"),
    (28, 1024, 2, 3, "ring", "rws"),
    (5, 1024, 4, 4, "torus", "rws"),
    (5, 64, 16, 2, "all2all", "vose"),
    (2, 256, 64, 1, "all2all", "rws"),
    # more sub-filters than resident groups: groups merge several sub-filters'
    # best t into their running pool candidates (All-to-All, t >= 2)
    (5, 32, 8192, 2, "all2all", "rws"),
    (5, 32, 8192, 4, "all2all", "vose"),
    # deg t = 2 and 4 with four slots per thread (the specialised worst-slot selections)
    (5, 256, 2048, 2, "ring", "rws"),
    (5, 256, 1024, 1, "torus", "vose"),
    (5, 256, 1024, 1, "ring", "rws"),
])
def test_full_filter_variants(P, orc, W, nj, m, N, t, topo, res):
    _run_compare(P, orc, W, nj, m, N, 12, t=t, topo=topo, res=res, seed=nj * 1000 + m)


def test_set_particles_resume(P, orc, W):
    # checkpoint / resume from a generator-made weighted set, then 5 steps
    nj, m, N = 5, 64, 16
    tr, g, o = _pair(P, orc, W, nj, m, N, T=20, res="vose", topo="torus")
    s0 = W.random_particles(tr, m * N, 9)
    w0 = W.random_logw(N, m, 9).ravel()
    g.set_particles(s0, w0, 7)
    o.set(s0, w0, 7)
    for k in range(8, 13):
        g.step(tr["Z"][k], tr["U"][k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        assert g.estimate()[2] == o.estimate()[2]
    np.testing.assert_array_equal(g.get_particles()[0], o.get()[0])


@pytest.mark.parametrize("res", ["rws", "vose"])
def test_full_size_c2(P, orc, W, res):
    # BASELINE config 2 at full size: medium arm, 4096 x 256 = 2^20, ring t=1,
    # in the launch configuration bench.py times; 3 steps vs the oracle
    tr, g, o = _pair(P, orc, W, 5, 256, 4096, T=10, res=res, seed=2013)
    for k in range(1, 4):
        g.step(tr["Z"][k], tr["U"][k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        xg, lg, ig = g.estimate()
        xo, lo, io = o.estimate()
        assert ig == io
        np.testing.assert_array_equal(xg, xo)
    sg, wg, _ = g.get_particles()
    so, wo, _ = o.get()
    np.testing.assert_array_equal(sg, so)
    np.testing.assert_array_equal(wg, wo)


def test_step_batch_matches_streaming(P, W):
    import torch
    nj, m, N, T = 5, 128, 32, 20
    tr = W.make_trajectory(nj, T, 3)
    a = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=m, n_filters=N, seed=9)
    b = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=m, n_filters=N, seed=9)
    zs = torch.tensor(tr["Z"][1:T + 1], device="cuda")
    us = torch.tensor(tr["U"][0:T], device="cuda")
    est = torch.zeros(T, 4 + nj + 4, device="cuda")
    b.step_batch(zs, us, est)
    torch.cuda.synchronize()
    for k in range(1, T + 1):
        a.step(tr["Z"][k], tr["U"][k - 1])
        x, lw, idx = a.estimate()
        np.testing.assert_array_equal(est[k - 1, 4:].cpu().numpy(), x)
        assert est[k - 1, 2].item() == lw


@pytest.mark.parametrize("topo,N,world", [("ring", 16, 2), ("torus", 16, 2), ("ring", 12, 4), ("torus", 64, 4),
                                          ("all2all", 16, 2), ("all2all", 24, 4)])
def test_sharded_loopback_bit_identical(P, orc, W, topo, N, world):
    # world shards of one filter in one process on one GPU, halos exchanged
    # by the same plan the NCCL path uses: identical to the unsharded filter
    # and to the oracle (global Philox counters, exact max reduce)
    import torch
    from paper_conf_ipps_chitchianasks13_b200 import distributed as Dd
    nj, m, T = 5, 64, 6
    tr = W.make_trajectory(nj, T, 4)
    t = 2 if topo == "all2all" else 1
    kw = dict(m=m, n_filters=N, t=t, topo=topo, resampler="vose", seed=99)
    shards = [P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), rank=r, world=world, **kw)
              for r in range(world)]
    o = orc.Filter(orc.Config(m=m, n_filters=N, t=t, topo=topo, resampler="vose", seed=99),
                   orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"])
    plan = Dd.halo_plan(topo, N, world)
    nl = int(shards[0].shard.n_local)
    recs = torch.zeros(world, 4 + nj + 4, device="cuda")
    for k in range(1, T + 1):
        if k > 1:
            Dd.loopback_exchange([s.mailbox[(k - 1) & 1] for s in shards], plan)
        for s in shards:
            s.step(tr["Z"][k], tr["U"][k - 1])
        if topo == "all2all":   # the all-gather of every shard's best-t row, then the exact reduce
            for r in range(world):
                for s in shards:
                    s.mailbox[k & 1][nl + r].copy_(shards[r].mailbox[k & 1][nl + r])
            for s in shards:
                s.reduce_pool()
        for r, s in enumerate(shards):
            recs[r] = s.record
        shards[0].reduce_records(recs)
        o.step(tr["Z"][k], tr["U"][k - 1])
        xg, lg, ig = shards[0].estimate()
        xo, lo, io = o.estimate()
        assert ig == io and np.array_equal(xg, xo), k
    so, wo, _ = o.get()
    sg = np.concatenate([s.get_particles()[0] for s in shards], axis=1)
    np.testing.assert_array_equal(sg, so)


@pytest.mark.parametrize("name,nj,m,N,t,topo,res", [
    ("C4 high-DOF arm 16M, Vose", 28, 256, 65536, 1, "ring", "vose"),
    ("C5 per-GPU shard 16M, RWS", 5, 256, 65536, 1, "ring", "rws"),
    ("C3 m=32 at 4M, torus t=4", 5, 32, 131072, 4, "torus", "rws"),
    ("C3 m=1024 at 4M, torus t=2", 5, 1024, 4096, 2, "torus", "vose"),
])
def test_full_size_sampled(P, orc, W, name, nj, m, N, t, topo, res):
    # BASELINE configs at full size in the bench's launch configuration: one
    # step from a generator-made weighted set; the oracle recomputes a sample
    # of sub-filters one by one (exchange, resample, sample, weight)
    tr = W.make_trajectory(nj, 10, 2)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=m, n_filters=N, t=t, topo=topo,
                         resampler=res, seed=31337)
    s0 = W.random_particles(tr, m * N, 5)
    w0 = W.random_logw(N, m, 5).ravel()
    g.set_particles(s0, w0, 4)
    g.step(tr["Z"][5], tr["U"][4])
    sg, wg, k = g.get_particles()
    assert k == 5
    rng = np.random.default_rng(N + m)
    subs = np.unique(np.concatenate([[0, N - 1, N // 2], rng.integers(0, N, 21)]))
    cfg = orc.Config(m=m, n_filters=N, t=t, topo=topo, resampler=res, seed=31337)
    so, wo = orc.step_subset(cfg, orc.Model(n_joints=nj), s0, w0, 5, tr["Z"][5], tr["U"][4], subs)
    for i, n in enumerate(subs):
        np.testing.assert_array_equal(sg[:, n * m:(n + 1) * m], so[:, i * m:(i + 1) * m], err_msg=f"{name} sf {n}")
        np.testing.assert_array_equal(wg[n * m:(n + 1) * m], wo[i * m:(i + 1) * m], err_msg=f"{name} sf {n}")
    # the estimate is the global argmax of the new log-weights (R6)
    x, lw, idx = g.estimate()
    assert lw == wg.max() and idx == int(np.flatnonzero(wg == wg.max())[0])
    np.testing.assert_array_equal(x, sg[:, idx])
    g.close()


def test_rmse_100_seeds_c1(P, orc, W):
    # north_star: end-to-end tracking RMSE within 5 % of the oracle's over 100
    # seeds (config C1: 2-link arm, 16 x 64, RWS, ring t = 1, 100 steps).
    # With the fp32 contract the estimates are bit-identical, so the RMSEs agree exactly.
    nj, T = 2, 100
    rg, ro = [], []
    for seed in range(100):
        tr = W.make_trajectory(nj, T, seed)
        g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=64, n_filters=16, t=1,
                             topo="ring", resampler="rws", seed=seed)
        o = orc.Filter(orc.Config(m=64, n_filters=16, t=1, topo="ring", resampler="rws", seed=seed),
                       orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"])
        eg, eo = [], []
        for k in range(1, T + 1):
            g.step(tr["Z"][k], tr["U"][k - 1])
            o.step(tr["Z"][k], tr["U"][k - 1])
            truth = tr["X"][k][nj:nj + 2]
            eg.append(np.hypot(*(g.estimate()[0][nj:nj + 2] - truth)))
            eo.append(np.hypot(*(o.estimate()[0][nj:nj + 2] - truth)))
        g.close()
        rg.append(np.sqrt(np.mean(np.square(eg))))
        ro.append(np.sqrt(np.mean(np.square(eo))))
    mg, mo = float(np.mean(rg)), float(np.mean(ro))
    assert abs(mg - mo) <= 0.05 * mo, (mg, mo)
    np.testing.assert_array_equal(rg, ro)
    assert mo < 0.25   # tracks the lemniscate (Fig.8)


@pytest.mark.parametrize("nj,m,N,t,topo,res,rows,cols", [
    (5, 64, 16, 1, "torus", "rws", 2, 8),      # non-square torus
    (5, 64, 16, 2, "torus", "vose", 8, 2),
    (2, 32, 1, 1, "ring", "rws", 0, 0),       # one sub-filter: both ring neighbours are itself
    (2, 32, 1, 3, "all2all", "vose", 0, 0),   # one sub-filter receiving its own best back
    (5, 32, 4, 7, "torus", "rws", 0, 0),      # deg*t = 28 = m - 4 (R19 bound)
    (5, 1024, 4, 8, "torus", "vose", 0, 0),   # deg*t = 32 = KMAX
    (28, 32, 8, 0, "none", "rws", 0, 0),      # independent sub-filters
])
def test_edge_configs(P, orc, W, nj, m, N, t, topo, res, rows, cols):
    tr = W.make_trajectory(nj, 8, 6)
    kw = dict(m=m, n_filters=N, t=t, topo=topo, resampler=res, seed=(1 << 40) + 17, torus_rows=rows,
              torus_cols=cols)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), **kw)
    o = orc.Filter(orc.Config(**kw), orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"])
    for k in range(1, 7):
        g.step(tr["Z"][k], tr["U"][k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        assert g.estimate()[2] == o.estimate()[2]
    np.testing.assert_array_equal(g.get_particles()[0], o.get()[0])


def test_error_behaviour(P, W):
    from paper_conf_ipps_chitchianasks13_b200 import binding as B
    tr = W.make_trajectory(2, 4, 0)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=2), m=64, n_filters=4)
    x = np.zeros(6, np.float32)
    assert B.lib().pf_estimate(g.h, x.ctypes.data, None, None) == B.PF_ESTATE    # before the first step
    assert B.lib().pf_reduce_pool(g.h) == B.PF_ESTATE                          # not All-to-All
    assert B.lib().pf_step(g.h, None, None) == B.PF_EINVAL
    assert B.lib().pf_destroy(None) == B.PF_OK
    g.step(tr["Z"][1], tr["U"][0])
    assert B.lib().pf_estimate(g.h, x.ctypes.data, None, None) == B.PF_OK
    assert B.pf_last_error(g.h) == B.PF_OK
    with pytest.raises(B.PFError):
        P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=29), m=64, n_filters=4)   # d > 32: not compiled


@pytest.mark.parametrize("central", [False, True])
def test_device_inputs_streamed_and_batched(P, orc, W, central):
    """Device-resident inputs (the bench's timed path): per-step pf_step +
    pf_estimate (record copied from the device) and pf_step_batch (records
    written on the device) both equal the oracle's estimates, step by step."""
    import torch
    nj, T = 5, 8
    m, N = (8192, 1) if central else (64, 16)
    topo, t = ("none", 0) if central else ("ring", 1)
    tr = W.make_trajectory(nj, T, 3)
    kw = dict(m=m, n_filters=N, t=t, topo=topo, resampler="rws", seed=5)
    zs = torch.tensor(tr["Z"][1:T + 1], device="cuda")
    us = torch.tensor(tr["U"][:T], device="cuda")
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), device_inputs=True, **kw)
    gb = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), device_inputs=True, **kw)
    o = orc.Filter(orc.Config(**kw), orc.Model(n_joints=nj), tr["mu0"], tr["sigma0"])
    d = nj + 4
    est = torch.zeros(T, 4 + d, device="cuda")
    gb.step_batch(zs, us, est)
    est = est.cpu().numpy()
    for k in range(1, T + 1):
        g.step(zs[k - 1], us[k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        xg, lg, ig = g.estimate()
        xo, lo, io = o.estimate()
        assert ig == io, (k, ig, io)
        np.testing.assert_array_equal(xg, xo)
        np.testing.assert_array_equal(est[k - 1, 4:], xo)
        assert est[k - 1, 2] == np.float32(lo)
    xb, _, ib = gb.estimate()
    assert ib == io
    np.testing.assert_array_equal(xb, xo)
    g.close()
    gb.close()


@pytest.mark.parametrize("nj,m,N,t,topo,sig", [
    (5, 32, 1, 1, "ring", 0.1),      # one sub-filter: its ring neighbours are itself (both sides)
    (5, 32, 2, 3, "ring", 0.1),      # two sub-filters: both neighbours are the other one
    (2, 64, 4, 1, "torus", 0.1),     # 2 x 2 torus: duplicate neighbours deliver the same particle twice
    (2, 64, 8, 1, "ring", 0.0),      # zero process noise: deterministic motion, ties everywhere
])
def test_degenerate_filters(P, orc, W, nj, m, N, t, topo, sig):
    tr = W.make_trajectory(nj, 8, 1)
    gm = P.ArmModel(n_joints=nj, sigma_theta=sig, sigma_pos=sig, sigma_vel=sig)
    om = orc.Model(n_joints=nj, sigma_theta=sig, sigma_pos=sig, sigma_vel=sig)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], gm, m=m, n_filters=N, t=t, topo=topo, seed=6)
    o = orc.Filter(orc.Config(m=m, n_filters=N, t=t, topo=topo, seed=6), om, tr["mu0"], tr["sigma0"])
    for k in range(1, 9):
        g.step(tr["Z"][k], tr["U"][k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        assert g.estimate()[2] == o.estimate()[2]
    sg, wg, _ = g.get_particles()
    so, wo, _ = o.get()
    np.testing.assert_array_equal(sg, so)
    np.testing.assert_array_equal(wg, wo)
    g.close()
