"""Every compiled step-kernel mapping (include/pf.h pf_query_mapping; the
PF_VARIANT tuning knob of pf_init) against the oracle: warps per group, groups
per CTA, TMA stages (double-buffered loads), sample-loop unroll, register cap
and the split first load (DESIGN.md §6 step 1) change how the work is laid
out, never the result — states, log-weights and every step's estimate stay
bit-identical to Algorithm 2 (§IV).  Sizes leave a ragged last
round of sub-filters, so groups run one to several sub-filters (split and
unsplit loads)."""
import os

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


def _run(P, orc, W, nj, m, N, res, topo, t, variant, steps=3):
    from paper_conf_ipps_chitchianasks13_b200 import binding as B
    tr = W.make_trajectory(nj, steps + 2, 3)
    old = os.environ.get("PF_VARIANT")
    os.environ["PF_VARIANT"] = str(variant)
    try:
        g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=nj), m=m, n_filters=N, t=t, topo=topo,
                             resampler=res, seed=404)
    finally:
        if old is None:
            del os.environ["PF_VARIANT"]
        else:
            os.environ["PF_VARIANT"] = old
    mp = B.pf_query_mapping(g.h)
    o = orc.Filter(orc.Config(m=m, n_filters=N, t=t, topo=topo, resampler=res, seed=404), orc.Model(n_joints=nj),
                   tr["mu0"], tr["sigma0"])
    for k in range(1, steps + 1):
        g.step(tr["Z"][k], tr["U"][k - 1])
        o.step(tr["Z"][k], tr["U"][k - 1])
        xg, lg, ig = g.estimate()
        xo, lo, io = o.estimate()
        assert ig == io, (variant, mp, k)
        np.testing.assert_array_equal(xg, xo)
    sg, wg, _ = g.get_particles()
    so, wo, _ = o.get()
    np.testing.assert_array_equal(sg, so)
    np.testing.assert_array_equal(wg, wo)
    g.close()
    return mp


@pytest.mark.parametrize("nj,m,N,res,topo,t", [
    (5, 256, 4000, "rws", "ring", 1),      # C2's m: 16 compiled RWS mappings
    (5, 256, 3072, "vose", "torus", 1),    # the Vose mappings; torus 32 x 96
    (28, 256, 600, "rws", "ring", 2),      # high-DOF arm
    (28, 256, 600, "vose", "ring", 1),
])
def test_every_mapping_bit_exact(P, orc, W, nj, m, N, res, topo, t):
    # (the variants are the compiled entries for this n_j and the generic-arm
    # buckets that hold it, pf_registry.h)
    mp0 = _run(P, orc, W, nj, m, N, res, topo, t, 0)
    assert mp0["n_variants"] >= 5
    for v in range(1, mp0["n_variants"]):
        mp = _run(P, orc, W, nj, m, N, res, topo, t, v)
        assert mp["n_variants"] == mp0["n_variants"]


def test_query_mapping_defaults(P, W):
    # the runtime's choices: C2 -> 2 warps x 4 groups, 3 CTAs/SM, split first load;
    # a 16M shard -> the large-shard mapping without the split; few sub-filters -> one particle per thread
    from paper_conf_ipps_chitchianasks13_b200 import binding as B
    tr = W.make_trajectory(5, 3, 0)
    def mapping(N, res="rws"):
        g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=5), m=256, n_filters=N, resampler=res)
        mp = B.pf_query_mapping(g.h)
        g.close()
        return mp
    c2 = mapping(4096)
    assert (c2["warps_per_group"], c2["groups_per_cta"], c2["min_ctas_per_sm"], c2["split_first_load"]) == (2, 4, 3, 1)
    c2v = mapping(4096, "vose")
    assert (c2v["warps_per_group"], c2v["groups_per_cta"], c2v["min_ctas_per_sm"]) == (2, 4, 3)
    big = mapping(65536)
    assert (big["warps_per_group"], big["groups_per_cta"], big["min_ctas_per_sm"], big["split_first_load"]) == (2, 4, 4, 0)
    bigv = mapping(65536, "vose")
    assert (bigv["groups_per_cta"], bigv["min_ctas_per_sm"], bigv["split_first_load"]) == (7, 2, 0)
    small = mapping(16)
    assert small["warps_per_group"] == 8


def test_query_mapping_errors(P, W):
    # include/pf.h: NULL -> PF_EINVAL; the centralized filter (fixed kernel shapes) -> PF_ESTATE
    import ctypes as C
    from paper_conf_ipps_chitchianasks13_b200 import binding as B
    tr = W.make_trajectory(5, 3, 0)
    g = P.ParticleFilter(tr["mu0"], tr["sigma0"], P.ArmModel(n_joints=5), m=8192, n_filters=1, t=0, topo="none")
    out = (C.c_int32 * 8)()
    assert B.lib().pf_query_mapping(g.h, out) == B.PF_ESTATE
    assert B.lib().pf_query_mapping(g.h, None) == B.PF_EINVAL
    assert B.lib().pf_query_mapping(None, out) == B.PF_EINVAL
    g.close()
