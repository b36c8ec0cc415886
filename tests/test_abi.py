"""C-ABI boundary (include/pf.h) without a GPU: the library loads and exports
every declared entry point; configuration validation needs no device."""
import ctypes as C
import os
import re
import subprocess

import pytest

from conftest import ROOT

HEADER = os.path.join(ROOT, "include", "pf.h")


def _declared():
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"^\s*(?:pf_status|const char\*|int32_t)\s+(pf_\w+)\(", txt, re.M)))


@pytest.fixture(scope="module")
def B():
    from paper_conf_ipps_chitchianasks13_b200 import binding, build
    build.build()
    return binding


def test_header_declares_entry_points(B):
    assert _declared() == sorted(B.ENTRY_POINTS)


def test_library_exports_every_declared_symbol(B):
    lib = B.lib()
    out = subprocess.check_output(["nm", "-D", "--defined-only", B.LIB_PATH], text=True)
    exported = {line.split()[-1] for line in out.splitlines() if " T " in line}
    for name in _declared():
        assert name in exported, name
        assert hasattr(lib, name)


def test_library_is_sm100a_with_tma(B):
    out = subprocess.check_output(["cuobjdump", "--list-elf", B.LIB_PATH], text=True)
    assert "sm_100a" in out
    sass = subprocess.check_output(["cuobjdump", "-sass", B.LIB_PATH], text=True)
    assert "UBLKCP" in sass          # cp.async.bulk (TMA bulk copy) in the step kernel
    assert "REDUX" in sass           # warp-level max/min reductions


def _cfg(B, **kw):
    c = dict(m=64, n_filters=16, t=1, topo=B.PF_TOPO_RING, torus_rows=0, torus_cols=0,
             resampler=B.PF_RESAMPLE_RWS, seed=0, rank=0, world=1, flags=0)
    c.update(kw)
    return B.pf_config(**c)


def _model(B, nj=2):
    return B.pf_model_params(B.PF_MODEL_ARM_PLANAR, nj, 1.0, 0.1, 0.1, 0.1, 0.1, 0.1, 0.1)


def test_query_sizes(B):
    s = B.pf_query_sizes(_cfg(B), _model(B, 2))
    d, M = 6, 16 * 64
    assert s.state == 4 * (d + 1) * M          # blocked [n][d+1][m]: states + log-weights
    assert s.mailbox == 4 * 2 * 16 * 1 * (d + 2)
    # sharded ring: 2 halo rows
    s2 = B.pf_query_sizes(_cfg(B, world=4, rank=1, t=2), _model(B, 5))
    assert s2.state == 4 * 10 * 4 * 64
    assert s2.mailbox == 4 * 2 * (4 + 2) * 2 * 11
    # All-to-All, t = 2: one pool row, then the per-group best-t candidates (16384 groups x t x 16 B)
    s3 = B.pf_query_sizes(_cfg(B, topo=B.PF_TOPO_ALL2ALL, t=2), _model(B, 2))
    assert s3.mailbox == 4 * 2 * (16 + 1) * 2 * (d + 2) + 16 * 16384 * 2


@pytest.mark.parametrize("kw,code", [
    (dict(m=48), -1), (dict(m=16), -1), (dict(m=2048), -1),
    (dict(t=32, m=64), -1),                          # deg*t >= m (R19)
    (dict(topo=2, n_filters=12, torus_rows=3, torus_cols=5), -1),
    (dict(world=3), -1),                              # N % world != 0
    (dict(rank=2, world=2), -1),
    (dict(resampler=7), -1),
])
def test_invalid_configs(B, kw, code):
    out = B.pf_sizes()
    assert B.lib().pf_query_sizes(C.byref(_cfg(B, **kw)), C.byref(_model(B)), C.byref(out)) == code


def test_unsupported_model(B):
    out = B.pf_sizes()
    # any n_joints <= 28 runs (compiled n_j in {2, 5, 28}, the generic arm for the rest); 29+ is not compiled
    assert B.lib().pf_query_sizes(C.byref(_cfg(B)), C.byref(_model(B, 7)), C.byref(out)) == B.PF_OK
    assert out.state == 4 * (7 + 4 + 1) * 16 * 64
    assert B.lib().pf_query_sizes(C.byref(_cfg(B)), C.byref(_model(B, 29)), C.byref(out)) == B.PF_EUNSUPPORTED
    # the centralized filter too (the generic arm for n_j = 7)
    assert B.lib().pf_query_sizes(C.byref(_cfg(B, m=8192, n_filters=1, t=0, topo=0)), C.byref(_model(B, 7)),
                                  C.byref(out)) == B.PF_OK
    assert (5, 256) in B.pf_supported() and (28, 256) in B.pf_supported()
    assert B.pf_strerror(B.PF_EINVAL).startswith("invalid")


def test_model_selection(B):
    # the model id selects the compiled model instance (pf.h pf_model_id)
    lg = B.pf_model_params(B.PF_MODEL_LINEAR_GAUSS_1D, 0, 0.0, 0.1, 0.1, 0.0, 0.0, 0.0, 0.2)
    s = B.pf_query_sizes(_cfg(B, m=256, n_filters=8), lg)
    assert s.state == 4 * (1 + 1) * 256 * 8                 # d = 1: one state row + the log-weight row
    assert s.mailbox == 4 * 2 * 8 * 1 * (1 + 2)
    out = B.pf_sizes()
    # centralized linear-Gaussian filter (m = 10^5-class, a multiple of 4096)
    assert B.lib().pf_query_sizes(C.byref(_cfg(B, m=102400, n_filters=1, t=0, topo=0)), C.byref(lg),
                                  C.byref(out)) == B.PF_OK
    bad = B.pf_model_params(7, 5, 1.0, 0.1, 0.1, 0.1, 0.1, 0.1, 0.1)
    assert B.lib().pf_query_sizes(C.byref(_cfg(B)), C.byref(bad), C.byref(out)) == B.PF_EINVAL
    lg_bad = B.pf_model_params(B.PF_MODEL_LINEAR_GAUSS_1D, 0, 0.0, 0.1, 0.1, 0.0, 0.0, 0.0, 0.0)   # sigma_meas = 0
    assert B.lib().pf_query_sizes(C.byref(_cfg(B)), C.byref(lg_bad), C.byref(out)) == B.PF_EINVAL
