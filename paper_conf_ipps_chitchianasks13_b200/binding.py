"""Thin ctypes binding of libpf_b200.so (include/pf.h) — argument marshalling only.

Every function has the C name and argument order; pointers are passed as
integers (``tensor.data_ptr()`` for device memory, numpy ``ctypes.data`` for
host memory).  Loading fails loudly if the library is missing: there is no
CPU fallback.
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("PF_LIB") or os.path.join(HERE, "libpf_b200.so")   # PF_LIB: dev A/B builds

PF_OK, PF_EINVAL, PF_ENOMEM, PF_ECUDA, PF_ESTATE, PF_EUNSUPPORTED, PF_ETIMEOUT = 0, -1, -2, -3, -5, -6, -7
PF_TOPO_NONE, PF_TOPO_RING, PF_TOPO_TORUS2D, PF_TOPO_ALL2ALL = 0, 1, 2, 3
PF_RESAMPLE_RWS, PF_RESAMPLE_VOSE = 0, 1
PF_POLICY_ALWAYS, PF_POLICY_ESS, PF_POLICY_FREQ = 0, 1, 2
PF_MODEL_ARM_PLANAR, PF_MODEL_LINEAR_GAUSS_1D = 0, 1
PF_DEVICE_INPUTS = 1

ENTRY_POINTS = [
    "pf_query_sizes", "pf_init", "pf_step", "pf_step_batch", "pf_estimate", "pf_record_ptr",
    "pf_reduce_records", "pf_reduce_pool", "pf_get_shard", "pf_get_particles", "pf_set_particles", "pf_debug_sample_weight",
    "pf_debug_resample", "pf_debug_exchange", "pf_set_trace", "pf_get_trace", "pf_destroy", "pf_strerror",
    "pf_last_error", "pf_supported", "pf_debug_math", "pf_debug_check_sqrt", "pf_estimate_mean", "pf_mean_partial",
    "pf_reduce_means", "pf_peer_export", "pf_peer_connect", "pf_peer_connect_local", "pf_peer_connected",
    "pf_query_mapping",
]
PF_MATH = {"sin": 0, "cos": 1, "log": 2, "expq": 3, "sqrt": 4, "sincos2pi": 5, "normal_pair": 6, "philox": 7}


class pf_model_params(C.Structure):
    _fields_ = [("model", C.c_int32), ("n_joints", C.c_int32), ("arm_length", C.c_float), ("h_s", C.c_float),
                ("sigma_theta", C.c_float), ("sigma_pos", C.c_float), ("sigma_vel", C.c_float),
                ("sigma_cam", C.c_float), ("sigma_theta_meas", C.c_float)]


class pf_config(C.Structure):
    _fields_ = [("m", C.c_int32), ("n_filters", C.c_int64), ("t", C.c_int32), ("topo", C.c_int32),
                ("torus_rows", C.c_int32), ("torus_cols", C.c_int32), ("resampler", C.c_int32),
                ("seed", C.c_uint64), ("rank", C.c_int32), ("world", C.c_int32), ("flags", C.c_uint32),
                ("resample_policy", C.c_int32), ("resample_param", C.c_uint64)]


class pf_sizes(C.Structure):
    _fields_ = [("state", C.c_uint64), ("mailbox", C.c_uint64), ("scratch", C.c_uint64)]


class pf_buffers(C.Structure):
    _fields_ = [("state", C.c_void_p), ("mailbox", C.c_void_p), ("scratch", C.c_void_p)]


class pf_shard(C.Structure):
    _fields_ = [("g0", C.c_int64), ("n_local", C.c_int64), ("n_ext", C.c_int64), ("torus_rows", C.c_int64),
                ("torus_cols", C.c_int64), ("entry_floats", C.c_int32), ("t", C.c_int32), ("d", C.c_int32),
                ("record_floats", C.c_int32)]


class PFError(RuntimeError):
    pass


_lib = None


def lib() -> C.CDLL:
    """Load libpf_b200.so (built by __graft_entry__.build / build.py)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise PFError(f"{LIB_PATH} missing: run `python -m paper_conf_ipps_chitchianasks13_b200.build` "
                          "(the CUDA path has no fallback)")
        L = C.CDLL(LIB_PATH)
        P, I32, I64, ST = C.c_void_p, C.c_int32, C.c_int64, C.c_int
        sig = {
            "pf_query_sizes": [P, P, P],
            "pf_init": [P, P, P, P, P, P, P],
            "pf_step": [P, P, P],
            "pf_step_batch": [P, I32, P, P, P],
            "pf_estimate": [P, P, P, P],
            "pf_record_ptr": [P, P, P],
            "pf_estimate_mean": [P, P],
            "pf_mean_partial": [P, P, P],
            "pf_reduce_means": [P, P, I32, P],
            "pf_reduce_records": [P, P, I32],
            "pf_reduce_pool": [P],
            "pf_get_shard": [P, P],
            "pf_get_particles": [P, P, P, P],
            "pf_set_particles": [P, P, P, I64],
            "pf_debug_sample_weight": [P, P, P, P, I64, P, P],
            "pf_debug_resample": [P, P, P, P, P, P, P],
            "pf_debug_exchange": [P, P, P],
            "pf_set_trace": [P, I32],
            "pf_get_trace": [P, P, P],
            "pf_destroy": [P],
            "pf_last_error": [P],
            "pf_query_mapping": [P, P],
        }
        for name, args in sig.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = ST
        L.pf_strerror.argtypes = [ST]
        L.pf_strerror.restype = C.c_char_p
        L.pf_supported.argtypes = [P, P, I32]
        L.pf_supported.restype = I32
        L.pf_debug_math.argtypes = [I32, P, P, I64]
        L.pf_debug_math.restype = ST
        L.pf_debug_check_sqrt.argtypes = [C.c_uint32, C.c_uint32, P]
        L.pf_debug_check_sqrt.restype = ST
        if hasattr(L, "pf_peer_export"):   # (dev A/B builds of older sources lack the peer transport)
            for name, args in {"pf_peer_export": [P, P], "pf_peer_connect": [P, P],
                               "pf_peer_connect_local": [P, I32]}.items():
                getattr(L, name).argtypes = args
                getattr(L, name).restype = ST
            L.pf_peer_connected.argtypes = [P]
            L.pf_peer_connected.restype = I32
        _lib = L
    return _lib


def check(status: int, what: str = "") -> None:
    if status != PF_OK:
        msg = lib().pf_strerror(status).decode()
        raise PFError(f"{what}: {msg} ({status})")


def _ptr(x) -> int | None:
    """Pointer of a torch tensor / numpy array / int / None."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    return x.ctypes.data


def pf_query_sizes(cfg: pf_config, model: pf_model_params) -> pf_sizes:
    out = pf_sizes()
    check(lib().pf_query_sizes(C.byref(cfg), C.byref(model), C.byref(out)), "pf_query_sizes")
    return out


def pf_init(cfg, model, buffers: pf_buffers, stream: int, mu0, sigma0) -> C.c_void_p:
    h = C.c_void_p()
    check(lib().pf_init(C.byref(cfg), C.byref(model), C.byref(buffers), stream, _ptr(mu0), _ptr(sigma0),
                        C.byref(h)), "pf_init")
    return h


def pf_step(h, z, u) -> None:
    check(lib().pf_step(h, _ptr(z), _ptr(u)), "pf_step")


def pf_step_batch(h, T: int, zs, us, est) -> None:
    check(lib().pf_step_batch(h, T, _ptr(zs), _ptr(us), _ptr(est)), "pf_step_batch")


def pf_estimate(h, x_hat) -> tuple[float, int]:
    lw, idx = C.c_float(), C.c_int64()
    check(lib().pf_estimate(h, _ptr(x_hat), C.byref(lw), C.byref(idx)), "pf_estimate")
    return lw.value, idx.value


def pf_estimate_mean(h, x_mean) -> None:
    check(lib().pf_estimate_mean(h, _ptr(x_mean)), "pf_estimate_mean")


def pf_mean_partial(h) -> tuple[int, int]:
    p, n = C.c_void_p(), C.c_int32()
    check(lib().pf_mean_partial(h, C.byref(p), C.byref(n)), "pf_mean_partial")
    return p.value, n.value


def pf_reduce_means(h, partials_dev, count: int, x_mean) -> None:
    check(lib().pf_reduce_means(h, _ptr(partials_dev), count, _ptr(x_mean)), "pf_reduce_means")


def pf_record_ptr(h) -> tuple[int, int]:
    p, n = C.c_void_p(), C.c_int32()
    check(lib().pf_record_ptr(h, C.byref(p), C.byref(n)), "pf_record_ptr")
    return p.value, n.value


def pf_reduce_records(h, records_dev, count: int) -> None:
    check(lib().pf_reduce_records(h, _ptr(records_dev), count), "pf_reduce_records")


def pf_reduce_pool(h) -> None:
    check(lib().pf_reduce_pool(h), "pf_reduce_pool")


def pf_get_shard(h) -> pf_shard:
    out = pf_shard()
    check(lib().pf_get_shard(h, C.byref(out)), "pf_get_shard")
    return out


def pf_get_particles(h, state, logw) -> int:
    k = C.c_int64()
    check(lib().pf_get_particles(h, _ptr(state), _ptr(logw), C.byref(k)), "pf_get_particles")
    return k.value


def pf_set_particles(h, state, logw, step: int) -> None:
    check(lib().pf_set_particles(h, _ptr(state), _ptr(logw), step), "pf_set_particles")


def pf_debug_sample_weight(h, state_in, z, u, k: int, state_out, logw_out) -> None:
    check(lib().pf_debug_sample_weight(h, _ptr(state_in), _ptr(z), _ptr(u), k, _ptr(state_out), _ptr(logw_out)),
          "pf_debug_sample_weight")


def pf_debug_resample(h, q, ua, ub, ancestors, prob=None, alias=None) -> None:
    check(lib().pf_debug_resample(h, _ptr(q), _ptr(ua), _ptr(ub), _ptr(ancestors), _ptr(prob), _ptr(alias)),
          "pf_debug_resample")


def pf_debug_exchange(h, logw, src) -> None:
    check(lib().pf_debug_exchange(h, _ptr(logw), _ptr(src)), "pf_debug_exchange")


def pf_set_trace(h, enable: bool) -> None:
    check(lib().pf_set_trace(h, 1 if enable else 0), "pf_set_trace")


def pf_get_trace(h, src, ancestors) -> None:
    check(lib().pf_get_trace(h, _ptr(src), _ptr(ancestors)), "pf_get_trace")


def pf_destroy(h) -> None:
    check(lib().pf_destroy(h), "pf_destroy")


def pf_last_error(h) -> int:
    return lib().pf_last_error(h)


def pf_strerror(status: int) -> str:
    return lib().pf_strerror(status).decode()


def pf_supported() -> list[tuple[int, int]]:
    n = lib().pf_supported(None, None, 0)
    nj = (C.c_int32 * n)()
    m = (C.c_int32 * n)()
    lib().pf_supported(nj, m, n)
    return list(zip(list(nj), list(m)))


def pf_debug_math(fn: str, words, n: int, x2: bool = False):
    """Evaluate a contract function on the device; words: uint32 numpy array.
    x2: through the packed f32x2 code path (element pairs; n even)."""
    import numpy as np
    k = PF_MATH[fn] | (0x100 if x2 else 0)
    w = np.ascontiguousarray(words, dtype=np.uint32)
    out_n = 2 * n if fn in ("sincos2pi", "normal_pair") else 4 * n if fn == "philox" else n
    out = np.zeros(max(out_n, 1), np.uint32)
    check(lib().pf_debug_math(k, w.ctypes.data, out.ctypes.data, n), "pf_debug_math")
    return out[:out_n]


def pf_debug_check_sqrt(lo_bits: int, hi_bits: int) -> int:
    bad = C.c_uint64()
    check(lib().pf_debug_check_sqrt(lo_bits, hi_bits, C.byref(bad)), "pf_debug_check_sqrt")
    return bad.value


PF_PEER_BLOB_BYTES = 160


def pf_peer_export(h) -> bytes:
    buf = (C.c_uint8 * PF_PEER_BLOB_BYTES)()
    check(lib().pf_peer_export(h, buf), "pf_peer_export")
    return bytes(buf)


def pf_peer_connect(h, blobs: bytes) -> None:
    buf = (C.c_uint8 * len(blobs)).from_buffer_copy(blobs)
    check(lib().pf_peer_connect(h, buf), "pf_peer_connect")


def pf_peer_connect_local(handles) -> None:
    arr = (C.c_void_p * len(handles))(*[h.value for h in handles])
    check(lib().pf_peer_connect_local(arr, len(handles)), "pf_peer_connect_local")


def pf_query_mapping(h) -> dict:
    """The step kernel's launch configuration of handle h (include/pf.h pf_query_mapping)."""
    out = (C.c_int32 * 8)()
    check(lib().pf_query_mapping(h, out), "pf_query_mapping")
    keys = ("warps_per_group", "groups_per_cta", "tma_stages", "unroll", "min_ctas_per_sm", "split_first_load",
            "grid", "n_variants")
    return dict(zip(keys, list(out)))


def pf_peer_connected(h) -> bool:
    return bool(lib().pf_peer_connected(h))
