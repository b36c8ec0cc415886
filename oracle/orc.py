"""oracle/orc.py — ctypes wrapper around the CPU oracle liborc.so.

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / ``--impl reference`` leg; never by the product
package.  Argument marshalling only — every computation is in orc.c /
orc_impl.inc (plain C, Algorithm 2 of PAPER.md:16; see orc.h).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "liborc.so")
SOURCES = [os.path.join(HERE, f) for f in ("orc.c", "orc_impl.inc", "orc.h")]

TOPO = {"none": 0, "ring": 1, "torus": 2, "all2all": 3}
RESAMPLER = {"rws": 0, "vose": 1}
POLICY = {"always": 0, "ess": 1, "freq": 2}


def policy_param(policy: str, value: float) -> int:
    """R21 integer parameter: ESS threshold tau (fraction of m) in 1/65536;
    resampling ratio in [0, 1] as a threshold on a 32-bit Philox word."""
    if policy == "ess":
        return int(round(value * 65536))
    if policy == "freq":
        return min(1 << 32, max(0, int(round(value * 2.0**32))))
    return 0

CFLAGS = ["-O2", "-std=c11", "-Wall", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared"]


def build(force: bool = False) -> str:
    """Compile liborc.so with gcc (no contraction: F-contract of DESIGN.md §4)."""
    stale = force or not os.path.exists(LIB_PATH) or any(
        os.path.getmtime(s) > os.path.getmtime(LIB_PATH) for s in SOURCES)
    if stale:
        tmp = LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, os.path.join(HERE, "orc.c"), "-lm"])
        os.replace(tmp, LIB_PATH)
    return LIB_PATH


class OrcConfig(C.Structure):
    _fields_ = [("m", C.c_int32), ("n_filters", C.c_int64), ("t", C.c_int32), ("topo", C.c_int32),
                ("torus_rows", C.c_int32), ("torus_cols", C.c_int32), ("resampler", C.c_int32),
                ("seed", C.c_uint64), ("policy", C.c_int32), ("policy_param", C.c_uint64)]


MODEL = {"arm": 0, "lg1": 1}


class OrcModel(C.Structure):
    _fields_ = [("model", C.c_int32), ("n_joints", C.c_int32), ("arm_length", C.c_float), ("h_s", C.c_float),
                ("sigma_theta", C.c_float), ("sigma_pos", C.c_float), ("sigma_vel", C.c_float),
                ("sigma_cam", C.c_float), ("sigma_theta_meas", C.c_float)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(LIB_PATH)
        P = C.c_void_p
        sig = {
            "orc_philox4x32_10": (None, [P, P, P]),
            "orc_s_sin": (C.c_float, [C.c_float]),
            "orc_s_cos": (C.c_float, [C.c_float]),
            "orc_s_log": (C.c_float, [C.c_float]),
            "orc_s_sincos2pi": (None, [C.c_uint32, P, P]),
            "orc_s_expq": (C.c_uint32, [C.c_float]),
            "orc_s_normal_pair": (None, [C.c_uint32, C.c_uint32, P]),
            "orc_d_normal_pair": (None, [C.c_uint32, C.c_uint32, P]),
            "orc_s_camera": (None, [P, P, P]),
            "orc_d_camera": (None, [P, P, P]),
            "orc_s_loglik": (C.c_float, [P, P, P]),
            "orc_d_loglik": (C.c_double, [P, P, P]),
            "orc_s_sample_weight": (None, [P, C.c_uint64, C.c_int64, C.c_int64, P, P, P, C.c_int64, P, P]),
            "orc_d_sample_weight": (None, [P, C.c_uint64, C.c_int64, C.c_int64, P, P, P, C.c_int64, P, P]),
            "orc_rws_draw": (C.c_int32, [P, C.c_int32, C.c_uint32]),
            "orc_vose_build": (None, [P, C.c_int32, P, P]),
            "orc_s_weighted_mean": (None, [P, P, C.c_int64, C.c_int32, P]),
            "orc_d_weighted_mean": (None, [P, P, C.c_int64, C.c_int32, P]),
            "orc_s_estimate_mean": (C.c_int, [P, P]),
            "orc_d_estimate_mean": (C.c_int, [P, P]),
            "orc_should_resample": (C.c_int, [C.c_int32, C.c_uint64, P, C.c_int32, C.c_uint64, C.c_int64,
                                              C.c_int64]),
            "orc_vose_draw": (C.c_int32, [P, P, C.c_int32, C.c_uint64, C.c_uint32, C.c_uint32]),
            "orc_resample_q": (C.c_int, [P, C.c_int64, C.c_int32, C.c_int32, P, P, P]),
            "orc_s_normalise": (None, [P, C.c_int32, P]),
            "orc_s_resample_logw": (C.c_int, [P, P, C.c_int64, P, P]),
            "orc_neighbors": (C.c_int32, [P, C.c_int64, P]),
            "orc_torus_shape": (None, [P, P, P]),
            "orc_s_exchange": (C.c_int, [P, P, P]),
            "orc_s_create": (P, [P, P, P, P]),
            "orc_s_step": (C.c_int, [P, P, P]),
            "orc_s_estimate": (C.c_int, [P, P, P, P]),
            "orc_s_get": (C.c_int, [P, P, P, P]),
            "orc_s_set": (C.c_int, [P, P, P, C.c_int64]),
            "orc_s_trace": (C.c_int, [P, P, P]),
            "orc_s_destroy": (None, [P]),
            "orc_s_step_subset": (C.c_int, [P, P, P, P, C.c_int64, P, P, P, C.c_int64, P, P]),
            "orc_s_central_slots": (C.c_int, [P, P, P, P, C.c_int64, P, P, P, C.c_int64, P, P]),
            "orc_d_create": (P, [P, P, P, P]),
            "orc_d_step": (C.c_int, [P, P, P]),
            "orc_d_estimate": (C.c_int, [P, P, P, P]),
            "orc_d_get": (C.c_int, [P, P, P, P]),
            "orc_d_destroy": (None, [P]),
        }
        for name, (res, args) in sig.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


def _f64(a):
    return np.ascontiguousarray(a, dtype=np.float64)


def _u32(a):
    return np.ascontiguousarray(a, dtype=np.uint32)


@dataclass
class Model:
    """Table II model parameters — reading R15/R16 defaults."""
    n_joints: int = 5
    arm_length: float = 1.0
    h_s: float = 0.1
    sigma_theta: float = 0.1
    sigma_pos: float = 0.1
    sigma_vel: float = 0.1
    sigma_cam: float = 0.1
    sigma_theta_meas: float = 0.1
    kind: str = "arm"          # "arm" | "lg1" (1-D linear-Gaussian: one joint + its sensor)

    @property
    def d(self) -> int:
        return 1 if self.kind == "lg1" else self.n_joints + 4

    def c(self) -> OrcModel:
        return OrcModel(MODEL[self.kind], self.n_joints, self.arm_length, self.h_s, self.sigma_theta, self.sigma_pos,
                        self.sigma_vel, self.sigma_cam, self.sigma_theta_meas)


@dataclass
class Config:
    """Table I filter parameters: m, N, X, t (+ resampler, seed)."""
    m: int = 64
    n_filters: int = 16
    t: int = 1
    topo: str = "ring"
    resampler: str = "rws"
    seed: int = 0
    torus_rows: int = 0
    torus_cols: int = 0
    policy: str = "always"     # R21: "always" | "ess" | "freq"
    policy_param: int = 0      # ess: tau * 2^16; freq: ratio * 2^32 (integers, see policy_param())

    def c(self) -> OrcConfig:
        return OrcConfig(self.m, self.n_filters, self.t, TOPO[self.topo], self.torus_rows,
                         self.torus_cols, RESAMPLER[self.resampler], self.seed, POLICY[self.policy],
                         self.policy_param)


# ---- component functions --------------------------------------------------
def philox(ctr, key) -> np.ndarray:
    c, k, out = _u32(ctr), _u32(key), np.zeros(4, np.uint32)
    lib().orc_philox4x32_10(_p(c), _p(k), _p(out))
    return out


def s_sin(x: float) -> float:
    return lib().orc_s_sin(x)


def s_cos(x: float) -> float:
    return lib().orc_s_cos(x)


def s_log(x: float) -> float:
    return lib().orc_s_log(x)


def s_sincos2pi(m23: int):
    s, c = C.c_float(), C.c_float()
    lib().orc_s_sincos2pi(m23, C.byref(s), C.byref(c))
    return s.value, c.value


def s_expq(delta: float) -> int:
    return lib().orc_s_expq(delta)


def s_normal_pair(x0: int, x1: int) -> np.ndarray:
    out = np.zeros(2, np.float32)
    lib().orc_s_normal_pair(x0, x1, _p(out))
    return out


def d_normal_pair(x0: int, x1: int) -> np.ndarray:
    out = np.zeros(2, np.float64)
    lib().orc_d_normal_pair(x0, x1, _p(out))
    return out


def camera(model: Model, x, fp64: bool = False) -> np.ndarray:
    mc = model.c()
    if fp64:
        xx, out = _f64(x), np.zeros(2, np.float64)
        lib().orc_d_camera(C.byref(mc), _p(xx), _p(out))
    else:
        xx, out = _f32(x), np.zeros(2, np.float32)
        lib().orc_s_camera(C.byref(mc), _p(xx), _p(out))
    return out


def loglik(model: Model, x, z, fp64: bool = False) -> float:
    mc = model.c()
    if fp64:
        return lib().orc_d_loglik(C.byref(mc), _p(_f64(x)), _p(_f64(z)))
    return lib().orc_s_loglik(C.byref(mc), _p(_f32(x)), _p(_f32(z)))


def sample_weight(model: Model, seed: int, state_in, z, u, k: int, p_offset: int = 0, fp64=False):
    """a1–a3 for SoA state_in [d][M]: returns (state_out [d][M], logw [M])."""
    mc = model.c()
    conv = _f64 if fp64 else _f32
    s_in = conv(state_in)
    d, M = s_in.shape
    assert d == model.d
    s_out = np.empty_like(s_in)
    w = np.empty(M, s_in.dtype)
    fn = lib().orc_d_sample_weight if fp64 else lib().orc_s_sample_weight
    fn(C.byref(mc), seed, M, p_offset, _p(s_in), _p(conv(z)), _p(conv(u)), k, _p(s_out), _p(w))
    return s_out, w


def rws_draw(q, U: int) -> int:
    qq = _u32(q)
    return lib().orc_rws_draw(_p(qq), len(qq), U)


def weighted_mean(state, logw, fp64: bool = False) -> np.ndarray:
    """R22: integer-weighted average of a weighted set (state [d][M], logw [M])."""
    conv = _f64 if fp64 else _f32
    st, lw = conv(state), conv(logw)
    d, M = st.shape
    out = np.zeros(d, st.dtype)
    (lib().orc_d_weighted_mean if fp64 else lib().orc_s_weighted_mean)(_p(st), _p(lw), M, d, _p(out))
    return out


def should_resample(policy: str, param: int, q, seed: int, n: int, k: int) -> bool:
    qq = _u32(q)
    return bool(lib().orc_should_resample(POLICY[policy], param, _p(qq), len(qq), seed, n, k))


def vose_build(q):
    qq = _u32(q)
    m = len(qq)
    prob, alias = np.zeros(m, np.uint64), np.zeros(m, np.int32)
    lib().orc_vose_build(_p(qq), m, _p(prob), _p(alias))
    return prob, alias


def vose_draw(prob, alias, Q: int, Ua: int, Ub: int) -> int:
    pr = np.ascontiguousarray(prob, np.uint64)
    al = np.ascontiguousarray(alias, np.int32)
    return lib().orc_vose_draw(_p(pr), _p(al), len(pr), Q, Ua, Ub)


def resample_q(q, resampler: str, ua, ub) -> np.ndarray:
    """q [N][m] u32 integer weights, explicit uniforms [N][m] -> ancestors [N][m]."""
    qq = _u32(q)
    N, m = qq.shape
    anc = np.zeros((N, m), np.int32)
    rc = lib().orc_resample_q(_p(qq), N, m, RESAMPLER[resampler], _p(_u32(ua)), _p(_u32(ub)), _p(anc))
    if rc:
        raise ValueError(f"orc_resample_q failed: {rc}")
    return anc


def normalise(logw) -> np.ndarray:
    w = _f32(logw)
    q = np.zeros(len(w), np.uint32)
    lib().orc_s_normalise(_p(w), len(w), _p(q))
    return q


def resample_logw(cfg: Config, logw, k: int):
    """logw [N][m] -> (ancestors [N][m], q [N][m]) with Philox (p, k, 0, 0) draws."""
    w = _f32(logw).reshape(cfg.n_filters, cfg.m)
    anc = np.zeros(w.shape, np.int32)
    q = np.zeros(w.shape, np.uint32)
    cc = cfg.c()
    rc = lib().orc_s_resample_logw(C.byref(cc), _p(w), k, _p(anc), _p(q))
    if rc:
        raise ValueError(f"orc_s_resample_logw failed: {rc}")
    return anc, q


def neighbors(cfg: Config, n: int) -> list[int]:
    nb = np.zeros(4, np.int64)
    cc = cfg.c()
    deg = lib().orc_neighbors(C.byref(cc), n, _p(nb))
    return [int(v) for v in nb[:deg]]


def torus_shape(cfg: Config):
    r, c = C.c_int64(), C.c_int64()
    cc = cfg.c()
    lib().orc_torus_shape(C.byref(cc), C.byref(r), C.byref(c))
    return r.value, c.value


def exchange(cfg: Config, logw) -> np.ndarray:
    """logw [N][m] -> src [N][m] (global source index of every slot)."""
    w = _f32(logw).reshape(cfg.n_filters, cfg.m)
    src = np.zeros(w.shape, np.int64)
    cc = cfg.c()
    rc = lib().orc_s_exchange(C.byref(cc), _p(w), _p(src))
    if rc:
        raise ValueError(f"orc_s_exchange failed: {rc}")
    return src


def step_subset(cfg: Config, model: Model, state, logw, k: int, z, u, subs):
    """Step k of the listed sub-filters from the full weighted set of step k-1:
    returns (state [d][len(subs)*m], logw [len(subs)*m])."""
    st, lw = _f32(state), _f32(logw)
    sb = np.ascontiguousarray(subs, np.int64)
    d, m = model.d, cfg.m
    out_s = np.zeros((d, len(sb) * m), np.float32)
    out_w = np.zeros(len(sb) * m, np.float32)
    cc, mc = cfg.c(), model.c()
    rc = lib().orc_s_step_subset(C.byref(cc), C.byref(mc), _p(st), _p(lw), k, _p(_f32(z)), _p(_f32(u)), _p(sb),
                                 len(sb), _p(out_s), _p(out_w))
    if rc:
        raise ValueError(f"orc_s_step_subset failed: {rc}")
    return out_s, out_w


def central_slots(cfg: Config, model: Model, state, logw, k: int, z, u, slots):
    """Centralized filter: step k of the listed slots from the weighted set of
    step k-1: returns (state [d][len(slots)], logw [len(slots)])."""
    st, lw = _f32(state), _f32(logw)
    sl = np.ascontiguousarray(slots, np.int64)
    out_s = np.zeros((model.d, len(sl)), np.float32)
    out_w = np.zeros(len(sl), np.float32)
    cc, mc = cfg.c(), model.c()
    rc = lib().orc_s_central_slots(C.byref(cc), C.byref(mc), _p(st), _p(lw), k, _p(_f32(z)), _p(_f32(u)), _p(sl),
                                   len(sl), _p(out_s), _p(out_w))
    if rc:
        raise ValueError(f"orc_s_central_slots failed: {rc}")
    return out_s, out_w


# ---- the filter -------------------------------------------------------------
class Filter:
    """Algorithm 2, one call of step() per time step."""

    def __init__(self, cfg: Config, model: Model, mu0, sigma0, fp64: bool = False):
        self.cfg, self.model, self.fp64 = cfg, model, fp64
        self._cc, self._mc = cfg.c(), model.c()
        self._conv = _f64 if fp64 else _f32
        self.d = model.d
        self.M = cfg.m * cfg.n_filters
        L = lib()
        pre = "orc_d_" if fp64 else "orc_s_"
        self._fn = {n: getattr(L, pre + n) for n in ("create", "step", "estimate", "estimate_mean", "get", "destroy")}
        if not fp64:
            self._fn["set"] = L.orc_s_set
            self._fn["trace"] = L.orc_s_trace
        h = self._fn["create"](C.byref(self._cc), C.byref(self._mc), _p(self._conv(mu0)),
                               _p(self._conv(sigma0)))
        if not h:
            raise ValueError("oracle rejected the configuration")
        self._h = h

    def __del__(self):
        h = getattr(self, "_h", None)
        if h:
            self._fn["destroy"](h)
            self._h = None

    def step(self, z, u) -> None:
        rc = self._fn["step"](self._h, _p(self._conv(z)), _p(self._conv(u)))
        if rc:
            raise RuntimeError(f"oracle step failed: {rc}")

    def estimate(self):
        dt = np.float64 if self.fp64 else np.float32
        x = np.zeros(self.d, dt)
        w = (C.c_double if self.fp64 else C.c_float)()
        idx = C.c_int64()
        rc = self._fn["estimate"](self._h, _p(x), C.byref(w), C.byref(idx))
        if rc:
            raise RuntimeError("no estimate before the first step")
        return x, w.value, idx.value

    def estimate_mean(self) -> np.ndarray:
        """R22: the weighted-average estimate of the current set."""
        x = np.zeros(self.d, np.float64 if self.fp64 else np.float32)
        if self._fn["estimate_mean"](self._h, _p(x)):
            raise RuntimeError("no estimate before the first step")
        return x

    def get(self):
        dt = np.float64 if self.fp64 else np.float32
        s = np.zeros((self.d, self.M), dt)
        w = np.zeros(self.M, dt)
        k = C.c_int64()
        self._fn["get"](self._h, _p(s), _p(w), C.byref(k))
        return s, w, k.value

    def set(self, state, logw, step: int) -> None:
        s, w = _f32(state), _f32(logw)
        assert s.shape == (self.d, self.M) and w.shape == (self.M,)
        if self._fn["set"](self._h, _p(s), _p(w), step):
            raise ValueError("bad step")

    def trace(self):
        src = np.zeros(self.M, np.int64)
        anc = np.zeros(self.M, np.int32)
        self._fn["trace"](self._h, _p(src), _p(anc))
        return src, anc
