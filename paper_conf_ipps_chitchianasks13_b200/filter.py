"""ParticleFilter — torch-owned device buffers + the C-ABI handle.

Torch is plumbing here: it allocates the caller-owned buffers of pf.h
(pf_query_sizes) and provides the CUDA stream.  Every step of the hot path
runs in libpf_b200.so; this class only marshals arguments (binding.py).
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass

import numpy as np
import torch

from . import binding as B

_cchar, _addressof = ctypes.c_char, ctypes.addressof

TOPO = {"none": B.PF_TOPO_NONE, "ring": B.PF_TOPO_RING, "torus": B.PF_TOPO_TORUS2D, "all2all": B.PF_TOPO_ALL2ALL}
RESAMPLER = {"rws": B.PF_RESAMPLE_RWS, "vose": B.PF_RESAMPLE_VOSE}


@dataclass
class ArmModel:
    """Robotic arm of PAPER.md:22–24 §VII-A, Table II defaults (readings R15, R16)."""
    n_joints: int = 5
    arm_length: float = 1.0
    h_s: float = 0.1
    sigma_theta: float = 0.1
    sigma_pos: float = 0.1
    sigma_vel: float = 0.1
    sigma_cam: float = 0.1
    sigma_theta_meas: float = 0.1

    @property
    def d(self) -> int:
        return self.n_joints + 4

    def c(self) -> B.pf_model_params:
        return B.pf_model_params(B.PF_MODEL_ARM_PLANAR, self.n_joints, self.arm_length, self.h_s, self.sigma_theta,
                                 self.sigma_pos, self.sigma_vel, self.sigma_cam, self.sigma_theta_meas)


@dataclass
class LinearGaussModel:
    """1-D linear-Gaussian model (pf.h PF_MODEL_LINEAR_GAUSS_1D; pf_model.cuh):
    theta_k = theta_{k-1} + h_s u + w, w ~ N(0, sigma_theta^2); z = theta + v,
    v ~ N(0, sigma_theta_meas^2) — one joint of the arm with its angle sensor,
    the Kalman special case of SURVEY §8(c)."""
    h_s: float = 0.1
    sigma_theta: float = 0.1
    sigma_theta_meas: float = 0.1
    n_joints: int = 1

    @property
    def d(self) -> int:
        return 1

    def c(self) -> B.pf_model_params:
        return B.pf_model_params(B.PF_MODEL_LINEAR_GAUSS_1D, 1, 0.0, self.h_s, self.sigma_theta, 0.0, 0.0, 0.0,
                                 self.sigma_theta_meas)


def _dims(model) -> tuple[int, int]:
    """(measurement, control) dimensions of a model."""
    if isinstance(model, LinearGaussModel):
        return 1, 1
    return model.n_joints + 2, model.n_joints


POLICY = {"always": B.PF_POLICY_ALWAYS, "ess": B.PF_POLICY_ESS, "freq": B.PF_POLICY_FREQ}


def _policy_param(policy: str, value: float) -> int:
    """pf_config.resample_param (pf.h pf_policy): ESS tau in 1/65536 of m;
    resampling ratio as a threshold on a 32-bit Philox word."""
    if policy == "ess":
        return int(round(value * 65536))
    if policy == "freq":
        return int(round(value * 2.0**32))   # > 2^32 is rejected by pf_init (PF_EINVAL)
    return 0


def _f32(a) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.float32)


class ParticleFilter:
    """Distributed particle filter (Algorithm 2) on one GPU shard.

    Table I parameters: ``m`` particles per sub-filter,
    ``n_filters`` (global N), exchange scheme ``topo`` and ``t`` particles per
    exchange; ``resampler`` 'rws' | 'vose'.  ``rank``/``world`` select this
    process's shard of the sub-filters (pf.h).

    ``n_filters=1`` with ``m > 1024`` (a multiple of 4096) is the paper's
    centralized filter (§VI, Fig. 9): one filter resampled
    globally over all ``m`` particles (RWS or Vose; pf_central.cu).

    ``policy`` (reading R21, §IV): 'always' (default), 'ess'
    (resample a sub-filter when its effective sample size falls below
    ``policy_value`` x m) or 'freq' (each sub-filter resamples with
    probability ``policy_value`` per step).
    """

    def __init__(self, mu0, sigma0, model: ArmModel | LinearGaussModel | None = None, m: int = 256, n_filters: int = 4096,
                 t: int = 1, topo: str = "ring", resampler: str = "rws", seed: int = 0, rank: int = 0,
                 world: int = 1, torus_rows: int = 0, torus_cols: int = 0, device_inputs: bool = False,
                 device: torch.device | int | None = None, stream: torch.cuda.Stream | None = None,
                 policy: str = "always", policy_value: float = 1.0):
        self.model = model or ArmModel()
        self.device = torch.device("cuda", torch.cuda.current_device() if device is None else
                                   (device if isinstance(device, int) else device.index or 0))
        self.cfg = B.pf_config(m, n_filters, t, TOPO[topo], torus_rows, torus_cols, RESAMPLER[resampler],
                               seed, rank, world, B.PF_DEVICE_INPUTS if device_inputs else 0,
                               POLICY[policy], _policy_param(policy, policy_value))
        self.m, self.n_filters, self.t, self.topo, self.resampler = m, n_filters, t, topo, resampler
        self.rank, self.world = rank, world
        self.d = self.model.d
        self.nj = self.model.n_joints
        mc = self.model.c()
        sizes = B.pf_query_sizes(self.cfg, mc)
        with torch.cuda.device(self.device):
            self.stream = stream or torch.cuda.current_stream(self.device)
            alloc = lambda n: torch.empty(max(int(n), 16), dtype=torch.uint8, device=self.device)
            self._parts = alloc(sizes.state)
            self._mailbox = alloc(sizes.mailbox)
            self._scratch = alloc(sizes.scratch)
            bufs = B.pf_buffers(self._parts.data_ptr(), self._mailbox.data_ptr(), self._scratch.data_ptr())
            self.h = B.pf_init(self.cfg, mc, bufs, self.stream.cuda_stream, _f32(mu0), _f32(sigma0))
        self.shard = B.pf_get_shard(self.h)
        self.M_local = self.shard.n_local * m
        self.central = n_filters == 1 and m > 1024
        self._k = 0
        self._xhat = np.zeros(self.d, np.float32)
        # per-step host path (e2e): persistent input / output buffers with
        # their pointers taken once (numpy pointer extraction costs ~1 us)
        self._device_inputs = bool(self.cfg.flags & B.PF_DEVICE_INPUTS)
        self.zd, self.ud = _dims(self.model)
        self._zin = np.zeros(self.zd, np.float32)
        self._uin = np.zeros(self.ud, np.float32)
        self._zin_p, self._uin_p, self._xhat_p = self._zin.ctypes.data, self._uin.ctypes.data, self._xhat.ctypes.data
        self._step_fn, self._est_fn = B.lib().pf_step, B.lib().pf_estimate
        self._lw, self._idx = B.C.c_float(), B.C.c_int64()
        self._lw_ref, self._idx_ref = B.C.byref(self._lw), B.C.byref(self._idx)

    # -- views of the caller-owned buffers (torch, device) -------------------
    @property
    def particles(self) -> torch.Tensor:
        """Device particle blocks [n_local][d+1][m] (rows 0..d-1 state, row d log-weight).
        Centralized filter: the AoS state records [m][S] (S = d rounded up to even) of the
        current step's buffer (ping-pong, k & 1); its log-weights are `central_logw`."""
        if self.central:
            S = (self.d + 1) & ~1
            n = self.m * S
            off = 4 * n * (self._k & 1)
            return self._parts[off: off + 4 * n].view(torch.float32).view(self.m, S)
        n = self.shard.n_local * (self.d + 1) * self.m
        return self._parts[: 4 * n].view(torch.float32).view(self.shard.n_local, self.d + 1, self.m)

    @property
    def central_logw(self) -> torch.Tensor:
        """Centralized filter: the log-weights [m] of the current step (device)."""
        S = (self.d + 1) & ~1
        off = 4 * (2 * self.m * S + (self._k & 1) * self.m)
        return self._parts[off: off + 4 * self.m].view(torch.float32)

    @property
    def mailbox(self) -> torch.Tensor:
        s = self.shard
        n = 2 * s.n_ext * s.t * s.entry_floats
        return self._mailbox[: 4 * n].view(torch.float32).view(2, s.n_ext, s.t, s.entry_floats)

    @property
    def record(self) -> torch.Tensor:
        ptr, n = B.pf_record_ptr(self.h)
        off = ptr - self._scratch.data_ptr()
        return self._scratch[off: off + 4 * n].view(torch.float32)

    # -- the path -----------------------------------------------------------
    def step(self, z, u) -> None:
        """One time step (host numpy z/u, or device tensors with device_inputs)."""
        if self._device_inputs:
            st = self._step_fn(self.h, z.data_ptr(), u.data_ptr())
        else:   # copied into the launch by pf_step (host inputs travel with the kernel)
            if (type(z) is np.ndarray and type(u) is np.ndarray and z.dtype == np.float32 and u.dtype == np.float32
                    and z.flags.c_contiguous and u.flags.c_contiguous and z.size == self.zd and u.size == self.ud):
                # no staging copy; the address through the buffer protocol (writable
                # arrays) costs a third of ndarray.ctypes.data, which builds an object
                zf, uf = z.flags, u.flags
                zp = _addressof(_cchar.from_buffer(z)) if zf.writeable else z.ctypes.data
                up = _addressof(_cchar.from_buffer(u)) if uf.writeable else u.ctypes.data
                st = self._step_fn(self.h, zp, up)
            else:
                np.copyto(self._zin, z, casting="same_kind")
                np.copyto(self._uin, u, casting="same_kind")
                st = self._step_fn(self.h, self._zin_p, self._uin_p)
        if st != B.PF_OK:
            B.check(st, "pf_step")
        self._k += 1

    def step_batch(self, zs: torch.Tensor, us: torch.Tensor, est: torch.Tensor | None = None) -> None:
        """T steps with device-resident inputs zs [T][zd], us [T][ud]; est [T][4+d]."""
        assert zs.is_cuda and us.is_cuda and zs.dtype == torch.float32 and us.dtype == torch.float32
        B.pf_step_batch(self.h, zs.shape[0], zs.data_ptr(), us.data_ptr(), None if est is None else est.data_ptr())
        self._k += zs.shape[0]

    # -- peer transport (include/pf.h: halo + global estimate inside the step
    #    kernel over NVLink peer memory) ------------------------------------
    def peer_export(self) -> bytes:
        return B.pf_peer_export(self.h)

    def peer_connect(self, blobs: bytes) -> None:
        B.pf_peer_connect(self.h, blobs)

    @staticmethod
    def peer_connect_local(filters) -> None:
        """Connect the shards of ONE process (tests on one device; each shard
        must step on its own stream)."""
        B.pf_peer_connect_local([f.h for f in filters])

    @property
    def peer_connected(self) -> bool:
        return B.pf_peer_connected(self.h)

    def estimate(self):
        """(x_hat [d], logw, global index) of the particle with the highest weight."""
        st = self._est_fn(self.h, self._xhat_p, self._lw_ref, self._idx_ref)
        if st != B.PF_OK:
            B.check(st, "pf_estimate")
        return self._xhat.copy(), self._lw.value, self._idx.value

    def estimate_mean(self) -> np.ndarray:
        """Weighted-average estimate x [d] of the last step's set (R22; §VI-D)."""
        x = np.zeros(self.d, np.float32)
        B.pf_estimate_mean(self.h, x)
        return x

    def mean_partial(self) -> torch.Tensor:
        """World > 1: this shard's partial record (device float64 [d+1]; slot 0 = uint64 bits)."""
        ptr, n = B.pf_mean_partial(self.h)
        off = ptr - self._scratch.data_ptr()
        return self._scratch[off: off + 8 * n].view(torch.float64)

    def reduce_means(self, partials: torch.Tensor) -> np.ndarray:
        """Mean of gathered partial records [count][d+1] (device float64)."""
        x = np.zeros(self.d, np.float32)
        B.pf_reduce_means(self.h, partials.data_ptr(), partials.shape[0], x)
        return x

    def reduce_records(self, records: torch.Tensor) -> None:
        B.pf_reduce_records(self.h, records.data_ptr(), records.shape[0])

    def reduce_pool(self) -> None:
        """All-to-All, world > 1: global best t from the gathered pool rows."""
        B.pf_reduce_pool(self.h)

    def get_particles(self):
        s = np.zeros((self.d, self.M_local), np.float32)
        w = np.zeros(self.M_local, np.float32)
        k = B.pf_get_particles(self.h, s, w)
        self._k = k
        return s, w, k

    def set_particles(self, state, logw, step: int) -> None:
        B.pf_set_particles(self.h, _f32(state), _f32(logw), step)
        self._k = step

    # -- test hooks ----------------------------------------------------------
    def debug_sample_weight(self, state_in, z, u, k: int):
        s_out = np.zeros((self.d, self.M_local), np.float32)
        w_out = np.zeros(self.M_local, np.float32)
        B.pf_debug_sample_weight(self.h, _f32(state_in), _f32(z), _f32(u), k, s_out, w_out)
        self._k = k
        return s_out, w_out

    def debug_resample(self, q, ua, ub):
        q = np.ascontiguousarray(q, np.uint32)
        anc = np.zeros(q.shape, np.int32)
        prob = np.zeros(q.shape, np.uint64)
        alias = np.zeros(q.shape, np.int32)
        B.pf_debug_resample(self.h, q, np.ascontiguousarray(ua, np.uint32), np.ascontiguousarray(ub, np.uint32),
                            anc, prob, alias)
        return anc, prob, alias

    def debug_exchange(self, logw):
        src = np.zeros(self.M_local, np.int64)
        B.pf_debug_exchange(self.h, _f32(logw), src)
        return src

    def set_trace(self, enable: bool = True) -> None:
        B.pf_set_trace(self.h, enable)

    def trace(self):
        src = np.zeros(self.M_local, np.int64)
        anc = np.zeros(self.M_local, np.int32)
        B.pf_get_trace(self.h, src, anc)
        return src, anc

    def close(self) -> None:
        if getattr(self, "h", None):
            B.pf_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
