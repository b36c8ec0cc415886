"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This module holds NONE of the filter's arithmetic.  It is the simulated
plant: a robotic arm tracking an object on a lemniscate (§VIII-A,
Fig.8 "starts by heading up from the right side"), with the recipe of reading
R16:

* object on a Bernoulli lemniscate a = 1 m, tau_k = 2 pi k / T; velocity by
  finite difference / h_s;
* true joint angles theta_0 = linspace(0.3, -0.3, n_j), theta_k = theta_{k-1}
  + h_s u_{k-1} + 0.1 xi, controls u_{i,k} = 0.5 sin(2 pi k / T + i);
* measurements z_k = (camera-frame object position + 0.1 xi, theta_k + 0.1 xi);
* prior mu0 = X_0 with the object x shifted by -0.2 m, sigma0 = (0.1 rad per
  angle, 0.25 m, 0.25 m, 0.25 m/s, 0.25 m/s);
* generator RNG numpy default_rng(10000 + seed).

The camera geometry of the plant is evaluated here in float64 numpy, written
independently of both the oracle (C) and the kernels (CUDA).
"""
from __future__ import annotations

import numpy as np


def lemniscate(tau: np.ndarray, a: float = 1.0):
    s, c = np.sin(tau), np.cos(tau)
    den = 1.0 + s * s
    return a * c / den, a * s * c / den


def _plant_camera(theta: np.ndarray, obj: np.ndarray, arm_length: float) -> np.ndarray:
    nj = theta.shape[-1]
    phi = np.cumsum(theta, axis=-1)
    link = arm_length / nj
    px = link * np.cos(phi).sum(-1)
    py = link * np.sin(phi).sum(-1)
    ph = phi[..., -1]
    dx, dy = obj[..., 0] - px, obj[..., 1] - py
    return np.stack([np.cos(ph) * dx + np.sin(ph) * dy, -np.sin(ph) * dx + np.cos(ph) * dy], -1)


def make_trajectory(n_joints: int, T: int, seed: int = 0, h_s: float = 0.1, noise: float = 0.1,
                    arm_length: float = 1.0) -> dict:
    """Ground truth X[T+1, d], measurements Z[T+1, n_j+2] (Z[0] unused), controls
    U[T+1, n_j] (step k uses U[k-1]), prior mu0[d], sigma0[d]; all float32."""
    rng = np.random.default_rng(10000 + seed)
    nj, d = n_joints, n_joints + 4
    k = np.arange(-1, T + 1)
    ox, oy = lemniscate(2 * np.pi * k / T)
    obj = np.stack([ox, oy], -1)
    vel = (obj[1:] - obj[:-1]) / h_s
    obj = obj[1:]
    U = np.stack([0.5 * np.sin(2 * np.pi * np.arange(T + 1) / T + i) for i in range(nj)], -1)
    theta = np.zeros((T + 1, nj))
    theta[0] = np.linspace(0.3, -0.3, nj)
    for t in range(1, T + 1):
        theta[t] = theta[t - 1] + h_s * U[t - 1] + noise * rng.standard_normal(nj)
    X = np.concatenate([theta, obj, vel], -1)
    cam = _plant_camera(theta, obj, arm_length)
    Z = np.concatenate([cam + noise * rng.standard_normal((T + 1, 2)),
                        theta + noise * rng.standard_normal((T + 1, nj))], -1)
    mu0 = X[0].copy()
    mu0[nj] -= 0.2
    sigma0 = np.concatenate([np.full(nj, 0.1), np.full(4, 0.25)])
    f = lambda a: np.ascontiguousarray(a, np.float32)
    return {"X": f(X), "Z": f(Z), "U": f(U), "mu0": f(mu0), "sigma0": f(sigma0), "T": T,
            "n_joints": nj, "d": d}


def random_particles(traj: dict, M: int, seed: int, spread: float = 0.2):
    """SoA particle set [d][M] scattered around the true state X[1] (float32)."""
    rng = np.random.default_rng(20000 + seed)
    x = rng.standard_normal((traj["d"], M), dtype=np.float32)   # float32 throughout: 16M x 32 fits
    x *= np.float32(spread)
    x += traj["X"][1][:, None].astype(np.float32)
    return x


def random_logw(N: int, m: int, seed: int, ties: bool = True, scale: float = 30.0) -> np.ndarray:
    """Log-weights [N][m] shaped like the path's (negative, spread over tens of
    nats, R7), with deliberate exact ties when ``ties`` (tie-breaks, R6)."""
    rng = np.random.default_rng(30000 + seed)
    w = -np.abs(rng.standard_normal((N, m)) * scale) - rng.exponential(2.0, (N, m))
    if ties:
        w = np.round(w * 4) / 4
    return np.ascontiguousarray(w, np.float32)


def random_q(N: int, m: int, seed: int, kind: str = "mixed") -> np.ndarray:
    """Integer weights q [N][m] in [0, 2^22] with at least one 2^22 per row."""
    rng = np.random.default_rng(40000 + seed)
    if kind == "uniform":
        q = np.full((N, m), 1 << 22, np.uint32)
    elif kind == "onehot":
        q = np.zeros((N, m), np.uint32)
        q[np.arange(N), rng.integers(0, m, N)] = 1 << 22
    else:
        ell = -rng.exponential(4.0, (N, m))
        ell[rng.random((N, m)) < 0.2] = -30.0
        q = np.floor(np.exp(ell - ell.max(1, keepdims=True)) * (1 << 22)).astype(np.uint32)
    return q


def make_lg_trajectory(T: int, seed: int = 0, h_s: float = 0.1, sigma_theta: float = 0.1,
                       sigma_meas: float = 0.1, prior_offset: float = 0.2, prior_std: float = 0.25) -> dict:
    """The 1-D linear-Gaussian plant (pf_model.cuh LinearGauss1D: one joint with
    its angle sensor): theta_k = theta_{k-1} + h_s u_{k-1} + sigma_theta xi,
    z_k = theta_k + sigma_meas xi, u_k = 0.5 sin(2 pi k / T).  Arrays shaped
    like make_trajectory's with d = zd = ud = 1: X[T+1, 1], Z[T+1, 1] (Z[0]
    unused), U[T+1, 1]; prior mu0 = theta_0 + prior_offset, sigma0 = prior_std."""
    rng = np.random.default_rng(50000 + seed)
    U = 0.5 * np.sin(2 * np.pi * np.arange(T + 1) / T)[:, None]
    theta = np.zeros((T + 1, 1))
    theta[0] = 0.3
    for t in range(1, T + 1):
        theta[t] = theta[t - 1] + h_s * U[t - 1] + sigma_theta * rng.standard_normal(1)
    Z = theta + sigma_meas * rng.standard_normal((T + 1, 1))
    f = lambda a: np.ascontiguousarray(a, np.float32)
    return {"X": f(theta), "Z": f(Z), "U": f(U), "mu0": f(theta[0] + prior_offset),
            "sigma0": f(np.full(1, prior_std)), "T": T, "n_joints": 1, "d": 1}
