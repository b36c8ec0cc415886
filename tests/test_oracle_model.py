"""Oracle pins: robotic-arm model hooks (§VII-A; readings
R14–R16, contract F8–F10) against closed forms and invariants."""
import json
import math
import os

import numpy as np

from conftest import GOLDEN

G = json.load(open(os.path.join(GOLDEN, "model_golden.json")))


def _state(theta, obj, vel=(0.0, 0.0)):
    return np.array(list(theta) + list(obj) + list(vel), np.float64)


def test_two_link_closed_forms(orc):
    g = G["two_link"]
    md = orc.Model(n_joints=2, arm_length=g["arm_length"])
    for case in g["cases"]:
        x = _state(case["theta"], case["obj"])
        for fp64 in (False, True):
            got = orc.camera(md, x, fp64=fp64)
            np.testing.assert_allclose(got, case["camera"], atol=1e-6)


def test_five_link_golden_and_loglik(orc):
    g = G["five_link"]
    md = orc.Model(n_joints=5, arm_length=g["arm_length"], sigma_cam=g["sigma"],
                   sigma_theta_meas=g["sigma"])
    x = _state(g["theta"], g["obj"])
    cam = orc.camera(md, x)
    np.testing.assert_allclose(cam, g["camera"], atol=1e-6)
    dz = g["z_offset"]
    z = np.array([cam[0] + dz[0], cam[1] + dz[1]] + [t + dz[2] for t in g["theta"]])
    assert abs(orc.loglik(md, x, z) - g["logw"]) <= 1e-5
    # sigma is an fp32 model parameter (0.1f), so fp64 is exact only to ~1e-7
    assert abs(orc.loglik(md, x, z, fp64=True) - g["logw"]) <= 1e-6


def test_loglik_unit_residuals(orc):
    # residual = sigma in exactly one component -> logw = -1/2 exactly
    md = orc.Model(n_joints=3, sigma_cam=0.25, sigma_theta_meas=0.5)
    x = _state([0.2, -0.1, 0.05], [0.7, 0.3])
    cam = orc.camera(md, x)
    base = np.concatenate([cam, x[:3]]).astype(np.float32)
    assert orc.loglik(md, x, base) == 0.0
    for comp, sig in [(0, 0.25), (1, 0.25), (2, 0.5), (4, 0.5)]:
        z = base.copy()
        z[comp] += np.float32(sig)
        # fp32: the residual (z - h) is exact here only up to rounding of z
        assert abs(orc.loglik(md, x, z) + 0.5) < 1e-5
        assert abs(orc.loglik(md, x, z.astype(np.float64), fp64=True) + 0.5) < 1e-6


def test_camera_rotation_invariance(orc):
    # rotating the world about the base (theta_0 + a, object rotated by a)
    # leaves the camera-frame measurement unchanged
    rng = np.random.default_rng(0)
    for nj in (2, 5, 28):
        md = orc.Model(n_joints=nj)
        for _ in range(20):
            th = rng.uniform(-1, 1, nj)
            ob = rng.uniform(-2, 2, 2)
            a = rng.uniform(-np.pi, np.pi)
            ob2 = np.array([math.cos(a) * ob[0] - math.sin(a) * ob[1],
                            math.sin(a) * ob[0] + math.cos(a) * ob[1]])
            th2 = th.copy()
            th2[0] += a
            c1 = orc.camera(md, _state(th, ob), fp64=True)
            c2 = orc.camera(md, _state(th2, ob2), fp64=True)
            np.testing.assert_allclose(c1, c2, atol=1e-12)
            c1s = orc.camera(md, _state(th, ob))
            np.testing.assert_allclose(c1s, c1, atol=2e-5)


def test_camera_translation(orc):
    # moving the object by (dx, dy) in the camera frame axes moves the measurement by it
    md = orc.Model(n_joints=4)
    th = np.array([0.3, -0.2, 0.1, 0.4])
    phi = th.sum()
    ob = np.array([0.4, -0.6])
    c0 = orc.camera(md, _state(th, ob), fp64=True)
    e1 = np.array([math.cos(phi), math.sin(phi)])
    c1 = orc.camera(md, _state(th, ob + 0.3 * e1), fp64=True)
    np.testing.assert_allclose(c1 - c0, [0.3, 0.0], atol=1e-12)


def test_sample_zero_noise_is_closed_form(orc, W):
    # sigma = 0 -> theta' = theta + h_s u, x' = x + h_s v_x, v' = v  (motion model)
    md = orc.Model(n_joints=5, sigma_theta=0.0, sigma_pos=0.0, sigma_vel=0.0)
    tr = W.make_trajectory(5, 10, 0)
    s = W.random_particles(tr, 300, 0)
    u = tr["U"][0]
    out, _ = orc.sample_weight(md, 3, s, tr["Z"][1], u, 1)
    hs = np.float32(0.1)
    exp = s.copy()
    exp[:5] = s[:5] + hs * u[:, None]
    exp[5] = s[5] + hs * s[7]
    exp[6] = s[6] + hs * s[8]
    np.testing.assert_array_equal(out[:5], exp[:5])
    np.testing.assert_allclose(out[5:7], exp[5:7], rtol=0, atol=1e-6)   # fma vs mul+add
    np.testing.assert_array_equal(out[7:], s[7:])


def test_sample_noise_layout(orc, W):
    # (x' - deterministic part)/sigma equals the Box–Muller normals of the
    # Philox words 2.. of counter (p, k, 0, j), in state order (R12, R13, F8)
    md = orc.Model(n_joints=5, sigma_theta=0.1, sigma_pos=0.2, sigma_vel=0.3)
    tr = W.make_trajectory(5, 10, 0)
    s = W.random_particles(tr, 40, 1).astype(np.float64)
    u = tr["U"][2].astype(np.float64)
    k, seed, off = 3, (7 << 32) | 9, 1000
    out, _ = orc.sample_weight(md, seed, s, tr["Z"][3], u, k, p_offset=off, fp64=True)
    det = s.copy()
    det[:5] = s[:5] + 0.1 * u[:, None].astype(np.float32).astype(np.float64)
    det[5] += np.float64(np.float32(0.1)) * s[7]
    det[6] += np.float64(np.float32(0.1)) * s[8]
    sig = np.array([0.1] * 5 + [0.2, 0.2, 0.3, 0.3], np.float32).astype(np.float64)
    xi = (out - det) / sig[:, None]
    for p in range(40):
        w = []
        for j in range(3):
            w += list(orc.philox([off + p, k, 0, j], [9, 7]))
        ref = []
        for q in range(5):
            x0, x1 = int(w[2 + 2 * q]), int(w[3 + 2 * q])
            u1 = 1 - ((x0 >> 9) + 0.5) * 2.0**-23
            u2 = (x1 >> 9) * 2.0**-23
            r = math.sqrt(-2 * math.log(u1))
            ref += [r * math.cos(2 * math.pi * u2), r * math.sin(2 * math.pi * u2)]
        np.testing.assert_allclose(xi[:, p], ref[:9], atol=1e-6)


def test_sample_weight_fp32_vs_fp64(orc, W):
    md = orc.Model(n_joints=28)
    tr = W.make_trajectory(28, 10, 0)
    s = W.random_particles(tr, 500, 2)
    o32, w32 = orc.sample_weight(md, 5, s, tr["Z"][1], tr["U"][0], 1)
    o64, w64 = orc.sample_weight(md, 5, s, tr["Z"][1], tr["U"][0], 1, fp64=True)
    np.testing.assert_allclose(o32, o64, rtol=1e-5, atol=1e-5)
    np.testing.assert_allclose(w32, w64, rtol=2e-5, atol=1e-4)
