// pf_model.cuh — model hooks of the particle filter (sm_100a).
//
// "Our application separates generic particle filtering from model-specific
// routines.  New dynamical system models can be easily added" (PAPER.md:10
// §I).  The generic step kernel (pf_kernels.cuh) is a template over a Model
// policy type; a model supplies, as compile-time hooks (no device function
// pointers, which would block fusion):
//
//   D, ZD, UD          state, measurement and control dimensions
//   Acc, Acc2          per-particle accumulator of the streamed weight
//                      (scalar / packed pair)
//   take<c>(...)       F8: component c (compile-time, increasing) of the new
//                      particle drawn from p(x_k | x_{k-1}) with the normal xi,
//                      folded into the accumulator at once (streamed weight)
//   finish(...)        F10: log p(z_k | x_k) from the accumulator
//   take2 / finish2    the same on two particles (packed f32x2, bit-identical)
//   CHUNKED, NC,
//   joint / joint2     optional: a runtime loop over chunks of four identical
//                      components (instruction-cache economy for large D)
//
// Constants (ModelConsts) are fp32 values the host derives from
// pf_model_params once per filter; each model documents which fields it uses.
// The control input enters as hs_u[i] = h_s u_i (one fp32 product, F8).
// Written from DESIGN.md §4 independently of oracle/.
#pragma once
#include <cstdint>

#include "pf_device.cuh"

#ifndef PF_CHUNK_MIN_D
#define PF_CHUNK_MIN_D 16
#endif

namespace pf {

enum : int { MODEL_ARM_PLANAR = 0, MODEL_LINEAR_GAUSS_1D = 1 };

// fp32 model constants (meaning per model, see each model)
struct ModelConsts {
  float lj;        // arm: link length L / n_joints
  float hs;        // sampling time h_s (every model: control term h_s u)
  float s_th, s_pos, s_vel;   // process-noise std
  float inv_cam, inv_thm;     // 1 / measurement-noise std
};
// the same with every field duplicated (packed f32x2 operands)
struct ModelConsts2 {
  f2 lj, hs, s_th, s_pos, s_vel, inv_cam, inv_thm;
};

// ------------------------------------------------------------ robotic arm ---
// PAPER.md:22–24 §VII-A; readings R14–R16.  State x = (theta_0..theta_{NJ-1},
// x, y, v_x, v_y), measurement z = (x_C, y_C, theta_hat_0..NJ-1), control
// u = joint velocities.  Uses every ModelConsts field.
struct ArmAcc {
  float phi = 0.0f, px = 0.0f, py = 0.0f, s = 0.0f, c = 1.0f, acc = 0.0f, xn = 0.0f, yn = 0.0f;
};
struct ArmAcc2 {
  f2 phi = 0ull, px = 0ull, py = 0ull, s = 0ull, c = 0ull, acc = 0ull, xn = 0ull, yn = 0ull;
};

template <int NJ_>
struct ArmPlanar {
  static constexpr int kId = MODEL_ARM_PLANAR;
  static constexpr int NJ = NJ_;
  static constexpr int D = NJ + 4, ZD = NJ + 2, UD = NJ;
  static constexpr bool RUNTIME = false;   // dimensions fixed at compile time
  // large states (the high-DOF arm): the joint chain runs as a loop over
  // chunks of four joints instead of being unrolled d times, so the
  // per-particle code fits the instruction cache (ncu: no_instruction stalls)
  static constexpr bool CHUNKED = D > PF_CHUNK_MIN_D;
  static constexpr int NC = NJ >= 6 ? (NJ - 2) / 4 : 0;   // chunks of four joints 2 + 4i .. 5 + 4i
  using Acc = ArmAcc;
  using Acc2 = ArmAcc2;

  // F8 + F9 + F10 streamed: component c of the new particle is sampled and
  // immediately folded into the forward kinematics and the log-likelihood,
  // so no state vector stays live.  x(c') reads component c' of the ancestor.
  template <int c, typename X>
  __device__ __forceinline__ static float take(const ModelConsts& mc, const float* hs_u, const float* z, const X& x,
                                               float xi, Acc& A) {
    if constexpr (c < NJ) {
      const float th = __fmaf_rn(mc.s_th, xi, x(c) + hs_u[c]);
      A.phi = A.phi + th;                               // F9
      sincos_c(A.phi, A.s, A.c);
      A.px = __fmaf_rn(mc.lj, A.c, A.px);
      A.py = __fmaf_rn(mc.lj, A.s, A.py);
      const float r = (z[2 + c] - th) * mc.inv_thm;     // F10, joint residuals first
      A.acc = (c == 0) ? r * r : __fmaf_rn(r, r, A.acc);
      return th;
    } else if constexpr (c == NJ) {
      A.xn = __fmaf_rn(mc.s_pos, xi, __fmaf_rn(mc.hs, x(NJ + 2), x(NJ)));
      return A.xn;
    } else if constexpr (c == NJ + 1) {
      A.yn = __fmaf_rn(mc.s_pos, xi, __fmaf_rn(mc.hs, x(NJ + 3), x(NJ + 1)));
      return A.yn;
    } else {
      return __fmaf_rn(mc.s_vel, xi, x(c));
    }
  }
  // F9 camera frame + F10 camera residuals
  __device__ __forceinline__ static float finish(const ModelConsts& mc, const float* z, const Acc& A) {
    const float dx = A.xn - A.px;
    const float dy = A.yn - A.py;
    const float sdy = A.s * dy;
    const float sdx = A.s * dx;
    const float xc = __fmaf_rn(A.c, dx, sdy);
    const float yc = __fmaf_rn(A.c, dy, -sdx);
    const float r0 = (z[0] - xc) * mc.inv_cam;
    const float r1 = (z[1] - yc) * mc.inv_cam;
    float acc = __fmaf_rn(r0, r0, A.acc);
    acc = __fmaf_rn(r1, r1, acc);
    return -0.5f * acc;
  }
  // joint c >= 2 of the chunked loop (runtime index): as take<c> for c < NJ
  template <typename X>
  __device__ __forceinline__ static float joint(int c, const ModelConsts& mc, const float* hsu, const float* z,
                                                const X& x, float xi, Acc& A) {
    const float th = __fmaf_rn(mc.s_th, xi, x(c) + hsu[c]);
    A.phi = A.phi + th;
    sincos_c(A.phi, A.s, A.c);
    A.px = __fmaf_rn(mc.lj, A.c, A.px);
    A.py = __fmaf_rn(mc.lj, A.s, A.py);
    const float r = (z[2 + c] - th) * mc.inv_thm;
    A.acc = __fmaf_rn(r, r, A.acc);   // c >= 2: never the first joint
    return th;
  }

  // The same on a pair of particles (packed, bit-identical to the above);
  // z2[i] = (z_i, z_i), hs_u2[c] = (h_s u_c, h_s u_c).
  template <int c, typename X>
  __device__ __forceinline__ static f2 take2(const ModelConsts2& mc, const f2* hs_u2, const f2* z2, const X& x, f2 xi,
                                             Acc2& A) {
    if constexpr (c < NJ) {
      const f2 th = fma2(mc.s_th, xi, add2(x(c), hs_u2[c]));
      A.phi = add2(A.phi, th);
      sincos_c2(A.phi, A.s, A.c);
      A.px = fma2(mc.lj, A.c, A.px);
      A.py = fma2(mc.lj, A.s, A.py);
      const f2 r = mul2(sub2(z2[2 + c], th), mc.inv_thm);
      A.acc = (c == 0) ? mul2(r, r) : fma2(r, r, A.acc);
      return th;
    } else if constexpr (c == NJ) {
      A.xn = fma2(mc.s_pos, xi, fma2(mc.hs, x(NJ + 2), x(NJ)));
      return A.xn;
    } else if constexpr (c == NJ + 1) {
      A.yn = fma2(mc.s_pos, xi, fma2(mc.hs, x(NJ + 3), x(NJ + 1)));
      return A.yn;
    } else {
      return fma2(mc.s_vel, xi, x(c));
    }
  }
  // -(s dx) = s (p_x - x_n) exactly
  __device__ __forceinline__ static f2 finish2(const ModelConsts2& mc, const f2* z2, const Acc2& A) {
    const f2 dx = sub2(A.xn, A.px);
    const f2 dy = sub2(A.yn, A.py);
    const f2 xc = fma2(A.c, dx, mul2(A.s, dy));
    const f2 yc = fma2(A.c, dy, mul2(A.s, sub2(A.px, A.xn)));
    const f2 r0 = mul2(sub2(z2[0], xc), mc.inv_cam);
    const f2 r1 = mul2(sub2(z2[1], yc), mc.inv_cam);
    return mul2(bc(-0.5f), fma2(r1, r1, fma2(r0, r0, A.acc)));
  }
  template <typename X>
  __device__ __forceinline__ static f2 joint2(int c, const ModelConsts2& mc, const f2* hsu2, const f2* z2, const X& x,
                                              f2 xi, Acc2& A) {
    const f2 th = fma2(mc.s_th, xi, add2(x(c), hsu2[c]));
    A.phi = add2(A.phi, th);
    sincos_c2(A.phi, A.s, A.c);
    A.px = fma2(mc.lj, A.c, A.px);
    A.py = fma2(mc.lj, A.s, A.py);
    const f2 r = mul2(sub2(z2[2 + c], th), mc.inv_thm);
    A.acc = fma2(r, r, A.acc);   // c >= 2
    return th;
  }
};

// --------------------------------------------- the generic (runtime) arm ---
// The arm for ANY n_joints <= NJMAX (the fallback behind the compiled
// instances n_j in {2, 5, 28}): the same F8–F10 arithmetic in the same order
// as ArmPlanar<n_j>, with the joint count a runtime value (take_rt / take_rt2,
// one component at a time; SampleRuntime(2) in pf_kernels.cuh pairs the
// normals), so its results are bit-identical to a compiled instance of that
// n_j.  The kernel's shared-memory stage is sized for NJMAX + 4 components
// (instantiated for NJMAX = 8, 16, 28: the smallest bucket that holds n_j is
// taken); the HBM block and mailbox entries use the runtime d.
template <int NJMAX_>
struct ArmDyn {
  static constexpr int kId = MODEL_ARM_PLANAR;
  static constexpr int NJ = NJMAX_;                      // (the largest supported)
  static constexpr int D = NJMAX_ + 4, ZD = NJMAX_ + 2, UD = NJMAX_;   // upper bounds
  static constexpr bool RUNTIME = true;
  static constexpr bool CHUNKED = false;
  static constexpr int NC = 0;
  using Acc = ArmAcc;
  using Acc2 = ArmAcc2;
  template <typename X>
  __device__ __forceinline__ static float take_rt(int c, int nj, const ModelConsts& mc, const float* hs_u, const float* z,
                                                  const X& x, float xi, Acc& A) {
    if (c < nj) {
      const float th = __fmaf_rn(mc.s_th, xi, x(c) + hs_u[c]);
      A.phi = A.phi + th;                               // F9
      sincos_c(A.phi, A.s, A.c);
      A.px = __fmaf_rn(mc.lj, A.c, A.px);
      A.py = __fmaf_rn(mc.lj, A.s, A.py);
      const float r = (z[2 + c] - th) * mc.inv_thm;     // F10, joint residuals first
      A.acc = (c == 0) ? r * r : __fmaf_rn(r, r, A.acc);
      return th;
    } else if (c == nj) {
      A.xn = __fmaf_rn(mc.s_pos, xi, __fmaf_rn(mc.hs, x(nj + 2), x(nj)));
      return A.xn;
    } else if (c == nj + 1) {
      A.yn = __fmaf_rn(mc.s_pos, xi, __fmaf_rn(mc.hs, x(nj + 3), x(nj + 1)));
      return A.yn;
    } else {
      return __fmaf_rn(mc.s_vel, xi, x(c));
    }
  }
  __device__ __forceinline__ static float finish(const ModelConsts& mc, const float* z, const Acc& A) {
    return ArmPlanar<1>::finish(mc, z, A);   // camera frame + residuals: independent of n_j
  }
  // the same on a pair of particles (packed, bit-identical lane by lane)
  template <typename X>
  __device__ __forceinline__ static f2 take_rt2(int c, int nj, const ModelConsts2& mc, const f2* hs_u2, const f2* z2,
                                                const X& x, f2 xi, Acc2& A) {
    if (c < nj) {
      const f2 th = fma2(mc.s_th, xi, add2(x(c), hs_u2[c]));
      A.phi = add2(A.phi, th);
      sincos_c2(A.phi, A.s, A.c);
      A.px = fma2(mc.lj, A.c, A.px);
      A.py = fma2(mc.lj, A.s, A.py);
      const f2 r = mul2(sub2(z2[2 + c], th), mc.inv_thm);
      A.acc = (c == 0) ? mul2(r, r) : fma2(r, r, A.acc);
      return th;
    } else if (c == nj) {
      A.xn = fma2(mc.s_pos, xi, fma2(mc.hs, x(nj + 2), x(nj)));
      return A.xn;
    } else if (c == nj + 1) {
      A.yn = fma2(mc.s_pos, xi, fma2(mc.hs, x(nj + 3), x(nj + 1)));
      return A.yn;
    } else {
      return fma2(mc.s_vel, xi, x(c));
    }
  }
  __device__ __forceinline__ static f2 finish2(const ModelConsts2& mc, const f2* z2, const Acc2& A) {
    return ArmPlanar<1>::finish2(mc, z2, A);
  }
};

// ------------------------------------------------- 1-D linear Gaussian ---
// The linear-Gaussian special case of SURVEY §8(c) whole-filter pin (ii): one
// joint of the arm with its angle sensor and no camera —
//   theta_k = theta_{k-1} + h_s u_{k-1} + w,  w ~ N(0, sigma_theta^2)   (F8 joint row)
//   z_k     = theta_k + v,                    v ~ N(0, sigma_theta_meas^2)
//   log p(z | theta) = -1/2 ((z - theta) / sigma_theta_meas)^2           (F10 joint term)
// for which the Kalman filter is the exact posterior (tests/).  Uses
// ModelConsts hs, s_th, inv_thm.  D = ZD = UD = 1.
struct LgAcc {
  float acc = 0.0f;
};
struct LgAcc2 {
  f2 acc = 0ull;
};
struct LinearGauss1D {
  static constexpr int kId = MODEL_LINEAR_GAUSS_1D;
  static constexpr int NJ = 1;   // (one "joint")
  static constexpr int D = 1, ZD = 1, UD = 1;
  static constexpr bool RUNTIME = false;
  static constexpr bool CHUNKED = false;
  static constexpr int NC = 0;
  using Acc = LgAcc;
  using Acc2 = LgAcc2;
  template <int c, typename X>
  __device__ __forceinline__ static float take(const ModelConsts& mc, const float* hs_u, const float* z, const X& x,
                                               float xi, Acc& A) {
    static_assert(c == 0, "one state component");
    const float th = __fmaf_rn(mc.s_th, xi, x(0) + hs_u[0]);
    const float r = (z[0] - th) * mc.inv_thm;
    A.acc = r * r;
    return th;
  }
  __device__ __forceinline__ static float finish(const ModelConsts&, const float*, const Acc& A) {
    return -0.5f * A.acc;
  }
  template <typename X>
  __device__ __forceinline__ static float joint(int, const ModelConsts&, const float*, const float*, const X&, float,
                                                Acc&) {
    return 0.0f;   // never used (CHUNKED = false)
  }
  template <int c, typename X>
  __device__ __forceinline__ static f2 take2(const ModelConsts2& mc, const f2* hs_u2, const f2* z2, const X& x, f2 xi,
                                             Acc2& A) {
    static_assert(c == 0, "one state component");
    const f2 th = fma2(mc.s_th, xi, add2(x(0), hs_u2[0]));
    const f2 r = mul2(sub2(z2[0], th), mc.inv_thm);
    A.acc = mul2(r, r);
    return th;
  }
  __device__ __forceinline__ static f2 finish2(const ModelConsts2&, const f2*, const Acc2& A) {
    return mul2(bc(-0.5f), A.acc);
  }
  template <typename X>
  __device__ __forceinline__ static f2 joint2(int, const ModelConsts2&, const f2*, const f2*, const X&, f2, Acc2&) {
    return 0ull;
  }
};

}  // namespace pf
