// pf_kernels.cuh — sm_100a kernels of the distributed particle filter.
//
// pf_step_kernel<NJ, M, RES> is the ROTATED STEP: launch k
// performs, for every sub-filter of this shard,
//   a6 exchange   merge the neighbours' best t of step k-1 (mailbox) into the
//                 own worst deg*t slots                  (Alg.2 l.10–14, R2–R5)
//   a7 normalise  q_i = floor(2^22 exp(l_i - l_max))     (§VI-F, R7–R8)
//   a8 resample   RWS (scan + binary search) or Vose (alias table, sweep
//                 closed form)                           (Alg.2 l.15–19, R9–R11)
//   a9 gather     ancestor state from shared memory      (§VI-F)
//   a1 RNG        Philox4x32-10 in registers             (R12, R13)
//   a2 sample, a3 weight (fused, §VI-B)      (F8–F10)
//   a4 local reduce: argmax / best t -> mailbox (k&1)    (Alg.2 l.8, replaces the sort)
//   a5 global estimate: u64 atomicMax + last-CTA copy    (Alg.2 l.9, R6)
//   a10 store state + log-weight (in place)
// so each launch streams the particle set through HBM once (read + write).
//
// Mapping: one CTA of M threads per sub-filter (one thread per particle, as
// the paper's one work-group per sub-filter, §VI), persistent
// grid-stride loop over the shard's sub-filters.  A sub-filter's d state
// rows and log-weight row (SoA, contiguous m floats each) are brought into
// shared memory by d+1 TMA bulk copies (cp.async.bulk + mbarrier); all
// reductions / scans are warp-shuffle / REDUX + one cross-warp level.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "pf_device.cuh"

namespace pf {

typedef unsigned long long u64;

enum : int { MODE_STEP = 0, MODE_PUBLISH = 1, MODE_EXCHANGE = 2, MODE_SAMPLE = 3 };
enum : int { TOPO_NONE = 0, TOPO_RING = 1, TOPO_TORUS = 2 };
enum : int { RES_RWS = 0, RES_VOSE = 1 };

struct StepParams {
  ArmConsts mc;
  float* state;            // [d][stride]
  float* logw;             // [stride]
  long long stride;        // M_local
  const float* mb_prev;    // mailbox parity (k-1)&1 : [n_ext][tt][E]
  float* mb_cur;           // mailbox parity k&1
  const float* z;          // [NJ+2] device
  const float* u;          // [NJ]   device
  u64* key_cur;            // global best key of this step (0 on entry)
  u64* key_next;           // reset to 0 for the next step
  unsigned int* counter;   // CTA completion counter (0 on entry, reset by the last CTA)
  float* record;           // [4 + d] estimate record of this shard
  float* est_out;          // nullable [4 + d] (batched mode)
  long long* dbg_src;      // nullable [M_local] exchange sources (global index)
  int* dbg_anc;            // nullable [M_local] ancestors
  long long n_local, g0, n_global, R, C;
  int t, tt, topo, deg;
  uint32_t key0, key1, k;
  int mode, first;
};

// ------------------------------------------------------------- PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(u64* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(u64* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, u64* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(u64* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "PF_WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra PF_WAIT_%=;\n}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

// ------------------------------------------------------ block primitives
// All take the two-slot reduction buffer `red` ([2][32] u64) and a uniform
// buffer toggle; every call with NW > 1 contains one __syncthreads, which
// makes a slot reusable two calls later.
template <int NW>
__device__ __forceinline__ u64 block_max_u64(u64 v, u64* red, int& rb) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint32_t hi = __reduce_max_sync(0xFFFFFFFFu, static_cast<uint32_t>(v >> 32));
  uint32_t lo = __reduce_max_sync(0xFFFFFFFFu, (static_cast<uint32_t>(v >> 32) == hi) ? static_cast<uint32_t>(v) : 0u);
  if (NW == 1) return (static_cast<u64>(hi) << 32) | lo;
  u64* r = red + rb * 32;
  rb ^= 1;
  if (lane == 0) r[warp] = (static_cast<u64>(hi) << 32) | lo;
  __syncthreads();
  const u64 w = lane < NW ? r[lane] : 0ull;
  hi = __reduce_max_sync(0xFFFFFFFFu, static_cast<uint32_t>(w >> 32));
  lo = __reduce_max_sync(0xFFFFFFFFu, (static_cast<uint32_t>(w >> 32) == hi) ? static_cast<uint32_t>(w) : 0u);
  return (static_cast<u64>(hi) << 32) | lo;
}

template <int NW>
__device__ __forceinline__ u64 block_min_u64(u64 v, u64* red, int& rb) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint32_t hi = __reduce_min_sync(0xFFFFFFFFu, static_cast<uint32_t>(v >> 32));
  uint32_t lo = __reduce_min_sync(0xFFFFFFFFu,
                                  (static_cast<uint32_t>(v >> 32) == hi) ? static_cast<uint32_t>(v) : 0xFFFFFFFFu);
  if (NW == 1) return (static_cast<u64>(hi) << 32) | lo;
  u64* r = red + rb * 32;
  rb ^= 1;
  if (lane == 0) r[warp] = (static_cast<u64>(hi) << 32) | lo;
  __syncthreads();
  const u64 w = lane < NW ? r[lane] : ~0ull;
  hi = __reduce_min_sync(0xFFFFFFFFu, static_cast<uint32_t>(w >> 32));
  lo = __reduce_min_sync(0xFFFFFFFFu,
                         (static_cast<uint32_t>(w >> 32) == hi) ? static_cast<uint32_t>(w) : 0xFFFFFFFFu);
  return (static_cast<u64>(hi) << 32) | lo;
}

template <int NW>
__device__ __forceinline__ uint32_t block_max_u32(uint32_t v, u64* red, int& rb) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint32_t m = __reduce_max_sync(0xFFFFFFFFu, v);
  if (NW == 1) return m;
  u64* r = red + rb * 32;
  rb ^= 1;
  if (lane == 0) r[warp] = m;
  __syncthreads();
  return __reduce_max_sync(0xFFFFFFFFu, lane < NW ? static_cast<uint32_t>(r[lane]) : 0u);
}

__device__ __forceinline__ u64 warp_incl_scan_u64(u64 x) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const u64 y = __shfl_up_sync(0xFFFFFFFFu, x, o);
    if (lane >= o) x += y;
  }
  return x;
}

// Exclusive prefix sum over threads in tid order; `total` = block sum.
template <int NW>
__device__ __forceinline__ u64 block_excl_scan_u64(u64 v, u64* red, int& rb, u64& total) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const u64 x = warp_incl_scan_u64(v);
  if (NW == 1) {
    total = __shfl_sync(0xFFFFFFFFu, x, 31);
    return x - v;
  }
  u64* r = red + rb * 32;
  rb ^= 1;
  if (lane == 31) r[warp] = x;
  __syncthreads();
  const u64 wt = warp_incl_scan_u64(lane < NW ? r[lane] : 0ull);
  const u64 off = __shfl_sync(0xFFFFFFFFu, wt, (warp + 31) & 31);
  total = __shfl_sync(0xFFFFFFFFu, wt, NW - 1);
  return (warp > 0 ? off : 0ull) + x - v;
}

// first index i in [0, n) with a[i] >= x (n if none)
__device__ __forceinline__ int lower_bound_u64(const u64* a, int n, u64 x) {
  int lo = 0;
  while (n > 0) {
    const int half = n >> 1;
    if (a[lo + half] < x) {
      lo += half + 1;
      n -= half + 1;
    } else {
      n = half;
    }
  }
  return lo;
}
// first index i in [0, n) with a[i] > x (n if none)
__device__ __forceinline__ int upper_bound_u64(const u64* a, int n, u64 x) {
  int lo = 0;
  while (n > 0) {
    const int half = n >> 1;
    if (a[lo + half] <= x) {
      lo += half + 1;
      n -= half + 1;
    } else {
      n = half;
    }
  }
  return lo;
}

// ---------------------------------------------------------- resampling
// Shared-memory scratch of the resampler (RWS uses only `scan`).
struct ResampleSmem {
  u64* scan;    // [M] RWS: inclusive sums C; Vose: D over L, then E over H
  u64* prob;    // [M] Vose
  int* alias;   // [M] Vose
  int* lists;   // [M] Vose: L ascending then H ascending
};

// Ancestor of slot `tid` (a8) from its integer weight q (a7) and uniforms.
// Every thread of the CTA must call it (barriers inside).
template <int M, int RES>
__device__ __forceinline__ int resample_slot(uint32_t q, uint32_t Ua, uint32_t Ub, const ResampleSmem& S,
                                             u64* red, int& rb, u64* prob_out, int* alias_out) {
  constexpr int NW = M / 32;
  const int tid = threadIdx.x;
  u64 Q;
  const u64 excl = block_excl_scan_u64<NW>(q, red, rb, Q);
  if (RES == RES_RWS) {
    // Roulette Wheel Selection (§VI-F): inclusive sums C, draw
    // c = floor(U Q / 2^32), ancestor = first j with C_j > c (R9).
    S.scan[tid] = excl + q;
    __syncthreads();
    const u64 c = (static_cast<u64>(Ua) * Q) >> 32;
    int pos = 0;
#pragma unroll
    for (int s = M / 2; s >= 1; s >>= 1)
      if (S.scan[pos + s - 1] <= c) pos += s;
    return pos;
  } else {
    // Vose's alias method (PAPER.md:18 §IV, :20–22 §VI-F), table by the
    // closed form of the sequential sweep (R10): a_j = M q_j, small L = {a < Q},
    // D = inclusive deficits over L, E = inclusive excesses over H.
    const u64 a = static_cast<u64>(M) * q;
    const bool small = a < Q;
    u64 nL, Dtot, Etot;
    const uint32_t ls = static_cast<uint32_t>(block_excl_scan_u64<NW>(small ? 1ull : 0ull, red, rb, nL));
    const u64 def = small ? Q - a : 0ull;
    const u64 exc = small ? 0ull : a - Q;
    const u64 Dincl = block_excl_scan_u64<NW>(def, red, rb, Dtot) + def;
    const u64 Eincl = block_excl_scan_u64<NW>(exc, red, rb, Etot) + exc;
    const int nl = static_cast<int>(nL);
    const int h = tid - static_cast<int>(ls);
    if (small) {
      S.lists[ls] = tid;
      S.scan[ls] = Dincl;
    } else {
      S.lists[nl + h] = tid;
      S.scan[nl + h] = Eincl;
    }
    __syncthreads();
    u64 pr;
    int al;
    if (small) {
      pr = a;
      const int hh = lower_bound_u64(S.scan + nl, M - nl, Dincl - def);
      al = S.lists[nl + hh];
    } else if (Eincl < Dtot) {
      const int ii = upper_bound_u64(S.scan, nl, Eincl);
      pr = Q + Eincl - S.scan[ii];
      al = S.lists[nl + h + 1];
    } else {
      pr = Q;
      al = tid;
    }
    S.prob[tid] = pr;
    S.alias[tid] = al;
    if (prob_out) {
      prob_out[tid] = pr;
      alias_out[tid] = al;
    }
    __syncthreads();
    const int b = static_cast<int>((static_cast<u64>(Ua) * M) >> 32);
    const u64 c = (static_cast<u64>(Ub) * Q) >> 32;
    return c < S.prob[b] ? b : S.alias[b];
  }
}

// ------------------------------------------------------------ topology
__device__ __forceinline__ long long neighbor_of(const StepParams& P, long long g, int qi) {
  if (P.topo == TOPO_RING) return qi == 0 ? (g - 1 + P.n_global) % P.n_global : (g + 1) % P.n_global;
  const long long r = g / P.C, c = g % P.C;
  switch (qi) {
    case 0: return ((r - 1 + P.R) % P.R) * P.C + c;
    case 1: return ((r + 1) % P.R) * P.C + c;
    case 2: return r * P.C + (c - 1 + P.C) % P.C;
    default: return r * P.C + (c + 1) % P.C;
  }
}
// mailbox row of global sub-filter q: local rows, then halo rows (pf.h pf_shard)
__device__ __forceinline__ long long mailbox_row(const StepParams& P, long long q) {
  const long long loc = q - P.g0;
  if (loc >= 0 && loc < P.n_local) return loc;
  if (P.topo == TOPO_RING) return q == (P.g0 - 1 + P.n_global) % P.n_global ? P.n_local : P.n_local + 1;
  const long long rq = q / P.C, cq = q % P.C, r0 = P.g0 / P.C;
  return rq == (r0 - 1 + P.R) % P.R ? P.n_local + cq : P.n_local + P.C + cq;
}

// ---------------------------------------------------------- smem layout
template <int NJ, int M, int RES>
struct StepSmem {
  static constexpr int D = NJ + 4;
  static constexpr size_t xs = 0;                                  // float [D][M]
  static constexpr size_t ws = xs + sizeof(float) * D * M;         // float [M]
  static constexpr size_t scan = ws + sizeof(float) * M;           // u64 [M]
  static constexpr size_t prob = scan + sizeof(u64) * M;           // u64 [M]   (Vose)
  static constexpr size_t alias = prob + (RES == RES_VOSE ? sizeof(u64) * M : 0);
  static constexpr size_t lists = alias + (RES == RES_VOSE ? sizeof(int) * M : 0);
  static constexpr size_t red = lists + (RES == RES_VOSE ? sizeof(int) * M : 0);   // u64 [2][32]
  static constexpr size_t misc = red + sizeof(u64) * 64;          // int [128]
  static constexpr size_t zin = misc + sizeof(int) * 128;         // float [64]: z (NJ+2), h_s u (NJ)
  static constexpr size_t bar = zin + sizeof(float) * 64;         // mbarrier
  static constexpr size_t bytes = bar + 16;
};

// ------------------------------------------------------------ the kernel
template <int NJ, int M, int RES>
__global__ void __launch_bounds__(M) pf_step_kernel(const __grid_constant__ StepParams P) {
  constexpr int D = NJ + 4;
  constexpr int E = D + 2;   // mailbox entry: [logw, index bits, x_0..x_{D-1}]
  constexpr int NW = M / 32;
  using L = StepSmem<NJ, M, RES>;
  extern __shared__ __align__(128) unsigned char smem[];
  float* xs = reinterpret_cast<float*>(smem + L::xs);
  float* ws = reinterpret_cast<float*>(smem + L::ws);
  u64* red = reinterpret_cast<u64*>(smem + L::red);
  int* misc = reinterpret_cast<int*>(smem + L::misc);
  float* z_s = reinterpret_cast<float*>(smem + L::zin);
  float* hsu_s = z_s + NJ + 2;
  u64* bar = reinterpret_cast<u64*>(smem + L::bar);
  ResampleSmem S;
  S.scan = reinterpret_cast<u64*>(smem + L::scan);
  S.prob = reinterpret_cast<u64*>(smem + L::prob);
  S.alias = reinterpret_cast<int*>(smem + L::alias);
  S.lists = reinterpret_cast<int*>(smem + L::lists);

  const int tid = threadIdx.x;
  const int mode = P.mode;
  const bool do_merge = (mode == MODE_EXCHANGE) || (mode == MODE_STEP && !P.first);
  const bool do_resample = (mode == MODE_STEP && !P.first);
  const bool do_sample = (mode == MODE_STEP || mode == MODE_SAMPLE);
  const int K = P.deg * P.t;

  if (tid == 0) {
    mbar_init(bar, 1);
    fence_mbar_init();
  }
  if (do_sample) {
    if (tid < NJ + 2) z_s[tid] = P.z[tid];
    if (tid < NJ) hsu_s[tid] = P.mc.hs * P.u[tid];
  }
  __syncthreads();

  int rb = 0;
  uint32_t parity = 0;
  for (long long n = blockIdx.x; n < P.n_local; n += gridDim.x) {
    const long long g = P.g0 + n;
    const uint32_t pbase = static_cast<uint32_t>(g * M);
    const uint32_t pidx = pbase + tid;
    // ---- load the sub-filter's D state rows + log-weight row (TMA bulk)
    if (tid == 0) {
      mbar_arrive_expect_tx(bar, (D + 1) * M * sizeof(float));
#pragma unroll 1
      for (int c = 0; c < D; ++c) bulk_g2s(xs + c * M, P.state + c * P.stride + n * M, M * sizeof(float), bar);
      bulk_g2s(ws, P.logw + n * M, M * sizeof(float), bar);
    }
    mbar_wait(bar, parity);
    parity ^= 1;

    // ---- a6 exchange: neighbours' best t (mailbox of step k-1) overwrite
    //      the own deg*t worst slots (R2–R5)
    if (do_merge && K > 0) {
      u64 mk = order_key(ws[tid], static_cast<uint32_t>(tid));
#pragma unroll 1
      for (int j = 0; j < K; ++j) {
        const u64 wk = block_min_u64<NW>(mk, red, rb);
        const int slot = static_cast<int>(0xFFFFFFFFu - static_cast<uint32_t>(wk));
        if (slot == tid) mk = ~0ull;
        if (tid == 0) misc[j] = slot;
      }
      __syncthreads();
#pragma unroll 1
      for (int e = tid; e < K * E; e += M) {
        const int j = e / E, c = e - j * E;
        const int qi = j / P.t, jj = j - qi * P.t;
        const long long row = mailbox_row(P, neighbor_of(P, g, qi));
        const float v = P.mb_prev[(row * P.tt + jj) * E + c];
        const int slot = misc[j];
        if (c == 0) ws[slot] = v;
        else if (c >= 2) xs[(c - 2) * M + slot] = v;
      }
      if (P.dbg_src) {
        long long src = pidx;
#pragma unroll 1
        for (int j = 0; j < K; ++j)
          if (misc[j] == tid) {
            const int qi = j / P.t, jj = j - qi * P.t;
            const long long row = mailbox_row(P, neighbor_of(P, g, qi));
            src = __float_as_uint(P.mb_prev[(row * P.tt + jj) * E + 1]);
          }
        P.dbg_src[n * M + tid] = src;
      }
      __syncthreads();
    } else if ((do_merge || mode == MODE_STEP) && P.dbg_src) {
      P.dbg_src[n * M + tid] = pidx;   // no exchange (k = 1 or deg*t = 0): identity
    }

    if (mode == MODE_EXCHANGE) {
      fence_proxy_async_smem();
      __syncthreads();
      continue;
    }

    // ---- a7 normalise + a8 resample (slot order, R11)
    int anc = tid;
    u32x4 b0;
    bool have_b0 = false;
    if (do_resample) {
      const float lw = ws[tid];
      const uint32_t lmax_o = block_max_u32<NW>(ord_f32(lw), red, rb);
      const uint32_t q = expq_c(lw - unord_f32(lmax_o));
      b0 = philox4x32_10(pidx, P.k, 0u, 0u, P.key0, P.key1);
      have_b0 = true;
      anc = resample_slot<M, RES>(q, b0.x, b0.y, S, red, rb, nullptr, nullptr);
      if (P.dbg_anc) P.dbg_anc[n * M + tid] = anc;
    } else if (mode == MODE_STEP && P.dbg_anc) {
      P.dbg_anc[n * M + tid] = tid;
    }

    float lnew;
    float xo[D];
    if (do_sample) {
      // ---- a9 gather + a1 RNG + a2 sample + a3 weight
      float xin[D], xi[D];
#pragma unroll
      for (int c = 0; c < D; ++c) xin[c] = xs[c * M + anc];
      if (!have_b0) b0 = philox4x32_10(pidx, P.k, 0u, 0u, P.key0, P.key1);
      u32x4 blk = b0;
#pragma unroll
      for (int qp = 0; qp < (D + 1) / 2; ++qp) {
        const int w = 2 + 2 * qp;
        if ((w & 3) == 0) blk = philox4x32_10(pidx, P.k, 0u, static_cast<uint32_t>(w >> 2), P.key0, P.key1);
        const uint32_t x0 = (w & 3) == 2 ? blk.z : blk.x;
        const uint32_t x1 = (w & 3) == 2 ? blk.w : blk.y;
        float z0, z1;
        normal_pair(x0, x1, z0, z1);
        xi[2 * qp] = z0;
        if (2 * qp + 1 < D) xi[2 * qp + 1] = z1;
      }
      arm_sample<NJ>(P.mc, hsu_s, xin, xi, xo);
      lnew = arm_loglik<NJ>(P.mc, z_s, xo);
      // ---- a10 store (coalesced: consecutive threads, consecutive columns)
#pragma unroll
      for (int c = 0; c < D; ++c) P.state[c * P.stride + n * M + tid] = xo[c];
      P.logw[n * M + tid] = lnew;
    } else {   // MODE_PUBLISH: the loaded set is the step's weighted set
      lnew = ws[tid];
#pragma unroll
      for (int c = 0; c < D; ++c) xo[c] = xs[c * M + tid];
    }

    // ---- a4 local reduce: best t -> mailbox (k&1); a5 global best key
    u64 key = order_key(lnew, pidx);
    const int nbest = P.t > 0 ? P.t : 1;
#pragma unroll 1
    for (int j = 0; j < nbest; ++j) {
      const u64 best = block_max_u64<NW>(key, red, rb);
      if (best == key) {   // unique owner (index is part of the key)
        if (j < P.t) {
          float* e = P.mb_cur + (n * P.tt + j) * E;
          e[0] = lnew;
          e[1] = __uint_as_float(pidx);
#pragma unroll
          for (int c = 0; c < D; ++c) e[2 + c] = xo[c];
        }
        if (j == 0) atomicMax(P.key_cur, best);
        key = 0ull;
      }
    }
    fence_proxy_async_smem();
    __syncthreads();
  }

  // ---- a5: the last CTA to finish copies the winning particle (R6)
  __shared__ unsigned int s_last;
  if (tid == 0) {
    __threadfence();
    const unsigned int prev = atomicAdd(P.counter, 1u);
    s_last = (prev == gridDim.x - 1) ? 1u : 0u;
  }
  __syncthreads();
  if (s_last) {
    __threadfence();
    if (mode != MODE_EXCHANGE) {
      const u64 key = __ldcg(P.key_cur);
      const uint32_t gidx = 0xFFFFFFFFu - static_cast<uint32_t>(key);
      const long long col = static_cast<long long>(gidx) - P.g0 * M;
      if (tid < D) {
        const float v = __ldcg(P.state + tid * P.stride + col);
        P.record[4 + tid] = v;
        if (P.est_out) P.est_out[4 + tid] = v;
      }
      if (tid == 0) {
        const float r0 = __uint_as_float(static_cast<uint32_t>(key));
        const float r1 = __uint_as_float(static_cast<uint32_t>(key >> 32));
        const float r2 = unord_f32(static_cast<uint32_t>(key >> 32));
        P.record[0] = r0;
        P.record[1] = r1;
        P.record[2] = r2;
        P.record[3] = 0.0f;
        if (P.est_out) {
          P.est_out[0] = r0;
          P.est_out[1] = r1;
          P.est_out[2] = r2;
          P.est_out[3] = 0.0f;
        }
      }
    }
    if (tid == 0) {
      *P.key_next = 0ull;
      *P.counter = 0u;
    }
  }
}

// Resampling test hook: one CTA per row of integer weights, explicit uniforms.
template <int M, int RES>
__global__ void __launch_bounds__(M) pf_resample_debug_kernel(const uint32_t* __restrict__ q,
                                                              const uint32_t* __restrict__ ua,
                                                              const uint32_t* __restrict__ ub, int* anc,
                                                              u64* prob, int* alias, long long N) {
  __shared__ u64 scan[M];
  __shared__ u64 pr[RES == RES_VOSE ? M : 1];
  __shared__ int al[RES == RES_VOSE ? M : 1];
  __shared__ int lists[RES == RES_VOSE ? M : 1];
  __shared__ u64 red[64];
  ResampleSmem S{scan, pr, al, lists};
  int rb = 0;
  for (long long n = blockIdx.x; n < N; n += gridDim.x) {
    const long long i = n * M + threadIdx.x;
    const int a = resample_slot<M, RES>(q[i], ua[i], ub[i], S, red, rb, prob ? prob + n * M : nullptr,
                                        alias ? alias + n * M : nullptr);
    anc[i] = a;
    __syncthreads();
  }
}

// Host-side launch helpers (one explicit instantiation set per n_joints TU).
template <int NJ, int M, int RES>
struct StepKernel {
  static constexpr size_t smem() { return StepSmem<NJ, M, RES>::bytes; }
  static cudaError_t prepare(int* blocks_per_sm) {
    cudaError_t e = cudaFuncSetAttribute(pf_step_kernel<NJ, M, RES>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         static_cast<int>(smem()));
    if (e != cudaSuccess) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, pf_step_kernel<NJ, M, RES>, M, smem());
  }
  static cudaError_t launch(const StepParams& p, int grid, cudaStream_t s) {
    pf_step_kernel<NJ, M, RES><<<grid, M, smem(), s>>>(p);
    return cudaGetLastError();
  }
};

}  // namespace pf
