// pf_central.cu — the centralized particle filter on the whole GPU (SURVEY.md
// NEXT-2): ONE filter of M > 1024 particles, resampled globally — the paper's
// reference scheme ("a sequential, centralized particle filter", PAPER.md:18
// §VI; Fig.5 and Fig.9).  Same arithmetic contract, counter
// layout and log-weight semantics as the distributed step (a1–a3, a5, a7–a10);
// no exchange.  Three launches per step (k > 1):
//   cz_tile_scan  q_i = expq(l_i - l_max) (l_max = the previous step's best,
//                 from its estimate record) and per-tile inclusive u64 sums
//   cz_tile_prefix  inclusive prefix of the tile totals (one CTA), Q
//   cz_step       per particle: RWS draw (Philox (p, k, 0, 0) word 0, R9),
//                 two-level binary search (tiles, then inside the tile),
//                 gather from the previous buffer, sample + weight, store to
//                 the other buffer, block argmax + u64 atomicMax; the last CTA
//                 copies the winning particle to the estimate record.
// Particle buffers ping-pong: step k reads buffer (k-1)&1 and writes k&1.
#include <cuda_runtime.h>

#include <cstdint>

#include "pf_central.h"
#include "pf_kernels.cuh"

namespace pf {
namespace {

constexpr int kScanThreads = 256;
constexpr int kPerThread = kCentralTile / kScanThreads;   // 16 consecutive particles per thread

__device__ __forceinline__ u64 block_excl_scan(u64 v, u64* sm, u64& total) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const u64 x = warp_incl_scan<u64>(v, lane);
  if (lane == 31) sm[warp] = x;
  __syncthreads();
  const u64 wt = warp_incl_scan<u64>(lane < nw ? sm[lane] : 0ull, lane);
  const u64 off = __shfl_sync(0xFFFFFFFFu, wt, (warp + 31) & 31);
  total = __shfl_sync(0xFFFFFFFFu, wt, nw - 1);
  __syncthreads();
  return (warp > 0 ? off : 0ull) + x - v;
}

// a7: integer weights of one tile and their inclusive sums (u64).
__global__ void __launch_bounds__(kScanThreads) cz_tile_scan(const float* __restrict__ logw, const float* record,
                                                             u64* __restrict__ cl, u64* __restrict__ tile_sum) {
  __shared__ u64 sm[32];
  const float lmax = unord_f32(__float_as_uint(record[1]));   // ordered(l_max) is the key's high word
  const long long base = static_cast<long long>(blockIdx.x) * kCentralTile + threadIdx.x * kPerThread;
  u64 run[kPerThread];
  u64 acc = 0;
#pragma unroll
  for (int j = 0; j < kPerThread; j += 4) {
    const float4 w4 = *reinterpret_cast<const float4*>(logw + base + j);
    const float w[4] = {w4.x, w4.y, w4.z, w4.w};
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      acc += expq_c(w[e] - lmax);
      run[j + e] = acc;
    }
  }
  u64 total;
  const u64 off = block_excl_scan(acc, sm, total);
#pragma unroll
  for (int j = 0; j < kPerThread; ++j) cl[base + j] = off + run[j];
  if (threadIdx.x == 0) tile_sum[blockIdx.x] = total;
}

// Inclusive prefix of the tile totals (one CTA of 1024 threads).
__global__ void __launch_bounds__(1024) cz_tile_prefix(const u64* __restrict__ tile_sum, u64* __restrict__ tile_incl,
                                                       int tiles) {
  __shared__ u64 sm[32];
  const int per = (tiles + 1023) / 1024;
  const int b0 = threadIdx.x * per;
  u64 acc = 0;
  for (int j = 0; j < per; ++j)
    if (b0 + j < tiles) acc += tile_sum[b0 + j];
  u64 total;
  u64 run = block_excl_scan(acc, sm, total);
  for (int j = 0; j < per; ++j)
    if (b0 + j < tiles) {
      run += tile_sum[b0 + j];
      tile_incl[b0 + j] = run;
    }
}

// ---- Vose over all M slots (§VI-F; the sweep closed form of
// reading R10, device-wide): a_j = M q_j, small L = {a_j < Q} and large H
// (both ascending), D = inclusive deficits (Q - a) over L, E = inclusive
// excesses (a - Q) over H.  Three passes over the tiles + one prefix:
//   vz_class   per tile: small flags, inclusive small counts / deficits
//   (prefix)   tile totals -> inclusive prefixes
//   vz_lists   global list positions: L[ls] = j with D, H[j - ls] = j with E
//   vz_table   per slot: prob / alias by binary search in the other list
// q_j is recovered from the per-tile inclusive sums cl of cz_tile_scan.

__device__ __forceinline__ u64 q_of(const u64* __restrict__ cl, long long j) {
  return (j % kCentralTile) == 0 ? cl[j] : cl[j] - cl[j - 1];
}

// block inclusive scan of a (count, sum) pair: returns the exclusive offsets
__device__ __forceinline__ void block_excl_scan2(u64 c, u64 d, u64* sm, u64& oc, u64& od, u64& tc, u64& td) {
  oc = block_excl_scan(c, sm, tc);
  od = block_excl_scan(d, sm, td);
}

__global__ void __launch_bounds__(kScanThreads) vz_class(const CentralParams C) {
  __shared__ u64 sm[32];
  const long long M = C.M;
  const u64 Q = C.tile_incl[M / kCentralTile - 1];
  const long long base = static_cast<long long>(blockIdx.x) * kCentralTile + threadIdx.x * kPerThread;
  uint32_t rc[kPerThread];
  u64 rd[kPerThread];
  uint32_t cnt = 0;
  u64 dsum = 0;
#pragma unroll
  for (int j = 0; j < kPerThread; ++j) {
    const u64 a = static_cast<u64>(M) * q_of(C.cl, base + j);
    if (a < Q) {
      ++cnt;
      dsum += Q - a;
    }
    rc[j] = cnt;
    rd[j] = dsum;
  }
  u64 oc, od, tc, td;
  block_excl_scan2(cnt, dsum, sm, oc, od, tc, td);
#pragma unroll
  for (int j = 0; j < kPerThread; ++j) {
    C.cn[base + j] = static_cast<uint32_t>(oc) + rc[j];
    C.dl[base + j] = od + rd[j];
  }
  if (threadIdx.x == 0) {
    C.tile_cnt[blockIdx.x] = tc;
    C.tile_D[blockIdx.x] = td;
  }
}

struct VoseSlot {
  u64 a, def, Dinc, Einc;
  long long ls;   // small slots before j
  bool small;
};
__device__ __forceinline__ VoseSlot vose_slot(const CentralParams& C, long long j, u64 Q) {
  const long long M = C.M;
  const long long t = j / kCentralTile;
  VoseSlot v;
  const u64 q = q_of(C.cl, j);
  v.a = static_cast<u64>(M) * q;
  v.small = v.a < Q;
  v.def = v.small ? Q - v.a : 0ull;
  const u64 cnt_incl = (t > 0 ? C.tile_cnt_incl[t - 1] : 0ull) + C.cn[j];
  v.ls = static_cast<long long>(cnt_incl) - (v.small ? 1 : 0);
  v.Dinc = (t > 0 ? C.tile_D_incl[t - 1] : 0ull) + C.dl[j];
  const u64 Cinc = (t > 0 ? C.tile_incl[t - 1] : 0ull) + C.cl[j];
  // sum_{j' <= j} (a_j' - Q) = E_j - D_j  (wraps harmlessly in u64)
  v.Einc = v.Dinc + static_cast<u64>(M) * Cinc - static_cast<u64>(j + 1) * Q;
  return v;
}

__global__ void __launch_bounds__(256) vz_lists(const CentralParams C) {
  const long long M = C.M;
  const u64 Q = C.tile_incl[M / kCentralTile - 1];
  const long long nL = static_cast<long long>(C.tile_cnt_incl[M / kCentralTile - 1]);
  for (long long j = blockIdx.x * static_cast<long long>(blockDim.x) + threadIdx.x; j < M;
       j += static_cast<long long>(gridDim.x) * blockDim.x) {
    const VoseSlot v = vose_slot(C, j, Q);
    const long long pos = v.small ? v.ls : nL + (j - v.ls);
    C.lists[pos] = static_cast<int>(j);
    C.vals[pos] = v.small ? v.Dinc : v.Einc;
  }
}

// first index i in [0, n) with a[i] >= x
__device__ __forceinline__ long long first_not_less(const u64* __restrict__ a, long long n, u64 x) {
  long long lo = 0;
  while (n > 0) {
    const long long half = n >> 1;
    if (__ldg(a + lo + half) < x) {
      lo += half + 1;
      n -= half + 1;
    } else {
      n = half;
    }
  }
  return lo;
}
// first index i in [0, n) with a[i] > x
__device__ __forceinline__ long long first_above(const u64* __restrict__ a, long long n, u64 x) {
  long long lo = 0;
  while (n > 0) {
    const long long half = n >> 1;
    if (__ldg(a + lo + half) <= x) {
      lo += half + 1;
      n -= half + 1;
    } else {
      n = half;
    }
  }
  return lo;
}

__global__ void __launch_bounds__(256) vz_table(const CentralParams C) {
  const long long M = C.M;
  const u64 Q = C.tile_incl[M / kCentralTile - 1];
  const long long nL = static_cast<long long>(C.tile_cnt_incl[M / kCentralTile - 1]);
  const u64 Dtot = C.tile_D_incl[M / kCentralTile - 1];
  for (long long j = blockIdx.x * static_cast<long long>(blockDim.x) + threadIdx.x; j < M;
       j += static_cast<long long>(gridDim.x) * blockDim.x) {
    const VoseSlot v = vose_slot(C, j, Q);
    u64 pr;
    int al;
    if (v.small) {
      pr = v.a;
      al = C.lists[nL + first_not_less(C.vals + nL, M - nL, v.Dinc - v.def)];
    } else if (v.Einc < Dtot) {
      pr = Q + v.Einc - C.vals[first_above(C.vals, nL, v.Einc)];
      al = C.lists[nL + (j - v.ls) + 1];
    } else {
      pr = Q;
      al = static_cast<int>(j);
    }
    C.prob[j] = pr;
    C.alias[j] = al;
  }
}

// first index i in [0, n) with a[i] > x (n if none)
__device__ __forceinline__ long long first_greater(const u64* __restrict__ a, long long n, u64 x) {
  long long lo = 0;
  while (n > 0) {
    const long long half = n >> 1;
    if (__ldg(a + lo + half) <= x) {
      lo += half + 1;
      n -= half + 1;
    } else {
      n = half;
    }
  }
  return lo;
}

// a8 over all M slots: the ancestor of a slot from its uniforms (U_a, U_b).
__device__ __forceinline__ long long central_ancestor(const CentralParams& C, u64 Q, int tiles, uint32_t ua,
                                                      uint32_t ub) {
  if (C.vose) {
    // Vose draw (§VI-F, R10): column b = floor(U_a M / 2^32),
    // c = floor(U_b Q / 2^32); a = b if c < prob[b] else alias[b]
    const long long b = static_cast<long long>((static_cast<u64>(ua) * static_cast<u64>(C.M)) >> 32);
    const u64 c = static_cast<u64>((static_cast<unsigned __int128>(ub) * Q) >> 32);
    return c < __ldg(C.prob + b) ? b : __ldg(C.alias + b);
  }
  // RWS (§VI-F, R9): c = floor(U Q / 2^32), first j with C_j > c
  const u64 c = static_cast<u64>((static_cast<unsigned __int128>(ua) * Q) >> 32);
  const long long b = first_greater(C.tile_incl, tiles, c);
  const u64 excl = b > 0 ? __ldg(C.tile_incl + b - 1) : 0ull;
  return b * kCentralTile + first_greater(C.cl + b * kCentralTile, kCentralTile, c - excl);
}

// Test hook: per-tile inclusive sums of given integer weights q (instead of
// cz_tile_scan's q from the log-weights), then the ancestors for given uniforms.
__global__ void __launch_bounds__(kScanThreads) cz_tile_scan_q(const uint32_t* __restrict__ q, u64* __restrict__ cl,
                                                               u64* __restrict__ tile_sum) {
  __shared__ u64 sm[32];
  const long long base = static_cast<long long>(blockIdx.x) * kCentralTile + threadIdx.x * kPerThread;
  u64 run[kPerThread];
  u64 acc = 0;
#pragma unroll
  for (int j = 0; j < kPerThread; ++j) {
    acc += q[base + j];
    run[j] = acc;
  }
  u64 total;
  const u64 off = block_excl_scan(acc, sm, total);
#pragma unroll
  for (int j = 0; j < kPerThread; ++j) cl[base + j] = off + run[j];
  if (threadIdx.x == 0) tile_sum[blockIdx.x] = total;
}
__global__ void __launch_bounds__(256) cz_draw_debug(const CentralParams C, const uint32_t* __restrict__ ua,
                                                     const uint32_t* __restrict__ ub, int* __restrict__ anc) {
  const int tiles = static_cast<int>(C.M / kCentralTile);
  const u64 Q = C.tile_incl[tiles - 1];
  for (long long j = blockIdx.x * static_cast<long long>(blockDim.x) + threadIdx.x; j < C.M;
       j += static_cast<long long>(gridDim.x) * blockDim.x)
    anc[j] = static_cast<int>(central_ancestor(C, Q, tiles, ua[j], ub[j]));
}

template <class Model>
__global__ void __launch_bounds__(256) cz_step(const CentralParams C) {
  constexpr int D = Model::D, ZD = Model::ZD, UD = Model::UD;
  __shared__ float z_s[ZD];
  __shared__ float hsu_s[UD];
  __shared__ u64 red[32];
  __shared__ unsigned int s_last;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid < ZD) z_s[tid] = C.z ? C.z[tid] : C.zin[tid];
  if (tid < UD) hsu_s[tid] = C.mc.hs * (C.u ? C.u[tid] : C.uin[tid]);   // control term h_s u_i (F8)
  __syncthreads();
  const long long M = C.M;
  const int tiles = static_cast<int>(M / kCentralTile);
  const u64 Q = C.first ? 0ull : C.tile_incl[tiles - 1];
  u64 best = 0ull;
  for (long long i = blockIdx.x * static_cast<long long>(blockDim.x) + tid; i < M;
       i += static_cast<long long>(gridDim.x) * blockDim.x) {
    const uint32_t p = static_cast<uint32_t>(i);
    if (C.publish) {   // restore: the loaded set is the step's weighted set
      const u64 key = order_key(C.in[static_cast<long long>(D) * M + i], p);
      best = key > best ? key : best;
      continue;
    }
    const u32x4 b0 = philox4x32_10_rk(p, C.k, 0u, 0u, C.rk);
    const long long a = C.first ? i : central_ancestor(C, Q, tiles, b0.x, b0.y);
    const float* xa = C.in + a;
    auto x = [xa, M](int c) { return __ldg(xa + c * M); };
    NoiseGen gen{p, C.k, C.rk, u32x4{0u, 0u, b0.z, b0.w}};
    typename Model::Acc A;
    float* out = C.out + i;
    SampleStream<Model, 0>::run(C.mc, hsu_s, z_s, x, gen, A, [out, M](int c, float v) { out[c * M] = v; });
    const float l = Model::finish(C.mc, z_s, A);
    out[D * M] = l;
    const u64 key = order_key(l, p);
    best = key > best ? key : best;
  }
  // a5: block argmax -> one atomicMax; the last CTA copies the winner
  const u64 w = warp_max_u64(best);
  if (lane == 0) red[warp] = w;
  __syncthreads();
  if (warp == 0) {
    const u64 v = warp_max_u64(lane < static_cast<int>(blockDim.x >> 5) ? red[lane] : 0ull);
    if (lane == 0) atomicMax(C.key_cur, v);
  }
  __threadfence();
  __syncthreads();
  if (tid == 0) s_last = (atomicAdd(C.counter, 1u) == gridDim.x - 1) ? 1u : 0u;
  __syncthreads();
  if (s_last) {
    __threadfence();
    const u64 key = __ldcg(C.key_cur);
    const uint32_t gidx = 0xFFFFFFFFu - static_cast<uint32_t>(key);
    float* outs[3] = {C.record, C.est_out, C.record_host};
    const float* src = C.publish ? C.in : C.out;
    if (tid < D) {
      const float v = __ldcg(src + static_cast<long long>(tid) * M + gidx);
      for (int o = 0; o < 3; ++o)
        if (outs[o]) outs[o][4 + tid] = v;
    }
    if (tid == 0) {
      const float r[4] = {__uint_as_float(static_cast<uint32_t>(key)), __uint_as_float(static_cast<uint32_t>(key >> 32)),
                          unord_f32(static_cast<uint32_t>(key >> 32)), 0.0f};
      for (int o = 0; o < 3; ++o)
        if (outs[o])
          for (int c = 0; c < 4; ++c) outs[o][c] = r[c];
      *C.key_next = 0ull;
      *C.counter = 0u;
    }
    if (C.record_host) {   // completion word polled by pf_estimate (after the record, system scope)
      __threadfence_system();
      __syncthreads();
      if (tid == 0) *reinterpret_cast<volatile uint32_t*>(C.record_host + kRecordSeq) = C.k;
    }
  }
}

// the alias table; Q = tile_incl[tiles - 1] is read on the device
void vose_table(const CentralParams& c, cudaStream_t s) {
  const int tiles = static_cast<int>(c.M / kCentralTile);
  const int g2 = static_cast<int>(c.M / 256 < 148 * 8 ? c.M / 256 : 148 * 8);
  vz_class<<<tiles, kScanThreads, 0, s>>>(c);
  cz_tile_prefix<<<1, 1024, 0, s>>>(c.tile_cnt, c.tile_cnt_incl, tiles);
  cz_tile_prefix<<<1, 1024, 0, s>>>(c.tile_D, c.tile_D_incl, tiles);
  vz_lists<<<g2, 256, 0, s>>>(c);
  vz_table<<<g2, 256, 0, s>>>(c);
}

template <class Model>
cudaError_t central_step_m(const CentralParams& c, int grid, cudaStream_t s) {
  const int tiles = static_cast<int>(c.M / kCentralTile);
  if (!c.first && !c.publish) {
    cz_tile_scan<<<tiles, kScanThreads, 0, s>>>(c.in + static_cast<long long>(Model::D) * c.M, c.record_prev, c.cl,
                                                c.tile_sum);
    cz_tile_prefix<<<1, 1024, 0, s>>>(c.tile_sum, c.tile_incl, tiles);
    if (c.vose) vose_table(c, s);
  }
  cz_step<Model><<<grid, 256, 0, s>>>(c);
  return cudaGetLastError();
}

}  // namespace

cudaError_t central_step(int model, int nj, const CentralParams& c, int grid, cudaStream_t s) {
  if (model == MODEL_LINEAR_GAUSS_1D) return central_step_m<LinearGauss1D>(c, grid, s);
  switch (nj) {
    case 2: return central_step_m<ArmPlanar<2>>(c, grid, s);
    case 5: return central_step_m<ArmPlanar<5>>(c, grid, s);
    case 28: return central_step_m<ArmPlanar<28>>(c, grid, s);
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t central_resample_debug(const CentralParams& c, const uint32_t* q, const uint32_t* ua, const uint32_t* ub,
                                   int* anc, cudaStream_t s) {
  const int tiles = static_cast<int>(c.M / kCentralTile);
  cz_tile_scan_q<<<tiles, kScanThreads, 0, s>>>(q, c.cl, c.tile_sum);
  cz_tile_prefix<<<1, 1024, 0, s>>>(c.tile_sum, c.tile_incl, tiles);
  if (c.vose) vose_table(c, s);
  cz_draw_debug<<<static_cast<int>(c.M / 256 < 148 * 8 ? c.M / 256 : 148 * 8), 256, 0, s>>>(c, ua, ub, anc);
  return cudaGetLastError();
}

int central_grid(int model, int nj, int sms) {
  int bps = 0;
  cudaError_t e = cudaErrorInvalidValue;
  if (model == MODEL_LINEAR_GAUSS_1D) {
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, cz_step<LinearGauss1D>, 256, 0);
  } else {
    switch (nj) {
      case 2: e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, cz_step<ArmPlanar<2>>, 256, 0); break;
      case 5: e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, cz_step<ArmPlanar<5>>, 256, 0); break;
      case 28: e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, cz_step<ArmPlanar<28>>, 256, 0); break;
      default: break;
    }
  }
  return (e == cudaSuccess && bps > 0) ? bps * sms : 0;
}

}  // namespace pf
