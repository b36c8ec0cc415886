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

template <int NJ>
__global__ void __launch_bounds__(256) cz_step(const CentralParams C) {
  constexpr int D = NJ + 4;
  __shared__ float z_s[NJ + 2];
  __shared__ float hsu_s[NJ > 0 ? NJ : 1];
  __shared__ u64 red[32];
  __shared__ unsigned int s_last;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid < NJ + 2) z_s[tid] = C.z ? C.z[tid] : C.zin[tid];
  if (tid < NJ) hsu_s[tid] = C.mc.hs * (C.u ? C.u[tid] : C.uin[tid]);
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
    long long a = i;
    if (!C.first) {
      // RWS (§VI-F, R9): c = floor(U Q / 2^32), first j with C_j > c
      const u64 c = static_cast<u64>((static_cast<unsigned __int128>(b0.x) * Q) >> 32);
      const long long b = first_greater(C.tile_incl, tiles, c);
      const u64 excl = b > 0 ? __ldg(C.tile_incl + b - 1) : 0ull;
      a = b * kCentralTile + first_greater(C.cl + b * kCentralTile, kCentralTile, c - excl);
    }
    const float* xa = C.in + a;
    auto x = [xa, M](int c) { return __ldg(xa + c * M); };
    NoiseGen gen{p, C.k, C.rk, u32x4{0u, 0u, b0.z, b0.w}};
    ArmAcc A;
    float* out = C.out + i;
    SampleStream<NJ, 0>::run(C.mc, hsu_s, z_s, x, gen, A, [out, M](int c, float v) { out[c * M] = v; });
    const float l = arm_finish(C.mc, z_s, A);
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
  }
}

template <int NJ>
cudaError_t central_step_nj(const CentralParams& c, int grid, cudaStream_t s) {
  const int tiles = static_cast<int>(c.M / kCentralTile);
  if (!c.first && !c.publish) {
    cz_tile_scan<<<tiles, kScanThreads, 0, s>>>(c.in + static_cast<long long>(NJ + 4) * c.M, c.record_prev, c.cl,
                                                c.tile_sum);
    cz_tile_prefix<<<1, 1024, 0, s>>>(c.tile_sum, c.tile_incl, tiles);
  }
  cz_step<NJ><<<grid, 256, 0, s>>>(c);
  return cudaGetLastError();
}

}  // namespace

cudaError_t central_step(int nj, const CentralParams& c, int grid, cudaStream_t s) {
  switch (nj) {
    case 2: return central_step_nj<2>(c, grid, s);
    case 5: return central_step_nj<5>(c, grid, s);
    case 28: return central_step_nj<28>(c, grid, s);
    default: return cudaErrorInvalidValue;
  }
}

int central_grid(int nj, int sms) {
  int bps = 0;
  cudaError_t e = cudaErrorInvalidValue;
  switch (nj) {
    case 2: e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, cz_step<2>, 256, 0); break;
    case 5: e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, cz_step<5>, 256, 0); break;
    case 28: e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, cz_step<28>, 256, 0); break;
    default: break;
  }
  return (e == cudaSuccess && bps > 0) ? bps * sms : 0;
}

}  // namespace pf
