// pf_mean.cu — weighted-average estimate (§VI-D:
// "The reduction operator can compute the particle with the highest weight,
// a weighted average, or any other associative operator"; reading R22).
//
// Over the weighted set of the last step (blocked SoA [n][d+1][m]):
//   omega_p = expq(l_p - L)  (F7, L = the global best log-weight of the
//                             estimate record, so omega_max = 2^22)
//   x_c     = sum_p omega_p x_cp / sum_p omega_p
// Integer weights (u64 sum, exact); each product omega x is exact in double
// and the numerators are summed in double in a fixed tree order (per-thread
// grid-stride partials, warp shuffles, warps in order, CTAs in order), so
// the result is deterministic for a launch configuration.  A second,
// one-CTA kernel adds the CTA partials (or the per-rank partial records of a
// sharded filter) and divides once.  One extra read pass over the set: the
// max-weight estimate is fused into the step, this operator is on demand.
#include <cuda_runtime.h>

#include <cstdint>

#include "pf_device.cuh"
#include "pf_mean.h"

namespace pf {
namespace {

typedef unsigned long long u64;

// D: the state dimension (compiled d) or an upper bound with the runtime d
// in dr (the generic arm: components c >= dr contribute 0 and are not stored)
template <int D>
__global__ void __launch_bounds__(kMeanThreads) mean_partial_kernel(const float* __restrict__ parts, long long n_blocks,
                                                                    int m, long long row, const float* record,
                                                                    double* __restrict__ partials, int aos,
                                                                    const float* __restrict__ lw, int dr) {
  __shared__ double sm[kMeanThreads / 32][D + 1];
  const float L = record[2];   // log-weight of the (global) best particle
  const long long total = n_blocks * m;
  u64 Q = 0;
  double S[D];
#pragma unroll
  for (int c = 0; c < D; ++c) S[c] = 0.0;
  for (long long p = blockIdx.x * static_cast<long long>(blockDim.x) + threadIdx.x; p < total;
       p += static_cast<long long>(gridDim.x) * blockDim.x) {
    const long long n = p / m, i = p - n * m;
    const float* b = aos ? parts + p * aos : parts + n * row + i;
    const long long cs = aos ? 1 : m;   // component stride
    const uint32_t q = expq_c((aos ? __ldg(lw + p) : __ldg(b + static_cast<long long>(dr) * m)) - L);
    if (q) {
      Q += q;
      const double qd = static_cast<double>(q);
#pragma unroll
      for (int c = 0; c < D; ++c)
        if (c < dr) S[c] = fma(qd, static_cast<double>(__ldg(b + c * cs)), S[c]);
    }
  }
#pragma unroll
  for (int o = 16; o >= 1; o >>= 1) {
    Q += __shfl_xor_sync(0xFFFFFFFFu, Q, o);
#pragma unroll
    for (int c = 0; c < D; ++c) S[c] += __shfl_xor_sync(0xFFFFFFFFu, S[c], o);
  }
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (lane == 0) {
    sm[warp][0] = __longlong_as_double(static_cast<long long>(Q));
#pragma unroll
    for (int c = 0; c < D; ++c) sm[warp][1 + c] = S[c];
  }
  __syncthreads();
  if (threadIdx.x <= dr) {
    const int c = threadIdx.x;
    double* out = partials + static_cast<long long>(blockIdx.x) * (dr + 1);
    if (c == 0) {
      u64 t = 0;
      for (int w = 0; w < kMeanThreads / 32; ++w) t += static_cast<u64>(__double_as_longlong(sm[w][0]));
      out[0] = __longlong_as_double(static_cast<long long>(t));
    } else {
      double t = 0.0;
      for (int w = 0; w < kMeanThreads / 32; ++w) t += sm[w][c];
      out[c] = t;
    }
  }
}

}  // namespace

// Sum `count` partial records [count][d+1] (slot 0 = the u64 weight sum,
// bit pattern) in order; write the summed record and / or the mean.
__global__ void mean_final_kernel(const double* __restrict__ partials, int count, int d, double* sum_out,
                                  float* mean_dev, float* mean_host) {
  __shared__ u64 Qs;
  const int c = threadIdx.x;
  if (c == 0) {
    u64 t = 0;
    for (int b = 0; b < count; ++b) t += static_cast<u64>(__double_as_longlong(partials[static_cast<long long>(b) * (d + 1)]));
    Qs = t;
    if (sum_out) sum_out[0] = __longlong_as_double(static_cast<long long>(t));
  }
  __syncthreads();
  if (c >= 1 && c <= d) {
    double t = 0.0;
    for (int b = 0; b < count; ++b) t += partials[static_cast<long long>(b) * (d + 1) + c];
    if (sum_out) sum_out[c] = t;
    const float v = static_cast<float>(t / static_cast<double>(Qs));
    if (mean_dev) mean_dev[c - 1] = v;
    if (mean_host) mean_host[c - 1] = v;
  }
}

cudaError_t mean_partials(const MeanParams& mp, cudaStream_t s) {
#define PF_MEAN(DD) mean_partial_kernel<DD><<<kMeanGrid, kMeanThreads, 0, s>>>(mp.parts, mp.n_blocks, mp.m, mp.row, \
                                                                          mp.record, mp.partials, mp.aos_stride, mp.lw, mp.d)
  switch (mp.d) {
    case 1: PF_MEAN(1); break;   // the linear-Gaussian model
    case 6: PF_MEAN(6); break;
    case 9: PF_MEAN(9); break;
    case 32: PF_MEAN(32); break;
    default:
      if (mp.d < 1 || mp.d > 32) return cudaErrorInvalidValue;
      if (mp.d <= 12) PF_MEAN(12);   // the generic arm (runtime d)
      else PF_MEAN(32);
  }
#undef PF_MEAN
  return cudaGetLastError();
}

cudaError_t mean_final(const double* partials, int count, int d, double* sum_out, float* mean_dev, float* mean_host,
                       cudaStream_t s) {
  mean_final_kernel<<<1, 64, 0, s>>>(partials, count, d, sum_out, mean_dev, mean_host);
  return cudaGetLastError();
}

}  // namespace pf
