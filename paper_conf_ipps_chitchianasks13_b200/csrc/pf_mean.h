// pf_mean.h — launch interface of the weighted-average estimate (pf_mean.cu).
#pragma once
#include <cuda_runtime.h>

namespace pf {

constexpr int kMeanGrid = 256;      // CTAs of the partial-sum pass (fixed: fixed summation order)
constexpr int kMeanThreads = 256;

struct MeanParams {
  const float* parts;   // weighted set, blocked SoA [n_blocks][d+1][m]
  long long n_blocks;   // sub-filters of the shard (the centralized filter: 1)
  int m;                // particles per block
  int d;                // state dimension (1, 6, 9 or 32)
  long long row;        // floats per block, (d+1) m
  int aos_stride;       // > 0: AoS records parts[p * aos_stride + c] and log-weights lw[p] (the centralized filter)
  const float* lw;
  const float* record;  // estimate record: record[2] = log-weight of the (global) best particle
  double* partials;     // [kMeanGrid][d+1] scratch
};

// per-CTA partial records [kMeanGrid][d+1]: slot 0 = sum of the integer
// weights (u64 bit pattern), slots 1..d = sum omega x_c (double)
cudaError_t mean_partials(const MeanParams& mp, cudaStream_t s);
// sum `count` partial records in order -> sum_out [d+1] (nullable) and the
// mean (float [d], device and / or mapped host pointers, nullable)
cudaError_t mean_final(const double* partials, int count, int d, double* sum_out, float* mean_dev, float* mean_host,
                       cudaStream_t s);

}  // namespace pf
