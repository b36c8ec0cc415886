// Cost of publishing a small record into mapped pinned host memory at the end
// of a kernel, by ordering scheme (dev micro-benchmark).
#include <chrono>
#include <cstdio>
#include <cuda_runtime.h>
using clk = std::chrono::high_resolution_clock;
template <int V>
__global__ void pub_k(float* rec, unsigned* seq, unsigned k) {
  const int tid = threadIdx.x;
  if (tid < 16) rec[tid] = static_cast<float>(k + tid);
  if (V == 0) return;                                   // record only (device or host memory)
  if (V == 1) { __syncthreads(); if (tid == 0) *(volatile unsigned*)seq = k; }   // no fence
  if (V == 2) { __threadfence_system(); __syncthreads(); if (tid == 0) *(volatile unsigned*)seq = k; }
  if (V == 3) { if (tid < 16) __threadfence_system(); __syncthreads(); if (tid == 0) *(volatile unsigned*)seq = k; }
  if (V == 4) {
    __syncthreads();
    if (tid == 0) asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(seq), "r"(k) : "memory");
  }
  if (V == 6) {   // 13 words, each with the sequence number in its upper half (no fence)
    if (tid < 13) {
      const unsigned long long w = (static_cast<unsigned long long>(k) << 32) | __float_as_uint(static_cast<float>(k + tid));
      asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(reinterpret_cast<unsigned long long*>(seq) + 8 + tid), "l"(w) : "memory");
    }
    return;
  }
  if (V == 5) {
    __syncthreads();
    if (tid == 0) { __threadfence_system(); *(volatile unsigned*)seq = k; }
  }
}
template <int V>
void run(const char* name, float* rec, unsigned* seq_d, volatile unsigned* seq_h, cudaStream_t s) {
  const int R = 400;
  static unsigned k = 1;
  for (int i = 0; i < 20; ++i) pub_k<V><<<1, 256, 0, s>>>(rec, seq_d, k++);
  cudaStreamSynchronize(s);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0, s);
  for (int i = 0; i < R; ++i) pub_k<V><<<1, 256, 0, s>>>(rec, seq_d, k++);
  cudaEventRecord(e1, s);
  cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  double rt = -1;
  if (V >= 1 && seq_h) {
    auto a = clk::now();
    for (int i = 0; i < R; ++i) {
      const unsigned want = k++;
      pub_k<V><<<1, 256, 0, s>>>(rec, seq_d, want);
      if (V == 6) {
        const unsigned long long* w = reinterpret_cast<const unsigned long long*>(const_cast<unsigned*>(seq_h)) + 8;
        for (int j = 0; j < 13; ++j)
          while ((__atomic_load_n(w + j, __ATOMIC_RELAXED) >> 32) != want) {}
      } else {
        while (__atomic_load_n(seq_h, __ATOMIC_ACQUIRE) != want) {}
      }
    }
    rt = std::chrono::duration<double, std::micro>(clk::now() - a).count() / R;
    cudaStreamSynchronize(s);
  }
  printf("%-40s back-to-back %6.2f us/launch   round trip %6.2f us\n", name, 1000.0 * ms / R, rt);
}
int main() {
  cudaStream_t s; cudaStreamCreate(&s);
  float *rh, *rd, *dev; unsigned *sh, *sd;
  cudaHostAlloc(&rh, 256, cudaHostAllocMapped); cudaHostGetDevicePointer(&rd, rh, 0);
  cudaHostAlloc(&sh, 256, cudaHostAllocMapped); cudaHostGetDevicePointer(&sd, sh, 0);
  cudaMalloc(&dev, 256);
  run<0>("record -> device memory", dev, sd, nullptr, s);
  run<0>("record -> host memory", rd, sd, nullptr, s);
  for (int rep = 0; rep < 2; ++rep) {
    run<1>("host, no fence", rd, sd, sh, s);
    run<2>("host, all threads fence.sc.sys", rd, sd, sh, s);
    run<3>("host, writers fence.sc.sys", rd, sd, sh, s);
    run<4>("host, bar + st.release.sys", rd, sd, sh, s);
    run<5>("host, bar + tid0 fence.sc.sys", rd, sd, sh, s);
    run<6>("host, 13 x u64 {word, seq}, no fence", rd, sd, sh, s);
  }
  return 0;
}
