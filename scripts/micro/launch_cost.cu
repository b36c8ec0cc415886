// Host cost of a kernel launch vs parameter size and launch API (dev micro-benchmark).
#include <chrono>
#include <cstdio>
#include <cuda_runtime.h>
template <int B> struct Par { char b[B]; };
template <int B> __global__ void k(const __grid_constant__ Par<B> p) { if (p.b[0] == 123 && threadIdx.x == 999) printf("x"); }
template <int B> double run(bool ex, cudaStream_t s) {
  Par<B> p{};
  for (int i = 0; i < 100; ++i) k<B><<<148, 256, 0, s>>>(p);
  cudaStreamSynchronize(s);
  auto t0 = std::chrono::high_resolution_clock::now();
  const int n = 2000;
  for (int i = 0; i < n; ++i) {
    if (!ex) { k<B><<<148, 256, 0, s>>>(p); continue; }
    cudaLaunchConfig_t cfg = {}; cfg.gridDim = dim3(148); cfg.blockDim = dim3(256); cfg.stream = s;
    cudaLaunchAttribute a[1]; a[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    a[0].val.programmaticStreamSerializationAllowed = 1; cfg.attrs = a; cfg.numAttrs = 1;
    cudaLaunchKernelEx(&cfg, k<B>, p);
  }
  auto t1 = std::chrono::high_resolution_clock::now();
  cudaStreamSynchronize(s);
  return std::chrono::duration<double, std::micro>(t1 - t0).count() / n;
}
int main() {
  cudaStream_t s; cudaStreamCreate(&s);
  printf("params  64 B: <<<>>> %.2f us  Ex+PDL %.2f us\n", run<64>(false, s), run<64>(true, s));
  printf("params 256 B: <<<>>> %.2f us  Ex+PDL %.2f us\n", run<256>(false, s), run<256>(true, s));
  printf("params 768 B: <<<>>> %.2f us  Ex+PDL %.2f us\n", run<768>(false, s), run<768>(true, s));
  printf("params 2048 B: <<<>>> %.2f us  Ex+PDL %.2f us\n", run<2048>(false, s), run<2048>(true, s));
  return 0;
}
