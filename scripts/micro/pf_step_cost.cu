// Host round-trip cost of a step through the C ABI (dev micro-benchmark):
// the launch + completion-signal floor of this box vs pf_step + pf_estimate.
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>
#include "../../include/pf.h"
using clk = std::chrono::high_resolution_clock;
static double us(clk::time_point a, clk::time_point b) { return std::chrono::duration<double, std::micro>(b - a).count(); }
__global__ void empty_k() {}
__global__ void flag_k(volatile unsigned* f, unsigned v) {
  __threadfence_system();
  *f = v;
}
int main(int argc, char** argv) {
  const long long m = argc > 1 ? atoll(argv[1]) : 32, N = argc > 2 ? atoll(argv[2]) : 4;
  cudaStream_t s;
  cudaStreamCreate(&s);
  const int R = 300;
  {  // launch + stream sync floor
    for (int i = 0; i < 20; ++i) { empty_k<<<1, 32, 0, s>>>(); cudaStreamSynchronize(s); }
    auto a = clk::now();
    for (int i = 0; i < R; ++i) { empty_k<<<1, 32, 0, s>>>(); cudaStreamSynchronize(s); }
    printf("empty kernel + cudaStreamSynchronize    %6.2f us\n", us(a, clk::now()) / R);
  }
  unsigned* fh;
  unsigned* fd;
  cudaHostAlloc(&fh, 64, cudaHostAllocMapped);
  cudaHostGetDevicePointer(&fd, fh, 0);
  {  // launch + mapped flag poll floor
    for (unsigned i = 1; i <= 20; ++i) { flag_k<<<1, 1, 0, s>>>(fd, i); while (__atomic_load_n(fh, __ATOMIC_ACQUIRE) != i) {} }
    auto a = clk::now();
    for (unsigned i = 21; i < 21 + R; ++i) { flag_k<<<1, 1, 0, s>>>(fd, i); while (__atomic_load_n(fh, __ATOMIC_ACQUIRE) != i) {} }
    printf("flag kernel + mapped poll               %6.2f us\n", us(a, clk::now()) / R);
    auto b = clk::now();
    for (int i = 0; i < R; ++i) empty_k<<<1, 32, 0, s>>>();
    auto c = clk::now();
    cudaStreamSynchronize(s);
    printf("empty kernel enqueue only               %6.2f us\n", us(b, c) / R);
  }
  pf_config cfg = {};
  cfg.m = m; cfg.n_filters = N; cfg.t = N > 1 ? 1 : 0; cfg.topo = N > 1 ? PF_TOPO_RING : PF_TOPO_NONE;
  cfg.resampler = PF_RESAMPLE_RWS; cfg.world = 1;
  pf_model_params mp = {PF_MODEL_ARM_PLANAR, 5, 1.0f, 0.1f, 0.1f, 0.1f, 0.1f, 0.1f, 0.1f};
  pf_sizes sz;
  if (pf_query_sizes(&cfg, &mp, &sz) != PF_OK) return 1;
  pf_buffers b;
  cudaMalloc(&b.state, sz.state); cudaMalloc(&b.mailbox, sz.mailbox); cudaMalloc(&b.scratch, sz.scratch);
  std::vector<float> mu(9, 0.1f), sg(9, 0.2f), z(7, 0.0f), u(5, 0.0f), x(9);
  pf_handle* h = nullptr;
  if (pf_init(&cfg, &mp, &b, s, mu.data(), sg.data(), &h) != PF_OK) return 2;
  for (int i = 0; i < 50; ++i) pf_step(h, z.data(), u.data());
  cudaStreamSynchronize(s);
  {
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0, s);
    for (int i = 0; i < R; ++i) pf_step(h, z.data(), u.data());
    cudaEventRecord(e1, s);
    cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    printf("pf_step back-to-back, device            %6.2f us/step (m=%lld N=%lld)\n", 1000.0 * ms / R, m, N);
  }
  {
    auto a = clk::now();
    for (int i = 0; i < R; ++i) { pf_step(h, z.data(), u.data()); cudaStreamSynchronize(s); }
    printf("pf_step + cudaStreamSynchronize         %6.2f us\n", us(a, clk::now()) / R);
  }
  {
    double tl = 0;
    auto a = clk::now();
    for (int i = 0; i < R; ++i) {
      auto q = clk::now();
      pf_step(h, z.data(), u.data());
      tl += us(q, clk::now());
      pf_estimate(h, x.data(), nullptr, nullptr);
    }
    printf("pf_step + pf_estimate                   %6.2f us (pf_step call %.2f us)\n", us(a, clk::now()) / R, tl / R);
  }
  pf_destroy(h);
  return 0;
}
