// pf_debug.cu — test hooks evaluating the device fp32 contract
// element-wise, so tests can compare it bit for bit with the oracle, and an
// exhaustive on-device check of the branch-free sqrt against sqrt.rn.
#include <cuda_runtime.h>

#include <cstdint>

#include "../../include/pf.h"
#include "pf_device.cuh"

namespace {

__global__ void math_kernel(int fn, const uint32_t* in, uint32_t* out, long long n) {
  for (long long i = blockIdx.x * static_cast<long long>(blockDim.x) + threadIdx.x; i < n;
       i += static_cast<long long>(gridDim.x) * blockDim.x) {
    const uint32_t a = in[i];
    const float x = __uint_as_float(a);
    float s, c;
    switch (fn) {
      case PF_MATH_SIN: pf::sincos_c(x, s, c); out[i] = __float_as_uint(s); break;
      case PF_MATH_COS: pf::sincos_c(x, s, c); out[i] = __float_as_uint(c); break;
      case PF_MATH_LOG: out[i] = __float_as_uint(pf::log_c(x)); break;
      case PF_MATH_EXPQ: out[i] = pf::expq_c(x); break;
      case PF_MATH_SQRT: out[i] = __float_as_uint(pf::sqrt_pos(x)); break;
      case PF_MATH_SINCOS2PI: pf::sincos2pi_c(a, s, c); out[2 * i] = __float_as_uint(s);
        out[2 * i + 1] = __float_as_uint(c); break;
      case PF_MATH_NORMAL_PAIR: {
        float z0, z1;
        pf::normal_pair(a, in[n + i], z0, z1);
        out[2 * i] = __float_as_uint(z0);
        out[2 * i + 1] = __float_as_uint(z1);
        break;
      }
      case PF_MATH_PHILOX: {   // in: [4][n] counters + key in the first two of a second block
        const pf::u32x4 r = pf::philox4x32_10(a, in[n + i], in[2 * n + i], in[3 * n + i], in[4 * n], in[4 * n + 1]);
        out[4 * i] = r.x; out[4 * i + 1] = r.y; out[4 * i + 2] = r.z; out[4 * i + 3] = r.w;
        break;
      }
      default: break;
    }
  }
}

// The packed (f32x2) evaluation of the same functions on element pairs
// (2i, 2i+1); n even.
__global__ void math_x2_kernel(int fn, const uint32_t* in, uint32_t* out, long long n) {
  for (long long i = blockIdx.x * static_cast<long long>(blockDim.x) + threadIdx.x; 2 * i < n;
       i += static_cast<long long>(gridDim.x) * blockDim.x) {
    const uint32_t a = in[2 * i], b = in[2 * i + 1];
    const pf::f2 x = pf::pk(__uint_as_float(a), __uint_as_float(b));
    pf::f2 s, c;
    switch (fn) {
      case PF_MATH_SIN: pf::sincos_c2(x, s, c); out[2 * i] = __float_as_uint(pf::lo2(s));
        out[2 * i + 1] = __float_as_uint(pf::hi2(s)); break;
      case PF_MATH_COS: pf::sincos_c2(x, s, c); out[2 * i] = __float_as_uint(pf::lo2(c));
        out[2 * i + 1] = __float_as_uint(pf::hi2(c)); break;
      case PF_MATH_LOG: s = pf::log_c2(x); out[2 * i] = __float_as_uint(pf::lo2(s));
        out[2 * i + 1] = __float_as_uint(pf::hi2(s)); break;
      case PF_MATH_EXPQ: pf::expq_c2(x, out[2 * i], out[2 * i + 1]); break;
      case PF_MATH_SQRT: s = pf::sqrt_pos2(x, pf::pk(-__uint_as_float(a), -__uint_as_float(b)));
        out[2 * i] = __float_as_uint(pf::lo2(s)); out[2 * i + 1] = __float_as_uint(pf::hi2(s)); break;
      case PF_MATH_SINCOS2PI: pf::sincos2pi_c2(a, b, s, c);
        out[4 * i] = __float_as_uint(pf::lo2(s)); out[4 * i + 1] = __float_as_uint(pf::lo2(c));
        out[4 * i + 2] = __float_as_uint(pf::hi2(s)); out[4 * i + 3] = __float_as_uint(pf::hi2(c)); break;
      case PF_MATH_NORMAL_PAIR: {
        pf::f2 z0, z1;
        pf::normal_pair2(a, in[n + 2 * i], b, in[n + 2 * i + 1], z0, z1);
        out[4 * i] = __float_as_uint(pf::lo2(z0)); out[4 * i + 1] = __float_as_uint(pf::lo2(z1));
        out[4 * i + 2] = __float_as_uint(pf::hi2(z0)); out[4 * i + 3] = __float_as_uint(pf::hi2(z1));
        break;
      }
      default: break;
    }
  }
}

__global__ void sqrt_check_kernel(uint32_t lo, uint32_t hi, unsigned long long* bad) {
  unsigned long long local = 0;
  for (unsigned long long b = lo + blockIdx.x * static_cast<unsigned long long>(blockDim.x) + threadIdx.x; b <= hi;
       b += static_cast<unsigned long long>(gridDim.x) * blockDim.x) {
    const float x = __uint_as_float(static_cast<uint32_t>(b));
    if (__float_as_uint(pf::sqrt_pos(x)) != __float_as_uint(__fsqrt_rn(x))) ++local;
  }
  if (local) atomicAdd(bad, local);
}

}  // namespace

extern "C" {

pf_status pf_debug_math(int32_t fn_flags, const uint32_t* in, uint32_t* out, int64_t n) {
  const bool x2 = (fn_flags & PF_MATH_X2) != 0;
  const int32_t fn = fn_flags & ~PF_MATH_X2;
  if (!in || !out || n < 0 || fn < PF_MATH_SIN || fn > PF_MATH_PHILOX) return PF_EINVAL;
  if (x2 && ((n & 1) || fn == PF_MATH_PHILOX)) return PF_EINVAL;
  const long long in_words = fn == PF_MATH_NORMAL_PAIR ? 2 * n : fn == PF_MATH_PHILOX ? 4 * n + 2 : n;
  const long long out_words = (fn == PF_MATH_SINCOS2PI || fn == PF_MATH_NORMAL_PAIR) ? 2 * n
                              : fn == PF_MATH_PHILOX                                  ? 4 * n
                                                                                      : n;
  uint32_t *din = nullptr, *dout = nullptr;
  cudaError_t e = cudaMalloc(&din, 4 * (in_words ? in_words : 1));
  if (e == cudaSuccess) e = cudaMalloc(&dout, 4 * (out_words ? out_words : 1));
  if (e == cudaSuccess) e = cudaMemcpy(din, in, 4 * in_words, cudaMemcpyHostToDevice);
  if (e == cudaSuccess && n > 0) {
    const int grid = static_cast<int>((n + 255) / 256 < 4096 ? (n + 255) / 256 : 4096);
    if (x2) {
      math_x2_kernel<<<grid, 256>>>(fn, din, dout, n);
    } else {
      math_kernel<<<grid, 256>>>(fn, din, dout, n);
    }
    e = cudaGetLastError();
  }
  if (e == cudaSuccess) e = cudaMemcpy(out, dout, 4 * out_words, cudaMemcpyDeviceToHost);
  cudaFree(din);
  cudaFree(dout);
  return e == cudaSuccess ? PF_OK : PF_ECUDA;
}

pf_status pf_debug_check_sqrt(uint32_t lo_bits, uint32_t hi_bits, uint64_t* mismatches) {
  if (!mismatches || hi_bits < lo_bits) return PF_EINVAL;
  unsigned long long* d = nullptr;
  cudaError_t e = cudaMalloc(&d, 8);
  if (e == cudaSuccess) e = cudaMemset(d, 0, 8);
  if (e == cudaSuccess) {
    sqrt_check_kernel<<<148 * 16, 256>>>(lo_bits, hi_bits, d);
    e = cudaGetLastError();
  }
  unsigned long long h = 0;
  if (e == cudaSuccess) e = cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  cudaFree(d);
  *mismatches = h;
  return e == cudaSuccess ? PF_OK : PF_ECUDA;
}

}  // extern "C"
