// pf_inst_nj5.cu — pf_step_kernel instantiations for the paper's medium arm
// (5 joints incl. the base, d = 9; Table II), with alternative
// mappings of m = 256 (configs C2 / C5) for tuning.
#include "pf_kernels.cuh"
#include "pf_registry.h"

namespace pf {
const KernelEntry kEntriesNJ5[] = {
    PF_SMALL_D_ENTRIES(5, 0), PF_SMALL_D_ENTRIES(5, 1),
    PF_LATENCY_ENTRIES(5, 0), PF_LATENCY_ENTRIES(5, 1),
    // measured best for large shards (C5: 16M particles per GPU)
    PF_ENTRY_LARGE(5, 256, 0, 2, 4, 1, 1, 4), PF_ENTRY_LARGE(5, 256, 1, 2, 7, 1, 1, 2),
    PF_ENTRY_LARGE(5, 512, 0, 4, 1, 1, 1, 3),
    // alternatives for PF_VARIANT tuning of configs C2 / C5 (m = 256)
    PF_ENTRY(5, 256, 0, 8, 1, 2, 1, 4), PF_ENTRY(5, 256, 0, 1, 8, 1, 1, 3), PF_ENTRY(5, 256, 0, 4, 2, 1, 1, 3),
    PF_ENTRY(5, 256, 1, 8, 1, 2, 1, 2), PF_ENTRY(5, 256, 1, 4, 2, 1, 1, 2),
    PF_ENTRY(5, 256, 0, 2, 3, 1, 1, 4), PF_ENTRY(5, 256, 0, 1, 6, 1, 1, 4), PF_ENTRY(5, 256, 0, 2, 3, 1, 1, 3),
    PF_ENTRY(5, 256, 0, 4, 2, 1, 1, 4), PF_ENTRY(5, 256, 0, 1, 8, 1, 1, 4), PF_ENTRY(5, 256, 0, 2, 4, 1, 4, 2),
    PF_ENTRY(5, 256, 0, 2, 3, 1, 4, 3),
    PF_ENTRY(5, 256, 1, 2, 4, 1, 1, 4), PF_ENTRY(5, 256, 1, 2, 3, 1, 1, 4),
    PF_ENTRY(5, 256, 0, 2, 3, 2, 1, 3), PF_ENTRY(5, 256, 0, 2, 4, 2, 1, 2), PF_ENTRY(5, 256, 0, 2, 2, 2, 1, 4),
    // Vose with the round-2 table footprint (RWS + 2 KB per group): 14 groups per SM
    PF_ENTRY(5, 256, 1, 2, 2, 1, 1, 7), PF_ENTRY(5, 256, 1, 1, 7, 1, 1, 2),
    // one 2-warp group per CTA, 12 CTAs per SM: the same 12 groups per SM as the default, with the
    // group index and its shared-memory base compile-time constants (the compiler otherwise
    // rematerialises them under register pressure).  C2 RWS 43.1 vs 43.9 us on one box, 43.9 vs
    // 44.0 on another; Vose 48.0 vs 47.1 us — not the default
    PF_ENTRY(5, 256, 0, 2, 1, 1, 1, 12), PF_ENTRY(5, 256, 1, 2, 1, 1, 1, 12),
};
const int kNumEntriesNJ5 = sizeof(kEntriesNJ5) / sizeof(kEntriesNJ5[0]);
}  // namespace pf

#ifdef PF_TIMELINE
extern "C" int pf_debug_timeline(unsigned long long* out, long long cap, int reset) {
  if (reset) {
    static unsigned long long zero = 0;
    static unsigned long long init2[4] = {~0ull, 0ull, 0ull, 0ull};
    if (cudaMemcpyToSymbol(pf::pf_tl2, init2, sizeof(init2)) != cudaSuccess) return -3;
    return cudaMemcpyToSymbol(pf::pf_tl, &zero, sizeof(zero)) == cudaSuccess ? 0 : -3;
  }
  if (cap == -2) return cudaMemcpyFromSymbol(out, pf::pf_tl3, sizeof(unsigned long long) * 3 * 4096) == cudaSuccess ? 0 : -3;
  if (cap < 0) return cudaMemcpyFromSymbol(out, pf::pf_tl2, sizeof(unsigned long long) * 4) == cudaSuccess ? 0 : -3;
  return cudaMemcpyFromSymbol(out, pf::pf_tl, sizeof(unsigned long long) * cap) == cudaSuccess ? 0 : -3;
}
#endif
