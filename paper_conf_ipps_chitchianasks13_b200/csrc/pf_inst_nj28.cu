// pf_inst_nj28.cu — pf_step_kernel instantiations for the high-DOF arm
// (28 joints, d = 32; config C4): larger groups (fewer particles per thread)
// because a sub-filter's state block is 4 (d+1) m bytes of shared memory.
#include "pf_kernels.cuh"
#include "pf_registry.h"

namespace pf {
// (m = 256 without the split first load: C4's 16M-particle launches are
// tens of rounds of sub-filters, where it measured +0.6 %)
#define PF_LARGE_D_ENTRIES(NJ, RES, GW256, MINB256)                                                \
  PF_ENTRY(NJ, 32, RES, 1, 4, 1, 1, 1), PF_ENTRY(NJ, 64, RES, 2, 2, 1, 1, 1),                       \
      PF_ENTRY(NJ, 128, RES, 4, 1, 1, 1, 1), PF_ENTRY_NOSPLIT(NJ, 256, RES, GW256, 1, 1, 1, MINB256), \
      PF_ENTRY(NJ, 512, RES, 16, 1, 1, 1, 1), PF_ENTRY(NJ, 1024, RES, 16, 1, 1, 1, 1)
const KernelEntry kEntriesNJ28[] = {
    // m = 256 (config C4), measured: two particles per thread (packed f32x2 path with the
    // chunked joint loop): RWS 6 CTAs of 4 warps per SM, Vose 4 (one particle per thread
    // was the better Vose mapping before the chunked loop: 1834 -> 1469 us)
    PF_LARGE_D_ENTRIES(28, 0, 4, 6), PF_LARGE_D_ENTRIES(28, 1, 4, 4),
    PF_ENTRY(28, 256, 1, 8, 1, 1, 1, 4),
    PF_ENTRY(28, 256, 0, 8, 1, 1, 1, 4),
    PF_ENTRY(28, 256, 0, 8, 1, 1, 1, 3), PF_ENTRY(28, 256, 0, 4, 1, 1, 1, 4), PF_ENTRY(28, 256, 0, 8, 1, 2, 1, 3),
    PF_ENTRY(28, 256, 1, 8, 1, 1, 1, 3), PF_ENTRY(28, 256, 1, 4, 1, 1, 1, 4),
    PF_ENTRY(28, 256, 1, 4, 1, 1, 1, 6),
};
const int kNumEntriesNJ28 = sizeof(kEntriesNJ28) / sizeof(kEntriesNJ28[0]);
}  // namespace pf
