// pf_inst_nj2.cu — pf_step_kernel instantiations for the 2-link arm (d = 6).
#include "pf_kernels.cuh"
#include "pf_registry.h"

namespace pf {
const KernelEntry kEntriesNJ2[] = {PF_SMALL_D_ENTRIES(2, 0), PF_SMALL_D_ENTRIES(2, 1),
    PF_LATENCY_ENTRIES(2, 0), PF_LATENCY_ENTRIES(2, 1)};
const int kNumEntriesNJ2 = sizeof(kEntriesNJ2) / sizeof(kEntriesNJ2[0]);
}  // namespace pf
