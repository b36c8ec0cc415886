// pf_inst_lg1.cu — pf_step_kernel instantiations for the 1-D linear-Gaussian
// model (pf_model.cuh LinearGauss1D: the Kalman special case of SURVEY §8(c),
// whole-filter pin (ii)), every m in {32, ..., 1024}, RWS and Vose, with the
// small-state mapping and the one-particle-per-thread latency mapping.
#include "pf_kernels.cuh"
#include "pf_registry.h"

namespace pf {
#define PF_LG(M, RES, GW, S) PF_ENTRY_MT(LinearGauss1D, 1, 0, M, RES, GW, S, 1, 1, 3)
const KernelEntry kEntriesLG1[] = {
    PF_LG(32, 0, 1, 8),  PF_LG(64, 0, 1, 8),  PF_LG(128, 0, 1, 8), PF_LG(256, 0, 2, 4), PF_LG(512, 0, 4, 2),
    PF_LG(1024, 0, 4, 1), PF_LG(32, 1, 1, 8), PF_LG(64, 1, 1, 8),  PF_LG(128, 1, 1, 8), PF_LG(256, 1, 2, 4),
    PF_LG(512, 1, 4, 2), PF_LG(1024, 1, 4, 1),
    PF_LG(64, 0, 2, 4),  PF_LG(128, 0, 4, 2), PF_LG(256, 0, 8, 1), PF_LG(64, 1, 2, 4), PF_LG(128, 1, 4, 2),
    PF_LG(256, 1, 8, 1),
};
const int kNumEntriesLG1 = sizeof(kEntriesLG1) / sizeof(kEntriesLG1[0]);
}  // namespace pf
