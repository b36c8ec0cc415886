// pf_inst_armg.cu — the generic arm (pf_model.cuh ArmDyn<NJMAX>): ANY n_joints
// in [1, 28] with runtime dimensions, bit-identical to a compiled instance of
// the same n_j (the fallback behind n_j in {2, 5, 28}).  Three
// buckets by the shared-memory stage they need — d <= 12, d <= 20, d <= 32 —
// keyed n_joints = -NJMAX in the kernel table (the runtime takes the first,
// i.e. the smallest, bucket that holds n_j), each with the mapping of the
// compiled arm of that state size (packed pairs where a thread owns two slots).
#include "pf_kernels.cuh"
#include "pf_registry.h"

namespace pf {
#define PF_ARMG(NJM, M, RES, GW, S, MINB) PF_ENTRY_MT(ArmDyn<NJM>, -(NJM), 0, M, RES, GW, S, 1, 1, MINB)
#define PF_ARMG_SET(NJM, RES, G32, S32, G64, S64, G128, S128, G256, S256, M256, G512, S512, G1K, S1K, MINB)          \
  PF_ARMG(NJM, 32, RES, G32, S32, MINB), PF_ARMG(NJM, 64, RES, G64, S64, MINB),                                    \
      PF_ARMG(NJM, 128, RES, G128, S128, MINB), PF_ARMG(NJM, 256, RES, G256, S256, M256),                          \
      PF_ARMG(NJM, 512, RES, G512, S512, MINB), PF_ARMG(NJM, 1024, RES, G1K, S1K, MINB)
const KernelEntry kEntriesARMG[] = {
    // d <= 12: the small-state mapping (about four particles per thread)
    PF_ARMG_SET(8, 0, 1, 8, 1, 8, 1, 8, 2, 4, 3, 4, 2, 4, 1, 3),
    PF_ARMG_SET(8, 1, 1, 8, 1, 8, 1, 8, 2, 4, 3, 4, 2, 4, 1, 3),
    // d <= 20: two particles per thread at m >= 256
    PF_ARMG_SET(16, 0, 1, 4, 2, 2, 4, 1, 4, 2, 2, 8, 1, 8, 1, 1),
    PF_ARMG_SET(16, 1, 1, 4, 2, 2, 4, 1, 4, 2, 2, 8, 1, 8, 1, 1),
    // d <= 32: the high-DOF arm's mapping
    PF_ARMG_SET(28, 0, 1, 4, 2, 2, 4, 1, 4, 1, 4, 16, 1, 16, 1, 1),
    PF_ARMG_SET(28, 1, 1, 4, 2, 2, 4, 1, 4, 1, 4, 16, 1, 16, 1, 1),
};
const int kNumEntriesARMG = sizeof(kEntriesARMG) / sizeof(kEntriesARMG[0]);
}  // namespace pf
