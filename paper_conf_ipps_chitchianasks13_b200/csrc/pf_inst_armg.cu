// pf_inst_armg.cu — the generic arm (pf_model.cuh ArmDyn<28>): ANY n_joints in
// [1, 28] with runtime dimensions, bit-identical to a compiled instance of the
// same n_j (the fallback behind n_j in {2, 5, 28}).  Table key
// n_joints = 0 ("any"); one particle per thread up to m = 512 (the stage is
// sized for d = 32, as the high-DOF arm's).
#include "pf_kernels.cuh"
#include "pf_registry.h"

namespace pf {
#define PF_ARMG(M, RES, GW, S, MINB) PF_ENTRY_MT(ArmDyn<28>, 0, 0, M, RES, GW, S, 1, 1, MINB)
const KernelEntry kEntriesARMG[] = {
    PF_ARMG(32, 0, 1, 4, 1),   PF_ARMG(64, 0, 2, 2, 1),   PF_ARMG(128, 0, 4, 1, 1),  PF_ARMG(256, 0, 8, 1, 1),
    PF_ARMG(512, 0, 16, 1, 1), PF_ARMG(1024, 0, 16, 1, 1), PF_ARMG(32, 1, 1, 4, 1),  PF_ARMG(64, 1, 2, 2, 1),
    PF_ARMG(128, 1, 4, 1, 1),  PF_ARMG(256, 1, 8, 1, 1),  PF_ARMG(512, 1, 16, 1, 1), PF_ARMG(1024, 1, 16, 1, 1),
};
const int kNumEntriesARMG = sizeof(kEntriesARMG) / sizeof(kEntriesARMG[0]);
}  // namespace pf
