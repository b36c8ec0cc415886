// pf_inst_nj2.cu — pf_step_kernel instantiations for the n_joints = 2 arm
// (d = 6), every m in {32..1024}, RWS and Vose.
#include "pf_kernels.cuh"
#include "pf_registry.h"

namespace pf {
const KernelEntry kEntriesNJ2[] = {PF_ENTRIES_FOR(2)};
}  // namespace pf
