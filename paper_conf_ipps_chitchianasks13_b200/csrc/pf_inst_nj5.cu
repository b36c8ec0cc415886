// pf_inst_nj5.cu — pf_step_kernel instantiations for the n_joints = 5 arm
// (d = 9), every m in {32..1024}, RWS and Vose.
#include "pf_kernels.cuh"
#include "pf_registry.h"

namespace pf {
const KernelEntry kEntriesNJ5[] = {PF_ENTRIES_FOR(5)};
}  // namespace pf
