// pf_inst_nj28.cu — pf_step_kernel instantiations for the n_joints = 28 arm
// (d = 32), every m in {32..1024}, RWS and Vose.
#include "pf_kernels.cuh"
#include "pf_registry.h"

namespace pf {
const KernelEntry kEntriesNJ28[] = {PF_ENTRIES_FOR(28)};
}  // namespace pf
