// pf_registry.h — table of compiled pf_step_kernel<NJ, M, RES> instantiations.
// Each pf_inst_nj*.cu translation unit instantiates one n_joints value for
// every m in {32, ..., 1024} and both resamplers; the runtime looks entries
// up by (n_joints, m, resampler).
#pragma once
#include <cuda_runtime.h>

#include <cstddef>

namespace pf {
struct StepParams;

struct KernelEntry {
  int nj, m, res;
  cudaError_t (*prepare)(int* blocks_per_sm);
  cudaError_t (*launch)(const StepParams& p, int grid, cudaStream_t s);
  size_t smem;
};

extern const KernelEntry kEntriesNJ2[];
extern const KernelEntry kEntriesNJ5[];
extern const KernelEntry kEntriesNJ28[];
extern const int kNumEntriesPerNJ;
}  // namespace pf

#define PF_ENTRY(NJ, M, RES) \
  { NJ, M, RES, &StepKernel<NJ, M, RES>::prepare, &StepKernel<NJ, M, RES>::launch, StepKernel<NJ, M, RES>::smem() }
#define PF_ENTRIES_FOR(NJ)                                                                                  \
  PF_ENTRY(NJ, 32, 0), PF_ENTRY(NJ, 32, 1), PF_ENTRY(NJ, 64, 0), PF_ENTRY(NJ, 64, 1), PF_ENTRY(NJ, 128, 0), \
      PF_ENTRY(NJ, 128, 1), PF_ENTRY(NJ, 256, 0), PF_ENTRY(NJ, 256, 1), PF_ENTRY(NJ, 512, 0),               \
      PF_ENTRY(NJ, 512, 1), PF_ENTRY(NJ, 1024, 0), PF_ENTRY(NJ, 1024, 1)
