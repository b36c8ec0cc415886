// pf_registry.h — table of compiled pf_step_kernel instantiations.
//
// Each pf_inst_*.cu translation unit instantiates one model (pf_model.cuh:
// the arm for one n_joints value, or the 1-D linear-Gaussian model) for every
// m in {32, ..., 1024} and both resamplers (plus alternative mappings of the
// hottest configurations).  The runtime takes the FIRST entry that matches
// (model, n_joints, m, resampler); PF_VARIANT=<i> in the environment selects
// the i-th matching entry instead (tuning knob, default 0).
#pragma once
#include <cuda_runtime.h>

#include <cstddef>
#include <cstdint>

namespace pf {
struct StepParams;

struct KernelEntry {
  int model, nj, m, res;          // pf_model_id; n_joints (arm; -NJMAX = a generic bucket) or 1
  int gw, s, nstage, unr, minb;   // warps per group, groups per CTA, TMA stages, sample unroll, min CTAs/SM
  int large;                      // preferred when the shard has >= kLargeNLocal sub-filters
  int split;                      // KCfg::SPLIT0: a group's first block in two bulk copies
  cudaError_t (*prepare)(int* blocks_per_sm);
  cudaError_t (*launch)(const StepParams& p, int grid, cudaStream_t s, bool pdl);
  cudaError_t (*resample_debug)(const uint32_t* q, const uint32_t* ua, const uint32_t* ub, int* anc,
                                unsigned long long* prob, int* alias, long long N, cudaStream_t s);
  size_t smem;
};

extern const KernelEntry kEntriesNJ2[];
extern const int kNumEntriesNJ2;
extern const KernelEntry kEntriesNJ5[];
extern const int kNumEntriesNJ5;
extern const KernelEntry kEntriesNJ28[];
extern const int kNumEntriesNJ28;
extern const KernelEntry kEntriesLG1[];
extern const int kNumEntriesLG1;
extern const KernelEntry kEntriesARMG[];   // the generic arm: n_joints key -NJMAX = any n_j <= NJMAX
extern const int kNumEntriesARMG;
}  // namespace pf

// one table entry for model type MT (its kId, n_joints NJ); SPLIT = KCfg::SPLIT0
#define PF_ENTRY_MTS(MT, NJ, LARGE, SPLIT, M, RES, GW, S, NST, UNR, MINB)                               \
  {MT::kId, NJ, M, RES, GW, S, NST, UNR, MINB, LARGE, SPLIT,                                        \
   &StepKernel<KCfg<MT, M, RES, GW, S, NST, UNR, MINB, 0, PF_X2_DEFAULT, SPLIT>>::prepare,           \
   &StepKernel<KCfg<MT, M, RES, GW, S, NST, UNR, MINB, 0, PF_X2_DEFAULT, SPLIT>>::launch,            \
   &StepKernel<KCfg<MT, M, RES, GW, S, NST, UNR, MINB, 0, PF_X2_DEFAULT, SPLIT>>::resample_debug,    \
   StepKernel<KCfg<MT, M, RES, GW, S, NST, UNR, MINB, 0, PF_X2_DEFAULT, SPLIT>>::smem()}
#define PF_ENTRY_MT(MT, NJ, LARGE, M, RES, GW, S, NST, UNR, MINB) \
  PF_ENTRY_MTS(MT, NJ, LARGE, 1, M, RES, GW, S, NST, UNR, MINB)
#define PF_ENTRY(NJ, M, RES, GW, S, NST, UNR, MINB) PF_ENTRY_MT(ArmPlanar<NJ>, NJ, 0, M, RES, GW, S, NST, UNR, MINB)
// Default mapping for small states (d <= 12), measured on B200:
// about four particles per thread (P = m / 32 GW), one warp per sub-filter up
// to m = 128, several sub-filters per CTA, at most ~80 registers (3 CTAs/SM).
#define PF_SMALL_D_ENTRIES(NJ, RES)                                                                  \
  PF_ENTRY(NJ, 32, RES, 1, 8, 1, 1, 3), PF_ENTRY(NJ, 64, RES, 1, 8, 1, 1, 3),                       \
      PF_ENTRY(NJ, 128, RES, 1, 8, 1, 1, 3), PF_ENTRY(NJ, 256, RES, 2, 4, 1, 1, 3),                 \
      PF_ENTRY(NJ, 512, RES, 4, 2, 1, 1, 3), PF_ENTRY(NJ, 1024, RES, 4, 1, 1, 1, 3)
// Lowest-latency mappings (one particle per thread) for small problems
// (selected by the runtime when the default leaves most groups idle).
#define PF_LATENCY_ENTRIES(NJ, RES)                                                                  \
  PF_ENTRY(NJ, 64, RES, 2, 4, 1, 1, 3), PF_ENTRY(NJ, 128, RES, 4, 2, 1, 1, 3),                      \
      PF_ENTRY(NJ, 256, RES, 8, 1, 1, 1, 3)
// large-shard mappings (tens of rounds of sub-filters per launch): no split first load (KCfg::SPLIT0)
#define PF_ENTRY_LARGE(NJ, M, RES, GW, S, NST, UNR, MINB) \
  PF_ENTRY_MTS(ArmPlanar<NJ>, NJ, 1, 0, M, RES, GW, S, NST, UNR, MINB)
#define PF_ENTRY_NOSPLIT(NJ, M, RES, GW, S, NST, UNR, MINB) \
  PF_ENTRY_MTS(ArmPlanar<NJ>, NJ, 0, 0, M, RES, GW, S, NST, UNR, MINB)
