// pf_central.h — launch interface of the centralized filter (pf_central.cu).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

#include "pf_model.cuh"

namespace pf {

constexpr int kCentralTile = 4096;   // particles per scan tile (M must be a multiple)
// floats per particle record of the centralized filter's AoS state buffers:
// d rounded up to even (8-byte aligned records)
__host__ __device__ constexpr int central_stride(int d) { return (d + 1) & ~1; }

struct CentralParams {
  ModelConsts mc;           // model constants (pf_model.cuh)
  const float* in;          // [M][S] states of step k-1 (AoS records, S = central_stride(D); buffer (k-1)&1)
  float* out;               // [M][S] states of step k (buffer k&1)
  const float* lw_in;       // [M] log-weights of step k-1
  float* lw_out;            // [M] log-weights of step k
  long long M;
  int d, nj;                // state dimension and joints (read by runtime-dimension models only)
  unsigned long long* cl;   // [M] per-tile inclusive sums of q
  unsigned long long* tile_sum;    // [M / tile]
  unsigned long long* tile_incl;   // [M / tile] inclusive prefix of the tile sums
  const float* z;           // device or nullptr (zin)
  const float* u;
  float zin[32];
  float uin[32];
  unsigned long long* key_cur;
  unsigned long long* key_next;
  unsigned int* counter;
  const float* record_prev;   // estimate record of step k-1 (its key gives l_max)
  float* record;
  float* est_out;
  unsigned long long* record_host;   // nullable: tagged words of the mapped host record (put_tagged)
  uint32_t rk[20];
  uint32_t k;
  int first;     // k == 1 (or the sample-only test hook): no resampling
  int publish;   // only the argmax / record of the set in `in` (checkpoint restore)
  // Vose (resampler 1): the alias table over all M slots (sweep closed form, R10)
  int vose;
  unsigned long long* vscal;       // [3] nL, D_last, Q (vz_lists -> vz_merge)
  uint32_t* q32;                   // [M] integer weights q (u32)
  int* lists;                      // [M] small slots ascending, then large slots ascending
  unsigned long long* vals;        // [M] exclusive D over the small list, then inclusive E over the large list
  unsigned long long* prob;        // [M] alias-table threshold (units of Q / M)
  int* alias;                      // [M]
  unsigned long long* tile_cnt;    // [tiles] small count per tile, then its inclusive prefix
  unsigned long long* tile_cnt_incl;
  unsigned long long* tile_D;      // [tiles] deficit sum per tile, then its inclusive prefix
  unsigned long long* tile_D_incl;
};

// Largest centralized filter resampled by Vose: the deficit / excess sums
// (<= M Q <= M^2 2^22) stay below 2^64.
constexpr long long kCentralVoseMax = 1ll << 20;

// model: pf_model_id; nj: the arm's n_joints (2, 5, 28), ignored for the 1-D linear-Gaussian model
cudaError_t central_step(int model, int nj, const CentralParams& c, int grid, cudaStream_t s);
// test hook: RWS / Vose ancestors over all M slots from integer weights q [M]
// and uniforms ua, ub [M] (device); the Vose table is left in c.prob / c.alias
cudaError_t central_resample_debug(const CentralParams& c, const uint32_t* q, const uint32_t* ua, const uint32_t* ub,
                                   int* anc, cudaStream_t s);
int central_grid(int model, int nj, int sms);

}  // namespace pf
