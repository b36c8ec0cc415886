// pf_central.cu — the centralized particle filter on the whole GPU (SURVEY.md
// NEXT-2): ONE filter of M > 1024 particles, resampled globally — the paper's
// reference scheme ("a sequential, centralized particle filter", PAPER.md:18
// §VI; Fig.5 and Fig.9).  Same arithmetic contract, counter
// layout and log-weight semantics as the distributed step (a1–a3, a5, a7–a10);
// no exchange.  RWS, two launches per step (k > 1):
//   cz_tile_scan  q_i = expq(l_i - l_max) (l_max = the previous step's best,
//                 from its estimate record) and per-tile inclusive u64 sums
//                 (one CTA of 1024 threads per 4096-slot tile)
//   cz_step       prologue: each CTA scans the tile totals into the tile
//                 prefix in its shared memory (and Q; above 4M particles a
//                 cz_tile_prefix launch does it instead); per particle: RWS
//                 draw (Philox (p, k, 0, 0) word 0, R9), binary search (tiles
//                 in shared memory, then inside the tile), gather from the
//                 previous buffer, sample + weight, store to the other buffer,
//                 block argmax + u64 atomicMax; the last CTA copies the
//                 winning particle to the estimate record.
// Particle buffers ping-pong: step k reads buffer (k-1)&1 and writes k&1.
#include <cuda_runtime.h>

#include <cstdint>

#include "pf_central.h"
#include "pf_kernels.cuh"

namespace pf {
namespace {

constexpr int kScanThreads = 1024;
constexpr int kPerThread = kCentralTile / kScanThreads;   // 4 consecutive particles per thread

__device__ __forceinline__ u64 block_excl_scan(u64 v, u64* sm, u64& total) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const u64 x = warp_incl_scan<u64>(v, lane);
  if (lane == 31) sm[warp] = x;
  __syncthreads();
  const u64 wt = warp_incl_scan<u64>(lane < nw ? sm[lane] : 0ull, lane);
  const u64 off = __shfl_sync(0xFFFFFFFFu, wt, (warp + 31) & 31);
  total = __shfl_sync(0xFFFFFFFFu, wt, nw - 1);
  __syncthreads();
  return (warp > 0 ? off : 0ull) + x - v;
}

// The inclusive sums of one tile (one CTA of 1024 threads, 4 consecutive
// slots per thread: a warp covers 128 slots, sum < 2^29, so the warp scan is
// u32; the warp offsets are u64, tile < 2^34) and the tile total.
__device__ __forceinline__ void tile_sums(const uint32_t (&q)[kPerThread], u64* __restrict__ cl,
                                          u64* __restrict__ tile_sum) {
  __shared__ uint32_t wtot[32];
  __shared__ u64 woff_s[33];
  const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
  uint32_t run[kPerThread];
  uint32_t acc = 0;
#pragma unroll
  for (int j = 0; j < kPerThread; ++j) {
    acc += q[j];
    run[j] = acc;
  }
  const uint32_t x = warp_incl_scan<uint32_t>(acc, lane);
  if (lane == 31) wtot[warp] = x;
  __syncthreads();
  if (warp == 0) {
    const u64 wt = wtot[lane];
    const u64 wi = warp_incl_scan<u64>(wt, lane);
    woff_s[lane] = wi - wt;
    if (lane == 31) woff_s[32] = wi;
  }
  __syncthreads();
  const u64 off = woff_s[warp] + (x - acc);
  ulonglong2* dst = reinterpret_cast<ulonglong2*>(cl + static_cast<long long>(blockIdx.x) * kCentralTile + t * kPerThread);
  dst[0] = make_ulonglong2(off + run[0], off + run[1]);
  dst[1] = make_ulonglong2(off + run[2], off + run[3]);
  if (t == 0) tile_sum[blockIdx.x] = woff_s[32];
}

// a7: integer weights of one tile and their inclusive sums (u64).
__global__ void __launch_bounds__(kScanThreads) cz_tile_scan(const float* __restrict__ logw, const float* record,
                                                             u64* __restrict__ cl, u64* __restrict__ tile_sum) {
  const float lmax = unord_f32(__float_as_uint(record[1]));   // ordered(l_max) is the key's high word
  const long long base = static_cast<long long>(blockIdx.x) * kCentralTile + threadIdx.x * kPerThread;
  const float4 w4 = *reinterpret_cast<const float4*>(logw + base);
  const uint32_t q[kPerThread] = {expq_c(w4.x - lmax), expq_c(w4.y - lmax), expq_c(w4.z - lmax), expq_c(w4.w - lmax)};
  tile_sums(q, cl, tile_sum);
}

// Inclusive prefix of the tile totals (one CTA of 1024 threads).
__global__ void __launch_bounds__(1024) cz_tile_prefix(const u64* __restrict__ tile_sum, u64* __restrict__ tile_incl,
                                                       int tiles) {
  __shared__ u64 sm[32];
  const int per = (tiles + 1023) / 1024;
  const int b0 = threadIdx.x * per;
  u64 acc = 0;
  for (int j = 0; j < per; ++j)
    if (b0 + j < tiles) acc += tile_sum[b0 + j];
  u64 total;
  u64 run = block_excl_scan(acc, sm, total);
  for (int j = 0; j < per; ++j)
    if (b0 + j < tiles) {
      run += tile_sum[b0 + j];
      tile_incl[b0 + j] = run;
    }
}

// ---- Vose over all M slots (§VI-F; the sweep closed form of
// reading R10, device-wide, as a MERGE): a_j = M q_j, small L = {a_j < Q} and
// large H (both ascending), A_i = exclusive deficit sum (Q - a) over L, E_j =
// inclusive excess sum (a - Q) over H.  Small L[i]: alias = H[#E < A_i],
// prob = a; large H[j] with E_j < D_last: prob = Q + E_j - (first A > E_j, or
// D_last), alias = H[j + 1]; else prob = Q, alias = itself — i.e. one merge of
// the sorted sequences A and E (A first on ties), as in the sub-filter kernel.
// Four passes (Vose is limited to M <= 2^20, so tiles <= 256 = one per thread):
//   vz_q      per tile: q_j = expq(l_j - l_max) (u32) and the tile sum
//   vz_count  Q = sum of the tile sums (every CTA); per tile: small count and
//             deficit sum; CTA 0 writes the inclusive tile prefix (Q for the draw)
//   vz_lists  global list positions from the tile prefixes + block scans:
//             A at [0, nL), E at [nL, M), slot indices alongside
//   vz_merge  merge path: one global diagonal search per CTA for its 4096
//             outputs, the two list segments staged in shared memory, one
//             shared-memory diagonal search per thread, 16 merge steps each
constexpr int kVoseTiles = static_cast<int>(kCentralVoseMax / kCentralTile);   // 256
constexpr int kVThreads = 1024;                       // Vose passes: one CTA of 1024 threads per tile
constexpr int kVPer = kCentralTile / kVThreads;      // 4 consecutive particles per thread
static_assert(kVoseTiles <= kVThreads, "one tile per thread in the tile-prefix scans");

// a7 for Vose: integer weights (u32) of one tile and the tile sum (from
// log-weights, or given q for the test hook)
__global__ void __launch_bounds__(kVThreads) vz_q(const float* __restrict__ logw, const float* record,
                                                     const uint32_t* __restrict__ qin, uint32_t* __restrict__ q32,
                                                     u64* __restrict__ tile_sum) {
  __shared__ u64 sm[32];
  const long long base = static_cast<long long>(blockIdx.x) * kCentralTile + threadIdx.x * kVPer;
  u64 acc = 0;
  if (qin) {
#pragma unroll
    for (int j = 0; j < kVPer; j += 4) {
      const uint4 v = *reinterpret_cast<const uint4*>(qin + base + j);
      *reinterpret_cast<uint4*>(q32 + base + j) = v;
      acc += static_cast<u64>(v.x) + v.y + v.z + v.w;
    }
  } else {
    const float lmax = unord_f32(__float_as_uint(record[1]));   // ordered(l_max) is the key's high word
#pragma unroll
    for (int j = 0; j < kVPer; j += 4) {
      const float4 w4 = *reinterpret_cast<const float4*>(logw + base + j);
      uint4 v;
      v.x = expq_c(w4.x - lmax);
      v.y = expq_c(w4.y - lmax);
      v.z = expq_c(w4.z - lmax);
      v.w = expq_c(w4.w - lmax);
      *reinterpret_cast<uint4*>(q32 + base + j) = v;
      acc += static_cast<u64>(v.x) + v.y + v.z + v.w;
    }
  }
  u64 total;
  block_excl_scan(acc, sm, total);
  if (threadIdx.x == 0) tile_sum[blockIdx.x] = total;
}

// Q = sum of all tile sums (one tile per thread); CTA 0 also writes the
// inclusive prefix of the tile sums (tile_incl: Q for the draws).
__device__ __forceinline__ u64 vz_total_q(const CentralParams& C, int tiles, u64* sm, bool write_prefix) {
  const u64 v = threadIdx.x < tiles ? C.tile_sum[threadIdx.x] : 0ull;
  u64 Q;
  const u64 excl = block_excl_scan(v, sm, Q);
  if (write_prefix && threadIdx.x < tiles) C.tile_incl[threadIdx.x] = excl + v;
  return Q;
}

__global__ void __launch_bounds__(kVThreads) vz_count(const CentralParams C) {
  __shared__ u64 sm[32];
  const long long M = C.M;
  const int tiles = static_cast<int>(M / kCentralTile);
  const u64 Q = vz_total_q(C, tiles, sm, blockIdx.x == 0);
  const long long base = static_cast<long long>(blockIdx.x) * kCentralTile + threadIdx.x * kVPer;
  u64 cnt = 0, dsum = 0;
#pragma unroll
  for (int j = 0; j < kVPer; j += 4) {
    const uint4 v = *reinterpret_cast<const uint4*>(C.q32 + base + j);
    const uint32_t qq[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const u64 a = static_cast<u64>(M) * qq[e];
      if (a < Q) {
        ++cnt;
        dsum += Q - a;
      }
    }
  }
  u64 tc, td;
  block_excl_scan(cnt, sm, tc);
  block_excl_scan(dsum, sm, td);
  if (threadIdx.x == 0) {
    C.tile_cnt[blockIdx.x] = tc;
    C.tile_D[blockIdx.x] = td;
  }
}

__global__ void __launch_bounds__(kVThreads) vz_lists(const CentralParams C) {
  extern __shared__ __align__(16) unsigned char lsm[];   // u64 [4096] values + int [4096] slots
  __shared__ u64 sm[32];
  __shared__ u64 pre[3];   // this tile's exclusive prefixes: weight sum, small count, deficit sum
  __shared__ u64 tot[3];   // nL, D_last, Q
  const long long M = C.M;
  const int tiles = static_cast<int>(M / kCentralTile);
  const int t = blockIdx.x, tid = threadIdx.x;
  {
    const u64 Q0 = tid < tiles ? C.tile_sum[tid] : 0ull;
    const u64 c0 = tid < tiles ? C.tile_cnt[tid] : 0ull;
    const u64 d0 = tid < tiles ? C.tile_D[tid] : 0ull;
    u64 tq, tcn, tdd;
    const u64 eq = block_excl_scan(Q0, sm, tq);
    const u64 ec = block_excl_scan(c0, sm, tcn);
    const u64 ed = block_excl_scan(d0, sm, tdd);
    if (tid == t) {
      pre[0] = eq;
      pre[1] = ec;
      pre[2] = ed;
    }
    if (tid == 0) {
      tot[0] = tcn;
      tot[1] = tdd;
      tot[2] = tq;
    }
  }
  __syncthreads();
  const u64 Q = tot[2];
  const long long nL = static_cast<long long>(tot[0]);
  const long long base = static_cast<long long>(t) * kCentralTile + tid * kVPer;
  uint32_t q[kVPer];
#pragma unroll
  for (int j = 0; j < kVPer; j += 4) {
    const uint4 v = *reinterpret_cast<const uint4*>(C.q32 + base + j);
    q[j] = v.x;
    q[j + 1] = v.y;
    q[j + 2] = v.z;
    q[j + 3] = v.w;
  }
  u64 sq = 0, sc = 0, sd = 0;
#pragma unroll
  for (int j = 0; j < kVPer; ++j) {
    const u64 a = static_cast<u64>(M) * q[j];
    sq += q[j];
    if (a < Q) {
      ++sc;
      sd += Q - a;
    }
  }

  u64 tq, tc, td;
  u64 oq = block_excl_scan(sq, sm, tq) + pre[0];
  u64 oc = block_excl_scan(sc, sm, tc) + pre[1];
  u64 od = block_excl_scan(sd, sm, td) + pre[2];
  // positions inside the tile (small at [0, cnt), large at [cnt, 4096)),
  // staged in shared memory, then copied out as two contiguous runs
  u64* v_s = reinterpret_cast<u64*>(lsm);
  int* l_s = reinterpret_cast<int*>(v_s + kCentralTile);
  const u64 oc0 = pre[1];                                  // smalls before the tile
  const int cnt_t = static_cast<int>(tc);                  // smalls in the tile
#pragma unroll
  for (int j = 0; j < kVPer; ++j) {
    const long long slot = base + j;
    const u64 a = static_cast<u64>(M) * q[j];
    oq += q[j];                                    // inclusive weight sum C_j
    if (a < Q) {                                   // small: rank oc, exclusive deficit od
      const int x = static_cast<int>(oc - oc0);
      v_s[x] = od;
      l_s[x] = static_cast<int>(slot);
      ++oc;
      od += Q - a;
    } else {                                       // large: E_j = D_j + M C_j - (j + 1) Q
      const int x = cnt_t + static_cast<int>((slot - t * static_cast<long long>(kCentralTile)) -
                                             static_cast<long long>(oc - oc0));
      v_s[x] = od + static_cast<u64>(M) * oq - static_cast<u64>(slot + 1) * Q;
      l_s[x] = static_cast<int>(slot);
    }
  }
  __syncthreads();
  const long long h0 = nL + (t * static_cast<long long>(kCentralTile) - static_cast<long long>(oc0));   // first large
#pragma unroll
  for (int r = 0; r < kCentralTile / kVThreads; ++r) {
    const int x = tid + r * kVThreads;
    const long long pos = x < cnt_t ? static_cast<long long>(oc0) + x : h0 + (x - cnt_t);
    C.vals[pos] = v_s[x];
    C.lists[pos] = l_s[x];
  }
  if (t == 0 && tid == 0) {
    C.vscal[0] = static_cast<u64>(nL);   // (scalars for vz_merge)
    C.vscal[1] = tot[1];
    C.vscal[2] = Q;
  }
}

// merge-path split of diagonal `diag` between A = vals[0, nL) and
// E = vals[nL, M): the number of A elements among the first diag merged
// (A before E on ties)
__device__ __forceinline__ long long merge_split(const u64* __restrict__ A, long long nA, const u64* __restrict__ B,
                                                 long long nB, long long diag) {
  long long lo = diag - nB > 0 ? diag - nB : 0, hi = diag < nA ? diag : nA;
  while (lo < hi) {
    const long long mid = (lo + hi) >> 1;
    if (A[mid] <= B[diag - 1 - mid]) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

// The same split found by the whole CTA: 256-ary search (each round one
// probe per thread, __syncthreads_count of the false probes), so a CTA spends
// ~3 rounds of L2 latency instead of ~20 dependent steps.  i >= lo0 is known.
__device__ long long merge_split_cta(const u64* __restrict__ A, long long nA, const u64* __restrict__ B, long long nB,
                                     long long diag, long long lo0, long long hi0) {
  long long lo = diag - nB > lo0 ? diag - nB : lo0;
  long long hi = diag < hi0 ? diag : hi0;
  while (lo < hi) {   // answer in [lo, hi]: the first i with A_i > B_{diag-1-i} (or hi)
    const long long n = hi - lo;
    const long long step = (n + blockDim.x - 1) / blockDim.x;
    const long long i = lo + (threadIdx.x + 1) * step - 1;
    const bool p = i >= hi || A[i] > B[diag - 1 - i];
    const int f = __syncthreads_count(!p);
    lo += f * step;
    const long long h2 = lo + step - 1;
    hi = h2 < hi ? h2 : hi;
  }
  return lo;
}

constexpr int kMergeW = kCentralTile;   // merged outputs per CTA
constexpr size_t kVoseMergeSmem = sizeof(u64) * (kMergeW + 2) + sizeof(int) * (kMergeW + 2);

__global__ void __launch_bounds__(kVThreads) vz_merge(const CentralParams C) {
  extern __shared__ __align__(16) unsigned char vsm[];
  u64* a_s = reinterpret_cast<u64*>(vsm);                 // [kMergeW + 1] A then E segment values
  int* l_s = reinterpret_cast<int*>(a_s + kMergeW + 2);   // [kMergeW + 2] their slot indices (+ E's next)
  __shared__ long long sp[2];
  const long long M = C.M;
  const long long nL = static_cast<long long>(C.vscal[0]), nH = M - nL;
  const u64 Dtot = C.vscal[1], Q = C.vscal[2];
  const u64* A = C.vals;
  const u64* E = C.vals + nL;
  const long long d0 = static_cast<long long>(blockIdx.x) * kMergeW, d1 = d0 + kMergeW;
  sp[0] = merge_split_cta(A, nL, E, nH, d0, 0, nL);
  sp[1] = merge_split_cta(A, nL, E, nH, d1, sp[0], nL);
  const long long i0 = sp[0], i1 = sp[1], j0 = d0 - i0, j1 = d1 - i1;
  const int na = static_cast<int>(i1 - i0), nb = static_cast<int>(j1 - j0);
  // stage A[i0, i1) at [0, na), E[j0, j1) at [na, na + nb), and E's next
  // list entry (alias of the last large slot) at l_s[na + nb]
  {
    constexpr int R = kMergeW / kVThreads;   // staged values per thread, loads issued together
    u64 v[R];
    int l[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const int x = threadIdx.x + r * kVThreads;
      const long long g = x < na ? i0 + x : nL + j0 + (x - na);   // vals / lists index
      v[r] = __ldcg(C.vals + g);
      l[r] = __ldcg(C.lists + g);
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
      a_s[threadIdx.x + r * kVThreads] = v[r];
      l_s[threadIdx.x + r * kVThreads] = l[r];
    }
  }
  if (threadIdx.x == 0) {
    a_s[kMergeW] = i1 < nL ? A[i1] : Dtot;       // the A head after the segment
    a_s[kMergeW + 1] = j1 < nH ? E[j1] : ~0ull;  // the E head after the segment
    l_s[kMergeW] = j1 < nH ? C.lists[nL + j1] : -1;
    l_s[kMergeW + 1] = j1 + 1 < nH ? C.lists[nL + j1 + 1] : -1;
  }
  __syncthreads();
  auto Aat = [&](int i) { return i < na ? a_s[i] : a_s[kMergeW]; };              // i <= na
  auto Bat = [&](int j) { return j < nb ? a_s[na + j] : a_s[kMergeW + 1]; };     // j <= nb
  auto Hl = [&](int j) { return j < nb ? l_s[na + j] : l_s[kMergeW + (j - nb)]; };   // H[j0 + j], j <= nb + 1
  constexpr int PT = kMergeW / kVThreads;   // 4 outputs per thread
  const int diag = threadIdx.x * PT;
  int lo = diag - nb > 0 ? diag - nb : 0, hi = diag < na ? diag : na;
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if (a_s[mid] <= a_s[na + diag - 1 - mid]) lo = mid + 1;
    else hi = mid;
  }
  int i = lo, j = diag - lo;
  u64 Ai = Aat(i), Bj = Bat(j);
  for (int e = 0; e < PT; ++e) {
    int s, al;
    u64 pr;
    if (i < na && Ai <= Bj) {   // small slot L[i0 + i]: alias = H[#E before it]
      s = l_s[i];
      const u64 An = Aat(i + 1);
      pr = Q - (An - Ai);
      al = Hl(j);
      ++i;
      Ai = An;
    } else {                    // large slot H[j0 + j]
      s = Hl(j);
      if (Bj < Dtot) {
        pr = Q + Bj - Ai;
        al = Hl(j + 1);
      } else {
        pr = Q;
        al = s;
      }
      ++j;
      Bj = Bat(j);
    }
    C.prob[s] = pr;
    C.alias[s] = al;
  }
}

// first index i in [0, n) with a[i] > x (n if none)
__device__ __forceinline__ long long first_greater(const u64* __restrict__ a, long long n, u64 x) {
  long long lo = 0;
  while (n > 0) {
    const long long half = n >> 1;
    if (__ldg(a + lo + half) <= x) {
      lo += half + 1;
      n -= half + 1;
    } else {
      n = half;
    }
  }
  return lo;
}

// a8 over all M slots: the ancestor of a slot from its uniforms (U_a, U_b).
// RWS: the tile by a binary search over the inclusive tile prefix (in shared
// memory, tidx, when it fits: kTidxMax tiles), then inside the tile in two
// levels — every 64th inclusive sum first (6 probes), then the 64-slot block
// (6 probes within 512 B) — the same first j with C_j > c as one search.
constexpr int kTidxMax = 1024;   // tiles whose prefix a CTA keeps in shared memory (8 KB)
__device__ __forceinline__ long long central_ancestor(const CentralParams& C, u64 Q, int tiles, uint32_t ua,
                                                      uint32_t ub, const u64* tidx) {
  if (C.vose) {
    // Vose draw (§VI-F, R10): column b = floor(U_a M / 2^32),
    // c = floor(U_b Q / 2^32); a = b if c < prob[b] else alias[b]
    const long long b = static_cast<long long>((static_cast<u64>(ua) * static_cast<u64>(C.M)) >> 32);
    const u64 c = static_cast<u64>((static_cast<unsigned __int128>(ub) * Q) >> 32);
    return c < __ldg(C.prob + b) ? b : __ldg(C.alias + b);
  }
  // RWS (§VI-F, R9): c = floor(U Q / 2^32), first j with C_j > c
  const u64 c = static_cast<u64>((static_cast<unsigned __int128>(ua) * Q) >> 32);
  long long b;
  u64 excl;
  if (tidx) {
    int lo = 0, n = tiles;
    while (n > 0) {
      const int half = n >> 1;
      if (tidx[lo + half] <= c) {
        lo += half + 1;
        n -= half + 1;
      } else {
        n = half;
      }
    }
    b = lo;
    excl = b > 0 ? tidx[b - 1] : 0ull;
  } else {
    b = first_greater(C.tile_incl, tiles, c);
    excl = b > 0 ? __ldg(C.tile_incl + b - 1) : 0ull;
  }
  const u64 cr = c - excl;
  const u64* cl = C.cl + b * kCentralTile;
  int blk = 0;   // first 64-slot block whose last inclusive sum exceeds cr
#pragma unroll
  for (int s = 32; s >= 1; s >>= 1)
    if (__ldg(cl + (blk + s) * 64 - 1) <= cr) blk += s;
  int pos = blk * 64;   // (the tile's last sum exceeds cr: blk <= 63)
#pragma unroll
  for (int s = 32; s >= 1; s >>= 1)
    if (__ldg(cl + pos + s - 1) <= cr) pos += s;
  return b * kCentralTile + pos;
}

// Test hook: per-tile inclusive sums of given integer weights q (instead of
// cz_tile_scan's q from the log-weights), then the ancestors for given uniforms.
__global__ void __launch_bounds__(kScanThreads) cz_tile_scan_q(const uint32_t* __restrict__ qin, u64* __restrict__ cl,
                                                               u64* __restrict__ tile_sum) {
  const long long base = static_cast<long long>(blockIdx.x) * kCentralTile + threadIdx.x * kPerThread;
  uint32_t q[kPerThread];
#pragma unroll
  for (int j = 0; j < kPerThread; ++j) q[j] = qin[base + j];
  tile_sums(q, cl, tile_sum);
}
__global__ void __launch_bounds__(256) cz_draw_debug(const CentralParams C, const uint32_t* __restrict__ ua,
                                                     const uint32_t* __restrict__ ub, int* __restrict__ anc) {
  const int tiles = static_cast<int>(C.M / kCentralTile);
  const u64 Q = C.tile_incl[tiles - 1];
  for (long long j = blockIdx.x * static_cast<long long>(blockDim.x) + threadIdx.x; j < C.M;
       j += static_cast<long long>(gridDim.x) * blockDim.x)
    anc[j] = static_cast<int>(central_ancestor(C, Q, tiles, ua[j], ub[j], nullptr));
}

template <class Model>
__global__ void __launch_bounds__(256) cz_step(const CentralParams C) {
  // dimensions: compile-time, or from the launch for the generic arm
  // (Model::RUNTIME: the stage is sized for its largest d, records use the runtime d)
  constexpr bool RT = Model::RUNTIME;
  constexpr int SMAX = central_stride(Model::D);
  const int D = RT ? C.d : Model::D;
  const int S = RT ? central_stride(C.d) : SMAX;
  const int ZD = RT ? C.nj + 2 : Model::ZD, UD = RT ? C.nj : Model::UD;
  __shared__ float z_s[Model::ZD];
  __shared__ float hsu_s[Model::UD];
  __shared__ u64 red[32];
  __shared__ unsigned int s_last;
  __shared__ float stage_s[256 / 32][32 * SMAX];   // each warp's 32 new records, written out coalesced
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  float* st = stage_s[warp];
  if (tid < ZD) z_s[tid] = C.z ? C.z[tid] : C.zin[tid];
  if (tid < UD) hsu_s[tid] = C.mc.hs * (C.u ? C.u[tid] : C.uin[tid]);   // control term h_s u_i (F8)
  const long long M = C.M;
  const int tiles = static_cast<int>(M / kCentralTile);
  __shared__ u64 tidx_s[kTidxMax];   // RWS: the inclusive tile prefix
  const bool use_tidx = !C.vose && !C.first && !C.publish && tiles <= kTidxMax;
  u64 Q = 0ull;
  if (use_tidx) {   // the inclusive prefix of the tile totals (in place of a cz_tile_prefix launch)
    const int per = (tiles + 255) / 256;   // <= 4 consecutive tiles per thread
    u64 v[kTidxMax / 256], acc = 0;
#pragma unroll
    for (int j = 0; j < kTidxMax / 256; ++j) {
      const int tt = tid * per + j;
      v[j] = (j < per && tt < tiles) ? __ldg(C.tile_sum + tt) : 0ull;
      acc += v[j];
    }
    u64 run = block_excl_scan(acc, red, Q);
#pragma unroll
    for (int j = 0; j < kTidxMax / 256; ++j) {
      const int tt = tid * per + j;
      run += v[j];
      if (j < per && tt < tiles) tidx_s[tt] = run;
    }
  }
  const u64* tidx = use_tidx ? tidx_s : nullptr;
  __syncthreads();
  if (!use_tidx && !C.first) Q = C.tile_incl[tiles - 1];
  u64 best = 0ull;
  // one particle per thread (grid-stride): the gather from random ancestors
  // is latency-bound, so occupancy (registers) matters more than the packed
  // pairs' instruction savings (measured: pairs at 74 registers no faster)
  for (long long i = blockIdx.x * static_cast<long long>(blockDim.x) + tid; i < M;
       i += static_cast<long long>(gridDim.x) * blockDim.x) {
    const uint32_t p = static_cast<uint32_t>(i);
    if (C.publish) {   // restore: the loaded set is the step's weighted set
      const u64 key = order_key(C.lw_in[i], p);
      best = key > best ? key : best;
      continue;
    }
    const u32x4 b0 = philox4x32_10_rk(p, C.k, 0u, 0u, C.rk);
    const long long a = C.first ? i : central_ancestor(C, Q, tiles, b0.x, b0.y, tidx);
    // AoS records: the ancestor's d components are one contiguous run (two
    // or three sectors), not d rows M apart
    const float* xa = C.in + a * S;
    auto x = [xa](int c) { return __ldg(xa + c); };
    NoiseGen gen{p, C.k, C.rk, u32x4{0u, 0u, b0.z, b0.w}};
    typename Model::Acc A;
    float* rec = st + lane * S;
    if constexpr (RT) {
      SampleRuntime<Model>::run(C.mc, C.nj, hsu_s, z_s, x, gen, A, [rec](int c, float v) { rec[c] = v; });
    } else if constexpr (Model::CHUNKED) {
      SampleChunked<Model>::run(C.mc, hsu_s, z_s, x, gen, A, [rec](int c, float v) { rec[c] = v; });
    } else {
      SampleStream<Model, 0>::run(C.mc, hsu_s, z_s, x, gen, A, [rec](int c, float v) { rec[c] = v; });
    }
    const float l = Model::finish(C.mc, z_s, A);
    C.lw_out[i] = l;
    // the warp's 32 consecutive records (i - lane .. i - lane + 31; M is a
    // multiple of the grid stride's 32-aligned warps) as contiguous stores
    __syncwarp();
    float* dst = C.out + (i - lane) * S;
#pragma unroll
    for (int f = lane; f < 32 * S; f += 32) dst[f] = st[f];
    __syncwarp();
    const u64 key = order_key(l, p);
    best = key > best ? key : best;
  }
  // a5: block argmax -> one atomicMax; the last CTA copies the winner
  const u64 w = warp_max_u64(best);
  if (lane == 0) red[warp] = w;
  __syncthreads();
  if (warp == 0) {
    const u64 v = warp_max_u64(lane < static_cast<int>(blockDim.x >> 5) ? red[lane] : 0ull);
    if (lane == 0) atomicMax(C.key_cur, v);
  }
  // the barrier orders every thread's writes (records, key) before thread 0's
  // completion count, a gpu-scope acquire-release RMW (cumulative); the last
  // CTA's acquire orders its reads below after every other CTA's release
  __syncthreads();
  if (tid == 0) {
    unsigned int prev;
    asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(prev) : "l"(C.counter) : "memory");
    s_last = (prev == gridDim.x - 1) ? 1u : 0u;
  }
  __syncthreads();
  if (s_last) {
    const u64 key = __ldcg(C.key_cur);
    const uint32_t gidx = 0xFFFFFFFFu - static_cast<uint32_t>(key);
    float* outs[2] = {C.record, C.est_out};
    const float* src = C.publish ? C.in : C.out;
    if (tid < D) {
      const float v = __ldcg(src + static_cast<long long>(gidx) * S + tid);
      for (int o = 0; o < 2; ++o)
        if (outs[o]) outs[o][4 + tid] = v;
      if (C.record_host) put_tagged(C.record_host, 4 + tid, v, C.k);
    }
    if (tid == 0) {
      const float r[4] = {__uint_as_float(static_cast<uint32_t>(key)), __uint_as_float(static_cast<uint32_t>(key >> 32)),
                          unord_f32(static_cast<uint32_t>(key >> 32)), 0.0f};
      for (int o = 0; o < 2; ++o)
        if (outs[o])
          for (int c = 0; c < 4; ++c) outs[o][c] = r[c];
      if (C.record_host)
        for (int c = 0; c < 4; ++c) put_tagged(C.record_host, c, r[c], C.k);
      *C.key_next = 0ull;
      *C.counter = 0u;
    }
  }
}

// the alias table (from C.q32 = q u32 and the tile sums of vz_q); Q is left in
// tile_incl[tiles - 1] for the draws
void vose_table(const CentralParams& c, cudaStream_t s) {
  const int tiles = static_cast<int>(c.M / kCentralTile);
  vz_count<<<tiles, kVThreads, 0, s>>>(c);
  vz_lists<<<tiles, kVThreads, kVoseMergeSmem, s>>>(c);
  vz_merge<<<tiles, kVThreads, kVoseMergeSmem, s>>>(c);
}

template <class Model>
cudaError_t central_step_m(const CentralParams& c, int grid, cudaStream_t s) {
  const int tiles = static_cast<int>(c.M / kCentralTile);
  if (!c.first && !c.publish) {
    const float* logw = c.lw_in;
    if (c.vose) {
      vz_q<<<tiles, kVThreads, 0, s>>>(logw, c.record_prev, nullptr, c.q32, c.tile_sum);
      vose_table(c, s);
    } else {
      cz_tile_scan<<<tiles, kScanThreads, 0, s>>>(logw, c.record_prev, c.cl, c.tile_sum);
      // the tile prefix: in every cz_step CTA's prologue when it fits its shared memory
      if (tiles > kTidxMax) cz_tile_prefix<<<1, 1024, 0, s>>>(c.tile_sum, c.tile_incl, tiles);
    }
  }
  cz_step<Model><<<grid, 256, 0, s>>>(c);
  return cudaGetLastError();
}

}  // namespace

cudaError_t central_step(int model, int nj, const CentralParams& c, int grid, cudaStream_t s) {
  if (model == MODEL_LINEAR_GAUSS_1D) return central_step_m<LinearGauss1D>(c, grid, s);
  switch (nj) {
    case 2: return central_step_m<ArmPlanar<2>>(c, grid, s);
    case 5: return central_step_m<ArmPlanar<5>>(c, grid, s);
    case 28: return central_step_m<ArmPlanar<28>>(c, grid, s);
    default:   // the generic arm, the smallest record stage that holds n_j
      if (nj >= 1 && nj <= 8) return central_step_m<ArmDyn<8>>(c, grid, s);
      return nj >= 1 && nj <= 28 ? central_step_m<ArmDyn<28>>(c, grid, s) : cudaErrorInvalidValue;
  }
}

cudaError_t central_resample_debug(const CentralParams& c, const uint32_t* q, const uint32_t* ua, const uint32_t* ub,
                                   int* anc, cudaStream_t s) {
  const int tiles = static_cast<int>(c.M / kCentralTile);
  if (c.vose) {
    vz_q<<<tiles, kVThreads, 0, s>>>(nullptr, nullptr, q, c.q32, c.tile_sum);
    vose_table(c, s);
  } else {
    cz_tile_scan_q<<<tiles, kScanThreads, 0, s>>>(q, c.cl, c.tile_sum);
    cz_tile_prefix<<<1, 1024, 0, s>>>(c.tile_sum, c.tile_incl, tiles);
  }
  cz_draw_debug<<<static_cast<int>(c.M / 256 < 148 * 8 ? c.M / 256 : 148 * 8), 256, 0, s>>>(c, ua, ub, anc);
  return cudaGetLastError();
}

int central_grid(int model, int nj, int sms) {
  int bps = 0;
  if (cudaFuncSetAttribute(vz_merge, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(kVoseMergeSmem)) !=
          cudaSuccess ||
      cudaFuncSetAttribute(vz_lists, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(kVoseMergeSmem)) !=
          cudaSuccess)
    return 0;
  cudaError_t e = cudaErrorInvalidValue;
  if (model == MODEL_LINEAR_GAUSS_1D) {
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, cz_step<LinearGauss1D>, 256, 0);
  } else {
    switch (nj) {
      case 2: e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, cz_step<ArmPlanar<2>>, 256, 0); break;
      case 5: e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, cz_step<ArmPlanar<5>>, 256, 0); break;
      case 28: e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, cz_step<ArmPlanar<28>>, 256, 0); break;
      default:
        if (nj >= 1 && nj <= 8) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, cz_step<ArmDyn<8>>, 256, 0);
        else if (nj >= 1 && nj <= 28)
          e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, cz_step<ArmDyn<28>>, 256, 0);
        break;
    }
  }
  return (e == cudaSuccess && bps > 0) ? bps * sms : 0;
}

}  // namespace pf
