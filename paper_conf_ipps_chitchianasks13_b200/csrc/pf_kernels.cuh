// pf_kernels.cuh — sm_100a kernels of the distributed particle filter.
//
// pf_step_kernel<Cfg> is the ROTATED STEP: launch k performs,
// for every sub-filter of this shard,
//   a6 exchange   merge the neighbours' best t of step k-1 (mailbox) into the
//                 own worst deg*t slots                  (Alg.2 l.10–14, R2–R5)
//   a7 normalise  q_i = floor(2^22 exp(l_i - l_max))     (§VI-F, R7–R8)
//   a8 resample   RWS (scan + binary search) or Vose (alias table, sweep
//                 closed form)                           (Alg.2 l.15–19, R9–R11)
//   a9 gather     ancestor state from shared memory      (§VI-F)
//   a1 RNG        Philox4x32-10 in registers             (R12, R13)
//   a2 sample, a3 weight (fused, §VI-B)      (F8–F10)
//   a4 local reduce: argmax / best t -> mailbox (k&1)    (Alg.2 l.8, replaces the sort)
//   a5 global estimate: u64 atomicMax + last-CTA copy    (Alg.2 l.9, R6)
//   a10 store state + log-weight (in place)
// so each launch streams the particle set through HBM once (read + write).
//
// Data layout (blocked SoA): sub-filter n of the shard owns one contiguous
// block of (D+1) rows x M floats — rows 0..D-1 the state components, row D
// the log-weight — so a sub-filter arrives in shared memory with ONE TMA bulk
// copy and every per-component store is a coalesced row store at an
// immediate offset.
//
// Mapping: a GROUP of GW warps owns one sub-filter at a time (GW = 1: one
// warp per sub-filter, no CTA barrier at all); thread t of the group owns the
// P = M / (32 GW) strided slots t, t + 32GW, ...; a CTA holds S groups;
// persistent grid-stride loop over sub-filters; NSTAGE = 2 double-buffers the
// TMA load of the group's next sub-filter behind the current one.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <type_traits>

#include "pf_device.cuh"
#include "pf_model.cuh"

namespace pf {

typedef unsigned long long u64;

enum : int { MODE_STEP = 0, MODE_PUBLISH = 1, MODE_EXCHANGE = 2, MODE_SAMPLE = 3 };
enum : int { TOPO_NONE = 0, TOPO_RING = 1, TOPO_TORUS = 2, TOPO_A2A = 3 };
enum : int { RES_RWS = 0, RES_VOSE = 1 };
enum : int { POLICY_ALWAYS = 0, POLICY_ESS = 1, POLICY_FREQ = 2 };

// mapped host buffer (128 floats): u64 words [0, 4 + d) the estimate record of
// the last step, each tagged with the step number (put_tagged; pf_estimate
// polls them instead of synchronizing the stream), floats [kMeanHost,
// kMeanHost + d) the weighted mean
constexpr int kMeanHost = 80;

// Peer transport (world > 1 on one node, NVLink/NVSwitch peer memory): every
// rank's runtime owns a small "peer block" that the other ranks write into:
// [kMaxRanks] u64 rendezvous flags, then [2][kMaxRanks][kPeerRec] float
// records, then [2][kMaxRanks][kPeerPool] float All-to-All pool rows — the
// records and pool rows double-buffered by the parity of the rendezvous
// number (see the ordering argument at the rendezvous and DESIGN.md §8).
constexpr int kMaxRanks = 8;
constexpr int kPeerRec = 40;   // 4 + d <= 36 floats, padded
constexpr int kPeerPool = 32 * 34;   // All-to-All: t <= 32 entries of E = d + 2 <= 34 floats
constexpr size_t kPeerBlockUsed =
    sizeof(unsigned long long) * kMaxRanks + sizeof(float) * 2 * kMaxRanks * (kPeerRec + kPeerPool);
// record word 3 (a status, 0 = ok): the rendezvous timed out (a rank did not
// arrive within peer_timeout_ns) — the record is not the global estimate
constexpr uint32_t kStatusPeerTimeout = 1u;

struct StepParams {
  ModelConsts mc;          // model constants (pf_model.cuh)
  ModelConsts2 mc2;        // mc with every field duplicated (packed f32x2 operands)
  float* parts;            // [n_local][D+1][M] blocked SoA (row D = log-weight)
  const float* mb_prev;    // mailbox parity (k-1)&1 : [n_ext][tt][E]
  float* mb_cur;           // mailbox parity k&1
  const float* z;          // [ZD] device, or nullptr: use zin
  const float* u;          // [UD] device, or nullptr: use uin
  u64* key_cur;            // global best key of this step (0 on entry)
  u64* key_next;           // reset to 0 for the next step
  unsigned int* counter;   // CTA completion counter (0 on entry, reset by the last CTA)
  unsigned int* work;      // dynamic sub-filter counter (0 on entry, reset by the last CTA)
  float* record;           // [4 + d] estimate record of this shard
  float* est_out;          // nullable [4 + d] (batched mode)
  u64* record_host;        // nullable [4 + d]: mapped pinned host copy of the record (tagged words)
  long long* dbg_src;      // nullable [M_local] exchange sources (global index)
  int* dbg_anc;            // nullable [M_local] ancestors
  long long n_local, g0, n_global, R, C;
  long long pool_row;      // All-to-All: the row every sub-filter reads (global best t)
  long long pool_local_row;  // All-to-All: where the last CTA writes this shard's best t
  u64* pool_cta;             // All-to-All, t >= 2: [groups][tt] x {order key, mailbox entry}: each
                             // group's best t (the last CTA merges these instead of the whole mailbox)
  int t, tt, topo, deg;
  uint32_t t_inv;          // ceil(2^16 / t): lane / t = (lane * t_inv) >> 16 for lane < 2^16 / t
  uint32_t k;
  int mode, first;
  int policy;              // R21: POLICY_ALWAYS / _ESS / _FREQ
  unsigned long long policy_param;   // ESS: tau 2^16; FREQ: threshold on a Philox word
  uint32_t rk[20];         // Philox round keys (key0 + r W0, key1 + r W1), r = 0..9
  // peer transport (nullable peer_mb[0] = off): the prev / next neighbour
  // rank's mailbox base (ring: r -1 / r + 1; torus: the rank above / below),
  // every rank's peer block (own included), this rank and the world size
  float* peer_mb[2];
  unsigned char* peer_blk[kMaxRanks];
  int rank, world;
  long long mb_parity;     // floats per mailbox parity (n_ext * tt * E), same on every rank
  int d, nj;               // state dimension and joints (read by runtime-dimension models only)
  unsigned long long rv;   // peer rendezvous number of this launch (>= 1, +1 per peer-mode launch on every rank)
  unsigned long long peer_timeout_ns;   // give up waiting at the rendezvous after this long (status word)
  float zin[32];           // step inputs carried by the launch itself (host-input mode)
  float uin[32];
};

// ------------------------------------------------------------- PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(u64* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(u64* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, u64* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void bulk_prefetch_l2(const void* src, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(src), "r"(bytes) : "memory");
}
// relaxed fetch-and-add of 1 on the launch's work counter, not aggregated
// across the warp: the result register is consumed only where it is used
__device__ __forceinline__ unsigned int ticket_add(unsigned int* p) {
  unsigned int r;
  // atom.inc with a limit the counter never reaches is an add of 1 that ptxas
  // does not aggregate (it rewrites atom.add, and inc with limit 2^32-1, into
  // a warp-aggregated atomic + shuffle)
  asm volatile("atom.relaxed.gpu.global.inc.u32 %0, [%1], 0x7FFFFFFF;" : "=r"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ void mbar_arrive(u64* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(u64* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "PF_WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra PF_WAIT_%=;\n}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

#ifdef PF_TIMELINE
// dev-only timeline (scripts/timeline.py): one record of 8 u64 per sub-filter
__device__ unsigned long long pf_tl[1 + 8 * 65536];
__device__ unsigned long long pf_tl2[4];   // min CTA entry, last-CTA epilogue start, its end
__device__ unsigned long long pf_tl3[3 * 4096];   // per CTA: entry, after griddepcontrol.wait, after the prologue
__device__ __forceinline__ unsigned long long tl_now() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define TL(v) unsigned long long v = tl_now()
#else
#define TL(v)
#endif

// ------------------------------------------------------- configuration
// Model (pf_model.cuh: D state components, the sample / weight hooks), M
// particles per sub-filter, resampler RES; a group
// of GW warps owns one sub-filter; S groups per CTA; NSTAGE TMA stages per
// group; the per-particle sample/weight loop over a thread's P slots is
// unrolled UNR times (P for full unrolling; 1 keeps one copy of the
// ~10–40 KB per-particle code in the instruction cache).
#ifndef PF_X2_DEFAULT
#define PF_X2_DEFAULT 1
#endif
template <class Model_, int M_, int RES_, int GW_, int S_, int NSTAGE_, int UNR_, int MINB_, int EARLY_ = 0,
          int X2_ = PF_X2_DEFAULT, int SPLIT0_ = 1>
struct KCfg {
  using Model = Model_;
  static constexpr int EARLY = EARLY_;       // start the next TMA load right after the sample loop
  // a group's first block in two bulk copies (log-weight row, then state
  // rows): for mappings whose launch is a few rounds of sub-filters (the
  // launch's first burst is a visible share of the step); the large-shard
  // mappings (tens of rounds) measured +2.5 % with it and leave it out
  static constexpr bool SPLIT0 = SPLIT0_ != 0;
  static constexpr int M = M_, RES = RES_, GW = GW_, S = S_, NSTAGE = NSTAGE_, UNR = UNR_;
  static constexpr int MINB = MINB_;         // __launch_bounds__ min CTAs per SM (register cap)
  static constexpr int D = Model::D;
  static constexpr int E = D + 2;            // mailbox entry: [logw, index bits, x_0..x_{D-1}]
  static constexpr int T = 32 * GW;          // threads per group
  static constexpr int P = M / T;            // particles per thread
  static constexpr int ROW = (D + 1) * M;    // floats per sub-filter block
  static constexpr bool SCAN32 = (M <= 512);  // Q <= M 2^22 fits 32 bits
  static constexpr bool STAGED = UNR < P;    // rolled sample loop: per-slot values via smem
  static constexpr bool X2 = X2_ && (P % 2 == 0);   // two particles at once (packed f32x2)
  static constexpr bool CHUNKED = Model::CHUNKED;   // runtime loop over joint chunks (pf_model.cuh)
  static_assert(P >= 1 && P * T == M, "M must be a multiple of the group size");
  static_assert(P <= 32, "exclusion masks are 32-bit");
  static_assert(S >= 1 && S <= 15, "named barriers 1..S");
  static constexpr int KMAX = 32;            // deg * t <= 32 (validated by the runtime)
  // per-group shared memory
  static constexpr size_t stage_bytes = sizeof(float) * ROW;
  static constexpr size_t g_stage = 0;
  static constexpr size_t g_scan = NSTAGE * stage_bytes;                          // u64 [M]; after the
                                                                                  // resample: Philox words
  // Vose: the second scan, then the alias table: prob u32 [M] + alias u16 [M]
  // when Q <= M 2^22 fits 32 bits (m <= 512), else prob u64 [M] + alias int [M]
  // (the small/large lists live in the stage's log-weight row, free by then)
  static constexpr bool PROB32 = (RES == RES_VOSE) && M <= 512;
  static constexpr size_t g_prob = g_scan + sizeof(u64) * M;                      // u64 [M]  (Vose)
  static constexpr size_t g_alias = g_prob + (RES == RES_VOSE ? sizeof(u64) * M : 0);   // int [M] (!PROB32)
  static constexpr size_t g_red = g_alias + ((RES == RES_VOSE && !PROB32) ? sizeof(int) * M : 0);   // u64 [2][32]
  static constexpr size_t g_cand = g_red + sizeof(u64) * 64;                     // u64 [GW KMAX + GW]
  static constexpr size_t g_misc = g_cand + sizeof(u64) * GW * (KMAX + 1);       // int [GW][2][KMAX]
  // mbarriers: [2] log-weight row of stage 0/1, [2] state rows of stage 0/1; then next [2]
  static constexpr size_t g_bar = g_misc + sizeof(int) * GW * 2 * KMAX;
  static constexpr size_t group_bytes = (g_bar + 48 + 127) / 128 * 128;
  // per-CTA
  static constexpr size_t c_zin = 0;          // float [64]: z (ZD), h_s u (UD)
  static constexpr size_t c_zin2 = 256;       // f2 [64]: the same, each value duplicated (packed operands)
  static constexpr size_t c_groups = 768;
  static constexpr size_t smem = c_groups + S * group_bytes;
  // slot j of group thread t: strided, so chunk j of the group covers the
  // contiguous slots [jT, (j+1)T) and every row store is coalesced
  __device__ __forceinline__ static int slot(int t, int j) { return j * T + t; }
};

// ------------------------------------------------------- group primitives
template <int GW>
__device__ __forceinline__ void gsync(int g) {
  if constexpr (GW == 1) {
    __syncwarp();
  } else {
    asm volatile("bar.sync %0, %1;" ::"r"(g + 1), "n"(32 * GW) : "memory");
  }
}

struct GroupCtx {
  int g;          // group index in the CTA
  int t;          // thread index in the group
  int lane, wig;  // lane, warp in group
  u64* red;       // [2][32] cross-warp reduction slots
  int rb;         // slot toggle (uniform in the group); each call with GW > 1
                  // syncs once, so a slot is reusable two calls later
};

__device__ __forceinline__ u64 warp_max_u64(u64 v) {
  const uint32_t hi = __reduce_max_sync(0xFFFFFFFFu, static_cast<uint32_t>(v >> 32));
  const uint32_t lo =
      __reduce_max_sync(0xFFFFFFFFu, (static_cast<uint32_t>(v >> 32) == hi) ? static_cast<uint32_t>(v) : 0u);
  return (static_cast<u64>(hi) << 32) | lo;
}
__device__ __forceinline__ u64 warp_min_u64(u64 v) {
  const uint32_t hi = __reduce_min_sync(0xFFFFFFFFu, static_cast<uint32_t>(v >> 32));
  const uint32_t lo = __reduce_min_sync(
      0xFFFFFFFFu, (static_cast<uint32_t>(v >> 32) == hi) ? static_cast<uint32_t>(v) : 0xFFFFFFFFu);
  return (static_cast<u64>(hi) << 32) | lo;
}

template <int GW>
__device__ __forceinline__ u64 gmax_u64(u64 v, GroupCtx& G) {
  const u64 w = warp_max_u64(v);
  if constexpr (GW == 1) {
    return w;
  } else {
    u64* r = G.red + G.rb * 32;
    G.rb ^= 1;
    if (G.lane == 0) r[G.wig] = w;
    gsync<GW>(G.g);
    return warp_max_u64(G.lane < GW ? r[G.lane] : 0ull);
  }
}

template <int GW>
__device__ __forceinline__ u64 gsum_u64(u64 v, GroupCtx& G) {
#pragma unroll
  for (int o = 16; o >= 1; o >>= 1) v += __shfl_xor_sync(0xFFFFFFFFu, v, o);
  if constexpr (GW == 1) {
    return v;
  } else {
    u64* r = G.red + G.rb * 32;
    G.rb ^= 1;
    if (G.lane == 0) r[G.wig] = v;
    gsync<GW>(G.g);
    u64 t = 0;
#pragma unroll
    for (int w = 0; w < GW; ++w) t += r[w];
    return t;
  }
}

template <typename X>
__device__ __forceinline__ X warp_incl_scan(X x, int lane) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const X y = __shfl_up_sync(0xFFFFFFFFu, x, o);
    if (lane >= o) x += y;
  }
  return x;
}

// P contiguous elements <-> registers with the widest shared-memory vectors
template <typename X, int P>
__device__ __forceinline__ void vload(const X* src, X (&v)[P]) {
  constexpr int B = P * static_cast<int>(sizeof(X));
  if constexpr (B % 16 == 0) {
#pragma unroll
    for (int i = 0; i < B / 16; ++i) reinterpret_cast<uint4*>(v)[i] = reinterpret_cast<const uint4*>(src)[i];
  } else if constexpr (B % 8 == 0) {
#pragma unroll
    for (int i = 0; i < B / 8; ++i) reinterpret_cast<uint2*>(v)[i] = reinterpret_cast<const uint2*>(src)[i];
  } else {
#pragma unroll
    for (int i = 0; i < P; ++i) v[i] = src[i];
  }
}
template <typename X, int P>
__device__ __forceinline__ void vstore(X* dst, const X (&v)[P]) {
  constexpr int B = P * static_cast<int>(sizeof(X));
  if constexpr (B % 16 == 0) {
#pragma unroll
    for (int i = 0; i < B / 16; ++i) reinterpret_cast<uint4*>(dst)[i] = reinterpret_cast<const uint4*>(v)[i];
  } else if constexpr (B % 8 == 0) {
#pragma unroll
    for (int i = 0; i < B / 8; ++i) reinterpret_cast<uint2*>(dst)[i] = reinterpret_cast<const uint2*>(v)[i];
  } else {
#pragma unroll
    for (int i = 0; i < P; ++i) dst[i] = v[i];
  }
}

// Slot-order inclusive prefix through shared memory: the strided per-thread
// values are transposed (buf[slot]), thread t scans the P contiguous slots
// [tP, tP + P) serially, ONE warp shuffle scan of the per-thread totals (plus
// one cross-warp level) instead of one shuffle scan per slot chunk, and
// buf[s] ends up holding the inclusive prefix of every slot s (slot order).
// Returns the group total.  Group barriers: 2 (+1 when GW > 1).
template <class C, typename X>
__device__ __forceinline__ X slot_scan_smem(const X (&val)[C::P], X* buf, GroupCtx& G) {
  constexpr int P = C::P, GW = C::GW;
#pragma unroll
  for (int j = 0; j < P; ++j) buf[C::slot(G.t, j)] = val[j];
  gsync<GW>(G.g);
  X v[P];
  vload<X, P>(buf + G.t * P, v);
#pragma unroll
  for (int j = 1; j < P; ++j) v[j] += v[j - 1];
  const X tot = v[P - 1];
  const X inc = warp_incl_scan<X>(tot, G.lane);
  X off = inc - tot;
  X total;
  if constexpr (GW == 1) {
    total = __shfl_sync(0xFFFFFFFFu, inc, 31);
  } else {
    X* r = reinterpret_cast<X*>(G.red + G.rb * 32);
    G.rb ^= 1;
    if (G.lane == 31) r[G.wig] = inc;
    gsync<GW>(G.g);
    X before = 0;
    total = 0;
#pragma unroll
    for (int w = 0; w < GW; ++w) {
      const X x = r[w];
      if (w < G.wig) before += x;
      total += x;
    }
    off += before;
  }
#pragma unroll
  for (int j = 0; j < P; ++j) v[j] += off;
  vstore<X, P>(buf + G.t * P, v);
  gsync<GW>(G.g);
  return total;
}

// One level of the RWS binary search over u32 inclusive sums in shared
// memory: a += INC if sums[a + OFF] <= c (byte addresses).
template <int OFF, int INC>
__device__ __forceinline__ void search_step(uint32_t& a, uint32_t c) {
  asm("{\n\t.reg .pred p;\n\t.reg .u32 v;\n\t"
      "ld.shared.u32 v, [%0+%2];\n\t"
      "setp.le.u32 p, v, %1;\n\t"
      "@p add.u32 %0, %0, %3;\n\t}"
      : "+r"(a)
      : "r"(c), "n"(OFF), "n"(INC));
}

template <int S>
__device__ __forceinline__ void search_levels(uint32_t& a, uint32_t c) {
  search_step<4 * (S - 1), 4 * S>(a, c);
  if constexpr (S > 1) search_levels<S / 2>(a, c);
}

// ---------------------------------------------------------- resampling
struct ResampleSmem {
  u64* scan;    // [M] RWS: inclusive sums C (u32 or u64); Vose: exclusive D over L, then E over H
  u64* prob;    // [M] Vose: the second scan, then the table (KCfg::PROB32: u32 prob [M] + u16 alias [M])
  int* alias;   // [M] Vose, !PROB32
  int* lists;   // [M] Vose: L ascending then H ascending (the stage's log-weight row)
};

// Ancestors anc[P] of the thread's slots (a8) from integer weights q[P]
// (a7) and uniforms ua/ub (R9–R11).  All threads of the group call it.
template <class C>
__device__ __forceinline__ void resample_group(const uint32_t (&q)[C::P], const uint32_t (&ua)[C::P],
                                               const uint32_t (&ub)[C::P], int (&anc)[C::P],
                                               const ResampleSmem& S, GroupCtx& G, u64* prob_out,
                                               int* alias_out) {
  constexpr int P = C::P, M = C::M;
  if constexpr (C::RES == RES_RWS) {
    // Roulette Wheel Selection (§VI-F): C = inclusive sums of q
    // in slot order, c = floor(U Q / 2^32), ancestor = first j with C_j > c.
    using X = typename std::conditional<C::SCAN32, uint32_t, u64>::type;
    X val[P];
#pragma unroll
    for (int j = 0; j < P; ++j) val[j] = q[j];
    X* Cs = reinterpret_cast<X*>(S.scan);
    const X Q = slot_scan_smem<C, X>(val, Cs, G);   // Cs[s] = inclusive sum of slot s
#pragma unroll
    for (int j = 0; j < P; ++j) {
      const X c = static_cast<X>((static_cast<u64>(ua[j]) * Q) >> 32);
      if constexpr (C::SCAN32) {
        // branch-free search on the shared-memory byte address: per level one
        // LDS at an immediate offset, one compare, one predicated add
        uint32_t a = smem_u32(Cs);
        const uint32_t a0 = a;
        search_levels<M / 2>(a, c);
        anc[j] = static_cast<int>((a - a0) >> 2);
      } else {
        int pos = 0;
#pragma unroll
        for (int s = M / 2; s >= 1; s >>= 1)
          if (Cs[pos + s - 1] <= c) pos += s;
        anc[j] = pos;
      }
    }
  } else {
    // Vose's alias method (PAPER.md:18 §IV, :20–22 §VI-F), table by the
    // closed form of the sequential sweep (R10): a_j = M q_j, small L =
    // {a < Q}, D = inclusive deficits over L, E = inclusive excesses over H.
    // Two slot-order prefix sums: the weights (-> the prefix of a = M q), and
    // the deficits over L with the count of L packed above bit 48 (D < 2^42).
    // E follows from sum_{j'<=j} (a_j' - Q) = E_j - D_j.
    u64 Qg, Dtot;
    int nL;
    if constexpr (C::SCAN32) {
      // Q <= M 2^22 fits 32 bits.  Q first (warp REDUX + one group barrier),
      // then ONE transposition of q into slot order: thread t classifies its
      // CONTIGUOUS slots [tP, tP + P) itself and scans, in registers, both the
      // weights (u32) and the packed deficits (u64) — one warp scan level and
      // one cross-warp level for the two — and writes its list entries
      // straight from registers (no scan results stored back to shared memory
      // and re-read).  4 group barriers per table instead of 8; the same
      // sums, hence the same table.
      uint32_t qs = 0;
#pragma unroll
      for (int j = 0; j < P; ++j) qs += q[j];
      qs = __reduce_add_sync(0xFFFFFFFFu, qs);
      if constexpr (C::GW > 1) {
        uint32_t* r = reinterpret_cast<uint32_t*>(G.red + G.rb * 32);
        G.rb ^= 1;
        if (G.lane == 0) r[G.wig] = qs;
        uint32_t* b32 = reinterpret_cast<uint32_t*>(S.scan);
#pragma unroll
        for (int j = 0; j < P; ++j) b32[C::slot(G.t, j)] = q[j];
        gsync<C::GW>(G.g);
        qs = 0;
#pragma unroll
        for (int w = 0; w < C::GW; ++w) qs += r[w];
      } else {
        uint32_t* b32 = reinterpret_cast<uint32_t*>(S.scan);
#pragma unroll
        for (int j = 0; j < P; ++j) b32[C::slot(G.t, j)] = q[j];
        __syncwarp();
      }
      const uint32_t Q32 = qs;
      Qg = Q32;
      uint32_t qc[P], qi[P];   // contiguous slots tP + e: weight, inclusive weight sum
      u64 pc[P];               // packed inclusive deficit sum (count of L above bit 48)
      vload<uint32_t, P>(reinterpret_cast<const uint32_t*>(S.scan) + G.t * P, qc);
#pragma unroll
      for (int e = 0; e < P; ++e) {
        const u64 a = static_cast<u64>(M) * qc[e];
        const u64 pk0 = a < Qg ? (Qg - a) + (1ull << 48) : 0ull;
        qi[e] = e ? qi[e - 1] + qc[e] : qc[e];
        pc[e] = e ? pc[e - 1] + pk0 : pk0;
      }
      const uint32_t tq = qi[P - 1];
      const u64 tp = pc[P - 1];
      const uint32_t iq = warp_incl_scan<uint32_t>(tq, G.lane);
      const u64 ip = warp_incl_scan<u64>(tp, G.lane);
      uint32_t oq = iq - tq;
      u64 op = ip - tp, ptot;
      if constexpr (C::GW == 1) {
        ptot = __shfl_sync(0xFFFFFFFFu, ip, 31);
      } else {
        u64* r = G.red + G.rb * 32;
        G.rb ^= 1;
        if (G.lane == 31) {
          r[G.wig] = ip;
          r[16 + G.wig] = iq;
        }
        gsync<C::GW>(G.g);
        ptot = 0;
#pragma unroll
        for (int w = 0; w < C::GW; ++w) {
          const u64 xp = r[w];
          if (w < G.wig) {
            op += xp;
            oq += static_cast<uint32_t>(r[16 + w]);
          }
          ptot += xp;
        }
      }
      nL = static_cast<int>(ptot >> 48);
      Dtot = ptot & ((1ull << 48) - 1);
      // (every thread's transposition reads precede the barrier above, so the
      // lists may now overwrite S.scan)
#pragma unroll
      for (int e = 0; e < P; ++e) {
        const int s = G.t * P + e;
        const u64 a = static_cast<u64>(M) * qc[e];
        const bool small = a < Qg;
        const u64 pinc = pc[e] + op;
        const u64 Dinc = pinc & ((1ull << 48) - 1);
        const int ls = static_cast<int>(pinc >> 48) - (small ? 1 : 0);   // smalls before the slot
        if (small) {
          S.lists[ls] = s;
          S.scan[ls] = Dinc - (Qg - a);
        } else {   // E_s = D_s + sum_{s' <= s} (a_s' - Q): 32 x 32 -> 64-bit products
          S.lists[nL + (s - ls)] = s;
          S.scan[nL + (s - ls)] = Dinc + static_cast<u64>(qi[e] + oq) * static_cast<uint32_t>(M) -
                                  static_cast<u64>(static_cast<uint32_t>(s) + 1u) * Q32;
        }
      }
    } else {   // m = 1024: Q up to 2^32, both scans in u64 through shared memory
      u64 qinc[P], pinc[P];
      u64 ptot;
      {
        u64 val[P];
#pragma unroll
        for (int j = 0; j < P; ++j) val[j] = q[j];
        Qg = slot_scan_smem<C, u64>(val, S.scan, G);
#pragma unroll
        for (int j = 0; j < P; ++j) qinc[j] = S.scan[C::slot(G.t, j)];
      }
      {
        u64 packed[P];
#pragma unroll
        for (int j = 0; j < P; ++j) {
          const u64 a = static_cast<u64>(M) * q[j];
          packed[j] = a < Qg ? (Qg - a) + (1ull << 48) : 0ull;
        }
        ptot = slot_scan_smem<C, u64>(packed, S.prob, G);
#pragma unroll
        for (int j = 0; j < P; ++j) pinc[j] = S.prob[C::slot(G.t, j)];
      }
      // (every thread read qinc before passing scan 2's barriers: S.scan is free)
      nL = static_cast<int>(ptot >> 48);
      Dtot = ptot & ((1ull << 48) - 1);
      // Lists: small slots ascending with their EXCLUSIVE deficit sums A_i =
      // D_{i-1} (A_0 = 0) at [0, nL), large slots ascending with their
      // inclusive excess sums E_j at [nL, M) (both sequences sorted).
#pragma unroll
      for (int j = 0; j < P; ++j) {
        const u64 a = static_cast<u64>(M) * q[j];
        const bool small = a < Qg;
        const u64 Dinc = pinc[j] & ((1ull << 48) - 1);
        const int ls = static_cast<int>(pinc[j] >> 48) - (small ? 1 : 0);   // smalls before the slot
        const int s = C::slot(G.t, j);
        if (small) {
          S.lists[ls] = s;
          S.scan[ls] = Dinc - (Qg - a);
        } else {   // E_s = D_s + sum_{s' <= s} (a_s' - Q)
          S.lists[nL + (s - ls)] = s;
          S.scan[nL + (s - ls)] = Dinc + static_cast<u64>(M) * qinc[j] - static_cast<u64>(s + 1) * Qg;
        }
      }
    }
    gsync<C::GW>(G.g);
    // The closed form of the sweep (R10) is a MERGE of the sorted sequences
    // A (small) and E (large) with "A first on ties":
    //   small L[i]: alias = H[lower_bound(E, A_i)] = H[#E before A_i],
    //               prob = a = Q - (A_{i+1} - A_i)   (A_nL := D_last);
    //   large H[j] with E_j < D_last: prob = Q + E_j - D[upper_bound(D, E_j)]
    //               = Q + E_j - (the next A after E_j in merge order, or D_last),
    //               alias = H[j + 1]; otherwise prob = Q, alias = itself.
    // Merge path: thread t emits merged positions [tP, tP + P) after ONE
    // binary search for its split on the diagonal (instead of one search per
    // slot), then P sequential merge steps.
    {
      const int nH = M - nL;
      const int diag = G.t * P;
      int lo = diag - nH > 0 ? diag - nH : 0, hi = diag < nL ? diag : nL;
      while (lo < hi) {   // first i with A_i > E_{diag-1-i} (A before E on ties)
        const int mid = (lo + hi) >> 1;
        if (S.scan[mid] <= S.scan[nL + diag - 1 - mid]) lo = mid + 1;
        else hi = mid;
      }
      int i = lo, jj = diag - lo;
      u64 Ai = i < nL ? S.scan[i] : Dtot;        // head of A (D_last past the end)
      u64 Bj = jj < nH ? S.scan[nL + jj] : ~0ull;
#pragma unroll
      for (int e = 0; e < P; ++e) {
        int s, al;
        u64 pr;
        if (i < nL && Ai <= Bj) {   // small slot L[i]
          s = S.lists[i];
          const u64 An = i + 1 < nL ? S.scan[i + 1] : Dtot;
          pr = Qg - (An - Ai);
          al = S.lists[nL + jj];
          ++i;
          Ai = An;
        } else {                    // large slot H[jj]
          s = S.lists[nL + jj];
          if (Bj < Dtot) {
            pr = Qg + Bj - Ai;
            al = S.lists[nL + jj + 1];
          } else {
            pr = Qg;
            al = s;
          }
          ++jj;
          Bj = jj < nH ? S.scan[nL + jj] : ~0ull;
        }
        if constexpr (C::PROB32) {
          reinterpret_cast<uint32_t*>(S.prob)[s] = static_cast<uint32_t>(pr);
          reinterpret_cast<uint16_t*>(reinterpret_cast<uint32_t*>(S.prob) + M)[s] = static_cast<uint16_t>(al);
        } else {
          S.prob[s] = pr;
          S.alias[s] = al;
        }
        if (prob_out) {
          prob_out[s] = pr;
          alias_out[s] = al;
        }
      }
    }
    const u64 Q2 = Qg;
    gsync<C::GW>(G.g);
#pragma unroll
    for (int j = 0; j < P; ++j) {
      const int b = static_cast<int>((static_cast<u64>(ua[j]) * M) >> 32);
      if constexpr (C::PROB32) {   // Q < 2^32: c = the high word of one 32 x 32 product
        const uint32_t c = __umulhi(ub[j], static_cast<uint32_t>(Q2));
        const uint32_t* p32 = reinterpret_cast<const uint32_t*>(S.prob);
        anc[j] = c < p32[b] ? b : reinterpret_cast<const uint16_t*>(p32 + M)[b];
      } else {
        const u64 c = (static_cast<u64>(ub[j]) * Q2) >> 32;
        anc[j] = c < S.prob[b] ? b : S.alias[b];
      }
    }
  }
}

// ------------------------------------------------------------ topology
// Mailbox row of neighbour qi of local sub-filter g (global index) — rows
// [0, n_local) are the shard's own sub-filters, [n_local, n_ext) the halo
// rows of pf.h pf_shard.  Ring (R3): [g-1, g+1] mod N; 2D torus (R4): [up,
// down, left, right] with wrap; a shard holds whole grid rows, so left/right
// are always local and up/down leave the shard only at its first/last row.
__device__ __forceinline__ long long neighbor_row(const StepParams& P, long long g64, int qi) {
  // 32-bit arithmetic: N m <= 2^32 with m >= 32 keeps every index below 2^27
  const int N = static_cast<int>(P.n_global), g = static_cast<int>(g64);
  const int g0 = static_cast<int>(P.g0), nl = static_cast<int>(P.n_local);
  if (P.topo == TOPO_A2A) return P.pool_row;
  if (P.topo == TOPO_RING) {
    const int q = qi == 0 ? (g == 0 ? N - 1 : g - 1) : (g == N - 1 ? 0 : g + 1);
    const int loc = q - g0;
    if (static_cast<unsigned>(loc) < static_cast<unsigned>(nl)) return loc;
    return qi == 0 ? nl : nl + 1;
  }
  const int C = static_cast<int>(P.C), R = static_cast<int>(P.R);
  const int loc = g - g0;
  const int lr = loc / C, c = loc - lr * C;
  const int rows = nl / C;
  switch (qi) {
    case 0: return lr > 0 ? loc - C : (rows == R ? (R - 1) * C + c : nl + c);
    case 1: return lr < rows - 1 ? loc + C : (rows == R ? c : nl + C + c);
    case 2: return lr * C + (c == 0 ? C - 1 : c - 1);
    default: return lr * C + (c == C - 1 ? 0 : c + 1);
  }
}

// ------------------------------------------------------------ sampling
// Process noise of one particle, Box–Muller pair by pair (R12, R13): pair qp
// uses Philox words w = 2+2qp, 3+2qp of block w/4; block 0 (words 0–1 = the
// resampling draw) is supplied by the caller (its words 2, 3 in blk.z/.w).
struct NoiseGen {
  uint32_t p, k;
  const uint32_t (&rk)[20];
  u32x4 blk;
  template <int QP>
  __device__ __forceinline__ void pair(float& z0, float& z1) {
    constexpr int w = 2 + 2 * QP;
    if constexpr ((w & 3) == 0) blk = philox4x32_10_rk(p, k, 0u, static_cast<uint32_t>(w >> 2), rk);
    const uint32_t x0 = (w & 3) == 2 ? blk.z : blk.x;
    const uint32_t x1 = (w & 3) == 2 ? blk.w : blk.y;
    normal_pair(x0, x1, z0, z1);
  }
};

// Streamed sample + weight of one particle (F8–F10) through the model's
// take<c> hooks, Box–Muller pair by pair; out(c, v) stores component c of
// the new state.
template <class Model, int QP>
struct SampleStream {
  static constexpr int D = Model::D;
  template <typename X, typename O>
  __device__ __forceinline__ static void run(const ModelConsts& mc, const float* hsu, const float* z, const X& x,
                                             NoiseGen& gen, typename Model::Acc& A, const O& out) {
    float z0, z1;
    gen.template pair<QP>(z0, z1);
    out(2 * QP, Model::template take<2 * QP>(mc, hsu, z, x, z0, A));
    if constexpr (2 * QP + 1 < D) out(2 * QP + 1, Model::template take<2 * QP + 1>(mc, hsu, z, x, z1, A));
    if constexpr (QP + 1 < (D + 1) / 2) SampleStream<Model, QP + 1>::run(mc, hsu, z, x, gen, A, out);
  }
};

// Two particles A, B at once: the same Philox words per particle, the
// Box–Muller arithmetic packed (normal_pair2).
struct NoiseGen2 {
  uint32_t pa, pb, k;
  const uint32_t (&rk)[20];
  u32x4 ba, bb;
  template <int QP>
  __device__ __forceinline__ void pair(f2& z0, f2& z1) {
    constexpr int w = 2 + 2 * QP;
    if constexpr ((w & 3) == 0) {
      ba = philox4x32_10_rk(pa, k, 0u, static_cast<uint32_t>(w >> 2), rk);
      bb = philox4x32_10_rk(pb, k, 0u, static_cast<uint32_t>(w >> 2), rk);
    }
    normal_pair2((w & 3) == 2 ? ba.z : ba.x, (w & 3) == 2 ? ba.w : ba.y, (w & 3) == 2 ? bb.z : bb.x,
                 (w & 3) == 2 ? bb.w : bb.y, z0, z1);
  }
};

template <class Model, int QP>
struct SampleStream2 {
  static constexpr int D = Model::D;
  template <typename X, typename O>
  __device__ __forceinline__ static void run(const ModelConsts2& mc, const f2* hsu2, const f2* z2, const X& x,
                                             NoiseGen2& gen, typename Model::Acc2& A, const O& out) {
    f2 z0, z1;
    gen.template pair<QP>(z0, z1);
    out(2 * QP, Model::template take2<2 * QP>(mc, hsu2, z2, x, z0, A));
    if constexpr (2 * QP + 1 < D) out(2 * QP + 1, Model::template take2<2 * QP + 1>(mc, hsu2, z2, x, z1, A));
    if constexpr (QP + 1 < (D + 1) / 2) SampleStream2<Model, QP + 1>::run(mc, hsu2, z2, x, gen, A, out);
  }
};

// The same streamed sample + weight as SampleStream / SampleStream2 for large
// states (Model::CHUNKED), with the middle of the chain as a runtime loop:
// pair 0 (components 0, 1; block 0 words 2-3 supplied) static, then NC
// chunks of four components 2 + 4i .. 5 + 4i (Model::joint) that use exactly
// Philox block i + 1 (words 4-7 of the chunk), then the remaining components
// static from pair 1 + 2 NC on.  One copy of four components' code instead of
// d (instruction cache), identical arithmetic in the same order.
template <class Model>
struct SampleChunked {
  static constexpr int NC = Model::NC;
  template <typename X, typename O>
  __device__ __forceinline__ static void run(const ModelConsts& mc, const float* hsu, const float* z, const X& x,
                                             NoiseGen& gen, typename Model::Acc& A, const O& out) {
    {
      float z0, z1;
      gen.template pair<0>(z0, z1);
      out(0, Model::template take<0>(mc, hsu, z, x, z0, A));
      out(1, Model::template take<1>(mc, hsu, z, x, z1, A));
    }
#pragma unroll 1
    for (int i = 0; i < NC; ++i) {
      const int c = 2 + 4 * i;
      const u32x4 b = philox4x32_10_rk(gen.p, gen.k, 0u, static_cast<uint32_t>(i + 1), gen.rk);
      float n0, n1, n2, n3;
      normal_pair(b.x, b.y, n0, n1);
      normal_pair(b.z, b.w, n2, n3);
      out(c, Model::joint(c, mc, hsu, z, x, n0, A));
      out(c + 1, Model::joint(c + 1, mc, hsu, z, x, n1, A));
      out(c + 2, Model::joint(c + 2, mc, hsu, z, x, n2, A));
      out(c + 3, Model::joint(c + 3, mc, hsu, z, x, n3, A));
    }
    SampleStream<Model, 1 + 2 * NC>::run(mc, hsu, z, x, gen, A, out);
  }
};

template <class Model>
struct SampleChunked2 {
  static constexpr int NC = Model::NC;
  template <typename X, typename O>
  __device__ __forceinline__ static void run(const ModelConsts2& mc, const f2* hsu2, const f2* z2, const X& x,
                                             NoiseGen2& gen, typename Model::Acc2& A, const O& out) {
    {
      f2 z0, z1;
      gen.template pair<0>(z0, z1);
      out(0, Model::template take2<0>(mc, hsu2, z2, x, z0, A));
      out(1, Model::template take2<1>(mc, hsu2, z2, x, z1, A));
    }
#pragma unroll 1
    for (int i = 0; i < NC; ++i) {
      const int c = 2 + 4 * i;
      const u32x4 ba = philox4x32_10_rk(gen.pa, gen.k, 0u, static_cast<uint32_t>(i + 1), gen.rk);
      const u32x4 bb = philox4x32_10_rk(gen.pb, gen.k, 0u, static_cast<uint32_t>(i + 1), gen.rk);
      f2 n0, n1, n2, n3;
      normal_pair2(ba.x, ba.y, bb.x, bb.y, n0, n1);
      normal_pair2(ba.z, ba.w, bb.z, bb.w, n2, n3);
      out(c, Model::joint2(c, mc, hsu2, z2, x, n0, A));
      out(c + 1, Model::joint2(c + 1, mc, hsu2, z2, x, n1, A));
      out(c + 2, Model::joint2(c + 2, mc, hsu2, z2, x, n2, A));
      out(c + 3, Model::joint2(c + 3, mc, hsu2, z2, x, n3, A));
    }
    SampleStream2<Model, 1 + 2 * NC>::run(mc, hsu2, z2, x, gen, A, out);
  }
};

// Streamed sample + weight with RUNTIME dimensions (the generic arm): the
// same Box–Muller pairing, Philox words and per-component arithmetic as
// SampleStream, as a loop over pairs (block 0 words 2-3 supplied).
template <class Model>
struct SampleRuntime {
  template <typename X, typename O>
  __device__ __forceinline__ static void run(const ModelConsts& mc, int nj, const float* hsu, const float* z,
                                             const X& x, NoiseGen& gen, typename Model::Acc& A, const O& out) {
    const int d = nj + 4;
    u32x4 blk = gen.blk;
#pragma unroll 1
    for (int q = 0; q < (d + 1) / 2; ++q) {
      const int w = 2 + 2 * q;
      if ((w & 3) == 0) blk = philox4x32_10_rk(gen.p, gen.k, 0u, static_cast<uint32_t>(w >> 2), gen.rk);
      float z0, z1;
      normal_pair((w & 3) == 2 ? blk.z : blk.x, (w & 3) == 2 ? blk.w : blk.y, z0, z1);
      out(2 * q, Model::take_rt(2 * q, nj, mc, hsu, z, x, z0, A));
      if (2 * q + 1 < d) out(2 * q + 1, Model::take_rt(2 * q + 1, nj, mc, hsu, z, x, z1, A));
    }
  }
};

template <class Model>
struct SampleRuntime2 {
  template <typename X, typename O>
  __device__ __forceinline__ static void run(const ModelConsts2& mc, int nj, const f2* hsu2, const f2* z2, const X& x,
                                             NoiseGen2& gen, typename Model::Acc2& A, const O& out) {
    const int d = nj + 4;
    u32x4 ba = gen.ba, bb = gen.bb;
#pragma unroll 1
    for (int q = 0; q < (d + 1) / 2; ++q) {
      const int w = 2 + 2 * q;
      if ((w & 3) == 0) {
        ba = philox4x32_10_rk(gen.pa, gen.k, 0u, static_cast<uint32_t>(w >> 2), gen.rk);
        bb = philox4x32_10_rk(gen.pb, gen.k, 0u, static_cast<uint32_t>(w >> 2), gen.rk);
      }
      const bool hi = (w & 3) == 2;
      f2 z0, z1;
      normal_pair2(hi ? ba.z : ba.x, hi ? ba.w : ba.y, hi ? bb.z : bb.x, hi ? bb.w : bb.y, z0, z1);
      out(2 * q, Model::take_rt2(2 * q, nj, mc, hsu2, z2, x, z0, A));
      if (2 * q + 1 < d) out(2 * q + 1, Model::take_rt2(2 * q + 1, nj, mc, hsu2, z2, x, z1, A));
    }
  }
};

// Peer transport, halo rows (reading R3/R4 and the halo plan of
// distributed.py): ring — local sub-filter 0 -> the previous rank's row
// n_local + 1, the last -> the next rank's row n_local; torus — the first grid
// row -> the rank above, rows n_local + C + c, the last grid row -> the rank
// below, rows n_local + c.  The rows' first t entries [logw, index bits, x],
// copied by the last CTA (every row is complete; no code in the step loop).
static __device__ void peer_halo_rows(const StepParams& P, int E) {   // whole CTA (the last one)
  const long long nl = P.n_local, par = static_cast<long long>(P.k & 1u) * P.mb_parity;
  const int per = P.t * E;                                  // the row's first t entries
  const long long Cc = P.topo == TOPO_RING ? 1 : P.C;       // rows per side
  const long long total = 2 * Cc * per;
  for (long long i = threadIdx.x; i < total; i += blockDim.x) {
    const int side = static_cast<int>(i / (Cc * per));      // 0: -> previous rank, 1: -> next rank
    const long long j = i - side * Cc * per;
    const long long c = j / per;
    const int e = static_cast<int>(j - c * per);
    long long src, dst;
    if (P.topo == TOPO_RING) {
      src = side == 0 ? 0 : nl - 1;
      dst = side == 0 ? nl + 1 : nl;
    } else {
      src = side == 0 ? c : nl - Cc + c;
      dst = side == 0 ? nl + Cc + c : nl + c;
    }
    P.peer_mb[side][par + dst * P.tt * E + e] = __ldcg(P.mb_cur + src * P.tt * E + e);
  }
}

__device__ __forceinline__ unsigned long long* peer_flags(unsigned char* blk) {
  return reinterpret_cast<unsigned long long*>(blk);
}
// record / pool row of rank r in buffer par (= rendezvous number & 1)
__device__ __forceinline__ float* peer_rec(unsigned char* blk, int par, int r) {
  return reinterpret_cast<float*>(blk + sizeof(unsigned long long) * kMaxRanks) + (par * kMaxRanks + r) * kPeerRec;
}
__device__ __forceinline__ float* peer_pool(unsigned char* blk, int par, int r) {
  return reinterpret_cast<float*>(blk + sizeof(unsigned long long) * kMaxRanks) + 2 * kMaxRanks * kPeerRec +
         (par * kMaxRanks + r) * kPeerPool;
}
__device__ __forceinline__ unsigned long long global_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Best t of the union of two descending lists held by lanes 0..t-1 (run list
// r, new list nb; keys unique or 0 = empty) into r, by t rounds of warp max.
__device__ __forceinline__ void top_t_merge(u64& rk, u64& rl, u64 nk, u64 nl, int t, int lane) {
  u64 a = lane < t ? rk : 0ull, b = lane < t ? nk : 0ull;
  u64 ok = 0ull, ol = 0ull;
  for (int r = 0; r < t; ++r) {
    const u64 c = a > b ? a : b;
    const u64 w = warp_max_u64(c);
    const bool own = w != 0ull && c == w;
    const int owner = __ffs(__ballot_sync(0xFFFFFFFFu, own)) - 1;
    const u64 wl = __shfl_sync(0xFFFFFFFFu, a == w ? rl : nl, owner < 0 ? 0 : owner);
    if (own) {
      if (a == w) a = 0ull;
      else b = 0ull;
    }
    if (lane == r) {
      ok = w;
      ol = owner < 0 ? 0ull : wl;
    }
  }
  rk = ok;
  rl = ol;
}

// All-to-All pool from the per-group best t (pool_cta rows of the groups
// that processed a sub-filter: static first index gid0 < n_local): the best t
// of those candidates, entries copied from the mailbox.  Whole CTA.
static __device__ void pool_top_t_cta(const StepParams& P, float* out, u64* red, long long groups, int E) {   // red: 66 u64
  u64* red_k = red;
  u64* red_l = red + 33;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nw = (blockDim.x + 31) >> 5;
  const long long count = (groups < P.n_local ? groups : P.n_local) * P.tt;
  u64 prev = ~0ull;
  for (int jb = 0; jb < P.t; ++jb) {
    u64 best = 0ull, bl = 0ull;
    for (long long i = tid; i < count; i += blockDim.x) {
      const u64 key = __ldcg(P.pool_cta + 2 * i);
      if (key < prev && key > best) {
        best = key;
        bl = __ldcg(P.pool_cta + 2 * i + 1);
      }
    }
    const u64 wbest = warp_max_u64(best);
    if (best == wbest && wbest != 0ull) {   // unique owner in the warp
      red_k[warp] = wbest;
      red_l[warp] = bl;
    } else if (lane == 0 && wbest == 0ull) {
      red_k[warp] = 0ull;
    }
    __syncthreads();
    if (warp == 0) {
      const u64 k = lane < nw ? red_k[lane] : 0ull;
      const u64 v = warp_max_u64(k);
      if (v != 0ull && k == v) {
        red_k[32] = v;
        red_l[32] = red_l[lane];
      }
      if (lane == 0 && v == 0ull) red_k[32] = 0ull;
    }
    __syncthreads();
    const u64 g = red_k[32];
    const float* en = P.mb_cur + static_cast<long long>(red_l[32]) * E;
    if (g != 0ull)
      for (int c = tid; c < E; c += blockDim.x) out[jb * E + c] = __ldcg(en + c);
    prev = g;
    __syncthreads();
  }
}

// All-to-All pool (§VI-E): the best t of `count` mailbox entries
// (entry e = row e / t, item e % t, E floats [logw, index bits, x]) by the
// order key of R6, copied to out[0..t) in order.  Whole CTA; t rounds.
static __device__ void pool_top_t(const StepParams& P, const float* mb, long long count, float* out, u64* pool_red, int E) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nw = (blockDim.x + 31) >> 5;
  u64 prev = ~0ull;
  for (int jb = 0; jb < P.t; ++jb) {
    u64 best = 0ull;
    long long be = -1;
    for (long long e = tid; e < count; e += blockDim.x) {
      const long long row = e / P.t, jj = e - row * P.t;
      const float* en = mb + (row * P.tt + jj) * E;
      const u64 key = order_key(__ldcg(en), __float_as_uint(__ldcg(en + 1)));
      if (key < prev && key > best) {
        best = key;
        be = e;
      }
    }
    const u64 wbest = warp_max_u64(best);
    if (lane == 0) pool_red[warp] = wbest;
    __syncthreads();
    if (warp == 0) {
      const u64 v = warp_max_u64(lane < nw ? pool_red[lane] : 0ull);
      if (lane == 0) pool_red[32] = v;
    }
    __syncthreads();
    const u64 g = pool_red[32];
    if (best == g && be >= 0) {   // unique owner (the index is part of the key)
      const long long row = be / P.t, jj = be - row * P.t;
      const float* en = mb + (row * P.tt + jj) * E;
      for (int c = 0; c < E; ++c) out[jb * E + c] = __ldcg(en + c);
    }
    prev = g;
    __syncthreads();
  }
}

// ------------------------------------------------------------ the kernel
template <class C>
__global__ void __launch_bounds__(C::T* C::S, C::MINB) pf_step_kernel(const __grid_constant__ StepParams P) {
#ifdef PF_TIMELINE
  const unsigned long long tl_entry = tl_now();
  if (threadIdx.x == 0) atomicMin(&pf_tl2[0], tl_entry);
#endif
  using Model = typename C::Model;
  constexpr int M = C::M, GW = C::GW, PP = C::P;
  // dimensions: compile-time for the compiled models; the generic arm
  // (Model::RUNTIME) takes them from the launch (its shared-memory stage is
  // sized for its largest state, the HBM block and mailbox entry are exact)
  constexpr bool RT = Model::RUNTIME;
  const int D = RT ? P.d : C::D;
  const int E = D + 2;
  const int ZD = RT ? P.nj + 2 : Model::ZD;
  const int UD = RT ? P.nj : Model::UD;
  const long long ROW = static_cast<long long>(D + 1) * M;                  // floats per HBM block
  const uint32_t stage_bytes = RT ? static_cast<uint32_t>(sizeof(float) * ROW) : static_cast<uint32_t>(C::stage_bytes);
  extern __shared__ __align__(128) unsigned char smem[];
  float* z_s = reinterpret_cast<float*>(smem + C::c_zin);
  float* hsu_s = z_s + ZD;
  f2* z2_s = reinterpret_cast<f2*>(smem + C::c_zin2);
  f2* hsu2_s = z2_s + ZD;

  const int g = threadIdx.x / C::T;
  unsigned char* gs = smem + C::c_groups + g * C::group_bytes;
  u64* bars = reinterpret_cast<u64*>(gs + C::g_bar);
  ResampleSmem S;
  S.scan = reinterpret_cast<u64*>(gs + C::g_scan);
  S.prob = reinterpret_cast<u64*>(gs + C::g_prob);
  S.alias = reinterpret_cast<int*>(gs + C::g_alias);
  S.lists = nullptr;   // per sub-filter: the stage's log-weight row
  uint2* bzw_s = reinterpret_cast<uint2*>(gs + C::g_scan);       // STAGED: Philox words after the resample
  volatile unsigned int* next_s = reinterpret_cast<unsigned int*>(gs + C::g_bar + 32);
  GroupCtx G;
  G.g = g;
  G.t = threadIdx.x - g * C::T;
  G.lane = threadIdx.x & 31;
  G.wig = G.t >> 5;
  G.red = reinterpret_cast<u64*>(gs + C::g_red);
  G.rb = 0;
  u64* cand = reinterpret_cast<u64*>(gs + C::g_cand);             // [GW * K] candidates, [GW] maxima at GW * KMAX
  int* wlist = reinterpret_cast<int*>(gs + C::g_misc) + G.wig * 2 * C::KMAX;   // this warp's copy: worst slots
  int* woff = wlist + C::KMAX;                                                  // mailbox offsets of the incoming

  const int mode = P.mode;
  const bool do_merge = (mode == MODE_EXCHANGE) || (mode == MODE_STEP && !P.first);
  const bool do_resample = (mode == MODE_STEP && !P.first);
  const bool do_sample = (mode == MODE_STEP || mode == MODE_SAMPLE);
  const int K = P.deg * P.t;
  const long long gid0 = static_cast<long long>(blockIdx.x) * C::S + g;
  const long long gstride = static_cast<long long>(gridDim.x) * C::S;

  // Work distribution: the group's first sub-filter is blockIdx.x * S + g;
  // later ones come from the launch's work counter (dynamic, so SMs that
  // finish early take more).  Thread 0 announces each next index through
  // next_s[barrier] before arriving on that barrier (release / acquire), and
  // a "no more work" index completes the barrier phase without a copy.
  // A group's FIRST sub-filter arrives in two bulk copies: its log-weight
  // row (row D of the block) on barrier b, and — requested only once that
  // row has landed, so that every group's log-weights come first — its D
  // state rows on barrier 2 + b.  The exchange selection, normalisation and
  // resampler need only the log-weights, so at the launch's start — when
  // every group's first block comes from HBM at once, ~18 MB at C2 — a group
  // works on them while the state rows (9/10 of the bytes) are in flight.  Later sub-filters
  // (their loads overlap the previous sub-filter's work, from L2 after the
  // prefetch) come in one copy on barrier b; barrier 2 + b then completes at
  // once.  (Splitting every load measured +3 % at 16M particles.)
  const uint32_t lw_bytes = static_cast<uint32_t>(sizeof(float) * M);
  const uint32_t st_bytes = stage_bytes - lw_bytes;
  auto issue = [&](int b, long long nn, bool split) {   // thread 0 only
    next_s[b] = static_cast<unsigned int>(nn < P.n_local ? nn : P.n_local);
    unsigned char* dst = gs + C::g_stage + b * C::stage_bytes;
    const float* src = P.parts + nn * ROW;
    if (C::SPLIT0 && nn < P.n_local && split) {   // (the state rows: issue_states)
      mbar_arrive_expect_tx(bars + b, lw_bytes);
      bulk_g2s(dst + st_bytes, src + static_cast<long long>(D) * M, lw_bytes, bars + b);
    } else {
      if (nn < P.n_local) {
        mbar_arrive_expect_tx(bars + b, stage_bytes);
        bulk_g2s(dst, src, stage_bytes, bars + b);
      } else {
        mbar_arrive(bars + b);
      }
      if constexpr (C::SPLIT0) mbar_arrive(bars + 2 + b);
    }
  };
  // thread 0 keeps one dynamic index in flight: the atomic's latency is
  // hidden behind a whole sub-filter of work.  The ticket is taken with a
  // plain PTX atom: atomicAdd() is compiled into a warp-aggregated atomic
  // whose result is shuffled to the lanes at once, i.e. consumed right away,
  // which stalled thread 0's warp (and at the next barrier its group) for the
  // atomic's round trip on every sub-filter, and the launch's prologue for
  // the burst of same-address atomics of all groups (~4 us at C2).
  unsigned int pending = 0;
  auto fetch_next = [&]() -> long long {
    const long long nn = gstride + pending;
    pending = ticket_add(P.work);
    return nn;
  };

  // a6, the mailbox part: the K incoming entries of sub-filter gsf_ (offsets
  // into woff, their log-weights in_w by lanes < K, this thread's first
  // element of the copy into vpre)
  auto mb_fetch = [&](long long gsf_, float& in_w_, float& vpre_) {
    if (G.lane < K) {
      const int qi = static_cast<int>((static_cast<uint32_t>(G.lane) * P.t_inv) >> 16);   // lane / t
      const int off = static_cast<int>((neighbor_row(P, gsf_, qi) * P.tt + (G.lane - qi * P.t)) * E);
      woff[G.lane] = off;
      in_w_ = P.mb_prev[off];
    }
    __syncwarp();
    if (G.t < K * E) {
      const int j = G.t / E;
      vpre_ = P.mb_prev[woff[j] + (G.t - j * E)];
    }
  };

  // programmatic dependent launch: the CTA's launch overlaps the previous
  // step's tail; nothing that step wrote (particle blocks, mailbox, counters,
  // key, device inputs) is read before its grid has completed (no-op otherwise)
  asm volatile("griddepcontrol.wait;" ::: "memory");
#ifdef PF_TIMELINE
  const unsigned long long tl_pw = tl_now();
#endif
  // z / u first: their (device-input) loads leave before the launch's burst
  // of first-sub-filter copies, not queued behind it
  float zv = 0.0f, uv = 0.0f;
  if (do_sample) {
    if (threadIdx.x < ZD) zv = P.z ? P.z[threadIdx.x] : P.zin[threadIdx.x];
    if (threadIdx.x < UD) uv = P.u ? P.u[threadIdx.x] : P.uin[threadIdx.x];
  }
  if (G.t == 0) {
#pragma unroll
    for (int b = 0; b < (C::SPLIT0 ? 4 : 2); ++b) mbar_init(bars + b, 1);
    fence_mbar_init();
    issue(0, gid0, true);
    if (gid0 < P.n_local) pending = ticket_add(P.work);
  }
  if (do_sample) {
    if (threadIdx.x < ZD) {
      z_s[threadIdx.x] = zv;
      z2_s[threadIdx.x] = bc(zv);
    }
    if (threadIdx.x < UD) {   // control term h_s u_i (F8)
      const float v = P.mc.hs * uv;
      hsu_s[threadIdx.x] = v;
      hsu2_s[threadIdx.x] = bc(v);
    }
  }
  __syncthreads();

  TL(tl_start);
#ifdef PF_TIMELINE
  if (threadIdx.x == 0 && blockIdx.x < 4096) {
    pf_tl3[3 * blockIdx.x] = tl_entry;
    pf_tl3[3 * blockIdx.x + 1] = tl_pw;
    pf_tl3[3 * blockIdx.x + 2] = tl_start;
  }
#endif
  for (int it = 0;; ++it) {
    const int st = (C::NSTAGE == 2) ? (it & 1) : 0;
    TL(tl_w0);
    const uint32_t bpar = C::NSTAGE == 2 ? (it >> 1) & 1 : it & 1;
    mbar_wait(bars + st, bpar);   // the log-weight row (and next_s)
    if constexpr (C::SPLIT0) {   // first sub-filter: now its state rows
      if (it == 0 && G.t == 0 && next_s[st] < P.n_local) {
        const long long n0 = next_s[st];
        mbar_arrive_expect_tx(bars + 2 + st, st_bytes);
        bulk_g2s(gs + C::g_stage + st * C::stage_bytes, P.parts + n0 * ROW, st_bytes, bars + 2 + st);
      }
    }
    TL(tl_ready);
    const long long n = next_s[st];
    if (n >= P.n_local) break;
    if constexpr (C::NSTAGE == 2) {   // prefetch the next sub-filter into the other stage
      if (G.t == 0) issue(st ^ 1, fetch_next(), false);
    }
    float* xs = reinterpret_cast<float*>(gs + C::g_stage + st * C::stage_bytes);
    float* ws = xs + D * M;
    S.lists = reinterpret_cast<int*>(ws);   // Vose lists: the log-weight row is read into registers by then
    const long long gsf = P.g0 + n;                    // global sub-filter
    const uint32_t pbase = static_cast<uint32_t>(gsf * M);
    float* gblk = P.parts + n * ROW;                   // this sub-filter's block in HBM
    bool issued = false;   // NSTAGE 1: next load already started (after the sample loop)
    auto release_stage = [&]() {   // all generic smem accesses to the stage done: start the next load
      fence_proxy_async_smem();
      gsync<GW>(g);
      if constexpr (C::NSTAGE == 1) {
        if (G.t == 0) issue(0, fetch_next(), false);
      }
      issued = true;
    };
    auto finish = [&]() {   // end of a sub-filter
      if (!issued) {
        release_stage();
      } else {
        gsync<GW>(g);   // the scan region (new log-weights) is reused by the next sub-filter
      }
    };

    float lw[PP];
#pragma unroll
    for (int j = 0; j < PP; ++j) lw[j] = ws[C::slot(G.t, j)];
    uint32_t lmax_o = 0;   // ordered max of the post-exchange log-weights
    bool defer_x = false;  // incoming state entry (this thread's vpre) not yet in the state rows
    float dvx = 0.0f;
    // the state rows: landed (bulk copy) + the deferred incoming entry, before the group barrier
    // that precedes any read of them
    auto states_in = [&]() {
      if constexpr (!C::SPLIT0) return;
      mbar_wait(bars + 2 + st, bpar);
      if (defer_x && G.t < K * E) {
        const int j = G.t / E, c = G.t - j * E;
        if (c >= 2) xs[(c - 2) * M + wlist[j]] = dvx;
      }
    };

    // ---- a6 exchange: neighbours' best t (mailbox of step k-1) overwrite
    //      the own deg*t worst slots (R2–R5)
    if (do_merge && K > 0) {
      // worst K by order key (ascending = worse, R6): per-warp bottom-K by
      // K rounds of warp REDUX, then a merge of the GW lists after one barrier
      u64 key[PP];
      uint32_t wmax = 0;
#pragma unroll
      for (int i = 0; i < PP; ++i) {
        key[i] = order_key(lw[i], static_cast<uint32_t>(C::slot(G.t, i)));
        wmax = max(wmax, static_cast<uint32_t>(key[i] >> 32));
      }
      wmax = __reduce_max_sync(0xFFFFFFFFu, wmax);
      // incoming item j = (neighbour j / t, its j % t-th best): mailbox offset
      // (its log-weight, loaded now, gives the incoming maximum without a
      // dependent shared-memory read after the copy)
      // All mailbox loads are issued here, before the selection rounds, and
      // consumed after them: the incoming log-weights (-> incoming maximum)
      // and this thread's first element of the copy below (one L2 round trip
      // overlapped with the selection instead of two dependent ones).
      float in_w = 0.0f, vpre = 0.0f;
      mb_fetch(gsf, in_w, vpre);
      int ws0 = 0, ws1 = 0;   // K = 2: the two worst slots, in every thread's registers
      if (K == 2) {
        // deg t = 2 (ring, t = 1: the benchmark configurations): each thread's
        // two smallest keys, two warp rounds (the owner of the first advances
        // to its second), then the group's two smallest of the GW sorted pairs
        // — the same worst two (keys are unique), in the same order, without
        // the K-round rescans and clears over every key
        u64 m1 = ~0ull, m2 = ~0ull;
#pragma unroll
        for (int i = 0; i < PP; ++i) {
          const u64 kk = key[i];
          const bool lt1 = kk < m1;
          m2 = lt1 ? m1 : (kk < m2 ? kk : m2);
          m1 = lt1 ? kk : m1;
        }
        const u64 w1 = warp_min_u64(m1);
        if (m1 == w1) m1 = m2;
        const u64 w2 = warp_min_u64(m1);
        u64 b1 = w1, b2 = w2;
        if constexpr (GW == 1) {
          lmax_o = wmax;
        } else {
          if (G.lane == 0) {
            cand[G.wig * 2] = w1;
            cand[G.wig * 2 + 1] = w2;
            cand[GW * C::KMAX + G.wig] = wmax;
          }
          gsync<GW>(g);
          uint32_t mo = 0;
          b1 = ~0ull;
          b2 = ~0ull;
#pragma unroll
          for (int ww = 0; ww < GW; ++ww) {
            mo = max(mo, static_cast<uint32_t>(cand[GW * C::KMAX + ww]));
            const u64 x1 = cand[2 * ww], x2 = cand[2 * ww + 1];   // x1 < x2
            if (x1 < b1) {
              b2 = b1 < x2 ? b1 : x2;
              b1 = x1;
            } else {
              b2 = b2 < x1 ? b2 : x1;
            }
          }
          lmax_o = mo;
        }
        ws0 = static_cast<int>(0xFFFFFFFFu - static_cast<uint32_t>(b1));
        ws1 = static_cast<int>(0xFFFFFFFFu - static_cast<uint32_t>(b2));
        if (G.lane < 2) wlist[G.lane] = G.lane == 0 ? ws0 : ws1;   // (states_in, the trace hook)
      } else {
        u64 my_cand = ~0ull;
  #pragma unroll 1
        for (int j = 0; j < K; ++j) {
          u64 mk = key[0];
  #pragma unroll
          for (int i = 1; i < PP; ++i) mk = key[i] < mk ? key[i] : mk;
          const u64 wk = warp_min_u64(mk);
  #pragma unroll
          for (int i = 0; i < PP; ++i)
            if (key[i] == wk) key[i] = ~0ull;   // keys are unique (slot in the low bits)
          if (G.lane == j) my_cand = wk;
        }
        if constexpr (GW == 1) {
          lmax_o = wmax;
          if (G.lane < K) wlist[G.lane] = static_cast<int>(0xFFFFFFFFu - static_cast<uint32_t>(my_cand));
        } else {
          // flat list: candidate i of the GW * K is cand[i] (warp i / K), the
          // per-warp maxima after the GW * KMAX candidate slots
          if (G.lane < K) cand[G.wig * K + G.lane] = my_cand;
          if (G.lane == 0) cand[GW * C::KMAX + G.wig] = wmax;
          gsync<GW>(g);
          // every warp merges the GW candidate lists (identical result in all warps)
          u64 c[GW];   // candidate i = lane + 32 r of the GW*K list
          const int ncand = GW * K;
  #pragma unroll
          for (int r = 0; r < GW; ++r) {
            const int i = G.lane + 32 * r;
            c[r] = i < ncand ? cand[i] : ~0ull;
          }
          uint32_t mo = 0;
  #pragma unroll
          for (int ww = 0; ww < GW; ++ww) mo = max(mo, static_cast<uint32_t>(cand[GW * C::KMAX + ww]));
          lmax_o = mo;
          u64 mine = ~0ull;
  #pragma unroll 1
          for (int j = 0; j < K; ++j) {
            u64 lo = ~0ull;
  #pragma unroll
            for (int r = 0; r < GW; ++r) lo = c[r] < lo ? c[r] : lo;
            const u64 wk = warp_min_u64(lo);
  #pragma unroll
            for (int r = 0; r < GW; ++r)
              if (c[r] == wk) c[r] = ~0ull;
            if (G.lane == j) mine = wk;
          }
          if (G.lane < K) wlist[G.lane] = static_cast<int>(0xFFFFFFFFu - static_cast<uint32_t>(mine));
        }
      }
      __syncwarp();
      // own slots among the worst K (slot s is owned by thread s mod T, index s / T)
      uint32_t excl = 0;
      if (K == 2) {
        excl = ((ws0 & (C::T - 1)) == G.t ? 1u << (ws0 / C::T) : 0u) |
               ((ws1 & (C::T - 1)) == G.t ? 1u << (ws1 / C::T) : 0u);
      } else {
#pragma unroll 1
        for (int j = 0; j < K; ++j) {
          const int s = wlist[j];
          if ((s & (C::T - 1)) == G.t) excl |= 1u << (s / C::T);
        }
      }
      const uint32_t in_max = __reduce_max_sync(0xFFFFFFFFu, G.lane < K ? ord_f32(in_w) : 0u);
      // incoming log-weights now; incoming states into the state rows only
      // once their bulk copy has landed: for the first (split) load deferred
      // to after the resampler when every entry value is one thread's vpre
      // (K E <= T), else waited for here (at once after an unsplit load)
      defer_x = C::SPLIT0 && it == 0 && K * E <= C::T;
      if (C::SPLIT0 && !defer_x) mbar_wait(bars + 2 + st, bpar);
#pragma unroll 1
      for (int e = G.t; e < K * E; e += C::T) {
        const int j = e / E, c = e - j * E;
        const float v = e == G.t ? vpre : P.mb_prev[woff[j] + c];
        const int slot = K == 2 ? (j == 0 ? ws0 : ws1) : wlist[j];
        if (c == 0) ws[slot] = v;
        else if (c >= 2 && !defer_x) xs[(c - 2) * M + slot] = v;
      }
      dvx = vpre;
      if (P.dbg_src) {
#pragma unroll
        for (int i = 0; i < PP; ++i) {
          const int s = C::slot(G.t, i);
          long long src = pbase + s;
          if ((excl >> i) & 1u)
#pragma unroll 1
            for (int j = 0; j < K; ++j)
              if (wlist[j] == s) src = __float_as_uint(P.mb_prev[woff[j] + 1]);
          P.dbg_src[n * M + s] = src;
        }
      }
      gsync<GW>(g);
      // post-exchange max = max(pre-exchange max, incoming): the pre-exchange
      // maximum value survives because deg*t < m (R19)
      lmax_o = max(lmax_o, in_max);
#pragma unroll
      for (int j = 0; j < PP; ++j)
        if ((excl >> j) & 1u) lw[j] = ws[C::slot(G.t, j)];
    } else if ((do_merge || mode == MODE_STEP) && P.dbg_src) {
#pragma unroll
      for (int j = 0; j < PP; ++j) {
        const int s = C::slot(G.t, j);
        P.dbg_src[n * M + s] = pbase + s;   // no exchange (k = 1 or deg*t = 0): identity
      }
    }

    if (mode == MODE_EXCHANGE) {
      states_in();   // (the copy must land before the stage is reused)
      finish();
      continue;
    }
    TL(tl_merged);

    // ---- a7 normalise + a8 resample (slot order, R11)
    int anc[PP];
    uint32_t bz[PP], bw[PP];   // Philox block 0, words 2-3 (first Box–Muller pair)
    bool resampled = true;     // false: conditional policy kept the set (R21)
    float carry[PP];
    {
      uint32_t ua[PP], ub[PP], q[PP];
#pragma unroll
      for (int j = 0; j < PP; ++j) {
        const int s = C::slot(G.t, j);
        anc[j] = s;
        ua[j] = ub[j] = bz[j] = bw[j] = 0u;
        if (do_sample || do_resample) {
          const u32x4 b0 = philox4x32_10_rk(pbase + s, P.k, 0u, 0u, P.rk);
          ua[j] = b0.x;
          ub[j] = b0.y;
          bz[j] = b0.z;
          bw[j] = b0.w;
        }
      }
      if (do_resample) {
        if (K == 0) {   // no exchange this step: group max of the loaded set
          uint32_t mo = 0;
#pragma unroll
          for (int j = 0; j < PP; ++j) mo = max(mo, ord_f32(lw[j]));
          mo = __reduce_max_sync(0xFFFFFFFFu, mo);
          if constexpr (GW > 1) {
            uint32_t* r = reinterpret_cast<uint32_t*>(G.red + G.rb * 32);
            G.rb ^= 1;
            if (G.lane == 0) r[G.wig] = mo;
            gsync<GW>(g);
            mo = __reduce_max_sync(0xFFFFFFFFu, G.lane < GW ? r[G.lane] : 0u);
          }
          lmax_o = mo;
        }
        const float lmax = unord_f32(lmax_o);
        if constexpr (PP % 2 == 0) {   // F7 on pairs (packed, bit-identical)
#pragma unroll
          for (int j = 0; j < PP; j += 2) expq_c2(sub2(pk(lw[j], lw[j + 1]), bc(lmax)), q[j], q[j + 1]);
        } else {
#pragma unroll
          for (int j = 0; j < PP; ++j) q[j] = expq_c(lw[j] - lmax);
        }
        // R21: does this sub-filter resample now?  (uniform in the group)
        if (P.policy == POLICY_ESS) {   // ESS = Q^2 / sum q^2 < tau m, exactly in integers
          u64 s1 = 0, s2 = 0;
#pragma unroll
          for (int j = 0; j < PP; ++j) {
            s1 += q[j];
            s2 += static_cast<u64>(q[j]) * q[j];
          }
          const u64 Qs = gsum_u64<GW>(s1, G), S2 = gsum_u64<GW>(s2, G);
          resampled = ((static_cast<unsigned __int128>(Qs) * Qs) << 16) <
                      static_cast<unsigned __int128>(P.policy_param) * static_cast<u64>(M) * S2;
        } else if (P.policy == POLICY_FREQ) {   // a coin per (sub-filter, step): Philox stream 1
          resampled = static_cast<u64>(philox4x32_10_rk(static_cast<uint32_t>(gsf), P.k, 1u, 0u, P.rk).x) <
                      P.policy_param;
        }
        if (resampled) {
          resample_group<C>(q, ua, ub, anc, S, G, nullptr, nullptr);
        } else {   // keep the particles, carry l - l_max into the next weight (F12)
#pragma unroll
          for (int j = 0; j < PP; ++j) carry[j] = lw[j] - lmax;
        }
      }
      if (mode == MODE_STEP && P.dbg_anc) {
#pragma unroll
        for (int j = 0; j < PP; ++j) P.dbg_anc[n * M + C::slot(G.t, j)] = anc[j];
      }
      states_in();
      // all resampler reads of the scan buffer and the log-weight row are done;
      // the state rows are complete (bulk copy + incoming entries)
      gsync<GW>(g);
      if constexpr (C::STAGED) {
        // rolled sample loop: per-slot ancestor -> the (now free) log-weight
        // row, Philox words -> the (now free) scan buffer; own slots only
#pragma unroll
        for (int j = 0; j < PP; ++j) {
          const int s = C::slot(G.t, j);
          if (resampled) {
            reinterpret_cast<int*>(ws)[s] = anc[j];
          } else {
            ws[s] = carry[j];   // ancestor = own slot
          }
          bzw_s[s] = make_uint2(bz[j], bw[j]);
        }
      }
    }

    TL(tl_res);
    if constexpr (C::NSTAGE == 1) {
      // one stage: the next sub-filter's block is loaded only after this one's
      // sample loop; pull it from HBM into L2 now, so that load hits L2.  Not
      // earlier: the index is the ticket thread 0 requested a sub-filter ago,
      // and the first one (the launch's burst of same-address atomics, one per
      // group) returns only microseconds into the launch.
      if (G.t == 0 && mode == MODE_STEP) {
        const long long nn = gstride + pending;
        if (nn < P.n_local) bulk_prefetch_l2(P.parts + nn * ROW, stage_bytes);
      }
    }
    if constexpr (C::X2) {
     if (do_sample) {
      // ---- a9 gather (smem) + a1 RNG + a2 sample + a3 weight + a10 store,
      //      two particles (slots j, j+1 of this thread) at a time with the
      //      floating-point work packed (f32x2, bit-identical lane by lane)
#pragma unroll(C::UNR > 1 ? C::UNR / 2 : 1)
      for (int j = 0; j < PP; j += 2) {
        const int sa = C::slot(G.t, j), sb = C::slot(G.t, j + 1);
        int a0, a1;
        uint32_t za2, za3, zb2, zb3;
        float c0 = 0.0f, c1 = 0.0f;
        if constexpr (C::STAGED) {
          if (resampled) {
            a0 = reinterpret_cast<const int*>(ws)[sa];
            a1 = reinterpret_cast<const int*>(ws)[sb];
          } else {
            a0 = sa;
            a1 = sb;
            c0 = ws[sa];
            c1 = ws[sb];
          }
          const uint2 pa = bzw_s[sa], pb = bzw_s[sb];
          za2 = pa.x;
          za3 = pa.y;
          zb2 = pb.x;
          zb3 = pb.y;
        } else {
          a0 = anc[j];
          a1 = anc[j + 1];
          if (!resampled) {
            c0 = carry[j];
            c1 = carry[j + 1];
          }
          za2 = bz[j];
          za3 = bw[j];
          zb2 = bz[j + 1];
          zb3 = bw[j + 1];
        }
        const float* xa = xs + a0;
        const float* xb = xs + a1;
        auto x = [xa, xb](int c) { return pk(xa[c * M], xb[c * M]); };
        float* outa = gblk + sa;
        float* outb = gblk + sb;
        NoiseGen2 gen{pbase + static_cast<uint32_t>(sa), pbase + static_cast<uint32_t>(sb), P.k, P.rk,
                      u32x4{0u, 0u, za2, za3}, u32x4{0u, 0u, zb2, zb3}};
        typename Model::Acc2 A;
        auto store2 = [outa, outb](int c, f2 v) {
          outa[c * M] = lo2(v);
          outb[c * M] = hi2(v);
        };
        if constexpr (RT) {
          SampleRuntime2<Model>::run(P.mc2, P.nj, hsu2_s, z2_s, x, gen, A, store2);
        } else if constexpr (C::CHUNKED) {
          SampleChunked2<Model>::run(P.mc2, hsu2_s, z2_s, x, gen, A, store2);
        } else {
          SampleStream2<Model, 0>::run(P.mc2, hsu2_s, z2_s, x, gen, A, store2);
        }
        f2 l = Model::finish2(P.mc2, z2_s, A);
        if (!resampled) l = add2(pk(c0, c1), l);   // F12
        outa[D * M] = lo2(l);
        outb[D * M] = hi2(l);
        reinterpret_cast<float*>(bzw_s)[2 * sa] = lo2(l);   // own slots, after their Philox words were read
        reinterpret_cast<float*>(bzw_s)[2 * sb] = hi2(l);
      }
     }
    } else if (do_sample) {
      // ---- a9 gather (smem) + a1 RNG + a2 sample + a3 weight + a10 store,
      //      one particle at a time (coalesced rows: consecutive threads,
      //      consecutive slots)
#pragma unroll C::UNR
      for (int j = 0; j < PP; ++j) {
        const int s = C::slot(G.t, j);
        int a;
        uint32_t z2, z3;
        float cr = 0.0f;
        if constexpr (C::STAGED) {
          if (resampled) {
            a = reinterpret_cast<const int*>(ws)[s];
          } else {
            a = s;
            cr = ws[s];
          }
          const uint2 bb = bzw_s[s];
          z2 = bb.x;
          z3 = bb.y;
        } else {
          a = anc[j];
          if (!resampled) cr = carry[j];
          z2 = bz[j];
          z3 = bw[j];
        }
        const float* xa = xs + a;
        auto x = [xa](int c) { return xa[c * M]; };
        float* out = gblk + s;
        NoiseGen gen{pbase + static_cast<uint32_t>(s), P.k, P.rk, u32x4{0u, 0u, z2, z3}};
        typename Model::Acc A;
        // (one particle per thread: the unrolled chain measured as fast as the chunked one)
        if constexpr (RT) {
          SampleRuntime<Model>::run(P.mc, P.nj, hsu_s, z_s, x, gen, A, [out](int c, float v) { out[c * M] = v; });
        } else {
          SampleStream<Model, 0>::run(P.mc, hsu_s, z_s, x, gen, A, [out](int c, float v) { out[c * M] = v; });
        }
        float l = Model::finish(P.mc, z_s, A);
        if (!resampled) l = cr + l;   // F12
        out[D * M] = l;
        reinterpret_cast<float*>(bzw_s)[2 * s] = l;   // own slot, after its Philox words were read

      }
    }

    TL(tl_smp);
    // the stage buffer is no longer read (new states live in HBM, new
    // log-weights in the scan buffer): start the next sub-filter's load now
    if (C::EARLY && do_sample) release_stage();

    // ---- a4 local reduce: best t -> mailbox (k&1); a5 global best key
    {
      float lnew[PP];
#pragma unroll
      for (int j = 0; j < PP; ++j)
        lnew[j] = do_sample ? reinterpret_cast<const float*>(bzw_s)[2 * C::slot(G.t, j)] : lw[j];
      uint32_t done = 0;
      const int nbest = P.t > 0 ? P.t : 1;
      u64 nb_k = 0ull, nb_l = 0ull;
#pragma unroll 1
      for (int jb = 0; jb < nbest; ++jb) {
        u64 mk = 0ull;
#pragma unroll
        for (int j = 0; j < PP; ++j) {
          const u64 key = (done >> j) & 1u ? 0ull : order_key(lnew[j], pbase + C::slot(G.t, j));
          mk = key > mk ? key : mk;
        }
        const u64 best = gmax_u64<GW>(mk, G);
        if (P.pool_cta && G.lane == jb) {   // All-to-All t >= 2: this sub-filter's jb-th best
          nb_k = best;
          nb_l = static_cast<u64>(n * P.tt + jb);
        }
        const int bslot = static_cast<int>(0xFFFFFFFFu - static_cast<uint32_t>(best) - pbase);
        if ((bslot & (C::T - 1)) == G.t) {   // the unique owner (slot bslot = j T + t)
          done |= 1u << (bslot / C::T);
          if (jb < P.t) {
            float* e = P.mb_cur + (n * P.tt + jb) * E;
            e[0] = unord_f32(static_cast<uint32_t>(best >> 32));   // = lnew[j] (ord is a bijection)
            e[1] = __uint_as_float(pbase + bslot);
          }
          if (jb == 0) atomicMax(P.key_cur, best);
        }
        if (jb < P.t && G.wig == 0) {
          // the state of the best particle, one component per lane (one L2
          // round trip): the owner's global stores of the sample loop are
          // ordered before these loads by the group barrier in gmax (GW > 1)
          // or the warp barrier (GW == 1); without sampling: the loaded set
          if constexpr (GW == 1) __syncwarp();
          if (G.lane < D) {
            const float* src = do_sample ? gblk + bslot : xs + bslot;
            P.mb_cur[(n * P.tt + jb) * E + 2 + G.lane] = src[G.lane * M];
          }
        }
      }
      if (P.pool_cta && G.wig == 0) {
        // All-to-All t >= 2: merge this sub-filter's best t into the group's
        // running best t (global row of the group, lanes < t; empty before
        // the group's first sub-filter)
        u64* row = P.pool_cta + (gid0 * P.tt + G.lane) * 2;
        u64 rk = 0ull, rl = 0ull;
        if (it > 0 && G.lane < P.t) {
          rk = __ldcg(row);
          rl = __ldcg(row + 1);
        }
        top_t_merge(rk, rl, nb_k, nb_l, P.t, G.lane);
        if (G.lane < P.t) {
          __stcg(row, rk);
          __stcg(row + 1, rl);
        }
      }
    }
    finish();
#ifdef PF_TIMELINE
    if (G.t == 0) {
      const unsigned long long tl_end = tl_now();
      unsigned int smid;
      asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
      const unsigned long long i = atomicAdd(&pf_tl[0], 1ull);
      if (i < 65536) {
        unsigned long long* r = pf_tl + 1 + 8 * i;
        r[0] = static_cast<unsigned long long>(n) | (static_cast<unsigned long long>(smid) << 32) |
               (static_cast<unsigned long long>(blockIdx.x * C::S + g) << 40);
        r[1] = tl_start; r[2] = tl_w0; r[3] = tl_ready; r[4] = tl_merged; r[5] = tl_res; r[6] = tl_smp; r[7] = tl_end;
      }
    }
#endif
  }

  // this CTA's sub-filters are done: the next step's grid may start launching
  // into the SMs the retiring CTAs free (it waits in griddepcontrol.wait)
  asm volatile("griddepcontrol.launch_dependents;");

  // ---- a5: the last CTA to finish copies the winning particle (R6)
#ifdef PF_TIMELINE
  const unsigned long long tl_epi = tl_now();
#endif
  __shared__ unsigned int s_last;
  __syncthreads();
  if (threadIdx.x == 0) {
    // the CTA barrier orders every thread's writes (mailbox rows, key) before
    // thread 0's completion count, a gpu-scope acquire-release RMW (cumulative:
    // it releases what the barrier ordered before it, and the last CTA's
    // acquire orders its reads below after every other CTA's release)
    unsigned int prev;
    asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(prev) : "l"(P.counter) : "memory");
    s_last = (prev == gridDim.x - 1) ? 1u : 0u;
  }
  __syncthreads();
  if (s_last) {
    const int tid = threadIdx.x;
    // All-to-All: this shard's best t -> pool row pool_local_row (first: the
    // peer transport also ships it to every rank before the rendezvous)
    if (P.topo == TOPO_A2A && P.t > 0 && mode != MODE_EXCHANGE) {
      float* pool = P.mb_cur + P.pool_local_row * P.tt * E;
      if (P.t == 1) {   // the pool's best is the shard's best particle: the record just written
        const u64 key = __ldcg(P.key_cur);
        const uint32_t gidx = 0xFFFFFFFFu - static_cast<uint32_t>(key);
        const long long col = static_cast<long long>(gidx) - P.g0 * M;
        const float* blk = P.parts + (col / M) * ROW + (col % M);
        if (tid < D) pool[2 + tid] = __ldcg(blk + tid * M);
        if (tid == 0) {
          pool[0] = unord_f32(static_cast<uint32_t>(key >> 32));
          pool[1] = __uint_as_float(gidx);
        }
      } else {
        // reduction scratch: group 0's stage buffer (no load in flight after the loop)
        u64* red = reinterpret_cast<u64*>(smem + C::c_groups + C::g_stage);
        if (P.pool_cta) pool_top_t_cta(P, pool, red, static_cast<long long>(gridDim.x) * C::S, E);
        else pool_top_t(P, P.mb_cur, P.n_local * P.t, pool, red, E);
      }
    }
    if (mode != MODE_EXCHANGE) {
      const u64 key = __ldcg(P.key_cur);
      const uint32_t gidx = 0xFFFFFFFFu - static_cast<uint32_t>(key);
      const long long col = static_cast<long long>(gidx) - P.g0 * M;
      const float* blk = P.parts + (col / M) * ROW + (col % M);
      float* outs[2] = {P.record, P.est_out};
      if (P.peer_mb[0] && (mode == MODE_STEP || mode == MODE_PUBLISH)) {
        // peer transport: the boundary sub-filters' best-t rows into the
        // neighbour ranks' halo rows, this shard's best record into slot
        // `rank` of every rank's peer block, then step flags, then wait for every rank's flag
        // (device-side rendezvous over NVLink), then the exact max over the
        // world records (the all-gather + pf_reduce_records of the NCCL path)
        const bool a2a = P.topo == TOPO_A2A && P.t > 0;
        const int par = static_cast<int>(P.rv & 1ull);
        if (a2a) {
          __syncthreads();   // the local pool row is complete
          const float* lp = P.mb_cur + P.pool_local_row * P.tt * E;
          for (int i = tid; i < P.world * P.t * E; i += blockDim.x) {
            const int r = i / (P.t * E), e = i - r * (P.t * E);
            peer_pool(P.peer_blk[r], par, P.rank)[e] = __ldcg(lp + e);
          }
        } else {
          peer_halo_rows(P, E);
        }
        if (tid < D) {
          const float v = __ldcg(blk + tid * M);
          for (int r = 0; r < P.world; ++r) peer_rec(P.peer_blk[r], par, P.rank)[4 + tid] = v;
        }
        if (tid == 0) {
          const float r4[4] = {__uint_as_float(static_cast<uint32_t>(key)),
                               __uint_as_float(static_cast<uint32_t>(key >> 32)),
                               unord_f32(static_cast<uint32_t>(key >> 32)), 0.0f};
          for (int r = 0; r < P.world; ++r)
            for (int c = 0; c < 4; ++c) peer_rec(P.peer_blk[r], par, P.rank)[c] = r4[c];
        }
        // the barrier orders every thread's peer writes before the flag
        // stores below, system-scope releases (cumulative)
        __syncthreads();
        // Rendezvous number rv (not the step number: flags only grow, also
        // across pf_set_particles).  Ordering: a rank writes the records /
        // pool rows of rendezvous rv into buffer rv & 1 BEFORE raising flag
        // rv, and starts rendezvous rv + 1 only after every rank raised flag
        // rv.  Rank B raises flag rv + 1 only after its rendezvous-rv reads
        // are done (they precede its kernel's completion), so rank A's writes
        // of rendezvous rv + 2 into buffer rv & 1 (issued after A passed
        // rendezvous rv + 1) cannot overwrite anything B still reads.
        const unsigned long long kk = P.rv;
        int late = 0;
        if (tid < P.world) {
          unsigned long long* f = peer_flags(P.peer_blk[tid]) + P.rank;
          asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(f), "l"(kk) : "memory");
          const unsigned long long* mine = peer_flags(P.peer_blk[P.rank]) + tid;
          const unsigned long long t0 = global_ns();
          unsigned long long seen;
          for (;;) {
            asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(seen) : "l"(mine) : "memory");
            if (seen >= kk) break;
            if (global_ns() - t0 > P.peer_timeout_ns) {   // a rank did not arrive: report, do not hang
              late = 1;
              break;
            }
          }
        }
        const bool timed_out = __syncthreads_or(late) != 0;
        if (tid < 32) {
          const float* rec0 = peer_rec(P.peer_blk[P.rank], par, 0);
          u64 k2 = 0ull;
          if (tid < P.world)
            k2 = static_cast<u64>(__float_as_uint(__ldcv(rec0 + tid * kPeerRec))) |
                 (static_cast<u64>(__float_as_uint(__ldcv(rec0 + tid * kPeerRec + 1))) << 32);
          const u64 w = warp_max_u64(k2);
          const int src = __ffs(__ballot_sync(0xFFFFFFFFu, tid < P.world && k2 == w)) - 1;
          for (int c = tid; c < 4 + D; c += 32) {
            const float v = c == 3 ? __uint_as_float(timed_out ? kStatusPeerTimeout : 0u)
                                   : __ldcv(rec0 + src * kPeerRec + c);
            for (int o = 0; o < 2; ++o)
              if (outs[o]) outs[o][c] = v;
            if (P.record_host) put_tagged(P.record_host, c, v, static_cast<uint32_t>(P.k));
          }
          if (a2a) {   // the global pool: best t of the world's pool rows (pf_reduce_pool, fused)
            float* out = P.mb_cur + P.pool_row * P.tt * E;
            u64 prev = ~0ull;
            for (int jb = 0; jb < P.t; ++jb) {
              u64 best = 0ull;
              int be = -1;
              for (int e = tid; e < P.world * P.t; e += 32) {
                const int r = e / P.t, jj = e - r * P.t;
                const float* en = peer_pool(P.peer_blk[P.rank], par, r) + jj * E;
                const u64 kk2 = order_key(__ldcv(en), __float_as_uint(__ldcv(en + 1)));
                if (kk2 < prev && kk2 > best) {
                  best = kk2;
                  be = e;
                }
              }
              const u64 g2 = warp_max_u64(best);
              const int own = __ffs(__ballot_sync(0xFFFFFFFFu, be >= 0 && best == g2)) - 1;
              const int bsel = __shfl_sync(0xFFFFFFFFu, be, own < 0 ? 0 : own);
              if (own >= 0) {
                const int r = bsel / P.t, jj = bsel - r * P.t;
                const float* en = peer_pool(P.peer_blk[P.rank], par, r) + jj * E;
                for (int c = tid; c < E; c += 32) out[jb * E + c] = __ldcv(en + c);
              }
              prev = g2;
            }
          }
        }
      } else {
        if (tid < D) {
          const float v = __ldcg(blk + tid * M);
#pragma unroll
          for (int o = 0; o < 2; ++o)
            if (outs[o]) outs[o][4 + tid] = v;
          if (P.record_host) put_tagged(P.record_host, 4 + tid, v, static_cast<uint32_t>(P.k));
        }
        if (tid == 0) {
          const float r[4] = {__uint_as_float(static_cast<uint32_t>(key)), __uint_as_float(static_cast<uint32_t>(key >> 32)),
                              unord_f32(static_cast<uint32_t>(key >> 32)), 0.0f};
#pragma unroll
          for (int o = 0; o < 2; ++o)
            if (outs[o])
#pragma unroll
              for (int c = 0; c < 4; ++c) outs[o][c] = r[c];
          if (P.record_host)
#pragma unroll
            for (int c = 0; c < 4; ++c) put_tagged(P.record_host, c, r[c], static_cast<uint32_t>(P.k));
        }
      }
    }
    if (tid == 0) {
      *P.key_next = 0ull;
      *P.counter = 0u;
#ifdef PF_TIMELINE
      pf_tl2[1] = tl_epi;
      pf_tl2[2] = tl_now();
#endif
      *P.work = 0u;
    }
  }
}

// Resampling test hook: the step kernel's group resampler on rows of integer
// weights q [N][M] with explicit uniforms (one group per row).
template <class C>
__global__ void __launch_bounds__(C::T* C::S) pf_resample_debug_kernel(const uint32_t* __restrict__ q,
                                                                        const uint32_t* __restrict__ ua,
                                                                        const uint32_t* __restrict__ ub, int* anc,
                                                                        u64* prob, int* alias, long long N) {
  extern __shared__ __align__(128) unsigned char smem[];
  const int g = threadIdx.x / C::T;
  unsigned char* gs = smem + C::c_groups + g * C::group_bytes;
  ResampleSmem S;
  S.scan = reinterpret_cast<u64*>(gs + C::g_scan);
  S.prob = reinterpret_cast<u64*>(gs + C::g_prob);
  S.alias = reinterpret_cast<int*>(gs + C::g_alias);
  S.lists = reinterpret_cast<int*>(gs + C::g_stage);   // (no particle stage in the test hook)
  GroupCtx G;
  G.g = g;
  G.t = threadIdx.x - g * C::T;
  G.lane = threadIdx.x & 31;
  G.wig = G.t >> 5;
  G.red = reinterpret_cast<u64*>(gs + C::g_red);
  G.rb = 0;
  for (long long n = static_cast<long long>(blockIdx.x) * C::S + g; n < N;
       n += static_cast<long long>(gridDim.x) * C::S) {
    uint32_t qq[C::P], a[C::P], b[C::P];
    int an[C::P];
#pragma unroll
    for (int j = 0; j < C::P; ++j) {
      const long long i = n * C::M + C::slot(G.t, j);
      qq[j] = q[i];
      a[j] = ua[i];
      b[j] = ub[i];
    }
    resample_group<C>(qq, a, b, an, S, G, prob ? prob + n * C::M : nullptr, alias ? alias + n * C::M : nullptr);
#pragma unroll
    for (int j = 0; j < C::P; ++j) anc[n * C::M + C::slot(G.t, j)] = an[j];
    gsync<C::GW>(g);
  }
}

// Host-side launch helpers (explicit instantiation sets per n_joints TU).
template <class C>
struct StepKernel {
  static constexpr size_t smem() { return C::smem; }
  static cudaError_t prepare(int* blocks_per_sm) {
    cudaError_t e = cudaFuncSetAttribute(pf_step_kernel<C>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         static_cast<int>(smem()));
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(pf_resample_debug_kernel<C>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               static_cast<int>(smem()));
    if (e != cudaSuccess) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, pf_step_kernel<C>, C::T * C::S, smem());
  }
  static cudaError_t launch(const StepParams& p, int grid, cudaStream_t s, bool pdl) {
    // programmatic stream serialization: back-to-back steps overlap the launch
    // and prologue of step k + 1 with the tail of step k (see the kernel)
    if (!pdl) {
      pf_step_kernel<C><<<grid, C::T * C::S, smem(), s>>>(p);
      return cudaGetLastError();
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(C::T * C::S);
    cfg.dynamicSmemBytes = smem();
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, pf_step_kernel<C>, p);
  }
  static cudaError_t resample_debug(const uint32_t* q, const uint32_t* ua, const uint32_t* ub, int* anc, u64* prob,
                                    int* alias, long long N, cudaStream_t s) {
    const long long ctas = (N + C::S - 1) / C::S;
    pf_resample_debug_kernel<C><<<static_cast<int>(ctas < 4096 ? ctas : 4096), C::T * C::S, smem(), s>>>(
        q, ua, ub, anc, prob, alias, N);
    return cudaGetLastError();
  }
};

}  // namespace pf
