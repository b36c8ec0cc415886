// pf_runtime.cu — host runtime behind the C ABI of include/pf.h.
//
// Owns host metadata only: configuration validation, shard geometry, the
// scratch carve-up of the caller's buffers, the kernel table lookup, the
// per-step launch parameters (step inputs travel inside the launch).
// Every computation of the path runs in the kernels of pf_kernels.cuh.
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <new>

#include "../../include/pf.h"
#include "pf_central.h"
#include "pf_mean.h"
#include "pf_kernels.cuh"
#include "pf_registry.h"

using pf::u64;

namespace {

constexpr int kMaxNJ = 28;

// scratch layout (bytes)
constexpr size_t kOffKeys = 0;        // u64[2]
constexpr size_t kOffCounter = 16;    // u32 CTA completion counter
constexpr size_t kOffWork = 20;       // u32 dynamic work counter
constexpr size_t kOffRecord = 64;     // float[4 + d]  (d <= 32 -> 144 B)
constexpr size_t kOffInputs = 256;    // float[64]: z at 0, u at 32
constexpr size_t kOffMu0 = 512;       // float[64]
constexpr size_t kOffSigma0 = 768;    // float[64]
constexpr size_t kOffMean = 1024;     // double[kMeanGrid + 1][33]: weighted-mean partials + summed record
constexpr size_t kScratchBytes = kOffMean + sizeof(double) * (pf::kMeanGrid + 1) * 33;

struct Table {
  const pf::KernelEntry* e;
  int n;
};
Table tables(int i) {
  switch (i) {
    case 0: return {pf::kEntriesNJ2, pf::kNumEntriesNJ2};
    case 1: return {pf::kEntriesNJ5, pf::kNumEntriesNJ5};
    case 2: return {pf::kEntriesNJ28, pf::kNumEntriesNJ28};
    case 3: return {pf::kEntriesLG1, pf::kNumEntriesLG1};
    default: return {pf::kEntriesARMG, pf::kNumEntriesARMG};   // last: compiled n_j come first
  }
}
constexpr int kTables = 5;
constexpr int kMaxGenericNJ = 28;   // the generic arm's stage holds d <= 32

bool matches(const pf::KernelEntry& e, int model, int nj, int m, int res) {
  // arm entries: a compiled n_j, or a generic bucket (key -NJMAX) that holds n_j
  return e.model == model && (model != PF_MODEL_ARM_PLANAR || e.nj == nj || (e.nj < 0 && nj <= -e.nj)) && e.m == m &&
         e.res == res;
}

// First entry matching (model, nj, m, res), or the PF_VARIANT-th one if set.
const pf::KernelEntry* find_entry(int model, int nj, int m, int res) {
  const char* v = std::getenv("PF_VARIANT");
  int want = v ? std::atoi(v) : 0;
  const pf::KernelEntry* first = nullptr;
  for (int ti = 0; ti < kTables; ++ti) {
    const Table t = tables(ti);
    for (int i = 0; i < t.n; ++i)
      if (matches(t.e[i], model, nj, m, res)) {
        if (!first) first = &t.e[i];
        if (want-- == 0) return &t.e[i];
      }
  }
  return first;
}

// Large shards take the entry flagged `large` when one is compiled.
constexpr long long kLargeNLocal = 8192;
const pf::KernelEntry* large_entry(int model, int nj, int m, int res) {
  for (int ti = 0; ti < kTables; ++ti) {
    const Table t = tables(ti);
    for (int i = 0; i < t.n; ++i)
      if (matches(t.e[i], model, nj, m, res) && t.e[i].large) return &t.e[i];
  }
  return nullptr;
}

// Small problems (too few sub-filters to keep the default mapping's groups
// busy) are latency-bound: take the matching entry with the fewest particles
// per thread.  PF_VARIANT, when set, wins.
const pf::KernelEntry* latency_entry(int model, int nj, int m, int res) {
  const pf::KernelEntry* best = nullptr;
  for (int ti = 0; ti < kTables; ++ti) {
    const Table t = tables(ti);
    for (int i = 0; i < t.n; ++i)
      if (matches(t.e[i], model, nj, m, res) && (!best || t.e[i].gw > best->gw))
        best = &t.e[i];
  }
  return best;
}

struct Geometry {
  int model;          // pf_model_id
  int nj, d, m, deg, tt, E;
  int zd, ud;         // measurement and control dimensions of the model
  long long N, R, C, n_local, g0, n_ext, M_local, ROW;
  bool central;   // one filter of m > 1024 particles, resampled globally (pf_central.cu)
  bool vose;      // resampler (central filter sizing)
  long long tiles;
};

pf_status validate(const pf_config* cfg, const pf_model_params* mp, Geometry* g) {
  if (!cfg || !mp) return PF_EINVAL;
  if (mp->model == PF_MODEL_ARM_PLANAR) {
    if (mp->n_joints < 1) return PF_EINVAL;
    if (mp->n_joints > kMaxGenericNJ) return PF_EUNSUPPORTED;
    if (!(mp->sigma_cam > 0.0f) || !(mp->sigma_theta_meas > 0.0f) || !(mp->sigma_theta >= 0.0f) ||
        !(mp->sigma_pos >= 0.0f) || !(mp->sigma_vel >= 0.0f))
      return PF_EINVAL;
    g->model = PF_MODEL_ARM_PLANAR;
    g->nj = mp->n_joints;
    g->d = mp->n_joints + 4;
    g->zd = mp->n_joints + 2;
    g->ud = mp->n_joints;
  } else if (mp->model == PF_MODEL_LINEAR_GAUSS_1D) {
    if (!(mp->sigma_theta_meas > 0.0f) || !(mp->sigma_theta >= 0.0f)) return PF_EINVAL;
    g->model = PF_MODEL_LINEAR_GAUSS_1D;
    g->nj = 1;
    g->d = g->zd = g->ud = 1;
  } else {
    return PF_EINVAL;
  }
  const int m = cfg->m;
  if (cfg->n_filters < 1 || cfg->t < 0 || cfg->world < 1 || cfg->rank < 0 || cfg->rank >= cfg->world)
    return PF_EINVAL;
  if (cfg->resample_policy < PF_POLICY_ALWAYS || cfg->resample_policy > PF_POLICY_FREQ ||
      cfg->resample_param > (1ull << 32))
    return PF_EINVAL;
  // Centralized filter (NEXT-2): a single filter of M > 1024 particles.
  g->central = cfg->n_filters == 1 && m > 1024;
  g->vose = false;
  if (g->central) {
    if (m % pf::kCentralTile != 0 || m > (1 << 26) || cfg->world != 1) return PF_EINVAL;
    if (cfg->topo != PF_TOPO_NONE && cfg->t != 0) return PF_EINVAL;
    if (cfg->resampler != PF_RESAMPLE_RWS && cfg->resampler != PF_RESAMPLE_VOSE) return PF_EINVAL;
    if (cfg->resampler == PF_RESAMPLE_VOSE && m > pf::kCentralVoseMax) return PF_EUNSUPPORTED;
    if (cfg->resample_policy != PF_POLICY_ALWAYS) return PF_EUNSUPPORTED;
    g->vose = cfg->resampler == PF_RESAMPLE_VOSE;
    g->m = m;   // (any n_j <= 28: compiled 2 / 5 / 28, the generic arm otherwise)
    g->N = 1;
    g->deg = 0;
    g->tt = 1;
    g->E = g->d + 2;
    g->R = g->C = 0;
    g->n_local = 1;
    g->g0 = 0;
    g->n_ext = 1;
    g->M_local = m;
    g->ROW = static_cast<long long>(g->d + 1) * m;
    g->tiles = m / pf::kCentralTile;
    return PF_OK;
  }
  if (m < 32 || m > 1024 || (m & (m - 1)) != 0) return PF_EINVAL;
  if (cfg->resampler != PF_RESAMPLE_RWS && cfg->resampler != PF_RESAMPLE_VOSE) return PF_EINVAL;
  if (cfg->topo != PF_TOPO_NONE && cfg->topo != PF_TOPO_RING && cfg->topo != PF_TOPO_TORUS2D &&
      cfg->topo != PF_TOPO_ALL2ALL)
    return PF_EINVAL;
  if (!find_entry(g->model, g->nj, m, cfg->resampler)) return PF_EUNSUPPORTED;
  g->m = m;
  g->N = cfg->n_filters;
  g->deg = cfg->topo == PF_TOPO_RING ? 2 : cfg->topo == PF_TOPO_TORUS2D ? 4 : cfg->topo == PF_TOPO_ALL2ALL ? 1 : 0;
  if (static_cast<long long>(g->deg) * cfg->t >= m && g->deg * cfg->t > 0) return PF_EINVAL;   // R19
  if (g->deg * cfg->t > 32) return PF_EINVAL;   // exchange list fits one warp (KMAX)
  g->tt = cfg->t > 0 ? cfg->t : 1;
  g->E = g->d + 2;
  g->R = g->C = 0;
  const long long W = cfg->world;
  if (cfg->topo == PF_TOPO_TORUS2D) {
    long long R = cfg->torus_rows, C = cfg->torus_cols;
    if (R <= 0 || C <= 0) {
      int lg = 0;
      while ((1ll << (lg + 1)) <= g->N) ++lg;
      R = 1ll << (lg / 2);
      C = g->N / R;
    }
    if (R * C != g->N || R % W != 0) return PF_EINVAL;
    g->R = R;
    g->C = C;
    const long long rows = R / W;
    g->n_local = rows * C;
    g->g0 = cfg->rank * rows * C;
    g->n_ext = g->n_local + (W > 1 ? 2 * C : 0);
  } else {
    if (g->N % W != 0) return PF_EINVAL;
    g->n_local = g->N / W;
    g->g0 = cfg->rank * g->n_local;
    g->n_ext = g->n_local + ((W > 1 && cfg->topo == PF_TOPO_RING) ? 2 : 0) +
               (cfg->topo == PF_TOPO_ALL2ALL ? (W > 1 ? W + 1 : 1) : 0);
  }
  g->M_local = g->n_local * m;
  g->ROW = static_cast<long long>(g->d + 1) * m;
  if (g->M_local > (1ll << 31) || g->N * m > (1ll << 32)) return PF_EINVAL;
  return PF_OK;
}

}  // namespace

struct pf_handle {
  pf_config cfg;
  pf_model_params mp;
  Geometry g;
  pf::ModelConsts mc;
  float* parts;      // [n_local][d+1][m] blocked SoA (row d = log-weight)
  float* mailbox;
  unsigned char* scratch;
  cudaStream_t stream;
  long long step;
  const pf::KernelEntry* ke;
  int grid;
  pf_status err;
  bool trace;
  long long* d_src;
  int* d_anc;
  // peer transport (pf_peer_connect*): the neighbour ranks' mailboxes and every
  // rank's peer block (flags + records), this rank's own block (cudaMalloc'd)
  bool peers;
  bool local_peers;   // connected by pf_peer_connect_local (one process, one device)
  bool shared_device; // some connected peer runs on this rank's device (PDL off, see launch())
  unsigned long long rv;          // peer rendezvous number of the last peer-mode launch
  unsigned long long peer_timeout_ns;
  bool pdl;           // programmatic dependent launch of the step kernel (PF_NO_PDL unset at init)
  float* peer_mb[2];
  unsigned char* peer_blk[pf::kMaxRanks];
  unsigned char* own_blk;
  void* opened[2 * pf::kMaxRanks];   // IPC mappings to close
  int n_opened;
  bool mapped;         // PF_NO_MAPPED unset at init
  bool last_mapped;    // the last step wrote its record (and step number) into rec_host
  float* rec_host;     // mapped pinned host floats: [0, 4+d) estimate record, [48, 48+d) weighted mean
  float* rec_host_dev; // its device alias
  float* d_reduce_tmp;
};

namespace {

pf_status sticky(pf_handle* h, cudaError_t e) {
  if (e != cudaSuccess && h->err == PF_OK) h->err = PF_ECUDA;
  return e == cudaSuccess ? h->err : PF_ECUDA;
}

u64* keys(pf_handle* h) { return reinterpret_cast<u64*>(h->scratch + kOffKeys); }
float* record(pf_handle* h) { return reinterpret_cast<float*>(h->scratch + kOffRecord); }
float* inputs(pf_handle* h) { return reinterpret_cast<float*>(h->scratch + kOffInputs); }

float* mailbox_parity(pf_handle* h, long long k) {
  return h->mailbox + (k & 1) * h->g.n_ext * h->g.tt * h->g.E;
}

// All-to-All with t >= 2: per-group best-t candidates after the mailbox parities
// ({order key, entry} u64 pairs for up to kPoolGroups groups of the step kernel).
constexpr long long kPoolGroups = 16384;
size_t pool_cta_bytes(const pf_config* cfg, const Geometry& g) {
  return (!g.central && cfg->topo == PF_TOPO_ALL2ALL && cfg->t >= 2) ? sizeof(u64) * 2 * kPoolGroups * g.tt : 0;
}

// Host-input steps of a single-rank filter stream their estimate record into
// mapped pinned host memory (pf_estimate polls it); device-input steps keep it
// on the device (record / est_out) and pf_estimate copies it on demand.
bool streams_record(const pf_handle* h) {
  return h->mapped && !(h->cfg.flags & PF_DEVICE_INPUTS) && (h->cfg.world == 1 || h->peers);
}

pf::StepParams base_params(pf_handle* h, long long k, int mode) {
  pf::StepParams p;
  std::memset(&p, 0, sizeof(p));
  p.mc = h->mc;
  auto dup = [](float v) {
    uint32_t b;
    std::memcpy(&b, &v, 4);
    return (static_cast<unsigned long long>(b) << 32) | b;
  };
  p.mc2 = {dup(h->mc.lj), dup(h->mc.hs), dup(h->mc.s_th), dup(h->mc.s_pos), dup(h->mc.s_vel), dup(h->mc.inv_cam),
           dup(h->mc.inv_thm)};
  p.parts = h->parts;
  p.mb_prev = mailbox_parity(h, k - 1);
  p.mb_cur = mailbox_parity(h, k);
  p.z = nullptr;   // host-input mode: zin / uin (filled by the caller)
  p.u = nullptr;
  p.key_cur = keys(h) + (k & 1);
  p.key_next = keys(h) + ((k + 1) & 1);
  p.counter = reinterpret_cast<unsigned int*>(h->scratch + kOffCounter);
  p.work = reinterpret_cast<unsigned int*>(h->scratch + kOffWork);
  p.record = record(h);
  p.record_host = streams_record(h) ? reinterpret_cast<u64*>(h->rec_host_dev) : nullptr;
  p.est_out = nullptr;
  p.dbg_src = nullptr;
  p.dbg_anc = nullptr;
  p.n_local = h->g.n_local;
  p.g0 = h->g.g0;
  p.n_global = h->g.N;
  p.R = h->g.R;
  p.C = h->g.C;
  p.pool_row = h->g.n_local + (h->cfg.world > 1 ? h->cfg.world : 0);
  p.pool_local_row = h->g.n_local + (h->cfg.world > 1 ? h->cfg.rank : 0);
  if (h->peers) {
    p.peer_mb[0] = h->peer_mb[0];
    p.peer_mb[1] = h->peer_mb[1];
    for (int r = 0; r < pf::kMaxRanks; ++r) p.peer_blk[r] = h->peer_blk[r];
  }
  p.rank = h->cfg.rank;
  p.world = h->cfg.world;
  p.mb_parity = h->g.n_ext * h->g.tt * h->g.E;
  p.d = h->g.d;
  p.nj = h->g.nj;
  p.pool_cta = pool_cta_bytes(&h->cfg, h->g)
                   ? reinterpret_cast<u64*>(h->mailbox + 2 * h->g.n_ext * h->g.tt * h->g.E)
                   : nullptr;
  p.t = h->cfg.t;
  p.t_inv = h->cfg.t > 0 ? (65536u + static_cast<uint32_t>(h->cfg.t) - 1u) / static_cast<uint32_t>(h->cfg.t) : 0u;
  p.tt = h->g.tt;
  p.topo = h->cfg.topo;
  p.deg = h->g.deg;
  const uint32_t key0 = static_cast<uint32_t>(h->cfg.seed);
  const uint32_t key1 = static_cast<uint32_t>(h->cfg.seed >> 32);
  for (int r = 0; r < 10; ++r) {
    p.rk[2 * r] = key0 + static_cast<uint32_t>(r) * 0x9E3779B9u;
    p.rk[2 * r + 1] = key1 + static_cast<uint32_t>(r) * 0xBB67AE85u;
  }
  p.k = static_cast<uint32_t>(k);
  p.policy = h->cfg.resample_policy;
  p.policy_param = h->cfg.resample_param;
  p.mode = mode;
  p.first = (k == 1) ? 1 : 0;
  return p;
}

// Host step inputs travel inside the launch (StepParams.zin / uin): no
// separate copy, no staging buffer, nothing to synchronize.
void host_inputs(pf_handle* h, pf::StepParams& p, const float* z, const float* u) {
  p.z = nullptr;
  p.u = nullptr;
  std::memcpy(p.zin, z, sizeof(float) * h->g.zd);
  std::memcpy(p.uin, u, sizeof(float) * h->g.ud);
}

// Centralized filter: AoS state records ping-pong ([2][M][S], S =
// central_stride(d): the random-ancestor gather reads one contiguous record),
// then the log-weights ping-pong ([2][M]), then the per-particle tile sums
// (u64 [M]) and two u64 arrays of tile totals.  Vose adds per slot vscal,
// vals, prob (u64) and q32, lists, alias (32-bit), and four u64 arrays of
// tile totals / prefixes.
long long central_S(const Geometry& g) { return pf::central_stride(g.d); }
long long central_floats(const Geometry& g) { return 2 * g.M_local * central_S(g) + 2 * g.M_local; }
size_t central_bytes(const Geometry& g) {
  const size_t vose = g.vose ? sizeof(u64) * (3 * g.M_local + 4 * g.tiles) + sizeof(uint32_t) * 3 * g.M_local : 0;
  return sizeof(float) * central_floats(g) + sizeof(u64) * (g.M_local + 2 * g.tiles) + vose;
}
// weighted set of step k lives in particle buffer (central: the state records of buffer k & 1; else
// the only blocked SoA buffer)
float* set_of_step(pf_handle* h, long long k) {
  return h->parts + (h->g.central ? (k & 1) * h->g.M_local * central_S(h->g) : 0);
}
// central: the log-weights that go with the state buffer `state`
float* central_lw_of(pf_handle* h, const float* state) {
  const long long idx = (state - h->parts) / (h->g.M_local * central_S(h->g));
  return h->parts + 2 * h->g.M_local * central_S(h->g) + idx * h->g.M_local;
}

pf::CentralParams central_params(pf_handle* h, long long k) {
  pf::CentralParams c;
  std::memset(&c, 0, sizeof(c));
  c.mc = h->mc;
  c.in = set_of_step(h, k - 1);
  c.out = set_of_step(h, k);
  c.lw_in = central_lw_of(h, c.in);
  c.lw_out = central_lw_of(h, c.out);
  c.M = h->g.M_local;
  c.d = h->g.d;
  c.nj = h->g.nj;
  u64* aux = reinterpret_cast<u64*>(h->parts + central_floats(h->g));
  c.cl = aux;
  c.tile_sum = aux + h->g.M_local;
  c.tile_incl = aux + h->g.M_local + h->g.tiles;
  if (h->g.vose) {
    const long long M = h->g.M_local, T = h->g.tiles;
    u64* v = aux + M + 2 * T;
    c.vose = 1;
    c.vscal = v;
    c.vals = v + M;
    c.prob = v + 2 * M;
    c.tile_cnt = v + 3 * M;
    c.tile_cnt_incl = v + 3 * M + T;
    c.tile_D = v + 3 * M + 2 * T;
    c.tile_D_incl = v + 3 * M + 3 * T;
    uint32_t* w = reinterpret_cast<uint32_t*>(v + 3 * M + 4 * T);
    c.q32 = w;
    c.lists = reinterpret_cast<int*>(w + M);
    c.alias = reinterpret_cast<int*>(w + 2 * M);
  }
  c.key_cur = keys(h) + (k & 1);
  c.key_next = keys(h) + ((k + 1) & 1);
  c.counter = reinterpret_cast<unsigned int*>(h->scratch + kOffCounter);
  c.record_prev = record(h);
  c.record = record(h);
  c.record_host = streams_record(h) ? reinterpret_cast<u64*>(h->rec_host_dev) : nullptr;
  const uint32_t key0 = static_cast<uint32_t>(h->cfg.seed), key1 = static_cast<uint32_t>(h->cfg.seed >> 32);
  for (int r = 0; r < 10; ++r) {
    c.rk[2 * r] = key0 + static_cast<uint32_t>(r) * 0x9E3779B9u;
    c.rk[2 * r + 1] = key1 + static_cast<uint32_t>(r) * 0xBB67AE85u;
  }
  c.k = static_cast<uint32_t>(k);
  c.first = k == 1 ? 1 : 0;
  return c;
}

pf_status launch(pf_handle* h, const pf::StepParams& p0) {
  pf::StepParams p = p0;
  if (h->peers && (p.mode == pf::MODE_STEP || p.mode == pf::MODE_PUBLISH)) {
    // every rank makes the same sequence of peer-mode launches (steps and
    // publishes are collective), so the rendezvous numbers agree
    p.rv = ++h->rv;
    p.peer_timeout_ns = h->peer_timeout_ns;
  }
  // programmatic dependent launch, except when a connected peer shares this
  // device (shards of one process, or processes on one GPU): a next step's
  // waiting CTAs could hold the SMs another shard's current step needs to
  // reach the rendezvous
  return sticky(h, h->ke->launch(p, h->grid, h->stream, h->pdl && !h->local_peers && !h->shared_device));
}
pf_status launch_central(pf_handle* h, const pf::CentralParams& c) {
  return sticky(h, pf::central_step(h->g.model, h->g.nj, c, h->grid, h->stream));
}
void host_inputs(pf_handle* h, pf::CentralParams& c, const float* z, const float* u) {
  c.z = nullptr;
  c.u = nullptr;
  std::memcpy(c.zin, z, sizeof(float) * h->g.zd);
  std::memcpy(c.uin, u, sizeof(float) * h->g.ud);
}

__global__ void pf_init_kernel(float* parts, int m, long long M_local, uint32_t p0, int d, const float* mu0,
                               const float* s0, uint32_t key0, uint32_t key1, int aos_stride, float* aos_lw) {
  // F11: x_c = fma(sigma0_c, xi_c, mu0_c); pair q of particle p from words
  // 2(q&1), 2(q&1)+1 of Philox (p, 0, 2, q>>1) (R13, stream 2 = init).
  // Layout: blocked SoA [n][d+1][m]; the centralized filter (aos_stride > 0):
  // AoS records [M][aos_stride] + log-weights aos_lw [M].
  const long long row = static_cast<long long>(d + 1) * m;
  for (long long col = blockIdx.x * static_cast<long long>(blockDim.x) + threadIdx.x; col < M_local;
       col += static_cast<long long>(gridDim.x) * blockDim.x) {
    const uint32_t p = p0 + static_cast<uint32_t>(col);
    const long long cs = aos_stride ? 1 : m;   // component stride
    float* blk = aos_stride ? parts + col * aos_stride : parts + (col / m) * row + (col % m);
    pf::u32x4 blk4{0, 0, 0, 0};
    for (int q = 0; q < (d + 1) / 2; ++q) {
      if ((q & 1) == 0) blk4 = pf::philox4x32_10(p, 0u, 2u, static_cast<uint32_t>(q >> 1), key0, key1);
      const uint32_t x0 = (q & 1) ? blk4.z : blk4.x;
      const uint32_t x1 = (q & 1) ? blk4.w : blk4.y;
      float z0, z1;
      pf::normal_pair(x0, x1, z0, z1);
      const int c = 2 * q;
      blk[c * cs] = __fmaf_rn(s0[c], z0, mu0[c]);
      if (c + 1 < d) blk[(c + 1) * cs] = __fmaf_rn(s0[c + 1], z1, mu0[c + 1]);
    }
    if (aos_stride) aos_lw[col] = 0.0f;
    else blk[d * m] = 0.0f;
  }
}

// All-to-All with world > 1: the global best t of the world gathered rows
// [n_local, n_local + world) (t entries of E floats each) -> row out.
__global__ void pf_reduce_pool_kernel(const float* rows, int world, int t, int tt, int E, float* out) {
  const int lane = threadIdx.x;
  pf::u64 prev = ~0ull;
  for (int jb = 0; jb < t; ++jb) {
    pf::u64 best = 0ull;
    int be = -1;
    for (int e = lane; e < world * t; e += 32) {
      const int r = e / t, jj = e - r * t;
      const float* en = rows + (static_cast<long long>(r) * tt + jj) * E;
      const pf::u64 key = pf::order_key(en[0], __float_as_uint(en[1]));
      if (key < prev && key > best) {
        best = key;
        be = e;
      }
    }
    const pf::u64 g = pf::warp_max_u64(best);
    if (best == g && be >= 0) {
      const int r = be / t, jj = be - r * t;
      const float* en = rows + (static_cast<long long>(r) * tt + jj) * E;
      for (int c = 0; c < E; ++c) out[jb * E + c] = en[c];
    }
    prev = g;
    __syncwarp();
  }
}

// Pick the record with the maximal key among `count` (exact, order-free).
__global__ void pf_reduce_records_kernel(const float* recs, int count, int rec_floats, float* out, float* out_host) {
  const int lane = threadIdx.x;
  u64 best = 0ull;
  int bi = 0;
  for (int i = lane; i < count; i += 32) {
    const u64 k = static_cast<u64>(__float_as_uint(recs[i * rec_floats])) |
                  (static_cast<u64>(__float_as_uint(recs[i * rec_floats + 1])) << 32);
    if (k > best) {
      best = k;
      bi = i;
    }
  }
  const uint32_t hi = __reduce_max_sync(0xFFFFFFFFu, static_cast<uint32_t>(best >> 32));
  const uint32_t lo =
      __reduce_max_sync(0xFFFFFFFFu, static_cast<uint32_t>(best >> 32) == hi ? static_cast<uint32_t>(best) : 0u);
  const u64 win = (static_cast<u64>(hi) << 32) | lo;
  const unsigned mask = __ballot_sync(0xFFFFFFFFu, best == win);
  const int src_lane = __ffs(mask) - 1;
  const int src = __shfl_sync(0xFFFFFFFFu, bi, src_lane);
  for (int c = lane; c < rec_floats; c += 32) {
    const float v = recs[src * rec_floats + c];
    out[c] = v;
    if (out_host) out_host[c] = v;
  }
}

// host [d][M_local] rows <-> device blocked [n_local][d+1][m]: row c of the
// host array maps to row c of every block (cudaMemcpy2D, pitch = block size).
cudaError_t rows_to_device(pf_handle* h, float* base, const float* host, int row0, int nrows);
cudaError_t rows_to_host(pf_handle* h, const float* base, float* host, int row0, int nrows);

template <typename T>
struct DevBuf {
  T* p = nullptr;
  cudaError_t alloc(size_t n) { return cudaMalloc(&p, sizeof(T) * (n ? n : 1)); }
  ~DevBuf() {
    if (p) cudaFree(p);
  }
};

}  // namespace


extern "C" {

pf_status pf_query_sizes(const pf_config* cfg, const pf_model_params* model, pf_sizes* out) {
  Geometry g;
  const pf_status s = validate(cfg, model, &g);
  if (s != PF_OK || !out) return s != PF_OK ? s : PF_EINVAL;
  out->state = g.central ? central_bytes(g) : sizeof(float) * g.ROW * g.n_local;
  out->mailbox = sizeof(float) * 2 * g.n_ext * g.tt * g.E + pool_cta_bytes(cfg, g);
  out->scratch = kScratchBytes;
  return PF_OK;
}

pf_status pf_init(const pf_config* cfg, const pf_model_params* model, const pf_buffers* buffers,
                  void* cuda_stream, const float* mu0, const float* sigma0, pf_handle** out) {
  if (!out || !buffers || !mu0 || !sigma0) return PF_EINVAL;
  *out = nullptr;
  Geometry g;
  pf_status s = validate(cfg, model, &g);
  if (s != PF_OK) return s;
  if (!buffers->state || !buffers->mailbox || !buffers->scratch) return PF_EINVAL;
  pf_handle* h = new (std::nothrow) pf_handle();
  if (!h) return PF_ENOMEM;
  h->cfg = *cfg;
  h->mp = *model;
  h->g = g;
  // F8-F10 model constants: fp32 operations, exactly as the contract states
  // (pf_model.cuh: the 1-D linear-Gaussian model reads hs, s_th, inv_thm)
  h->mc.lj = g.model == PF_MODEL_ARM_PLANAR ? model->arm_length / static_cast<float>(model->n_joints) : 0.0f;
  h->mc.hs = model->h_s;
  h->mc.s_th = model->sigma_theta;
  h->mc.s_pos = model->sigma_pos;
  h->mc.s_vel = model->sigma_vel;
  h->mc.inv_cam = g.model == PF_MODEL_ARM_PLANAR ? 1.0f / model->sigma_cam : 0.0f;
  h->mc.inv_thm = 1.0f / model->sigma_theta_meas;
  h->parts = static_cast<float*>(buffers->state);
  h->mailbox = static_cast<float*>(buffers->mailbox);
  h->scratch = static_cast<unsigned char*>(buffers->scratch);
  h->stream = static_cast<cudaStream_t>(cuda_stream);
  h->step = 0;
  h->ke = g.central ? nullptr : find_entry(g.model, g.nj, g.m, cfg->resampler);
  h->err = PF_OK;
  int dev = 0, sms = 0, bps = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (e == cudaSuccess && g.central) {
    bps = 1;
    h->grid = pf::central_grid(g.model, g.nj, sms);
    if (h->grid < 1) e = cudaErrorInvalidConfiguration;
  } else if (e == cudaSuccess) {
    e = h->ke->prepare(&bps);
  }
  if (e == cudaSuccess && bps < 1) e = cudaErrorInvalidConfiguration;
  if (e == cudaSuccess)
    e = cudaHostAlloc(reinterpret_cast<void**>(&h->rec_host), sizeof(float) * 128, cudaHostAllocMapped);
  if (e == cudaSuccess) e = cudaHostGetDevicePointer(reinterpret_cast<void**>(&h->rec_host_dev), h->rec_host, 0);
  if (e == cudaSuccess) {
    h->mapped = std::getenv("PF_NO_MAPPED") == nullptr;
    const char* to = std::getenv("PF_PEER_TIMEOUT_MS");
    const long long ms = to ? std::atoll(to) : 30000;
    h->peer_timeout_ns = static_cast<unsigned long long>(ms > 0 ? ms : 30000) * 1000000ull;
    h->pdl = std::getenv("PF_NO_PDL") == nullptr;
    h->last_mapped = false;
    for (int c = 0; c < 4 + 32; ++c)   // no step's tag
      reinterpret_cast<volatile uint64_t*>(h->rec_host)[c] = 0xFFFFFFFF00000000ull;
  }
  if (e != cudaSuccess) {
    pf_destroy(h);
    return PF_ECUDA;
  }
  if (!g.central && !std::getenv("PF_VARIANT") && g.n_local >= kLargeNLocal) {
    const pf::KernelEntry* le = large_entry(g.model, g.nj, g.m, cfg->resampler);
    if (le && le != h->ke) {
      int b2 = 0;
      if (le->prepare(&b2) == cudaSuccess && b2 >= 1) {
        h->ke = le;
        bps = b2;
      }
    }
  }
  // fewer sub-filters than a quarter of the default mapping's groups: switch
  // to the lowest-latency mapping (more threads per sub-filter)
  if (!g.central && !std::getenv("PF_VARIANT") && g.n_local * 4 <= static_cast<long long>(bps) * sms * h->ke->s) {
    const pf::KernelEntry* le = latency_entry(g.model, g.nj, g.m, cfg->resampler);
    if (le && le != h->ke) {
      int b2 = 0;
      if (le->prepare(&b2) == cudaSuccess && b2 >= 1) {
        h->ke = le;
        bps = b2;
      }
    }
  }
  if (!g.central) {
    const long long ctas_needed = (g.n_local + h->ke->s - 1) / h->ke->s;
    const long long grid = static_cast<long long>(bps) * sms;
    h->grid = static_cast<int>(grid < ctas_needed ? grid : ctas_needed);
    if (pool_cta_bytes(cfg, g) && static_cast<long long>(h->grid) * h->ke->s > kPoolGroups)
      h->grid = static_cast<int>(kPoolGroups / h->ke->s);
  }
  // scratch: zero keys / counter; prior parameters
  float prior[128];
  std::memset(prior, 0, sizeof(prior));
  std::memcpy(prior, mu0, sizeof(float) * g.d);
  std::memcpy(prior + 64, sigma0, sizeof(float) * g.d);
  e = cudaMemsetAsync(h->scratch, 0, kScratchBytes, h->stream);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(h->scratch + kOffMu0, prior, sizeof(prior), cudaMemcpyHostToDevice, h->stream);
  if (e == cudaSuccess) e = cudaMemsetAsync(h->mailbox, 0, sizeof(float) * 2 * g.n_ext * g.tt * g.E, h->stream);
  if (e == cudaSuccess) {
    const long long blocks = (g.M_local + 255) / 256;
    pf_init_kernel<<<static_cast<int>(blocks < 8 * sms ? blocks : 8 * sms), 256, 0, h->stream>>>(
        h->parts, g.m, g.M_local, static_cast<uint32_t>(g.g0 * g.m), g.d,
        reinterpret_cast<const float*>(h->scratch + kOffMu0), reinterpret_cast<const float*>(h->scratch + kOffSigma0),
        static_cast<uint32_t>(cfg->seed), static_cast<uint32_t>(cfg->seed >> 32),
        g.central ? static_cast<int>(central_S(g)) : 0, g.central ? central_lw_of(h, h->parts) : nullptr);
    e = cudaGetLastError();
  }
  // the prior copy reads a stack buffer: finish before returning
  if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
  if (e != cudaSuccess) {
    pf_destroy(h);
    return PF_ECUDA;
  }
  *out = h;
  return PF_OK;
}

pf_status pf_step(pf_handle* h, const float* z_k, const float* u_km1) {
  if (!h || !z_k || !u_km1) return PF_EINVAL;
  if (h->err != PF_OK) return h->err;
  const long long k = h->step + 1;
  if (h->g.central) {
    pf::CentralParams c = central_params(h, k);
    if (h->cfg.flags & PF_DEVICE_INPUTS) {
      c.z = z_k;
      c.u = u_km1;
    } else {
      host_inputs(h, c, z_k, u_km1);
    }
    const pf_status s = launch_central(h, c);
    if (s == PF_OK) {
      h->step = k;
      h->last_mapped = c.record_host != nullptr;
    }
    return s;
  }
  pf::StepParams p = base_params(h, k, pf::MODE_STEP);
  if (h->cfg.flags & PF_DEVICE_INPUTS) {
    p.z = z_k;
    p.u = u_km1;
  } else {
    host_inputs(h, p, z_k, u_km1);
  }
  if (h->trace) {
    p.dbg_src = h->d_src;
    p.dbg_anc = h->d_anc;
  }
  const pf_status s = launch(h, p);
  if (s == PF_OK) {
    h->step = k;
    h->last_mapped = p.record_host != nullptr;
  }
  return s;
}

pf_status pf_step_batch(pf_handle* h, int32_t T, const float* zs, const float* us, float* est) {
  if (!h || T < 0 || (T > 0 && (!zs || !us))) return PF_EINVAL;
  if (h->err != PF_OK) return h->err;
  if (h->cfg.world != 1) return PF_ESTATE;
  const int zd = h->g.zd, ud = h->g.ud;
  h->last_mapped = false;
  for (int32_t s = 0; s < T; ++s) {
    const long long k = h->step + 1;
    if (h->g.central) {
      pf::CentralParams c = central_params(h, k);
      c.z = zs + static_cast<long long>(s) * zd;
      c.u = us + static_cast<long long>(s) * ud;
      c.est_out = est ? est + static_cast<long long>(s) * (4 + h->g.d) : nullptr;
      c.record_host = nullptr;   // device-resident pipeline: records stay on the device
      const pf_status st = launch_central(h, c);
      if (st != PF_OK) return st;
      h->step = k;
      continue;
    }
    pf::StepParams p = base_params(h, k, pf::MODE_STEP);
    p.z = zs + static_cast<long long>(s) * zd;
    p.u = us + static_cast<long long>(s) * ud;
    p.est_out = est ? est + static_cast<long long>(s) * (4 + h->g.d) : nullptr;
    p.record_host = nullptr;   // device-resident pipeline: records stay on the device
    if (h->trace) {
      p.dbg_src = h->d_src;
      p.dbg_anc = h->d_anc;
    }
    const pf_status st = launch(h, p);
    if (st != PF_OK) return st;
    h->step = k;
  }
  return PF_OK;
}

pf_status pf_estimate(pf_handle* h, float* x_hat, float* logw, int64_t* idx) {
  if (!h || !x_hat) return PF_EINVAL;
  if (h->err != PF_OK) return h->err;
  if (h->step < 1) return PF_ESTATE;
  // Host-input steps (the streaming, real-time use): the kernel wrote the
  // record into mapped pinned host memory as 64-bit words tagged with the
  // step number, so waiting is polling those words until every one carries
  // this step — no stream synchronization, and no fence in the kernel, on the
  // critical path; a stream that completes without them (or any error) ends
  // the poll.  Otherwise (device inputs, several ranks over NCCL) the record
  // is copied from the device after a stream synchronization.
  cudaError_t e = cudaSuccess;
  float rec[4 + 32 + 4];
  const int nw = 4 + h->g.d;
  if (h->last_mapped) {
    const uint32_t want = static_cast<uint32_t>(h->step);
    const uint64_t* words = reinterpret_cast<const uint64_t*>(h->rec_host);
    auto tag = [](uint64_t w) { return static_cast<uint32_t>(w >> 32); };
    unsigned it = 1;
    for (int c = 0; c < nw && e == cudaSuccess; ++c) {
      // each word is single-copy atomic: its value half belongs to its tag
      uint64_t w = __atomic_load_n(words + c, __ATOMIC_ACQUIRE);
      while (tag(w) != want) {
        if ((it++ & 1023u) == 0u) {
          const cudaError_t q = cudaStreamQuery(h->stream);
          if (q != cudaErrorNotReady) {   // the stream is idle or failed: the word is final
            w = __atomic_load_n(words + c, __ATOMIC_ACQUIRE);
            if (q != cudaSuccess) e = q;
            else if (tag(w) != want) e = cudaErrorUnknown;   // completed without this step's record
            break;
          }
        }
        w = __atomic_load_n(words + c, __ATOMIC_ACQUIRE);
      }
      const uint32_t v = static_cast<uint32_t>(w);
      std::memcpy(&rec[c], &v, 4);
    }
    // an error raised after the record surfaces at the next call (sticky)
    if (e != cudaSuccess) return sticky(h, e);
  } else {
    e = cudaMemcpyAsync(h->rec_host, record(h), sizeof(float) * nw, cudaMemcpyDeviceToHost, h->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
    if (e != cudaSuccess) return sticky(h, e);
    std::memcpy(rec, const_cast<const float*>(h->rec_host), sizeof(float) * nw);
  }
  uint32_t lo, status;
  std::memcpy(&lo, &rec[0], 4);
  std::memcpy(&status, &rec[3], 4);
  if (status == pf::kStatusPeerTimeout) {   // the device rendezvous gave up on a rank (sticky)
    if (h->err == PF_OK) h->err = PF_ETIMEOUT;
    return PF_ETIMEOUT;
  }
  std::memcpy(x_hat, rec + 4, sizeof(float) * h->g.d);
  if (logw) *logw = rec[2];
  if (idx) *idx = static_cast<int64_t>(0xFFFFFFFFu - lo);
  return PF_OK;
}

// ---- weighted-average estimate (R22) -------------------------------------
static double* mean_scratch(pf_handle* h) { return reinterpret_cast<double*>(h->scratch + kOffMean); }

static pf_status mean_partials_launch(pf_handle* h) {
  pf::MeanParams mp;
  mp.parts = set_of_step(h, h->step);
  mp.n_blocks = h->g.central ? 1 : h->g.n_local;
  mp.m = h->g.central ? static_cast<int>(h->g.M_local) : h->g.m;
  mp.d = h->g.d;
  mp.row = h->g.ROW;
  mp.aos_stride = h->g.central ? static_cast<int>(central_S(h->g)) : 0;
  mp.lw = h->g.central ? central_lw_of(h, mp.parts) : nullptr;
  mp.record = record(h);
  mp.partials = mean_scratch(h);
  return sticky(h, pf::mean_partials(mp, h->stream));
}

pf_status pf_estimate_mean(pf_handle* h, float* x_mean) {
  if (!h || !x_mean) return PF_EINVAL;
  if (h->err != PF_OK) return h->err;
  if (h->step < 1) return PF_ESTATE;
  if (h->cfg.world != 1) return PF_ESTATE;
  pf_status st = mean_partials_launch(h);
  if (st != PF_OK) return st;
  float* out = h->rec_host_dev + pf::kMeanHost;   // mapped pinned host floats (the record's tagged words are below)
  st = sticky(h, pf::mean_final(mean_scratch(h), pf::kMeanGrid, h->g.d, nullptr, nullptr, out, h->stream));
  if (st != PF_OK) return st;
  cudaError_t e = cudaStreamSynchronize(h->stream);
  if (e != cudaSuccess) return sticky(h, e);
  std::memcpy(x_mean, const_cast<const float*>(h->rec_host) + pf::kMeanHost, sizeof(float) * h->g.d);
  return PF_OK;
}

pf_status pf_mean_partial(pf_handle* h, double** partial_dev, int32_t* partial_doubles) {
  if (!h || !partial_dev) return PF_EINVAL;
  if (h->err != PF_OK) return h->err;
  if (h->step < 1) return PF_ESTATE;
  pf_status st = mean_partials_launch(h);
  if (st != PF_OK) return st;
  double* rec = mean_scratch(h) + static_cast<long long>(pf::kMeanGrid) * 33;
  st = sticky(h, pf::mean_final(mean_scratch(h), pf::kMeanGrid, h->g.d, rec, nullptr, nullptr, h->stream));
  *partial_dev = rec;
  if (partial_doubles) *partial_doubles = h->g.d + 1;
  return st;
}

pf_status pf_reduce_means(pf_handle* h, const double* partials_dev, int32_t count, float* x_mean) {
  if (!h || !partials_dev || count < 1 || !x_mean) return PF_EINVAL;
  if (h->err != PF_OK) return h->err;
  float* out = h->rec_host_dev + pf::kMeanHost;
  pf_status st = sticky(h, pf::mean_final(partials_dev, count, h->g.d, nullptr, nullptr, out, h->stream));
  if (st != PF_OK) return st;
  cudaError_t e = cudaStreamSynchronize(h->stream);
  if (e != cudaSuccess) return sticky(h, e);
  std::memcpy(x_mean, const_cast<const float*>(h->rec_host) + pf::kMeanHost, sizeof(float) * h->g.d);
  return PF_OK;
}

pf_status pf_record_ptr(pf_handle* h, float** record_dev, int32_t* record_floats) {
  if (!h || !record_dev) return PF_EINVAL;
  *record_dev = record(h);
  if (record_floats) *record_floats = 4 + h->g.d;
  return h->err;
}

pf_status pf_reduce_records(pf_handle* h, const float* records_dev, int32_t count) {
  if (!h || !records_dev || count < 1) return PF_EINVAL;
  if (h->err != PF_OK) return h->err;
  pf_reduce_records_kernel<<<1, 32, 0, h->stream>>>(records_dev, count, 4 + h->g.d, record(h), nullptr);
  return sticky(h, cudaGetLastError());
}

pf_status pf_reduce_pool(pf_handle* h) {
  if (!h) return PF_EINVAL;
  if (h->err != PF_OK) return h->err;
  if (h->cfg.topo != PF_TOPO_ALL2ALL || h->cfg.world < 2 || h->cfg.t < 1 || h->step < 1) return PF_ESTATE;
  float* mb = mailbox_parity(h, h->step);
  const long long rowf = static_cast<long long>(h->g.tt) * h->g.E;
  pf_reduce_pool_kernel<<<1, 32, 0, h->stream>>>(mb + h->g.n_local * rowf, h->cfg.world, h->cfg.t, h->g.tt, h->g.E,
                                                 mb + (h->g.n_local + h->cfg.world) * rowf);
  return sticky(h, cudaGetLastError());
}

pf_status pf_get_shard(const pf_handle* h, pf_shard* out) {
  if (!h || !out) return PF_EINVAL;
  out->g0 = h->g.g0;
  out->n_local = h->g.n_local;
  out->n_ext = h->g.n_ext;
  out->torus_rows = h->g.R;
  out->torus_cols = h->g.C;
  out->entry_floats = h->g.E;
  out->t = h->g.tt;
  out->d = h->g.d;
  out->record_floats = 4 + h->g.d;
  return PF_OK;
}

pf_status pf_get_particles(pf_handle* h, float* state_host, float* logw_host, int64_t* step) {
  if (!h || !state_host) return PF_EINVAL;
  if (h->err != PF_OK) return h->err;
  cudaError_t e = cudaStreamSynchronize(h->stream);
  if (e == cudaSuccess)
    e = rows_to_host(h, set_of_step(h, h->step), state_host, 0, h->g.d);
  if (e == cudaSuccess && logw_host) e = rows_to_host(h, set_of_step(h, h->step), logw_host, h->g.d, 1);
  if (step) *step = h->step;
  return sticky(h, e);
}

static pf_status publish(pf_handle* h, long long step) {
  cudaError_t e = cudaMemsetAsync(keys(h), 0, 2 * sizeof(u64), h->stream);
  if (e != cudaSuccess) return sticky(h, e);
  if (h->g.central) {
    pf::CentralParams c = central_params(h, step);
    c.in = set_of_step(h, step);
    c.lw_in = central_lw_of(h, c.in);
    c.publish = 1;
    return launch_central(h, c);
  }
  pf::StepParams p = base_params(h, step, pf::MODE_PUBLISH);
  return launch(h, p);
}

pf_status pf_set_particles(pf_handle* h, const float* state_host, const float* logw_host, int64_t step) {
  if (!h || !state_host || !logw_host || step < 1) return PF_EINVAL;
  if (h->err != PF_OK) return h->err;
  cudaError_t e = cudaStreamSynchronize(h->stream);
  if (e == cudaSuccess)
    e = rows_to_device(h, set_of_step(h, step), state_host, 0, h->g.d);
  if (e == cudaSuccess) e = rows_to_device(h, set_of_step(h, step), logw_host, h->g.d, 1);
  if (e != cudaSuccess) return sticky(h, e);
  pf_status s = publish(h, step);
  if (s != PF_OK) return s;
  h->step = step;
  h->last_mapped = false;
  return sticky(h, cudaStreamSynchronize(h->stream));
}

pf_status pf_debug_sample_weight(pf_handle* h, const float* state_in, const float* z_k, const float* u_km1,
                                 int64_t k, float* state_out, float* logw_out) {
  if (!h || !state_in || !z_k || !u_km1 || !state_out || !logw_out || k < 1) return PF_EINVAL;
  if (h->err != PF_OK) return h->err;
  if (h->cfg.world != 1) return PF_ESTATE;
  cudaError_t e = cudaStreamSynchronize(h->stream);
  if (e == cudaSuccess)
    e = rows_to_device(h, set_of_step(h, k - 1), state_in, 0, h->g.d);
  if (e == cudaSuccess) e = cudaMemsetAsync(keys(h), 0, 2 * sizeof(u64), h->stream);
  if (e != cudaSuccess) return sticky(h, e);
  pf_status s;
  if (h->g.central) {
    pf::CentralParams c = central_params(h, k);
    c.first = 1;   // sample + weight only (a1-a3)
    host_inputs(h, c, z_k, u_km1);
    s = launch_central(h, c);
  } else {
    pf::StepParams p = base_params(h, k, pf::MODE_SAMPLE);
    host_inputs(h, p, z_k, u_km1);
    s = launch(h, p);
  }
  if (s != PF_OK) return s;
  h->step = k;
  h->last_mapped = false;
  e = cudaStreamSynchronize(h->stream);
  if (e == cudaSuccess)
    e = rows_to_host(h, set_of_step(h, k), state_out, 0, h->g.d);
  if (e == cudaSuccess) e = rows_to_host(h, set_of_step(h, k), logw_out, h->g.d, 1);
  return sticky(h, e);
}

pf_status pf_debug_resample(pf_handle* h, const uint32_t* q, const uint32_t* ua, const uint32_t* ub,
                            int32_t* ancestors, uint64_t* prob, int32_t* alias) {
  if (!h || !q || !ua || !ub || !ancestors) return PF_EINVAL;
  if (h->err != PF_OK) return h->err;
  const long long n = h->g.N * h->g.m;
  DevBuf<uint32_t> dq, dua, dub;
  DevBuf<int> danc, dal;
  DevBuf<u64> dpr;
  const bool vose = h->cfg.resampler == PF_RESAMPLE_VOSE;
  const bool want_table = vose && prob && alias;
  cudaError_t e = dq.alloc(n);
  if (e == cudaSuccess) e = dua.alloc(n);
  if (e == cudaSuccess) e = dub.alloc(n);
  if (e == cudaSuccess) e = danc.alloc(n);
  if (e == cudaSuccess && want_table) e = dpr.alloc(n);
  if (e == cudaSuccess && want_table) e = dal.alloc(n);
  if (e == cudaSuccess) e = cudaMemcpy(dq.p, q, 4 * n, cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(dua.p, ua, 4 * n, cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(dub.p, ub, 4 * n, cudaMemcpyHostToDevice);
  if (e == cudaSuccess && h->g.central) {
    // one filter over all M slots (clobbers the handle's scan / table arrays)
    const pf::CentralParams c = central_params(h, h->step + 1);
    e = pf::central_resample_debug(c, dq.p, dua.p, dub.p, danc.p, h->stream);
    if (e == cudaSuccess && want_table) e = cudaMemcpyAsync(dpr.p, c.prob, 8 * n, cudaMemcpyDeviceToDevice, h->stream);
    if (e == cudaSuccess && want_table) e = cudaMemcpyAsync(dal.p, c.alias, 4 * n, cudaMemcpyDeviceToDevice, h->stream);
  } else if (e == cudaSuccess) {
    e = h->ke->resample_debug(dq.p, dua.p, dub.p, danc.p, want_table ? dpr.p : nullptr, want_table ? dal.p : nullptr,
                              h->g.N, h->stream);
  }
  if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
  if (e == cudaSuccess) e = cudaMemcpy(ancestors, danc.p, 4 * n, cudaMemcpyDeviceToHost);
  if (e == cudaSuccess && want_table) e = cudaMemcpy(prob, dpr.p, 8 * n, cudaMemcpyDeviceToHost);
  if (e == cudaSuccess && want_table) e = cudaMemcpy(alias, dal.p, 4 * n, cudaMemcpyDeviceToHost);
  return sticky(h, e);
}

pf_status pf_debug_exchange(pf_handle* h, const float* logw, int64_t* src) {
  if (!h || !logw || !src) return PF_EINVAL;
  if (h->err != PF_OK) return h->err;
  if (h->cfg.world != 1 || h->g.central) return PF_ESTATE;
  const long long M = h->g.M_local;
  DevBuf<long long> dsrc;
  cudaError_t e = dsrc.alloc(M);
  if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
  if (e == cudaSuccess) e = rows_to_device(h, h->parts, logw, h->g.d, 1);
  if (e != cudaSuccess) return sticky(h, e);
  const long long s = h->step > 0 ? h->step : 1;
  pf_status st = publish(h, s);
  if (st != PF_OK) return st;
  pf::StepParams p = base_params(h, s + 1, pf::MODE_EXCHANGE);
  p.dbg_src = dsrc.p;
  st = launch(h, p);
  if (st != PF_OK) return st;
  h->step = s;
  h->last_mapped = false;
  e = cudaStreamSynchronize(h->stream);
  if (e == cudaSuccess) e = cudaMemcpy(src, dsrc.p, sizeof(long long) * M, cudaMemcpyDeviceToHost);
  return sticky(h, e);
}

pf_status pf_set_trace(pf_handle* h, int32_t enable) {
  if (!h) return PF_EINVAL;
  if (h->g.central) return enable ? PF_ESTATE : PF_OK;
  if (enable && !h->trace) {
    cudaError_t e = cudaStreamSynchronize(h->stream);
    if (e == cudaSuccess) e = cudaMalloc(&h->d_src, sizeof(long long) * h->g.M_local);
    if (e == cudaSuccess) e = cudaMalloc(&h->d_anc, sizeof(int) * h->g.M_local);
    if (e != cudaSuccess) return sticky(h, e);
    h->trace = true;
  } else if (!enable && h->trace) {
    cudaStreamSynchronize(h->stream);
    cudaFree(h->d_src);
    cudaFree(h->d_anc);
    h->d_src = nullptr;
    h->d_anc = nullptr;
    h->trace = false;
  }
  return h->err;
}

pf_status pf_get_trace(pf_handle* h, int64_t* src, int32_t* ancestors) {
  if (!h) return PF_EINVAL;
  if (!h->trace) return PF_ESTATE;
  cudaError_t e = cudaStreamSynchronize(h->stream);
  if (e == cudaSuccess && src)
    e = cudaMemcpy(src, h->d_src, sizeof(long long) * h->g.M_local, cudaMemcpyDeviceToHost);
  if (e == cudaSuccess && ancestors)
    e = cudaMemcpy(ancestors, h->d_anc, sizeof(int) * h->g.M_local, cudaMemcpyDeviceToHost);
  return sticky(h, e);
}

// ---- peer transport (NVLink / NVSwitch peer memory via CUDA IPC) ----------
namespace {
// [kMaxRanks] u64 flags + [2][kMaxRanks][kPeerRec] record floats + [2][kMaxRanks][kPeerPool] pool floats
constexpr size_t kPeerBlockBytes = 81920;
static_assert(pf::kPeerBlockUsed <= kPeerBlockBytes, "peer block");

pf_status peer_check(const pf_handle* h) {
  if (!h) return PF_EINVAL;
  if (h->err != PF_OK) return h->err;
  if (h->g.central || h->cfg.world < 2 || h->cfg.world > pf::kMaxRanks) return PF_ESTATE;
  if (h->cfg.topo != PF_TOPO_RING && h->cfg.topo != PF_TOPO_TORUS2D && h->cfg.topo != PF_TOPO_ALL2ALL)
    return PF_EUNSUPPORTED;
  if (h->step != 0 || h->peers) return PF_ESTATE;   // connect once, before the first step
  return PF_OK;
}
pf_status ensure_block(pf_handle* h) {
  if (h->own_blk) return PF_OK;
  cudaError_t e = cudaMalloc(&h->own_blk, kPeerBlockBytes);
  if (e == cudaSuccess) e = cudaMemset(h->own_blk, 0, kPeerBlockBytes);
  if (e != cudaSuccess) {
    h->own_blk = nullptr;
    return sticky(h, e);
  }
  return PF_OK;
}
void set_peers(pf_handle* h, float* prev_mb, float* next_mb, unsigned char* const* blks) {
  h->peer_mb[0] = prev_mb;
  h->peer_mb[1] = next_mb;
  for (int r = 0; r < pf::kMaxRanks; ++r) h->peer_blk[r] = r < h->cfg.world ? blks[r] : nullptr;
  h->peers = true;
}
}  // namespace

pf_status pf_peer_export(pf_handle* h, uint8_t* blob) {
  pf_status st = peer_check(h);
  if (st != PF_OK || !blob) return st != PF_OK ? st : PF_EINVAL;
  if ((st = ensure_block(h)) != PF_OK) return st;
  // the caller's mailbox lives inside some cudaMalloc allocation: export that
  // allocation and the mailbox's offset in it
  typedef int (*AddrRange)(unsigned long long*, size_t*, unsigned long long);
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaError_t e = cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &q);
  if (e != cudaSuccess || !fn) return sticky(h, e != cudaSuccess ? e : cudaErrorNotSupported);
  unsigned long long base = 0;
  size_t size = 0;
  if (reinterpret_cast<AddrRange>(fn)(&base, &size, reinterpret_cast<unsigned long long>(h->mailbox)) != 0)
    return sticky(h, cudaErrorInvalidValue);
  cudaIpcMemHandle_t hm, hb;
  e = cudaIpcGetMemHandle(&hm, reinterpret_cast<void*>(base));
  if (e == cudaSuccess) e = cudaIpcGetMemHandle(&hb, h->own_blk);
  if (e != cudaSuccess) return sticky(h, e);
  const unsigned long long off = reinterpret_cast<unsigned long long>(h->mailbox) - base;
  std::memset(blob, 0, PF_PEER_BLOB_BYTES);
  std::memcpy(blob, &hm, sizeof(hm));
  std::memcpy(blob + 64, &off, sizeof(off));
  std::memcpy(blob + 72, &hb, sizeof(hb));
  const int64_t rank = h->cfg.rank;
  std::memcpy(blob + 136, &rank, sizeof(rank));
  // the device's PCI bus id (peers on the same device turn PDL off)
  int dev = 0;
  e = cudaGetDevice(&dev);
  if (e == cudaSuccess) e = cudaDeviceGetPCIBusId(reinterpret_cast<char*>(blob + 144), 16, dev);
  if (e != cudaSuccess) return sticky(h, e);
  return PF_OK;
}

pf_status pf_peer_connect(pf_handle* h, const uint8_t* blobs) {
  pf_status st = peer_check(h);
  if (st != PF_OK || !blobs) return st != PF_OK ? st : PF_EINVAL;
  if (!h->own_blk) return PF_ESTATE;   // pf_peer_export first
  const int W = h->cfg.world, r = h->cfg.rank;
  const int prev = (r + W - 1) % W, next = (r + 1) % W;
  unsigned char* blks[pf::kMaxRanks] = {};
  float* mbs[pf::kMaxRanks] = {};
  const uint8_t* mine = blobs + static_cast<size_t>(r) * PF_PEER_BLOB_BYTES;
  bool shared = false;
  for (int q = 0; q < W; ++q) {
    const uint8_t* b = blobs + static_cast<size_t>(q) * PF_PEER_BLOB_BYTES;
    int64_t qr;
    std::memcpy(&qr, b + 136, sizeof(qr));
    if (qr != q) return PF_EINVAL;
    if (q != r && std::memcmp(b + 144, mine + 144, 16) == 0) shared = true;
    if (q == r) {
      blks[q] = h->own_blk;
      mbs[q] = h->mailbox;
      continue;
    }
    cudaIpcMemHandle_t hb;
    std::memcpy(&hb, b + 72, sizeof(hb));
    void* pb = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&pb, hb, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) return sticky(h, e);
    h->opened[h->n_opened++] = pb;
    blks[q] = static_cast<unsigned char*>(pb);
    if (q == prev || q == next) {
      cudaIpcMemHandle_t hm;
      unsigned long long off;
      std::memcpy(&hm, b, sizeof(hm));
      std::memcpy(&off, b + 64, sizeof(off));
      void* pm = nullptr;
      e = cudaIpcOpenMemHandle(&pm, hm, cudaIpcMemLazyEnablePeerAccess);
      if (e != cudaSuccess) return sticky(h, e);
      h->opened[h->n_opened++] = pm;
      mbs[q] = reinterpret_cast<float*>(static_cast<unsigned char*>(pm) + off);
    }
  }
  set_peers(h, mbs[prev], mbs[next], blks);
  h->shared_device = shared;
  return PF_OK;
}

pf_status pf_peer_connect_local(pf_handle* const* handles, int32_t world) {
  if (!handles || world < 2 || world > pf::kMaxRanks) return PF_EINVAL;
  unsigned char* blks[pf::kMaxRanks] = {};
  for (int q = 0; q < world; ++q) {
    pf_handle* h = handles[q];
    pf_status st = peer_check(h);
    if (st != PF_OK) return st;
    if (h->cfg.world != world || h->cfg.rank != q) return PF_EINVAL;
    if ((st = ensure_block(h)) != PF_OK) return st;
    blks[q] = h->own_blk;
  }
  for (int q = 0; q < world; ++q) {
    pf_handle* h = handles[q];
    set_peers(h, handles[(q + world - 1) % world]->mailbox, handles[(q + 1) % world]->mailbox, blks);
    h->local_peers = true;
  }
  return PF_OK;
}

int32_t pf_peer_connected(const pf_handle* h) { return h && h->peers ? 1 : 0; }

pf_status pf_query_mapping(const pf_handle* h, int32_t* out) {
  if (!h || !out) return PF_EINVAL;
  if (h->g.central || !h->ke) return PF_ESTATE;
  const pf::KernelEntry& e = *h->ke;
  int n = 0;   // compiled mappings of (model, n_joints, m, resampler): the range of PF_VARIANT
  for (int ti = 0; ti < kTables; ++ti) {
    const Table t = tables(ti);
    for (int i = 0; i < t.n; ++i)
      if (matches(t.e[i], h->g.model, h->g.nj, h->g.m, h->cfg.resampler)) ++n;
  }
  const int32_t v[8] = {e.gw, e.s, e.nstage, e.unr, e.minb, e.split, h->grid, n};
  std::memcpy(out, v, sizeof(v));
  return PF_OK;
}

pf_status pf_destroy(pf_handle* h) {
  if (!h) return PF_OK;
  cudaStreamSynchronize(h->stream);
  for (int i = 0; i < h->n_opened; ++i) cudaIpcCloseMemHandle(h->opened[i]);
  if (h->own_blk) cudaFree(h->own_blk);
  if (h->rec_host) cudaFreeHost(h->rec_host);
  if (h->d_src) cudaFree(h->d_src);
  if (h->d_anc) cudaFree(h->d_anc);
  delete h;
  return PF_OK;
}

const char* pf_strerror(pf_status s) {
  switch (s) {
    case PF_OK: return "ok";
    case PF_EINVAL: return "invalid argument or configuration";
    case PF_ENOMEM: return "host allocation failed";
    case PF_ECUDA: return "CUDA error";
    case PF_ESTATE: return "call not valid in the handle's state";
    case PF_EUNSUPPORTED: return "configuration not compiled (model, n_joints, m)";
    case PF_ETIMEOUT: return "peer rendezvous timed out (a rank did not arrive)";
    default: return "unknown pf_status";
  }
}

pf_status pf_last_error(const pf_handle* h) { return h ? h->err : PF_EINVAL; }

int32_t pf_supported(int32_t* n_joints, int32_t* m, int32_t cap) {
  int32_t n = 0;
  for (int ti = 0; ti < kTables; ++ti) {
    const Table t = tables(ti);
    for (int i = 0; i < t.n; ++i) {
      if (t.e[i].model != PF_MODEL_ARM_PLANAR || t.e[i].nj <= 0) continue;
      bool dup = false;
      for (int j = 0; j < i; ++j) dup = dup || (t.e[j].m == t.e[i].m && t.e[j].nj == t.e[i].nj);
      if (t.e[i].res != 0 || dup) continue;
      if (n < cap && n_joints && m) {
        n_joints[n] = t.e[i].nj;
        m[n] = t.e[i].m;
      }
      ++n;
    }
  }
  return n;
}

}  // extern "C"

namespace {
cudaError_t rows_to_device(pf_handle* h, float* base, const float* host, int row0, int nrows) {
  if (h->g.central) {   // AoS records + the log-weight array (transposed on the host)
    const long long M = h->g.M_local, S = central_S(h->g);
    const int d = h->g.d;
    if (row0 == d && nrows == 1)
      return cudaMemcpy(central_lw_of(h, base), host, sizeof(float) * M, cudaMemcpyHostToDevice);
    if (row0 != 0 || nrows != d) return cudaErrorInvalidValue;
    float* tmp = static_cast<float*>(std::calloc(static_cast<size_t>(M * S), sizeof(float)));
    if (!tmp) return cudaErrorMemoryAllocation;
    for (int c = 0; c < d; ++c)
      for (long long p = 0; p < M; ++p) tmp[p * S + c] = host[c * M + p];
    const cudaError_t e = cudaMemcpy(base, tmp, sizeof(float) * M * S, cudaMemcpyHostToDevice);
    std::free(tmp);
    return e;
  }
  const size_t m = h->g.m;
  for (int r = 0; r < nrows; ++r) {
    cudaError_t e = cudaMemcpy2D(base + (row0 + r) * m, sizeof(float) * h->g.ROW,
                                 host + static_cast<size_t>(r) * h->g.M_local, sizeof(float) * m, sizeof(float) * m,
                                 h->g.n_local, cudaMemcpyHostToDevice);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}
cudaError_t rows_to_host(pf_handle* h, const float* base, float* host, int row0, int nrows) {
  if (h->g.central) {
    const long long M = h->g.M_local, S = central_S(h->g);
    const int d = h->g.d;
    if (row0 == d && nrows == 1)
      return cudaMemcpy(host, central_lw_of(h, base), sizeof(float) * M, cudaMemcpyDeviceToHost);
    if (row0 != 0 || nrows != d) return cudaErrorInvalidValue;
    float* tmp = static_cast<float*>(std::malloc(sizeof(float) * M * S));
    if (!tmp) return cudaErrorMemoryAllocation;
    const cudaError_t e = cudaMemcpy(tmp, base, sizeof(float) * M * S, cudaMemcpyDeviceToHost);
    if (e == cudaSuccess)
      for (int c = 0; c < d; ++c)
        for (long long p = 0; p < M; ++p) host[c * M + p] = tmp[p * S + c];
    std::free(tmp);
    return e;
  }
  const size_t m = h->g.m;
  for (int r = 0; r < nrows; ++r) {
    cudaError_t e = cudaMemcpy2D(host + static_cast<size_t>(r) * h->g.M_local, sizeof(float) * m,
                                 base + (row0 + r) * m, sizeof(float) * h->g.ROW, sizeof(float) * m,
                                 h->g.n_local, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}
}  // namespace
