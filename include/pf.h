/*
 * include/pf.h — C ABI of libpf_b200.so, the B200 (sm_100a) hot path of the
 * fully distributed particle filter of Chitchian, van Amesfoort, Simonetto,
 * Keviczky, Sips, "Adapting Particle Filter Algorithms to Many-Core
 * Architectures", IPDPS 2013 (/root/reference/PAPER.md; "PAPER.md:16" = PDF
 * page 4).  Readings R1–R20 and the fp32 contract F1–F11 are
 * in DESIGN.md §3–§4.
 *
 * Conventions (all functions):
 *  - Return pf_status: PF_OK (0) or a negative code.  No exceptions, no
 *    printing.  CUDA errors are sticky on the handle (pf_last_error) and are
 *    returned by every later call until pf_destroy.
 *  - Device buffers (pf_buffers) are allocated and owned by the CALLER (the
 *    Python layer uses torch), sized by pf_query_sizes, 256-byte aligned, and
 *    must outlive the handle.  The caller owns the cudaStream_t.  The handle
 *    owns only host metadata and small pinned staging memory.
 *  - "host" pointers are ordinary CPU memory; "device" pointers are CUDA
 *    device memory of the handle's device.  Work is stream-ordered on the
 *    handle's stream; only pf_estimate / pf_get_particles / the debug hooks
 *    synchronize it.
 *  - A handle is used by one host thread at a time.
 *  - Device layout (blocked SoA): the particle buffer is float32
 *    [n_local][d+1][m] — for every local sub-filter one contiguous block
 *    whose rows 0..d-1 are the state components (d = n_joints + 4:
 *    theta_0..theta_{n_j-1}, x, y, v_x, v_y — PAPER.md:22 §VII-A) of its m
 *    particles and whose row d is their log-weight (reading R7).  The
 *    centralized filter (n_filters == 1, m > 1024) instead keeps AoS records:
 *    float [2][m][S] states (S = d rounded up to even; ping-pong by step
 *    parity), then float [2][m] log-weights, then its resampling tables — so
 *    the global resampler's random-ancestor gather reads one contiguous record.
 *  - Host layout (get/set/debug hooks): state float32 [d][M_local] (row c =
 *    component c of every local particle, column n_local*m + i for
 *    sub-filter n_local, slot i), log-weights float32 [M_local].
 */
#ifndef PF_H
#define PF_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  PF_OK = 0,
  PF_EINVAL = -1,        /* invalid argument / configuration                 */
  PF_ENOMEM = -2,        /* host allocation failed                           */
  PF_ECUDA = -3,         /* CUDA error (sticky)                              */
  PF_ESTATE = -5,        /* call not valid in the handle's state             */
  PF_EUNSUPPORTED = -6,  /* (model, n_joints, m) combination not compiled    */
  PF_ETIMEOUT = -7       /* peer transport: a rank did not reach the device  */
                         /* rendezvous within PF_PEER_TIMEOUT_MS (sticky)    */
} pf_status;

/* Exchange scheme X (PAPER.md:18 Table I; :16 Fig.1; :20 §VI-E): Ring and
 * 2D Torus exchange t particles per neighbour pair; All-to-All — "each
 * sub-filter supplies [t]. Then, all sub-filters read back the same t best
 * particles from the supplied set" (§VI-E). */
typedef enum { PF_TOPO_NONE = 0, PF_TOPO_RING = 1, PF_TOPO_TORUS2D = 2, PF_TOPO_ALL2ALL = 3 } pf_topology;
/* Resampler (PAPER.md:18 §IV; :20–22 §VI-F). */
typedef enum { PF_RESAMPLE_RWS = 0, PF_RESAMPLE_VOSE = 1 } pf_resampler;
/* Model hooks (the paper separates "generic particle filtering from
 * model-specific routines.  New dynamical system models can be easily
 * added", §I).  The step kernels are templates over a model
 * policy (csrc/pf_model.cuh: state / measurement / control dimensions and
 * the sample (F8) and weight (F10) hooks, fused into the step); a model id
 * selects the compiled instance.
 *  PF_MODEL_ARM_PLANAR       the robotic arm of PAPER.md:22–24 §VII-A with
 *                            h(x) of reading R14; d = n_joints + 4, z has
 *                            n_joints + 2 entries (x_C, y_C, joint angles),
 *                            u has n_joints; compiled for n_joints in
 *                            {2, 5, 28}, any other n_joints <= 28 through the
 *                            generic runtime-dimension arm (bit-identical);
 *                            > 28: PF_EUNSUPPORTED.
 *  PF_MODEL_LINEAR_GAUSS_1D  one joint with its angle sensor and no camera:
 *                            theta_k = theta_{k-1} + h_s u + w,
 *                            w ~ N(0, sigma_theta^2); z = theta + v,
 *                            v ~ N(0, sigma_theta_meas^2); d = 1, z and u
 *                            one entry each (the Kalman special case of
 *                            SURVEY §8(c)); n_joints, arm_length,
 *                            sigma_pos/vel/cam are ignored. */
typedef enum { PF_MODEL_ARM_PLANAR = 0, PF_MODEL_LINEAR_GAUSS_1D = 1 } pf_model_id;

/* pf_config.flags */
#define PF_DEVICE_INPUTS 1u   /* pf_step's z / u are device pointers         */

/* When a sub-filter resamples (§IV: "we have experimented with
 * the suggested metric to compute the effective sample size as well as a
 * simpler resampling frequency parameter (each sub-filter randomly decides to
 * resample at a fixed ratio of the time)"; reading R21).  A sub-filter that
 * does not resample keeps its particles and carries its normalised
 * log-weight l - l_max into the next weight (F12). */
typedef enum {
  PF_POLICY_ALWAYS = 0,   /* resample every step (the paper's choice)                     */
  PF_POLICY_ESS = 1,      /* resample iff Q^2 2^16 < param m sum q^2 (ESS < tau m, tau =   */
                          /* param / 2^16; q = the integer weights of F7, exact integers)  */
  PF_POLICY_FREQ = 2      /* resample iff word 0 of Philox (n, k, 1, 0) < param            */
                          /* (param = ratio 2^32 in [0, 2^32])                             */
} pf_policy;

typedef struct {
  int32_t model;            /* pf_model_id                                           */
  int32_t n_joints;         /* joints incl. base rotation; d = n_joints + 4          */
  float arm_length;         /* L (m); link length L / n_joints (R16)                 */
  float h_s;                /* sampling time (s) (R16)                               */
  float sigma_theta;        /* process noise std, joint angles (R15)                 */
  float sigma_pos;          /* process noise std, object x, y                        */
  float sigma_vel;          /* process noise std, object v_x, v_y                    */
  float sigma_cam;          /* measurement noise std, camera (x_C, y_C)              */
  float sigma_theta_meas;   /* measurement noise std, joint sensors                  */
} pf_model_params;

/* Table I: m, N, X, t; plus resampler, RNG seed and the shard
 * of this process.  Sharding: ring — rank r owns global
 * sub-filters [r N/W, (r+1) N/W); torus — rank r owns rows
 * [r R/W, (r+1) R/W) of the R x C grid. */
typedef struct {
  int32_t m;                /* particles per sub-filter, power of two in [32, 1024]; */
                            /* n_filters == 1 and m > 1024: the centralized filter  */
                            /* (multiple of 4096, <= 2^26; Vose <= 2^20), see below */
  int64_t n_filters;        /* N, GLOBAL number of sub-filters                       */
  int32_t t;                /* particles per exchange per neighbour; deg*t < m (R19) */
  int32_t topo;             /* pf_topology                                           */
  int32_t torus_rows;       /* 0 = default R = 2^floor(log2(N)/2) (R4)               */
  int32_t torus_cols;       /* 0 = default N / R                                     */
  int32_t resampler;        /* pf_resampler                                          */
  uint64_t seed;            /* Philox key = (seed & 0xffffffff, seed >> 32) (R12)    */
  int32_t rank;             /* shard index in [0, world)                             */
  int32_t world;            /* number of shards (processes / GPUs), >= 1             */
  uint32_t flags;           /* PF_DEVICE_INPUTS                                      */
  int32_t resample_policy;  /* pf_policy (sub-filters; the centralized filter: ALWAYS) */
  uint64_t resample_param;  /* see pf_policy; <= 2^32                                */
} pf_config;

/* Bytes of each caller-owned device buffer. */
typedef struct {
  uint64_t state;    /* float [n_local][d+1][m]: states + log-weights (blocked SoA); */
                     /* centralized filter: AoS records + tables, see above        */
  uint64_t mailbox;  /* float [2][n_ext][max(t,1)][d+2]: exchange mailbox, see below */
  uint64_t scratch;  /* keys, counters, estimate record, step inputs                */
} pf_sizes;

typedef struct {
  void* state;
  void* mailbox;
  void* scratch;
} pf_buffers;

/* Shard geometry (multi-rank plumbing).  Mailbox entry (d+2 floats) =
 * [logw, global particle index (uint32 bits), x_0..x_{d-1}]; mailbox parity
 * k&1 holds the best t of every local sub-filter after step k at rows
 * [0, n_local), and rows [n_local, n_ext) are halo rows the caller fills
 * with neighbour ranks' entries before step k+1: ring — row n_local holds
 * global sub-filter (g0-1) mod N, row n_local+1 holds (g0+n_local) mod N;
 * torus — rows n_local + c hold grid row (r0-1) mod R, rows
 * n_local + C + c hold grid row (r1) mod R (c = column).  All-to-All: the
 * kernel writes this shard's best t of the pool into row n_local + rank
 * (world > 1) or n_local (world == 1); with world > 1 the caller all-gathers
 * rows [n_local, n_local + world) and calls pf_reduce_pool, which writes the
 * global best t into row n_local + world — the row every sub-filter reads. */
typedef struct {
  int64_t g0;            /* first global sub-filter of this shard                  */
  int64_t n_local;       /* local sub-filters                                      */
  int64_t n_ext;         /* n_local + halo rows                                    */
  int64_t torus_rows;    /* R (torus) or 0                                         */
  int64_t torus_cols;    /* C (torus) or 0                                         */
  int32_t entry_floats;  /* d + 2                                                  */
  int32_t t;             /* entries per sub-filter row (max(t, 1))                 */
  int32_t d;             /* state dimension                                        */
  int32_t record_floats; /* 4 + d                                                  */
} pf_shard;

typedef struct pf_handle pf_handle;

/* Sizes of the caller-owned buffers for (cfg, model).  PF_EINVAL on an
 * invalid configuration (same checks as pf_init). */
pf_status pf_query_sizes(const pf_config* cfg, const pf_model_params* model, pf_sizes* out);

/* Create a handle on the current CUDA device and draw the initial particle
 * set X_0 ~ N(mu0, diag(sigma0^2)) (implicit input of Algorithm 2, PAPER.md:16;
 * F11, Philox stream 2).  mu0, sigma0: host float[d].  cuda_stream: a
 * cudaStream_t (NULL = legacy default stream).  Validation (PF_EINVAL): m a
 * power of two in [32, 1024]; deg*t < m; N % world == 0 (ring) or
 * R % world == 0 and R*C == N (torus); N*m per shard <= 2^31; global N*m <= 2^32;
 * 0 <= rank < world; unsupported n_joints -> PF_EUNSUPPORTED.
 * Centralized filter ("a sequential, centralized particle filter", PAPER.md:18
 * §VI; Fig. 5 and 9): n_filters == 1 and m > 1024 resamples
 * all m particles globally (RWS or Vose over every slot, no exchange:
 * topo NONE or t == 0; world == 1); m a multiple of 4096 and <= 2^26, Vose
 * m <= 2^20 (PF_EUNSUPPORTED above: its u64 alias sums reach m^2 2^22). */
pf_status pf_init(const pf_config* cfg, const pf_model_params* model, const pf_buffers* buffers,
                  void* cuda_stream, const float* mu0, const float* sigma0, pf_handle** out);

/* One time step k = (last step) + 1 of Algorithm 2: exchange
 * with the neighbours' best t of step k-1 (l.10–14), normalise + resample
 * locally (l.15–19), sample + weight (l.3–6), local/global estimate (l.8–9).
 * z_k: float[zd] and u_{k-1}: float[ud], the model's measurement and
 * control (arm: zd = n_joints + 2 = (x_C, y_C, theta_hat_0..), ud =
 * n_joints; linear-Gaussian: one each).  Host pointers — their values travel to
 * the device inside the kernel launch, so the buffers may be reused as soon
 * as the call returns — unless PF_DEVICE_INPUTS (device pointers, read by the
 * kernel).  Asynchronous.
 * With world > 1 the caller must have filled the halo rows of mailbox
 * parity (k-1)&1 (see pf_shard) and, after the step, reduce the per-rank
 * records (pf_reduce_records) for a global estimate. */
pf_status pf_step(pf_handle* h, const float* z_k, const float* u_km1);

/* T consecutive steps with device-resident inputs zs [T][zd] and
 * us [T][ud] (device), writing each step's estimate record
 * (4 + d floats, layout of pf_record_ptr) to est [T][4+d] (device, nullable).
 * world == 1 only (PF_ESTATE otherwise).  Asynchronous (T back-to-back
 * launches on the handle's stream, no host synchronization). */
pf_status pf_step_batch(pf_handle* h, int32_t T, const float* zs, const float* us, float* est);

/* The global estimate of the last step: the particle with the highest
 * weight (PAPER.md:16 §IV; :20 §VI-D; R6).  Blocks until that record is on
 * the host: after a host-input pf_step of a single-rank filter (or of a
 * peer-connected rank) the step kernel streams it into mapped pinned host
 * memory as 64-bit words, each tagged with the step number, and this call
 * polls them until every word carries this step (work queued after the step
 * may still be running); otherwise it synchronizes the stream and copies the
 * record.
 * Device errors of the step are reported either way.
 * x_hat: host float[d]; logw, idx (global particle index): host, nullable.
 * PF_ESTATE before the first step. */
pf_status pf_estimate(pf_handle* h, float* x_hat, float* logw, int64_t* idx);

/* Weighted-average estimate of the last step's weighted set ("The
 * reduction operator can compute the particle with the highest weight, a
 * weighted average, or any other associative operator", §VI-D;
 * reading R22): x_c = sum_p w_p x_cp / sum_p w_p with the integer weights
 * w_p = floor(2^22 exp(l_p - L)) of F7, L = the best log-weight of the
 * estimate record; numerators summed in double (each product exact),
 * divided once.  x_mean: host float[d].  One extra read pass over the
 * particle set; synchronizes.  world == 1 (else PF_ESTATE: use the two
 * calls below); PF_ESTATE before the first step. */
pf_status pf_estimate_mean(pf_handle* h, float* x_mean);

/* Sharded filters (world > 1), after pf_reduce_records made L global: this
 * shard's partial record, device double[d+1] = [sum w (uint64 bit pattern),
 * sum w x_0, ..., sum w x_{d-1}] (stream-ordered, asynchronous), and the
 * mean of `count` such records (device [count][d+1], e.g. an all-gather;
 * summed in order) into host float[d] (synchronizes). */
pf_status pf_mean_partial(pf_handle* h, double** partial_dev, int32_t* partial_doubles);
pf_status pf_reduce_means(pf_handle* h, const double* partials_dev, int32_t count, float* x_mean);

/* Device pointer to this shard's estimate record of the last step:
 * float[4 + d] = [key lo (u32 bits), key hi (u32 bits), logw, reserved, x[d]]
 * with key = (ordered(logw) << 32) | (0xffffffff - global index). */
pf_status pf_record_ptr(pf_handle* h, float** record_dev, int32_t* record_floats);

/* Global estimate from `count` records (device, [count][4+d], e.g. an
 * all-gather of every rank's record): picks the maximal key (exact,
 * order-free) and makes it this handle's estimate.  Asynchronous. */
pf_status pf_reduce_records(pf_handle* h, const float* records_dev, int32_t count);

/* All-to-All with world > 1: after the rows [n_local, n_local + world) of
 * the last step's mailbox parity hold every rank's best t (all-gather),
 * select the global best t (order key R6; exact) into row n_local + world.
 * Asynchronous.  PF_ESTATE unless topo == PF_TOPO_ALL2ALL and world > 1. */
pf_status pf_reduce_pool(pf_handle* h);

/* Shard geometry and mailbox layout for halo exchange. */
pf_status pf_get_shard(const pf_handle* h, pf_shard* out);

/* Checkpoint: copy the weighted particle set of the last step (host layout:
 * state [d][M_local], logw [M_local]) and its step index (step 0 = prior,
 * logw = 0).  Synchronizes. */
pf_status pf_get_particles(pf_handle* h, float* state_host, float* logw_host, int64_t* step);
/* Resume: load a weighted particle set as the result of step `step` >= 1
 * (host pointers), republish its best t to the mailbox and its estimate.
 * With the counter-based RNG, resuming is bit-exact.  Synchronizes. */
pf_status pf_set_particles(pf_handle* h, const float* state_host, const float* logw_host, int64_t step);

/* ---- test hooks: the same device code on isolated phases.  They clobber
 * the handle's particles, mailbox and estimate.  world == 1 only. ---- */

/* Sample + weight (a1–a3) every particle of state_in [d][M] (host) with no
 * resampling, Philox counter (p, k, 0, j) (R13): state_out [d][M],
 * logw_out [M] (host). */
pf_status pf_debug_sample_weight(pf_handle* h, const float* state_in, const float* z_k,
                                 const float* u_km1, int64_t k, float* state_out, float* logw_out);

/* Resampling (a8) of integer weights q [N][m] (host, each row with
 * sum > 0 and sum <= 2^32) with explicit uniforms ua, ub [N][m] (host):
 * ancestors [N][m] (host).  Vose only: prob [N][m] (uint64, units of the
 * row sum) and alias [N][m] (host, nullable) of the alias table (R10).
 * Centralized filter: one row of m (sum <= m 2^22), device-wide passes. */
pf_status pf_debug_resample(pf_handle* h, const uint32_t* q, const uint32_t* ua, const uint32_t* ub,
                            int32_t* ancestors, uint64_t* prob, int32_t* alias);

/* Exchange (a6) of log-weights logw [N][m] (host): src [N][m] (host) = the
 * global index of the particle each slot holds after the exchange (R2–R5). */
pf_status pf_debug_exchange(pf_handle* h, const float* logw, int64_t* src);

/* Exchange sources and ancestors of the last pf_step (host, [M_local] each,
 * nullable); recorded only when PF_TRACE was enabled with pf_set_trace. */
pf_status pf_set_trace(pf_handle* h, int32_t enable);
pf_status pf_get_trace(pf_handle* h, int64_t* src, int32_t* ancestors);

/* Element-wise evaluation of the device fp32 contract for
 * bit-exact comparison with the oracle.  Host arrays of 32-bit words:
 *   PF_MATH_SIN / COS / LOG / SQRT: in float[n] -> out float[n]  (F5, F6, sqrt of F2)
 *   PF_MATH_EXPQ: in float[n] (delta <= 0) -> out uint32[n]      (F7)
 *   PF_MATH_SINCOS2PI: in uint32 m23[n] -> out float[2n] (sin, cos)  (F3)
 *   PF_MATH_NORMAL_PAIR: in uint32 [x0[n], x1[n]] -> out float[2n] (z0, z1)  (F2)
 *   PF_MATH_PHILOX: in uint32 [c0[n], c1[n], c2[n], c3[n], k0, k1] -> out uint32[4n]  (R12)
 * fn | PF_MATH_X2 (not PHILOX; n even): the same functions evaluated by
 * the packed f32x2 code path on element pairs (2i, 2i+1), same output layout.
 * No handle; uses the current CUDA device; synchronous. */
enum { PF_MATH_SIN = 0, PF_MATH_COS = 1, PF_MATH_LOG = 2, PF_MATH_EXPQ = 3, PF_MATH_SQRT = 4,
       PF_MATH_SINCOS2PI = 5, PF_MATH_NORMAL_PAIR = 6, PF_MATH_PHILOX = 7, PF_MATH_X2 = 0x100 };
pf_status pf_debug_math(int32_t fn, const uint32_t* in, uint32_t* out, int64_t n);

/* Count the float bit patterns x in [lo_bits, hi_bits] for which the
 * kernels' branch-free sqrt differs from IEEE sqrt.rn (exhaustive, on device). */
pf_status pf_debug_check_sqrt(uint32_t lo_bits, uint32_t hi_bits, uint64_t* mismatches);

/* ---- Peer transport (multi-rank on one node) -------------
 * The exchange halo (Alg.2 l.10–14; "exchanged particles are
 * unique to neighbor pairs", §VI-E) and the global estimate (the
 * particle with the highest global weight, :16 §IV / :20 §VI-D) cross ranks
 * inside the step kernel itself, over NVLink / NVSwitch peer memory, instead of
 * NCCL send/recv + all-gather + pf_reduce_records around it:
 *  - the reduce phase writes each boundary sub-filter's best-t entries straight
 *    into the neighbour ranks' halo rows (the pf_shard layout: ring — local
 *    sub-filter 0 -> rank r-1's row n_local+1, the last -> rank r+1's row
 *    n_local; torus — the first grid row -> rank r-1's rows n_local+C.., the
 *    last -> rank r+1's rows n_local..);
 *  - the last CTA writes the shard's best record into every rank's peer block
 *    (buffer rv & 1 of a double buffer, rv = the rendezvous number: +1 per
 *    peer-mode launch — pf_step, pf_set_particles — on every rank), raises its
 *    flag there to rv (system-scope release) and waits for every rank's flag
 *    to reach rv (acquire): a device-side rendezvous per step, after which the
 *    exact max over the world records is the global estimate on every rank.
 *    A rank missing for PF_PEER_TIMEOUT_MS (environment, default 30000) ends
 *    the wait: pf_estimate then returns PF_ETIMEOUT (sticky) instead of the
 *    device hanging.
 * All-to-All: the shard's pool row (its best t) goes into every rank's peer
 * block and the global pool is reduced after the rendezvous (pf_reduce_pool,
 * fused).  Ring, 2D torus, All-to-All; world 2..8; every rank calls pf_step /
 * pf_set_particles in the same sequence.  Peers on the same device (by PCI bus
 * id) run without programmatic dependent launch.
 * pf_peer_export: this rank's blob (CUDA IPC handles of the caller's mailbox
 *   allocation + offset, and of an 80 KiB runtime-owned peer block; the rank;
 *   the device's PCI bus id).  Host blob[PF_PEER_BLOB_BYTES].  Call before the
 *   first step.
 * pf_peer_connect: blobs [world][PF_PEER_BLOB_BYTES] of all ranks in rank order
 *   (e.g. all-gathered through torch.distributed); opens the peers' blocks and
 *   the neighbours' mailboxes (cudaIpcOpenMemHandle, lazy peer access).
 * pf_peer_connect_local: the same for `world` handles of ONE process (tests on
 *   one device; their steps must run on different streams).
 * Errors: PF_ESTATE (world == 1, central filter, already stepped / connected,
 *   export missing), PF_ECUDA (IPC failure; the handle stays on the NCCL path). */
#define PF_PEER_BLOB_BYTES 160
pf_status pf_peer_export(pf_handle* h, uint8_t* blob);
pf_status pf_peer_connect(pf_handle* h, const uint8_t* blobs);
pf_status pf_peer_connect_local(pf_handle* const* handles, int32_t world);
int32_t pf_peer_connected(const pf_handle* h);

/* The step kernel's launch configuration chosen for this handle (tuning,
 * tests; DESIGN.md §6 "mappings"): out = int32[8] { warps per group, groups
 * per CTA, TMA stages, sample-loop unroll, min CTAs per SM (register cap),
 * split first load (0/1), grid size in CTAs, number of compiled mappings for
 * this (model, n_joints, m, resampler) — the range of the PF_VARIANT
 * environment variable read by pf_init }.  Host only, no synchronisation.
 * Errors: PF_EINVAL (NULL), PF_ESTATE (the centralized filter: its kernels
 * have fixed shapes). */
pf_status pf_query_mapping(const pf_handle* h, int32_t* out);

/* Release host metadata; NULL-safe.  Does not free caller buffers. */
pf_status pf_destroy(pf_handle* h);

const char* pf_strerror(pf_status s);
pf_status pf_last_error(const pf_handle* h);

/* Compiled configurations: writes up to `cap` (n_joints, m) pairs. */
int32_t pf_supported(int32_t* n_joints, int32_t* m, int32_t cap);

#ifdef __cplusplus
}
#endif
#endif
