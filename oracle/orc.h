/*
 * oracle/orc.h — the CPU ORACLE for the distributed particle filter of
 * Chitchian et al., "Adapting Particle Filter Algorithms to Many-Core
 * Architectures", IPDPS 2013 (/root/reference/PAPER.md; one line = one page,
 * see SURVEY.md §0 for the garbling key).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference leg may load liborc.so.  The
 * product (CUDA) path never includes, links or calls anything in oracle/, and
 * this tree includes nothing from the product tree (no shared headers,
 * kernels, helpers, constants or generators).
 *
 * The oracle is plain, slow, single-threaded C.  It executes Algorithm 2
 * (§IV "Distributed Particle Filter") literally: loops over
 * sub-filters and particles, a full sort per sub-filter, a snapshot copy for
 * the exchange, a sequential prefix sum for RWS and the sequential sweep for
 * Vose's alias table.  The readings of everything the paper leaves open
 * (h(x), noise, RNG, counter layout, integer weights, tie-breaks, where
 * exchanged particles go, …) are DESIGN.md §3 "Readings"; each function below
 * names the reading (R#) or the contract clause (F#) it implements.
 *
 * Two arithmetic variants are compiled from the same body (orc_impl.inc):
 *   orc_s_*  fp32 — the paper's precision ("All floating point operations in
 *            the parallel implementations are in single precision"
 *            §VI), with the fp32 arithmetic contract F1–F11 of DESIGN.md §4
 *            (specified polynomials for sin/cos/log/exp, explicit fmaf), so
 *            every floating-point value that decides an integer is defined.
 *   orc_d_*  fp64 with libm — the paper's "double precision reference"
 *            (§VI), used for the fp32-vs-fp64 accuracy pin (E12).
 *
 * Errors: functions returning int return 0 on success and a negative value on
 * invalid arguments (-1) or allocation failure (-2); nothing is printed.
 */
#ifndef ORC_H
#define ORC_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum { ORC_TOPO_NONE = 0, ORC_TOPO_RING = 1, ORC_TOPO_TORUS2D = 2, ORC_TOPO_ALL2ALL = 3 };
enum { ORC_RWS = 0, ORC_VOSE = 1 };
/* When a sub-filter resamples (§IV: "the suggested metric to
 * compute the effective sample size as well as a simpler resampling frequency
 * parameter (each sub-filter randomly decides to resample at a fixed ratio of
 * the time)"; reading R21). */
enum { ORC_POLICY_ALWAYS = 0, ORC_POLICY_ESS = 1, ORC_POLICY_FREQ = 2 };

/* Table I parameters: m, N, X, t; plus the RNG seed. */
typedef struct {
  int32_t m;            /* particles per sub-filter                        */
  int64_t n_filters;    /* N, number of sub-filters                        */
  int32_t t;            /* particles per exchange (per neighbour)          */
  int32_t topo;         /* X: ORC_TOPO_*                                   */
  int32_t torus_rows;   /* 0 = default R = 2^floor(log2(N)/2) (R4)         */
  int32_t torus_cols;   /* 0 = default N / R                               */
  int32_t resampler;    /* ORC_RWS | ORC_VOSE                              */
  uint64_t seed;        /* Philox key = (seed lo 32, seed hi 32)  (R12)    */
  int32_t policy;       /* ORC_POLICY_*                                    */
  uint64_t policy_param;/* ESS: tau in 1/65536 of m; FREQ: threshold in [0, 2^32] */
} orc_config;

/* R21: does sub-filter n (global) resample before the sample of step k?
 * q = its integer weights (F7).  ESS: Q^2 2^16 < param m S2 (Q = sum q,
 * S2 = sum q^2, i.e. ESS = Q^2/S2 < tau m; 128-bit integers); FREQ: word 0 of
 * Philox (n, k, 1, 0) < param. */
int orc_should_resample(int32_t policy, uint64_t param, const uint32_t* q, int32_t m, uint64_t seed, int64_t n,
                        int64_t k);

/* Models ("our application separates generic particle filtering from
 * model-specific routines", §I):
 *   ORC_MODEL_ARM_PLANAR       the robotic arm of PAPER.md:22–24 §VII-A (R14)
 *   ORC_MODEL_LINEAR_GAUSS_1D  one joint with its angle sensor, no camera:
 *       theta_k = theta_{k-1} + h_s u + w, w ~ N(0, sigma_theta^2),
 *       z_k = theta_k + v, v ~ N(0, sigma_theta_meas^2)  (d = 1; the Kalman
 *       special case of SURVEY §8(c), pinned against the Kalman filter) */
enum { ORC_MODEL_ARM_PLANAR = 0, ORC_MODEL_LINEAR_GAUSS_1D = 1 };

/* Table II model parameters (§VII-A) — fp32 values. */
typedef struct {
  int32_t model;           /* ORC_MODEL_*                                   */
  int32_t n_joints;        /* joints incl. base rotation; d = n_joints + 4  */
  float arm_length;        /* L; link length = L / n_joints            (R16)*/
  float h_s;               /* sampling time                            (R16)*/
  float sigma_theta;       /* process noise on joint angles            (R15)*/
  float sigma_pos;         /* process noise on object x, y             (R15)*/
  float sigma_vel;         /* process noise on object vx, vy           (R15)*/
  float sigma_cam;         /* measurement noise on (x_C, y_C)          (R15)*/
  float sigma_theta_meas;  /* measurement noise on joint sensors       (R15)*/
} orc_model;

/* ---- Philox4x32-10 (Salmon et al. SC'11; R12/R13) ---------------------- */
void orc_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);

/* ---- fp32 contract functions (F3–F7) ---------------------- */
float orc_s_sin(float x);                 /* F5 sin with Cody–Waite reduction */
float orc_s_cos(float x);                 /* F5 cos                            */
float orc_s_log(float x);                 /* F6 natural log, x normal > 0      */
void orc_s_sincos2pi(uint32_t m23, float* s, float* c);  /* F3 sin/cos(2π m/2^23) */
uint32_t orc_s_expq(float delta);         /* F7 floor(2^22 exp(delta)), delta<=0 */
void orc_s_normal_pair(uint32_t x0, uint32_t x1, float out[2]);   /* F2 */
void orc_d_normal_pair(uint32_t x0, uint32_t x1, double out[2]);  /* libm */

/* ---- model hooks (§VII-A; R14, R16) ---------------------- */
/* camera-frame object position h(x) = (x_C, y_C) (F9) */
void orc_s_camera(const orc_model* md, const float* x, float out[2]);
void orc_d_camera(const orc_model* md, const double* x, double out[2]);
/* log p(z | x) up to a constant (F10) */
float orc_s_loglik(const orc_model* md, const float* x, const float* z);
double orc_d_loglik(const orc_model* md, const double* x, const double* z);

/* Sample (a1–a2) + weight (a3) of M particles with no resampling: particle p
 * (global index p_offset + column) takes the Philox counter
 * (p, k, 0, j), words 2.. (F8).  state_* are SoA [d][M]; logw_out is [M]. */
void orc_s_sample_weight(const orc_model* md, uint64_t seed, int64_t M, int64_t p_offset,
                         const float* state_in, const float* z, const float* u, int64_t k,
                         float* state_out, float* logw_out);

/* ---- resampling (PAPER.md:18 §IV, :20–22 §VI-F; R8–R11) ----------------- */
/* RWS: a = min{ j : C_j > floor(U*Q/2^32) } over the inclusive sum C of q. */
int32_t orc_rws_draw(const uint32_t* q, int32_t m, uint32_t U);
/* Vose's alias table by the sequential sweep (R10); prob in units of Q. */
void orc_vose_build(const uint32_t* q, int32_t m, uint64_t* prob, int32_t* alias);
int32_t orc_vose_draw(const uint64_t* prob, const int32_t* alias, int32_t m, uint64_t Q,
                      uint32_t Ua, uint32_t Ub);
/* Whole [N][m] array with explicit uniforms: ancestors[n][i] in [0, m). */
int orc_resample_q(const uint32_t* q, int64_t N, int32_t m, int32_t resampler,
                   const uint32_t* ua, const uint32_t* ub, int32_t* ancestors);
/* Normalise (a7): q_i = F7(logw_i - max logw) for one sub-filter. */
void orc_s_normalise(const float* logw, int32_t m, uint32_t* q);
/* Normalise + resample [N][m] log-weights with the step-k Philox draws
 * (counter (p, k, 0, 0) words 0–1, R13). */
int orc_s_resample_logw(const orc_config* cfg, const float* logw, int64_t k, int32_t* ancestors,
                        uint32_t* q_out /* nullable */);

/* ---- exchange (PAPER.md:16 Alg.2 l.10–14, Fig.1; :20 §VI-E; R2–R5) ------ */
/* Neighbour list of sub-filter n, in exchange order; returns the degree. */
int32_t orc_neighbors(const orc_config* cfg, int64_t n, int64_t nb[4]);
void orc_torus_shape(const orc_config* cfg, int64_t* rows, int64_t* cols);
/* Global source particle index of every slot after the exchange. */
int orc_s_exchange(const orc_config* cfg, const float* logw, int64_t* src);

/* ---- the filter (Algorithm 2, one time step per call) ------------------- */
typedef struct orc_s_filter orc_s_filter;
typedef struct orc_d_filter orc_d_filter;

/* Draw X_0 ~ N(mu0, diag(sigma0^2)) with Philox counter (p, 0, 2, j) (F11). */
orc_s_filter* orc_s_create(const orc_config* cfg, const orc_model* md, const float* mu0,
                           const float* sigma0);
/* One step k = step+1: [k>1: exchange + normalise + resample of step k-1]
 * then sample + weight + estimate of step k.  z: n_joints+2, u: n_joints. */
int orc_s_step(orc_s_filter* f, const float* z, const float* u);
int orc_s_estimate(const orc_s_filter* f, float* x_hat, float* logw, int64_t* idx);
/* Weighted-average estimate of the current set (R22; §VI-D). */
int orc_s_estimate_mean(const orc_s_filter* f, float* x_mean);
void orc_s_weighted_mean(const float* state, const float* logw, int64_t M, int32_t d, float* out);
void orc_d_weighted_mean(const double* state, const double* logw, int64_t M, int32_t d, double* out);
/* The weighted (pre-exchange) set of the current step; step 0 = prior. */
int orc_s_get(const orc_s_filter* f, float* state, float* logw, int64_t* step);
int orc_s_set(orc_s_filter* f, const float* state, const float* logw, int64_t step);
/* Exchange sources and ancestors used by the last step (for diagnosis). */
int orc_s_trace(const orc_s_filter* f, int64_t* src, int32_t* ancestors);
void orc_s_destroy(orc_s_filter* f);

/* Centralized filter (n_filters == 1): step k >= 2 for the listed slots only
 * (normalise over all M, resample, sample, weight).  out_state [d][n]. */
int orc_s_central_slots(const orc_config* cfg, const orc_model* md, const float* state, const float* logw,
                        int64_t k, const float* z, const float* u, const int64_t* slots, int64_t n,
                        float* out_state, float* out_logw);

/* One step k >= 2 for the listed sub-filters only, from the full weighted
 * set of step k-1 (state [d][M], logw [M]) — exchange, normalise, resample,
 * sample, weight, one sub-filter at a time.  out_state [d][n_sub*m],
 * out_logw [n_sub*m].  For sampled checks at full size. */
int orc_s_step_subset(const orc_config* cfg, const orc_model* md, const float* state, const float* logw,
                      int64_t k, const float* z, const float* u, const int64_t* subs, int64_t n_sub,
                      float* out_state, float* out_logw);

orc_d_filter* orc_d_create(const orc_config* cfg, const orc_model* md, const double* mu0,
                           const double* sigma0);
int orc_d_step(orc_d_filter* f, const double* z, const double* u);
int orc_d_estimate(const orc_d_filter* f, double* x_hat, double* logw, int64_t* idx);
int orc_d_estimate_mean(const orc_d_filter* f, double* x_mean);
int orc_d_get(const orc_d_filter* f, double* state, double* logw, int64_t* step);
void orc_d_destroy(orc_d_filter* f);

#ifdef __cplusplus
}
#endif
#endif
