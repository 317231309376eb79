/*
 * capgpu.h -- C ABI of the B200-native CapGPU hot path.
 *
 * CapGPU (Ma, Subramaniyan, Wang, ICPP '25): per-control-period MIMO power
 * capping of a GPU server (1 host CPU knob + N_g GPU knobs), batched over many
 * servers.  Citations "P:NNN" are lines of the paper text; "Qn" are
 * the readings of DESIGN.md §2.  Implementation: hand-written CUDA for sm_100a
 * (paper_conf_icpp_masw25_b200/csrc/); no CPU fallback exists.
 *
 * Conventions (all entry points):
 *  - Return CAPGPU_OK (0) or a negative CAPGPU_E_* code.  All argument
 *    validation happens BEFORE any launch; on failure nothing is written.
 *    capgpu_last_error(ctx) gives a one-line reason.  No C++ exception crosses
 *    the ABI.
 *  - Per-server soft conditions are status bits (CAPGPU_ST_*), never errors
 *    (an unreachable cap is not an error: P:230).
 *  - Array arguments named *_d are DEVICE pointers (checked with
 *    cudaPointerGetAttributes), fp64 unless stated, laid out SoA "knob-major":
 *    element (j, i) of a [N][n] array lives at [j * n + i], n = the context's
 *    local server count.  The caller owns every argument buffer.
 *  - Calls are stream-ordered and asynchronous on `stream` (a cudaStream_t
 *    passed as void*, NULL = legacy default stream); the caller synchronises.
 *  - The context owns its state workspace (allocated at create, freed at
 *    destroy).  One context per stream/thread; contexts are independent.
 *  - Knob order: knob 0 = CPU, knobs 1..n_gpus = GPUs.  Frequencies in
 *    MHz, power in W (Q5).
 */
#ifndef CAPGPU_H
#define CAPGPU_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define CAPGPU_MAX_KNOBS 16   /* N = 1 + n_gpus <= 16 ("up to eight GPUs") */
#define CAPGPU_MAX_M 4        /* control horizon M <= 4 on the CUDA path */
#define CAPGPU_MAX_P 64
#define CAPGPU_MAX_LEVELS 32  /* discrete frequency levels per knob */

enum {
  CAPGPU_OK = 0,
  CAPGPU_E_INVALID = -1,     /* bad argument (size, bound, pointer kind) */
  CAPGPU_E_NOMEM = -2,       /* device allocation failed */
  CAPGPU_E_CUDA = -3,        /* CUDA runtime/launch error */
  CAPGPU_E_NCCL = -4,        /* NCCL error (hierarchical budget) */
  CAPGPU_E_ORDER = -5,       /* call order: e.g. control_step before a prior A0 exists */
  CAPGPU_E_UNSUPPORTED = -6  /* valid request this build does not implement */
};

/* per-server status bits (Q26) */
enum {
  CAPGPU_ST_CAP_INFEASIBLE = 1, /* no frequency vector in the box reaches P_s per the model */
  CAPGPU_ST_SLO_INFEASIBLE = 2, /* an SLO lower bound exceeds f_max (Eq. 10b-c) */
  CAPGPU_ST_SOLVER_CAP = 4,     /* QP iteration cap reached (never expected) */
  CAPGPU_ST_NONFINITE = 8       /* non-finite measurement: outputs pinned to the lower bounds */
};

typedef struct capgpu_ctx capgpu_ctx;

/* Prediction horizon P and control horizon M, 1 <= M <= P (P = 8, M = 2). */
typedef struct {
  int32_t P, M;
} capgpu_horizons;

/* One knob (P:126-127 f_min/f_max, P:242 discrete levels, Eq. 10b-c SLO bound). */
typedef struct {
  double f_min, f_max;  /* MHz, f_min < f_max */
  int32_t n_levels;     /* >= 2 uniform levels: f_min + l (f_max - f_min)/(n_levels - 1) (Q15) */
  int32_t sweep_base;   /* level index held while other knobs are swept */
  double f_lo;          /* lower bound l_j in [f_min, f_max] (SLO, Q14); 0 -> f_min */
  double r0;            /* base control penalty r0_j of R_j = r0_j/theta_j; 0 -> params.r0 */
} capgpu_knob_bounds;

/* Controller and plant constants; NULL -> defaults of DESIGN.md §2/§3. */
typedef struct {
  double q;           /* tracking weight Q(i) = q > 0 (Q6) */
  double r0;          /* default control penalty > 0 (Q6) */
  double theta_min;   /* 0 < theta_min <= 1 (Q8) */
  double lambda;      /* forgetting factor 0 < lambda <= 1 (Q1) */
  double rho;         /* ridge toward A0, > 0 (Q1) */
  double a_lo, a_hi;  /* clamp of Ahat to [a_lo, a_hi] A0, 0 <= a_lo <= a_hi (Q4) */
  double a_floor;     /* positivity guard of identified A0 (Q21), > 0 */
  double gamma;       /* latency exponent, > 0 */
  double noise_std;   /* synthetic meter noise sigma, W (>= 0) */
  int32_t substeps;   /* delta-sigma sub-steps per period S in {1,2,4,8} (Q22) */
  int32_t caps_per_server; /* simulated instances per server (cfg 5: 32), >= 1 */
  uint64_t seed;      /* synthetic-input seed */
  double wmove;       /* NEXT-3 move suppression (Q36): Eq. 9 + sum_{t<M} wmove |d(k+t|k)|^2,
                         >= 0 (W^2/MHz^2); 0 = the literal Eq. 9.  > 0 couples the M blocks: solved by a
                         per-instance active set on the block-tridiagonal Hessian (Woodbury: N tridiagonal
                         M x M solves + one M x M system per iteration), CUDA path for M * N <= 36,
                         capgpu_simulate only
                         (not control_step / hierarchical / SLO schedule: CAPGPU_E_UNSUPPORTED) */
  double ref_alpha;   /* NEXT-3 reference trajectory ("a reference trajectory"; Q37):
                         prediction step i tracks r(k+i|k) = P_s - ref_alpha^i (P_s - p(k)) instead of
                         P_s; ref_alpha = exp(-T/T_ref) in [0, 1), 0 = the literal Eq. 9 (r = P_s).
                         Every call and config (also control_step / hierarchical / move / SLO). */
} capgpu_params;

/* Contiguous server range of this process (one process per GPU, §8(e)). */
typedef struct {
  int32_t rank, world;       /* 0 <= rank < world */
  int64_t srv_begin;         /* first global server id of this shard */
  int64_t n_servers_global;  /* servers over all shards (cfg 4 budget) */
  int32_t use_nccl;          /* 1: create an NCCL communicator from nccl_id */
  uint8_t nccl_id[128];      /* ncclUniqueId from capgpu_nccl_unique_id on rank 0 */
} capgpu_shard;

/* Synthetic workload of capgpu_simulate. */
typedef struct {
  int32_t demand_kind;       /* 0: constant demand_frac * thr_max; 1: bursty */
  double demand_frac;
  double cap_frac0, cap_frac_rand, cap_frac_step; /* base cap = Pmin + frac (Pmax - Pmin) */
  int64_t cap_period, cap_lo, cap_hi;             /* step schedule: x cap_mult while k mod period in [lo, hi) */
  double cap_mult;
  int32_t hierarchical;      /* 1: caps from the rack/cluster budget (Q16, cfg 4) */
  int32_t rack;              /* servers per rack (16) */
  int32_t block;             /* servers per reduction block (1024) */
  double cluster_frac;       /* B_c = Pmin_tot + cluster_frac (Pmax_tot - Pmin_tot) */
  double rack_frac;          /* B_rack = rack_frac * sum_rack Pmax */
  const double *cap_base_d;  /* nullable device [n_inst]: operator-set base caps P_s (W) for this
                                call, replacing the generated ones (the step schedule still applies) */
  double gain_dlo, gain_step; /* gain-mismatch sweep (NEXT-4, §4.4): the plant of cap
                                 index c has true gains g_c a with g_c = 1 + gain_dlo + c gain_step
                                 (0, 0 -> the nominal plant) */
  /* Time-varying latency SLOs (NEXT-1, §6.4; Eq. 10b-c; DESIGN.md
   * Q29-Q31).  slo_a / slo_b [knob] = SLO_j / e_min,j (0 = no SLO for that knob).
   * Phase B is in force at instant k while slo_period > 0 and k mod slo_period lies
   * in [slo_lo, slo_hi); phase A otherwise (slo_period = 0: phase A throughout).
   * Knob j's lower bound at instant k is max(f_lo_j, level(q_j)), q_j = the lowest
   * grid level whose latency e_min (f_max/level)^gamma meets the SLO; an SLO no
   * level meets (ratio < 1) pins the bound to f_max and sets CAPGPU_ST_SLO_INFEASIBLE.
   * A delta-sigma sub-step whose level index is below q_j is a deadline miss
   * (capgpu_trace.n_miss_d).  Not supported with `hierarchical`. */
  int64_t slo_period, slo_lo, slo_hi;
  double slo_a[CAPGPU_MAX_KNOBS], slo_b[CAPGPU_MAX_KNOBS];
  /* Controller (NEXT-2, §6.1; Q32-Q35): CAPGPU_CTRL_*.  The
   * baselines replace S1-S3 on the same plant: Fixed-step moves the movable knob
   * with the highest (p < P_s) or lowest (p > P_s) theta by fs_levels grid levels
   * (ties round-robin; Safe Fixed-step uses P_s - safe_margin); GPU-only / CPU-only
   * run g(k) = clamp(g(k-1) + K (P_s - p(k))) on one common GPU (CPU) frequency
   * with the other knobs at f_max and the pole-placed gain K = (1 - p_pole) / sum_J A0_j;
   * CPU+GPU (Q39) runs one such loop per device class on its own meter (CPU
   * meter 0.3 C + a_0 fbar_0 + n/2, GPU meter the rest) toward gpu_share * P_s (GPUs)
   * and (1 - gpu_share) * P_s (CPU).
   * Traces: u row 0 = the command, theta, p, cap, levels; status 0; act_count 0.
   * The controller is fixed for a simulation (first call after create/sim_reset).
   * Not supported with `hierarchical`. */
  int32_t controller;
  int32_t fs_levels;   /* >= 1 */
  double safe_margin;  /* W, finite */
  double p_pole;       /* in [0, 1) */
  double gpu_share;    /* CPU+GPU: GPU share of the budget, in (0, 1) */
} capgpu_workload;

enum { CAPGPU_CTRL_CAPGPU = 0, CAPGPU_CTRL_FIXED_STEP = 1, CAPGPU_CTRL_SAFE_FIXED_STEP = 2,
       CAPGPU_CTRL_GPU_ONLY = 3, CAPGPU_CTRL_CPU_ONLY = 4, CAPGPU_CTRL_CPU_GPU = 5 };

/* Optional outputs of capgpu_simulate; every pointer may be NULL.
 * Summaries are over the last floor(0.8 K) of the K periods of the call (Q25).
 * Traces record n_trace sampled local instances per period, layout
 * [period][field...][slot] (slot fastest). */
typedef struct {
  double *sum_p_d, *sumsq_p_d, *max_p_d, *sum_theta_d; /* [n_inst] */
  int32_t *n_viol_d, *n_window_d;                      /* [n_inst] */
  int32_t *act_count_d;                                /* [M][n_inst] */
  double *final_p_d;                                   /* [n_inst] p(k0+K) */
  int32_t *n_miss_d;                                   /* [n_inst] SLO deadline misses (sub-steps x knobs) */
  int32_t n_trace;
  const int64_t *trace_inst_d;                         /* [n_trace] local instance ids */
  double *p_d, *cap_d;                                 /* [K][n_trace] p(k), P_s(k) */
  double *u_d;                                         /* [K][M][N][n_trace] */
  double *ahat_d, *theta_d;                            /* [K][N][n_trace] */
  uint32_t *active_d;                                  /* [K][M][n_trace] 2 bits/knob: 0 free, 1 lower, 2 upper */
  int8_t *rank_d;                                      /* [K][N][n_trace] */
  uint8_t *levels_d;                                   /* [K][S][N][n_trace] */
  uint32_t *status_d;                                  /* [K][n_trace] */
  double *agg_W_d, *agg_P_d;                           /* [K] cluster sums (hierarchical) */
} capgpu_trace;

/* ---------------------------------------------------------------------- */

const char *capgpu_version(void);
const char *capgpu_status_string(int code);
const char *capgpu_last_error(const capgpu_ctx *ctx);

/* Defaults of DESIGN.md §2 (q=1, r0=1e-4, theta_min=0.05, lambda=0.95, rho=100,
 * a in [0.25,4] A0, a_floor=1e-3, gamma=0.91, noise 11 W, S=4, 1 cap/server, seed 1). */
void capgpu_default_params(capgpu_params *out);

/* Create a context for n_servers LOCAL servers (this shard) with 1 CPU + n_gpus
 * GPU knobs, horizons h, bounds[1 + n_gpus].  shard = NULL -> rank 0 of 1,
 * srv_begin 0.  Validation (before anything is allocated): n_servers >= 1,
 * 1 <= n_gpus <= 15, 1 <= M <= min(P, CAPGPU_MAX_M), P <= CAPGPU_MAX_P,
 * f_min < f_max, 2 <= n_levels <= 32, 0 <= sweep_base < n_levels,
 * f_min <= f_lo <= f_max, params in range.  Allocates the SoA state (device
 * memory) on the current device.  *out = NULL on failure. */
int capgpu_create(capgpu_ctx **out, int64_t n_servers, int32_t n_gpus, capgpu_horizons h,
                  const capgpu_knob_bounds *bounds, const capgpu_params *params,
                  const capgpu_shard *shard);
int capgpu_destroy(capgpu_ctx *ctx);

/* Bytes of device state the context holds (for capacity planning). */
int64_t capgpu_state_bytes(const capgpu_ctx *ctx);

/* S0 identification: per server, least squares of the sweep rows
 * p ~ A.F + C.  F_d [rows][N][n] and p_d [rows][n]; F_d = p_d = NULL -> the
 * paper's sweep on the synthetic plant (each knob over its levels, others at
 * sweep_base; rows = sum_j n_levels_j).  Outputs (nullable) A_out_d [N][n],
 * C_out_d [n], r2_out_d [n].  The identified gains, floored at a_floor (Q21),
 * become the context's prior A0 for control_step / simulate. */
int capgpu_identify(capgpu_ctx *ctx, const double *F_d, const double *p_d, int32_t rows,
                    double *A_out_d, double *C_out_d, double *r2_out_d, void *stream);

/* Set the prior A0 [N][n] directly (all > 0). */
int capgpu_set_prior(capgpu_ctx *ctx, const double *A0_d, void *stream);

/* Reset the online LS state (w = 0, mu = 0, Sigma = 0): next Ahat = A0. */
int capgpu_model_reset(capgpu_ctx *ctx, void *stream);

/* S2 weight assignment (Q8-Q10) on thr_d, thr_max_d [N][n]:
 * theta = clamp(thr/thr_max, theta_min, 1) (IEEE division), R = r0/theta,
 * rank = stable descending order of theta (0 = highest, ties -> lower index).
 * Outputs nullable: theta_out_d, R_out_d [N][n], rank_out_d int8 [N][n]. */
int capgpu_assign_weights(capgpu_ctx *ctx, const double *thr_d, const double *thr_max_d,
                          double *theta_out_d, double *R_out_d, int8_t *rank_out_d, void *stream);

/* One control period on user measurements:
 *   S1 push z = (f_applied, p_meas) into the model state, solve Ahat;
 *   S2 weights from thr / thr_max;
 *   S3 MPC (Eq. 9-10a) with P_s = cap:  u_out_d [M][N][n] (row t = 0 is the
 *   frequency to apply now), active_out_d [M][n] (2 bits per knob).
 * Nullable extras: rank_out_d int8 [N][n], ahat_out_d [N][n], status_out_d [n].
 * Requires a prior (capgpu_identify or capgpu_set_prior), else CAPGPU_E_ORDER. */
int capgpu_control_step(capgpu_ctx *ctx, const double *p_meas_d, const double *f_applied_d,
                        const double *thr_d, const double *thr_max_d, const double *cap_d,
                        double *u_out_d, uint32_t *active_out_d, int8_t *rank_out_d,
                        double *ahat_out_d, uint32_t *status_out_d, void *stream);

/* Closed-loop simulation of `periods` control periods for every local instance
 * (n_servers * caps_per_server) on the synthetic plant of DESIGN.md §3, all
 * four steps S1-S4 per period (+ S5 when wl->hierarchical).  The first call
 * (or the first after capgpu_sim_reset) generates the plant, runs the
 * identification sweep (S0) and the initial period (Q23); later calls continue
 * from the stored state.  Outputs in tr (nullable).  cfgs 1-3, 5 run as one
 * fused multi-period kernel; the hierarchical mode runs one kernel per period
 * around the budget all-reduce. */
int capgpu_simulate(capgpu_ctx *ctx, int64_t periods, const capgpu_workload *wl,
                    const capgpu_trace *tr, void *stream);
int capgpu_sim_reset(capgpu_ctx *ctx);

/* Hierarchical budget (wl->hierarchical) for n_ctx shards that live on ONE
 * device in one process (ranks 0..n_ctx-1 of world n_ctx, created without
 * NCCL): the contexts step period by period together and the per-period
 * all-reduce is an in-process (loopback) sum of their zero-padded block
 * vectors.  Results are bitwise identical to one context holding all servers
 * and to n_ctx processes over NCCL.  trs: NULL or [n_ctx]. */
int capgpu_simulate_group(capgpu_ctx **ctxs, int32_t n_ctx, int64_t periods, const capgpu_workload *wl,
                          const capgpu_trace *const *trs, void *stream);

/* Host copy of the fixed-order pairwise tree the device uses for cluster sums
 * (zero-pad to 2^m >= n; for h = 2^(m-1)..1: v[i] += v[i+h]). */
int capgpu_tree_sum_host(const double *v, int64_t n, double *out);

/* Copy the device plant state of the simulation to host-visible buffers for
 * checkpointing / parity checks: fbar, acc, thr [N][n_inst]; p [n_inst]
 * (device pointers, nullable). */
int capgpu_sim_state(capgpu_ctx *ctx, double *fbar_d, double *acc_d, double *thr_d, double *p_d,
                     void *stream);

/* NEXT-3 explicit (multi-parametric) MPC ("an offline part and an
 * online part ... solved incrementally as a piecewise linear function").
 * Offline: from the context's current model state (the S1 solve: A-hat, as the
 * next control_step would compute it before its push) and the weights of
 * thr_d / thr_max_d [N][n] (S2), tabulate every server's applied control law
 * u_0(beta) of Eq. 9's first block (weight c_0): the critical regions are
 * nested in the tracking offset beta = p - P_s - A.f (knobs reach f_max in the
 * stable ascending order of b_j = (f_max - f_min) / (c_0 tau_j)), each with an
 * affine law.  The table (6N + 3 doubles per server) is owned by the context.
 * Online: u_out [N][n] (device) = the law at beta of p_meas [n], f_applied
 * [N][n], cap [n]; active_out [n] = block 0's 2-bit codes; status_out
 * (nullable) = CAP_INFEASIBLE as control_step.  No model update, no weights
 * (they are frozen in the table until the next build).  Convex literal Eq. 9
 * only (no f_lo / ref_alpha / wmove: CAPGPU_E_UNSUPPORTED); CAPGPU_E_ORDER
 * before identify/set_prior (build) or before a build (step). */
int capgpu_explicit_build(capgpu_ctx *ctx, const double *thr_d, const double *thr_max_d, void *stream);
int capgpu_explicit_step(capgpu_ctx *ctx, const double *p_meas_d, const double *f_applied_d, const double *cap_d,
                         double *u_out_d, uint32_t *active_out_d, uint32_t *status_out_d, void *stream);

/* Overwrite the plant state of the simulation (inverse of capgpu_sim_state;
 * device pointers, each nullable = keep).  Validated before anything is
 * written (synchronous on `stream`): every value finite and |acc_j| <=
 * step_j / 2 -- the first-order modulator's invariant (Q15) that the
 * plant's exactness rests on; else CAPGPU_E_INVALID and nothing changes.
 * CAPGPU_E_ORDER before the first capgpu_simulate. */
int capgpu_set_state(capgpu_ctx *ctx, const double *fbar_d, const double *acc_d, const double *thr_d,
                     const double *p_d, void *stream);

/* Checkpoint / resume of a whole context: the model state (S1),
 * plant state (S4), warm starts (S3), server constants, the period counter and
 * -- for the hierarchical budget -- the per-server weights and cluster
 * aggregates, as one device blob of capgpu_checkpoint_bytes(ctx) bytes
 * (caller-owned, e.g. a torch uint8 tensor; copy it to the host to persist).
 * Load into a context created with the SAME arguments (checked: else
 * CAPGPU_E_INVALID); a hierarchical checkpoint needs the budget allocated
 * first (one simulate call, else CAPGPU_E_ORDER).  A resumed run continues
 * bitwise identically.  save/load synchronise `stream`. */
int64_t capgpu_checkpoint_bytes(const capgpu_ctx *ctx);
int capgpu_checkpoint_save(capgpu_ctx *ctx, void *dst_d, void *stream);
int capgpu_checkpoint_load(capgpu_ctx *ctx, const void *src_d, void *stream);

/* Current base caps P_s of every local instance (device [n_inst], W); valid
 * after the first capgpu_simulate. */
int capgpu_sim_caps(capgpu_ctx *ctx, double *cap_base_d, void *stream);

/* Multi-GPU helper: ncclUniqueId (128 bytes) to broadcast from rank 0. */
int capgpu_nccl_unique_id(uint8_t out[128]);

/* Shard bookkeeping (host only, no device work): contiguous ranges in multiples
 * of `granule` servers; remainder to the last ranks.  Returns the count. */
int64_t capgpu_shard_range(int64_t n_servers_global, int32_t world, int32_t rank, int64_t granule,
                           int64_t *begin_out);

/* Test hook: device copy of the seeded generator for servers
 * [srv_begin, srv_begin + n): a_true, thr_max [N][n], c_true [n], demand at
 * period k [N][n], noise at period k [n].  Used to check host/device bit
 * identity of gen/capgpu_gen.h. */
int capgpu_debug_gen(capgpu_ctx *ctx, int64_t k, int32_t demand_kind, double demand_frac,
                     double *a_true_d, double *thr_max_d, double *c_true_d, double *dem_d,
                     double *noise_d, void *stream);

/* Profiling hook: per-instance cycle counters [8][n_inst] (int64, device,
 * accumulated, caller zeroes) of the fused kernel's phases; only libraries
 * built with -DCAPGPU_PHASE_TIMING write them.  NULL disables. */
int capgpu_debug_phase_counters(capgpu_ctx *ctx, long long *counters_d);

/* Microbenchmark: FP64 DFMA throughput of this device (TFLOP/s), for the
 * roofline denominator. */
int capgpu_fp64_peak(double *tflops_out, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* CAPGPU_H */
