/*
 * capgpu_oracle.h -- plain, slow, single-threaded CPU oracle of the CapGPU hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load or call this library.  The
 * product path (paper_conf_icpp_masw25_b200/) never links, imports or executes it.
 * It shares no code with the CUDA path except the seeded input generator
 * gen/capgpu_gen.h (no method arithmetic lives there).
 *
 * Every function follows PAPER.md (cited "P:NNN" = /root/reference/PAPER.md line)
 * or, where the paper is silent, the reading listed in DESIGN.md §2 (Q1..Q20).
 * Floating point is IEEE fp64 compiled with -O2 -fno-fast-math -ffp-contract=off.
 *
 * Pins (tests/test_oracle_*.py): see DESIGN.md §4 for which pin covers which
 * function.  Functions without an independent pin say "parity unpinned".
 */
#ifndef CAPGPU_ORACLE_H
#define CAPGPU_ORACLE_H

#include <stdint.h>

#define ORA_MAXN 16
#define ORA_MAXM 8
#define ORA_MAXL 32
#define ORA_MAXS 8

/* per-server status bits (same meaning as include/capgpu.h) */
#define ORA_ST_CAP_INFEASIBLE 1u
#define ORA_ST_SLO_INFEASIBLE 2u
#define ORA_ST_SOLVER_CAP 4u
#define ORA_ST_NONFINITE 8u

typedef struct {
  int32_t n;         /* knobs N = 1 + n_gpus; knob 0 = CPU */
  int32_t P, M;      /* prediction / control horizon */
  int32_t substeps;  /* S: delta-sigma sub-steps per control period */
  int32_t n_levels[ORA_MAXN];
  int32_t sweep_base[ORA_MAXN]; /* base level index held during the sweep */
  double f_min[ORA_MAXN], f_max[ORA_MAXN], f_lo[ORA_MAXN], r0[ORA_MAXN];
  double q;          /* Q(i) = q (Q6) */
  double theta_min;  /* Q8 */
  double lambda;     /* forgetting factor of the online LS (Q1) */
  double rho;        /* ridge toward A0 (Q1) */
  double a_lo, a_hi; /* clamp of Ahat to [a_lo, a_hi] * A0 (Q4) */
  double a_floor;    /* positivity guard on identified A0 (Q21) */
  double gamma;      /* latency exponent */
  double noise_std;  /* meter noise sigma (W) */
  uint64_t seed;
  double wmove;      /* NEXT-3 move suppression weight W (W^2/MHz^2, Q36); 0 = the literal Eq. 9 */
  double ref_alpha;  /* NEXT-3 reference trajectory alpha = exp(-T/T_ref) in [0, 1) (Q37); 0 = off */
} ora_cfg;

typedef struct {
  int32_t periods;      /* control periods to run */
  int32_t n_caps;       /* instances per server (cfg 5: 32) */
  int32_t demand_kind;  /* 0 = constant frac, 1 = bursty */
  double demand_frac;   /* constant demand fraction (cfg 1: 0.7) */
  double cap_frac0, cap_frac_rand, cap_frac_step;
  int64_t cap_period, cap_lo, cap_hi; /* step schedule */
  double cap_mult;
  double gain_dlo, gain_step; /* gain mismatch (NEXT-4): true gains g_c a, g_c = 1 + dlo + c step */
  /* SLO schedule (NEXT-1, §6.4; Eq. 10b-c; Q29-Q31): per knob the latency
   * SLO as a ratio SLO_j / e_min,j (0 = no SLO).  Phase B is in force at instant k
   * while slo_period > 0 and (k mod slo_period) lies in [slo_lo, slo_hi); phase A
   * otherwise. */
  int64_t slo_period, slo_lo, slo_hi;
  double slo_a[ORA_MAXN], slo_b[ORA_MAXN];
  /* Baseline controllers (NEXT-2, §6.1; Q32-Q35) replacing S1-S3:
   * 0 = CapGPU (MPC), 1 = Fixed-step, 2 = Safe Fixed-step, 3 = GPU-only, 4 = CPU-only,
   * 5 = CPU+GPU (two loops on separately metered CPU and GPU power; Q39). */
  int32_t controller;
  int32_t fs_levels;   /* Fixed-step size in grid levels (stepsize 1 or 5) */
  double safe_margin;  /* Safe Fixed-step: set point lowered by this many W */
  double p_pole;       /* GPU-/CPU-only: closed-loop pole z of the pole-placed P gain */
  double gpu_share;    /* CPU+GPU: GPU share of the server budget (50 % or 60 %) */
} ora_workload;

/* CPU+GPU (Q39): the CPU meter reads ORA_CPU_IDLE_SHARE * C + a_0 fbar_0 + n / 2,
 * the GPU meter the rest of the server power. */
#define ORA_CPU_IDLE_SHARE 0.3

/* per-instance summary over the last 80 % of periods */
typedef struct {
  double sum_p, sumsq_p, max_p, sum_theta;
  int32_t n_window, n_viol;
  int32_t act_count[ORA_MAXM]; /* periods where block t had >= 1 active bound */
  int32_t n_miss;              /* SLO deadline misses: sub-steps x knobs below the SLO level (Q31) */
} ora_summary;

#ifdef __cplusplus
extern "C" {
#endif

/* ---- frequency grid (Q15): level(l) = f_min + l*step, mid(l) = f_min + (l+0.5)*step */
void ora_levels(const ora_cfg *c, int j, double *level, double *mid, double *g);

/* ---- SLO bound (NEXT-1; Eq. 10b-c, Q14, Q30): the lowest grid level
 * of knob j whose latency e_min (f_max / level)^gamma meets SLO = ratio * e_min.
 * Returns its index q (n_levels if even f_max misses: SLO infeasible) and the
 * continuous bound f_req = f_max ratio^(-1/gamma) in *f_req (nullable). */
int ora_slo_level(const ora_cfg *c, int j, double ratio, double *f_req);
/* Lower bounds l_j and SLO level indices q_j at instant k of workload w
 * (static f_lo combined with the SLO level, Q29); returns status bits
 * (ORA_ST_SLO_INFEASIBLE when an SLO in force is unreachable). */
uint32_t ora_slo_bounds(const ora_cfg *c, const ora_workload *w, int64_t k, double *lo, int32_t *q);

/* ---- S0 identification */
int ora_identify_ls(int n, int rows, const double *F, const double *p, double *A, double *C, double *r2);
int ora_sweep_rows(const ora_cfg *c, uint64_t server, int noisy, double *F, double *p);
int ora_sweep_nrows(const ora_cfg *c);
int ora_identify_server(const ora_cfg *c, uint64_t server, double *A0, double *C0, double *r2);

/* ---- S1 model update (Eq. 5, LS P:173; online form Q1-Q4) */
typedef struct {
  double w, mu_f[ORA_MAXN], mu_p;
  double S_ff[ORA_MAXN][ORA_MAXN], S_fp[ORA_MAXN];
} ora_model;
void ora_model_reset(ora_model *m);
void ora_model_push(const ora_cfg *c, ora_model *m, const double *f, double p);
void ora_model_solve(const ora_cfg *c, const ora_model *m, const double *A0, double *Ahat);
void ora_model_definition(const ora_cfg *c, int count, const double *F_hist, const double *p_hist,
                          const double *A0, double *Ahat);

/* ---- S2 weights (Q8-Q10) */
void ora_weights(const ora_cfg *c, const double *thr, const double *thr_max, double *theta,
                 double *R, int8_t *rank);

/* ---- S3 MPC (Eq. 9-10a; Q11-Q13, Q17, Q19) */
int ora_block_weights(const ora_cfg *c, double *ct);
int ora_mpc_stacked(const ora_cfg *c, const double *Ahat, const double *R, double beta,
                    const double *lo, const double *hi, const double *m, double *u,
                    uint32_t *active, uint32_t *tie, int *iters);
int ora_mpc_bruteforce(const ora_cfg *c, const double *Ahat, const double *R, double beta,
                       const double *lo, const double *hi, const double *m, double *u);
/* NEXT-3 (Q36): Eq. 9 + sum_{t<M} wmove |d(k+t|k)|^2 with u_{-1} = fbar = f(k);
 * dense generic active set / brute force / literal cost. */
int ora_mpc_move(const ora_cfg *c, const double *Ahat, const double *R, double beta, const double *fbar,
                 const double *lo, const double *hi, const double *m, double *u, uint32_t *active, uint32_t *tie,
                 int *iters);
int ora_mpc_move_bruteforce(const ora_cfg *c, const double *Ahat, const double *R, double beta, const double *fbar,
                            const double *lo, const double *hi, const double *m, double *u);
double ora_mpc_move_cost(const ora_cfg *c, const double *Ahat, const double *R, double beta, const double *fbar,
                         const double *m, const double *u);
double ora_mpc_cost(const ora_cfg *c, const double *Ahat, const double *R, double beta,
                    const double *m, const double *u);
void ora_mpc_classify(const ora_cfg *c, const double *Ahat, const double *R, double beta,
                      const double *lo, const double *hi, const double *m, const double *u,
                      uint32_t *active, uint32_t *tie);
/* NEXT-3 reference trajectory (Q37): row i of the tracking term has the
 * offset beta + alpha^i dref, dref = P_s - p(k), alpha = cfg ref_alpha. */
double ora_ref_pow(const ora_cfg *c, int i);
double ora_mpc_cost_ref(const ora_cfg *c, const double *Ahat, const double *R, double beta, double dref,
                        const double *m, const double *u);
double ora_mpc_move_cost_ref(const ora_cfg *c, const double *Ahat, const double *R, double beta, double dref,
                             const double *fbar, const double *m, const double *u);
void ora_mpc_classify_ref(const ora_cfg *c, const double *Ahat, const double *R, double beta, double dref,
                          const double *lo, const double *hi, const double *m, const double *u,
                          uint32_t *active, uint32_t *tie);
int ora_mpc_stacked_ref(const ora_cfg *c, const double *Ahat, const double *R, double beta, double dref,
                        const double *lo, const double *hi, const double *m, double *u,
                        uint32_t *active, uint32_t *tie, int *iters);
int ora_mpc_move_ref(const ora_cfg *c, const double *Ahat, const double *R, double beta, double dref,
                     const double *fbar, const double *lo, const double *hi, const double *m, double *u,
                     uint32_t *active, uint32_t *tie, int *iters);
int ora_mpc_bruteforce_ref(const ora_cfg *c, const double *Ahat, const double *R, double beta, double dref,
                           const double *fbar, const double *lo, const double *hi, const double *m, double *u);

/* ---- S4 plant (P:242 delta-sigma, P:238/P:264 meter, Eq. 5, Eq. 8/10b) */
void ora_plant_step(const ora_cfg *c, const double *a_true, double c_true, const double *thr_max,
                    const double *dem, double noise, const double *u0, double *acc, double *fbar,
                    double *p, double *thr, uint8_t *levels);

/* ---- generator front-ends (exposed for the device-generator bit test) */
uint64_t ora_gen_mix64(uint64_t z);
void ora_gen_server(const ora_cfg *c, uint64_t server, double *a_true, double *c_true,
                    double *thr_max, double *base, double *amp);
double ora_gen_noise(const ora_cfg *c, uint64_t server, int64_t k);
void ora_gen_demand(const ora_cfg *c, const ora_workload *w, uint64_t server, int64_t k, double *dem);
double ora_gen_cap_base(const ora_cfg *c, const ora_workload *w, uint64_t server, int cap_idx);

/* ---- closed loop (P:90-96 loop, P:196 receding horizon).  Instances are
 * global ids inst = server * n_caps + cap.  Trace arrays are [periods][n_inst][...]
 * (any may be NULL).  Returns 0 or a negative error. */
int ora_simulate(const ora_cfg *c, const ora_workload *w, int n_inst, const int64_t *inst,
                 const double *caps_override /* [periods][n_inst] or NULL */,
                 double *tr_p /* p(k) seen at instant k */, double *tr_cap, double *tr_u /*[M][N]*/,
                 uint32_t *tr_active /*[M]*/, uint32_t *tr_tie /*[M]*/, int8_t *tr_rank /*[N]*/,
                 uint8_t *tr_levels /*[S][N]*/, double *tr_ahat /*[N]*/, double *tr_theta /*[N]*/,
                 uint32_t *tr_status, double *final_p /*[n_inst]: p(K)*/, ora_summary *summ,
                 double *A0_out /*[n_inst][N]*/, int use_definition_mode);

/* ---- baseline controllers (NEXT-2): same plant, S1-S3 replaced by the
 * controller of w->controller (Q32-Q35).  Traces as ora_simulate: tr_u holds
 * the command [N] (row 0 only), tr_theta the weights the controller saw. */
int ora_simulate_baseline(const ora_cfg *c, const ora_workload *w, int n_inst, const int64_t *inst,
                          double *tr_p, double *tr_cap, double *tr_u /*[N]*/, uint8_t *tr_levels /*[S][N]*/,
                          double *tr_theta /*[N]*/, double *final_p, ora_summary *summ);

/* ---- S5 hierarchical budget (cfg 4, Q16) */
int ora_simulate_hier(const ora_cfg *c, const ora_workload *w, int n_servers, int rack, double cluster_frac,
                      double rack_frac, const double *W_replay, double W0_replay, int n_total, int n_tr,
                      const int64_t *tr_srv,
                      double *tr_p, double *tr_cap, double *tr_u, uint32_t *tr_active, uint32_t *tr_tie,
                      uint8_t *tr_levels, double *tr_theta /*[N]: theta at instant k*/, double *agg_W, double *agg_P, double *final_p);
void ora_budget_caps(int n_servers, int rack, const double *pmin, const double *w, double W,
                     double B_c, double pmin_tot, const double *B_rack_max, double *cap);

#ifdef __cplusplus
}
#endif
#endif
