// capgpu_device.cuh -- per-instance device math of the CapGPU step (sm_100a, FP64).
//
// One CUDA thread owns one (server, cap) instance.  All loops over knobs are
// compile-time (template N) and fully unrolled, so the model, its LDL^T
// factors and the QP state live in registers.
//
// Instruction economy (the kernel is FP64-pipe / issue bound):
//   - clamps are plain compare+select (no fmin/fmax NaN handling), sums
//     are split in two partial accumulators for ILP;
//   - rarely executed code (QP phase 2, trace replays) is out of line so the
//     hot period loop fits the instruction cache;
//   - divisions that only feed continuous values use an MUFU seed + 2 Newton
//     steps; the one division that decides integers (theta -> ranks) is IEEE;
//   - frequency-grid arithmetic that must match the oracle bit for bit comes
//     from host-computed tables staged in shared memory.
//
// Citations: P:NNN = PAPER.md line; Qn = DESIGN.md §2 reading.
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

#include "../../gen/capgpu_gen.h"
#include "../../include/capgpu.h"

namespace capgpu {

constexpr int kMaxN = CAPGPU_MAX_KNOBS;
constexpr int kMaxM = CAPGPU_MAX_M;
constexpr int kMaxL = CAPGPU_MAX_LEVELS;
constexpr int kMaxS = 8;

template <int N>
struct Tri {
  static constexpr int size = N * (N + 1) / 2;
  // packed upper triangle, row-major: (i, j), i <= j
  static __host__ __device__ constexpr int idx(int i, int j) {
    return i <= j ? i * N - i * (i - 1) / 2 + (j - i) : j * N - j * (j - 1) / 2 + (i - j);
  }
};

// Uniform (per-launch) constants, passed by value (constant bank).
struct KnobConst {
  double f_min, f_max, step, inv_step;  // grid (Q15)
  double lo, hi, m;                     // box [l, h] (Eq. 10a, Q14) and penalty reference f_min (Q7)
  double span;                          // hi - m
  double r0, inv_r0;                    // r0_j and 1 / r0_j (Q6, Q9)
  double pos_tol;                       // plant_pair: distance to an interior grid point (in steps) that forces the exact path
  int32_t L;                            // levels
  int32_t sweep_base;
  int32_t cls;                          // grid class (knobs with identical grids share a table)
  int32_t pad;
};

// Per-class grid table entry, level l:  {mid(l-1) or -inf, mid(l) or +inf,
// level(l), g(l)}: decision thresholds, frequency and capacity factor (Q14, Q15).
struct GridEntry {
  double mid_lo, mid_hi, level, g;
};

// Per-class table of neighbouring level pairs (l, l+1), l = 0..L-2: the
// threshold mid(l) between them, both levels and both capacity factors --
// the same host-computed values as GridEntry (oracle formulas).  Row L-1
// duplicates row L-2 (never indexed).
struct PairEntry {
  double mid, lev0, lev1, g0, g1, pad;
};

struct DevParams {
  int32_t N, M, P, S;
  int32_t n_caps;            // instances per server
  int32_t demand_kind;
  int32_t n_class;
  int32_t convex;            // 1 iff lo_j == m_j (= f_min) for every knob: phi convex on s <= 0
  double demand_frac;
  double q, theta_min, lam, rho, a_lo, a_hi, a_floor;
  double inv_lam;             // 1 / lam (scaled Welford state of the fused kernel)
  int32_t fold_mask;         // R - 1: the fused kernel folds lam^-kk back into Sigma' at call periods
                             // kk = R - 1 mod R, R = 2^r <= 1024 with lam^-R <= 2^600 (host, from lam)
  double noise_scale;        // sigma * sqrt(3) (host-computed)
  double inv_S;              // 1/S, exact (S power of two, Q22)
  double inv_N;              // 1/N for the mean-theta summary
  double ct[kMaxM];          // block weights c_t (Q11)
  double cap_frac0, cap_frac_rand, cap_frac_step, cap_mult;
  double gain0, gain_step;   // plant gain mismatch g_c = gain0 + c * gain_step, gain0 = 1 + gain_dlo (NEXT-4)
  int64_t cap_period, cap_lo, cap_hi;
  uint64_t seed;
  int64_t srv_begin;         // global id of local server 0
  int64_t n_srv, n_inst;     // local counts
  const GridEntry *grid;     // device [n_class][kMaxL]
  const PairEntry *pair;     // device [n_class][kMaxL] (plant_pair)
  const KnobConst *k_dev;    // device copy of k[] for out-of-line code (keeps P in the param bank)
  // SLO schedule (NEXT-1, §6.4, Eq. 10b-c; Q29-Q31).  Phase B at instant k
  // while slo_period > 0 and k mod slo_period in [slo_lo, slo_hi).  k_dev_slo[ph]
  // = device copy of k[] with phase ph's lower bounds; q_slo[ph][j] = SLO level
  // index (0 = no SLO, L = unreachable); st_slo[ph] = SLO_INFEASIBLE or 0.
  int32_t slo;               // 1 iff an SLO is in force in either phase
  int64_t slo_period, slo_lo, slo_hi;
  const KnobConst *k_dev_slo[2];
  int32_t q_slo[2][kMaxN];
  uint32_t st_slo[2];
  // Baseline controllers (NEXT-2, §6.1; Q32-Q35): 0 = CapGPU MPC,
  // 1 = Fixed-step, 2 = Safe Fixed-step, 3 = GPU-only, 4 = CPU-only.
  int32_t bl_kind, bl_steps;
  double bl_margin, bl_pole;
  double bl_share;           // CPU+GPU: GPU share of the budget (Q39)
  double wmove;              // NEXT-3 move-suppression weight W (Q36); 0 = the literal Eq. 9
  int32_t ref;               // NEXT-3 reference trajectory on (Q37): block t tracks beta + ref_w[t] (P_s - p(k))
  double ref_w[kMaxM];
  int32_t no_chunking;       // 1: fused kernel without the chunked persistent schedule (env CAPGPU_NO_CHUNKING)
  long long *phase;          // [8][n_inst] cycle counters (builds with -DCAPGPU_PHASE_TIMING only)
  KnobConst k[kMaxN];
};

// ------------------------------------------------------------------ helpers

// Phase timing (profiling builds only): CAPGPU_MARK(P, id, i) adds the cycles
// since the previous mark to counter `id` of instance i.
#ifdef CAPGPU_PHASE_TIMING
struct PhaseClock {
  long long t;
};
#define CAPGPU_PHASE_DECL PhaseClock ph_clk{clock64()};
#define CAPGPU_MARK(P, id, i)                                                        \
  do {                                                                               \
    const long long t_ = clock64();                                                  \
    if ((P).phase) (P).phase[(int64_t)(id) * (P).n_inst + (i)] += t_ - ph_clk.t;     \
    ph_clk.t = clock64();                                                            \
  } while (0)
#else
#define CAPGPU_PHASE_DECL
#define CAPGPU_MARK(P, id, i) \
  do {                        \
  } while (0)
#endif

// True-gain factor of instance column `cidx` (NEXT-4, "A' = g A"):
// g = (1 + gain_dlo) + cidx * gain_step, rounded exactly as the oracle (no FMA).
__device__ __forceinline__ double plant_gain(const DevParams &P, int cidx) {
  return __dadd_rn(P.gain0, __dmul_rn((double)cidx, P.gain_step));
}

__device__ __forceinline__ double rcp_fast(double x) {
  // MUFU.RCP64H seed y0 with residual e = 1 - x y0, |e| < 2^-20, then
  // 1/x = y0 / (1 - e) = y0 (1 + e + e^2) + O(e^3): three dependent FMAs
  // (two Newton steps need four) for ~1 ulp (continuous quantities only;
  // tools/dbg/rcp_check.cu measures it on the device).
  double y;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
  const double e = fma(-x, y, 1.0);
  return fma(y, fma(e, e, e), y);
}

// One Newton step on the MUFU seed: |rel. error| <= e^2 < 2^-39 (~2e-12).
// Only for quantities whose error enters the outputs linearly and far below
// the 1e-9 parity bar (the weights theta that scale the MPC penalties).
__device__ __forceinline__ double rcp_nr1(double x) {
  double y;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
  return fma(y, fma(-x, y, 1.0), y);
}

// Position r = k mod cap_period in the cap step schedule of gen_cap_at,
// advanced by one per period instead of a 64-bit modulo (a software division)
// every period; the caps are bitwise those of gen_cap_at.  Used by the
// latency-bound lane-parallel kernel (cfg 2: 1.45 -> 1.35 us per period with
// the draws hoisted, capgpu_lanes.cuh); in k_simulate the extra live register
// cost more than the modulo saved (cfgs 3/5 -1.2 / -1.5 %, no cap schedule).
struct CapSched {
  int64_t r;
  __device__ __forceinline__ CapSched(const DevParams &P, int64_t k) : r(P.cap_period > 0 ? k % P.cap_period : 0) {}
  __device__ __forceinline__ double cap(const DevParams &P, double base) const {
    return (P.cap_period > 0 && r >= P.cap_lo && r < P.cap_hi) ? GEN_MUL(base, P.cap_mult) : base;
  }
  __device__ __forceinline__ void next(const DevParams &P) {
    if (P.cap_period > 0 && ++r == P.cap_period) r = 0;
  }
};

__device__ __forceinline__ long long dbits(double x) { return __double_as_longlong(x); }
__device__ __forceinline__ double bitsd(long long b) { return __longlong_as_double(b); }

// clamp without fmin/fmax NaN handling: one DSETP + two FSEL per side
__device__ __forceinline__ double pclamp(double x, double lo, double hi) {
  return x < lo ? lo : (x > hi ? hi : x);
}

// ------------------------------------------------------------------ S1 model
// Weighted Welford push (Q1-Q3): w <- lam w + 1, delta = z - mu,
// mu += delta / w, Sigma <- lam Sigma + (1 - 1/w) delta delta^T
// (= delta (z - mu_new)^T in exact arithmetic).
// Scaled form (fused kernel): the stored Sigma' = Sigma / Lambda with
// Lambda = lam^k since the start of the call, so the decay needs no multiply:
// Sigma' <- Sigma' + (e / Lambda_new) delta delta^T (inv_lam_k = 1 / Lambda_new);
// the solve uses rho / Lambda (same solution), and the caller multiplies
// Sigma' back by Lambda before it leaves the kernel (and every 1024 periods).
// SCALED = false: the plain form above (state in HBM, one period per launch).
template <int N, bool SCALED, class SAcc, class VAcc, class FAcc>
__device__ __forceinline__ void model_push(double lam, double inv_lam_k, double &w, VAcc mu_f, double &mu_p,
                                           SAcc S, FAcc Sfp, const double (&f)[N], double p) {
  w = fma(lam, w, 1.0);
  const double iw = rcp_fast(w);
  const double e = SCALED ? (1.0 - iw) * inv_lam_k : 1.0 - iw;
  double df[N];
#pragma unroll
  for (int j = 0; j < N; ++j) {
    const double m = mu_f.get(j);
    df[j] = f[j] - m;
    mu_f.set(j, fma(df[j], iw, m));
  }
  const double dp = p - mu_p;
  mu_p = fma(dp, iw, mu_p);
  const double edp = e * dp;
#pragma unroll
  for (int i = 0; i < N; ++i) {
    const double ei = e * df[i];
#pragma unroll
    for (int j = i; j < N; ++j) {
      const int t = Tri<N>::idx(i, j);
      if constexpr (SCALED)
        S.set(t, fma(ei, df[j], S.get(t)));
      else
        S.set(t, fma(lam, S.get(t), ei * df[j]));
    }
    if constexpr (SCALED)
      Sfp.set(i, fma(df[i], edp, Sfp.get(i)));
    else
      Sfp.set(i, fma(lam, Sfp.get(i), df[i] * edp));
  }
}

// In-register LDL^T solve of a packed SPD system: A (packed upper, destroyed
// into the factors), b -> x.  Used for the model (S1) and identification (S0).
//
// Critical path.  Column j waits for d_j, which waits for dinv_{j-1} through
// the last term L(j,j-1) W(j,j-1) of its sum, W(i,k) = L(i,k) D_k being the
// unnormalised column.  W(j,j-1) is kept from column j-1 (wp[]) instead of
// being re-formed as L(j,j-1) D_{j-1}, so the chain per column is one DMUL
// (L = W dinv), one DFMA and the 3-deep reciprocal; the other W(j,k) are
// re-formed off the critical path.
template <int N>
__device__ __forceinline__ void ldlt_solve(double (&L)[Tri<N>::size], const double (&b)[N], double (&x)[N]) {
  double dinv[N];
  double wp[N];  // wp[i] = W(i, j-1) of the previous column (rows i >= j)
#pragma unroll
  for (int j = 0; j < N; ++j) {
    double v[N > 1 ? N - 1 : 1];
    double d = L[Tri<N>::idx(j, j)];
#pragma unroll
    for (int k = 0; k < j; ++k) {
      // v_k = W(j,k) = L(j,k) D_k with the unit-lower factor L(j,k) of column k
      v[k] = k == j - 1 ? wp[j] : L[Tri<N>::idx(j, k)] * L[Tri<N>::idx(k, k)];
      d = fma(-L[Tri<N>::idx(j, k)], v[k], d);
    }
    L[Tri<N>::idx(j, j)] = d;
    dinv[j] = rcp_fast(d);
#pragma unroll
    for (int i = j + 1; i < N; ++i) {
      double y = L[Tri<N>::idx(i, j)];
#pragma unroll
      for (int k = 0; k < j; ++k) y = fma(-L[Tri<N>::idx(i, k)], v[k], y);
      wp[i] = y;
      L[Tri<N>::idx(i, j)] = y * dinv[j];
    }
  }
  double y[N];
#pragma unroll
  for (int i = 0; i < N; ++i) {
    double t = b[i];
#pragma unroll
    for (int k = 0; k < i; ++k) t = fma(-L[Tri<N>::idx(i, k)], y[k], t);
    y[i] = t;
  }
#pragma unroll
  for (int i = N - 1; i >= 0; --i) {
    // x_{i+1} (the most recent) enters last: a linear, not quadratic, chain
    double t = y[i] * dinv[i];
#pragma unroll
    for (int k = N - 1; k > i; --k) t = fma(-L[Tri<N>::idx(k, i)], x[k], t);
    x[i] = t;
  }
}

// (Sigma_ff + rho I) a = Sigma_fp + rho A0, then clamp to [a_lo A0, a_hi A0] (Q1, Q4).
template <int N, class SAcc, class VAcc, class A0Acc>
__device__ __forceinline__ void model_solve(double rho, double a_lo, double a_hi, SAcc S, VAcc Sfp, A0Acc A0,
                                            double (&ahat)[N]) {
  double L[Tri<N>::size];
#pragma unroll
  for (int t = 0; t < Tri<N>::size; ++t) L[t] = S.get(t);
#pragma unroll
  for (int j = 0; j < N; ++j) L[Tri<N>::idx(j, j)] += rho;
  double b[N];
#pragma unroll
  for (int i = 0; i < N; ++i) b[i] = fma(rho, A0.get(i), Sfp.get(i));
  ldlt_solve<N>(L, b, ahat);
#pragma unroll
  for (int j = 0; j < N; ++j) {
    const double a0 = A0.get(j);
    ahat[j] = pclamp(ahat[j], a_lo * a0, a_hi * a0);
  }
}

// ------------------------------------------------------------------ S2 weights
// theta = clamp(thr/thr_max, theta_min, 1) with IEEE division (ranks must be
// bit-exact, §8(c.4)); ranks: stable descending (Q10).
template <int N>
__device__ __forceinline__ void weights(double theta_min, const double (&thr)[N], const double (&thr_max)[N],
                                        double (&theta)[N]) {
#pragma unroll
  for (int j = 0; j < N; ++j) theta[j] = pclamp(__ddiv_rn(thr[j], thr_max[j]), theta_min, 1.0);
}

template <int N>
__device__ __forceinline__ void ranks(const double (&theta)[N], int8_t (&rk)[N]) {
#pragma unroll
  for (int j = 0; j < N; ++j) {
    int r = 0;
#pragma unroll
    for (int l = 0; l < N; ++l) {
      if (l == j) continue;
      const long long tl = dbits(theta[l]), tj = dbits(theta[j]);
      r += (tl > tj) || (l < j && tl == tj);
    }
    rk[j] = (int8_t)r;
  }
}

// ------------------------------------------------------------------ S3 MPC block
// Block t of the decoupled Eq. 9 (Q11):
//   min_{lo<=u<=hi} c (beta + a.u)^2 + sum_j R_j (u_j - m_j)^2
// KKT: u_j(s) = clamp(m_j - c tau_j s, lo_j, hi_j), tau_j = a_j / R_j, and
// s = beta + a.u(s) (the predicted tracking error).  phi(s) = s - beta - a.u(s)
// is strictly increasing and piecewise linear with slope
// phi'(s) = 1 + sum_{free j} c tau_j a_j >= 1, so the root is unique and is the
// exact root of the linear piece it lies on.
//   phase 1: Newton from the previous period's root s_prev (warm start):
//            s' = s - phi(s)/phi'(s).  When the active set at s' equals the one
//            at s, s' is the root of that piece: exact.  Two tries.
//   phase 2: otherwise the root's active set is read off phi at each knob's
//            two breakpoints (phi increasing: s* > b <=> phi(b) < 0; <= 2N
//            evaluations, no sorting) and the root of that piece is exact.

// phi, slope and active codes at s.  cta_j = c tau_j a_j.  Per knob: one
// DFMA for v, two DSETP, predicated accumulation (no selects on the FP64
// pipe beyond the clamp).  Two partial sums for ILP.
template <int N>
__device__ __forceinline__ uint32_t block_eval(const KnobConst *kc, const double (&a)[N], const double (&ctau)[N],
                                               const double (&cta)[N], double beta, double s, double &phi,
                                               double &slope) {
  uint32_t code = 0u;
  double f0 = s - beta, f1 = 0.0, d0 = 1.0, d1 = 0.0;
#pragma unroll
  for (int j = 0; j < N; ++j) {
    const double v = fma(-ctau[j], s, kc[j].m);
    const bool low = v < kc[j].lo, up = v > kc[j].hi;
    code |= (low ? 1u : 0u) << (2 * j);
    code |= (up ? 2u : 0u) << (2 * j);
    const double u = low ? kc[j].lo : (up ? kc[j].hi : v);
    if (j & 1) {
      f1 = fma(-a[j], u, f1);
      if (!(low || up)) d1 += cta[j];
    } else {
      f0 = fma(-a[j], u, f0);
      if (!(low || up)) d0 += cta[j];
    }
  }
  phi = f0 + f1;
  slope = d0 + d1;
  return code;
}

template <int N>
__device__ __forceinline__ uint32_t block_codes(const KnobConst *kc, const double (&ctau)[N], double s) {
  uint32_t code = 0u;
#pragma unroll
  for (int j = 0; j < N; ++j) {
    const double v = fma(-ctau[j], s, kc[j].m);
    code |= (v < kc[j].lo ? 1u : 0u) << (2 * j);
    code |= (v > kc[j].hi ? 2u : 0u) << (2 * j);
  }
  return code;
}

// phase 2 (rare): exact active set of the root read off phi at each knob's
// breakpoints.  Kept out of line so the hot loop stays small (I-cache).
template <int N>
__device__ __noinline__ double block_exact(const KnobConst *kc, const double *a_p, const double *ctau_p,
                                           double beta) {
  double a[N], ctau[N], cta[N];
#pragma unroll
  for (int j = 0; j < N; ++j) {
    a[j] = a_p[j];
    ctau[j] = ctau_p[j];
    cta[j] = ctau[j] * a[j];
  }
  double num = beta, den = 1.0;
#pragma unroll 1
  for (int j = 0; j < N; ++j) {
    double x;
    const double cj = ctau_p[j];
    if (!(cj > 0.0)) {
      x = pclamp(kc[j].m, kc[j].lo, kc[j].hi);
    } else {
      const double r = rcp_fast(cj);
      double fb, sl;
      block_eval<N>(kc, a, ctau, cta, beta, (kc[j].m - kc[j].lo) * r, fb, sl);
      if (fb < 0.0) {
        x = kc[j].lo;  // root right of b_l: lower
      } else {
        block_eval<N>(kc, a, ctau, cta, beta, (kc[j].m - kc[j].hi) * r, fb, sl);
        if (fb > 0.0) {
          x = kc[j].hi;  // root left of b_h: upper
        } else {
          x = kc[j].m;  // free
          den += cj * a_p[j];
        }
      }
    }
    num = fma(a_p[j], x, num);
  }
  return num * rcp_fast(den);
}

// One convex block (weight c), exact: iterate U <- U(s_U) from the start set
// `up` (upper bits 2j+1).  Any start set works: every piece line of the convex
// phi lies below phi, so s_U >= s* and U(s_U) is a subset of U(s*); s moves
// down monotonically and stops on the root's piece (<= N + 1 steps).  The set
// sums are predicated adds (no 0/1 masks); the classification is Q19's
// v_j = m_j - c tau_j s > h_j written as -(c s) tau_j > h_j - m_j.
//   ta_j = tau_j a_j, ad_j = a_j (h_j - m_j), TA = sum_j ta_j, base = beta + a.l < 0.
template <int N>
__device__ __forceinline__ double convex_root(const KnobConst *kc, double c, const double (&tau)[N],
                                              const double (&ta)[N], const double (&ad)[N], double base, double TA,
                                              uint32_t &up) {
  double s = 0.0;
#pragma unroll 1
  for (int it = 0; it <= N; ++it) {
    double n0 = base, n1 = 0.0, d0 = 0.0, d1 = 0.0;
#pragma unroll
    for (int j = 0; j < N; ++j) {
      if ((up >> (2 * j + 1)) & 1u) {
        if (j & 1) {
          n1 += ad[j];
          d1 += ta[j];
        } else {
          n0 += ad[j];
          d0 += ta[j];
        }
      }
    }
    s = (n0 + n1) * rcp_fast(fma(c, TA - (d0 + d1), 1.0));
    const double mcs = -c * s;
    uint32_t nu = 0u;
#pragma unroll
    for (int j = 0; j < N; ++j) nu |= (mcs * tau[j] > kc[j].span ? 2u : 0u) << (2 * j);
    if (nu == up) break;
    up = nu;
  }
  return s;
}

// Does the convex block with weight c have any bound active at its root?
// U(s*) is empty iff U(s_0) is, s_0 = base / (1 + c TA) being the all-free
// root (U only grows as s decreases, and s* <= s_0).  The fused kernel needs
// only this bit for the blocks it does not apply or trace (act_count summary).
template <int N>
__device__ __forceinline__ bool convex_any_upper(const KnobConst *kc, double c, const double (&tau)[N], double base,
                                                 double TA) {
  const double mcs = -c * (base * rcp_fast(fma(c, TA, 1.0)));
  bool any = false;
#pragma unroll
  for (int j = 0; j < N; ++j) any |= mcs * tau[j] > kc[j].span;
  return any;
}

// Branch-free exact block solve for small N: phi at all 2N breakpoints at
// once (independent clamp terms, no chain), the root's active set read off
// their signs exactly as block_exact decides it (phi increasing: knob j is
// lower iff phi(b_l,j) < 0, upper iff phi(b_h,j) > 0), then the root of that
// piece.  On the SLO bench Newton's first two pieces missed the root in
// 12.5 % of the lanes, so 98 % of the warps ran the out-of-line fallback.
template <int N>
__device__ __forceinline__ double phi_at(const KnobConst *kc, const double (&a)[N], const double (&ctau)[N],
                                         double beta, double s) {
  double f0 = s - beta, f1 = 0.0;
#pragma unroll
  for (int k = 0; k < N; ++k) {
    const double v = fma(-ctau[k], s, kc[k].m);
    const double u = v < kc[k].lo ? kc[k].lo : (v > kc[k].hi ? kc[k].hi : v);
    if (k & 1)
      f1 = fma(-a[k], u, f1);
    else
      f0 = fma(-a[k], u, f0);
  }
  return f0 + f1;
}

template <int N>
__device__ __forceinline__ double block_direct(const KnobConst *kc, const double (&a)[N], const double (&ctau)[N],
                                               double beta) {
  double bh[N], bl[N], ph[N], pl[N];
#pragma unroll
  for (int j = 0; j < N; ++j) {
    const double r = rcp_fast(ctau[j]);
    bh[j] = (kc[j].m - kc[j].hi) * r;
    bl[j] = (kc[j].m - kc[j].lo) * r;
  }
#pragma unroll
  for (int j = 0; j < N; ++j) {
    ph[j] = phi_at<N>(kc, a, ctau, beta, bh[j]);
    pl[j] = phi_at<N>(kc, a, ctau, beta, bl[j]);
  }
  double num = beta, den = 1.0;
#pragma unroll
  for (int j = 0; j < N; ++j) {
    double x;
    if (!(ctau[j] > 0.0)) {
      x = pclamp(kc[j].m, kc[j].lo, kc[j].hi);
    } else if (pl[j] < 0.0) {
      x = kc[j].lo;  // root right of b_l: lower
    } else if (ph[j] > 0.0) {
      x = kc[j].hi;  // root left of b_h: upper
    } else {
      x = kc[j].m;  // free
      den += ctau[j] * a[j];
    }
    num = fma(a[j], x, num);
  }
  return num * rcp_fast(den);
}

// Solve one block; returns the root s (u and codes follow from it).
template <int N>
__device__ __forceinline__ double solve_block(const KnobConst *kc, const KnobConst *kc_dev, const double (&a)[N],
                                              const double (&ctau)[N],
                                              double beta, double s_warm) {
#ifndef CAPGPU_BLOCK_DIRECT_MAX_N
#define CAPGPU_BLOCK_DIRECT_MAX_N 6  // 2N^2 clamp terms: small N only (larger N keep Newton + fallback)
#endif
  if constexpr (N <= CAPGPU_BLOCK_DIRECT_MAX_N) {
    (void)kc_dev;
    (void)s_warm;
    return block_direct<N>(kc, a, ctau, beta);
  }
  double cta[N];
#pragma unroll
  for (int j = 0; j < N; ++j) cta[j] = ctau[j] * a[j];
  double s = s_warm;
#ifndef CAPGPU_NEWTON_TRIES  // 3 / 4 / 6 tries measured 5 / 9 / 16 % slower on the SLO bench (lanes that
#define CAPGPU_NEWTON_TRIES 2  // leave Newton's first two pieces oscillate; tools/ab_slo.sh)
#endif
#pragma unroll 1
  for (int it = 0; it < CAPGPU_NEWTON_TRIES; ++it) {
    double phi, slope;
    const uint32_t c0 = block_eval<N>(kc, a, ctau, cta, beta, s, phi, slope);
    if (phi == 0.0) return s;
    const double s1 = fma(-phi, rcp_fast(slope), s);
    if (block_codes<N>(kc, ctau, s1) == c0) return s1;
    s = s1;
  }
  double a_l[N], c_l[N];
#pragma unroll
  for (int j = 0; j < N; ++j) {
    a_l[j] = a[j];
    c_l[j] = ctau[j];
  }
  return block_exact<N>(kc_dev, a_l, c_l, beta);
}

// u(s) and the 2-bit codes at the root (Q19: exact tie counts as free).
template <int N>
__device__ __forceinline__ uint32_t block_u(const KnobConst *kc, const double (&ctau)[N], double s, double (&u)[N]) {
  uint32_t code = 0u;
#pragma unroll
  for (int j = 0; j < N; ++j) {
    const double v = fma(-ctau[j], s, kc[j].m);
    const bool low = v < kc[j].lo, up = v > kc[j].hi;
    code |= (low ? 1u : 0u) << (2 * j);
    code |= (up ? 2u : 0u) << (2 * j);
    u[j] = low ? kc[j].lo : (up ? kc[j].hi : v);
  }
  return code;
}

// ------------------------------------------------------------------ S3 with move suppression (NEXT-3)
// Eq. 9 + sum_{t<M} W |u_t - u_{t-1}|^2, u_{-1} = f(k) (Q36): the M blocks
// couple through the increments, so the decoupled block solve no longer
// applies.  Generic primal active set on the stacked MN-variable box QP
// (Nocedal & Wright Alg. 16.3 for bounds), per thread, warm-started from last
// period's active set, fixed iteration cap 3 MN + 3 (CAPGPU_ST_SOLVER_CAP).
// The equality-constrained subproblem of each iteration is one masked LDL^T of
// the full MN x MN Hessian (fixed variables -> identity rows), so the code is
// branch-free and fully unrolled.  Half the Hessian (variable a = t N + j):
//   H(a, a)  = c_t A_j^2 + R_j + W (1 + [t < M-1])
//   H(a, b)  = c_t A_j A_k  (same t, k != j);  -W (same j, |t - t'| = 1)
//   g(a)     = c_t beta_t A_j - R_j m_j - [t = 0] W f_j,  beta_t = beta + ref_w[t] dref (Q37)
template <int N, int M>
__device__ __forceinline__ double move_h(const DevParams &P, const double (&a)[N], const double (&R)[N], int x,
                                         int y) {
  const int tx = x / N, jx = x - tx * N, ty = y / N, jy = y - ty * N;
  if (tx == ty) {
    double h = P.ct[tx] * a[jx] * a[jy];
    if (jx == jy) h += R[jx] + P.wmove * (tx < M - 1 ? 2.0 : 1.0);
    return h;
  }
  return (jx == jy && (tx - ty == 1 || ty - tx == 1)) ? -P.wmove : 0.0;
}

template <int N, int M>
__device__ __forceinline__ uint32_t move_qp(const DevParams &P, const KnobConst *kc, const double (&a)[N],
                                            const double (&R)[N], double beta, double dref, const double (&f)[N],
                                            uint32_t (&act)[M], double (&x)[M * N]) {
  constexpr int V = M * N;
  double g[V];
  uint32_t lo_m = 0u, up_m = 0u;  // working set: variable a fixed at its lower / upper bound
#pragma unroll
  for (int t = 0; t < M; ++t) {
#pragma unroll
    for (int j = 0; j < N; ++j) {
      const int v = t * N + j;
      g[v] = P.ct[t] * fma(P.ref_w[t], dref, beta) * a[j] - R[j] * kc[j].m - (t == 0 ? P.wmove * f[j] : 0.0);
      const uint32_t code = (act[t] >> (2 * j)) & 3u;
      lo_m |= (code == 1u ? 1u : 0u) << v;
      up_m |= (code == 2u ? 1u : 0u) << v;
      x[v] = code == 1u ? kc[j].lo : (code == 2u ? kc[j].hi : pclamp(f[j], kc[j].lo, kc[j].hi));
    }
  }
  double gscale = 1.0;
#pragma unroll
  for (int v = 0; v < V; ++v) gscale = fmax(gscale, fabs(g[v]));
  uint32_t status = CAPGPU_ST_SOLVER_CAP;
#pragma unroll 1
  for (int it = 0; it < 3 * V + 3; ++it) {
    const uint32_t fix = lo_m | up_m;
    // equality-constrained subproblem on the free set (masked LDL^T)
    double L[Tri<V>::size], rhs[V], xs[V];
#pragma unroll
    for (int u = 0; u < V; ++u) {
      const bool fu = (fix >> u) & 1u;
      double r = -g[u];
#pragma unroll
      for (int w = 0; w < V; ++w) {
        const bool fw = (fix >> w) & 1u;
        const double h = move_h<N, M>(P, a, R, u, w);
        if (w >= u) L[Tri<V>::idx(u, w)] = (fu || fw) ? (u == w ? 1.0 : 0.0) : h;
        if (fw) r = fma(-h, x[w], r);
      }
      rhs[u] = fu ? x[u] : r;
    }
    ldlt_solve<V>(L, rhs, xs);
    // ratio test along xs - x over the free variables
    double alpha = 1.0;
    int blk = -1;
    bool blk_up = false;
#pragma unroll
    for (int u = 0; u < V; ++u) {
      if ((fix >> u) & 1u) continue;
      const int j = u % N;
      const double d = xs[u] - x[u];
      if (xs[u] < kc[j].lo && d < 0.0) {
        const double al = (kc[j].lo - x[u]) / d;
        if (al < alpha) { alpha = al; blk = u; blk_up = false; }
      } else if (xs[u] > kc[j].hi && d > 0.0) {
        const double al = (kc[j].hi - x[u]) / d;
        if (al < alpha) { alpha = al; blk = u; blk_up = true; }
      }
    }
    if (blk >= 0) {  // blocked: step to the bound, fix the blocking variable
#pragma unroll
      for (int u = 0; u < V; ++u)
        if (!((fix >> u) & 1u)) x[u] = pclamp(fma(alpha, xs[u] - x[u], x[u]), kc[u % N].lo, kc[u % N].hi);
      x[blk] = blk_up ? kc[blk % N].hi : kc[blk % N].lo;
      if (blk_up) up_m |= 1u << blk; else lo_m |= 1u << blk;
      continue;
    }
#pragma unroll
    for (int u = 0; u < V; ++u) x[u] = xs[u];
    // stationary on the face: bound multipliers of the fixed variables
    int worst = -1;
    double most = -1e-12 * gscale;
#pragma unroll
    for (int u = 0; u < V; ++u) {
      if (!((fix >> u) & 1u)) continue;
      double gr = g[u];
#pragma unroll
      for (int w = 0; w < V; ++w) gr = fma(move_h<N, M>(P, a, R, u, w), x[w], gr);
      const double lam = ((lo_m >> u) & 1u) ? gr : -gr;
      if (lam < most) { most = lam; worst = u; }
    }
    if (worst < 0) { status = 0u; break; }
    lo_m &= ~(1u << worst);
    up_m &= ~(1u << worst);
  }
#pragma unroll
  for (int t = 0; t < M; ++t) {
    uint32_t c = 0u;
#pragma unroll
    for (int j = 0; j < N; ++j) {
      const int v = t * N + j;
      c |= ((((lo_m >> v) & 1u) ? 1u : 0u) | (((up_m >> v) & 1u) ? 2u : 0u)) << (2 * j);
    }
    act[t] = c;
  }
  return status;
}

// ------------------------------------------------------------------ S3 move suppression, structured (NEXT-3, M N <= 64)
// The same QP as move_qp (Q36), solved without forming the MN x MN Hessian.
// H = T + sum_t c_t v_t v_t^T: T is N independent M x M tridiagonal matrices
// (knob j: diagonal R_j + W (1 + [t < M-1]), off-diagonal -W between t and
// t + 1) and v_t = A on block t (the rank-1 tracking term of Eq. 9's block t).
// The equality-constrained subproblem of each active-set iteration keeps this
// form on the free variables (fixed rows -> identity, their couplings -> the
// right-hand side), so it is solved by the Woodbury identity:
//   y = T^-1 r - T^-1 V (C^-1 + V^T T^-1 V)^-1 V^T T^-1 r,
// N tridiagonal solves of size M plus one M x M system: O(M^2 N) per
// iteration instead of the dense O((MN)^3 / 6).  T is strictly diagonally
// dominant (R > 0) and the M x M capacitance matrix is SPD.

// LDL^T of one knob's masked tridiagonal (free: diagonal dd_t, coupling -W
// to a free neighbour; fixed: identity row) and its inverse G (symmetric).
template <int M>
__device__ __forceinline__ void tri_inverse(const double (&dd)[M], const bool (&fr)[M], double W, double (&G)[M][M],
                                            double (&dinv)[M], double (&ll)[M]) {
  // factor: D_0 = dd_0; l_t = e_t / D_{t-1}; D_t = dd_t - e_t l_t, e_t = -W if t-1, t both free
#pragma unroll
  for (int t = 0; t < M; ++t) {
    const double e = (t > 0 && fr[t] && fr[t - 1]) ? -W : 0.0;
    const double Dt = fr[t] ? (t > 0 ? fma(-e, e * dinv[t > 0 ? t - 1 : 0], dd[t]) : dd[t]) : 1.0;
    ll[t] = t > 0 ? e * dinv[t > 0 ? t - 1 : 0] : 0.0;
    dinv[t] = rcp_fast(Dt);
  }
  // columns of the inverse: solve L D L^T g = e_c
#pragma unroll
  for (int c = 0; c < M; ++c) {
    double y[M];
#pragma unroll
    for (int t = 0; t < M; ++t) y[t] = (t == c ? 1.0 : 0.0) - (t > 0 ? ll[t] * y[t > 0 ? t - 1 : 0] : 0.0);
#pragma unroll
    for (int t = M - 1; t >= 0; --t) G[t][c] = y[t] * dinv[t] - (t < M - 1 ? ll[t < M - 1 ? t + 1 : 0] * G[t < M - 1 ? t + 1 : 0][c] : 0.0);
  }
}

template <int M>
__device__ __forceinline__ void tri_solve(const double (&dinv)[M], const double (&ll)[M], const double (&b)[M],
                                          double (&x)[M]) {
  double y[M];
#pragma unroll
  for (int t = 0; t < M; ++t) y[t] = b[t] - (t > 0 ? ll[t] * y[t > 0 ? t - 1 : 0] : 0.0);
#pragma unroll
  for (int t = M - 1; t >= 0; --t) x[t] = y[t] * dinv[t] - (t < M - 1 ? ll[t < M - 1 ? t + 1 : 0] * x[t < M - 1 ? t + 1 : 0] : 0.0);
}

template <int N, int M>
__device__ __forceinline__ uint32_t move_qp_w(const DevParams &P, const KnobConst *kc, const double (&a)[N],
                                              const double (&R)[N], double beta, double dref, const double (&f)[N],
                                              uint32_t (&act)[M], double (&x)[M * N]) {
  constexpr int V = M * N;
  static_assert(V <= 64, "masks are 64-bit");
  const double W = P.wmove;
  double g[V];
  uint64_t lo_m = 0u, up_m = 0u;  // working set: variable fixed at its lower / upper bound
#pragma unroll
  for (int t = 0; t < M; ++t) {
#pragma unroll
    for (int j = 0; j < N; ++j) {
      const int v = t * N + j;
      g[v] = P.ct[t] * fma(P.ref_w[t], dref, beta) * a[j] - R[j] * kc[j].m - (t == 0 ? W * f[j] : 0.0);
      const uint32_t code = (act[t] >> (2 * j)) & 3u;
      lo_m |= (code == 1u ? 1ull : 0ull) << v;
      up_m |= (code == 2u ? 1ull : 0ull) << v;
      x[v] = code == 1u ? kc[j].lo : (code == 2u ? kc[j].hi : pclamp(f[j], kc[j].lo, kc[j].hi));
    }
  }
  double gscale = 1.0;
#pragma unroll
  for (int v = 0; v < V; ++v) gscale = fmax(gscale, fabs(g[v]));
  double cinv[M];
#pragma unroll
  for (int t = 0; t < M; ++t) cinv[t] = 1.0 / P.ct[t];
  uint32_t status = CAPGPU_ST_SOLVER_CAP;
#pragma unroll 1
  for (int it = 0; it < 3 * V + 3; ++it) {
    const uint64_t fix = lo_m | up_m;
    // rank-1 loads of the fixed variables per block: sX_t = sum_{j fixed at t} A_j x_tj
    double sX[M];
#pragma unroll
    for (int t = 0; t < M; ++t) {
      sX[t] = 0.0;
#pragma unroll
      for (int j = 0; j < N; ++j)
        if ((fix >> (t * N + j)) & 1ull) sX[t] = fma(a[j], x[t * N + j], sX[t]);
    }
    // pass 1, per knob: p_j = T_j^-1 r_j, Q += (a_j a_j^T) o G_j on the free entries, q = V^T p
    double Q[M][M], q[M];
#pragma unroll
    for (int s2 = 0; s2 < M; ++s2) {
      q[s2] = 0.0;
#pragma unroll
      for (int t = 0; t < M; ++t) Q[s2][t] = 0.0;
    }
#pragma unroll
    for (int j = 0; j < N; ++j) {
      double dd[M], r[M], G[M][M], dinv[M], ll[M], pj[M];
      bool fr[M];
#pragma unroll
      for (int t = 0; t < M; ++t) {
        const int v = t * N + j;
        fr[t] = !((fix >> v) & 1ull);
        dd[t] = R[j] + W * (t < M - 1 ? 2.0 : 1.0) + 0.0;
        // r = -g - H[:, fixed] x_fixed on the free rows: tridiagonal couplings
        // (-W to a fixed neighbour) and the block's rank-1 term
        double rv = -g[v] - P.ct[t] * a[j] * sX[t];
        if (t > 0 && ((fix >> (v >= N ? v - N : 0)) & 1ull)) rv = fma(W, x[v >= N ? v - N : 0], rv);
        if (t < M - 1 && ((fix >> (v + N < V ? v + N : 0)) & 1ull)) rv = fma(W, x[v + N < V ? v + N : 0], rv);
        r[t] = fr[t] ? rv : 0.0;
      }
      tri_inverse<M>(dd, fr, W, G, dinv, ll);
      tri_solve<M>(dinv, ll, r, pj);
#pragma unroll
      for (int s2 = 0; s2 < M; ++s2) {
        const double as = fr[s2] ? a[j] : 0.0;
        q[s2] = fma(as, pj[s2], q[s2]);
#pragma unroll
        for (int t = 0; t < M; ++t) Q[s2][t] = fma(as * (fr[t] ? a[j] : 0.0), G[s2][t], Q[s2][t]);
      }
    }
    // capacitance system (C^-1 + Q) z = q, M x M SPD: plain LDL^T
    double z[M];
    {
      double L[Tri<M>::size], b[M];
#pragma unroll
      for (int s2 = 0; s2 < M; ++s2) {
        b[s2] = q[s2];
#pragma unroll
        for (int t = s2; t < M; ++t) L[Tri<M>::idx(s2, t)] = Q[s2][t] + (s2 == t ? cinv[s2] : 0.0);
      }
      ldlt_solve<M>(L, b, z);
    }
    // pass 2, per knob: y_j = p_j - T_j^-1 (a_j z) on the free entries
    double xs[V];
#pragma unroll
    for (int j = 0; j < N; ++j) {
      double dd[M], r[M], G[M][M], dinv[M], ll[M], pj[M], c[M], cj[M];
      bool fr[M];
#pragma unroll
      for (int t = 0; t < M; ++t) {
        const int v = t * N + j;
        fr[t] = !((fix >> v) & 1ull);
        dd[t] = R[j] + W * (t < M - 1 ? 2.0 : 1.0) + 0.0;
        double rv = -g[v] - P.ct[t] * a[j] * sX[t];
        if (t > 0 && ((fix >> (v >= N ? v - N : 0)) & 1ull)) rv = fma(W, x[v >= N ? v - N : 0], rv);
        if (t < M - 1 && ((fix >> (v + N < V ? v + N : 0)) & 1ull)) rv = fma(W, x[v + N < V ? v + N : 0], rv);
        r[t] = fr[t] ? rv : 0.0;
        c[t] = fr[t] ? a[j] * z[t] : 0.0;
      }
      tri_inverse<M>(dd, fr, W, G, dinv, ll);
      tri_solve<M>(dinv, ll, r, pj);
      tri_solve<M>(dinv, ll, c, cj);
#pragma unroll
      for (int t = 0; t < M; ++t) xs[t * N + j] = fr[t] ? pj[t] - cj[t] : x[t * N + j];
    }
    // ratio test along xs - x over the free variables
    double alpha = 1.0;
    int blk = -1;
    bool blk_up = false;
#pragma unroll
    for (int u = 0; u < V; ++u) {
      if ((fix >> u) & 1ull) continue;
      const int j = u % N;
      const double d = xs[u] - x[u];
      if (xs[u] < kc[j].lo && d < 0.0) {
        const double al = (kc[j].lo - x[u]) / d;
        if (al < alpha) { alpha = al; blk = u; blk_up = false; }
      } else if (xs[u] > kc[j].hi && d > 0.0) {
        const double al = (kc[j].hi - x[u]) / d;
        if (al < alpha) { alpha = al; blk = u; blk_up = true; }
      }
    }
    if (blk >= 0) {  // blocked: step to the bound, fix the blocking variable
#pragma unroll
      for (int u = 0; u < V; ++u)
        if (!((fix >> u) & 1ull)) x[u] = pclamp(fma(alpha, xs[u] - x[u], x[u]), kc[u % N].lo, kc[u % N].hi);
      x[blk] = blk_up ? kc[blk % N].hi : kc[blk % N].lo;
      if (blk_up) up_m |= 1ull << blk; else lo_m |= 1ull << blk;
      continue;
    }
#pragma unroll
    for (int u = 0; u < V; ++u) x[u] = xs[u];
    // stationary on the face: bound multipliers of the fixed variables,
    // grad = g + H x = g + T x + c_t A_j (A . x_t)
    double ax[M];
#pragma unroll
    for (int t = 0; t < M; ++t) {
      ax[t] = 0.0;
#pragma unroll
      for (int j = 0; j < N; ++j) ax[t] = fma(a[j], x[t * N + j], ax[t]);
    }
    int worst = -1;
    double most = -1e-12 * gscale;
#pragma unroll
    for (int u = 0; u < V; ++u) {
      if (!((fix >> u) & 1ull)) continue;
      const int t = u / N, j = u % N;
      double gr = fma(P.ct[t] * a[j], ax[t], g[u]);
      gr = fma(R[j] + W * (t < M - 1 ? 2.0 : 1.0), x[u], gr);
      if (t > 0) gr = fma(-W, x[u >= N ? u - N : 0], gr);
      if (t < M - 1) gr = fma(-W, x[u + N < V ? u + N : 0], gr);
      const double lam = ((lo_m >> u) & 1ull) ? gr : -gr;
      if (lam < most) { most = lam; worst = u; }
    }
    if (worst < 0) { status = 0u; break; }
    lo_m &= ~(1ull << worst);
    up_m &= ~(1ull << worst);
  }
#pragma unroll
  for (int t = 0; t < M; ++t) {
    uint32_t c = 0u;
#pragma unroll
    for (int j = 0; j < N; ++j) {
      const int v = t * N + j;
      c |= ((((lo_m >> v) & 1ull) ? 1u : 0u) | (((up_m >> v) & 1ull) ? 2u : 0u)) << (2 * j);
    }
    act[t] = c;
  }
  return status;
}

// ------------------------------------------------------------------ S4 plant
// First-order delta-sigma over S sub-steps, period averages (Q22),
// throughput min(dem, thr_max g(l)) (Q18).  Exact arithmetic (no contraction;
// thresholds, levels and capacities from the host tables) so level indices,
// fbar and thr reproduce the oracle bit for bit given u0.  Sub-step loop
// outside (not unrolled: small code), knobs inside (unrolled: ILP across
// knobs).  grid = shared-memory copy of the per-class tables.
template <int N>
__device__ __forceinline__ int level_of(const KnobConst &kc, const GridEntry *tab, double v) {
  // estimate, then one exact correction each way against the thresholds
  int l = __double2int_rd(fma(v - kc.f_min, kc.inv_step, 0.5));
  l = min(max(l, 0), kc.L - 1);
  const double2 mm = __ldg(reinterpret_cast<const double2 *>(&tab[l].mid_lo));
  return l + (v > mm.y ? 1 : 0) - (v <= mm.x ? 1 : 0);
}

// MISS: also count the SLO deadline misses of the period (Q31): sub-steps whose
// level index lies below the SLO level q_slo[phase][j] of the instant.
template <int N, bool MISS = false>
__device__ __forceinline__ void plant_delta_sigma(const DevParams &P, const GridEntry *grid, const double (&u0)[N],
                                                  double (&acc)[N], const double (&dem)[N],
                                                  const double (&thr_max)[N], double (&fbar)[N], double (&thr)[N],
                                                  int phase = 0, int *miss = nullptr) {
  int nm = 0;
  double fs[N], ts[N];
#pragma unroll
  for (int j = 0; j < N; ++j) {
    fs[j] = 0.0;
    ts[j] = 0.0;
  }
#pragma unroll 1
  for (int s = 0; s < P.S; ++s) {
#pragma unroll
    for (int j = 0; j < N; ++j) {
      const KnobConst &kc = P.k[j];
      const GridEntry *tab = grid + kc.cls * kMaxL;
      const double v = __dadd_rn(u0[j], acc[j]);
      const int l = level_of<N>(kc, tab, v);
      if constexpr (MISS) nm += l < P.q_slo[phase][j] ? 1 : 0;
      const double2 lg = __ldg(reinterpret_cast<const double2 *>(&tab[l].level));
      acc[j] = __dadd_rn(v, -lg.x);
      fs[j] = __dadd_rn(fs[j], lg.x);
      const double capj = __dmul_rn(thr_max[j], lg.y);
      ts[j] = __dadd_rn(ts[j], dem[j] < capj ? dem[j] : capj);
    }
  }
#pragma unroll
  for (int j = 0; j < N; ++j) {
    fbar[j] = __dmul_rn(fs[j], P.inv_S);
    thr[j] = __dmul_rn(ts[j], P.inv_S);
  }
  if constexpr (MISS) *miss += nm;
}

// The same plant for a compile-time sub-step count S (the fused kernel's
// common case).  The period's input u_j is constant and |acc_j| <= step_j/2
// (u in [f_min, f_max]), so every sub-step value v = u + acc lies within
// 1.5 steps of the level l_u estimated for u: its level is l_u - 1, l_u or
// l_u + 1, decided by the thresholds mid(l_u - 1) and mid(l_u) exactly as
// level_of decides it.  The three candidate rows are read once per period
// (independent loads) instead of two dependent table reads per sub-step, and
// the capacities min(dem, thr_max g) are formed once per candidate.  Knobs
// outer, sub-steps unrolled: the knobs' serial acc chains interleave.  Same
// arithmetic, same order as plant_delta_sigma (bit-identical results).
template <int N, int S, bool MISS = false>
__device__ __forceinline__ void plant_delta_sigma_c(const DevParams &P, const GridEntry *grid, const double (&u0)[N],
                                                    double (&acc)[N], const double (&dem)[N],
                                                    const double (&thr_max)[N], double (&fbar)[N], double (&thr)[N],
                                                    int phase = 0, int *miss = nullptr) {
  int nm = 0;
#pragma unroll
  for (int j = 0; j < N; ++j) {
    const KnobConst &kc = P.k[j];
    const GridEntry *tab = grid + kc.cls * kMaxL;
    int l = __double2int_rd(fma(u0[j] - kc.f_min, kc.inv_step, 0.5));
    l = min(max(l, 0), kc.L - 1);
    const double2 mm = __ldg(reinterpret_cast<const double2 *>(&tab[l].mid_lo));
    const double2 c0 = __ldg(reinterpret_cast<const double2 *>(&tab[l].level));
    const double2 cl = __ldg(reinterpret_cast<const double2 *>(&tab[l > 0 ? l - 1 : 0].level));
    const double2 ch = __ldg(reinterpret_cast<const double2 *>(&tab[l < kc.L - 1 ? l + 1 : l].level));
    const double d = dem[j], tm = thr_max[j];
    const double k0 = __dmul_rn(tm, c0.y), kl = __dmul_rn(tm, cl.y), kh = __dmul_rn(tm, ch.y);
    const double t0 = d < k0 ? d : k0, tl = d < kl ? d : kl, th = d < kh ? d : kh;
    double a = acc[j], fs = 0.0, ts = 0.0;
    int qj = 0;
    if constexpr (MISS) qj = P.q_slo[phase][j] - l;  // miss <=> l + up - dn < q  <=>  up - dn < q - l
#pragma unroll
    for (int s = 0; s < S; ++s) {
      const double v = __dadd_rn(u0[j], a);
      const bool up = v > mm.y, dn = v <= mm.x;
      const double lev = up ? ch.x : (dn ? cl.x : c0.x);
      const double tt = up ? th : (dn ? tl : t0);
      a = __dadd_rn(v, -lev);
      fs = __dadd_rn(fs, lev);
      ts = __dadd_rn(ts, tt);
      if constexpr (MISS) nm += ((int)up - (int)dn) < qj ? 1 : 0;
    }
    acc[j] = a;
    fbar[j] = __dmul_rn(fs, P.inv_S);
    thr[j] = __dmul_rn(ts, P.inv_S);
  }
  if constexpr (MISS) *miss += nm;
}

// plant_pair: the same delta-sigma plant, bit for bit, with two candidate
// levels per knob and period instead of three.
//
// Why two suffice.  |acc| <= step/2 (+ a few ulps of the host's table
// rounding) after every sub-step, so every sub-step value v = u + acc lies
// within step/2 (+ ulps) of the period's command u.  Let l = floor of u's
// grid position (u - f_min)/step, clamped to [0, L-2]: when u is farther
// than pos_tol steps (1e-9, >> the ulps) from the grid points level(l) and
// level(l+1), no v can reach the thresholds mid(l-1) or mid(l+1), so the
// level index #{mid < v} of the oracle is l + [v > mid(l)] -- one compare,
// one two-way select of the level and of the served throughput per sub-step.
// At the grid ends (l = 0, l + 1 = L-1) there is no outer threshold, so a
// command sitting ON f_min or f_max (a knob at a bound: the common case) is
// still a two-level case.  A command within pos_tol of an interior grid
// point (rare unless an SLO bound is an interior level, which runs
// plant_delta_sigma_c) takes the generic three-way plant for the whole
// instance (out of line).  Same operations in the same order as the oracle
// (v = u + acc, acc = v - level, sums in ascending s): identical bits.
template <int N>
__device__ __noinline__ void plant_generic_ool(const KnobConst *k_dev, int S, double inv_S, const GridEntry *grid,
                                               const double *u0, double *acc, const double *dem,
                                               const double *thr_max, double *fbar, double *thr) {
  for (int j = 0; j < N; ++j) {
    const KnobConst &kc = k_dev[j];
    const GridEntry *tab = grid + kc.cls * kMaxL;
    double a = acc[j], fs = 0.0, ts = 0.0;
    for (int s = 0; s < S; ++s) {
      const double v = __dadd_rn(u0[j], a);
      const int l = level_of<N>(kc, tab, v);
      const double lev = tab[l].level;
      a = __dadd_rn(v, -lev);
      fs = __dadd_rn(fs, lev);
      const double capj = __dmul_rn(thr_max[j], tab[l].g);
      ts = __dadd_rn(ts, dem[j] < capj ? dem[j] : capj);
    }
    acc[j] = a;
    fbar[j] = __dmul_rn(fs, inv_S);
    thr[j] = __dmul_rn(ts, inv_S);
  }
}

// Grid position of u in steps, rounded to the nearest integer without a
// float->int conversion: r = (x + 1.5 2^52) - 1.5 2^52 is rint(x) exactly for
// |x| < 2^51 and the low word of x + 1.5 2^52 is rint(x) as an integer.
struct GridPos {
  int ln;     // rint(x)
  double d;   // x - rint(x) in [-1/2, 1/2]
};
__device__ __forceinline__ GridPos grid_pos(double u, const KnobConst &kc) {
  const double x = (u - kc.f_min) * kc.inv_step;
  const double magic = 6755399441055744.0;
  const double xm = x + magic;
  return GridPos{(int)__double2loint(xm), x - (xm - magic)};
}

// one knob over S sub-steps on the pair (lev0 | lev1 above mid), from acc
template <int S>
__device__ __forceinline__ void pair_substeps(double u, double &acc, double mid, double lev0, double lev1, double t0,
                                              double t1, double inv_S, double &fbar, double &thr) {
  double a = acc, fs, ts;
#pragma unroll
  for (int s = 0; s < S; ++s) {
    const double v = __dadd_rn(u, a);
    const bool up = v > mid;
    const double lev = up ? lev1 : lev0;
    const double tt = up ? t1 : t0;
    a = __dadd_rn(v, -lev);
    // s = 0: 0 + x = x exactly (x >= 0), so the oracle's first add is a copy
    fs = s == 0 ? lev : __dadd_rn(fs, lev);
    ts = s == 0 ? tt : __dadd_rn(ts, tt);
  }
  acc = a;
  fbar = __dmul_rn(fs, inv_S);
  thr = __dmul_rn(ts, inv_S);
}

template <int N, int S>
__device__ __forceinline__ void plant_pair(const DevParams &P, const double (&u0)[N], double (&acc)[N],
                                           const double (&dem)[N], const double (&thr_max)[N], double (&fbar)[N],
                                           double (&thr)[N]) {
  static_assert(S >= 1, "compile-time sub-steps");
  int lidx[N];
  bool exc = false;
#pragma unroll
  for (int j = 0; j < N; ++j) {
    const KnobConst &kc = P.k[j];
    const GridPos g = grid_pos(u0[j], kc);
    exc |= fabs(g.d) < kc.pos_tol && g.ln > 0 && g.ln < kc.L - 1;
    lidx[j] = min(max(g.ln - (g.d < 0.0 ? 1 : 0), 0), kc.L - 2);
  }
  if (exc) {
    double u_l[N], a_l[N], d_l[N], t_l[N], f_o[N], t_o[N];
#pragma unroll
    for (int j = 0; j < N; ++j) {
      u_l[j] = u0[j];
      a_l[j] = acc[j];
      d_l[j] = dem[j];
      t_l[j] = thr_max[j];
    }
    plant_generic_ool<N>(P.k_dev, S, P.inv_S, P.grid, u_l, a_l, d_l, t_l, f_o, t_o);
#pragma unroll
    for (int j = 0; j < N; ++j) {
      acc[j] = a_l[j];
      fbar[j] = f_o[j];
      thr[j] = t_o[j];
    }
    return;
  }
#pragma unroll
  for (int j = 0; j < N; ++j) {
    const KnobConst &kc = P.k[j];
    const PairEntry *e = P.pair + kc.cls * kMaxL + lidx[j];
    const double2 e0 = __ldg(reinterpret_cast<const double2 *>(&e->mid));
    const double2 e1 = __ldg(reinterpret_cast<const double2 *>(&e->lev1));
    const double g1v = __ldg(&e->g1);
    const double d = dem[j], tm = thr_max[j];
    const double k0 = __dmul_rn(tm, e1.y), k1 = __dmul_rn(tm, g1v);
    pair_substeps<S>(u0[j], acc[j], e0.x, e0.y, e1.x, d < k0 ? d : k0, d < k1 ? d : k1, P.inv_S, fbar[j], thr[j]);
  }
}

// Trace of the level indices (traced instances only): replays the same
// delta-sigma from the pre-period accumulators.  Out of line (I-cache).
template <int N>
__device__ __noinline__ void plant_trace_levels(const KnobConst *k_dev, int S, const GridEntry *grid,
                                                const double *u0, const double *acc_in, uint8_t *lv_out,
                                                int64_t lv_stride) {
  for (int j = 0; j < N; ++j) {
    const KnobConst &kc = k_dev[j];
    const GridEntry *tab = grid + kc.cls * kMaxL;
    double ac = acc_in[j];
    for (int s = 0; s < S; ++s) {
      const double v = __dadd_rn(u0[j], ac);
      const int l = level_of<N>(kc, tab, v);
      ac = __dadd_rn(v, -tab[l].level);
      lv_out[(int64_t)(s * N + j) * lv_stride] = (uint8_t)l;
    }
  }
}

}  // namespace capgpu
