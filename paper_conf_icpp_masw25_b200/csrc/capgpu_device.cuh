// capgpu_device.cuh -- per-server device math of the CapGPU step (sm_100a, FP64).
//
// One CUDA thread owns one (server, cap) instance.  All loops over knobs are
// compile-time (template N) and fully unrolled, so the per-server model,
// Hessian factors and QP state live in registers; the symmetric scatter
// Sigma_ff and the read-only per-server constants live in a per-thread
// shared-memory slab (SoA [field][thread], conflict-free 8-byte accesses).
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

// Uniform (per-launch) constants.  Passed by value as the kernel parameter
// (constant bank); the level-capacity table is staged into shared memory.
struct KnobConst {
  double f_min, f_max, step, inv_step;  // grid (Q15)
  double lo, hi, m;                     // box [l, h] (Eq. 10a, Q14) and penalty reference f_min (Q7)
  double r0, inv_r0;                    // r0_j and 1 / r0_j (Q6, Q9)
  int32_t L;                            // levels
  int32_t sweep_base;
};

struct DevParams {
  int32_t N, M, P, S;
  int32_t n_caps;            // instances per server
  int32_t demand_kind;
  double demand_frac;
  double q, theta_min, lam, rho, a_lo, a_hi, a_floor;
  double noise_scale;        // sigma * sqrt(3) (host-computed)
  double inv_S;              // 1/S, exact (S power of two, Q22)
  double ct[kMaxM];          // block weights c_t (Q11)
  double cap_frac0, cap_frac_rand, cap_frac_step, cap_mult;
  int64_t cap_period, cap_lo, cap_hi;
  uint64_t seed;
  int64_t srv_begin;         // global id of local server 0
  int64_t n_srv, n_inst;     // local counts
  KnobConst k[kMaxN];
  double g[kMaxN][kMaxL];    // capacity factor g_j(l) (Q14)
};

// ------------------------------------------------------------------ helpers

__device__ __forceinline__ double rcp_fast(double x) {
  // MUFU.RCP64H seed + two Newton steps: ~1 ulp (continuous quantities only).
  double y;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
  double e = fma(-x, y, 1.0);
  y = fma(y, e, y);
  e = fma(-x, y, 1.0);
  return fma(y, e, y);
}

__device__ __forceinline__ double clampd(double x, double lo, double hi) { return fmin(fmax(x, lo), hi); }

// Exact level arithmetic (Q15): must reproduce the host formulas bit for bit,
// so no FMA contraction here.
__device__ __forceinline__ double level_value(const KnobConst &kc, int l) {
  return __dadd_rn(kc.f_min, __dmul_rn((double)l, kc.step));
}
__device__ __forceinline__ double level_mid(const KnobConst &kc, int l) {
  return __dadd_rn(kc.f_min, __dmul_rn((double)l + 0.5, kc.step));
}
// #{midpoints < v}: estimate from the grid, then one exact correction each way.
__device__ __forceinline__ int level_index(const KnobConst &kc, double v) {
  double x = fma(v - kc.f_min, kc.inv_step, 0.5);
  int l = __double2int_rd(x);
  l = min(max(l, 0), kc.L - 1);
  if (l > 0 && v <= level_mid(kc, l - 1)) --l;
  else if (l < kc.L - 1 && v > level_mid(kc, l)) ++l;
  return l;
}

// ------------------------------------------------------------------ S1 model
// Weighted Welford push (Q1-Q3): w <- lam w + 1, delta = z - mu,
// mu += delta / w, Sigma <- lam Sigma + (1 - 1/w) delta delta^T
// (= delta (z - mu_new)^T in exact arithmetic).
template <int N, class SAcc>
__device__ __forceinline__ void model_push(double lam, double &w, double (&mu_f)[N], double &mu_p,
                                           SAcc S, double (&Sfp)[N], const double (&f)[N], double p) {
  w = fma(lam, w, 1.0);
  const double iw = rcp_fast(w);
  const double e = 1.0 - iw;
  double df[N];
#pragma unroll
  for (int j = 0; j < N; ++j) {
    df[j] = f[j] - mu_f[j];
    mu_f[j] = fma(df[j], iw, mu_f[j]);
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
      S.set(t, fma(lam, S.get(t), ei * df[j]));
    }
    Sfp[i] = fma(lam, Sfp[i], df[i] * edp);
  }
}

// In-register LDL^T solve of a packed SPD system: A (packed upper, destroyed
// into the factors), b -> x.  Used for the model (S1) and identification (S0).
template <int N>
__device__ __forceinline__ void ldlt_solve(double (&L)[Tri<N>::size], const double (&b)[N], double (&x)[N]) {
  double dinv[N];
#pragma unroll
  for (int j = 0; j < N; ++j) {
    double v[N > 1 ? N - 1 : 1];
    double d = L[Tri<N>::idx(j, j)];
#pragma unroll
    for (int k = 0; k < j; ++k) {
      // v_k = L(j,k) D_k with the unit-lower factor L(j,k) of column k
      v[k] = L[Tri<N>::idx(j, k)] * L[Tri<N>::idx(k, k)];
      d = fma(-L[Tri<N>::idx(j, k)], v[k], d);
    }
    L[Tri<N>::idx(j, j)] = d;
    dinv[j] = rcp_fast(d);
#pragma unroll
    for (int i = j + 1; i < N; ++i) {
      double y = L[Tri<N>::idx(i, j)];
#pragma unroll
      for (int k = 0; k < j; ++k) y = fma(-L[Tri<N>::idx(i, k)], v[k], y);
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
    double t = y[i] * dinv[i];
#pragma unroll
    for (int k = i + 1; k < N; ++k) t = fma(-L[Tri<N>::idx(k, i)], x[k], t);
    x[i] = t;
  }
}

// (Sigma_ff + rho I) a = Sigma_fp + rho A0, then clamp to [a_lo A0, a_hi A0] (Q1, Q4).
template <int N, class SAcc, class A0Acc>
__device__ __forceinline__ void model_solve(double rho, double a_lo, double a_hi, SAcc S,
                                            const double (&Sfp)[N], A0Acc A0, double (&ahat)[N]) {
  double L[Tri<N>::size];
#pragma unroll
  for (int t = 0; t < Tri<N>::size; ++t) L[t] = S.get(t);
#pragma unroll
  for (int j = 0; j < N; ++j) L[Tri<N>::idx(j, j)] += rho;
  double b[N];
#pragma unroll
  for (int i = 0; i < N; ++i) b[i] = fma(rho, A0.get(i), Sfp[i]);
  ldlt_solve<N>(L, b, ahat);
#pragma unroll
  for (int j = 0; j < N; ++j) {
    const double a0 = A0.get(j);
    ahat[j] = clampd(ahat[j], a_lo * a0, a_hi * a0);
  }
}

// ------------------------------------------------------------------ S2 weights
// theta = clamp(thr/thr_max, theta_min, 1) with IEEE division (ranks must be
// bit-exact, §8(c.4)); ranks: stable descending (Q10).
template <int N>
__device__ __forceinline__ void weights(double theta_min, const double (&thr)[N], const double (&thr_max)[N],
                                        double (&theta)[N]) {
#pragma unroll
  for (int j = 0; j < N; ++j) theta[j] = clampd(__ddiv_rn(thr[j], thr_max[j]), theta_min, 1.0);
}

template <int N>
__device__ __forceinline__ void ranks(const double (&theta)[N], int8_t (&rk)[N]) {
#pragma unroll
  for (int j = 0; j < N; ++j) {
    int r = 0;
#pragma unroll
    for (int l = 0; l < N; ++l) {
      if (l == j) continue;
      r += (theta[l] > theta[j]) || (l < j && theta[l] == theta[j]);
    }
    rk[j] = (int8_t)r;
  }
}

// ------------------------------------------------------------------ S3 MPC block
// Block t of the decoupled Eq. 9 (Q11):
//   min_{lo<=u<=hi} c (beta + a.u)^2 + sum_j R_j (u_j - m_j)^2
// KKT: u_j(s) = clamp(m_j - c tau_j s, lo_j, hi_j), tau_j = a_j / R_j, and
// s = beta + a.u(s).  phi(s) = s - beta - a.u(s) is strictly increasing and
// piecewise linear (slope >= 1, breakpoints where a knob meets a bound), so
// the root is unique and is the exact root of the linear piece it lies on.
//   phase 1: up to 3 Newton steps on phi from the warm-start active set (the
//            previous period's); ends when a Newton point reproduces its own
//            active set (then it is the exact root).
//   phase 2: otherwise the root's active set is read off phi at each knob's
//            two breakpoints (<= 2N evaluations, no sorting) and the root of
//            that piece is exact.  Bounded work, no iteration cap to hit.

// root of the linear piece with active codes `code`
template <int N>
__device__ __forceinline__ double piece_root(const KnobConst *kc, const double (&a)[N], const double (&ctau)[N],
                                             double beta, uint32_t code) {
  double num = beta, den = 1.0;
#pragma unroll
  for (int j = 0; j < N; ++j) {
    const uint32_t cj = (code >> (2 * j)) & 3u;
    const double x = cj == 0u ? kc[j].m : (cj == 1u ? kc[j].lo : kc[j].hi);
    num = fma(a[j], x, num);
    den = cj == 0u ? fma(ctau[j], a[j], den) : den;
  }
  return num * rcp_fast(den);
}

// active codes and phi at s
template <int N>
__device__ __forceinline__ uint32_t eval_phi(const KnobConst *kc, const double (&a)[N], const double (&ctau)[N],
                                             double beta, double s, double &phi) {
  uint32_t nc = 0u;
  double f = s - beta;
#pragma unroll
  for (int j = 0; j < N; ++j) {
    const double v = fma(-ctau[j], s, kc[j].m);
    const uint32_t cj = v < kc[j].lo ? 1u : (v > kc[j].hi ? 2u : 0u);
    nc |= cj << (2 * j);
    f = fma(-a[j], clampd(v, kc[j].lo, kc[j].hi), f);
  }
  phi = f;
  return nc;
}

template <int N>
__device__ __forceinline__ uint32_t solve_block(const KnobConst *kc, const double (&a)[N],
                                                const double (&tau)[N], double c, double beta,
                                                uint32_t code, double (&u)[N], bool &capped) {
  double ctau[N];
#pragma unroll
  for (int j = 0; j < N; ++j) ctau[j] = c * tau[j];
  double s = 0.0;
  bool done = false;
  // phase 1: a few Newton steps from the warm start (the common case ends in
  // the first: last period's active set is still right).
  constexpr int kNewton = 3;
#pragma unroll 1
  for (int it = 0; it < kNewton; ++it) {
    s = piece_root<N>(kc, a, ctau, beta, code);
    double phi;
    const uint32_t nc = eval_phi<N>(kc, a, ctau, beta, s, phi);
    if (nc == code || phi == 0.0) { done = true; break; }
    code = nc;
  }
  if (!done) {
    // phase 2: the active set of the root read off phi at each knob's own
    // breakpoints (phi increasing: s* > b  <=>  phi(b) < 0), no sorting:
    //   lower  iff s* > b_l = (m - lo)/(c tau),  upper iff s* < b_h = (m - hi)/(c tau).
    code = 0u;
#pragma unroll
    for (int j = 0; j < N; ++j) {
      uint32_t cj;
      if (!(ctau[j] > 0.0)) {
        cj = kc[j].m < kc[j].lo ? 1u : (kc[j].m > kc[j].hi ? 2u : 0u);
      } else {
        const double r = rcp_fast(ctau[j]);
        double fb;
        eval_phi<N>(kc, a, ctau, beta, (kc[j].m - kc[j].lo) * r, fb);
        if (fb < 0.0) {
          cj = 1u;
        } else {
          eval_phi<N>(kc, a, ctau, beta, (kc[j].m - kc[j].hi) * r, fb);
          cj = fb > 0.0 ? 2u : 0u;
        }
      }
      code |= cj << (2 * j);
    }
    s = piece_root<N>(kc, a, ctau, beta, code);
    // consistency: the classification at s must reproduce `code` (exact root);
    // a mismatch can only come from a rounding-level tie and is reported.
    double phi;
    if (eval_phi<N>(kc, a, ctau, beta, s, phi) != code && fabs(phi) > 1e-9 * (1.0 + fabs(beta))) capped = true;
  }
  uint32_t out = 0u;
#pragma unroll
  for (int j = 0; j < N; ++j) {
    const double v = fma(-ctau[j], s, kc[j].m);
    const uint32_t cj = v < kc[j].lo ? 1u : (v > kc[j].hi ? 2u : 0u);
    out |= cj << (2 * j);
    u[j] = clampd(v, kc[j].lo, kc[j].hi);
  }
  return out;
}

// ------------------------------------------------------------------ S4 plant
// First-order delta-sigma over S sub-steps, period averages (Q22),
// throughput min(dem, thr_max g(l)) (Q18).  Exact arithmetic (no contraction)
// so level indices, fbar and thr reproduce the oracle bit for bit given u0.
template <int N>
__device__ __forceinline__ void plant_delta_sigma(const DevParams &P, const double *sg /* smem [N][kMaxL] */,
                                                  const double (&u0)[N], double (&acc)[N],
                                                  const double (&dem)[N], const double (&thr_max)[N],
                                                  double (&fbar)[N], double (&thr)[N], uint8_t *lv_out,
                                                  int lv_stride) {
#pragma unroll
  for (int j = 0; j < N; ++j) {
    const KnobConst &kc = P.k[j];
    double fs = 0.0, ts = 0.0, ac = acc[j];
    for (int s = 0; s < P.S; ++s) {
      const double v = __dadd_rn(u0[j], ac);
      const int l = level_index(kc, v);
      const double lv = level_value(kc, l);
      ac = __dadd_rn(v, -lv);
      fs = __dadd_rn(fs, lv);
      ts = __dadd_rn(ts, fmin(dem[j], __dmul_rn(thr_max[j], sg[j * kMaxL + l])));
      if (lv_out) lv_out[(s * N + j) * lv_stride] = (uint8_t)l;
    }
    acc[j] = ac;
    fbar[j] = __dmul_rn(fs, P.inv_S);
    thr[j] = __dmul_rn(ts, P.inv_S);
  }
}

}  // namespace capgpu
