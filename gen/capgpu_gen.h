/*
 * capgpu_gen.h -- seeded synthetic-input generator for the CapGPU hot path.
 *
 * This module is the ONE piece of code shared by the CPU oracle (oracle/) and
 * the CUDA path (paper_conf_icpp_masw25_b200/csrc/).  It holds NO method
 * arithmetic (no model update, no weights, no MPC, no plant): only a
 * counter-based hash and the workload recipe of DESIGN.md §3 (per-server
 * parameters, demand traces, meter noise, cap schedules).  Every value it
 * produces is bit-identical on host and device:
 *   - integer splitmix64 arithmetic is exact;
 *   - uniforms are built by bit assembly (exact);
 *   - the few floating-point ops use explicit round-to-nearest intrinsics on the
 *     device (__dadd_rn / __dmul_rn / __fma_rn, never contracted) and plain
 *     operators / C99 fma() on the host, which must be compiled with
 *     -ffp-contract=off (fma() is correctly rounded: identical to __fma_rn).
 *
 * Per-period draws (demand jitter of every knob and the meter noise of one
 * server and period) come from ONE splitmix64 finaliser of the (stream,
 * period) key, expanded by a 64-bit LCG: state 1 and 2 give the four noise
 * uniforms, state 2 + q the jitter of knobs 2q and 2q + 1 (26-bit halves).
 * (Round 1 hashed every draw separately: ~2.5x the integer work per period.)
 *
 * Recipe citations (PAPER.md line numbers, "P:NNN"):
 *   - gains / offset of the linear power model p = A F + C: P:156-167 (Eq. 3-4)
 *   - meter noise / 4 s period averaged over 1 s samples: P:238
 *   - normalised throughput vs device maximum: P:93
 *   - bursty inference demand (Fig. 10 surge), SURVEY §8(d.2)
 *   - cap schedules: fixed, step 800->900->800 W (Fig. 10),
 *     set-point sweep (Fig. 6)
 */
#ifndef CAPGPU_GEN_H
#define CAPGPU_GEN_H

#include <stdint.h>
#ifndef __CUDACC__
#include <string.h>
#endif

#if defined(__CUDACC__)
#define GEN_HD __host__ __device__ __forceinline__
#else
#define GEN_HD static inline
#endif

#if defined(__CUDA_ARCH__)
#define GEN_ADD(a, b) __dadd_rn((a), (b))
#define GEN_MUL(a, b) __dmul_rn((a), (b))
#define GEN_FMA(a, b, c) __fma_rn((a), (b), (c))
#else
#include <math.h>
#define GEN_ADD(a, b) ((a) + (b))
#define GEN_MUL(a, b) ((a) * (b))
#define GEN_FMA(a, b, c) fma((a), (b), (c))
#endif

#define GEN_MAX_KNOBS 16

/* stream tags */
enum {
  GEN_TAG_PARAM = 1, /* per-server constants */
  GEN_TAG_JIT = 2,   /* per-period draws: demand jitter AND meter noise of period k */
  GEN_TAG_BURST = 3, /* demand bursts, held for GEN_BURST_HOLD periods */
  GEN_TAG_NOISE = 4, /* (unused since the per-period draws share GEN_TAG_JIT) */
  GEN_TAG_SWEEP = 5, /* meter noise of identification sweep row r */
};

/* parameter field indices for GEN_TAG_PARAM samples */
enum {
  GEN_F_A = 0,        /* + knob j : true gain a_j            */
  GEN_F_THRMAX = 16,  /* + knob j : device max throughput    */
  GEN_F_BASE = 32,    /* + knob j : demand base level        */
  GEN_F_AMP = 48,     /* + knob j : demand burst amplitude   */
  GEN_F_C = 64,       /* true constant offset C              */
  GEN_F_CAPU = 65,    /* per-server random cap fraction      */
};

#define GEN_BURST_HOLD 10

/* splitmix64 finaliser (Steele, Lea, Flood 2014) */
GEN_HD uint64_t gen_mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

/* Key of one (seed, tag, server) stream.  Fully mixed. */
GEN_HD uint64_t gen_stream_key(uint64_t seed, uint32_t tag, uint64_t server) {
  uint64_t s = gen_mix64(seed ^ ((uint64_t)tag * 0xD1B54A32D192ED03ULL));
  return gen_mix64(s + server * 0x9E3779B97F4A7C15ULL);
}

/* Sample (a, b) of a stream: a = small field/knob/slot index, b = period/row. */
GEN_HD uint64_t gen_sample(uint64_t key, uint64_t a, uint64_t b) {
  return gen_mix64(key + a * 0xC2B2AE3D27D4EB4FULL + b * 0xD6E8FEB86659FD93ULL);
}

GEN_HD double gen_bits_to_double(uint64_t b) {
#if defined(__CUDA_ARCH__)
  return __longlong_as_double((long long)b);
#else
  double d;
  memcpy(&d, &b, sizeof d);
  return d;
#endif
}

/* U52: uniform on [0,1) with 52 random bits, exact: (h >> 12) * 2^-52 */
GEN_HD double gen_u52(uint64_t h) {
  return gen_bits_to_double(0x3FF0000000000000ULL | (h >> 12)) - 1.0;
}

/* two 26-bit uniforms of one 64-bit word as doubles in [1, 2), exact:
 * 1 + x * 2^-26 (bits 63..38 and 37..12) */
GEN_HD double gen_v26_hi(uint64_t h) {
  return gen_bits_to_double(0x3FF0000000000000ULL | ((h >> 38) << 26));
}
GEN_HD double gen_v26_lo(uint64_t h) {
  return gen_bits_to_double(0x3FF0000000000000ULL | (((h >> 12) & 0x3FFFFFFULL) << 26));
}

/* ---------------------------------------------------------------- per-period draws */

/* seed of the draws of period (or sweep row) b of a stream */
GEN_HD uint64_t gen_period_seed(uint64_t key, int64_t b) {
  return gen_mix64(key + (uint64_t)b * 0xD6E8FEB86659FD93ULL);
}
/* 64-bit LCG step (Knuth's MMIX multiplier and increment) */
GEN_HD uint64_t gen_lcg(uint64_t x) { return x * 6364136223846793005ULL + 1442695040888963407ULL; }

/* Irwin-Hall-4 noise from the period seed h: states 1 and 2 of the LCG give
 * four 26-bit uniforms V_t in [1, 2); n = scale * (sum_t V_t - 6), i.e.
 * scale * (U0 + U1 + U2 + U3 - 2) with U_t = V_t - 1 (mean 0, variance
 * scale^2 / 3: scale = sigma sqrt(3)).  Sums in a fixed order. */
GEN_HD double gen_noise_h(uint64_t h, double scale) {
  const uint64_t s1 = gen_lcg(h), s2 = gen_lcg(s1);
  const double a = GEN_ADD(gen_v26_hi(s1), gen_v26_lo(s1));
  const double b = GEN_ADD(gen_v26_hi(s2), gen_v26_lo(s2));
  return GEN_MUL(scale, GEN_ADD(GEN_ADD(a, b), -6.0));
}

/* jitter word of knob pair q (knobs 2q, 2q+1) from the period seed: LCG state 3 + q */
GEN_HD uint64_t gen_jit_word(uint64_t h, int q) {
  uint64_t s = gen_lcg(gen_lcg(h));
  for (int t = 0; t <= q; ++t) s = gen_lcg(s);
  return s;
}
/* jitter uniform of knob j in [1, 2) from its pair's word */
GEN_HD double gen_jit_v(uint64_t w, int j) { return (j & 1) ? gen_v26_lo(w) : gen_v26_hi(w); }

/* ---------------------------------------------------------------- params */

/* one U52 of the per-server parameter stream */
GEN_HD double gen_param_u(uint64_t seed, uint64_t server, int field) {
  return gen_u52(gen_sample(gen_stream_key(seed, GEN_TAG_PARAM, server), (uint64_t)field, 0));
}

/* true gain of knob j (W/MHz): CPU 0.03+0.05U, GPU 0.15+0.10U */
GEN_HD double gen_a_true(uint64_t seed, uint64_t server, int j) {
  double u = gen_param_u(seed, server, GEN_F_A + j);
  return j == 0 ? GEN_ADD(0.03, GEN_MUL(0.05, u)) : GEN_ADD(0.15, GEN_MUL(0.10, u));
}
/* true offset C (W): 250 + 100U */
GEN_HD double gen_c_true(uint64_t seed, uint64_t server) {
  return GEN_ADD(250.0, GEN_MUL(100.0, gen_param_u(seed, server, GEN_F_C)));
}
/* device maximum throughput: CPU 50+100U, GPU 40+160U (units irrelevant) */
GEN_HD double gen_thr_max(uint64_t seed, uint64_t server, int j) {
  double u = gen_param_u(seed, server, GEN_F_THRMAX + j);
  return j == 0 ? GEN_ADD(50.0, GEN_MUL(100.0, u)) : GEN_ADD(40.0, GEN_MUL(160.0, u));
}
/* demand base level (fraction of thr_max): 0.2 + 0.7U */
GEN_HD double gen_dem_base(uint64_t seed, uint64_t server, int j) {
  return GEN_ADD(0.2, GEN_MUL(0.7, gen_param_u(seed, server, GEN_F_BASE + j)));
}
/* demand burst amplitude (fraction of thr_max): 0.2 + 0.4U */
GEN_HD double gen_dem_amp(uint64_t seed, uint64_t server, int j) {
  return GEN_ADD(0.2, GEN_MUL(0.4, gen_param_u(seed, server, GEN_F_AMP + j)));
}

/* ---------------------------------------------------------------- demand */

/* Bursty demand of knob j in period k:
 *   dem = thr_max * clamp(base + amp*[U_burst(k/10) < 0.2] + 0.05*(2U_jit(k) - 1), 0, 1.5)
 * key_jit / key_burst = gen_stream_key(seed, GEN_TAG_JIT / GEN_TAG_BURST, server). */
/* burst flags of burst epoch e = floor(k / GEN_BURST_HOLD): one seed per
 * epoch, LCG state j + 1 for knob j, flag iff its high 32 bits < 2^32 / 5
 * (probability 0.2) */
GEN_HD int gen_burst_flag(uint64_t key_burst, int j, int64_t epoch) {
  uint64_t s = gen_period_seed(key_burst, epoch);
  for (int t = 0; t <= j; ++t) s = gen_lcg(s);
  return (uint32_t)(s >> 32) < 858993460u;
}

/* demand from the jitter uniform v in [1, 2) and the burst flag:
 *   thr_max * min(base + amp*burst + (0.1 v - 0.15), 1.5)
 * (jitter 0.05 (2U - 1) with U = v - 1, one correctly rounded fma; the lower
 * clamp at 0 of the recipe never binds: base >= 0.2 > 0.05) */
GEN_HD double gen_demand_u(double v, int burst, double thr_max, double base, double amp) {
  double x = burst ? GEN_ADD(base, amp) : base;
  double y = GEN_ADD(x, GEN_FMA(0.1, v, -0.15));
  y = y > 1.5 ? 1.5 : y;
  return GEN_MUL(thr_max, y);
}

/* demand given the burst flag of the period's epoch */
GEN_HD double gen_demand_flag(uint64_t key_jit, int j, int64_t k, int burst, double thr_max,
                              double base, double amp) {
  const uint64_t w = gen_jit_word(gen_period_seed(key_jit, k), j >> 1);
  return gen_demand_u(gen_jit_v(w, j), burst, thr_max, base, amp);
}

GEN_HD double gen_demand_bursty(uint64_t key_jit, uint64_t key_burst, int j, int64_t k,
                                double thr_max, double base, double amp) {
  return gen_demand_flag(key_jit, j, k, gen_burst_flag(key_burst, j, k / GEN_BURST_HOLD), thr_max,
                         base, amp);
}

/* Constant demand: dem = thr_max * frac */
GEN_HD double gen_demand_const(double thr_max, double frac) { return GEN_MUL(thr_max, frac); }

/* ---------------------------------------------------------------- noise */

/* Irwin-Hall-4 meter noise with standard deviation sigma (scale = sigma*sqrt(3),
 * computed once on the host) of slot b of a stream: the period k of the
 * GEN_TAG_JIT stream (shared with the demand jitter of period k) or the row r
 * of the identification sweep stream (GEN_TAG_SWEEP). */
GEN_HD double gen_noise(uint64_t key, int64_t b, double scale) {
  return gen_noise_h(gen_period_seed(key, b), scale);
}

/* ---------------------------------------------------------------- caps */

/* P_min / P_max of a server from its true model: C + sum_j a_j f_j, j ascending */
GEN_HD double gen_power_at(double c_true, const double *a_true, const double *f, int n) {
  double p = c_true;
  for (int j = 0; j < n; ++j) p = GEN_ADD(p, GEN_MUL(a_true[j], f[j]));
  return p;
}

/* Cap fraction of instance (server, cap index c):
 *   frac = (frac0 + frac_rand*U_capu) + frac_step*(c + 0.5)
 * cfg1: 0.6/0/0; cfg2: 0.45/0/0; cfg3: 0.3/0.5/0; cfg5: 0/0/(1/32). */
GEN_HD double gen_cap_frac(uint64_t seed, uint64_t server, int c, double frac0, double frac_rand,
                           double frac_step) {
  double f = frac0;
  if (frac_rand != 0.0) f = GEN_ADD(f, GEN_MUL(frac_rand, gen_param_u(seed, server, GEN_F_CAPU)));
  if (frac_step != 0.0) f = GEN_ADD(f, GEN_MUL(frac_step, GEN_ADD((double)c, 0.5)));
  return f;
}

/* base cap = P_min + frac * (P_max - P_min) */
GEN_HD double gen_cap_base(double pmin, double pmax, double frac) {
  return GEN_ADD(pmin, GEN_MUL(frac, GEN_ADD(pmax, -pmin)));
}

/* Step schedule (Fig. 10 analogue): cap(k) = base * (k mod period in
 * [lo, hi) ? mult : 1).  period <= 0 disables the schedule. */
GEN_HD double gen_cap_at(double base, int64_t k, int64_t period, int64_t lo, int64_t hi, double mult) {
  if (period > 0) {
    int64_t r = k % period;
    if (r >= lo && r < hi) return GEN_MUL(base, mult);
  }
  return base;
}

/* ---------------------------------------------------------------- sweep */

/* Identification sweep design: row r enumerates knob-major
 * (knob j over all its levels l = 0..L_j-1 while the others sit at their base
 * level).  Returns the knob varied in row r and writes its level index. */
GEN_HD int gen_sweep_row(const int *n_levels, int n, int r, int *level_out) {
  for (int j = 0; j < n; ++j) {
    if (r < n_levels[j]) { *level_out = r; return j; }
    r -= n_levels[j];
  }
  *level_out = -1;
  return -1;
}

#endif /* CAPGPU_GEN_H */
