// capgpu_lanes.cuh -- lane-parallel fused kernel for SMALL batches (sm_100a).
//
// k_simulate runs one instance per thread: with few instances (cfg 1: 1
// server, cfg 2: 1,024 servers on 148 SMs) each warp is alone on its
// scheduler and the period time is one thread's dependency chain over all N
// knobs.  k_simulate_lp gives each instance a group of G >= N lanes, lane j
// owning knob j: the knob-parallel parts of the period -- the S4 plant and
// its demand draw, the S1 Welford row updates, the S2 weights, the block-0
// frequency -- run one knob per lane; the parts that couple the knobs (the
// LDL^T solve, the convex block root, the sums) run redundantly in every lane
// of the group on the gathered per-knob values, IN THE SAME OPERATION ORDER as
// k_simulate, so the two kernels give bitwise identical results (the shard
// invariance tests compare them).  Gathers go through a per-instance
// shared-memory exchange row; the model state Sigma' lives in a per-instance
// shared-memory slab.  Scope: the convex MPC path (no SLO schedule, no move
// suppression, no reference trajectory), S = 4 sub-steps; other workloads use
// k_simulate.  Citations as in capgpu_device.cuh.
#pragma once

#include "capgpu_device.cuh"

namespace capgpu {

// one knob of plant_pair (identical arithmetic; the three-way generic plant
// for this knob when its command sits on an interior grid point)
template <int S>
__device__ __noinline__ void plant_knob_generic_ool(const KnobConst *kc, double inv_S, const GridEntry *grid, double u,
                                                    double *acc, double dem, double tm, double *fbar, double *thr) {
  const GridEntry *tab = grid + kc->cls * kMaxL;
  double a = *acc, fs = 0.0, ts = 0.0;
  for (int s = 0; s < S; ++s) {
    const double v = __dadd_rn(u, a);
    int l = __double2int_rd(fma(v - kc->f_min, kc->inv_step, 0.5));
    l = min(max(l, 0), kc->L - 1);
    l = l + (v > tab[l].mid_hi ? 1 : 0) - (v <= tab[l].mid_lo ? 1 : 0);
    const double lev = tab[l].level;
    a = __dadd_rn(v, -lev);
    fs = __dadd_rn(fs, lev);
    const double capj = __dmul_rn(tm, tab[l].g);
    ts = __dadd_rn(ts, dem < capj ? dem : capj);
  }
  *acc = a;
  *fbar = __dmul_rn(fs, inv_S);
  *thr = __dmul_rn(ts, inv_S);
}

template <int S>
__device__ __forceinline__ void plant_knob(const DevParams &P, const KnobConst &kc, double u, double &acc, double dem,
                                           double tm, double &fbar, double &thr) {
  const GridPos g = grid_pos(u, kc);
  const bool exc = fabs(g.d) < kc.pos_tol && g.ln > 0 && g.ln < kc.L - 1;
  if (exc) {
    double a = acc, f, t;
    plant_knob_generic_ool<S>(&kc, P.inv_S, P.grid, u, &a, dem, tm, &f, &t);
    acc = a;
    fbar = f;
    thr = t;
    return;
  }
  const int l = min(max(g.ln - (g.d < 0.0 ? 1 : 0), 0), kc.L - 2);
  const PairEntry *e = P.pair + kc.cls * kMaxL + l;
  const double2 e0 = __ldg(reinterpret_cast<const double2 *>(&e->mid));
  const double2 e1 = __ldg(reinterpret_cast<const double2 *>(&e->lev1));
  const double g1v = __ldg(&e->g1);
  const double k0 = __dmul_rn(tm, e1.y), k1 = __dmul_rn(tm, g1v);
  pair_substeps<S>(u, acc, e0.x, e0.y, e1.x, dem < k0 ? dem : k0, dem < k1 ? dem : k1, P.inv_S, fbar, thr);
}

// gather the group's per-knob values v (lane j = knob j) into out[N]:
// warp shuffles within the G-lane segment (every lane of the warp calls it)
template <int N, int G>
__device__ __forceinline__ void lp_gather(double v, double (&out)[N]) {
#pragma unroll
  for (int j = 0; j < N; ++j) out[j] = __shfl_sync(0xffffffffu, v, j, G);
}

template <int N, int M, int S, int G>
__global__ void __launch_bounds__(128) k_simulate_lp(DevParams P, StatePtrs st, TracePtrs tr, int64_t k0call, int Ktot) {
  static_assert(G >= N && G <= 32 && (G & (G - 1)) == 0, "one knob per lane");
  constexpr int T = Tri<N>::size;
  const int gl = threadIdx.x & (G - 1);
  const int64_t iraw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) / G;
  const bool ivalid = iraw < P.n_inst;
  const int64_t i = ivalid ? iraw : P.n_inst - 1;  // surplus groups shadow the last instance, write nothing
  const bool own = gl < N;
  const int j = own ? gl : 0;  // idle lanes shadow knob 0 and write nothing
  const KnobConst kc = P.k_dev[j];
  const int64_t si = i / P.n_caps, ls = P.n_srv, li = P.n_inst;
  const uint64_t srv = (uint64_t)(P.srv_begin + si);
  const double gain = plant_gain(P, (int)(i - si * P.n_caps));
  // jitter word of this lane's knob pair: LCG state 3 + j/2 of the period seed
  uint64_t jump_a = 1ull, jump_c = 0ull;
  for (int t = 0; t < 3 + (j >> 1); ++t) {
    jump_a = jump_a * 6364136223846793005ULL;
    jump_c = jump_c * 6364136223846793005ULL + 1442695040888963407ULL;
  }

  // ---- stage in: the model (w, mu, Sigma') redundantly in every lane of the
  // group, the plant state and constants of the lane's own knob
  double fb = __ldcg(st.fbar + j * li + i), ac = __ldcg(st.acc + j * li + i), th_r = __ldcg(st.thr + j * li + i);
  const double tm = st.thr_max[j * ls + si], bas = st.base[j * ls + si], amp = st.amp[j * ls + si];
  double Sg[T], muf[N], sfp[N], A0a[N], ATa[N], fba[N];
#pragma unroll
  for (int t = 0; t < T; ++t) Sg[t] = __ldcg(st.S + t * li + i);
#pragma unroll
  for (int q = 0; q < N; ++q) {
    muf[q] = __ldcg(st.mu_f + q * li + i);
    sfp[q] = __ldcg(st.Sfp + q * li + i);
    A0a[q] = st.A0[q * ls + si];
    ATa[q] = __dmul_rn(gain, st.a_true[q * ls + si]);
  }
  lp_gather<N, G>(fb, fba);
  double p = __ldcg(st.p + i), w = __ldcg(st.w + i), mu_p = __ldcg(st.mu_p + i);
  const double c_true = st.c_true[si], cap_base = st.cap_base[i];
  double s_prev[M];
  uint32_t act[M];
#pragma unroll
  for (int t = 0; t < M; ++t) {
    s_prev[t] = __ldcg(st.s_prev + t * li + i);
    act[t] = __ldcg(st.act + t * li + i);
  }
  const int slot = tr.n_trace > 0 ? st.trace_slot[i] : -1;
  const uint64_t kjit = gen_stream_key(P.seed, GEN_TAG_JIT, srv);
  const uint64_t kburst = gen_stream_key(P.seed, GEN_TAG_BURST, srv);
  int64_t epoch = (k0call + 1) / GEN_BURST_HOLD;
  int left = (int)(GEN_BURST_HOLD - (k0call + 1) % GEN_BURST_HOLD);
  uint32_t bmask = 0u;
  if (P.demand_kind != 0) {
    uint64_t sb = gen_period_seed(kburst, epoch);
#pragma unroll
    for (int q = 0; q < N; ++q) {
      sb = gen_lcg(sb);
      bmask |= ((uint32_t)(sb >> 32) < 858993460u ? 1u : 0u) << q;
    }
  }
  const int kw = (int)(Ktot - (4 * (int64_t)Ktot) / 5);
  double sum_p = 0.0, sumsq_p = 0.0, max_p = 0.0, sum_theta = 0.0;
  int n_viol = 0, act_cnt[M];
#pragma unroll
  for (int t = 0; t < M; ++t) act_cnt[t] = 0;
  double inv_lam_k = 1.0;

  CapSched csch(P, k0call);
#pragma unroll 1
  for (int kk = 0; kk < Ktot; ++kk) {
    const int64_t k = k0call + kk;
    const double cap = csch.cap(P, cap_base);
    csch.next(P);
    // ---- S4's draws first (burst epoch, demand and meter noise of period
    // k + 1): they depend only on the seeds, so their integer hash chain
    // overlaps the FP64 chain of S1-S3 below instead of following it
    if (left == 0) {
      ++epoch;
      left = GEN_BURST_HOLD;
      bmask = 0u;
      if (P.demand_kind != 0) {
        uint64_t sb = gen_period_seed(kburst, epoch);
#pragma unroll
        for (int q = 0; q < N; ++q) {
          sb = gen_lcg(sb);
          bmask |= ((uint32_t)(sb >> 32) < 858993460u ? 1u : 0u) << q;
        }
      }
    }
    --left;
    const uint64_t hper = gen_period_seed(kjit, k + 1);
    const double dem = P.demand_kind == 0
                           ? gen_demand_const(tm, P.demand_frac)
                           : gen_demand_u(gen_jit_v(hper * jump_a + jump_c, j), (bmask >> j) & 1u, tm, bas, amp);
    const double noise = gen_noise_h(hper, P.noise_scale);
    if ((kk & P.fold_mask) == P.fold_mask) {  // fold lam^-kk back into Sigma' (as slab_rescale)
      const double f = rcp_fast(inv_lam_k);
#pragma unroll
      for (int t = 0; t < T; ++t) Sg[t] *= f;
#pragma unroll
      for (int q = 0; q < N; ++q) sfp[q] *= f;
      inv_lam_k = 1.0;
    }
    inv_lam_k *= P.inv_lam;
    // ---- S1 (model_push SCALED + model_solve), redundant in every lane
    double ahat[N];
    {
      w = fma(P.lam, w, 1.0);
      const double iw = rcp_fast(w);
      const double e = (1.0 - iw) * inv_lam_k;
      double df[N];
#pragma unroll
      for (int q = 0; q < N; ++q) {
        const double m = muf[q];
        df[q] = fba[q] - m;
        muf[q] = fma(df[q], iw, m);
      }
      const double dp = p - mu_p;
      mu_p = fma(dp, iw, mu_p);
      const double edp = e * dp;
#pragma unroll
      for (int a = 0; a < N; ++a) {
        const double ea = e * df[a];
#pragma unroll
        for (int b = a; b < N; ++b) Sg[Tri<N>::idx(a, b)] = fma(ea, df[b], Sg[Tri<N>::idx(a, b)]);
        sfp[a] = fma(df[a], edp, sfp[a]);
      }
      const double rho = P.rho * inv_lam_k;
      double L[T], bb[N];
#pragma unroll
      for (int t = 0; t < T; ++t) L[t] = Sg[t];
#pragma unroll
      for (int q = 0; q < N; ++q) L[Tri<N>::idx(q, q)] += rho;
#pragma unroll
      for (int q = 0; q < N; ++q) bb[q] = fma(rho, A0a[q], sfp[q]);
      ldlt_solve<N>(L, bb, ahat);
#pragma unroll
      for (int q = 0; q < N; ++q) ahat[q] = pclamp(ahat[q], P.a_lo * A0a[q], P.a_hi * A0a[q]);
    }
    // ---- S2 (own knob), then the gathered weights
    const double thj = pclamp(th_r * rcp_nr1(tm), P.theta_min, 1.0);
    const double tauj = ahat[j] * thj * kc.inv_r0;
    double tha[N], tau[N];
    lp_gather<N, G>(thj, tha);
    lp_gather<N, G>(tauj, tau);
    double tsum0 = 0.0, tsum1 = 0.0;
#pragma unroll
    for (int q = 0; q < N; ++q) {
      if (q & 1) tsum1 += tha[q]; else tsum0 += tha[q];
    }
    const double tbar = (tsum0 + tsum1) * P.inv_N;
    // ---- S3 convex path (control_instant), redundant
    double beta = p - cap;
#pragma unroll
    for (int q = 0; q < N; ++q) beta = fma(-ahat[q], fba[q], beta);
    double smin = 0.0, smax = 0.0;
#pragma unroll
    for (int q = 0; q < N; ++q) {
      smin = fma(ahat[q], P.k[q].lo, smin);
      smax = fma(ahat[q], P.k[q].hi, smax);
    }
    const uint32_t status = (beta + smin > 0.0 || beta + smax < 0.0) ? (uint32_t)CAPGPU_ST_CAP_INFEASIBLE : 0u;
    const double base = beta + smin;
    const bool full = slot >= 0;
    double s[M];
    if (!(base < 0.0)) {
      uint32_t c = 0u;
#pragma unroll
      for (int q = 0; q < N; ++q) c |= (base > 0.0 && tau[q] > 0.0 ? 1u : 0u) << (2 * q);
#pragma unroll
      for (int t = 0; t < M; ++t) {
        s[t] = base;
        act[t] = c;
      }
    } else {
      double ta[N], ad[N], TA0 = 0.0, TA1 = 0.0;
#pragma unroll
      for (int q = 0; q < N; ++q) {
        ta[q] = tau[q] * ahat[q];
        ad[q] = ahat[q] * P.k[q].span;
        if (q & 1) TA1 += ta[q]; else TA0 += ta[q];
      }
      const double TA = TA0 + TA1;
      const bool any_last = M > 1 && !full ? convex_any_upper<N>(P.k, P.ct[M - 1], tau, base, TA) : false;
      uint32_t up0 = act[0] & 0xAAAAAAAAu;
      const double s0 = convex_root<N>(P.k, P.ct[0], tau, ta, ad, base, TA, up0);
#pragma unroll
      for (int t = 0; t + 1 < M; ++t) {
        s[t] = s0;
        act[t] = up0;
      }
      if (M == 1) {
        s[0] = s0;
        act[0] = up0;
      } else if (full) {
        uint32_t upl = act[M - 1] & 0xAAAAAAAAu;
        s[M - 1] = convex_root<N>(P.k, P.ct[M - 1], tau, ta, ad, base, TA, upl);
        act[M - 1] = upl;
      } else {
        s[M - 1] = s0;
        act[M - 1] = any_last ? 2u : 0u;
      }
    }
#pragma unroll
    for (int t = 0; t < M; ++t) s_prev[t] = s[t];
    double u0j;
    {
      const double mcs = -P.ct[0] * s[0];
      uint32_t code = 0u;
#pragma unroll
      for (int q = 0; q < N; ++q) {
        const double v = fma(mcs, tau[q], P.k[q].m);
        code |= (v > P.k[q].hi ? 2u : 0u) << (2 * q);
      }
      const double v = fma(mcs, tau[j], kc.m);
      u0j = base < 0.0 ? (v > kc.hi ? kc.hi : v) : kc.lo;
      if (base < 0.0) act[0] = code;
    }
    // ---- traced outputs (as control_instant's InstantOut + sim_run's rows)
    if (slot >= 0) {
      const double thi = pclamp(__ddiv_rn(th_r, tm), P.theta_min, 1.0);  // IEEE weights (weights<N>)
      double thv[N];
      lp_gather<N, G>(thi, thv);
      if (ivalid) {
        const int64_t n_tr = tr.n_trace;
        if (own) {
          if (tr.u) {
#pragma unroll 1
            for (int t = 0; t < M; ++t) {
              const double ctau = P.ct[t] * tau[j];
              const double v = fma(-ctau, s_prev[t], kc.m);
              const double u = v < kc.lo ? kc.lo : (v > kc.hi ? kc.hi : v);
              tr.u[((int64_t)kk * M * N + t * N + j) * n_tr + slot] = u;
            }
          }
          if (tr.ahat) tr.ahat[((int64_t)kk * N + j) * n_tr + slot] = ahat[j];
          if (tr.theta) tr.theta[((int64_t)kk * N + j) * n_tr + slot] = thi;
          if (tr.rank) {
            int r = 0;
#pragma unroll
            for (int q = 0; q < N; ++q) {
              if (q == j) continue;
              const long long tl = dbits(thv[q]), tj = dbits(thi);
              r += (tl > tj) || (q < j && tl == tj);
            }
            tr.rank[((int64_t)kk * N + j) * n_tr + slot] = (int8_t)r;
          }
        }
        if (gl == 0) {
          const int64_t b = (int64_t)kk * n_tr + slot;
          if (tr.p) tr.p[b] = p;
          if (tr.cap) tr.cap[b] = cap;
          if (tr.status) tr.status[b] = status;
          if (tr.active) {
#pragma unroll
            for (int t = 0; t < M; ++t) tr.active[((int64_t)kk * M + t) * n_tr + slot] = act[t];
          }
        }
      }
    }
    // ---- S4 (own knob): plant (the draws were formed at the top of the period)
    if (slot >= 0 && ivalid && own && tr.levels) {
      const GridEntry *tab = P.grid + kc.cls * kMaxL;
      double a2 = ac;
      for (int sstep = 0; sstep < P.S; ++sstep) {
        const double v = __dadd_rn(u0j, a2);
        const int l = level_of<N>(kc, tab, v);
        a2 = __dadd_rn(v, -tab[l].level);
        tr.levels[((int64_t)kk * P.S * N + sstep * N + j) * tr.n_trace + slot] = (uint8_t)l;
      }
    }
    plant_knob<S>(P, kc, u0j, ac, dem, tm, fb, th_r);
    lp_gather<N, G>(fb, fba);
    double pw = c_true;
#pragma unroll
    for (int q = 0; q < N; ++q) pw = fma(ATa[q], fba[q], pw);
    p = pw + noise;
    if (kk >= kw) {
      sum_theta += tbar;
      sum_p += p;
      sumsq_p = fma(p, p, sumsq_p);
      max_p = kk == kw ? p : fmax(max_p, p);
      n_viol += p > cap;
#pragma unroll
      for (int t = 0; t < M; ++t) act_cnt[t] += act[t] != 0u;
    }
  }

  // ---- write back (Sigma = lam^kk Sigma' at the end of the call)
  const double lam_k = rcp_fast(inv_lam_k);
  if (ivalid) {
    if (own) {
      __stcg(st.fbar + j * li + i, fb);
      __stcg(st.acc + j * li + i, ac);
      __stcg(st.thr + j * li + i, th_r);
      __stcg(st.mu_f + j * li + i, muf[j]);
      __stcg(st.Sfp + j * li + i, sfp[j] * lam_k);
    }
#pragma unroll
    for (int t = 0; t < T; ++t)
      if (t % G == gl) __stcg(st.S + t * li + i, Sg[t] * lam_k);
    if (gl == 0) {
      __stcg(st.p + i, p);
      __stcg(st.w + i, w);
      __stcg(st.mu_p + i, mu_p);
#pragma unroll
      for (int t = 0; t < M; ++t) {
        __stcg(st.s_prev + t * li + i, s_prev[t]);
        __stcg(st.act + t * li + i, act[t]);
      }
      if (tr.sum_p) tr.sum_p[i] = sum_p;
      if (tr.sumsq_p) tr.sumsq_p[i] = sumsq_p;
      if (tr.max_p) tr.max_p[i] = max_p;
      if (tr.sum_theta) tr.sum_theta[i] = sum_theta;
      if (tr.n_viol) tr.n_viol[i] = n_viol;
      if (tr.n_miss) tr.n_miss[i] = 0;
      if (tr.n_window) tr.n_window[i] = (int)((4 * (int64_t)Ktot) / 5);
      if (tr.final_p) tr.final_p[i] = p;
      if (tr.act_count) {
#pragma unroll
        for (int t = 0; t < M; ++t) tr.act_count[t * li + i] = act_cnt[t];
      }
    }
  }
}

}  // namespace capgpu
