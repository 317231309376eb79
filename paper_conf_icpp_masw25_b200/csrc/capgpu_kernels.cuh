// capgpu_kernels.cuh -- CUDA kernels of the CapGPU hot path (sm_100a) and their
// templated launchers.  Instantiated per knob count N in inst_n*.cu.
//
//   k_init_servers   per-server synthetic plant constants
//   k_identify       S0: one WARP per server; sweep rows spread over lanes,
//                    normal equations reduced with warp shuffles
//   k_init_instances cap base + virtual period -1 (Q23)
//   k_simulate       S1-S4 fused over K periods, one THREAD per instance, state
//                    in registers + a per-thread shared-memory slab
//   k_period         S1-S4 for one period with state in HBM + rack/cluster
//                    budget (S5, cfg 4)
//   k_control_step   S1-S3 on user measurements (per-period mode)
//   k_assign_weights S2 alone
#pragma once

#include "capgpu_device.cuh"

namespace capgpu {

// ------------------------------------------------------------------ state layout

// Device state of a context.  Every array is SoA [field][ld].
struct StatePtrs {
  // per instance (ld = n_inst)
  double *fbar, *acc, *thr, *p;            // plant state S4
  double *w, *mu_f, *mu_p, *S, *Sfp;       // model state S1
  uint32_t *act;                           // [M] warm-start active codes
  double *cap_base;                        // [1]
  int32_t *trace_slot;                     // [1] -1 = not traced
  // per server (ld = n_srv)
  double *a_true, *c_true, *thr_max, *base, *amp, *A0, *pmin, *pmax;
};

struct TracePtrs {
  double *sum_p, *sumsq_p, *max_p, *sum_theta, *final_p;
  int32_t *n_viol, *n_window, *act_count;
  int32_t n_trace;
  double *p, *cap, *u, *ahat, *theta;
  uint32_t *active, *status;
  int8_t *rank;
  uint8_t *levels;
};

struct SlabAcc {
  double *p;
  int stride;
  __device__ __forceinline__ double get(int t) const { return p[t * stride]; }
  __device__ __forceinline__ void set(int t, double v) const { p[t * stride] = v; }
};

template <int N>
struct RegArr {
  double (&r)[N];
  __device__ __forceinline__ double get(int t) const { return r[t]; }
};

// global-memory accessor for the per-period kernels (state in HBM)
struct GlobAcc {
  double *p;
  int64_t ld;
  __device__ __forceinline__ double get(int t) const { return p[(int64_t)t * ld]; }
  __device__ __forceinline__ void set(int t, double v) const { p[(int64_t)t * ld] = v; }
};

__device__ __forceinline__ double plant_power(double c_true, const double *a, const double *f, int n, double noise) {
  double pw = c_true;
  for (int j = 0; j < n; ++j) pw = fma(a[j], f[j], pw);
  return pw + noise;
}

// ------------------------------------------------------------------ init

template <int N>
__global__ void k_init_servers(DevParams P, StatePtrs st) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= P.n_srv) return;
  const uint64_t srv = (uint64_t)(P.srv_begin + i);
  const int64_t ld = P.n_srv;
  double a[N], fmn[N], fmx[N];
  double c = gen_c_true(P.seed, srv);
#pragma unroll
  for (int j = 0; j < N; ++j) {
    a[j] = gen_a_true(P.seed, srv, j);
    st.a_true[j * ld + i] = a[j];
    st.thr_max[j * ld + i] = gen_thr_max(P.seed, srv, j);
    st.base[j * ld + i] = gen_dem_base(P.seed, srv, j);
    st.amp[j * ld + i] = gen_dem_amp(P.seed, srv, j);
    fmn[j] = P.k[j].f_min;
    fmx[j] = P.k[j].f_max;
  }
  st.c_true[i] = c;
  st.pmin[i] = gen_power_at(c, a, fmn, N);
  st.pmax[i] = gen_power_at(c, a, fmx, N);
}

// S0 identification: one warp per server.  Rows r = lane, lane+32, ... of the
// sweep (or of user F/p); three passes with xor-butterfly shuffle reductions:
// means, centred normal equations (Gram + rhs + SS_tot), residuals.
template <int N>
__global__ void k_identify(DevParams P, StatePtrs st, const double *F_user, const double *p_user, int rows,
                           double *A_out, double *C_out, double *r2_out) {
  const int lane = threadIdx.x & 31;
  const int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (i >= P.n_srv) return;
  const int64_t ld = P.n_srv;
  const bool synth = (F_user == nullptr);
  double a[N];
  double c = 0.0;
  int nl[N];
  uint64_t key = 0;
  double scale = P.noise_scale;
  if (synth) {
#pragma unroll
    for (int j = 0; j < N; ++j) a[j] = st.a_true[j * ld + i];
    c = st.c_true[i];
    key = gen_stream_key(P.seed, GEN_TAG_SWEEP, (uint64_t)(P.srv_begin + i));
  }
#pragma unroll
  for (int j = 0; j < N; ++j) nl[j] = P.k[j].L;

  auto row = [&](int r, double (&f)[N]) -> double {
    if (synth) {
      int l = -1;
      const int jv = gen_sweep_row(nl, N, r, &l);
#pragma unroll
      for (int j = 0; j < N; ++j) f[j] = level_value(P.k[j], j == jv ? l : P.k[j].sweep_base);
      double pw = c;
#pragma unroll
      for (int j = 0; j < N; ++j) pw = fma(a[j], f[j], pw);
      return pw + (scale > 0.0 ? gen_noise(key, r, scale) : 0.0);
    }
#pragma unroll
    for (int j = 0; j < N; ++j) f[j] = F_user[((int64_t)r * N + j) * ld + i];
    return p_user[(int64_t)r * ld + i];
  };
  auto allsum = [&](double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
  };

  // pass 1: means
  double mf[N], mp = 0.0;
#pragma unroll
  for (int j = 0; j < N; ++j) mf[j] = 0.0;
  for (int r = lane; r < rows; r += 32) {
    double f[N];
    mp += row(r, f);
#pragma unroll
    for (int j = 0; j < N; ++j) mf[j] += f[j];
  }
  const double inv_rows = 1.0 / (double)rows;
#pragma unroll
  for (int j = 0; j < N; ++j) mf[j] = allsum(mf[j]) * inv_rows;
  mp = allsum(mp) * inv_rows;

  // pass 2: centred Gram, rhs, SS_tot
  double G[Tri<N>::size], b[N], spp = 0.0;
#pragma unroll
  for (int t = 0; t < Tri<N>::size; ++t) G[t] = 0.0;
#pragma unroll
  for (int j = 0; j < N; ++j) b[j] = 0.0;
  for (int r = lane; r < rows; r += 32) {
    double f[N];
    const double pc = row(r, f) - mp;
#pragma unroll
    for (int j = 0; j < N; ++j) f[j] -= mf[j];
#pragma unroll
    for (int x = 0; x < N; ++x) {
#pragma unroll
      for (int y = x; y < N; ++y) G[Tri<N>::idx(x, y)] = fma(f[x], f[y], G[Tri<N>::idx(x, y)]);
      b[x] = fma(f[x], pc, b[x]);
    }
    spp = fma(pc, pc, spp);
  }
#pragma unroll
  for (int t = 0; t < Tri<N>::size; ++t) G[t] = allsum(G[t]);
#pragma unroll
  for (int j = 0; j < N; ++j) b[j] = allsum(b[j]);
  spp = allsum(spp);
  double A[N];
  ldlt_solve<N>(G, b, A);
  double C = mp;
#pragma unroll
  for (int j = 0; j < N; ++j) C = fma(-A[j], mf[j], C);

  // pass 3: residual sum of squares
  double ssr = 0.0;
  for (int r = lane; r < rows; r += 32) {
    double f[N];
    double res = row(r, f) - mp;
#pragma unroll
    for (int j = 0; j < N; ++j) res = fma(-A[j], f[j] - mf[j], res);
    ssr = fma(res, res, ssr);
  }
  ssr = allsum(ssr);
  if (lane == 0) {
#pragma unroll
    for (int j = 0; j < N; ++j) {
      if (A_out) A_out[j * ld + i] = A[j];
      st.A0[j * ld + i] = fmax(A[j], P.a_floor);
    }
    if (C_out) C_out[i] = C;
    if (r2_out) r2_out[i] = spp > 0.0 ? 1.0 - ssr / spp : 1.0;
  }
}

__device__ __forceinline__ double demand_of(const DevParams &P, uint64_t kjit, int j, int64_t k, int burst,
                                            double thr_max, double base, double amp) {
  return P.demand_kind == 0 ? gen_demand_const(thr_max, P.demand_frac)
                            : gen_demand_flag(kjit, j, k, burst, thr_max, base, amp);
}

template <int N>
__device__ __forceinline__ uint32_t burst_mask(const DevParams &P, uint64_t kburst, int64_t epoch) {
  uint32_t m = 0u;
  if (P.demand_kind != 0) {
#pragma unroll
    for (int j = 0; j < N; ++j) m |= (uint32_t)gen_burst_flag(kburst, j, epoch) << j;
  }
  return m;
}

// Per instance: base cap and the virtual period -1 (Q23): u0 = f_min, acc = 0.
template <int N>
__global__ void k_init_instances(DevParams P, StatePtrs st, int M) {
  __shared__ double sg[N * kMaxL];
  for (int t = threadIdx.x; t < N * kMaxL; t += blockDim.x) sg[t] = P.g[t / kMaxL][t % kMaxL];
  __syncthreads();
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= P.n_inst) return;
  const int64_t si = i / P.n_caps;
  const int cidx = (int)(i % P.n_caps);
  const uint64_t srv = (uint64_t)(P.srv_begin + si);
  const int64_t ls = P.n_srv, li = P.n_inst;
  double thr_max[N], dem[N], u0[N], acc[N], fbar[N], thr[N], a[N];
  const uint64_t kjit = gen_stream_key(P.seed, GEN_TAG_JIT, srv);
  const uint64_t kburst = gen_stream_key(P.seed, GEN_TAG_BURST, srv);
  const uint32_t bm = burst_mask<N>(P, kburst, 0);
#pragma unroll
  for (int j = 0; j < N; ++j) {
    thr_max[j] = st.thr_max[j * ls + si];
    a[j] = st.a_true[j * ls + si];
    dem[j] = demand_of(P, kjit, j, 0, (bm >> j) & 1u, thr_max[j], st.base[j * ls + si], st.amp[j * ls + si]);
    u0[j] = P.k[j].f_min;
    acc[j] = 0.0;
  }
  plant_delta_sigma<N>(P, sg, u0, acc, dem, thr_max, fbar, thr, nullptr, 0);
  const double noise = gen_noise(gen_stream_key(P.seed, GEN_TAG_NOISE, srv), 0, P.noise_scale);
  st.p[i] = plant_power(st.c_true[si], a, fbar, N, noise);
#pragma unroll
  for (int j = 0; j < N; ++j) {
    st.fbar[j * li + i] = fbar[j];
    st.acc[j * li + i] = acc[j];
    st.thr[j * li + i] = thr[j];
    st.mu_f[j * li + i] = 0.0;
    st.Sfp[j * li + i] = 0.0;
  }
#pragma unroll
  for (int t = 0; t < Tri<N>::size; ++t) st.S[t * li + i] = 0.0;
  st.w[i] = 0.0;
  st.mu_p[i] = 0.0;
  for (int t = 0; t < M; ++t) st.act[t * li + i] = 0u;
  const double fr = gen_cap_frac(P.seed, srv, cidx, P.cap_frac0, P.cap_frac_rand, P.cap_frac_step);
  st.cap_base[i] = gen_cap_base(st.pmin[si], st.pmax[si], fr);
}

// ------------------------------------------------------------------ shared step

// One control instant for one instance: S1, S2, S3.  Returns u0 and fills
// the trace of u/active/ahat/theta; status bits in *status.
template <int N, int M, class SAcc, class A0Acc>
__device__ __forceinline__ void control_instant(const DevParams &P, double cap, double &w, double (&mu_f)[N],
                                                double &mu_p, SAcc S, double (&Sfp)[N], A0Acc A0,
                                                const double (&fbar)[N], double p, const double (&thr)[N],
                                                const double (&thr_max)[N], uint32_t (&act)[M],
                                                double (&u0)[N], double (&ahat)[N], double (&theta)[N],
                                                uint32_t &status, double *tr_u, int64_t tr_ld) {
  // S1 (Eq. 5; Q1-Q4)
  model_push<N>(P.lam, w, mu_f, mu_p, S, Sfp, fbar, p);
  model_solve<N>(P.rho, P.a_lo, P.a_hi, S, Sfp, A0, ahat);
  // S2
  weights<N>(P.theta_min, thr, thr_max, theta);
  double tau[N];
#pragma unroll
  for (int j = 0; j < N; ++j) tau[j] = ahat[j] * theta[j] * P.k[j].inv_r0;
  // S3 (Eq. 9-10a)
  double beta = p - cap, smin = 0.0, smax = 0.0;
#pragma unroll
  for (int j = 0; j < N; ++j) {
    beta = fma(-ahat[j], fbar[j], beta);
    smin = fma(ahat[j], P.k[j].lo, smin);
    smax = fma(ahat[j], P.k[j].hi, smax);
  }
  status = 0u;
  if (beta + smin > 0.0 || beta + smax < 0.0) status |= CAPGPU_ST_CAP_INFEASIBLE;
  bool capped = false;
#pragma unroll
  for (int t = 0; t < M; ++t) {
    double u[N];
    act[t] = solve_block<N>(P.k, ahat, tau, P.ct[t], beta, act[t], u, capped);
    if (t == 0) {
#pragma unroll
      for (int j = 0; j < N; ++j) u0[j] = u[j];
    }
    if (tr_u) {
#pragma unroll
      for (int j = 0; j < N; ++j) tr_u[(int64_t)(t * N + j) * tr_ld] = u[j];
    }
  }
  if (capped) status |= CAPGPU_ST_SOLVER_CAP;
}

// ------------------------------------------------------------------ fused simulate

// Slab fields (per thread): S[T] | A0[N] | a_true[N] | thr_max[N] | base[N] | amp[N]
template <int N>
struct Slab {
  static constexpr int T = Tri<N>::size;
  static constexpr int fields = T + 5 * N;
};

template <int N, int M>
__global__ void __launch_bounds__(128) k_simulate(DevParams P, StatePtrs st, TracePtrs tr, int64_t k0, int K) {
  extern __shared__ double slab_mem[];
  __shared__ double sg[N * kMaxL];
  for (int t = threadIdx.x; t < N * kMaxL; t += blockDim.x) sg[t] = P.g[t / kMaxL][t % kMaxL];
  __syncthreads();
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= P.n_inst) return;
  constexpr int T = Slab<N>::T;
  const int stride = blockDim.x;
  double *my = slab_mem + threadIdx.x;
  const SlabAcc S{my, stride};
  const SlabAcc A0{my + T * stride, stride};
  const SlabAcc AT{my + (T + N) * stride, stride};
  const SlabAcc TM{my + (T + 2 * N) * stride, stride};
  const SlabAcc BA{my + (T + 3 * N) * stride, stride};
  const SlabAcc AM{my + (T + 4 * N) * stride, stride};

  const int64_t si = i / P.n_caps;
  const uint64_t srv = (uint64_t)(P.srv_begin + si);
  const int64_t ls = P.n_srv, li = P.n_inst;

  // ---- stage state into registers / slab
  double fbar[N], acc[N], thr[N], mu_f[N], Sfp[N];
#pragma unroll
  for (int j = 0; j < N; ++j) {
    fbar[j] = st.fbar[j * li + i];
    acc[j] = st.acc[j * li + i];
    thr[j] = st.thr[j * li + i];
    mu_f[j] = st.mu_f[j * li + i];
    Sfp[j] = st.Sfp[j * li + i];
    A0.set(j, st.A0[j * ls + si]);
    AT.set(j, st.a_true[j * ls + si]);
    TM.set(j, st.thr_max[j * ls + si]);
    BA.set(j, st.base[j * ls + si]);
    AM.set(j, st.amp[j * ls + si]);
  }
#pragma unroll
  for (int t = 0; t < T; ++t) S.set(t, st.S[t * li + i]);
  double p = st.p[i], w = st.w[i], mu_p = st.mu_p[i];
  const double c_true = st.c_true[si], cap_base = st.cap_base[i];
  uint32_t act[M];
#pragma unroll
  for (int t = 0; t < M; ++t) act[t] = st.act[t * li + i];
  const int slot = tr.n_trace > 0 ? st.trace_slot[i] : -1;
  const uint64_t kjit = gen_stream_key(P.seed, GEN_TAG_JIT, srv);
  const uint64_t kburst = gen_stream_key(P.seed, GEN_TAG_BURST, srv);
  const uint64_t knoise = gen_stream_key(P.seed, GEN_TAG_NOISE, srv);
  int64_t epoch = -1;
  uint32_t bmask = 0u;

  // ---- summaries (Q25)
  const int kw = K - (4 * K) / 5;
  double sum_p = 0.0, sumsq_p = 0.0, max_p = -INFINITY, sum_theta = 0.0;
  int n_viol = 0, n_win = 0;
  int act_cnt[M];
#pragma unroll
  for (int t = 0; t < M; ++t) act_cnt[t] = 0;

  for (int kk = 0; kk < K; ++kk) {
    const int64_t k = k0 + kk;
    const double cap = gen_cap_at(cap_base, k, P.cap_period, P.cap_lo, P.cap_hi, P.cap_mult);
    double thr_max[N];
#pragma unroll
    for (int j = 0; j < N; ++j) thr_max[j] = TM.get(j);
    double u0[N], ahat[N], theta[N];
    uint32_t status;
    double *tr_u = slot >= 0 && tr.u ? tr.u + (int64_t)kk * M * N * tr.n_trace + slot : nullptr;
    control_instant<N, M>(P, cap, w, mu_f, mu_p, S, Sfp, A0, fbar, p, thr, thr_max, act, u0, ahat, theta,
                          status, tr_u, tr.n_trace);
    if (slot >= 0) {
      const int64_t b = (int64_t)kk * tr.n_trace + slot;
      if (tr.p) tr.p[b] = p;
      if (tr.cap) tr.cap[b] = cap;
      if (tr.status) tr.status[b] = status;
      if (tr.active) {
#pragma unroll
        for (int t = 0; t < M; ++t) tr.active[((int64_t)kk * M + t) * tr.n_trace + slot] = act[t];
      }
      int8_t rk[N];
      ranks<N>(theta, rk);
#pragma unroll
      for (int j = 0; j < N; ++j) {
        const int64_t e = ((int64_t)kk * N + j) * tr.n_trace + slot;
        if (tr.ahat) tr.ahat[e] = ahat[j];
        if (tr.theta) tr.theta[e] = theta[j];
        if (tr.rank) tr.rank[e] = rk[j];
      }
    }
    // ---- S4: period k -> k+1
    const int64_t kn = k + 1;
    if (kn / GEN_BURST_HOLD != epoch) {
      epoch = kn / GEN_BURST_HOLD;
      bmask = burst_mask<N>(P, kburst, epoch);
    }
    double dem[N];
#pragma unroll
    for (int j = 0; j < N; ++j) dem[j] = demand_of(P, kjit, j, kn, (bmask >> j) & 1u, thr_max[j], BA.get(j), AM.get(j));
    uint8_t *lv = slot >= 0 && tr.levels ? tr.levels + (int64_t)kk * P.S * N * tr.n_trace + slot : nullptr;
    plant_delta_sigma<N>(P, sg, u0, acc, dem, thr_max, fbar, thr, lv, tr.n_trace);
    const double noise = gen_noise(knoise, kn, P.noise_scale);
    double pw = c_true;
#pragma unroll
    for (int j = 0; j < N; ++j) pw = fma(AT.get(j), fbar[j], pw);
    p = pw + noise;
    if (kk >= kw) {
      double tb = 0.0;
#pragma unroll
      for (int j = 0; j < N; ++j) tb += theta[j];
      sum_theta += tb / (double)N;
      sum_p += p;
      sumsq_p = fma(p, p, sumsq_p);
      max_p = fmax(max_p, p);
      n_viol += p > cap;
      ++n_win;
#pragma unroll
      for (int t = 0; t < M; ++t) act_cnt[t] += act[t] != 0u;
    }
  }

  // ---- write back
#pragma unroll
  for (int j = 0; j < N; ++j) {
    st.fbar[j * li + i] = fbar[j];
    st.acc[j * li + i] = acc[j];
    st.thr[j * li + i] = thr[j];
    st.mu_f[j * li + i] = mu_f[j];
    st.Sfp[j * li + i] = Sfp[j];
  }
#pragma unroll
  for (int t = 0; t < T; ++t) st.S[t * li + i] = S.get(t);
  st.p[i] = p;
  st.w[i] = w;
  st.mu_p[i] = mu_p;
#pragma unroll
  for (int t = 0; t < M; ++t) st.act[t * li + i] = act[t];
  if (tr.sum_p) tr.sum_p[i] = sum_p;
  if (tr.sumsq_p) tr.sumsq_p[i] = sumsq_p;
  if (tr.max_p) tr.max_p[i] = max_p;
  if (tr.sum_theta) tr.sum_theta[i] = sum_theta;
  if (tr.n_viol) tr.n_viol[i] = n_viol;
  if (tr.n_window) tr.n_window[i] = n_win;
  if (tr.final_p) tr.final_p[i] = p;
  if (tr.act_count) {
#pragma unroll
    for (int t = 0; t < M; ++t) tr.act_count[t * li + i] = act_cnt[t];
  }
}

// ------------------------------------------------------------------ control step (per-period mode)

template <int N, int M>
__global__ void __launch_bounds__(128) k_control_step(DevParams P, StatePtrs st, const double *p_meas,
                                                      const double *f_app, const double *thr_in,
                                                      const double *thr_max_in, const double *cap_in,
                                                      double *u_out, uint32_t *act_out, int8_t *rank_out,
                                                      double *ahat_out, uint32_t *status_out) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= P.n_inst) return;
  const int64_t ld = P.n_inst;
  double fbar[N], thr[N], thr_max[N], mu_f[N], Sfp[N], A0r[N];
  bool finite = true;
  const double p = p_meas[i], cap = cap_in[i];
  finite &= isfinite(p) && isfinite(cap);
#pragma unroll
  for (int j = 0; j < N; ++j) {
    fbar[j] = f_app[j * ld + i];
    thr[j] = thr_in[j * ld + i];
    thr_max[j] = thr_max_in[j * ld + i];
    finite &= isfinite(fbar[j]) && isfinite(thr[j]) && isfinite(thr_max[j]) && thr_max[j] > 0.0;
    mu_f[j] = st.mu_f[j * ld + i];
    Sfp[j] = st.Sfp[j * ld + i];
    A0r[j] = st.A0[j * ld + i];
  }
  uint32_t act[M];
#pragma unroll
  for (int t = 0; t < M; ++t) act[t] = st.act[t * ld + i];
  if (!finite) {
    // Q26: hold the model, pin outputs to the lower bounds
#pragma unroll
    for (int t = 0; t < M; ++t) {
#pragma unroll
      for (int j = 0; j < N; ++j) u_out[((int64_t)t * N + j) * ld + i] = P.k[j].lo;
      uint32_t all = 0u;
#pragma unroll
      for (int j = 0; j < N; ++j) all |= 1u << (2 * j);
      act_out[(int64_t)t * ld + i] = all;
    }
    if (status_out) status_out[i] = CAPGPU_ST_NONFINITE;
    if (ahat_out) {
#pragma unroll
      for (int j = 0; j < N; ++j) ahat_out[j * ld + i] = A0r[j];
    }
    if (rank_out) {
#pragma unroll
      for (int j = 0; j < N; ++j) rank_out[j * ld + i] = (int8_t)j;
    }
    return;
  }
  double w = st.w[i], mu_p = st.mu_p[i];
  const GlobAcc S{st.S + i, ld};
  double u0[N], ahat[N], theta[N];
  uint32_t status;
  control_instant<N, M>(P, cap, w, mu_f, mu_p, S, Sfp, RegArr<N>{A0r}, fbar, p, thr, thr_max, act, u0, ahat,
                        theta, status, u_out + i, ld);
  st.w[i] = w;
  st.mu_p[i] = mu_p;
#pragma unroll
  for (int j = 0; j < N; ++j) {
    st.mu_f[j * ld + i] = mu_f[j];
    st.Sfp[j * ld + i] = Sfp[j];
  }
#pragma unroll
  for (int t = 0; t < M; ++t) {
    st.act[t * ld + i] = act[t];
    act_out[(int64_t)t * ld + i] = act[t];
  }
  if (status_out) status_out[i] = status;
  if (ahat_out) {
#pragma unroll
    for (int j = 0; j < N; ++j) ahat_out[j * ld + i] = ahat[j];
  }
  if (rank_out) {
    int8_t rk[N];
    ranks<N>(theta, rk);
#pragma unroll
    for (int j = 0; j < N; ++j) rank_out[j * ld + i] = rk[j];
  }
}

template <int N>
__global__ void k_assign_weights(DevParams P, const double *thr_in, const double *thr_max_in, double *theta_out,
                                 double *R_out, int8_t *rank_out, int64_t n) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  double thr[N], tm[N], th[N];
#pragma unroll
  for (int j = 0; j < N; ++j) {
    thr[j] = thr_in[j * n + i];
    tm[j] = thr_max_in[j * n + i];
  }
  weights<N>(P.theta_min, thr, tm, th);
#pragma unroll
  for (int j = 0; j < N; ++j) {
    if (theta_out) theta_out[j * n + i] = th[j];
    if (R_out) R_out[j * n + i] = __ddiv_rn(P.k[j].r0, th[j]);
  }
  if (rank_out) {
    int8_t rk[N];
    ranks<N>(th, rk);
#pragma unroll
    for (int j = 0; j < N; ++j) rank_out[j * n + i] = rk[j];
  }
}

template <int N>
__global__ void k_debug_gen(DevParams P, StatePtrs st, int64_t k, double *a_true, double *thr_max, double *c_true,
                            double *dem, double *noise) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= P.n_srv) return;
  const uint64_t srv = (uint64_t)(P.srv_begin + i);
  const int64_t ld = P.n_srv;
  const uint64_t kjit = gen_stream_key(P.seed, GEN_TAG_JIT, srv);
  const uint64_t kburst = gen_stream_key(P.seed, GEN_TAG_BURST, srv);
  const uint32_t bm = burst_mask<N>(P, kburst, k / GEN_BURST_HOLD);
#pragma unroll
  for (int j = 0; j < N; ++j) {
    const double tm = gen_thr_max(P.seed, srv, j);
    a_true[j * ld + i] = gen_a_true(P.seed, srv, j);
    thr_max[j * ld + i] = tm;
    dem[j * ld + i] = demand_of(P, kjit, j, k, (bm >> j) & 1u, tm, gen_dem_base(P.seed, srv, j),
                                gen_dem_amp(P.seed, srv, j));
  }
  c_true[i] = gen_c_true(P.seed, srv);
  noise[i] = gen_noise(gen_stream_key(P.seed, GEN_TAG_NOISE, srv), k, P.noise_scale);
}

// ------------------------------------------------------------------ launchers

struct Launchers {
  int (*init_servers)(const DevParams &, const StatePtrs &, cudaStream_t);
  int (*identify)(const DevParams &, const StatePtrs &, const double *, const double *, int, double *, double *,
                  double *, cudaStream_t);
  int (*init_instances)(const DevParams &, const StatePtrs &, cudaStream_t);
  int (*simulate)(const DevParams &, const StatePtrs &, const TracePtrs &, int64_t, int, cudaStream_t);
  int (*control_step)(const DevParams &, const StatePtrs &, const double *, const double *, const double *,
                      const double *, const double *, double *, uint32_t *, int8_t *, double *, uint32_t *,
                      cudaStream_t);
  int (*assign_weights)(const DevParams &, const double *, const double *, double *, double *, int8_t *, int64_t,
                        cudaStream_t);
  int (*debug_gen)(const DevParams &, const StatePtrs &, int64_t, double *, double *, double *, double *, double *,
                   cudaStream_t);
  int (*sim_smem_bytes)(int block);
};

inline int grid_for(int64_t n, int block) { return (int)((n + block - 1) / block); }

template <int N>
struct LaunchN {
  static int init_servers(const DevParams &P, const StatePtrs &st, cudaStream_t s) {
    k_init_servers<N><<<grid_for(P.n_srv, 128), 128, 0, s>>>(P, st);
    return (int)cudaGetLastError();
  }
  static int identify(const DevParams &P, const StatePtrs &st, const double *F, const double *p, int rows,
                      double *A, double *C, double *r2, cudaStream_t s) {
    k_identify<N><<<grid_for(P.n_srv * 32, 128), 128, 0, s>>>(P, st, F, p, rows, A, C, r2);
    return (int)cudaGetLastError();
  }
  static int init_instances(const DevParams &P, const StatePtrs &st, cudaStream_t s) {
    k_init_instances<N><<<grid_for(P.n_inst, 128), 128, 0, s>>>(P, st, P.M);
    return (int)cudaGetLastError();
  }
  static int assign_weights(const DevParams &P, const double *thr, const double *tm, double *th, double *R,
                            int8_t *rk, int64_t n, cudaStream_t s) {
    k_assign_weights<N><<<grid_for(n, 128), 128, 0, s>>>(P, thr, tm, th, R, rk, n);
    return (int)cudaGetLastError();
  }
  static int debug_gen(const DevParams &P, const StatePtrs &st, int64_t k, double *a, double *tm, double *c,
                       double *dem, double *noise, cudaStream_t s) {
    k_debug_gen<N><<<grid_for(P.n_srv, 128), 128, 0, s>>>(P, st, k, a, tm, c, dem, noise);
    return (int)cudaGetLastError();
  }
  static int sim_smem_bytes(int block) { return (int)(sizeof(double) * Slab<N>::fields * block); }
};

template <int N, int M>
struct LaunchNM {
  static int simulate(const DevParams &P, const StatePtrs &st, const TracePtrs &tr, int64_t k0, int K,
                      cudaStream_t s) {
    const int block = 128;
    const int smem = LaunchN<N>::sim_smem_bytes(block);
    static bool attr = false;
    if (!attr) {
      cudaFuncSetAttribute(k_simulate<N, M>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      attr = true;
    }
    k_simulate<N, M><<<grid_for(P.n_inst, block), block, smem, s>>>(P, st, tr, k0, K);
    return (int)cudaGetLastError();
  }
  static int control_step(const DevParams &P, const StatePtrs &st, const double *p, const double *f,
                          const double *thr, const double *tm, const double *cap, double *u, uint32_t *act,
                          int8_t *rk, double *ahat, uint32_t *status, cudaStream_t s) {
    k_control_step<N, M><<<grid_for(P.n_inst, 128), 128, 0, s>>>(P, st, p, f, thr, tm, cap, u, act, rk, ahat,
                                                                  status);
    return (int)cudaGetLastError();
  }
};

template <int N>
Launchers make_launchers(int M) {
  Launchers L{};
  L.init_servers = &LaunchN<N>::init_servers;
  L.identify = &LaunchN<N>::identify;
  L.init_instances = &LaunchN<N>::init_instances;
  L.assign_weights = &LaunchN<N>::assign_weights;
  L.debug_gen = &LaunchN<N>::debug_gen;
  L.sim_smem_bytes = &LaunchN<N>::sim_smem_bytes;
  switch (M) {
    case 1: L.simulate = &LaunchNM<N, 1>::simulate; L.control_step = &LaunchNM<N, 1>::control_step; break;
    case 2: L.simulate = &LaunchNM<N, 2>::simulate; L.control_step = &LaunchNM<N, 2>::control_step; break;
    case 3: L.simulate = &LaunchNM<N, 3>::simulate; L.control_step = &LaunchNM<N, 3>::control_step; break;
    case 4: L.simulate = &LaunchNM<N, 4>::simulate; L.control_step = &LaunchNM<N, 4>::control_step; break;
    default: break;
  }
  return L;
}

// one per instantiation unit (inst_n*.cu)
#define CAPGPU_DECL_N(NN) Launchers launchers_n##NN(int M);
CAPGPU_DECL_N(2) CAPGPU_DECL_N(3) CAPGPU_DECL_N(4) CAPGPU_DECL_N(5) CAPGPU_DECL_N(6) CAPGPU_DECL_N(7)
CAPGPU_DECL_N(8) CAPGPU_DECL_N(9) CAPGPU_DECL_N(10) CAPGPU_DECL_N(11) CAPGPU_DECL_N(12) CAPGPU_DECL_N(13)
CAPGPU_DECL_N(14) CAPGPU_DECL_N(15) CAPGPU_DECL_N(16)
#undef CAPGPU_DECL_N

}  // namespace capgpu
