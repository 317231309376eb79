// capgpu_api.cu -- the C ABI of include/capgpu.h: validation, device state
// ownership, dispatch to the per-N kernel instantiations.
//
// Nothing here computes the method on the host: every step (S0-S5) runs in the
// kernels of capgpu_kernels.cuh.  Host code only validates, allocates, builds
// the per-launch constant block (grid, bounds, horizon weights, capacity table)
// and launches.
#include <cmath>
#include <cstdarg>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <new>

#include "capgpu_kernels.cuh"
#include "capgpu_budget.cuh"

using namespace capgpu;

struct capgpu_ctx {
  int64_t n_srv = 0, n_inst = 0;
  int32_t N = 0, M = 0, P = 0, T = 0;
  capgpu_params prm{};
  capgpu_shard shard{};
  capgpu_knob_bounds bounds[CAPGPU_MAX_KNOBS]{};
  DevParams dp{};
  StatePtrs st{};
  Launchers L{};
  void *ws = nullptr;
  int64_t ws_bytes = 0;
  bool servers_ready = false, has_prior = false, sim_ready = false;
  int32_t convex_static = 1;       // dp.convex of the static bounds (control_step, SLO-free runs)
  KnobConst *kdev_slo = nullptr;   // device [2][CAPGPU_MAX_KNOBS]: knob constants of the SLO phases
  int64_t k_global = 0;
  capgpu_workload wl{};
  Budget budget{};
  double *explicit_tab = nullptr;  // NEXT-3 explicit MPC tables (allocated by the first capgpu_explicit_build)
  bool explicit_ready = false;
  char err[512] = {0};
};

static thread_local char g_err[512];

static int fail(capgpu_ctx *c, int code, const char *fmt, ...) {
  char *buf = c ? c->err : g_err;
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, 512, fmt, ap);
  va_end(ap);
  return code;
}

static int cuda_fail(capgpu_ctx *c, cudaError_t e, const char *where) {
  return fail(c, CAPGPU_E_CUDA, "%s: %s", where, cudaGetErrorString(e));
}

#define CK_CUDA(ctx, call)                                   \
  do {                                                       \
    cudaError_t e_ = (call);                                 \
    if (e_ != cudaSuccess) return cuda_fail(ctx, e_, #call); \
  } while (0)

static bool is_device_ptr(const void *p) {
  if (!p) return false;
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

#define NEED_DEV(ctx, ptr)                                                                  \
  do {                                                                                      \
    if (!is_device_ptr(ptr)) return fail(ctx, CAPGPU_E_INVALID, "%s is not a device pointer", #ptr); \
  } while (0)
#define OPT_DEV(ctx, ptr)                        \
  do {                                           \
    if ((ptr) != nullptr) NEED_DEV(ctx, ptr);    \
  } while (0)

static Launchers launchers(int N, int M) {
  // experiment builds may compile a subset of the knob counts (build.py --only-n)
#ifdef CAPGPU_SUBSET
#define CAPGPU_CASE(NN) CAPGPU_CASE_IF_##NN
#else
#define CAPGPU_CASE(NN) \
  case NN: return launchers_n##NN(M);
#endif
  switch (N) {
    CAPGPU_CASE(2) CAPGPU_CASE(3) CAPGPU_CASE(4) CAPGPU_CASE(5) CAPGPU_CASE(6) CAPGPU_CASE(7) CAPGPU_CASE(8)
    CAPGPU_CASE(9) CAPGPU_CASE(10) CAPGPU_CASE(11) CAPGPU_CASE(12) CAPGPU_CASE(13) CAPGPU_CASE(14)
    CAPGPU_CASE(15) CAPGPU_CASE(16)
#undef CAPGPU_CASE
    default: return Launchers{};
  }
}

extern "C" {

const char *capgpu_version(void) { return "capgpu-b200 0.1 (sm_100a)"; }

const char *capgpu_status_string(int code) {
  switch (code) {
    case CAPGPU_OK: return "ok";
    case CAPGPU_E_INVALID: return "invalid argument";
    case CAPGPU_E_NOMEM: return "out of device memory";
    case CAPGPU_E_CUDA: return "CUDA error";
    case CAPGPU_E_NCCL: return "NCCL error";
    case CAPGPU_E_ORDER: return "call order (no prior / not initialised)";
    case CAPGPU_E_UNSUPPORTED: return "unsupported by this build";
    default: return "unknown";
  }
}

const char *capgpu_last_error(const capgpu_ctx *ctx) { return ctx ? ctx->err : g_err; }

void capgpu_default_params(capgpu_params *o) {
  if (!o) return;
  std::memset(o, 0, sizeof *o);
  o->q = 1.0;
  o->r0 = 1e-4;
  o->theta_min = 0.05;
  o->lambda = 0.95;
  o->rho = 100.0;
  o->a_lo = 0.25;
  o->a_hi = 4.0;
  o->a_floor = 1e-3;
  o->gamma = 0.91;
  o->noise_std = 11.0;
  o->substeps = 4;
  o->caps_per_server = 1;
  o->seed = 1;
}

int64_t capgpu_shard_range(int64_t n_global, int32_t world, int32_t rank, int64_t granule, int64_t *begin_out) {
  if (n_global <= 0 || world <= 0 || rank < 0 || rank >= world || granule <= 0) return -1;
  const int64_t units = (n_global + granule - 1) / granule;
  const int64_t base = units / world, rem = units % world;
  // the first (world - rem) ranks get `base` units, the last `rem` ranks base + 1
  const int64_t lo_ranks = world - rem;
  int64_t u0 = rank < lo_ranks ? rank * base : lo_ranks * base + (rank - lo_ranks) * (base + 1);
  int64_t nu = rank < lo_ranks ? base : base + 1;
  int64_t b = u0 * granule, e = (u0 + nu) * granule;
  if (e > n_global) e = n_global;
  if (b > n_global) b = n_global;
  if (begin_out) *begin_out = b;
  return e - b;
}

int capgpu_create(capgpu_ctx **out, int64_t n_servers, int32_t n_gpus, capgpu_horizons h,
                  const capgpu_knob_bounds *bounds, const capgpu_params *params, const capgpu_shard *shard) {
  if (!out) return fail(nullptr, CAPGPU_E_INVALID, "out is NULL");
  *out = nullptr;
  capgpu_params prm;
  if (params) prm = *params;
  else capgpu_default_params(&prm);
  const int N = 1 + n_gpus;
  if (n_servers < 1) return fail(nullptr, CAPGPU_E_INVALID, "n_servers < 1");
  if (n_gpus < 1 || N > CAPGPU_MAX_KNOBS) return fail(nullptr, CAPGPU_E_INVALID, "n_gpus must be in [1, 15]");
  if (h.M < 1 || h.M > h.P || h.P > CAPGPU_MAX_P) return fail(nullptr, CAPGPU_E_INVALID, "need 1 <= M <= P <= 64");
  if (h.M > CAPGPU_MAX_M) return fail(nullptr, CAPGPU_E_UNSUPPORTED, "M > %d", CAPGPU_MAX_M);
  if (!bounds) return fail(nullptr, CAPGPU_E_INVALID, "bounds is NULL");
  if (!(prm.q > 0) || !(prm.r0 > 0) || !(prm.theta_min > 0 && prm.theta_min <= 1) ||
      !(prm.lambda > 0 && prm.lambda <= 1) || !(prm.rho > 0) || !(prm.a_lo >= 0 && prm.a_lo <= prm.a_hi) ||
      !(prm.a_floor > 0) || !(prm.gamma > 0) || !(prm.noise_std >= 0) || prm.caps_per_server < 1)
    return fail(nullptr, CAPGPU_E_INVALID, "params out of range");
  if (!(prm.substeps == 1 || prm.substeps == 2 || prm.substeps == 4 || prm.substeps == 8))
    return fail(nullptr, CAPGPU_E_INVALID, "substeps must be 1, 2, 4 or 8");
  if (!(prm.wmove >= 0.0) || !std::isfinite(prm.wmove)) return fail(nullptr, CAPGPU_E_INVALID, "wmove must be >= 0");
  if (!(prm.ref_alpha >= 0.0 && prm.ref_alpha < 1.0))
    return fail(nullptr, CAPGPU_E_INVALID, "ref_alpha must be in [0, 1)");
  if (prm.wmove > 0.0 && h.M * N > kMoveMaxVars)
    return fail(nullptr, CAPGPU_E_UNSUPPORTED, "move suppression needs M * N <= %d on the CUDA path", kMoveMaxVars);
  for (int j = 0; j < N; ++j) {
    const capgpu_knob_bounds &b = bounds[j];
    if (!(b.f_min < b.f_max) || !std::isfinite(b.f_min) || !std::isfinite(b.f_max))
      return fail(nullptr, CAPGPU_E_INVALID, "knob %d: need f_min < f_max", j);
    if (b.n_levels < 2 || b.n_levels > CAPGPU_MAX_LEVELS)
      return fail(nullptr, CAPGPU_E_INVALID, "knob %d: n_levels in [2, 32]", j);
    if (b.sweep_base < 0 || b.sweep_base >= b.n_levels) return fail(nullptr, CAPGPU_E_INVALID, "knob %d: sweep_base", j);
    const double flo = b.f_lo == 0.0 ? b.f_min : b.f_lo;
    if (!(flo >= b.f_min && flo <= b.f_max)) return fail(nullptr, CAPGPU_E_INVALID, "knob %d: f_lo outside [f_min, f_max]", j);
    if (b.r0 < 0) return fail(nullptr, CAPGPU_E_INVALID, "knob %d: r0 < 0", j);
  }
  capgpu_shard sh{};
  if (shard) sh = *shard;
  else {
    sh.rank = 0;
    sh.world = 1;
    sh.srv_begin = 0;
    sh.n_servers_global = n_servers;
  }
  if (sh.world < 1 || sh.rank < 0 || sh.rank >= sh.world || sh.srv_begin < 0)
    return fail(nullptr, CAPGPU_E_INVALID, "bad shard");
  if (sh.n_servers_global < sh.srv_begin + n_servers) sh.n_servers_global = sh.srv_begin + n_servers;

  capgpu_ctx *c = new (std::nothrow) capgpu_ctx();
  if (!c) return fail(nullptr, CAPGPU_E_NOMEM, "host allocation");
  c->n_srv = n_servers;
  c->n_inst = n_servers * prm.caps_per_server;
  c->N = N;
  c->M = h.M;
  c->P = h.P;
  c->T = N * (N + 1) / 2;
  c->prm = prm;
  c->shard = sh;
  for (int j = 0; j < N; ++j) c->bounds[j] = bounds[j];
  c->L = launchers(N, h.M);
  if (!c->L.simulate || !c->L.init_servers) {  // an experiment build without this knob count
    delete c;
    return fail(nullptr, CAPGPU_E_UNSUPPORTED, "this library was built without N = %d knobs", N);
  }

  // ---- per-launch constants
  DevParams &d = c->dp;
  d.N = N;
  d.M = h.M;
  d.P = h.P;
  d.S = prm.substeps;
  d.n_caps = prm.caps_per_server;
  d.q = prm.q;
  d.theta_min = prm.theta_min;
  d.lam = prm.lambda;
  d.rho = prm.rho;
  d.a_lo = prm.a_lo;
  d.a_hi = prm.a_hi;
  d.a_floor = prm.a_floor;
  d.noise_scale = prm.noise_std * std::sqrt(3.0);
  d.inv_S = 1.0 / (double)prm.substeps;
  d.inv_lam = 1.0 / prm.lambda;
  {
    // fold interval of the fused kernel's scaled model state: lam^-R <= 2^600
    // keeps Sigma' = Sigma lam^-kk and rho lam^-kk finite and lam^kk above the
    // FTZ range of the reciprocal (a fixed 1024 overflows for lam <~ 0.5)
    int R = 1024;
    const double l2 = -std::log2(prm.lambda);
    while (R > 1 && (double)R * l2 > 600.0) R >>= 1;
    d.fold_mask = R - 1;
  }
  d.wmove = prm.wmove;
  // Q37: block t's tracking offset is beta + ref_w[t] (P_s - p(k)), ref_w[t] =
  // mean of alpha^i over the prediction steps i whose prediction uses u_t
  d.ref = prm.ref_alpha > 0.0 ? 1 : 0;
  for (int t = 0; t < h.M; ++t) {
    double sum = 0.0, ai = 1.0;
    int cnt = 0;
    for (int i = 1; i <= h.P; ++i) {
      ai *= prm.ref_alpha;
      if ((i < h.M ? i : h.M) - 1 == t) {
        sum += ai;
        ++cnt;
      }
    }
    d.ref_w[t] = d.ref ? sum / cnt : 0.0;
  }
  // Q11: c_t = Q for t < M-1, c_{M-1} = (P - M + 1) Q
  for (int t = 0; t < h.M; ++t) d.ct[t] = t < h.M - 1 ? prm.q : (double)(h.P - h.M + 1) * prm.q;
  d.seed = prm.seed;
  d.srv_begin = sh.srv_begin;
  d.n_srv = c->n_srv;
  d.n_inst = c->n_inst;
  d.inv_N = 1.0 / (double)N;
  // Frequency-grid classes: knobs with the same (f_min, f_max, L, CPU/GPU)
  // share one table of thresholds, levels and capacity factors (Q14, Q15),
  // computed here with the oracle's formulas (host, no FP contraction).
  static_assert(sizeof(GridEntry) == 32, "GridEntry layout");
  GridEntry grid[CAPGPU_MAX_KNOBS][CAPGPU_MAX_LEVELS];
  int n_class = 0;
  int cls_of[CAPGPU_MAX_KNOBS];
  for (int j = 0; j < N; ++j) {
    const capgpu_knob_bounds &b = bounds[j];
    int found = -1;
    for (int q = 0; q < j; ++q) {
      const capgpu_knob_bounds &o = bounds[q];
      if (o.f_min == b.f_min && o.f_max == b.f_max && o.n_levels == b.n_levels && (q == 0) == (j == 0)) {
        found = cls_of[q];
        break;
      }
    }
    if (found < 0) {
      found = n_class++;
      const double step = (b.f_max - b.f_min) / (double)(b.n_levels - 1);
      for (int l = 0; l < CAPGPU_MAX_LEVELS; ++l) {
        GridEntry &e = grid[found][l];
        const int ll = l < b.n_levels ? l : b.n_levels - 1;
        e.level = b.f_min + (double)ll * step;
        e.g = j == 0 ? e.level / b.f_max : std::pow(e.level / b.f_max, prm.gamma);  // Q14
        e.mid_lo = ll == 0 ? -INFINITY : b.f_min + ((double)(ll - 1) + 0.5) * step;
        e.mid_hi = ll >= b.n_levels - 1 ? INFINITY : b.f_min + ((double)ll + 0.5) * step;
      }
    }
    cls_of[j] = found;
  }
  d.n_class = n_class;
  for (int j = 0; j < N; ++j) {
    const capgpu_knob_bounds &b = bounds[j];
    KnobConst &k = d.k[j];
    k.f_min = b.f_min;
    k.f_max = b.f_max;
    k.L = b.n_levels;
    k.sweep_base = b.sweep_base;
    k.cls = cls_of[j];
    k.step = (b.f_max - b.f_min) / (double)(b.n_levels - 1);
    k.inv_step = 1.0 / k.step;
    k.lo = b.f_lo == 0.0 ? b.f_min : b.f_lo;
    k.hi = b.f_max;
    k.m = b.f_min;  // Q7
    k.span = k.hi - k.m;
    k.r0 = b.r0 == 0.0 ? prm.r0 : b.r0;
    k.inv_r0 = 1.0 / k.r0;
    k.pos_tol = 1e-9;  // grid steps: >> the table and sub-step rounding (ulps of f_max; plant_pair)
  }
  // two-level pair tables of plant_pair: row l = {mid(l), level(l), level(l+1), g(l), g(l+1)}
  PairEntry pairs[CAPGPU_MAX_KNOBS][CAPGPU_MAX_LEVELS];
  for (int c2 = 0; c2 < n_class; ++c2)
    for (int l = 0; l < CAPGPU_MAX_LEVELS; ++l) {
      const int l0 = l + 1 < CAPGPU_MAX_LEVELS ? l : l - 1;
      const GridEntry &a = grid[c2][l0], &b = grid[c2][l0 + 1];
      pairs[c2][l] = PairEntry{a.mid_hi, a.level, b.level, a.g, b.g, 0.0};
    }
  d.convex = 1;
  for (int j = 0; j < N; ++j) d.convex &= d.k[j].lo == d.k[j].m ? 1 : 0;
  c->convex_static = d.convex;
  d.slo = 0;

  // ---- state workspace (SoA)
  const int64_t ni = c->n_inst, ns = c->n_srv;
  const int64_t nd_inst = (int64_t)(5 * N + c->T + 5);
  const int64_t nd_srv = (int64_t)(5 * N + 3);
  const int64_t grid_bytes = (int64_t)(sizeof(GridEntry) + sizeof(PairEntry)) * n_class * CAPGPU_MAX_LEVELS;
  const int64_t sched_words = ni + 2;  // chunked schedule of the fused kernel: counter + done[instance]
  const int64_t bytes = 8 * (nd_inst * ni + nd_srv * ns) + 12 * (int64_t)h.M * ni + 4 * ni + 4 * sched_words +
                        grid_bytes + (int64_t)sizeof(KnobConst) * CAPGPU_MAX_KNOBS * 3 + 256;
  cudaError_t e = cudaMalloc(&c->ws, (size_t)bytes);
  if (e != cudaSuccess) {
    cudaGetLastError();
    delete c;
    return fail(nullptr, CAPGPU_E_NOMEM, "cudaMalloc(%lld): %s", (long long)bytes, cudaGetErrorString(e));
  }
  c->ws_bytes = bytes;
  // every CUDA call of create is checked: on failure nothing is left allocated
  auto ck = [&](cudaError_t ce, const char *what) -> bool {
    if (ce == cudaSuccess) return true;
    cudaGetLastError();
    fail(nullptr, CAPGPU_E_CUDA, "%s: %s", what, cudaGetErrorString(ce));
    cudaFree(c->ws);
    delete c;
    return false;
  };
  if (!ck(cudaMemset(c->ws, 0, (size_t)bytes), "cudaMemset(workspace)")) return CAPGPU_E_CUDA;
  double *q = (double *)c->ws;
  auto take = [&](int64_t n) { double *r = q; q += n; return r; };
  StatePtrs &s = c->st;
  s.fbar = take(N * ni);
  s.acc = take(N * ni);
  s.thr = take(N * ni);
  s.p = take(ni);
  s.w = take(ni);
  s.mu_p = take(ni);
  // mu_f | Sigma | Sigma_fp are consecutive rows (ld n_inst) and a_true ..
  // A0 below are consecutive rows (ld n_srv): k_period stages each block
  // with one 2D TMA box per 32 servers
  s.mu_f = take(N * ni);
  s.S = take(c->T * ni);
  s.Sfp = take(N * ni);
  s.cap_base = take(ni);
  s.lamk = take(ni);
  s.a_true = take(N * ns);
  s.c_true = take(ns);
  s.thr_max = take(N * ns);
  s.base = take(N * ns);
  s.amp = take(N * ns);
  s.A0 = take(N * ns);
  s.pmin = take(ns);
  s.pmax = take(ns);
  s.s_prev = take((int64_t)h.M * ni);
  q = (double *)(((uintptr_t)q + 31) & ~(uintptr_t)31);  // 16-byte vector loads of the grid table
  GridEntry *gdev = (GridEntry *)take(4 * (int64_t)n_class * CAPGPU_MAX_LEVELS);
  PairEntry *pdev = (PairEntry *)take(6 * (int64_t)n_class * CAPGPU_MAX_LEVELS);
  KnobConst *kdev = (KnobConst *)take((int64_t)(sizeof(KnobConst) * CAPGPU_MAX_KNOBS + 7) / 8);
  if (!ck(cudaMemcpy(kdev, d.k, sizeof(KnobConst) * CAPGPU_MAX_KNOBS, cudaMemcpyHostToDevice), "cudaMemcpy(knobs)"))
    return CAPGPU_E_CUDA;
  d.k_dev = kdev;
  c->kdev_slo = (KnobConst *)take((int64_t)(sizeof(KnobConst) * CAPGPU_MAX_KNOBS * 2 + 7) / 8);
  d.k_dev_slo[0] = c->kdev_slo;
  d.k_dev_slo[1] = c->kdev_slo + CAPGPU_MAX_KNOBS;
  s.trace_slot = (int32_t *)q;
  s.act = (uint32_t *)(s.trace_slot + ni);
  s.sched = (int32_t *)(s.act + (int64_t)h.M * ni);
  {
    const char *nc = getenv("CAPGPU_NO_CHUNKING");
    d.no_chunking = (nc && nc[0] && nc[0] != '0') ? 1 : 0;
  }
  for (int c2 = 0; c2 < n_class; ++c2)
    if (!ck(cudaMemcpy(gdev + c2 * CAPGPU_MAX_LEVELS, grid[c2], sizeof(GridEntry) * CAPGPU_MAX_LEVELS,
                       cudaMemcpyHostToDevice), "cudaMemcpy(grid)"))
      return CAPGPU_E_CUDA;
  d.grid = gdev;
  for (int c2 = 0; c2 < n_class; ++c2)
    if (!ck(cudaMemcpy(pdev + c2 * CAPGPU_MAX_LEVELS, pairs[c2], sizeof(PairEntry) * CAPGPU_MAX_LEVELS,
                       cudaMemcpyHostToDevice), "cudaMemcpy(pairs)"))
      return CAPGPU_E_CUDA;
  d.pair = pdev;

  if (sh.use_nccl) {
    int rc = budget_init_nccl(c->budget, sh.nccl_id, sh.world, sh.rank, c->err);
    if (rc != CAPGPU_OK) {
      cudaFree(c->ws);
      delete c;
      return fail(nullptr, rc, "nccl init failed");
    }
  }
  *out = c;
  return CAPGPU_OK;
}

int capgpu_destroy(capgpu_ctx *c) {
  if (!c) return CAPGPU_OK;
  budget_free(c->budget);
  if (c->explicit_tab) cudaFree(c->explicit_tab);
  if (c->ws) cudaFree(c->ws);
  delete c;
  return CAPGPU_OK;
}

int64_t capgpu_state_bytes(const capgpu_ctx *c) { return c ? c->ws_bytes : 0; }

static int ensure_servers(capgpu_ctx *c, cudaStream_t s) {
  if (c->servers_ready) return CAPGPU_OK;
  int e = c->L.init_servers(c->dp, c->st, s);
  if (e) return cuda_fail(c, (cudaError_t)e, "init_servers");
  c->servers_ready = true;
  return CAPGPU_OK;
}

int capgpu_identify(capgpu_ctx *c, const double *F_d, const double *p_d, int32_t rows, double *A_out_d,
                    double *C_out_d, double *r2_out_d, void *stream) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  cudaStream_t s = (cudaStream_t)stream;
  if ((F_d == nullptr) != (p_d == nullptr)) return fail(c, CAPGPU_E_INVALID, "F_d and p_d must both be set or both NULL");
  if (F_d) {
    NEED_DEV(c, F_d);
    NEED_DEV(c, p_d);
    if (rows < c->N + 1) return fail(c, CAPGPU_E_INVALID, "rows < N + 1");
  } else {
    rows = 0;
    for (int j = 0; j < c->N; ++j) rows += c->bounds[j].n_levels;
  }
  OPT_DEV(c, A_out_d);
  OPT_DEV(c, C_out_d);
  OPT_DEV(c, r2_out_d);
  if (!F_d) {
    int rc = ensure_servers(c, s);
    if (rc) return rc;
  }
  int e = c->L.identify(c->dp, c->st, F_d, p_d, rows, A_out_d, C_out_d, r2_out_d, s);
  if (e) return cuda_fail(c, (cudaError_t)e, "identify");
  c->has_prior = true;
  return CAPGPU_OK;
}

int capgpu_set_prior(capgpu_ctx *c, const double *A0_d, void *stream) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  NEED_DEV(c, A0_d);
  CK_CUDA(c, cudaMemcpyAsync(c->st.A0, A0_d, sizeof(double) * c->N * c->n_srv, cudaMemcpyDeviceToDevice,
                             (cudaStream_t)stream));
  c->has_prior = true;
  return CAPGPU_OK;
}

int capgpu_model_reset(capgpu_ctx *c, void *stream) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  cudaStream_t s = (cudaStream_t)stream;
  const int64_t ni = c->n_inst;
  CK_CUDA(c, cudaMemsetAsync(c->st.w, 0, sizeof(double) * ni, s));
  CK_CUDA(c, cudaMemsetAsync(c->st.mu_f, 0, sizeof(double) * c->N * ni, s));
  CK_CUDA(c, cudaMemsetAsync(c->st.mu_p, 0, sizeof(double) * ni, s));
  CK_CUDA(c, cudaMemsetAsync(c->st.S, 0, sizeof(double) * c->T * ni, s));
  CK_CUDA(c, cudaMemsetAsync(c->st.Sfp, 0, sizeof(double) * c->N * ni, s));
  CK_CUDA(c, cudaMemsetAsync(c->st.s_prev, 0, sizeof(double) * c->M * ni, s));
  CK_CUDA(c, cudaMemsetAsync(c->st.act, 0, sizeof(uint32_t) * c->M * ni, s));
  return CAPGPU_OK;
}

int capgpu_assign_weights(capgpu_ctx *c, const double *thr_d, const double *thr_max_d, double *theta_out_d,
                          double *R_out_d, int8_t *rank_out_d, void *stream) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  NEED_DEV(c, thr_d);
  NEED_DEV(c, thr_max_d);
  OPT_DEV(c, theta_out_d);
  OPT_DEV(c, R_out_d);
  OPT_DEV(c, rank_out_d);
  int e = c->L.assign_weights(c->dp, thr_d, thr_max_d, theta_out_d, R_out_d, rank_out_d, c->n_srv,
                              (cudaStream_t)stream);
  if (e) return cuda_fail(c, (cudaError_t)e, "assign_weights");
  return CAPGPU_OK;
}

int capgpu_control_step(capgpu_ctx *c, const double *p_meas_d, const double *f_applied_d, const double *thr_d,
                        const double *thr_max_d, const double *cap_d, double *u_out_d, uint32_t *active_out_d,
                        int8_t *rank_out_d, double *ahat_out_d, uint32_t *status_out_d, void *stream) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  if (c->prm.caps_per_server != 1) return fail(c, CAPGPU_E_INVALID, "control_step needs caps_per_server == 1");
  NEED_DEV(c, p_meas_d);
  NEED_DEV(c, f_applied_d);
  NEED_DEV(c, thr_d);
  NEED_DEV(c, thr_max_d);
  NEED_DEV(c, cap_d);
  NEED_DEV(c, u_out_d);
  NEED_DEV(c, active_out_d);
  OPT_DEV(c, rank_out_d);
  OPT_DEV(c, ahat_out_d);
  OPT_DEV(c, status_out_d);
  if (!c->has_prior) return fail(c, CAPGPU_E_ORDER, "no prior A0: call capgpu_identify or capgpu_set_prior first");
  if (c->prm.wmove > 0.0) return fail(c, CAPGPU_E_UNSUPPORTED, "move suppression (wmove > 0) in control_step");
  DevParams dp = c->dp;  // static bounds: no SLO schedule on user measurements
  dp.slo = 0;
  dp.convex = c->convex_static;
  int e = c->L.control_step(dp, c->st, p_meas_d, f_applied_d, thr_d, thr_max_d, cap_d, u_out_d, active_out_d,
                            rank_out_d, ahat_out_d, status_out_d, (cudaStream_t)stream);
  if (e) return cuda_fail(c, (cudaError_t)e, "control_step");
  return CAPGPU_OK;
}

// NEXT-3 explicit (multi-parametric) MPC: offline part + online part
int capgpu_explicit_build(capgpu_ctx *c, const double *thr_d, const double *thr_max_d, void *stream) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  if (c->prm.caps_per_server != 1) return fail(c, CAPGPU_E_INVALID, "explicit MPC needs caps_per_server == 1");
  NEED_DEV(c, thr_d);
  NEED_DEV(c, thr_max_d);
  if (!c->has_prior) return fail(c, CAPGPU_E_ORDER, "no prior A0: call capgpu_identify or capgpu_set_prior first");
  if (!c->convex_static || c->prm.ref_alpha > 0.0 || c->prm.wmove > 0.0)
    return fail(c, CAPGPU_E_UNSUPPORTED, "explicit MPC tabulates the convex literal Eq. 9 (no f_lo, reference "
                                         "trajectory or move suppression)");
  if (!c->explicit_tab) {
    const size_t bytes = sizeof(double) * (size_t)c->L.explicit_fields * (size_t)c->n_srv;
    cudaError_t e = cudaMalloc(&c->explicit_tab, bytes);
    if (e != cudaSuccess) {
      cudaGetLastError();
      c->explicit_tab = nullptr;
      return fail(c, CAPGPU_E_NOMEM, "explicit table (%zu bytes): %s", bytes, cudaGetErrorString(e));
    }
  }
  int e = c->L.explicit_build(c->dp, c->st, thr_d, thr_max_d, c->explicit_tab, (cudaStream_t)stream);
  if (e) return cuda_fail(c, (cudaError_t)e, "explicit_build");
  c->explicit_ready = true;
  return CAPGPU_OK;
}

int capgpu_explicit_step(capgpu_ctx *c, const double *p_meas_d, const double *f_applied_d, const double *cap_d,
                         double *u_out_d, uint32_t *active_out_d, uint32_t *status_out_d, void *stream) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  NEED_DEV(c, p_meas_d);
  NEED_DEV(c, f_applied_d);
  NEED_DEV(c, cap_d);
  NEED_DEV(c, u_out_d);
  NEED_DEV(c, active_out_d);
  OPT_DEV(c, status_out_d);
  if (!c->explicit_ready) return fail(c, CAPGPU_E_ORDER, "no explicit table: call capgpu_explicit_build first");
  int e = c->L.explicit_step(c->dp, c->explicit_tab, p_meas_d, f_applied_d, cap_d, u_out_d, active_out_d,
                             status_out_d, (cudaStream_t)stream);
  if (e) return cuda_fail(c, (cudaError_t)e, "explicit_step");
  return CAPGPU_OK;
}

__global__ void k_trace_slots(int32_t *slot, int64_t n, const int64_t *inst, int32_t n_trace) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) slot[i] = -1;
  __syncthreads();
}
__global__ void k_trace_slots_set(int32_t *slot, int64_t n, const int64_t *inst, int32_t n_trace) {
  const int t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t < n_trace) {
    const int64_t i = inst[t];
    if (i >= 0 && i < n) slot[i] = t;
  }
}

int capgpu_sim_reset(capgpu_ctx *c) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  c->sim_ready = false;
  c->budget.ready = false;
  c->k_global = 0;
  return CAPGPU_OK;
}

// NEXT-1: the SLO schedule's per-phase bounds (§6.4, Eq. 10b-c
// P:205-208; Q29-Q31).  Host-side constants only (like the grid table): for
// each phase and knob the SLO level q = the lowest grid level whose latency
// e_min (f_max/level)^gamma meets SLO = ratio e_min, i.e. level >= f_max
// ratio^(-1/gamma); bound = max(f_lo, level(q)), or f_max + SLO_INFEASIBLE when
// no level meets it.  Validation happens before anything is launched.
// validation of the SLO schedule alone (no side effects); *any = a ratio is set
static int slo_validate(capgpu_ctx *c, const capgpu_workload &w, bool *any_out) {
  bool any = false;
  for (int j = 0; j < CAPGPU_MAX_KNOBS; ++j) {
    if (!(w.slo_a[j] >= 0.0) || !(w.slo_b[j] >= 0.0) || !std::isfinite(w.slo_a[j]) || !std::isfinite(w.slo_b[j]))
      return fail(c, CAPGPU_E_INVALID, "slo ratios must be finite and >= 0");
    if (j >= c->N && (w.slo_a[j] != 0.0 || w.slo_b[j] != 0.0))
      return fail(c, CAPGPU_E_INVALID, "slo ratio set for knob %d >= N", j);
    any |= w.slo_a[j] != 0.0 || w.slo_b[j] != 0.0;
  }
  *any_out = any;
  if (!any) return CAPGPU_OK;
  if (w.hierarchical) return fail(c, CAPGPU_E_UNSUPPORTED, "SLO schedule with the hierarchical budget");
  if (c->prm.wmove > 0.0 && w.controller == CAPGPU_CTRL_CAPGPU)
    return fail(c, CAPGPU_E_UNSUPPORTED, "SLO schedule with move suppression");
  if (w.slo_period < 0 || (w.slo_period > 0 && !(w.slo_lo >= 0 && w.slo_lo <= w.slo_hi)))
    return fail(c, CAPGPU_E_INVALID, "slo schedule");
  return CAPGPU_OK;
}

static int apply_slo(capgpu_ctx *c, const capgpu_workload &w, cudaStream_t s) {
  DevParams &d = c->dp;
  d.slo = 0;
  d.convex = c->convex_static;
  bool any = false;
  for (int j = 0; j < CAPGPU_MAX_KNOBS; ++j) {
    if (!(w.slo_a[j] >= 0.0) || !(w.slo_b[j] >= 0.0) || !std::isfinite(w.slo_a[j]) || !std::isfinite(w.slo_b[j]))
      return fail(c, CAPGPU_E_INVALID, "slo ratios must be finite and >= 0");
    if (j >= c->N && (w.slo_a[j] != 0.0 || w.slo_b[j] != 0.0))
      return fail(c, CAPGPU_E_INVALID, "slo ratio set for knob %d >= N", j);
    any |= w.slo_a[j] != 0.0 || w.slo_b[j] != 0.0;
  }
  if (!any) return CAPGPU_OK;
  if (w.hierarchical) return fail(c, CAPGPU_E_UNSUPPORTED, "SLO schedule with the hierarchical budget");
  if (c->prm.wmove > 0.0 && w.controller == CAPGPU_CTRL_CAPGPU)
    return fail(c, CAPGPU_E_UNSUPPORTED, "SLO schedule with move suppression");
  if (w.slo_period < 0 || (w.slo_period > 0 && !(w.slo_lo >= 0 && w.slo_lo <= w.slo_hi)))
    return fail(c, CAPGPU_E_INVALID, "slo schedule");
  KnobConst kk[2][CAPGPU_MAX_KNOBS];
  int convex = 1;
  for (int ph = 0; ph < 2; ++ph) {
    uint32_t st = 0u;
    for (int j = 0; j < CAPGPU_MAX_KNOBS; ++j) {
      kk[ph][j] = d.k[j];
      d.q_slo[ph][j] = 0;
      if (j >= c->N) continue;
      const double ratio = ph ? w.slo_b[j] : w.slo_a[j];
      if (ratio > 0.0) {
        const capgpu_knob_bounds &b = c->bounds[j];
        const double step = (b.f_max - b.f_min) / (double)(b.n_levels - 1);
        const double f_req = b.f_max * std::pow(ratio, -1.0 / c->prm.gamma);
        int q = b.n_levels;
        double lev = b.f_max;
        for (int l = 0; l < b.n_levels; ++l) {
          const double lv = b.f_min + (double)l * step;
          if (lv >= f_req) {
            q = l;
            lev = lv;
            break;
          }
        }
        if (q >= b.n_levels) st |= CAPGPU_ST_SLO_INFEASIBLE;
        kk[ph][j].lo = q >= b.n_levels ? b.f_max : (lev > d.k[j].lo ? lev : d.k[j].lo);
        d.q_slo[ph][j] = q;
      }
      convex &= kk[ph][j].lo == kk[ph][j].m ? 1 : 0;
    }
    d.st_slo[ph] = st;
  }
  CK_CUDA(c, cudaMemcpyAsync(c->kdev_slo, kk, sizeof kk, cudaMemcpyHostToDevice, s));
  d.slo = 1;
  d.slo_period = w.slo_period;
  d.slo_lo = w.slo_lo;
  d.slo_hi = w.slo_hi;
  d.convex = convex;
  return CAPGPU_OK;
}

static void apply_workload(DevParams &d, const capgpu_workload &w) {
  d.demand_kind = w.demand_kind;
  d.demand_frac = w.demand_frac;
  d.cap_frac0 = w.cap_frac0;
  d.cap_frac_rand = w.cap_frac_rand;
  d.cap_frac_step = w.cap_frac_step;
  d.cap_period = w.cap_period;
  d.cap_lo = w.cap_lo;
  d.cap_hi = w.cap_hi;
  d.cap_mult = w.cap_mult;
  d.gain0 = 1.0 + w.gain_dlo;
  d.gain_step = w.gain_step;
  d.bl_kind = w.controller;
  d.bl_steps = w.fs_levels;
  d.bl_margin = w.safe_margin;
  d.bl_pole = w.p_pole;
  d.bl_share = w.gpu_share;
}

}  // extern "C"

// Validation of workload + trace, first-call initialisation (plant, S0 sweep,
// virtual period -1), base-cap override and trace slots.  Nothing is launched
// before all arguments are validated.
// Validation of one simulate call (no side effects: nothing launched or written)
static int sim_validate(capgpu_ctx *c, const capgpu_workload *wl, const capgpu_trace *tr, TracePtrs &t) {
  t = TracePtrs{};
  if (wl->demand_kind != 0 && wl->demand_kind != 1) return fail(c, CAPGPU_E_INVALID, "demand_kind");
  if (wl->cap_period < 0 || (wl->cap_period > 0 && !(wl->cap_lo >= 0 && wl->cap_lo <= wl->cap_hi)))
    return fail(c, CAPGPU_E_INVALID, "cap schedule");
  if (wl->hierarchical && c->prm.caps_per_server != 1)
    return fail(c, CAPGPU_E_INVALID, "hierarchical budget needs caps_per_server == 1");
  if (wl->hierarchical && (wl->rack < 1 || wl->rack > 32 || (wl->rack & (wl->rack - 1)) != 0))
    return fail(c, CAPGPU_E_INVALID, "rack must be a power of two <= 32");
  if (wl->hierarchical && (c->shard.n_servers_global % wl->rack != 0 || c->n_srv % wl->rack != 0))
    return fail(c, CAPGPU_E_INVALID, "server count %lld (shard %lld) is not a multiple of the rack size %d (Q16)",
                (long long)c->shard.n_servers_global, (long long)c->n_srv, wl->rack);
  if (!std::isfinite(wl->gain_dlo) || !std::isfinite(wl->gain_step))
    return fail(c, CAPGPU_E_INVALID, "gain_dlo / gain_step must be finite");
  if (wl->hierarchical && (wl->gain_dlo != 0.0 || wl->gain_step != 0.0))
    return fail(c, CAPGPU_E_INVALID, "gain mismatch is not supported with the hierarchical budget");
  if (wl->controller < CAPGPU_CTRL_CAPGPU || wl->controller > CAPGPU_CTRL_CPU_GPU)
    return fail(c, CAPGPU_E_INVALID, "controller");
  if (wl->controller != CAPGPU_CTRL_CAPGPU) {
    if (wl->hierarchical) return fail(c, CAPGPU_E_UNSUPPORTED, "baseline controllers with the hierarchical budget");
    if (wl->fs_levels < 1 || !std::isfinite(wl->safe_margin) || !(wl->p_pole >= 0.0 && wl->p_pole < 1.0))
      return fail(c, CAPGPU_E_INVALID, "baseline parameters (fs_levels >= 1, finite safe_margin, 0 <= p_pole < 1)");
    if (wl->controller == CAPGPU_CTRL_CPU_GPU && !(wl->gpu_share > 0.0 && wl->gpu_share < 1.0))
      return fail(c, CAPGPU_E_INVALID, "CPU+GPU needs 0 < gpu_share < 1");
  }
  if (c->prm.wmove > 0.0 && wl->hierarchical)
    return fail(c, CAPGPU_E_UNSUPPORTED, "move suppression with the hierarchical budget");
  if (c->sim_ready && wl->controller != c->wl.controller)
    return fail(c, CAPGPU_E_ORDER, "the controller is fixed for a simulation: call capgpu_sim_reset first");
  if (tr) {
    OPT_DEV(c, tr->sum_p_d);
    OPT_DEV(c, tr->sumsq_p_d);
    OPT_DEV(c, tr->max_p_d);
    OPT_DEV(c, tr->sum_theta_d);
    OPT_DEV(c, tr->n_viol_d);
    OPT_DEV(c, tr->n_window_d);
    OPT_DEV(c, tr->act_count_d);
    OPT_DEV(c, tr->final_p_d);
    if (tr->n_trace < 0) return fail(c, CAPGPU_E_INVALID, "n_trace < 0");
    if (tr->n_trace > 0) {
      NEED_DEV(c, tr->trace_inst_d);
      OPT_DEV(c, tr->p_d);
      OPT_DEV(c, tr->cap_d);
      OPT_DEV(c, tr->u_d);
      OPT_DEV(c, tr->ahat_d);
      OPT_DEV(c, tr->theta_d);
      OPT_DEV(c, tr->active_d);
      OPT_DEV(c, tr->rank_d);
      OPT_DEV(c, tr->levels_d);
      OPT_DEV(c, tr->status_d);
    }
    OPT_DEV(c, tr->agg_W_d);
    OPT_DEV(c, tr->agg_P_d);
    t.sum_p = tr->sum_p_d;
    t.sumsq_p = tr->sumsq_p_d;
    t.max_p = tr->max_p_d;
    t.sum_theta = tr->sum_theta_d;
    t.final_p = tr->final_p_d;
    t.n_viol = tr->n_viol_d;
    t.n_window = tr->n_window_d;
    t.act_count = tr->act_count_d;
    t.n_miss = tr->n_miss_d;
    t.n_trace = tr->n_trace;
    t.p = tr->p_d;
    t.cap = tr->cap_d;
    t.u = tr->u_d;
    t.ahat = tr->ahat_d;
    t.theta = tr->theta_d;
    t.active = tr->active_d;
    t.status = tr->status_d;
    t.rank = tr->rank_d;
    t.levels = tr->levels_d;
  }
  if (wl->cap_base_d) NEED_DEV(c, wl->cap_base_d);
  OPT_DEV(c, tr ? tr->n_miss_d : nullptr);
  bool any_slo = false;
  return slo_validate(c, *wl, &any_slo);
}

// Side effects of a validated simulate call: SLO bounds, workload constants,
// first-call initialisation (identify + virtual period -1), cap bases, trace slots.
static int sim_apply(capgpu_ctx *c, const capgpu_workload *wl, const capgpu_trace *tr, const TracePtrs &t,
                     cudaStream_t s) {
  {
    int rc = apply_slo(c, *wl, s);
    if (rc) return rc;
  }
  apply_workload(c->dp, *wl);
  if (!c->sim_ready) {
    int rc = ensure_servers(c, s);
    if (rc) return rc;
    int rows = 0;
    for (int j = 0; j < c->N; ++j) rows += c->bounds[j].n_levels;
    int e = c->L.identify(c->dp, c->st, nullptr, nullptr, rows, nullptr, nullptr, nullptr, s);
    if (e) return cuda_fail(c, (cudaError_t)e, "identify (simulate init)");
    c->has_prior = true;
    e = c->L.init_instances(c->dp, c->st, s);
    if (e) return cuda_fail(c, (cudaError_t)e, "init_instances");
    c->sim_ready = true;
    c->k_global = 0;
    c->wl = *wl;
  }
  if (wl->cap_base_d)
    CK_CUDA(c, cudaMemcpyAsync(c->st.cap_base, wl->cap_base_d, sizeof(double) * c->n_inst,
                               cudaMemcpyDeviceToDevice, s));
  if (t.n_trace > 0) {
    k_trace_slots<<<grid_for(c->n_inst, 256), 256, 0, s>>>(c->st.trace_slot, c->n_inst, nullptr, 0);
    k_trace_slots_set<<<grid_for(t.n_trace, 256), 256, 0, s>>>(c->st.trace_slot, c->n_inst, tr->trace_inst_d,
                                                               t.n_trace);
    CK_CUDA(c, cudaGetLastError());
  }
  return CAPGPU_OK;
}

// S5 setup for a set of shards stepping together (1 = this process only,
// NCCL if world > 1; n > 1 = loopback shards on one GPU): allocation, w_i(0),
// cluster constants (Pmin_tot, Pmax_tot -> B_c) and W(0), all through the
// same deterministic block-sum / all-reduce / tree path as every period.
static int budget_setup_group(capgpu_ctx **cs, int n, const capgpu_workload &wl, cudaStream_t s) {
  Budget *bs[64];
  for (int q = 0; q < n; ++q) {
    capgpu_ctx *c = cs[q];
    bs[q] = &c->budget;
    if (c->prm.caps_per_server != 1) return fail(c, CAPGPU_E_INVALID, "hierarchical budget needs caps_per_server == 1");
    int rc = budget_alloc(c->budget, c->dp, wl, c->shard, c->err);
    if (!rc) rc = budget_setup_local(c->budget, c->dp, c->st, c->L, s, c->err);
    if (rc) return rc;
  }
  int rc = budget_reduce(bs, n, true, s, cs[0]->err);
  for (int q = 0; q < n && !rc; ++q) rc = budget_tree(*bs[q], nullptr, nullptr, 0, s, cs[q]->err);
  for (int q = 0; q < n && !rc; ++q) rc = budget_finish_setup(*bs[q], s, cs[q]->err);
  if (!rc) rc = budget_reduce(bs, n, false, s, cs[0]->err);
  for (int q = 0; q < n && !rc; ++q) rc = budget_tree(*bs[q], nullptr, nullptr, 0, s, cs[q]->err);
  if (rc) return rc;
  for (int q = 0; q < n; ++q) bs[q]->ready = true;
  return CAPGPU_OK;
}

extern "C" {

int capgpu_simulate(capgpu_ctx *c, int64_t periods, const capgpu_workload *wl, const capgpu_trace *tr,
                    void *stream) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  if (!wl) return fail(c, CAPGPU_E_INVALID, "workload is NULL");
  if (periods < 1 || periods > (1ll << 30)) return fail(c, CAPGPU_E_INVALID, "periods out of range");
  if (tr && tr->n_trace > 0 && periods > (1ll << 24))
    return fail(c, CAPGPU_E_INVALID, "traced runs are limited to 2^24 periods");
  if (wl->hierarchical && c->shard.world > 1 && !c->budget.comm)
    return fail(c, CAPGPU_E_INVALID, "world > 1 hierarchical runs need NCCL (shard.use_nccl) or capgpu_simulate_group");
  TracePtrs t;
  cudaStream_t s = (cudaStream_t)stream;
  int rc = sim_validate(c, wl, tr, t);
  if (rc) return rc;
  rc = sim_apply(c, wl, tr, t, s);
  if (rc) return rc;
  if (wl->hierarchical) {
    if (!c->budget.ready) {
      capgpu_ctx *cs[1] = {c};
      rc = budget_setup_group(cs, 1, *wl, s);
      if (rc) return rc;
    }
    rc = budget_simulate(c->budget, c->dp, c->st, t, c->L, c->k_global, periods, tr ? tr->agg_W_d : nullptr,
                         tr ? tr->agg_P_d : nullptr, s, c->err);
    if (rc) return rc;
  } else if (wl->controller != CAPGPU_CTRL_CAPGPU) {
    int e = c->L.baseline(c->dp, c->st, t, c->k_global, (int)periods, s);
    if (e) return cuda_fail(c, (cudaError_t)e, "simulate (baseline controller)");
  } else {
    int e = c->L.simulate(c->dp, c->st, t, c->k_global, (int)periods, s);
    if (e) return cuda_fail(c, (cudaError_t)e, "simulate");
  }
  c->k_global += periods;
  return CAPGPU_OK;
}

int capgpu_simulate_group(capgpu_ctx **ctxs, int32_t n_ctx, int64_t periods, const capgpu_workload *wl,
                          const capgpu_trace *const *trs, void *stream) {
  if (!ctxs || n_ctx < 1 || n_ctx > 64) return fail(nullptr, CAPGPU_E_INVALID, "bad context list");
  if (!wl || !wl->hierarchical) return fail(nullptr, CAPGPU_E_INVALID, "group simulation is for the hierarchical budget");
  if (periods < 1 || periods > (1ll << 30)) return fail(nullptr, CAPGPU_E_INVALID, "periods out of range");
  for (int q = 0; q < n_ctx; ++q) {
    capgpu_ctx *c = ctxs[q];
    if (!c) return fail(nullptr, CAPGPU_E_INVALID, "NULL context in group");
    if (c->shard.world != n_ctx || c->shard.rank != q || c->budget.comm)
      return fail(c, CAPGPU_E_INVALID, "group member %d must be rank %d of world %d without NCCL", q, q, n_ctx);
    if (c->N != ctxs[0]->N || c->M != ctxs[0]->M || c->shard.n_servers_global != ctxs[0]->shard.n_servers_global)
      return fail(c, CAPGPU_E_INVALID, "group members must share N, M and the global server count");
  }
  cudaStream_t s = (cudaStream_t)stream;
  TracePtrs t[64];
  // every member is validated before any member is initialised or launched
  for (int q = 0; q < n_ctx; ++q) {
    capgpu_ctx *c = ctxs[q];
    if (c->wl.hierarchical && c->sim_ready && c->k_global != ctxs[0]->k_global)
      return fail(c, CAPGPU_E_ORDER, "group members are out of step");
    int rc = sim_validate(c, wl, trs ? trs[q] : nullptr, t[q]);
    if (rc) return rc;
  }
  for (int q = 0; q < n_ctx; ++q) {
    int rc = sim_apply(ctxs[q], wl, trs ? trs[q] : nullptr, t[q], s);
    if (rc) return rc;
  }
  if (!ctxs[0]->budget.ready) {
    int rc = budget_setup_group(ctxs, n_ctx, *wl, s);
    if (rc) return rc;
  }
  Budget *bs[64];
  for (int q = 0; q < n_ctx; ++q) bs[q] = &ctxs[q]->budget;
  const int64_t k0 = ctxs[0]->k_global;
  DevParams Ps[64];
  StatePtrs Ss[64];
  Launchers Ls[64];
  double *aW[64], *aP[64];
  for (int q = 0; q < n_ctx; ++q) {
    Ps[q] = ctxs[q]->dp;
    Ss[q] = ctxs[q]->st;
    Ls[q] = ctxs[q]->L;
    const capgpu_trace *tq = trs ? trs[q] : nullptr;
    aW[q] = tq ? tq->agg_W_d : nullptr;
    aP[q] = tq ? tq->agg_P_d : nullptr;
  }
  {
    int rc = budget_simulate_group(bs, n_ctx, Ps, Ss, t, Ls, k0, periods, aW, aP, s, ctxs[0]->err);
    if (rc) return rc;
  }
  for (int q = 0; q < n_ctx; ++q) ctxs[q]->k_global += periods;
  return CAPGPU_OK;
}

int capgpu_sim_state(capgpu_ctx *c, double *fbar_d, double *acc_d, double *thr_d, double *p_d, void *stream) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  OPT_DEV(c, fbar_d);
  OPT_DEV(c, acc_d);
  OPT_DEV(c, thr_d);
  OPT_DEV(c, p_d);
  cudaStream_t s = (cudaStream_t)stream;
  const size_t nb = sizeof(double) * c->N * c->n_inst;
  if (fbar_d) CK_CUDA(c, cudaMemcpyAsync(fbar_d, c->st.fbar, nb, cudaMemcpyDeviceToDevice, s));
  if (acc_d) CK_CUDA(c, cudaMemcpyAsync(acc_d, c->st.acc, nb, cudaMemcpyDeviceToDevice, s));
  if (thr_d) CK_CUDA(c, cudaMemcpyAsync(thr_d, c->st.thr, nb, cudaMemcpyDeviceToDevice, s));
  if (p_d) CK_CUDA(c, cudaMemcpyAsync(p_d, c->st.p, sizeof(double) * c->n_inst, cudaMemcpyDeviceToDevice, s));
  return CAPGPU_OK;
}

// ---- state setter and checkpoint / resume

// |acc_j| <= step_j / 2 (+ rounding) is the modulator invariant the plant relies
// on (plant_pair); flags violations of a candidate acc array
__global__ void k_check_acc(const double *acc, int64_t n, const KnobConst *k, int N, int *bad) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  for (int j = 0; j < N; ++j) {
    const double a = acc[(int64_t)j * n + i];
    if (!(fabs(a) <= 0.5 * k[j].step * (1.0 + 1e-9))) atomicOr(bad, 1);
  }
}
__global__ void k_check_finite(const double *x, int64_t n, int *bad) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n && !isfinite(x[i])) atomicOr(bad, 2);
}

int capgpu_set_state(capgpu_ctx *c, const double *fbar_d, const double *acc_d, const double *thr_d,
                     const double *p_d, void *stream) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  if (!c->sim_ready) return fail(c, CAPGPU_E_ORDER, "simulation not initialised (call capgpu_simulate first)");
  OPT_DEV(c, fbar_d);
  OPT_DEV(c, acc_d);
  OPT_DEV(c, thr_d);
  OPT_DEV(c, p_d);
  cudaStream_t s = (cudaStream_t)stream;
  const int64_t nn = (int64_t)c->N * c->n_inst;
  // validation before anything is written: finite values, |acc| <= step / 2
  int *bad = nullptr;
  CK_CUDA(c, cudaMalloc(&bad, sizeof(int)));
  int hbad = 0;
  cudaError_t e = cudaMemsetAsync(bad, 0, sizeof(int), s);
  const double *arrs[4] = {fbar_d, acc_d, thr_d, p_d};
  const int64_t lens[4] = {nn, nn, nn, c->n_inst};
  for (int q = 0; q < 4 && e == cudaSuccess; ++q)
    if (arrs[q]) {
      k_check_finite<<<grid_for(lens[q], 256), 256, 0, s>>>(arrs[q], lens[q], bad);
      e = cudaGetLastError();
    }
  if (e == cudaSuccess && acc_d) {
    k_check_acc<<<grid_for(c->n_inst, 256), 256, 0, s>>>(acc_d, c->n_inst, c->dp.k_dev, c->N, bad);
    e = cudaGetLastError();
  }
  if (e == cudaSuccess) e = cudaMemcpyAsync(&hbad, bad, sizeof(int), cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  cudaFree(bad);
  if (e != cudaSuccess) return cuda_fail(c, e, "set_state validation");
  if (hbad & 2) return fail(c, CAPGPU_E_INVALID, "set_state: non-finite value");
  if (hbad & 1) return fail(c, CAPGPU_E_INVALID, "set_state: |acc| exceeds half a grid step (modulator invariant)");
  const size_t nb = sizeof(double) * (size_t)nn;
  if (fbar_d) CK_CUDA(c, cudaMemcpyAsync(c->st.fbar, fbar_d, nb, cudaMemcpyDeviceToDevice, s));
  if (acc_d) CK_CUDA(c, cudaMemcpyAsync(c->st.acc, acc_d, nb, cudaMemcpyDeviceToDevice, s));
  if (thr_d) CK_CUDA(c, cudaMemcpyAsync(c->st.thr, thr_d, nb, cudaMemcpyDeviceToDevice, s));
  if (p_d) CK_CUDA(c, cudaMemcpyAsync(c->st.p, p_d, sizeof(double) * c->n_inst, cudaMemcpyDeviceToDevice, s));
  return CAPGPU_OK;
}

// Checkpoint blob: a fixed header, the whole state workspace (model, plant,
// warm starts, server constants, grid tables -- identical for identical
// create() arguments), and for the hierarchical budget its per-server weights
// and cluster aggregates.
namespace {
struct CkptHeader {
  uint64_t magic;
  int64_t n_srv, n_inst, ws_bytes, k_global, budget_doubles;
  int32_t N, M, P, flags;
  capgpu_workload wl;
  double B_c, pmin_tot, pmax_tot;
};
constexpr uint64_t kCkptMagic = 0x3150434B55504743ull;  // "CGPUKCP1"
int64_t budget_doubles(const capgpu_ctx *c) { return c->budget.ready ? c->n_srv + 4 : 0; }
}  // namespace

int64_t capgpu_checkpoint_bytes(const capgpu_ctx *c) {
  if (!c) return 0;
  const int64_t hb = ((int64_t)sizeof(CkptHeader) + 255) & ~(int64_t)255;
  return hb + c->ws_bytes + 8 * budget_doubles(c);
}

int capgpu_checkpoint_save(capgpu_ctx *c, void *dst_d, void *stream) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  NEED_DEV(c, dst_d);
  cudaStream_t s = (cudaStream_t)stream;
  CkptHeader h{};
  h.magic = kCkptMagic;
  h.n_srv = c->n_srv;
  h.n_inst = c->n_inst;
  h.ws_bytes = c->ws_bytes;
  h.k_global = c->k_global;
  h.budget_doubles = budget_doubles(c);
  h.N = c->N;
  h.M = c->M;
  h.P = c->P;
  h.flags = (c->servers_ready ? 1 : 0) | (c->has_prior ? 2 : 0) | (c->sim_ready ? 4 : 0) | (c->budget.ready ? 8 : 0);
  h.wl = c->wl;
  h.B_c = c->budget.B_c;
  h.pmin_tot = c->budget.pmin_tot;
  h.pmax_tot = c->budget.pmax_tot;
  const int64_t hb = ((int64_t)sizeof(CkptHeader) + 255) & ~(int64_t)255;
  char *d = (char *)dst_d;
  CK_CUDA(c, cudaMemcpyAsync(d + hb, c->ws, (size_t)c->ws_bytes, cudaMemcpyDeviceToDevice, s));
  if (h.budget_doubles) {
    double *bd = (double *)(d + hb + c->ws_bytes);
    CK_CUDA(c, cudaMemcpyAsync(bd, c->budget.srv_w, sizeof(double) * c->n_srv, cudaMemcpyDeviceToDevice, s));
    CK_CUDA(c, cudaMemcpyAsync(bd + c->n_srv, c->budget.agg, sizeof(double) * 2, cudaMemcpyDeviceToDevice, s));
    CK_CUDA(c, cudaMemcpyAsync(bd + c->n_srv + 2, c->budget.consts, sizeof(double) * 2, cudaMemcpyDeviceToDevice, s));
  }
  // the header comes from host memory: synchronous, so h may go out of scope
  CK_CUDA(c, cudaStreamSynchronize(s));
  CK_CUDA(c, cudaMemcpy(d, &h, sizeof h, cudaMemcpyHostToDevice));
  return CAPGPU_OK;
}

int capgpu_checkpoint_load(capgpu_ctx *c, const void *src_d, void *stream) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  NEED_DEV(c, src_d);
  cudaStream_t s = (cudaStream_t)stream;
  CkptHeader h{};
  CK_CUDA(c, cudaStreamSynchronize(s));
  CK_CUDA(c, cudaMemcpy(&h, src_d, sizeof h, cudaMemcpyDeviceToHost));
  if (h.magic != kCkptMagic) return fail(c, CAPGPU_E_INVALID, "checkpoint: bad magic");
  if (h.n_srv != c->n_srv || h.n_inst != c->n_inst || h.ws_bytes != c->ws_bytes || h.N != c->N || h.M != c->M ||
      h.P != c->P)
    return fail(c, CAPGPU_E_INVALID, "checkpoint: shape differs from this context (create it with the same arguments)");
  if ((h.flags & 8) && !c->budget.srv_w)
    return fail(c, CAPGPU_E_ORDER, "checkpoint holds a hierarchical budget: run one capgpu_simulate with the "
                                   "hierarchical workload (or simulate_group) before loading");
  const int64_t hb = ((int64_t)sizeof(CkptHeader) + 255) & ~(int64_t)255;
  const char *d = (const char *)src_d;
  CK_CUDA(c, cudaMemcpyAsync(c->ws, d + hb, (size_t)c->ws_bytes, cudaMemcpyDeviceToDevice, s));
  if (h.budget_doubles) {
    const double *bd = (const double *)(d + hb + c->ws_bytes);
    CK_CUDA(c, cudaMemcpyAsync(c->budget.srv_w, bd, sizeof(double) * c->n_srv, cudaMemcpyDeviceToDevice, s));
    CK_CUDA(c, cudaMemcpyAsync(c->budget.agg, bd + c->n_srv, sizeof(double) * 2, cudaMemcpyDeviceToDevice, s));
    CK_CUDA(c, cudaMemcpyAsync(c->budget.consts, bd + c->n_srv + 2, sizeof(double) * 2, cudaMemcpyDeviceToDevice, s));
    c->budget.B_c = h.B_c;
    c->budget.pmin_tot = h.pmin_tot;
    c->budget.pmax_tot = h.pmax_tot;
    c->budget.ready = true;
  }
  c->servers_ready = h.flags & 1;
  c->has_prior = (h.flags & 2) != 0;
  c->sim_ready = (h.flags & 4) != 0;
  c->k_global = h.k_global;
  c->wl = h.wl;
  return CAPGPU_OK;
}

int capgpu_sim_caps(capgpu_ctx *c, double *cap_base_d, void *stream) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  NEED_DEV(c, cap_base_d);
  if (!c->sim_ready) return fail(c, CAPGPU_E_ORDER, "simulation not initialised");
  CK_CUDA(c, cudaMemcpyAsync(cap_base_d, c->st.cap_base, sizeof(double) * c->n_inst, cudaMemcpyDeviceToDevice,
                             (cudaStream_t)stream));
  return CAPGPU_OK;
}

int capgpu_debug_gen(capgpu_ctx *c, int64_t k, int32_t demand_kind, double demand_frac, double *a_true_d,
                     double *thr_max_d, double *c_true_d, double *dem_d, double *noise_d, void *stream) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  NEED_DEV(c, a_true_d);
  NEED_DEV(c, thr_max_d);
  NEED_DEV(c, c_true_d);
  NEED_DEV(c, dem_d);
  NEED_DEV(c, noise_d);
  DevParams d = c->dp;
  d.demand_kind = demand_kind;
  d.demand_frac = demand_frac;
  int e = c->L.debug_gen(d, c->st, k, a_true_d, thr_max_d, c_true_d, dem_d, noise_d, (cudaStream_t)stream);
  if (e) return cuda_fail(c, (cudaError_t)e, "debug_gen");
  return CAPGPU_OK;
}

// FP64 pipe microbenchmark: 8 independent DFMA chains per thread.
__global__ void k_dfma_peak(double *out, int iters, double a, double b) {
  double x[8];
#pragma unroll
  for (int c = 0; c < 8; ++c) x[c] = threadIdx.x * 1e-3 + c;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int c = 0; c < 8; ++c) x[c] = fma(x[c], a, b);
  }
  double s = 0;
#pragma unroll
  for (int c = 0; c < 8; ++c) s += x[c];
  if (s == 12345.678) out[0] = s;
}

int capgpu_debug_phase_counters(capgpu_ctx *c, long long *counters_d) {
  if (!c) return fail(nullptr, CAPGPU_E_INVALID, "ctx is NULL");
  OPT_DEV(c, counters_d);
  c->dp.phase = counters_d;
  return CAPGPU_OK;
}

int capgpu_fp64_peak(double *tflops_out, void *stream) {
  if (!tflops_out) return fail(nullptr, CAPGPU_E_INVALID, "out is NULL");
  cudaStream_t s = (cudaStream_t)stream;
  int dev = 0, sms = 0;
  CK_CUDA(nullptr, cudaGetDevice(&dev));
  CK_CUDA(nullptr, cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  double *d = nullptr;
  CK_CUDA(nullptr, cudaMalloc(&d, 64));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int blocks = sms * 4, thr = 256, iters = 1 << 14;
  k_dfma_peak<<<blocks, thr, 0, s>>>(d, 64, 1.0000001, 1e-9);
  cudaEventRecord(e0, s);
  for (int r = 0; r < 5; ++r) k_dfma_peak<<<blocks, thr, 0, s>>>(d, iters, 1.0000001, 1e-9);
  cudaEventRecord(e1, s);
  cudaError_t e = cudaEventSynchronize(e1);
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaFree(d);
  if (e != cudaSuccess) return cuda_fail(nullptr, e, "fp64 peak");
  *tflops_out = 5.0 * blocks * thr * (double)iters * 8 * 2 / (ms * 1e-3) / 1e12;
  return CAPGPU_OK;
}

}  // extern "C"
