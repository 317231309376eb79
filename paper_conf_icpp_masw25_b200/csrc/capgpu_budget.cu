// capgpu_budget.cu -- S5 hierarchical budget (cfg 4, Q16): deterministic
// cluster aggregates and the per-period loop around k_period.
//
// Determinism: each 1024-server block sum is computed by exactly one GPU in a
// fixed order (CTA partials in index order); the all-reduce runs over a
// zero-padded vector in which every element has exactly one non-zero
// contributor, so any reduction order (NCCL ring/tree/NVLS, loopback) is exact;
// the cluster sum is a fixed pairwise tree over the padded block vector.  The
// result is bitwise identical on every GPU and for 1, 2, 4 or 8 GPUs.
#include <cstdio>
#include <cstdlib>
#include <cstring>

#define CAPGPU_UNUSED(x) (void)(x)

#include <nccl.h>

#include "capgpu_budget.cuh"

namespace capgpu {

__global__ void k_block_sums(const double *part, int64_t n_cta, int64_t nb_local, int64_t blk_begin, int64_t nb_g,
                             double *send) {
  const int64_t b = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= nb_local) return;
  double a = 0.0, c = 0.0;
#pragma unroll
  for (int q = 0; q < kCtasPerBlock; ++q) {
    const int64_t ci = b * kCtasPerBlock + q;
    if (ci < n_cta) {
      a += part[ci];
      c += part[n_cta + ci];
    }
  }
  send[blk_begin + b] = a;
  send[nb_g + blk_begin + b] = c;
}

// Fixed pairwise tree over the zero-padded vector (length len = 2^m >= nb_g):
// for h = len/2 .. 1: v[i] += v[i + h], i < h.  Same order as
// capgpu_tree_sum_host.  Single CTA; two vectors (w, p) side by side.
__global__ void k_tree(const double *recv, int64_t nb_g, int64_t len, double *scratch, double *agg, double *tW,
                       double *tP, int kk, int64_t *kdev) {
  if (kdev) kk = (int)kdev[1];  // graph replay: call period from device memory, advanced below
  for (int64_t i = threadIdx.x; i < len; i += blockDim.x) {
    scratch[i] = i < nb_g ? recv[i] : 0.0;
    scratch[len + i] = i < nb_g ? recv[nb_g + i] : 0.0;
  }
  __syncthreads();
  for (int64_t h = len / 2; h >= 1; h /= 2) {
    for (int64_t i = threadIdx.x; i < h; i += blockDim.x) {
      scratch[i] = scratch[i] + scratch[i + h];
      scratch[len + i] = scratch[len + i] + scratch[len + i + h];
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    agg[0] = scratch[0];
    agg[1] = scratch[len];
    if (tW) tW[kk] = scratch[0];
    if (tP) tP[kk] = scratch[len];
    if (kdev) kdev[1] = kk + 1;  // every thread read kdev[1] before the first __syncthreads
  }
}

__global__ void k_set_period(int64_t *kdev, int64_t k0) {
  kdev[0] = k0;
  kdev[1] = 0;
}

__global__ void k_accumulate(double *dst, const double *src, int64_t n, int first) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) dst[i] = first ? src[i] : dst[i] + src[i];
}

static BudgetDev dev_view(Budget &b) {
  BudgetDev d{};
  d.agg = b.agg;
  d.srv_w = b.srv_w;
  d.cta_part = b.part;
  d.B_c = b.B_c;
  d.pmin_tot = b.pmin_tot;
  d.rack_frac = b.rack_frac;
  d.rack = b.rack;
  d.kdev = b.graph_mode ? b.kdev : nullptr;
  return d;
}

#define BCK(call)                                                               \
  do {                                                                          \
    cudaError_t e_ = (call);                                                    \
    if (e_ != cudaSuccess) {                                                    \
      snprintf(err, 512, "%s: %s", #call, cudaGetErrorString(e_));              \
      return CAPGPU_E_CUDA;                                                     \
    }                                                                           \
  } while (0)

int budget_init_nccl(Budget &b, const uint8_t *id, int world, int rank, char *err) {
  ncclUniqueId uid;
  std::memcpy(&uid, id, sizeof uid);
  ncclComm_t comm;
  ncclResult_t r = ncclCommInitRank(&comm, world, uid, rank);
  if (r != ncclSuccess) {
    snprintf(err, 512, "ncclCommInitRank: %s", ncclGetErrorString(r));
    return CAPGPU_E_NCCL;
  }
  b.comm = comm;
  b.world = world;
  b.rank = rank;
  return CAPGPU_OK;
}

void budget_free(Budget &b) {
  if (b.comm) ncclCommDestroy((ncclComm_t)b.comm);
  b.comm = nullptr;
  double *bufs[] = {b.srv_w, b.part, b.part_c, b.send, b.recv, b.scratch, b.agg, b.consts};
  for (double *p : bufs)
    if (p) cudaFree(p);
  b.srv_w = b.part = b.part_c = b.send = b.recv = b.scratch = b.agg = b.consts = nullptr;
  if (b.kdev) cudaFree(b.kdev);
  b.kdev = nullptr;
  b.ready = false;
}

int budget_alloc(Budget &b, const DevParams &P, const capgpu_workload &wl, const capgpu_shard &sh, char *err) {
  if (wl.rack < 1 || wl.rack > 32 || (wl.rack & (wl.rack - 1)) != 0) {
    snprintf(err, 512, "rack must be a power of two <= 32");
    return CAPGPU_E_INVALID;
  }
  if (sh.n_servers_global % wl.rack != 0 || P.n_srv % wl.rack != 0) {  // whole racks (Q16; the oracle's rule too)
    snprintf(err, 512, "server count %lld (shard %lld) is not a multiple of the rack size %d",
             (long long)sh.n_servers_global, (long long)P.n_srv, wl.rack);
    return CAPGPU_E_INVALID;
  }
  if (wl.block != 0 && wl.block != kBudgetBlock) {
    snprintf(err, 512, "reduction block must be %d servers", kBudgetBlock);
    return CAPGPU_E_UNSUPPORTED;
  }
  if (!(wl.cluster_frac >= 0.0) || !(wl.rack_frac > 0.0)) {
    snprintf(err, 512, "cluster_frac / rack_frac out of range");
    return CAPGPU_E_INVALID;
  }
  if (sh.srv_begin % kBudgetBlock != 0) {
    snprintf(err, 512, "hierarchical shards must start on a %d-server block", kBudgetBlock);
    return CAPGPU_E_INVALID;
  }
  if (b.srv_w) {  // re-setup after capgpu_sim_reset: keep the communicator
    void *comm = b.comm;
    b.comm = nullptr;
    budget_free(b);
    b.comm = comm;
  }
  b.world = sh.world;
  b.rank = sh.rank;
  b.rack = wl.rack;
  b.rack_frac = wl.rack_frac;
  b.cluster_frac = wl.cluster_frac;
  b.n_cta = (P.n_srv + kCta - 1) / kCta;
  b.nb_local = (P.n_srv + kBudgetBlock - 1) / kBudgetBlock;
  b.blk_begin = sh.srv_begin / kBudgetBlock;
  b.nb_g = (sh.n_servers_global + kBudgetBlock - 1) / kBudgetBlock;
  b.tree_len = 1;
  while (b.tree_len < b.nb_g) b.tree_len *= 2;
  BCK(cudaMalloc(&b.srv_w, sizeof(double) * P.n_srv));
  BCK(cudaMalloc(&b.part, sizeof(double) * 2 * b.n_cta));
  BCK(cudaMalloc(&b.part_c, sizeof(double) * 2 * b.n_cta));
  BCK(cudaMalloc(&b.send, sizeof(double) * 2 * b.nb_g));
  BCK(cudaMalloc(&b.recv, sizeof(double) * 2 * b.nb_g));
  BCK(cudaMalloc(&b.scratch, sizeof(double) * 2 * b.tree_len));
  BCK(cudaMalloc(&b.agg, sizeof(double) * 2));
  BCK(cudaMalloc(&b.consts, sizeof(double) * 2));
  BCK(cudaMalloc(&b.kdev, sizeof(int64_t) * 2));
  BCK(cudaMemset(b.send, 0, sizeof(double) * 2 * b.nb_g));
  BCK(cudaMemset(b.recv, 0, sizeof(double) * 2 * b.nb_g));
  return CAPGPU_OK;
}

// Local part of the setup: w_i(0) and the CTA partials of (w, p) and of
// (pmin, pmax); block sums of the constants into `send`.
int budget_setup_local(Budget &b, const DevParams &P, const StatePtrs &st, const Launchers &L, cudaStream_t s,
                       char *err) {
  BudgetDev d = dev_view(b);
  int e = L.budget_init(P, st, d, b.part_c, s);
  if (e) {
    snprintf(err, 512, "budget_init: %s", cudaGetErrorString((cudaError_t)e));
    return CAPGPU_E_CUDA;
  }
  k_block_sums<<<grid_for(b.nb_local, 128), 128, 0, s>>>(b.part_c, b.n_cta, b.nb_local, b.blk_begin, b.nb_g,
                                                          b.send);
  BCK(cudaGetLastError());
  return CAPGPU_OK;
}

// All-reduce of the zero-padded block vectors of n budgets: NCCL (one budget
// per process), identity (one shard), or an in-process loopback sum (several
// shards of one GPU).  Exact: one non-zero contributor per element.
int budget_reduce(Budget **bs, int n, bool /*consts*/, cudaStream_t s, char *err) {
  const int64_t cnt = 2 * bs[0]->nb_g;
  if (n == 1) {
    Budget &b = *bs[0];
    if (b.world > 1 && !b.comm) {
      snprintf(err, 512, "world > 1 needs an NCCL communicator (capgpu_shard.use_nccl) or simulate_group");
      return CAPGPU_E_INVALID;
    }
    if (b.comm) {  // any communicator, also a one-rank one (the single-GPU test of the NCCL path)
      ncclResult_t r = ncclAllReduce(b.send, b.recv, (size_t)cnt, ncclDouble, ncclSum, (ncclComm_t)b.comm, s);
      if (r != ncclSuccess) {
        snprintf(err, 512, "ncclAllReduce: %s", ncclGetErrorString(r));
        return CAPGPU_E_NCCL;
      }
    } else {
      BCK(cudaMemcpyAsync(b.recv, b.send, sizeof(double) * cnt, cudaMemcpyDeviceToDevice, s));
    }
    return CAPGPU_OK;
  }
  for (int q = 0; q < n; ++q) {
    k_accumulate<<<grid_for(cnt, 256), 256, 0, s>>>(bs[0]->recv, bs[q]->send, cnt, q == 0);
    BCK(cudaGetLastError());
  }
  for (int q = 1; q < n; ++q)
    BCK(cudaMemcpyAsync(bs[q]->recv, bs[0]->recv, sizeof(double) * cnt, cudaMemcpyDeviceToDevice, s));
  return CAPGPU_OK;
}

int budget_tree(Budget &b, double *agg_W, double *agg_P, int kk, cudaStream_t s, char *err) {
  k_tree<<<1, 1024, 0, s>>>(b.recv, b.nb_g, b.tree_len, b.scratch, b.agg, agg_W, agg_P, kk,
                            b.graph_mode ? b.kdev : nullptr);
  BCK(cudaGetLastError());
  return CAPGPU_OK;
}

// After the constants were reduced and tree-summed into b.agg: read them,
// form B_c (Q16) and put the (w, p) block sums of instant 0 into `send`.
int budget_finish_setup(Budget &b, cudaStream_t s, char *err) {
  double h[2];
  BCK(cudaMemcpyAsync(h, b.agg, sizeof h, cudaMemcpyDeviceToHost, s));
  BCK(cudaStreamSynchronize(s));
  b.pmin_tot = h[0];
  b.pmax_tot = h[1];
  b.B_c = b.pmin_tot + b.cluster_frac * (b.pmax_tot - b.pmin_tot);
  BCK(cudaMemcpyAsync(b.consts, b.agg, sizeof h, cudaMemcpyDeviceToDevice, s));
  k_block_sums<<<grid_for(b.nb_local, 128), 128, 0, s>>>(b.part, b.n_cta, b.nb_local, b.blk_begin, b.nb_g, b.send);
  BCK(cudaGetLastError());
  return CAPGPU_OK;
}

int budget_period_local(Budget &b, const DevParams &P, const StatePtrs &st, const TracePtrs &tr, const Launchers &L,
                        int64_t k, int kk, int K, cudaStream_t s, char *err) {
  BudgetDev d = dev_view(b);
  int e = L.period(P, st, d, tr, k, kk, K, s);
  if (e) {
    snprintf(err, 512, "period: %s", cudaGetErrorString((cudaError_t)e));
    return CAPGPU_E_CUDA;
  }
  k_block_sums<<<grid_for(b.nb_local, 128), 128, 0, s>>>(b.part, b.n_cta, b.nb_local, b.blk_begin, b.nb_g, b.send);
  BCK(cudaGetLastError());
  return CAPGPU_OK;
}

int budget_simulate(Budget &b, const DevParams &P, const StatePtrs &st, const TracePtrs &tr, const Launchers &L,
                    int64_t k0, int64_t K, double *agg_W, double *agg_P, cudaStream_t s, char *err) {
  Budget *bs[1] = {&b};
  CAPGPU_UNUSED(bs);
  return budget_simulate_group(bs, 1, &P, &st, &tr, &L, k0, K, agg_W ? &agg_W : nullptr, agg_P ? &agg_P : nullptr, s,
                               err);
}

// The K periods of a call for n budgets (1 = one context on its GPU, NCCL if
// world > 1; n > 1 = loopback shards of one GPU).  One period = k_period +
// block sums of every context, the all-reduce, every context's tree.  With
// CUDA-graph replay (default for K >= 8; env CAPGPU_NO_GRAPH=1 disables) the
// period's launches are captured once (R periods unrolled, R <= 16) with the
// period index read from device memory (k_set_period / k_tree), and the
// graph is replayed: no per-period host launch gaps.  Same kernels, same
// order: bitwise identical results.
int budget_simulate_group(Budget **bs, int n, const DevParams *P, const StatePtrs *st, const TracePtrs *tr,
                          const Launchers *L, int64_t k0, int64_t K, double **agg_W, double **agg_P, cudaStream_t s,
                          char *err) {
  auto period = [&](int64_t kk) -> int {
    for (int q = 0; q < n; ++q) {
      int rc = budget_period_local(*bs[q], P[q], st[q], tr[q], L[q], k0 + kk, (int)kk, (int)K, s, err);
      if (rc) return rc;
    }
    int rc = budget_reduce(bs, n, false, s, err);
    if (rc) return rc;
    for (int q = 0; q < n; ++q) {
      rc = budget_tree(*bs[q], agg_W ? agg_W[q] : nullptr, agg_P ? agg_P[q] : nullptr, (int)kk, s, err);
      if (rc) return rc;
    }
    return CAPGPU_OK;
  };
  const char *ng = getenv("CAPGPU_NO_GRAPH");
  const bool graph = K >= 8 && !(ng && ng[0] && ng[0] != '0');
  if (!graph) {
    for (int64_t kk = 0; kk < K; ++kk) {
      int rc = period(kk);
      if (rc) return rc;
    }
    return CAPGPU_OK;
  }
  for (int q = 0; q < n; ++q) {
    k_set_period<<<1, 1, 0, s>>>(bs[q]->kdev, k0);
    BCK(cudaGetLastError());
    bs[q]->graph_mode = true;
  }
  const int R = (int)(K < 16 ? K : 16);
  cudaStream_t cs;
  BCK(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
  cudaGraph_t g = nullptr;
  cudaGraphExec_t ge = nullptr;
  int rc = CAPGPU_OK;
  cudaError_t e = cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal);
  if (e == cudaSuccess) {
    cudaStream_t s_save = s;
    s = cs;
    for (int r = 0; r < R && !rc; ++r) rc = period(r);  // kk in the captured launches is overridden by kdev
    s = s_save;
    e = cudaStreamEndCapture(cs, &g);
  }
  if (!rc && e == cudaSuccess) e = cudaGraphInstantiate(&ge, g, 0);
  if (!rc && e == cudaSuccess) {
    int64_t done = 0;
    for (; done + R <= K && e == cudaSuccess; done += R) e = cudaGraphLaunch(ge, s);
    for (int64_t kk = done; kk < K && !rc && e == cudaSuccess; ++kk) rc = period(kk);  // remainder, kdev-driven
  }
  for (int q = 0; q < n; ++q) bs[q]->graph_mode = false;
  if (ge) cudaGraphExecDestroy(ge);
  if (g) cudaGraphDestroy(g);
  cudaStreamDestroy(cs);
  if (rc) return rc;
  if (e != cudaSuccess) {
    cudaGetLastError();
    snprintf(err, 512, "period graph: %s", cudaGetErrorString(e));
    return CAPGPU_E_CUDA;
  }
  return CAPGPU_OK;
}

}  // namespace capgpu

extern "C" int capgpu_nccl_unique_id(uint8_t out[128]) {
  ncclUniqueId uid;
  if (ncclGetUniqueId(&uid) != ncclSuccess) return CAPGPU_E_NCCL;
  std::memcpy(out, &uid, sizeof uid);
  return CAPGPU_OK;
}

// Host reference of the device tree (same pairwise order), used to check the
// deterministic aggregation and by multi-process tests.
extern "C" int capgpu_tree_sum_host(const double *v, int64_t n, double *out) {
  if (!v || !out || n < 1) return CAPGPU_E_INVALID;
  int64_t len = 1;
  while (len < n) len *= 2;
  double *w = new double[len];
  for (int64_t i = 0; i < len; ++i) w[i] = i < n ? v[i] : 0.0;
  for (int64_t h = len / 2; h >= 1; h /= 2)
    for (int64_t i = 0; i < h; ++i) w[i] = w[i] + w[i + h];
  *out = w[0];
  delete[] w;
  return CAPGPU_OK;
}
