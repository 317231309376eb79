// capgpu_budget.cuh -- S5 hierarchical rack/cluster budget (cfg 4, Q16): the
// per-period orchestration around k_period, the deterministic block sums and
// fixed-order tree, and the all-reduce (NCCL over NVLink, identity for one
// shard, or an in-process loopback sum for several shards on one GPU).
#pragma once

#include "capgpu_kernels.cuh"

namespace capgpu {

constexpr int kBudgetBlock = 1024;  // servers per reduction block (fixed granularity)
constexpr int kCta = kPeriodCta;    // servers per CTA of k_period
constexpr int kCtasPerBlock = kBudgetBlock / kCta;

struct Budget {
  void *comm = nullptr;  // ncclComm_t (world > 1 with NCCL)
  int world = 1, rank = 0;
  int64_t n_cta = 0, nb_local = 0, blk_begin = 0, nb_g = 0, tree_len = 0;
  double *srv_w = nullptr;    // [n_srv]
  double *part = nullptr;     // [2][n_cta]
  double *part_c = nullptr;   // [2][n_cta] (pmin, pmax) at setup
  double *send = nullptr;     // [2][nb_g] zero-padded block sums (only local blocks non-zero)
  double *recv = nullptr;     // [2][nb_g] all-reduced block sums
  double *scratch = nullptr;  // [2][tree_len] tree workspace
  double *agg = nullptr;      // [2] W, P
  double *consts = nullptr;   // [2] Pmin_tot, Pmax_tot
  double B_c = 0.0, pmin_tot = 0.0, pmax_tot = 0.0, rack_frac = 0.9, cluster_frac = 0.55;
  int rack = 16;
  bool ready = false;
  int64_t *kdev = nullptr;  // [2] {first period of the call, call period} for CUDA-graph replay
  bool graph_mode = false;  // launches read the period from kdev (while a call is captured / replayed)
};

int budget_init_nccl(Budget &b, const uint8_t *id, int world, int rank, char *err);
void budget_free(Budget &b);
// Allocation + setup.  loopback: if non-null, the all-reduce is replaced by
// summing the `send` buffers of the n_loop budgets (one GPU, several shards).
int budget_alloc(Budget &b, const DevParams &P, const capgpu_workload &wl, const capgpu_shard &sh, char *err);
int budget_setup_local(Budget &b, const DevParams &P, const StatePtrs &st, const Launchers &L, cudaStream_t s,
                       char *err);
int budget_reduce(Budget **bs, int n, bool consts, cudaStream_t s, char *err);
int budget_finish_setup(Budget &b, cudaStream_t s, char *err);
int budget_period_local(Budget &b, const DevParams &P, const StatePtrs &st, const TracePtrs &tr, const Launchers &L,
                        int64_t k, int kk, int K, cudaStream_t s, char *err);
int budget_tree(Budget &b, double *agg_W, double *agg_P, int kk, cudaStream_t s, char *err);
int budget_simulate(Budget &b, const DevParams &P, const StatePtrs &st, const TracePtrs &tr, const Launchers &L,
                    int64_t k0, int64_t K, double *agg_W, double *agg_P, cudaStream_t s, char *err);
int budget_simulate_group(Budget **bs, int n, const DevParams *P, const StatePtrs *st, const TracePtrs *tr,
                          const Launchers *L, int64_t k0, int64_t K, double **agg_W, double **agg_P, cudaStream_t s,
                          char *err);

}  // namespace capgpu
