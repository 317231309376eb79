// capgpu_budget.cuh -- S5 hierarchical rack/cluster budget (cfg 4, Q16) and the
// NCCL plumbing for the per-period all-reduce.  (Filled in by capgpu_budget.cu.)
#pragma once

#include "capgpu_kernels.cuh"

namespace capgpu {

struct Budget {
  void *comm = nullptr;  // ncclComm_t
  int world = 1, rank = 0;
  double *blk = nullptr;      // [3][2 * n_blocks_global] rotating block-sum buffers (w, p)
  double *agg = nullptr;      // scratch
  double *srv_w = nullptr;    // per-server w_i of the last instant
  double *caps = nullptr;     // per-server caps for the next instant
  double *rack_max = nullptr; // per-rack B_rack
  int64_t n_blocks_global = 0, blk_begin = 0, n_blocks_local = 0;
  double B_c = 0.0, pmin_tot = 0.0;
  int rack = 16, block = 1024;
  bool ready = false;
  void *stream_comm = nullptr;
  void *ev[3] = {nullptr, nullptr, nullptr};
};

int budget_init_nccl(Budget &b, const uint8_t *id, int world, int rank, char *err);
void budget_free(Budget &b);
int budget_setup(Budget &b, const DevParams &P, const StatePtrs &st, const capgpu_workload &wl,
                 const capgpu_shard &sh, cudaStream_t s, char *err);
int budget_simulate(Budget &b, const DevParams &P, const StatePtrs &st, const TracePtrs &tr, const Launchers &L,
                    int64_t k0, int64_t K, double *agg_W, double *agg_P, cudaStream_t s, char *err);

}  // namespace capgpu
