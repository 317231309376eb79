// capgpu_budget.cu -- S5 hierarchical budget (cfg 4).  Round-1 placeholder:
// the per-period kernel path lands with the multi-GPU milestone.
#include <cstdio>
#include <cstring>

#include <nccl.h>

#include "capgpu_budget.cuh"

namespace capgpu {

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
}

int budget_setup(Budget &, const DevParams &, const StatePtrs &, const capgpu_workload &, const capgpu_shard &,
                 cudaStream_t, char *err) {
  snprintf(err, 512, "hierarchical budget not built yet");
  return CAPGPU_E_UNSUPPORTED;
}

int budget_simulate(Budget &, const DevParams &, const StatePtrs &, const TracePtrs &, const Launchers &, int64_t,
                    int64_t, double *, double *, cudaStream_t, char *err) {
  snprintf(err, 512, "hierarchical budget not built yet");
  return CAPGPU_E_UNSUPPORTED;
}

}  // namespace capgpu

extern "C" int capgpu_nccl_unique_id(uint8_t out[128]) {
  ncclUniqueId uid;
  if (ncclGetUniqueId(&uid) != ncclSuccess) return CAPGPU_E_NCCL;
  std::memcpy(out, &uid, sizeof uid);
  return CAPGPU_OK;
}
