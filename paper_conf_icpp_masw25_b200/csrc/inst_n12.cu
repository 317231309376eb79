// Instantiation unit: kernels for N = 12 knobs (1 CPU + 11 GPUs).
#include "capgpu_kernels.cuh"

namespace capgpu {
Launchers launchers_n12(int M) { return make_launchers<12>(M); }
}  // namespace capgpu
