// Instantiation unit: kernels for N = 2 knobs (1 CPU + 1 GPUs).
#include "capgpu_kernels.cuh"

namespace capgpu {
Launchers launchers_n2(int M) { return make_launchers<2>(M); }
}  // namespace capgpu
