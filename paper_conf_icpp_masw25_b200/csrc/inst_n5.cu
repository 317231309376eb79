// Instantiation unit: kernels for N = 5 knobs (1 CPU + 4 GPUs).
#include "capgpu_kernels.cuh"

namespace capgpu {
Launchers launchers_n5(int M) { return make_launchers<5>(M); }
}  // namespace capgpu
