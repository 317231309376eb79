// Instantiation unit: kernels for N = 6 knobs (1 CPU + 5 GPUs).
#include "capgpu_kernels.cuh"

namespace capgpu {
Launchers launchers_n6(int M) { return make_launchers<6>(M); }
}  // namespace capgpu
