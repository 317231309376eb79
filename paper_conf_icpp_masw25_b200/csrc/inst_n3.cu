// Instantiation unit: kernels for N = 3 knobs (1 CPU + 2 GPUs).
#include "capgpu_kernels.cuh"

namespace capgpu {
Launchers launchers_n3(int M) { return make_launchers<3>(M); }
}  // namespace capgpu
