// Instantiation unit: kernels for N = 4 knobs (1 CPU + 3 GPUs).
#include "capgpu_kernels.cuh"

namespace capgpu {
Launchers launchers_n4(int M) { return make_launchers<4>(M); }
}  // namespace capgpu
