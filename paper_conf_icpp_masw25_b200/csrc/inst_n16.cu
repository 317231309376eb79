// Instantiation unit: kernels for N = 16 knobs (1 CPU + 15 GPUs).
#include "capgpu_kernels.cuh"

namespace capgpu {
Launchers launchers_n16(int M) { return make_launchers<16>(M); }
}  // namespace capgpu
