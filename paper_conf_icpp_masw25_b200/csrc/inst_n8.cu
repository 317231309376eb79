// Instantiation unit: kernels for N = 8 knobs (1 CPU + 7 GPUs).
#include "capgpu_kernels.cuh"

namespace capgpu {
Launchers launchers_n8(int M) { return make_launchers<8>(M); }
}  // namespace capgpu
