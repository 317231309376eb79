// Instantiation unit: kernels for N = 15 knobs (1 CPU + 14 GPUs).
#include "capgpu_kernels.cuh"

namespace capgpu {
Launchers launchers_n15(int M) { return make_launchers<15>(M); }
}  // namespace capgpu
