// Instantiation unit: kernels for N = 11 knobs (1 CPU + 10 GPUs).
#include "capgpu_kernels.cuh"

namespace capgpu {
Launchers launchers_n11(int M) { return make_launchers<11>(M); }
}  // namespace capgpu
