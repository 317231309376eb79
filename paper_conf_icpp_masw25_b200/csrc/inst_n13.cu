// Instantiation unit: kernels for N = 13 knobs (1 CPU + 12 GPUs).
#include "capgpu_kernels.cuh"

namespace capgpu {
Launchers launchers_n13(int M) { return make_launchers<13>(M); }
}  // namespace capgpu
