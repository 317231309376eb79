// Instantiation unit: kernels for N = 10 knobs (1 CPU + 9 GPUs).
#include "capgpu_kernels.cuh"

namespace capgpu {
Launchers launchers_n10(int M) { return make_launchers<10>(M); }
}  // namespace capgpu
