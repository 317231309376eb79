// Instantiation unit: kernels for N = 7 knobs (1 CPU + 6 GPUs).
#include "capgpu_kernels.cuh"

namespace capgpu {
Launchers launchers_n7(int M) { return make_launchers<7>(M); }
}  // namespace capgpu
