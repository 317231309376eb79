// Instantiation unit: kernels for N = 14 knobs (1 CPU + 13 GPUs).
#include "capgpu_kernels.cuh"

namespace capgpu {
Launchers launchers_n14(int M) { return make_launchers<14>(M); }
}  // namespace capgpu
