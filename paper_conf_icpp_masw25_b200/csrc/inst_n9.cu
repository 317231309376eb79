// Instantiation unit: kernels for N = 9 knobs (1 CPU + 8 GPUs).
#include "capgpu_kernels.cuh"

namespace capgpu {
Launchers launchers_n9(int M) { return make_launchers<9>(M); }
}  // namespace capgpu
