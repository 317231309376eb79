// Device accuracy of the fast reciprocal (capgpu_device.cuh rcp_fast):
// max |e| of the MUFU.RCP64H seed (e = 1 - x y0) and the max relative error of
// y0 (1 + e + e^2) against the IEEE quotient, over log-uniform x in [2^-30, 2^30].
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o rcp_check rcp_check.cu
#include <cstdio>
#include <cstdint>
#include <cmath>

__global__ void k(int n, unsigned long long seed, double *out) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  double emax = 0, rmax = 0, r2max = 0;
  for (int t = i; t < n; t += gridDim.x * blockDim.x) {
    unsigned long long z = seed + 0x9E3779B97F4A7C15ull * (t + 1);
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; z ^= z >> 31;
    double u = (double)(z >> 11) * 0x1p-53;
    double x = exp2(60.0 * u - 30.0);
    double y0; asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(y0) : "d"(x));
    double e = fma(-x, y0, 1.0);
    double y3 = fma(y0, fma(e, e, e), y0);
    double e1 = fma(-x, y0, 1.0); double y = fma(y0, e1, y0); e1 = fma(-x, y, 1.0); y = fma(y, e1, y);
    double q = __ddiv_rn(1.0, x);
    emax = fmax(emax, fabs(e));
    rmax = fmax(rmax, fabs(y3 - q) / q);
    r2max = fmax(r2max, fabs(y - q) / q);
  }
  atomicMax((unsigned long long *)&out[0], __double_as_longlong(emax));
  atomicMax((unsigned long long *)&out[1], __double_as_longlong(rmax));
  atomicMax((unsigned long long *)&out[2], __double_as_longlong(r2max));
}

int main() {
  double *d; cudaMalloc(&d, 24); cudaMemset(d, 0, 24);
  k<<<1184, 256>>>(1 << 28, 12345, d);
  double h[3]; cudaMemcpy(h, d, 24, cudaMemcpyDeviceToHost);
  printf("rcp64h seed: max|e| = %.3e (2^%.2f)\n", h[0], log2(h[0]));
  printf("y0(1+e+e^2): max rel err = %.3e (%.2f ulp)\n", h[1], h[1] / 0x1p-53);
  printf("two Newton : max rel err = %.3e (%.2f ulp)\n", h[2], h[2] / 0x1p-53);
  return 0;
}
