#include <cstdio>
#include "../../paper_conf_icpp_masw25_b200/csrc/capgpu_device.cuh"
using namespace capgpu;
__global__ void k(KnobConst k0, KnobConst k1, double beta, double a0, double a1, double t0, double t1, double c, uint32_t warm) {
  KnobConst kc[2] = {k0, k1};
  double a[2] = {a0, a1}, tau[2] = {t0, t1}, u[2];
  bool capped = false;
  uint32_t code = solve_block<2>(kc, a, tau, c, beta, warm, u, capped);
  printf("warm %u c %g -> code %u u %.9f %.9f capped %d\n", warm, c, code, u[0], u[1], (int)capped);
}
int main() {
  KnobConst k0{}, k1{};
  k0.f_min = 1100; k0.f_max = 2400; k0.lo = 1100; k0.hi = 2400; k0.m = 1100;
  k1.f_min = 435; k1.f_max = 1350; k1.lo = 435; k1.hi = 1350; k1.m = 435;
  double beta = -250.36917592279434, a0 = 0.07210369, a1 = 0.21226392;
  double t0 = a0 * 0.05 / 1e-4, t1 = a1 * 0.46361646 / 1e-4;
  for (uint32_t w : {0u, 5u, 10u, 1u, 4u}) for (double c : {1.0, 3.0}) k<<<1,1>>>(k0, k1, beta, a0, a1, t0, t1, c, w);
  cudaDeviceSynchronize();
}
