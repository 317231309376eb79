// Microbenchmark: dependent-issue latency (cycles) of the instruction kinds the
// fused kernel's period chain is made of (DFMA, DADD, DSETP+FSEL select,
// 64-bit integer compare+select, MUFU.RCP64H, LDS.64, SHFL of a double), and
// the DFMA chain throughput per SM at 1..8 warps per scheduler with ILP 1/2/4.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/lat tools/microbench/lat.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

constexpr int IT = 4096;

__global__ void lat_dfma(double *o, long long *c, double a, double b) {
  double x = threadIdx.x;
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < IT; ++i) x = fma(x, a, b);
  long long t1 = clock64();
  o[threadIdx.x] = x; if (threadIdx.x == 0) c[0] = t1 - t0;
}
__global__ void lat_dadd(double *o, long long *c, double a, double b) {
  double x = threadIdx.x;
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < IT; ++i) x = x + a;
  long long t1 = clock64();
  o[threadIdx.x] = x; if (threadIdx.x == 0) c[0] = t1 - t0;
}
// x = (x > a) ? x - b : x + b  : DSETP -> FSEL x2 -> DADD chain (per iteration)
__global__ void lat_dsel(double *o, long long *c, double a, double b) {
  double x = threadIdx.x;
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < IT; ++i) x = (x > a) ? x * b : x;
  long long t1 = clock64();
  o[threadIdx.x] = x; if (threadIdx.x == 0) c[0] = t1 - t0;
}
// same with the compare on the IEEE bits (non-negative doubles)
__global__ void lat_isel(double *o, long long *c, double a, double b) {
  double x = threadIdx.x + 1.0;
  const long long ab = __double_as_longlong(a);
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < IT; ++i) x = (__double_as_longlong(x) > ab) ? x * b : x;
  long long t1 = clock64();
  o[threadIdx.x] = x; if (threadIdx.x == 0) c[0] = t1 - t0;
}
__global__ void lat_dmul(double *o, long long *c, double a, double b) {
  double x = threadIdx.x + 1.0;
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < IT; ++i) x = x * a;
  long long t1 = clock64();
  o[threadIdx.x] = x; if (threadIdx.x == 0) c[0] = t1 - t0;
}
__global__ void lat_rcp(double *o, long long *c, double a, double b) {
  double x = threadIdx.x + 1.5;
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < IT; ++i) {
    double y;
    asm volatile("rcp.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
    x = y;
  }
  long long t1 = clock64();
  o[threadIdx.x] = x; if (threadIdx.x == 0) c[0] = t1 - t0;
}
__global__ void lat_lds(double *o, long long *c, double a, double b) {
  __shared__ double s[256];
  for (int i = threadIdx.x; i < 256; i += blockDim.x) s[i] = (double)((i * 7 + 1) & 255);
  __syncthreads();
  double x = (double)(threadIdx.x & 31);
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < IT; ++i) x = s[(int)x];
  long long t1 = clock64();
  o[threadIdx.x] = x; if (threadIdx.x == 0) c[0] = t1 - t0;
}
__global__ void lat_shfl(double *o, long long *c, double a, double b) {
  double x = threadIdx.x;
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < IT; ++i) x = __shfl_xor_sync(0xffffffffu, x, 1);
  long long t1 = clock64();
  o[threadIdx.x] = x; if (threadIdx.x == 0) c[0] = t1 - t0;
}
__global__ void lat_iadd64(double *o, long long *c, double a, double b) {
  long long x = threadIdx.x; const long long d = (long long)a;
  long long t0 = clock64();
#pragma unroll 16
  for (int i = 0; i < IT; ++i) x = x * 3 + d;
  long long t1 = clock64();
  o[threadIdx.x] = (double)x; if (threadIdx.x == 0) c[0] = t1 - t0;
}

// throughput: W warps per SM, each with ILP independent DFMA chains
template <int ILP>
__global__ void tput(double *o, int iters, double a, double b) {
  double x[ILP];
#pragma unroll
  for (int c = 0; c < ILP; ++c) x[c] = threadIdx.x + c;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int c = 0; c < ILP; ++c) x[c] = fma(x[c], a, b);
  }
  double s = 0;
#pragma unroll
  for (int c = 0; c < ILP; ++c) s += x[c];
  if (s == 1234.5) o[0] = s;
}

typedef void (*LK)(double *, long long *, double, double);

int main() {
  double *o; long long *c, hc;
  CK(cudaMalloc(&o, 1 << 20)); CK(cudaMalloc(&c, 64));
  struct { const char *n; LK k; double a, b; } L[] = {
      {"dfma", lat_dfma, 0.999, 1e-3}, {"dadd", lat_dadd, 1e-3, 0}, {"dmul", lat_dmul, 0.9999, 0},
      {"dsetp+fsel (+dmul)", lat_dsel, 0.5, 0.9999}, {"isetp64+sel (+dmul)", lat_isel, 0.5, 0.9999},
      {"mufu.rcp64h (rcp.approx.ftz.f64)", lat_rcp, 0, 0}, {"lds.64 (dep. address)", lat_lds, 0, 0},
      {"shfl.xor double", lat_shfl, 0, 0}, {"imad64", lat_iadd64, 5, 0}};
  for (auto &l : L) {
    for (int r = 0; r < 2; ++r) { l.k<<<1, 32>>>(o, c, l.a, l.b); }
    CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(&hc, c, 8, cudaMemcpyDeviceToHost));
    printf("latency %-36s %.2f cycles/iter\n", l.n, (double)hc / IT);
  }
  int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  int clk; CK(cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int iters = 1 << 16;
  for (int w = 4; w <= 32; w *= 2) {
    auto run = [&](auto kern, int ilp) {
      kern<<<sms, w * 32>>>(o, iters, 0.999, 1e-3);
      cudaEventRecord(e0);
      kern<<<sms, w * 32>>>(o, iters, 0.999, 1e-3);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      double fl = 2.0 * iters * ilp * (double)w * 32 * sms;
      printf("tput warps/SM %2d ILP %d: %.2f TF/s  (%.1f%% of %.1f derived)\n", w, ilp, fl / ms * 1e-9,
             100 * fl / ms * 1e-9 / (sms * 128.0 * clk * 1e-6), sms * 128.0 * clk * 1e-6);
    };
    run(tput<1>, 1); run(tput<2>, 2); run(tput<4>, 4);
  }
  CK(cudaGetLastError());
  return 0;
}
