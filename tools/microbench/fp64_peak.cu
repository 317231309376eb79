// Microbenchmark: FP64 pipe peak on B200 (DFMA/DDIV/DSQRT throughput, DFMA latency,
// splitmix64 integer-hash throughput).  Used to derive the "alu" roofline peak
// for the fused CapGPU kernel.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

template <int CH>
__global__ void dfma_tput(double *out, int iters, double a, double b) {
  double x[CH];
#pragma unroll
  for (int c = 0; c < CH; ++c) x[c] = threadIdx.x * 1e-3 + c;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = fma(x[c], a, b);
  }
  double s = 0;
#pragma unroll
  for (int c = 0; c < CH; ++c) s += x[c];
  if (s == 12345.678) out[0] = s;
}

__global__ void dfma_lat(double *out, long long *cyc, int iters, double a, double b) {
  double x = threadIdx.x;
  long long t0 = clock64();
  for (int i = 0; i < iters; ++i) x = fma(x, a, b);
  long long t1 = clock64();
  out[0] = x; cyc[0] = t1 - t0;
}

template <int CH>
__global__ void ddiv_tput(double *out, int iters, double b) {
  double x[CH];
#pragma unroll
  for (int c = 0; c < CH; ++c) x[c] = 1.0 + threadIdx.x * 1e-3 + c;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = b / x[c] + 1.0;
  }
  double s = 0;
#pragma unroll
  for (int c = 0; c < CH; ++c) s += x[c];
  if (s == 12345.678) out[0] = s;
}

template <int CH>
__global__ void dsqrt_tput(double *out, int iters) {
  double x[CH];
#pragma unroll
  for (int c = 0; c < CH; ++c) x[c] = 2.0 + threadIdx.x * 1e-3 + c;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = sqrt(x[c]) + 1.5;
  }
  double s = 0;
#pragma unroll
  for (int c = 0; c < CH; ++c) s += x[c];
  if (s == 12345.678) out[0] = s;
}

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
  return z ^ (z >> 31);
}

template <int CH>
__global__ void hash_tput(uint64_t *out, int iters) {
  uint64_t x[CH];
#pragma unroll
  for (int c = 0; c < CH; ++c) x[c] = threadIdx.x + 77 * c + blockIdx.x * 1000003ull;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = mix64(x[c] + 0x9e3779b97f4a7c15ULL);
  }
  uint64_t s = 0;
#pragma unroll
  for (int c = 0; c < CH; ++c) s ^= x[c];
  if (s == 12345) out[0] = s;
}

int main() {
  int dev = 0; cudaDeviceProp pr; CK(cudaGetDeviceProperties(&pr, dev));
  int clk_khz = 0; cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, dev);
  printf("{\"gpu\":\"%s\",\"sms\":%d,\"clock_khz_attr\":%d,\"l2_bytes\":%d}\n", pr.name, pr.multiProcessorCount, clk_khz, pr.l2CacheSize);
  double *d; CK(cudaMalloc(&d, 64)); long long *c; CK(cudaMalloc(&c, 8)); uint64_t *u; CK(cudaMalloc(&u, 8));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int sms = pr.multiProcessorCount;
  float ms;
  // DFMA throughput at several occupancies
  for (int bpsm : {2, 4, 8}) {
    int blocks = sms * bpsm, thr = 256, iters = 1 << 14;
    dfma_tput<8><<<blocks, thr>>>(d, 16, 1.0000001, 1e-9);
    cudaEventRecord(e0);
    for (int r = 0; r < 5; ++r) dfma_tput<8><<<blocks, thr>>>(d, iters, 1.0000001, 1e-9);
    cudaEventRecord(e1); CK(cudaEventSynchronize(e1)); cudaEventElapsedTime(&ms, e0, e1);
    double fl = 5.0 * blocks * thr * (double)iters * 8 * 2;
    printf("{\"test\":\"dfma_tput\",\"blocks_per_sm\":%d,\"tflops\":%.3f}\n", bpsm, fl / (ms * 1e-3) / 1e12);
  }
  dfma_lat<<<1, 1>>>(d, c, 4096, 1.0000001, 1e-9);
  long long cyc; CK(cudaMemcpy(&cyc, c, 8, cudaMemcpyDeviceToHost));
  printf("{\"test\":\"dfma_latency_cycles\",\"value\":%.2f}\n", cyc / 4096.0);
  {
    int blocks = sms * 4, thr = 256, iters = 1 << 11;
    ddiv_tput<4><<<blocks, thr>>>(d, 16, 3.0);
    cudaEventRecord(e0);
    for (int r = 0; r < 5; ++r) ddiv_tput<4><<<blocks, thr>>>(d, iters, 3.0);
    cudaEventRecord(e1); CK(cudaEventSynchronize(e1)); cudaEventElapsedTime(&ms, e0, e1);
    double n = 5.0 * blocks * thr * (double)iters * 4;
    printf("{\"test\":\"ddiv_tput\",\"gdiv_per_s\":%.3f}\n", n / (ms * 1e-3) / 1e9);
    dsqrt_tput<4><<<blocks, thr>>>(d, 16);
    cudaEventRecord(e0);
    for (int r = 0; r < 5; ++r) dsqrt_tput<4><<<blocks, thr>>>(d, iters);
    cudaEventRecord(e1); CK(cudaEventSynchronize(e1)); cudaEventElapsedTime(&ms, e0, e1);
    printf("{\"test\":\"dsqrt_tput\",\"gsqrt_per_s\":%.3f}\n", n / (ms * 1e-3) / 1e9);
    hash_tput<4><<<blocks, thr>>>(u, 16);
    cudaEventRecord(e0);
    for (int r = 0; r < 5; ++r) hash_tput<4><<<blocks, thr>>>(u, iters * 4);
    cudaEventRecord(e1); CK(cudaEventSynchronize(e1)); cudaEventElapsedTime(&ms, e0, e1);
    double nh = 5.0 * blocks * thr * (double)iters * 4 * 4;
    printf("{\"test\":\"splitmix_tput\",\"ghash_per_s\":%.3f}\n", nh / (ms * 1e-3) / 1e9);
  }
  return 0;
}
