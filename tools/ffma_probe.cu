// FFMA throughput probe: independent chains, register operands (3-reg form) vs immediate.
#include <cstdio>
#include <cuda_runtime.h>
template <int CH>
__global__ void ffma_reg(float* out, int iters, float b, float c) {
  float a[CH];
#pragma unroll
  for (int k = 0; k < CH; ++k) a[k] = threadIdx.x * 1e-3f + k;
  float bb = b + threadIdx.x * 1e-7f, cc = c;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < CH; ++k) a[k] = fmaf(a[k], bb, cc);
  }
  float s = 0;
#pragma unroll
  for (int k = 0; k < CH; ++k) s += a[k];
  if (s == 1.2345f) out[0] = s;
}
// outer-product style like SGEMM: acc[r][q] = fma(av[r], bv[q], acc[r][q])
__global__ void ffma_outer(float* out, int iters) {
  float acc[8][8], av[8], bv[8];
#pragma unroll
  for (int r = 0; r < 8; ++r) { av[r] = threadIdx.x + r; bv[r] = 1.0001f + r * 1e-6f;
#pragma unroll
    for (int q = 0; q < 8; ++q) acc[r][q] = 0; }
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int r = 0; r < 8; ++r)
#pragma unroll
      for (int q = 0; q < 8; ++q) acc[r][q] = fmaf(av[r], bv[q], acc[r][q]);
#pragma unroll
    for (int r = 0; r < 8; ++r) av[r] = av[r] * 0.9999f;
  }
  float s = 0;
#pragma unroll
  for (int r = 0; r < 8; ++r)
#pragma unroll
    for (int q = 0; q < 8; ++q) s += acc[r][q];
  if (s == 1.2345f) out[0] = s;
}

// packed fp32 (sm_100a FFMA2): two independent IEEE fmas per instruction
__device__ __forceinline__ unsigned long long f2fma(unsigned long long a, unsigned long long b, unsigned long long c) {
  unsigned long long d;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
  return d;
}
__device__ __forceinline__ unsigned long long pk(float x, float y) {
  return (unsigned long long)__float_as_uint(x) | ((unsigned long long)__float_as_uint(y) << 32);
}
template <int CH>
__global__ void ffma2_reg(float* out, int iters, float b, float c) {
  unsigned long long a[CH];
#pragma unroll
  for (int k = 0; k < CH; ++k) a[k] = pk(threadIdx.x * 1e-3f + k, k * 0.5f);
  const unsigned long long bb = pk(b + threadIdx.x * 1e-7f, b), cc = pk(c, c * 0.5f);
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < CH; ++k) a[k] = f2fma(a[k], bb, cc);
  }
  float s = 0;
#pragma unroll
  for (int k = 0; k < CH; ++k) s += __uint_as_float(unsigned(a[k])) + __uint_as_float(unsigned(a[k] >> 32));
  if (s == 1.2345f) out[0] = s;
}
// outer product 8 x 8 with packed pairs along q: acc[r][q2] (2 columns) = fma2(av[r] (dup), bv[q2], acc)
__global__ void ffma2_outer(float* out, int iters) {
  unsigned long long acc[8][4], av[8], bv[4];
#pragma unroll
  for (int r = 0; r < 8; ++r) { av[r] = pk(threadIdx.x + r, threadIdx.x + r);
#pragma unroll
    for (int q = 0; q < 4; ++q) acc[r][q] = 0; }
#pragma unroll
  for (int q = 0; q < 4; ++q) bv[q] = pk(1.0001f + q * 1e-6f, 1.0002f + q * 1e-6f);
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int r = 0; r < 8; ++r)
#pragma unroll
      for (int q = 0; q < 4; ++q) acc[r][q] = f2fma(av[r], bv[q], acc[r][q]);
#pragma unroll
    for (int r = 0; r < 8; ++r) av[r] = f2fma(av[r], pk(0.9999f, 0.9999f), 0ull);
  }
  float s = 0;
#pragma unroll
  for (int r = 0; r < 8; ++r)
#pragma unroll
    for (int q = 0; q < 4; ++q) s += __uint_as_float(unsigned(acc[r][q])) + __uint_as_float(unsigned(acc[r][q] >> 32));
  if (s == 1.2345f) out[0] = s;
}
int main() {
  float* out; cudaMalloc(&out, 4);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  int iters = 20000;
  for (int thr : {256, 512, 1024}) {
    int G = 148 * (2048 / thr);
    ffma_reg<8><<<G, thr>>>(out, 10, 1.0001f, 0.5f);
    cudaEventRecord(e0); ffma_reg<8><<<G, thr>>>(out, iters, 1.0001f, 0.5f); cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double flop = 2.0 * G * thr * 8.0 * iters;
    printf("ffma 3-reg chains=8 thr=%d: %.1f TFLOP/s\n", thr, flop / (ms * 1e-3) / 1e12);
    cudaEventRecord(e0); ffma_outer<<<G, thr>>>(out, iters / 8); cudaEventRecord(e1); cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    flop = 2.0 * G * thr * 64.0 * (iters / 8);
    printf("ffma outer 8x8 thr=%d: %.1f TFLOP/s\n", thr, flop / (ms * 1e-3) / 1e12);
    ffma2_reg<8><<<G, thr>>>(out, 10, 1.0001f, 0.5f);
    cudaEventRecord(e0); ffma2_reg<8><<<G, thr>>>(out, iters, 1.0001f, 0.5f); cudaEventRecord(e1); cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    flop = 2.0 * G * thr * 16.0 * iters;
    printf("ffma2 3-reg chains=8 (16 fma) thr=%d: %.1f TFLOP/s\n", thr, flop / (ms * 1e-3) / 1e12);
    cudaEventRecord(e0); ffma2_outer<<<G, thr>>>(out, iters / 8); cudaEventRecord(e1); cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    flop = 2.0 * G * thr * (64.0 + 16.0) * (iters / 8);
    printf("ffma2 outer 8x8 thr=%d: %.1f TFLOP/s (incl. 16 scaling fmas)\n", thr, flop / (ms * 1e-3) / 1e12);
  }
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("nominal 148 SM x 128 lanes x 2 x %.0f MHz = %.1f TFLOP/s\n", clk / 1e3, 148.0 * 128 * 2 * clk * 1e3 / 1e12);
  return 0;
}
