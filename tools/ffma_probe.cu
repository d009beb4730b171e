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
  }
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("nominal 148 SM x 128 lanes x 2 x %.0f MHz = %.1f TFLOP/s\n", clk / 1e3, 148.0 * 128 * 2 * clk * 1e3 / 1e12);
  return 0;
}
