// Per-warp FFMA2 rate: the 8 x 8 outer product of ffma_probe (broadcast .F32
// row operand, column pairs reused), at 8 / 16 / 32 warps per SM (one CTA per
// SM), to tell whether a few warps per SM can keep the FMA pipe busy.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/warp_rate_probe tools/warp_rate_probe.cu
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ unsigned long long f2fma(unsigned long long a, unsigned long long b, unsigned long long c) {
  unsigned long long d;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
  return d;
}
__device__ __forceinline__ unsigned long long pk(float x, float y) {
  return (unsigned long long)__float_as_uint(x) | ((unsigned long long)__float_as_uint(y) << 32);
}
// the row operand as a true register pair (x, x), duplicated by a volatile
// mov each step (not folded into the .F32 broadcast operand form)
__device__ __forceinline__ unsigned long long dup(float x) {
  unsigned long long r;
  asm volatile("mov.b64 %0, {%1, %1};" : "=l"(r) : "f"(x));
  return r;
}
__global__ void outer_dup(float* out, int iters) {
  unsigned long long acc[8][4];
  float av[8];
  unsigned long long bv[4];
#pragma unroll
  for (int r = 0; r < 8; ++r) {
    av[r] = threadIdx.x + r;
#pragma unroll
    for (int q = 0; q < 4; ++q) acc[r][q] = 0;
  }
#pragma unroll
  for (int q = 0; q < 4; ++q) bv[q] = pk(1.0001f + q * 1e-6f, 1.0002f + q * 1e-6f);
  for (int i = 0; i < iters; ++i) {
    unsigned long long ap[8];
#pragma unroll
    for (int r = 0; r < 8; ++r) ap[r] = dup(av[r]);
#pragma unroll
    for (int q = 0; q < 4; ++q)
#pragma unroll
      for (int r = 0; r < 8; ++r) acc[r][q] = f2fma(ap[r], bv[q], acc[r][q]);
#pragma unroll
    for (int r = 0; r < 8; ++r) av[r] = av[r] * 0.9999f;
  }
  float s = 0;
#pragma unroll
  for (int r = 0; r < 8; ++r)
#pragma unroll
    for (int q = 0; q < 4; ++q) s += __uint_as_float(unsigned(acc[r][q])) + __uint_as_float(unsigned(acc[r][q] >> 32));
  if (s == 1.2345f) out[0] = s;
}

template <bool PAIR_OUTER>
__global__ void outer(float* out, int iters) {
  unsigned long long acc[8][4];
  float av[8];
  unsigned long long bv[4];
#pragma unroll
  for (int r = 0; r < 8; ++r) {
    av[r] = threadIdx.x + r;
#pragma unroll
    for (int q = 0; q < 4; ++q) acc[r][q] = 0;
  }
#pragma unroll
  for (int q = 0; q < 4; ++q) bv[q] = pk(1.0001f + q * 1e-6f, 1.0002f + q * 1e-6f);
  for (int i = 0; i < iters; ++i) {
    if (PAIR_OUTER) {
#pragma unroll
      for (int q = 0; q < 4; ++q)
#pragma unroll
        for (int r = 0; r < 8; ++r) acc[r][q] = f2fma(pk(av[r], av[r]), bv[q], acc[r][q]);
    } else {
#pragma unroll
      for (int r = 0; r < 8; ++r)
#pragma unroll
        for (int q = 0; q < 4; ++q) acc[r][q] = f2fma(pk(av[r], av[r]), bv[q], acc[r][q]);
    }
#pragma unroll
    for (int r = 0; r < 8; ++r) av[r] = av[r] * 0.9999f;
  }
  float s = 0;
#pragma unroll
  for (int r = 0; r < 8; ++r)
#pragma unroll
    for (int q = 0; q < 4; ++q) s += __uint_as_float(unsigned(acc[r][q])) + __uint_as_float(unsigned(acc[r][q] >> 32));
  if (s == 1.2345f) out[0] = s;
}
int main() {
  float* out;
  cudaMalloc(&out, 4);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int iters = 20000;
  for (int po = 0; po < 2; ++po)
    for (int thr : {128, 256, 384, 512, 768, 1024}) {
      auto k = po ? outer<true> : outer<false>;
      k<<<148, thr>>>(out, 10);
      cudaEventRecord(e0);
      k<<<148, thr>>>(out, iters);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      const double flop = 2.0 * 148 * thr * 64.0 * iters;
      printf("%s warps/SM %2d: %6.1f TFLOP/s (%s)\n", po ? "pair-outer" : "row-outer ", thr / 32, flop / (ms * 1e-3) / 1e12,
             cudaGetErrorString(cudaGetLastError()));
    }
  for (int thr : {256, 512}) {
    outer_dup<<<148, thr>>>(out, 10);
    cudaEventRecord(e0);
    outer_dup<<<148, thr>>>(out, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    const double flop = 2.0 * 148 * thr * 64.0 * iters;
    printf("pair-dup   warps/SM %2d: %6.1f TFLOP/s (%s)\n", thr / 32, flop / (ms * 1e-3) / 1e12,
           cudaGetErrorString(cudaGetLastError()));
  }
  return 0;
}
