// T2 inner step from shared memory (4 LDS.128 + 32 FFMA2 per k), row operand as a .F32 broadcast
// (bcast) vs rows as register pairs with diagonal/anti-diagonal accumulators (diag).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/diag_pair_probe tools/diag_pair_probe.cu
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ unsigned long long f2fma(unsigned long long a, unsigned long long b, unsigned long long c) {
  unsigned long long d; asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c)); return d; }
__device__ __forceinline__ unsigned long long swp(unsigned long long x) {
  unsigned long long r; asm("{ .reg .b32 lo, hi; mov.b64 {lo, hi}, %1; mov.b64 %0, {hi, lo}; }" : "=l"(r) : "l"(x)); return r; }
__device__ __forceinline__ unsigned long long pk(float x, float y) {
  return (unsigned long long)__float_as_uint(x) | ((unsigned long long)__float_as_uint(y) << 32); }
// T2's inner step from shared memory: per k, the warp's 8 rows (broadcast) and each lane's 8 columns
template <bool DIAG>
__global__ void __launch_bounds__(256, 2) step(float* out, int iters) {
  __shared__ __align__(16) float srow[16][64];
  __shared__ __align__(16) float scol[16][256];
  const int lane = threadIdx.x & 31, ty = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < 16 * 64; i += 256) srow[i / 64][i % 64] = 1.0f + i * 1e-6f;
  for (int i = threadIdx.x; i < 16 * 256; i += 256) scol[i / 256][i % 256] = 0.5f + i * 1e-7f;
  __syncthreads();
  unsigned long long acc[32];
#pragma unroll
  for (int q = 0; q < 32; ++q) acc[q] = 0;
  for (int it = 0; it < iters; ++it) {
#pragma unroll 4
    for (int kk = 0; kk < 16; ++kk) {
      const float4 r0 = *reinterpret_cast<const float4*>(&srow[kk][ty * 4]);
      const float4 r1 = *reinterpret_cast<const float4*>(&srow[kk][32 + ty * 4]);
      const float4 c0 = *reinterpret_cast<const float4*>(&scol[kk][lane * 4]);
      const float4 c1 = *reinterpret_cast<const float4*>(&scol[kk][128 + lane * 4]);
      const float rv[8] = {r0.x, r0.y, r0.z, r0.w, r1.x, r1.y, r1.z, r1.w};
      const unsigned long long cp[4] = {pk(c0.x, c0.y), pk(c0.z, c0.w), pk(c1.x, c1.y), pk(c1.z, c1.w)};
      if (DIAG) {
        const unsigned long long rp[4] = {pk(rv[0], rv[1]), pk(rv[2], rv[3]), pk(rv[4], rv[5]), pk(rv[6], rv[7])};
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const unsigned long long cs = swp(cp[q]);
#pragma unroll
          for (int p = 0; p < 4; ++p) {
            acc[(p * 4 + q) * 2] = f2fma(rp[p], cp[q], acc[(p * 4 + q) * 2]);
            acc[(p * 4 + q) * 2 + 1] = f2fma(rp[p], cs, acc[(p * 4 + q) * 2 + 1]);
          }
        }
      } else {
#pragma unroll
        for (int q = 0; q < 4; ++q)
#pragma unroll
          for (int r = 0; r < 8; ++r) acc[r * 4 + q] = f2fma(pk(rv[r], rv[r]), cp[q], acc[r * 4 + q]);
      }
    }
  }
  float s = 0;
#pragma unroll
  for (int q = 0; q < 32; ++q) s += __uint_as_float(unsigned(acc[q])) + __uint_as_float(unsigned(acc[q] >> 32));
  if (s == 1.2345f) out[0] = s;
}
int main() {
  float* out; cudaMalloc(&out, 4);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const int iters = 2000;
  for (int v = 0; v < 2; ++v) for (int ctas : {148, 296}) {
    auto f = v ? step<true> : step<false>;
    f<<<ctas, 256>>>(out, 2);
    cudaEventRecord(e0); f<<<ctas, 256>>>(out, iters); cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    printf("%s CTAs %3d (warps/SM %2d): %6.1f TFLOP/s (%s)\n", v ? "diag " : "bcast", ctas, ctas / 148 * 8, 2.0 * ctas * 256 * 64.0 * 16 * iters / (ms * 1e-3) / 1e12, cudaGetErrorString(cudaGetLastError()));
  }
  return 0;
}
