// Shared-memory wavefronts of one warp-wide LDS.128 per lane->word pattern
// (16-byte words). Run under ncu: l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum
// per launch, 64 loads per thread -> wavefronts / 64 per pattern.
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ int word(int p, int l) {
  switch (p) {
    case 0: return 0;                                // broadcast
    case 1: return l & 1;                            // 2 distinct
    case 2: return l & 3;                            // 4 distinct, 64 B
    case 3: return l & 7;                            // 8 distinct, 128 B
    case 4: return l >> 3;                           // quarter-uniform, 4 distinct
    case 5: return l >> 2;                           // 8 distinct, 2 per quarter
    case 6: return l & 15;                           // 16 distinct, 256 B
    case 7: return l;                                // 32 distinct
    case 8: return (l & 3) + 4 * (l >> 4);           // 8 distinct, halves differ
    case 9: return (l >> 4);                         // half-uniform, 2 distinct
    case 10: return (l & 7) + 8 * (l >> 4);          // 16 distinct, halves differ
    case 11: return (l >> 3) * 8;                    // quarter-uniform, 4 distinct, 128 B apart
    default: return 0;
  }
}
__global__ void probe(int p, float* out) {
  __shared__ __align__(16) float s[4096];
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) s[i] = i;
  __syncthreads();
  const int w = word(p, threadIdx.x & 31);
  float4 acc = make_float4(0, 0, 0, 0);
#pragma unroll 1
  for (int it = 0; it < 64; ++it) {
    const float4 v = *reinterpret_cast<const float4*>(&s[(w * 4 + it * 128) & 4095]);
    acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
  }
  if (acc.x == -1.f) out[0] = acc.y + acc.z + acc.w;
}
int main() {
  float* o; cudaMalloc(&o, 16);
  for (int p = 0; p < 12; ++p) probe<<<1, 32>>>(p, o);
  cudaDeviceSynchronize();
  printf("done\n");
  return 0;
}
