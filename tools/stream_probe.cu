// Scratch probe: how fast can 1-D bulk copies (cp.async.bulk) through an
// smem ring stream 64 MiB / 256 MiB on B200, vs plain 16-B loads?
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("ERR %s %d: %s\n", #x, __LINE__, cudaGetErrorString(e)); return 1; } } while (0)
__device__ __forceinline__ uint32_t s32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void binit(uint64_t* b, uint32_t c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(s32(b)), "r"(c) : "memory"); }
__device__ __forceinline__ void btx(uint64_t* b, uint32_t n) { asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(s32(b)), "r"(n) : "memory"); }
__device__ __forceinline__ void bwait(uint64_t* b, uint32_t ph) { asm volatile("{\n.reg .pred P1;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n@P1 bra D;\nbra W;\nD:\n}\n" :: "r"(s32(b)), "r"(ph) : "memory"); }
__device__ __forceinline__ void bulk(void* d, const void* s, uint32_t n, uint64_t* b) { asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" :: "r"(s32(d)), "l"(s), "r"(n), "r"(s32(b)) : "memory"); }

__global__ void ring_kernel(const float* A, size_t total_bytes, int stage_bytes, int S, float* out) {
  extern __shared__ __align__(1024) unsigned char dyn[];
  uint64_t* full = (uint64_t*)dyn;
  unsigned char* ring = dyn + 1024;
  size_t per = total_bytes / gridDim.x;
  const char* base = (const char*)A + per * blockIdx.x;
  int nst = (int)(per / stage_bytes);
  if (threadIdx.x == 0) { for (int s = 0; s < S; ++s) binit(&full[s], 1); asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
  __syncthreads();
  if (threadIdx.x == 0) for (int c = 0; c < S && c < nst; ++c) { btx(&full[c], stage_bytes); bulk(ring + (size_t)c * stage_bytes, base + (size_t)c * stage_bytes, stage_bytes, &full[c]); }
  float acc = 0;
  for (int c = 0; c < nst; ++c) {
    int s = c % S;
    bwait(&full[s], (c / S) & 1);
    const float4* p = (const float4*)(ring + (size_t)s * stage_bytes);
    for (int q = threadIdx.x; q < stage_bytes / 16; q += blockDim.x) { float4 v = p[q]; acc += v.x + v.y + v.z + v.w; }
    __syncthreads();
    if (threadIdx.x == 0 && c + S < nst) { btx(&full[s], stage_bytes); bulk(ring + (size_t)s * stage_bytes, base + (size_t)(c + S) * stage_bytes, stage_bytes, &full[s]); }
  }
  if (acc == 12345.f) out[0] = acc;
}

__global__ void ldg_kernel(const float4* A, size_t n4, float* out) {
  float acc = 0;
  size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i + 7 * stride < n4; i += 8 * stride) {
    float4 v[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v[k].x), "=f"(v[k].y), "=f"(v[k].z), "=f"(v[k].w) : "l"(A + i + k * stride));
#pragma unroll
    for (int k = 0; k < 8; ++k) acc += v[k].x + v[k].y + v[k].z + v[k].w;
  }
  for (; i < n4; i += stride) { float4 v = A[i]; acc += v.x + v.y + v.z + v.w; }
  if (acc == 12345.f) out[0] = acc;
}

__global__ void read_sweep(const float4* B, size_t n4, float* out) {
  float acc = 0;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x) { float4 v = B[i]; acc += v.x; }
  if (acc == 12345.f) out[0] = acc;
}

int main() {
  size_t maxb = 256ull << 20;
  float *A, *out, *flush, *flush2; CK(cudaMalloc(&A, maxb)); CK(cudaMalloc(&out, 4)); CK(cudaMalloc(&flush, 256ull << 20)); CK(cudaMalloc(&flush2, 256ull << 20));
  CK(cudaMemset(A, 0, maxb)); CK(cudaMemset(flush2, 0, 256ull << 20));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const char* names[3] = {"write-flush", "write+read-flush", "warm (no flush)"};
  for (size_t total : {64ull << 20, 128ull << 20, 256ull << 20}) for (int mode = 0; mode < 3; ++mode) {
    for (int G : {296, 592}) for (int thr : {512}) {
      float best = 1e9, sum = 0;
      for (int r = 0; r < 7; ++r) {
        if (mode <= 1) CK(cudaMemset(flush, r, 256ull << 20));
        if (mode == 1) read_sweep<<<592, 512>>>((const float4*)flush2, (256ull << 20) / 16, out);
        if (mode == 2) ldg_kernel<<<G, thr>>>((const float4*)A, total / 16, out);
        cudaEventRecord(e0); ldg_kernel<<<G, thr>>>((const float4*)A, total / 16, out); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
        float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms; if (r >= 2) sum += ms;
      }
      printf("ldg %-18s total=%zuMB G=%d thr=%d : best %.1f us (%.0f GB/s)  mean %.1f us\n", names[mode], total >> 20, G, thr, best * 1e3, total / (best * 1e-3) / 1e9, sum / 5 * 1e3);
    }
  }
  // empty kernel: launch + event overhead
  float best = 1e9;
  for (int r = 0; r < 20; ++r) { cudaEventRecord(e0); read_sweep<<<1, 32>>>((const float4*)A, 0, out); cudaEventRecord(e1); CK(cudaEventSynchronize(e1)); float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms; }
  printf("empty kernel event time: %.2f us\n", best * 1e3);
  return 0;
}
