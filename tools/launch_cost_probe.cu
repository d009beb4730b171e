// launch_cost_probe.cu — what the ~6 us of CUDA-event time around an EMPTY
// launch after the bench's L2 flush is made of (profiles/r2/fused/floor.txt:
// 6.1 us event, 3.5 us ncu). Hypothesis: the SMs' L1 / shared-memory split.
// The flush kernel runs with the default (small) carveout; a kernel that
// needs 203 KB of shared memory makes every SM reconfigure the unified L1
// first. Cases (CUDA events, median of 21, each after a 256 MB flush and a
// GPU sleep):
//   empty  0 KB smem / 203 KB smem, after a small-carveout flush
//   empty 203 KB after a flush run at the maximum carveout (same split)
//   the same for a plain streaming read of 69.2 MB (KMEANS assign's bytes)
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/launch_cost_probe tools/launch_cost_probe.cu
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <vector>

__global__ void empty_k(float* out) {
  extern __shared__ float sm[];
  if (threadIdx.x == 0 && blockIdx.x == 100000) out[0] = sm[0];
}
__global__ void flush_k(float4* f, long long n4) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n4; i += (long long)gridDim.x * blockDim.x)
    f[i] = make_float4(1.f, 2.f, 3.f, 4.f);
}
// the same flush, launched with dynamic shared memory so the SMs take the maximum carveout
__global__ void flush_big_k(float4* f, long long n4) {
  extern __shared__ float sm[];
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n4; i += (long long)gridDim.x * blockDim.x)
    f[i] = make_float4(1.f, 2.f, 3.f, 4.f);
  if (n4 < 0) f[0].x = sm[threadIdx.x];
}
__global__ void sleep_k(long long ns) {
  const long long t0 = clock64();
  while (clock64() - t0 < ns) {
  }
}
__device__ __forceinline__ float4 ldnc(const float4* p) {
  float4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
  return r;
}
__global__ void read_k(const float4* __restrict__ a, long long n4, float* out) {
  extern __shared__ float sm[];
  const long long per = (n4 + gridDim.x - 1) / gridDim.x;
  const long long b0 = blockIdx.x * per, b1 = min(n4, b0 + per);
  float s = 0.f;
  long long i = b0 + threadIdx.x;
  constexpr int U = 8;
  for (; i + (U - 1) * (long long)blockDim.x < b1; i += U * (long long)blockDim.x) {
    float4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = ldnc(a + i + u * (long long)blockDim.x);
#pragma unroll
    for (int u = 0; u < U; ++u) s += v[u].x + v[u].y + v[u].z + v[u].w;
  }
  for (; i < b1; i += blockDim.x) {
    const float4 v = ldnc(a + i);
    s += v.x + v.y + v.z + v.w;
  }
  if (s == -1.f) out[blockIdx.x] = s + sm[0];
}

int main() {
  const long long bytes = 69152800ll / 16 * 16, n4 = bytes / 16;
  float4 *a, *f;
  float* out;
  cudaMalloc(&a, bytes);
  cudaMemset(a, 0, bytes);
  const long long fl = 256ll << 20;
  cudaMalloc(&f, fl);
  cudaMalloc(&out, 1 << 20);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int big = 203 * 1024;
  cudaFuncSetAttribute(empty_k, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaFuncSetAttribute(read_k, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaFuncSetAttribute(flush_big_k, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  auto timed = [&](const char* name, int flush_kind, auto launch) {
    std::vector<float> ts;
    for (int r = 0; r < 21; ++r) {
      if (flush_kind == 0) flush_k<<<148 * 4, 1024>>>(f, fl / 16);
      if (flush_kind == 1) flush_big_k<<<148, 1024, big>>>(f, fl / 16);
      sleep_k<<<1, 32>>>(400000);
      cudaEventRecord(e0);
      launch();
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms = 0;
      cudaEventElapsedTime(&ms, e0, e1);
      ts.push_back(ms * 1000.f);
    }
    std::sort(ts.begin(), ts.end());
    printf("%-60s median %8.2f us  min %8.2f  (%s)\n", name, ts[ts.size() / 2], ts[0],
           cudaGetErrorString(cudaGetLastError()));
  };
  for (int rep = 0; rep < 2; ++rep) {
    timed("empty 148x1024, 0 KB smem, small-carveout flush", 0, [&] { empty_k<<<148, 1024, 0>>>(out); });
    timed("empty 148x1024, 203 KB smem, small-carveout flush", 0, [&] { empty_k<<<148, 1024, big>>>(out); });
    timed("empty 148x1024, 203 KB smem, max-carveout flush", 1, [&] { empty_k<<<148, 1024, big>>>(out); });
    timed("empty 148x1024, 203 KB smem, no flush (sleep only)", 2, [&] { empty_k<<<148, 1024, big>>>(out); });
    timed("two empties 203 KB back to back, small-carveout flush", 0, [&] {
      empty_k<<<148, 1024, big>>>(out);
      empty_k<<<148, 1024, big>>>(out);
    });
    timed("read 69.2 MB 296x512, 0 KB smem, small-carveout flush", 0, [&] { read_k<<<296, 512, 0>>>(a, n4, out); });
    timed("read 69.2 MB 148x1024, 203 KB smem, small-carveout flush", 0, [&] { read_k<<<148, 1024, big>>>(a, n4, out); });
    timed("read 69.2 MB 148x1024, 203 KB smem, max-carveout flush", 1, [&] { read_k<<<148, 1024, big>>>(a, n4, out); });
  }
  return 0;
}
