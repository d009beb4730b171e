// fused_floor.cu — the floor under the fused BICG + MVT step (configs[1],
// 134.4 MB read once): CUDA-event time, after the bench's 256 MB flush and a
// GPU sleep, of (1) an empty launch of the fused kernel's shape, and (2) a
// plain streaming read of the same bytes with the fused kernel's load form
// (ld.global.nc.L1::no_allocate.v4, contiguous band per CTA, 8 x 16 B in
// flight per lane), at several grid shapes. Run plainly for event times and
// under ncu for gpu__time_duration / dram bytes.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/fused_floor tools/fused_floor.cu
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

__global__ void empty_k(float* out) {
  extern __shared__ float sm[];
  if (threadIdx.x == 0 && blockIdx.x == 100000) out[0] = sm[0];
}
__global__ void flush_k(float4* f, long long n4) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n4; i += (long long)gridDim.x * blockDim.x)
    f[i] = make_float4(1.f, 2.f, 3.f, 4.f);
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
// each CTA streams a contiguous band; lanes interleave 16-B chunks, U loads in flight
template <int U>
__global__ void read_k(const float4* __restrict__ a, long long n4, float* out) {
  const long long per = (n4 + gridDim.x - 1) / gridDim.x;
  const long long b0 = blockIdx.x * per, b1 = min(n4, b0 + per);
  float s = 0.f;
  long long i = b0 + threadIdx.x;
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
  if (s == -1.f) out[blockIdx.x] = s;
}

int main(int argc, char** argv) {
  // default: BICG + MVT 4096^2 (two matrices + vectors); argv[1]: other byte
  // counts, e.g. 69152800 (KMEANS assign 494020 x 34 + memberships)
  const long long bytes = argc > 1 ? atoll(argv[1]) / 16 * 16 : 134381568;
  const long long n4 = bytes / 16;
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
  cudaFuncSetAttribute(empty_k, cudaFuncAttributeMaxDynamicSharedMemorySize, 203 * 1024);
  auto timed = [&](const char* name, auto launch) {
    std::vector<float> ts;
    for (int r = 0; r < 21; ++r) {
      flush_k<<<148 * 4, 1024>>>(f, fl / 16);
      sleep_k<<<1, 32>>>(400000);
      cudaEventRecord(e0);
      launch();
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      if (r) ts.push_back(ms * 1e3f);
    }
    std::sort(ts.begin(), ts.end());
    const float med = ts[ts.size() / 2];
    printf("%-44s median %7.2f us  min %7.2f  -> %6.0f GB/s over %.1f MB  (%s)\n", name, med, ts.front(),
           bytes / (med * 1e-6) / 1e9, bytes / 1e6, cudaGetErrorString(cudaGetLastError()));
  };
  timed("empty, 148 x 1024, 203 KB smem", [&] { empty_k<<<148, 1024, 203 * 1024>>>(out); });
  timed("read, 148 x 1024, U=8", [&] { read_k<8><<<148, 1024>>>(a, n4, out); });
  timed("read, 296 x 512, U=8", [&] { read_k<8><<<296, 512>>>(a, n4, out); });
  timed("read, 148 x 1024, U=4", [&] { read_k<4><<<148, 1024>>>(a, n4, out); });
  timed("read, 592 x 256, U=8", [&] { read_k<8><<<592, 256>>>(a, n4, out); });
  timed("read, 1184 x 256, U=4", [&] { read_k<4><<<1184, 256>>>(a, n4, out); });
  return 0;
}
