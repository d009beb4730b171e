// launch_probe.cu — CUDA-event time of an (almost) empty 148-CTA launch after
// a 256 MB flush kernel, by launch form: plain, with ~200 KB of dynamic shared
// memory (carveout switch), cooperative, cooperative + cluster attribute, and
// the same after a kernel that already used the large carveout.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/launch_probe tools/launch_probe.cu
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <vector>

__global__ void empty_k(int* out) {
  extern __shared__ int sm[];
  if (threadIdx.x == 0 && blockIdx.x == 100000) out[0] = sm[0];
}
__global__ void flush_k(float4* f, long long n4) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n4; i += (long long)gridDim.x * blockDim.x)
    f[i] = make_float4(1.f, 2.f, 3.f, 4.f);
}

int main() {
  float4* f;
  int* out;
  const long long fl = 256ll << 20;
  cudaMalloc(&f, fl);
  cudaMalloc(&out, 64);
  cudaFuncSetAttribute(empty_k, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  auto run = [&](const char* name, size_t smem, bool coop, bool cluster, bool preflush) {
    std::vector<float> t;
    for (int r = 0; r < 25; ++r) {
      if (preflush) flush_k<<<148 * 4, 1024>>>(f, fl / 16);
      cudaEventRecord(e0);
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(148);
      cfg.blockDim = dim3(544);
      cfg.dynamicSmemBytes = smem;
      cudaLaunchAttribute at[2];
      int na = 0;
      if (coop) {
        at[na].id = cudaLaunchAttributeCooperative;
        at[na].val.cooperative = 1;
        ++na;
      }
      if (cluster) {
        at[na].id = cudaLaunchAttributeClusterDimension;
        at[na].val.clusterDim.x = 1;
        at[na].val.clusterDim.y = 1;
        at[na].val.clusterDim.z = 1;
        ++na;
      }
      cfg.attrs = at;
      cfg.numAttrs = na;
      void* args[] = {&out};
      cudaLaunchKernelExC(&cfg, (const void*)empty_k, args);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      if (r >= 5) t.push_back(ms * 1e3f);
    }
    std::sort(t.begin(), t.end());
    printf("%-44s median %6.2f us  min %6.2f  max %6.2f  (%s)\n", name, t[t.size() / 2], t[0], t.back(),
           cudaGetErrorString(cudaGetLastError()));
  };
  for (int pf = 0; pf < 2; ++pf) {
    printf("-- %s\n", pf ? "after a 256 MB flush kernel" : "back to back");
    run("plain, 0 smem", 0, false, false, pf);
    run("plain, 203 KB smem", 203 * 1024, false, false, pf);
    run("cooperative, 0 smem", 0, true, false, pf);
    run("cooperative, 203 KB smem", 203 * 1024, true, false, pf);
    run("cooperative + cluster(1), 203 KB smem", 203 * 1024, true, true, pf);
    run("plain + cluster(1), 203 KB smem", 203 * 1024, false, true, pf);
  }
  return 0;
}
