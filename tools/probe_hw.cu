// Scratch hardware probe (round 1): device props, effective L1D capacity per
// carveout percentage (Fig 3-style footprint sweep), CTA residency vs smem.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("ERR %s at %d: %s\n", #x, __LINE__, cudaGetErrorString(e)); return 1; } } while (0)

__global__ void chase(const int* __restrict__ next, int nlines, int passes, long long* out_cyc, int* sink) {
  int cur = 0;
  // warm pass
  for (int i = 0; i < nlines; ++i) cur = __ldca(next + cur);
  long long t0 = clock64();
  for (int p = 0; p < passes; ++p)
    for (int i = 0; i < nlines; ++i) cur = __ldca(next + cur);
  long long t1 = clock64();
  out_cyc[0] = t1 - t0;
  sink[0] = cur;
}

__device__ __forceinline__ unsigned smid() { unsigned r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }
__device__ __forceinline__ unsigned long long gtime() { unsigned long long r; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(r)); return r; }

__global__ void resid(unsigned long long* rec, unsigned long long spin_ns, int use_pad) {
  extern __shared__ int pad[];
  if (threadIdx.x == 0) {
    unsigned long long t0 = gtime();
    while (gtime() - t0 < spin_ns) {}
    unsigned long long t1 = gtime();
    rec[blockIdx.x * 3 + 0] = smid();
    rec[blockIdx.x * 3 + 1] = t0;
    rec[blockIdx.x * 3 + 2] = t1;
    if (use_pad) pad[0] = 1;
  }
  __syncthreads();
}

int max_conc(std::vector<unsigned long long>& r, int nb, int nsm) {
  int best = 0;
  for (int s = 0; s < nsm; ++s) {
    std::vector<std::pair<unsigned long long,int>> ev;
    for (int b = 0; b < nb; ++b) if ((int)r[b*3] == s) { ev.push_back({r[b*3+1], 1}); ev.push_back({r[b*3+2], -1}); }
    std::sort(ev.begin(), ev.end(), [](auto&a, auto&b){ return a.first < b.first || (a.first == b.first && a.second < b.second); });
    int c = 0; for (auto& e : ev) { c += e.second; best = std::max(best, c); }
  }
  return best;
}

int main() {
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, 0));
  printf("name=%s sms=%d cc=%d.%d smemPerSM=%zu smemPerBlockOptin=%zu reservedPerBlock=%zu regsPerSM=%d maxBlocksPerSM=%d maxThreadsPerSM=%d l2=%d persistL2max=%d\n",
    p.name, p.multiProcessorCount, p.major, p.minor, p.sharedMemPerMultiprocessor, p.sharedMemPerBlockOptin, p.reservedSharedMemPerBlock,
    p.regsPerMultiprocessor, p.maxBlocksPerMultiProcessor, p.maxThreadsPerMultiProcessor, p.l2CacheSize, p.persistingL2CacheMaxSize);
  int v; cudaDeviceGetAttribute(&v, cudaDevAttrClockRate, 0); printf("clockRate_khz=%d\n", v);
  // L1 capacity sweep
  const int maxbytes = 320 * 1024;
  int nl_max = maxbytes / 128;
  std::vector<int> h(nl_max * 32, 0);
  int *d_next, *d_sink; long long* d_cyc;
  CK(cudaMalloc(&d_next, h.size() * 4)); CK(cudaMalloc(&d_sink, 4)); CK(cudaMalloc(&d_cyc, 8));
  int pcts[] = {0, 3, 10, 20, 35, 50, 65, 80, 90};
  for (int pct : pcts) {
    CK(cudaFuncSetAttribute(chase, cudaFuncAttributePreferredSharedMemoryCarveout, pct));
    printf("pct=%d:", pct);
    int cap = -1;
    for (int kb = 8; kb <= 320; kb += (kb < 8 ? 4 : 1)) {
      int nl = kb * 1024 / 128;
      for (int l = 0; l < nl; ++l) h[l * 32] = ((l + 1) % nl) * 32;
      CK(cudaMemcpy(d_next, h.data(), nl * 32 * 4, cudaMemcpyHostToDevice));
      chase<<<1, 1>>>(d_next, nl, 4, d_cyc, d_sink);
      CK(cudaDeviceSynchronize());
      long long cyc; CK(cudaMemcpy(&cyc, d_cyc, 8, cudaMemcpyDeviceToHost));
      double per = (double)cyc / (4.0 * nl);
      if (per < 80) cap = kb;
      if (kb % 32 == 0 || per > 45) printf(" %d:%.0f", kb, per);
      if (per > 150 && kb > cap + 8) break;
    }
    printf("  => L1cap~%dKB\n", cap);
  }
  // residency
  unsigned long long* d_rec; int nb = p.multiProcessorCount * 40;
  CK(cudaMalloc(&d_rec, nb * 3 * 8));
  std::vector<unsigned long long> r(nb * 3);
  int rp[] = {0, 3, 20, 90};
  int dyn[] = {0, 128, 1024, 3072, 7168, 15360};
  for (int threads : {256, 64}) for (int pct : rp) for (int d : dyn) {
    CK(cudaFuncSetAttribute(resid, cudaFuncAttributePreferredSharedMemoryCarveout, pct));
    CK(cudaFuncSetAttribute(resid, cudaFuncAttributeMaxDynamicSharedMemorySize, 16384));
    resid<<<nb, threads, d>>>(d_rec, 200000, d > 0);
    CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(r.data(), d_rec, nb * 3 * 8, cudaMemcpyDeviceToHost));
    int occ; CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, resid, threads, d));
    printf("resid threads=%d pct=%d dyn=%d -> maxconc=%d occAPI=%d\n", threads, pct, d, max_conc(r, nb, p.multiProcessorCount), occ);
  }
  cudaFuncAttributes fa; CK(cudaFuncGetAttributes(&fa, resid));
  printf("resid attrs: regs=%d static_smem=%zu\n", fa.numRegs, fa.sharedSizeBytes);
  return 0;
}
