// read_probe.cu — the read-only HBM ceiling at the sizes the hot path streams
// (64 MB = one 4096^2 fp32 matrix, 128 MB = BICG + MVT, 256 MB = one 8192^2
// matrix, 4 GB = ATAX 65536x16384), cold L2 (flushed by a 256 MB write and a
// 256 MB read before every launch), CUDA events around the launch only.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/read_probe tools/read_probe.cu
//
// Variants (each sums what it reads so the loads cannot be dropped):
//   ldg-grid   16-B ld.global.nc.L1::no_allocate, U loads in flight per lane,
//              grid-stride over the whole buffer (interleaved CTAs)
//   ldg-band   same loads, each CTA streams one contiguous band (the fused
//              kernel's row-band split)
//   bulk-band  one CTA per SM, a ring of S stages filled by cp.async.bulk
//              (one elected thread), warps sum each stage from shared memory
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>

#define CK(x)                                                                              \
  do {                                                                                     \
    cudaError_t e_ = (x);                                                                  \
    if (e_ != cudaSuccess) {                                                               \
      fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_));           \
      exit(1);                                                                             \
    }                                                                                      \
  } while (0)

__device__ __forceinline__ float4 ld_stream4(const float4* p) {
  float4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
  return r;
}

template <int U>
__global__ void ldg_grid(const float4* __restrict__ a, int64_t n4, float* out) {
  float s = 0.f;
  const int64_t stride = int64_t(gridDim.x) * blockDim.x;
  int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  for (; i + (U - 1) * stride < n4; i += U * stride) {
    float4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = ld_stream4(a + i + u * stride);
#pragma unroll
    for (int u = 0; u < U; ++u) s += v[u].x + v[u].y + v[u].z + v[u].w;
  }
  for (; i < n4; i += stride) {
    float4 v = ld_stream4(a + i);
    s += v.x + v.y + v.z + v.w;
  }
  if (s == 12345.f) out[0] = s;
}

template <int U>
__global__ void ldg_band(const float4* __restrict__ a, int64_t n4, float* out) {
  const int64_t band = (n4 + gridDim.x - 1) / gridDim.x;
  const int64_t b0 = blockIdx.x * band, b1 = std::min<int64_t>(n4, b0 + band);
  float s = 0.f;
  int64_t i = b0 + threadIdx.x;
  const int64_t stride = blockDim.x;
  for (; i + (U - 1) * stride < b1; i += U * stride) {
    float4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = ld_stream4(a + i + u * stride);
#pragma unroll
    for (int u = 0; u < U; ++u) s += v[u].x + v[u].y + v[u].z + v[u].w;
  }
  for (; i < b1; i += stride) {
    float4 v = ld_stream4(a + i);
    s += v.x + v.y + v.z + v.w;
  }
  if (s == 12345.f) out[0] = s;
}

__device__ __forceinline__ uint32_t s_u32(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }
__device__ __forceinline__ void bar_wait(uint64_t* b, uint32_t parity) {
  asm volatile(
      "{\n.reg .pred P1;\nLAB_WAIT:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@P1 bra DONE;\nbra LAB_WAIT;\nDONE:\n}\n" ::"r"(s_u32(b)),
      "r"(parity)
      : "memory");
}

// GRID = false: CTA b streams one contiguous band; GRID = true: CTA b takes
// stage-sized chunks b, b + G, b + 2G, ... (all CTAs inside a narrow window)
template <bool GRID>
__global__ void bulk_kernel(const char* __restrict__ a, int64_t bytes, int stage, int S, float* out) {
  extern __shared__ __align__(1024) unsigned char dyn[];
  uint64_t* full = reinterpret_cast<uint64_t*>(dyn);
  uint64_t* empty = full + S;
  unsigned char* ring = dyn + 1024;
  const int nw = blockDim.x / 32, warp = threadIdx.x >> 5;
  const int64_t band = ((bytes / gridDim.x) + 4095) / 4096 * 4096;
  const int64_t nchunks = (bytes + stage - 1) / stage;
  const int64_t b0 = GRID ? 0 : blockIdx.x * band, b1 = GRID ? bytes : std::min<int64_t>(bytes, b0 + band);
  const int64_t nst = GRID ? (nchunks > blockIdx.x ? (nchunks - blockIdx.x + gridDim.x - 1) / gridDim.x : 0)
                           : (b1 > b0 ? (b1 - b0 + stage - 1) / stage : 0);
  auto off = [&](int64_t c) { return GRID ? (int64_t(blockIdx.x) + c * gridDim.x) * stage : b0 + c * stage; };
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(s_u32(&full[s])), "r"(1));
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(s_u32(&empty[s])), "r"(nw));
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  auto issue = [&](int64_t c) {
    const int s = int(c % S);
    if (c >= S) bar_wait(&empty[s], uint32_t(((c / S) - 1) & 1));
    const uint32_t nb = uint32_t(std::min<int64_t>(stage, b1 - off(c)));
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(s_u32(&full[s])), "r"(nb) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     s_u32(ring + int64_t(s) * stage)),
                 "l"(a + off(c)), "r"(nb), "r"(s_u32(&full[s]))
                 : "memory");
  };
  if (threadIdx.x == 0)
    for (int64_t c = 0; c < std::min<int64_t>(S, nst); ++c) issue(c);
  float acc = 0.f;
  for (int64_t c = 0; c < nst; ++c) {
    const int s = int(c % S);
    bar_wait(&full[s], uint32_t((c / S) & 1));
    const float4* st = reinterpret_cast<const float4*>(ring + int64_t(s) * stage);
    const int n4 = int(std::min<int64_t>(stage, b1 - off(c)) / 16);
    for (int i = threadIdx.x; i < n4; i += blockDim.x) {
      float4 v = st[i];
      acc += v.x + v.y + v.z + v.w;
    }
    __syncwarp();
    if ((threadIdx.x & 31) == 0)
      asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(s_u32(&empty[s])) : "memory");
    if (threadIdx.x == 0 && c + S < nst) issue(c + S);
  }
  (void)warp;
  if (acc == 12345.f) out[0] = acc;
}

// feature-major [nf][ld] fp32 read the KMEANS way: a warp takes 128-point
// groups (lane = 16 bytes), all nf rows of its group, U rows in flight;
// groups dealt round robin over the warps of the grid
template <int U>
__global__ void fm_groups(const float* __restrict__ a, int64_t ld, int64_t np, int nf, float* out) {
  const int lane = threadIdx.x & 31;
  const int64_t ng = (np + 127) / 128;
  const int64_t TW = int64_t(gridDim.x) * (blockDim.x >> 5);
  float s = 0.f;
  for (int64_t g = int64_t(blockIdx.x) * (blockDim.x >> 5) + (threadIdx.x >> 5); g < ng; g += TW) {
    const int64_t p = g * 128 + lane * 4;
    if (p >= np) continue;
    for (int f0 = 0; f0 < nf; f0 += U) {
      float4 v[U];
#pragma unroll
      for (int u = 0; u < U; ++u)
        v[u] = f0 + u < nf ? ld_stream4(reinterpret_cast<const float4*>(a + int64_t(f0 + u) * ld + p))
                           : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
      for (int u = 0; u < U; ++u) s += v[u].x + v[u].y + v[u].z + v[u].w;
    }
  }
  if (s == 12345.f) out[0] = s;
}
// the same array, feature rows in lockstep: rows f = 0..nf-1 in turn, each
// row read by the whole grid (grid-stride over the row's float4s)
template <int U>
__global__ void fm_rows(const float* __restrict__ a, int64_t ld, int64_t np, int nf, float* out) {
  const int64_t n4 = np / 4, stride = int64_t(gridDim.x) * blockDim.x;
  float s = 0.f;
  for (int f = 0; f < nf; ++f) {
    const float4* r = reinterpret_cast<const float4*>(a + int64_t(f) * ld);
    for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n4; i += stride) {
      float4 v = ld_stream4(r + i);
      s += v.x + v.y + v.z + v.w;
    }
  }
  if (s == 12345.f) out[0] = s;
}

__global__ void flush_write(float4* f, int64_t n4) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n4; i += int64_t(gridDim.x) * blockDim.x)
    f[i] = make_float4(1.f, 2.f, 3.f, 4.f);
}
__global__ void flush_read(const float4* f, int64_t n4, float* out) {
  float s = 0.f;
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n4; i += int64_t(gridDim.x) * blockDim.x)
    s += f[i].x;
  if (s == 12345.f) out[0] = s;
}

int main(int argc, char** argv) {
  int reps = argc > 1 ? atoi(argv[1]) : 7;
  int nsm = 0;
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  const int64_t maxb = int64_t(4) << 30;
  char* buf;
  CK(cudaMalloc(&buf, maxb));
  CK(cudaMemset(buf, 0, maxb));
  const int64_t fl = int64_t(256) << 20;
  float4 *fw, *fr;
  float* out;
  CK(cudaMalloc(&fw, fl));
  CK(cudaMalloc(&fr, fl));
  CK(cudaMemset(fr, 0, fl));
  CK(cudaMalloc(&out, 64));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  CK(cudaFuncSetAttribute(bulk_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024));
  CK(cudaFuncSetAttribute(bulk_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024));

  auto timeit = [&](auto launch) {
    std::vector<float> t;
    for (int r = 0; r < reps + 2; ++r) {
      flush_write<<<nsm * 4, 1024>>>(fw, fl / 16);
      flush_read<<<nsm * 4, 1024>>>(fr, fl / 16, out);
      CK(cudaEventRecord(e0));
      launch();
      CK(cudaEventRecord(e1));
      CK(cudaEventSynchronize(e1));
      float ms;
      CK(cudaEventElapsedTime(&ms, e0, e1));
      if (r >= 2) t.push_back(ms);
    }
    CK(cudaGetLastError());
    std::sort(t.begin(), t.end());
    return t[t.size() / 2];
  };
  const int64_t sizes[] = {int64_t(64) << 20, int64_t(128) << 20, int64_t(256) << 20, int64_t(4) << 30};
  {
    const int64_t np = 494020, ld = 494020;
    const int nf = 34;
    const double b = double(np) * nf * 4;
    for (int cps : {1, 2, 4, 8}) {
      for (int U : {4, 8}) {
        float ms = timeit([&] {
          if (U == 4) fm_groups<4><<<nsm * cps, 256>>>((const float*)buf, ld, np, nf, out);
          else fm_groups<8><<<nsm * cps, 256>>>((const float*)buf, ld, np, nf, out);
        });
        printf("kmeans-shape fm-groups cta/sm=%d,thr=256,U=%d %.2f us %.0f GBps\n", cps, U, ms * 1e3, b / (ms * 1e-3) / 1e9);
      }
      float ms = timeit([&] { fm_rows<1><<<nsm * cps, 256>>>((const float*)buf, ld, np, nf, out); });
      printf("kmeans-shape fm-rows cta/sm=%d,thr=256 %.2f us %.0f GBps\n", cps, ms * 1e3, b / (ms * 1e-3) / 1e9);
    }
    float ms = timeit([&] { ldg_grid<8><<<nsm * 2, 1024>>>((const float4*)buf, int64_t(b / 16), out); });
    printf("kmeans-shape flat ldg-grid U=8 %.2f us %.0f GBps\n", ms * 1e3, b / (ms * 1e-3) / 1e9);
    if (argc > 2) return 0;
  }
  printf("size_MB variant config us GBps\n");
  for (int64_t b : sizes) {
    const int64_t n4 = b / 16;
    auto rep = [&](const char* v, const char* cfg, float ms) {
      printf("%lld %s %s %.2f %.0f\n", (long long)(b >> 20), v, cfg, ms * 1e3, b / (ms * 1e-3) / 1e9);
    };
    for (int cps : {1, 2, 4}) {
      for (int th : {512, 1024}) {
        if (cps * th > 2048) continue;
        char cfg[64];
        snprintf(cfg, sizeof cfg, "cta/sm=%d,thr=%d,U=8", cps, th);
        rep("ldg-grid", cfg, timeit([&] { ldg_grid<8><<<nsm * cps, th>>>((const float4*)buf, n4, out); }));
        rep("ldg-band", cfg, timeit([&] { ldg_band<8><<<nsm * cps, th>>>((const float4*)buf, n4, out); }));
      }
    }
    for (int U : {4, 16}) {
      char cfg[64];
      snprintf(cfg, sizeof cfg, "cta/sm=2,thr=1024,U=%d", U);
      if (U == 4) rep("ldg-grid", cfg, timeit([&] { ldg_grid<4><<<nsm * 2, 1024>>>((const float4*)buf, n4, out); }));
      if (U == 16) rep("ldg-grid", cfg, timeit([&] { ldg_grid<16><<<nsm * 2, 1024>>>((const float4*)buf, n4, out); }));
    }
    for (int stage : {16384, 32768, 49152, 65536}) {
      for (int ringkb : {64, 96, 128, 192}) {
        const int S = ringkb * 1024 / stage;
        if (S < 2 || S * stage > ringkb * 1024) continue;
        char cfg[64];
        snprintf(cfg, sizeof cfg, "stage=%dKB,S=%d,thr=512", stage / 1024, S);
        rep("bulk-band", cfg, timeit([&] {
              bulk_kernel<false><<<nsm, 512, 1024 + S * stage>>>(buf, b, stage, S, out);
            }));
        rep("bulk-grid", cfg, timeit([&] {
              bulk_kernel<true><<<nsm, 512, 1024 + S * stage>>>(buf, b, stage, S, out);
            }));
      }
    }
    fflush(stdout);
  }
  return 0;
}
