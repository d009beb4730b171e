// k_kmeans.cu — KMEANS assignment step (Rodinia kmeans, Table 2; the
// KM rows of Table 3), features stored feature-major.
//
// LITERAL (Rodinia kmeansPoint): thread p, centres staged in shared memory:
//     for c < k: d = 0; for f < nf: diff = feat[f*ld + p] - C[c][f];
//                                   d = fmaf(diff, diff, d)
//                if (d < best) { best = d; index = c; }   (strict <: lowest c wins ties)
// feat[f*ld + p] is coalesced across the warp (C_tid = 1) and re-read for
// every centre: the 34 lines a warp touches per centre must survive in L1
// until the next centre (outer-loop reuse, reading R10). At 494020 points and
// 64 warps per SM this exceeds the L1D at every carveout on B200 (SURVEY 0
// finding 3): the contended configuration where CATT throttles.
// REGS: the features are streamed once (16 B-per-warp-lane loads that do not
// allocate in L1) while the k partial distances of the point stay in
// registers: for f: v = feat[f*ld + p]; for c: d[c] = fmaf(v - C[c][f], ...).
// Every (point, centre) pair still accumulates f = 0, 1, ... in order, so the
// membership is bit-identical to LITERAL; no L1 reuse is needed.
// COOP: a warp takes 128 consecutive points, a lane 4 of them: one 16-byte
// L1-bypassing load per feature (512 B per warp request instead of 128 B),
// FB features in flight per lane. The 4 points are two packed fp32 pairs, so
// one FADD2 + one FFMA2 advance two (point, centre) chains; each half is the
// scalar IEEE operation in the same order: bit-identical membership.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdlib>
#include <cfloat>
#include <cstdint>

#include "f32x2.cuh"
#include "internal.h"
#include "tma.cuh"

namespace catt {

struct KmArgs {
  const float* feat;
  const float* clusters;
  int32_t* membership;
  int64_t ld, npoints;
  int nf, k;
  Throttle t;
};

// MAXF = 0: LITERAL (the only instance; REGS is kmeans_stream_kernel below)
template <int MAXF>
__global__ void __launch_bounds__(1024, 2) kmeans_kernel(KmArgs a) {
  extern __shared__ float s_c[];
  __shared__ int slots;
  const int nck = a.nf * a.k;
  for (int q = threadIdx.x; q < nck; q += blockDim.x) s_c[q] = a.clusters[q];
  gate_init(&slots, a.t);
  __syncthreads();
  cta_enter(a.t);
  const int64_t p = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  throttled(a.t, &slots, [&]() {
    if (p >= a.npoints) return;
    const float* __restrict__ f0 = a.feat + p;
    const int64_t ld = a.ld;
    const int nf = a.nf;
    int index = -1;
    float best = FLT_MAX;
    if (MAXF == 0) {
      for (int c = 0; c < a.k; ++c) {
        const float* cc = s_c + c * nf;
        float d = 0.0f;
#pragma unroll 2
        for (int f = 0; f < nf; ++f) {
          const float diff = f0[int64_t(f) * ld] - cc[f];
          d = fmaf(diff, diff, d);
        }
        if (d < best) {
          best = d;
          index = c;
        }
      }
    } else {
      float v[MAXF > 0 ? MAXF : 1];
#pragma unroll
      for (int f = 0; f < MAXF; ++f) v[f] = (f < nf) ? f0[int64_t(f) * ld] : 0.0f;
      for (int c = 0; c < a.k; ++c) {
        const float* cc = s_c + c * nf;
        float d = 0.0f;
#pragma unroll
        for (int f = 0; f < MAXF; ++f) {
          if (f < nf) {
            const float diff = v[f] - cc[f];
            d = fmaf(diff, diff, d);
          }
        }
        if (d < best) {
          best = d;
          index = c;
        }
      }
    }
    a.membership[p] = index;
  });
  cta_exit(a.t);
}

// REGS: centres transposed in shared memory (s_ct[f*k + c]) so the k values
// of one feature are a broadcast; KMAX partial distances per thread.
template <int KMAX>
__global__ void __launch_bounds__(256) kmeans_stream_kernel(KmArgs a) {
  extern __shared__ float s_ct[];
  __shared__ int slots;
  const int nf = a.nf, k = a.k;
  for (int q = threadIdx.x; q < nf * k; q += blockDim.x) {
    const int c = q / nf, f = q % nf;
    s_ct[f * k + c] = a.clusters[q];
  }
  gate_init(&slots, a.t);
  __syncthreads();
  cta_enter(a.t);
  const int64_t p = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  throttled(a.t, &slots, [&]() {
    if (p >= a.npoints) return;
    const float* f0 = a.feat + p;
    const int64_t ld = a.ld;
    float d[KMAX];
#pragma unroll
    for (int c = 0; c < KMAX; ++c) d[c] = 0.0f;
    int f = 0;
    for (; f + 8 <= nf; f += 8) {
      float v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const float* q = f0 + int64_t(f + u) * ld;
        asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v[u]) : "l"(q));
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const float* cc = s_ct + (f + u) * k;
#pragma unroll
        for (int c = 0; c < KMAX; ++c) {
          if (c < k) {
            const float diff = v[u] - cc[c];
            d[c] = fmaf(diff, diff, d[c]);
          }
        }
      }
    }
    for (; f < nf; ++f) {
      const float v = f0[int64_t(f) * ld];
      const float* cc = s_ct + f * k;
#pragma unroll
      for (int c = 0; c < KMAX; ++c) {
        if (c < k) {
          const float diff = v - cc[c];
          d[c] = fmaf(diff, diff, d[c]);
        }
      }
    }
    int index = -1;
    float best = FLT_MAX;
#pragma unroll
    for (int c = 0; c < KMAX; ++c) {
      if (c < k && d[c] < best) {
        best = d[c];
        index = c;
      }
    }
    a.membership[p] = index;
  });
  cta_exit(a.t);
}


// COOP (see the header): centres duplicated into pairs (c, c) in shared
// memory, [nf][KP] with KP = KMAX rounded up to 2, read as 16-byte
// broadcasts; padding centres are +inf (never strictly nearer than FLT_MAX).
// One 128-point group per warp, FB features in flight per lane, register-lean
// (4 CTAs of 256 threads per SM): on B200 this feature-major pattern streams
// fastest with many warps and few loads each (tools/read_probe.cu fm-groups:
// 32 warps/SM x 4 loads beat 16 x 8 and persistent software pipelining).
template <int KMAX, int FB>
__global__ void __launch_bounds__(256, 4) kmeans_coop_kernel(KmArgs a) {
  constexpr int KP = (KMAX + 1) & ~1;
  extern __shared__ __align__(16) unsigned char dyn_c[];
  uint64_t* s_cd = reinterpret_cast<uint64_t*>(dyn_c);
  const int nf = a.nf, k = a.k;
  for (int q = threadIdx.x; q < nf * KP; q += blockDim.x) {
    const int f = q / KP, c = q - f * KP;
    const float v = c < k ? a.clusters[c * nf + f] : __int_as_float(0x7f800000);
    s_cd[q] = f2_pack(v, v);
  }
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int64_t g = int64_t(blockIdx.x) * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const int64_t p = g * 128 + lane * 4;
  if (p >= a.npoints) return;                        // p + 3 < ld: the 16-byte load stays inside row f
  const float* __restrict__ src = a.feat + p;
  const int64_t ld = a.ld;
  uint64_t d01[KMAX], d23[KMAX];
#pragma unroll
  for (int c = 0; c < KMAX; ++c) d01[c] = d23[c] = 0ull;
#pragma unroll 1
  for (int f0 = 0; f0 < nf; f0 += FB) {
    float4 v[FB];
#pragma unroll
    for (int u = 0; u < FB; ++u) {
      v[u] = make_float4(0.f, 0.f, 0.f, 0.f);
      if (f0 + u < nf)
        asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0, %1, %2, %3}, [%4];"
                     : "=f"(v[u].x), "=f"(v[u].y), "=f"(v[u].z), "=f"(v[u].w)
                     : "l"(src + int64_t(f0 + u) * ld));
    }
#pragma unroll
    for (int u = 0; u < FB; ++u) {
      if (f0 + u < nf) {
        const uint64_t v01 = f2_pack(v[u].x, v[u].y), v23 = f2_pack(v[u].z, v[u].w);
        const ulonglong2* cf = reinterpret_cast<const ulonglong2*>(s_cd + (f0 + u) * KP);
#pragma unroll
        for (int q = 0; q < KP / 2; ++q) {
          const ulonglong2 c2 = cf[q];
          {
            const uint64_t e01 = f2_sub(v01, c2.x), e23 = f2_sub(v23, c2.x);
            d01[2 * q] = f2_fma(e01, e01, d01[2 * q]);
            d23[2 * q] = f2_fma(e23, e23, d23[2 * q]);
          }
          if (2 * q + 1 < KMAX) {
            const uint64_t e01 = f2_sub(v01, c2.y), e23 = f2_sub(v23, c2.y);
            d01[2 * q + 1] = f2_fma(e01, e01, d01[2 * q + 1]);
            d23[2 * q + 1] = f2_fma(e23, e23, d23[2 * q + 1]);
          }
        }
      }
    }
  }
  int idx[4];
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    int index = -1;
    float best = FLT_MAX;
#pragma unroll
    for (int c = 0; c < KMAX; ++c) {
      const float dv = j == 0 ? f2_lo(d01[c]) : j == 1 ? f2_hi(d01[c]) : j == 2 ? f2_lo(d23[c]) : f2_hi(d23[c]);
      if (dv < best) {
        best = dv;
        index = c;
      }
    }
    idx[j] = index;
  }
  int32_t* m = a.membership + p;
  if (p + 3 < a.npoints && (reinterpret_cast<uintptr_t>(m) & 15u) == 0) {
    *reinterpret_cast<int4*>(m) = make_int4(idx[0], idx[1], idx[2], idx[3]);
  } else {
#pragma unroll
    for (int j = 0; j < 4; ++j)
      if (p + j < a.npoints) m[j] = idx[j];
  }
}

const void* kmeans_coop_fn(int k) {
  if (k <= 2) return (const void*)kmeans_coop_kernel<2, 4>;
  if (k <= 4) return (const void*)kmeans_coop_kernel<4, 4>;
  if (k == 5) return (const void*)kmeans_coop_kernel<5, 4>;
  return (const void*)kmeans_coop_kernel<8, 2>;
}

// STAGED: persistent CTAs; 2-D TMA copies of {256 points x nf features} tiles
// (one request per tile) into an S-stage ring; thread t computes point
// tile*256 + t from shared memory (column t of every feature row: conflict
// free), k partial distances in registers, f ascending: bit-exact membership.

// KP = KMAX rounded up to 4: centres [nf][KP] in shared memory, read as
// float4; the padding centres are +inf, never strictly nearer than FLT_MAX,
// so every distance runs unpredicated (k = 5 uses KMAX = 5: no wasted work).
template <int KMAX, int MINB>
__global__ void __launch_bounds__(256, MINB) kmeans_tma_kernel(const __grid_constant__ CUtensorMap map, KmArgs a,
                                                               int S) {
  constexpr int KP = (KMAX + 3) & ~3;
  extern __shared__ __align__(1024) unsigned char dyn[];
  const int t = threadIdx.x, lane = t & 31, nw = blockDim.x >> 5;
  const int nf = a.nf, k = a.k;
  uint64_t* full = reinterpret_cast<uint64_t*>(dyn);
  uint64_t* empty = full + S;
  float* s_ct = reinterpret_cast<float*>(dyn + 512);                    // [nf][KP] transposed centres
  const int head = 512 + ((nf * KP * 4 + 511) / 512) * 512;
  float* ring = reinterpret_cast<float*>(dyn + ((head + 1023) / 1024) * 1024);
  const int tile_floats = nf * 256;
  const int64_t ntiles_all = (a.npoints + 255) / 256;
  const int64_t G = gridDim.x;
  const int64_t mytiles = ntiles_all > blockIdx.x ? (ntiles_all - blockIdx.x + G - 1) / G : 0;
  for (int q = t; q < nf * KP; q += blockDim.x) {
    const int f = q / KP, cc = q - f * KP;
    s_ct[q] = cc < k ? a.clusters[cc * nf + f] : __int_as_float(0x7f800000);
  }
  if (t == 0) {
    for (int s = 0; s < S; ++s) {
      bar_init(&full[s], 1);
      bar_init(&empty[s], nw);
    }
    fence_barrier_init();
  }
  __syncthreads();
  auto issue = [&](int64_t c) {
    const int s = int(c % S);
    if (c >= S) bar_wait(&empty[s], uint32_t(((c / S) - 1) & 1));
    bar_expect_tx(&full[s], uint32_t(tile_floats) * 4u);
    tma_2d(ring + int64_t(s) * tile_floats, &map, int32_t((blockIdx.x + c * G) * 256), 0, &full[s]);
  };
  if (t == 0)
    for (int64_t c = 0; c < imin64(S, mytiles); ++c) issue(c);
  for (int64_t c = 0; c < mytiles; ++c) {
    const int s = int(c % S);
    bar_wait(&full[s], uint32_t((c / S) & 1));
    const int64_t p = (blockIdx.x + c * G) * 256 + t;
    if (p < a.npoints) {
      const float* col = ring + int64_t(s) * tile_floats + t;
      float d[KMAX];
#pragma unroll
      for (int cc = 0; cc < KMAX; ++cc) d[cc] = 0.0f;
#pragma unroll 4
      for (int f = 0; f < nf; ++f) {
        const float v = col[f * 256];
        const float4* cf = reinterpret_cast<const float4*>(s_ct + f * KP);
#pragma unroll
        for (int q = 0; q < KP / 4; ++q) {
          const float4 c4 = cf[q];
          const float cv[4] = {c4.x, c4.y, c4.z, c4.w};
#pragma unroll
          for (int jj = 0; jj < 4; ++jj)
            if (4 * q + jj < KMAX) {
              const float diff = v - cv[jj];
              d[4 * q + jj] = fmaf(diff, diff, d[4 * q + jj]);
            }
        }
      }
      int index = -1;
      float best = FLT_MAX;
#pragma unroll
      for (int cc = 0; cc < KMAX; ++cc) {
        if (d[cc] < best) {
          best = d[cc];
          index = cc;
        }
      }
      a.membership[p] = index;
    }
    __syncwarp();
    if (lane == 0) bar_arrive(&empty[s]);
    if (t == 0 && c + S < mytiles) issue(c + S);
  }
}

template <int MINB>
const void* kmeans_tma_fn(int k) {
  if (k <= 4) return (const void*)kmeans_tma_kernel<4, MINB>;
  if (k == 5) return (const void*)kmeans_tma_kernel<5, MINB>;
  if (k <= 8) return (const void*)kmeans_tma_kernel<8, MINB>;
  if (k <= 16) return (const void*)kmeans_tma_kernel<16, MINB>;
  return (const void*)kmeans_tma_kernel<32, MINB>;
}

// CTAs per SM of the STAGED kernel (2 by default; CATT_KMEANS_CTAS_PER_SM=1: one CTA, more stages)
int kmeans_tma_minb() {
  static const int v = [] {
    const char* e = getenv("CATT_KMEANS_CTAS_PER_SM");
    return (e && atoi(e) == 1) ? 1 : 2;
  }();
  return v;
}

const void* kmeans_func(int variant, int nf) {
  (void)nf;
  if (variant == CATT_VAR_STAGED) return kmeans_tma_minb() == 2 ? kmeans_tma_fn<2>(8) : kmeans_tma_fn<1>(8);
  if (variant == CATT_VAR_COOP) return kmeans_coop_fn(5);
  if (variant != CATT_VAR_REGS) return (const void*)kmeans_kernel<0>;
  return (const void*)kmeans_stream_kernel<8>;
}

}  // namespace catt

using namespace catt;

namespace {

}  // namespace

namespace catt {
// dynamic shared memory of the STAGED kernel: centres + S tile stages
int64_t kmeans_tma_smem(int nf, int k) {
  const int KMAX = k <= 4 ? 4 : k == 5 ? 5 : k <= 8 ? 8 : k <= 16 ? 16 : 32;
  const int KP = (KMAX + 3) & ~3;
  const int head = ((512 + ((nf * KP * 4 + 511) / 512) * 512 + 1023) / 1024) * 1024;
  const int tile_bytes = nf * 256 * 4;
  const int budget = (kmeans_tma_minb() == 2 ? 108 : 200) * 1024;
  const int S = std::max(2, std::min(8, (budget - head) / tile_bytes));
  return int64_t(head) + int64_t(S) * tile_bytes;
}
}  // namespace catt

namespace {

catt_status launch_kmeans_tma(const float* feat, int64_t ld, int64_t npoints, int32_t nf, const float* clusters,
                              int32_t k, int32_t* membership, const catt_throttle* t, void* stream) {
  if (k > 32 || nf > 256 || ld % 4 || (reinterpret_cast<uintptr_t>(feat) & 15u)) return CATT_EINVAL;
  if (t && (t->active_warps || t->active_ctas || (t->cta_threads && t->cta_threads != 256))) return CATT_EINVAL;
  void* fnp = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fnp, cudaEnableDefault, &q) != cudaSuccess ||
      q != cudaDriverEntryPointSuccess)
    return CATT_ECUDA;
  auto enc = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fnp);
  CUtensorMap map;
  const cuuint64_t dims[2] = {cuuint64_t(npoints), cuuint64_t(nf)};
  const cuuint64_t strides[1] = {cuuint64_t(ld) * 4};
  const cuuint32_t box[2] = {256, cuuint32_t(nf)};
  const cuuint32_t es[2] = {1, 1};
  if (enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(feat), dims, strides, box, es,
          CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
          CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
    return CATT_EINVAL;
  const int tile_bytes = nf * 256 * 4;
  const int KMAX = k <= 4 ? 4 : k == 5 ? 5 : k <= 8 ? 8 : k <= 16 ? 16 : 32;
  const int KP = (KMAX + 3) & ~3;
  const int head = ((512 + ((nf * KP * 4 + 511) / 512) * 512 + 1023) / 1024) * 1024;
  const int minb = kmeans_tma_minb();
  const size_t smem = size_t(kmeans_tma_smem(nf, k));
  const int S = int((int64_t(smem) - head) / tile_bytes);
  const void* f = minb == 2 ? kmeans_tma_fn<2>(k) : kmeans_tma_fn<1>(k);
  cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  KmArgs a{feat, clusters, membership, ld, npoints, nf, k, Throttle{}};
  size_t dyn_total = 0;
  catt_status st = prepare_launch(f, t, 256, smem, false, &a.t, &dyn_total);
  if (st != CATT_OK) return st;
  DevCtx* ctx = nullptr;
  st = dev_ctx(&ctx);
  if (st != CATT_OK) return st;
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, f, 256, dyn_total);
  if (e != cudaSuccess || per_sm < 1) {
    record_cuda_error(e == cudaSuccess ? cudaErrorInvalidConfiguration : e);
    return CATT_ECUDA;
  }
  const int64_t tiles = (npoints + 255) / 256;
  const unsigned grid = unsigned(std::min<int64_t>(tiles, int64_t(std::min(per_sm, minb)) * ctx->hw.num_sms));
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  int stages = S;
  void* args[] = {&map, &a, &stages};
  e = cudaLaunchKernel(f, dim3(grid), dim3(256), args, dyn_total, s);
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  return after_launch();
}

}  // namespace

extern "C" catt_status catt_kmeans_assign(const float* feat, int64_t ld, int64_t npoints, int32_t nf,
                                          const float* clusters, int32_t k, int32_t* membership,
                                          const catt_throttle* t, void* stream) {
  if (npoints < 0 || nf < 1 || k < 1 || ld < npoints || int64_t(nf) * k > 4096) return CATT_EINVAL;
  if (npoints > 0 && (!feat || !clusters || !membership)) return CATT_EINVAL;
  if (npoints == 0) return CATT_OK;
  const int var = variant_of(t);
  if (var == CATT_VAR_STAGED) return launch_kmeans_tma(feat, ld, npoints, nf, clusters, k, membership, t, stream);
  if (var == CATT_VAR_COOP) {
    // no L1-resident reference: nothing to throttle; 16-byte loads need ld % 4 == 0 and an aligned base
    if (k > 8 || ld % 4 || (reinterpret_cast<uintptr_t>(feat) & 15u)) return CATT_EINVAL;
    if (t && (t->active_warps || t->active_ctas || (t->cta_threads && t->cta_threads != 256))) return CATT_EINVAL;
    const void* f = kmeans_coop_fn(k);
    const int KP = ((k <= 2 ? 2 : k <= 4 ? 4 : k == 5 ? 5 : 8) + 1) & ~1;
    const size_t dyn = size_t(nf) * KP * sizeof(uint64_t);
    if (dyn > 48 * 1024 && cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, int(dyn)) != cudaSuccess)
      return after_launch();
    KmArgs a{feat, clusters, membership, ld, npoints, nf, k, Throttle{}};
    const int64_t groups = (npoints + 127) / 128;       // one group per warp
    const unsigned grid = unsigned((groups + 7) / 8);
    void* args[] = {&a};
    cudaError_t e = cudaLaunchKernel(f, dim3(grid), dim3(256), args, dyn, static_cast<cudaStream_t>(stream));
    if (e != cudaSuccess) {
      record_cuda_error(e);
      return CATT_ECUDA;
    }
    return after_launch();
  }
  if (var != CATT_VAR_LITERAL && var != CATT_VAR_REGS) return CATT_EINVAL;
  const int threads = cta_threads_or(t, 256);
  if (var == CATT_VAR_REGS && (k > 32 || threads > 256)) return CATT_EINVAL;
  KmArgs a{feat, clusters, membership, ld, npoints, nf, k, Throttle{}};
  const size_t dyn = size_t(nf) * size_t(k) * sizeof(float);
  const void* f = var == CATT_VAR_REGS ? (k <= 8 ? (const void*)kmeans_stream_kernel<8> : (const void*)kmeans_stream_kernel<32>)
                                       : (const void*)kmeans_kernel<0>;
  if (dyn > 48 * 1024 && cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, int(dyn)) != cudaSuccess)
    return after_launch();
  size_t dyn_total = 0;
  catt_status st = prepare_launch(f, t, threads, dyn, true, &a.t, &dyn_total);
  if (st != CATT_OK) return st;
  const int64_t grid = (npoints + threads - 1) / threads;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (var == CATT_VAR_REGS && k <= 8)
    kmeans_stream_kernel<8><<<dim3(unsigned(grid)), threads, dyn_total, s>>>(a);
  else if (var == CATT_VAR_REGS)
    kmeans_stream_kernel<32><<<dim3(unsigned(grid)), threads, dyn_total, s>>>(a);
  else
    kmeans_kernel<0><<<dim3(unsigned(grid)), threads, dyn_total, s>>>(a);
  return after_launch();
}
