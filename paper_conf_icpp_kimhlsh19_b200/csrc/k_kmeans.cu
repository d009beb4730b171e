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
// REGS: the point's features are read once into registers (same arithmetic
// order, bit-identical membership); no L1 reuse is needed.
#include <cfloat>
#include <cstdint>

#include "internal.h"

namespace catt {

struct KmArgs {
  const float* feat;
  const float* clusters;
  int32_t* membership;
  int64_t ld, npoints;
  int nf, k;
  Throttle t;
};

constexpr int kMaxRegsFeatures = 64;

// MAXF = 0: LITERAL; MAXF > 0: REGS with up to MAXF features in registers
template <int MAXF>
__global__ void __launch_bounds__(MAXF == 0 ? 1024 : 256, MAXF == 0 ? 2 : (MAXF <= 40 ? 2 : 1)) kmeans_kernel(KmArgs a) {
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

const void* kmeans_func(int variant, int nf) {
  if (variant != CATT_VAR_REGS) return (const void*)kmeans_kernel<0>;
  return nf <= 40 ? (const void*)kmeans_kernel<40> : (const void*)kmeans_kernel<kMaxRegsFeatures>;
}

}  // namespace catt

using namespace catt;

extern "C" catt_status catt_kmeans_assign(const float* feat, int64_t ld, int64_t npoints, int32_t nf,
                                          const float* clusters, int32_t k, int32_t* membership,
                                          const catt_throttle* t, void* stream) {
  if (npoints < 0 || nf < 1 || k < 1 || ld < npoints || int64_t(nf) * k > 4096) return CATT_EINVAL;
  if (npoints > 0 && (!feat || !clusters || !membership)) return CATT_EINVAL;
  if (npoints == 0) return CATT_OK;
  const int var = variant_of(t);
  if (var != CATT_VAR_LITERAL && var != CATT_VAR_REGS) return CATT_EINVAL;
  const int threads = cta_threads_or(t, 256);
  if (var == CATT_VAR_REGS && (nf > kMaxRegsFeatures || threads > 256)) return CATT_EINVAL;
  KmArgs a{feat, clusters, membership, ld, npoints, nf, k, Throttle{}};
  const size_t dyn = size_t(nf) * size_t(k) * sizeof(float);
  const void* f = kmeans_func(var, nf);
  if (dyn > 48 * 1024 && cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, int(dyn)) != cudaSuccess)
    return after_launch();
  size_t dyn_total = 0;
  catt_status st = prepare_launch(f, t, threads, dyn, true, &a.t, &dyn_total);
  if (st != CATT_OK) return st;
  const int64_t grid = (npoints + threads - 1) / threads;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (var == CATT_VAR_REGS && nf <= 40)
    kmeans_kernel<40><<<dim3(unsigned(grid)), threads, dyn_total, s>>>(a);
  else if (var == CATT_VAR_REGS)
    kmeans_kernel<kMaxRegsFeatures><<<dim3(unsigned(grid)), threads, dyn_total, s>>>(a);
  else
    kmeans_kernel<0><<<dim3(unsigned(grid)), threads, dyn_total, s>>>(a);
  return after_launch();
}
