// k_syrk.cu — SYRK, C = beta*C + alpha*A*A^T over the full n x n square
// (PolyBench/GPU syrk, Table 2; the 2-D thread-block case of P:246).
//
// LITERAL: block 32 x BY, thread (i = by*BY + ty, j = bx*32 + tx):
//     c = C[i][j] * beta;  for k < m: c = fmaf(alpha * a[i][k], a[j][k], c)
// a[j][k] is memory-divergent across the warp (32 rows of A) and reused for
// 32 consecutive k; a[i][k] is a broadcast. CATT throttles this loop.
// STAGED: 128 x 128 output tiles, 16 k per stage in shared memory (alpha*a_i
// pre-multiplied with the same rounding), 8 x 8 outputs per thread held in
// registers; every output still accumulates k = 0, 1, ..., m-1 in order, so
// the result is bit-identical to LITERAL. FP32 CUDA-core bound (no tensor
// cores: TF32 would break the 1e-5 bar, BASELINE north_star).
#include <cstdint>

#include "internal.h"

namespace catt {

struct SyrkArgs {
  const float* A;
  float* C;
  int64_t n, m;
  float alpha, beta;
  Throttle t;
};

__global__ void __launch_bounds__(1024, 2) syrk_thread_kernel(SyrkArgs a) {
  __shared__ int slots;
  gate_init(&slots, a.t);
  __syncthreads();
  cta_enter(a.t);
  const int64_t j = int64_t(blockIdx.x) * 32 + threadIdx.x;
  const int64_t i = int64_t(blockIdx.y) * blockDim.y + threadIdx.y;
  throttled(a.t, &slots, [&]() {
    if (i >= a.n || j >= a.n) return;
    const int64_t m = a.m;
    const float* __restrict__ ai = a.A + i * m;
    const float* __restrict__ aj = a.A + j * m;
    float c = __fmul_rn(a.C[i * a.n + j], a.beta);
#pragma unroll 8
    for (int64_t k = 0; k < m; ++k) c = fmaf(__fmul_rn(a.alpha, ai[k]), aj[k], c);
    a.C[i * a.n + j] = c;
  });
  cta_exit(a.t);
}

constexpr int BM = 128, BK = 16, TM = 8;
constexpr int PITCH = BM + 4;  // transposed tiles: 16-B aligned rows, spread store banks

// One k-step of the 8 x 8 register tile: c[r][q] = fmaf(alpha*a_i[r], a_j[q], c[r][q]).
__device__ __forceinline__ void syrk_kstep(float (&c)[TM][TM], const float* as, const float* bs, int ty, int tx) {
  const float4 a0 = *reinterpret_cast<const float4*>(as + ty * TM);
  const float4 a1 = *reinterpret_cast<const float4*>(as + ty * TM + 4);
  const float4 b0 = *reinterpret_cast<const float4*>(bs + tx * TM);
  const float4 b1 = *reinterpret_cast<const float4*>(bs + tx * TM + 4);
  const float av[TM] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
  const float bv[TM] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
  for (int r = 0; r < TM; ++r)
#pragma unroll
    for (int q = 0; q < TM; ++q) c[r][q] = fmaf(av[r], bv[q], c[r][q]);
}

__global__ void __launch_bounds__(256, 2) syrk_tiled_kernel(SyrkArgs a) {
  __shared__ __align__(16) float As[2][BK][PITCH];  // alpha * a[i][k], transposed
  __shared__ __align__(16) float Bs[2][BK][PITCH];  // a[j][k], transposed
  cta_enter(a.t);
  const int tid = threadIdx.x;
  const int tx = tid & 15, ty = tid >> 4;
  const int64_t i0 = int64_t(blockIdx.y) * BM, j0 = int64_t(blockIdx.x) * BM;
  const int64_t n = a.n, m = a.m;
  // loader: thread -> row lr = tid / 2 of the tile, k sub-block (tid & 1) * 8 (two float4)
  const int lr = tid >> 1, lk = (tid & 1) * 8;
  const bool vec = (m % 4) == 0 && (reinterpret_cast<uintptr_t>(a.A) & 15u) == 0;
  float c[TM][TM];
#pragma unroll
  for (int r = 0; r < TM; ++r)
#pragma unroll
    for (int q = 0; q < TM; ++q) {
      const int64_t gi = i0 + ty * TM + r, gj = j0 + tx * TM + q;
      c[r][q] = (gi < n && gj < n) ? __fmul_rn(a.C[gi * n + gj], a.beta) : 0.0f;
    }
  float ra[8], rb[8];
  auto gload = [&](int64_t k0) {
    const int64_t gi = i0 + lr, gj = j0 + lr, kb = k0 + lk;
    if (vec && kb + 8 <= m) {
      const float4* pa = reinterpret_cast<const float4*>(a.A + gi * m + kb);
      const float4* pb = reinterpret_cast<const float4*>(a.A + gj * m + kb);
      const float4 z = make_float4(0.f, 0.f, 0.f, 0.f);
      const float4 a0 = gi < n ? pa[0] : z, a1 = gi < n ? pa[1] : z;
      const float4 b0 = gj < n ? pb[0] : z, b1 = gj < n ? pb[1] : z;
      ra[0] = __fmul_rn(a.alpha, a0.x); ra[1] = __fmul_rn(a.alpha, a0.y);
      ra[2] = __fmul_rn(a.alpha, a0.z); ra[3] = __fmul_rn(a.alpha, a0.w);
      ra[4] = __fmul_rn(a.alpha, a1.x); ra[5] = __fmul_rn(a.alpha, a1.y);
      ra[6] = __fmul_rn(a.alpha, a1.z); ra[7] = __fmul_rn(a.alpha, a1.w);
      rb[0] = b0.x; rb[1] = b0.y; rb[2] = b0.z; rb[3] = b0.w;
      rb[4] = b1.x; rb[5] = b1.y; rb[6] = b1.z; rb[7] = b1.w;
    } else {
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int64_t k = kb + u;
        ra[u] = (gi < n && k < m) ? __fmul_rn(a.alpha, a.A[gi * m + k]) : 0.0f;
        rb[u] = (gj < n && k < m) ? a.A[gj * m + k] : 0.0f;
      }
    }
  };
  auto sstore = [&](int buf) {
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      As[buf][lk + u][lr] = ra[u];
      Bs[buf][lk + u][lr] = rb[u];
    }
  };
  const int64_t ktiles = (m + BK - 1) / BK;
  gload(0);
  sstore(0);
  __syncthreads();
  for (int64_t kt = 0; kt < ktiles; ++kt) {
    const int buf = int(kt & 1);
    if (kt + 1 < ktiles) gload((kt + 1) * BK);
    const int kvalid = int(imin64(BK, m - kt * BK));  // uniform: never run k >= m
    if (kvalid == BK) {
#pragma unroll
      for (int kk = 0; kk < BK; ++kk) syrk_kstep(c, &As[buf][kk][0], &Bs[buf][kk][0], ty, tx);
    } else {
      for (int kk = 0; kk < kvalid; ++kk) syrk_kstep(c, &As[buf][kk][0], &Bs[buf][kk][0], ty, tx);
    }
    if (kt + 1 < ktiles) sstore(buf ^ 1);
    __syncthreads();
  }
#pragma unroll
  for (int r = 0; r < TM; ++r) {
    const int64_t gi = i0 + ty * TM + r;
    if (gi >= n) continue;
    float* crow = a.C + gi * n + j0 + tx * TM;
    if (j0 + tx * TM + TM <= n && (n % 4) == 0) {
      reinterpret_cast<float4*>(crow)[0] = make_float4(c[r][0], c[r][1], c[r][2], c[r][3]);
      reinterpret_cast<float4*>(crow)[1] = make_float4(c[r][4], c[r][5], c[r][6], c[r][7]);
    } else {
#pragma unroll
      for (int q = 0; q < TM; ++q)
        if (j0 + tx * TM + q < n) crow[q] = c[r][q];
    }
  }
  cta_exit(a.t);
}

const void* syrk_func(int variant) {
  return variant == CATT_VAR_STAGED ? (const void*)syrk_tiled_kernel : (const void*)syrk_thread_kernel;
}

}  // namespace catt

using namespace catt;

extern "C" catt_status catt_syrk(const float* A, float* C, int64_t n, int64_t m, float alpha, float beta,
                                 const catt_throttle* t, void* stream) {
  if (n < 0 || m < 0 || n > (int64_t(1) << 31) || m > (int64_t(1) << 31)) return CATT_EINVAL;
  if (n > 0 && (!A || !C)) return CATT_EINVAL;
  if (n == 0) return CATT_OK;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  SyrkArgs a{A, C, n, m, alpha, beta, Throttle{}};
  const int var = variant_of(t);
  if (var == CATT_VAR_LITERAL) {
    const int threads = cta_threads_or(t, 256);
    if (threads % 32) return CATT_EINVAL;
    const int by = threads / 32;
    size_t dyn = 0;
    catt_status st = prepare_launch((const void*)syrk_thread_kernel, t, threads, 0, true, &a.t, &dyn);
    if (st != CATT_OK) return st;
    dim3 grid(unsigned((n + 31) / 32), unsigned((n + by - 1) / by));
    if (grid.y > 65535) return CATT_EINVAL;
    syrk_thread_kernel<<<grid, dim3(32, by), dyn, s>>>(a);
    return after_launch();
  }
  if (var == CATT_VAR_STAGED) {
    if (t && t->cta_threads != 0 && t->cta_threads != 256) return CATT_EINVAL;
    size_t dyn = 0;
    catt_status st = prepare_launch((const void*)syrk_tiled_kernel, t, 256, 0, false, &a.t, &dyn);
    if (st != CATT_OK) return st;
    dim3 grid(unsigned((n + BM - 1) / BM), unsigned((n + BM - 1) / BM));
    if (grid.y > 65535) return CATT_EINVAL;
    syrk_tiled_kernel<<<grid, 256, dyn, s>>>(a);
    return after_launch();
  }
  return CATT_EINVAL;
}
