// k_gemv.cu — the matrix-vector loop families of ATAX, BICG, MVT, GESUMMV.
//
// Row loops (memory-divergent, the loops CATT throttles; Fig 1):
//     thread i:  for j < N:  acc = fmaf(A[i*N + j], x[j], acc)
// Column loops (coalesced, CATT keeps full TLP):
//     thread j:  for i < M:  acc = fmaf(A[i*N + j], v[i], acc)
//
// Variants (catt.h): LITERAL and VEC4 are the paper's loop (the second with
// 16-byte loads) under the CATT throttle, bit-exact to the sequential oracle;
// STAGED keeps the per-thread sequential order but feeds the rows through
// shared memory with cp.async.bulk copies completing on mbarriers (no L1
// reliance: the B200 alternative to throttling, SURVEY 0 finding 4); COOP is
// the coalesced warp-per-row / column-block form with fixed-order shuffle and
// shared-memory reductions (the HBM-roofline variant).
#include <algorithm>
#include <cstdint>
#include <cstdlib>

#include <cooperative_groups.h>

#include "internal.h"

namespace catt {

enum { EPI_STORE = 0, EPI_ACCUM = 1, EPI_GESUMMV = 2, EPI_SUM3 = 3 };

struct RowArgs {
  const float* A;
  const float* B;   // second matrix (GESUMMV), the second and third back to back (SUM3), or nullptr
  const float* x;
  float* y;         // output (EPI_ACCUM: in/out)
  float* tmp;       // GESUMMV: A x
  int64_t M, N;
  float alpha, beta;
  Throttle t;
};

struct ColArgs {
  const float* A;
  const float* v;
  float* y;         // output (EPI_ACCUM: in/out)
  int64_t M, N;     // A is M x N; y has N entries
  Throttle t;
};

// 16-byte / 4-byte loads that do not allocate in L1 (streamed operands of the
// STAGED/COOP variants, flagged CATT_REF_NOT_L1 in their descriptors).
__device__ __forceinline__ float4 ld_na4(const float4* p) {
  float4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ float ld_na(const float* p) {
  float r;
  asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(r) : "l"(p));
  return r;
}

template <int NMAT, int EPI>
__device__ __forceinline__ void row_epilogue(const RowArgs& a, int64_t i, float acc, float acc2, float acc3 = 0.0f) {
  if (EPI == EPI_SUM3) {
    a.y[i] = __fadd_rn(__fadd_rn(acc, acc2), acc3);
  } else if (EPI == EPI_GESUMMV) {
    a.tmp[i] = acc;
    a.y[i] = __fmaf_rn(a.alpha, acc, __fmul_rn(a.beta, acc2));
  } else {
    a.y[i] = acc;
  }
}

// ---------------------------------------------------------------- row, thread per row
// VM: 0 = the literal scalar loop (loads through L1), 1 = VEC4 (16-byte loads),
// 2 = BYPASS (the literal loop with ld.global.cg matrix loads: cached in L2
// only, so the divergent rows never occupy L1; the alternative to throttling
// that the paper discusses as related work)
template <int NMAT, int EPI, int VM>
__global__ void __launch_bounds__(1024, (NMAT >= 2 && VM == 1) ? 1 : 2) row_thread_kernel(RowArgs a) {
  constexpr bool VEC = VM == 1, BYPASS = VM == 2;
  static_assert(NMAT < 3 || VM == 0, "the 3-matrix row loop is literal only");
  __shared__ int slots;
  gate_init(&slots, a.t);
  __syncthreads();
  cta_enter(a.t);
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  throttled(a.t, &slots, [&]() {
    if (i >= a.M) return;
    const int64_t N = a.N;
    const float* __restrict__ ar = a.A + i * N;
    const float* __restrict__ br = (NMAT >= 2) ? a.B + i * N : nullptr;
    const float* __restrict__ cr = (NMAT == 3) ? a.B + a.M * N + i * N : nullptr;
    const float* __restrict__ x = a.x;
    float acc = (EPI == EPI_ACCUM) ? a.y[i] : 0.0f;
    float acc2 = 0.0f, acc3 = 0.0f;
    if (!VEC) {
#pragma unroll 2
      for (int64_t j = 0; j < N; ++j) {
        const float xv = x[j];
        acc = fmaf(BYPASS ? __ldcg(ar + j) : ar[j], xv, acc);
        if (NMAT >= 2) acc2 = fmaf(BYPASS ? __ldcg(br + j) : br[j], xv, acc2);
        if (NMAT == 3) acc3 = fmaf(cr[j], xv, acc3);
      }
    } else {
      const float4* __restrict__ a4 = reinterpret_cast<const float4*>(ar);
      const float4* __restrict__ b4 = reinterpret_cast<const float4*>(br);
      const float4* __restrict__ x4 = reinterpret_cast<const float4*>(x);
      const float4* const aend = a4 + (N >> 2);
#pragma unroll 1
      for (; a4 < aend; ++a4, ++x4) {
        const float4 xv = *x4;
        const float4 av = *a4;
        acc = fmaf(av.x, xv.x, acc);
        acc = fmaf(av.y, xv.y, acc);
        acc = fmaf(av.z, xv.z, acc);
        acc = fmaf(av.w, xv.w, acc);
        if (NMAT == 2) {
          const float4 bv = *b4++;
          acc2 = fmaf(bv.x, xv.x, acc2);
          acc2 = fmaf(bv.y, xv.y, acc2);
          acc2 = fmaf(bv.z, xv.z, acc2);
          acc2 = fmaf(bv.w, xv.w, acc2);
        }
      }
    }
    row_epilogue<NMAT, EPI>(a, i, acc, acc2, acc3);
  });
  cta_exit(a.t);
}

// ---------------------------------------------------------------- row, warps per row (COOP)
// S warps share a row (S = 1, 2, 4, 8; 8 warps per CTA, 8/S rows per CTA):
// warp part p reads 16-byte chunks p*32 + lane + 32*S*t of the row, U chunks
// in flight per lane; lane partial sums are added by a fixed xor tree, the S
// warp partials in warp order (deterministic).
template <int NMAT, int EPI, bool VEC, int S>
__global__ void __launch_bounds__(256, VEC ? 2 : 3) row_warp_kernel(RowArgs a) {
  constexpr int U = NMAT == 2 ? 4 : 8;
  __shared__ int slots;
  __shared__ float red[2][8];
  gate_init(&slots, a.t);
  __syncthreads();
  cta_enter(a.t);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, part = warp % S;
  const int64_t i = int64_t(blockIdx.x) * (8 / S) + warp / S;
  float acc = 0.0f, acc2 = 0.0f;
  throttled(a.t, &slots, [&]() {
    if (i >= a.M) return;  // warp-uniform
    const int64_t N = a.N;
    if (VEC) {
      const float4* ar = reinterpret_cast<const float4*>(a.A + i * N);
      const float4* br = reinterpret_cast<const float4*>(NMAT == 2 ? a.B + i * N : a.A);
      const float4* x4 = reinterpret_cast<const float4*>(a.x);
      const int64_t n4 = N >> 2, step = 32 * S;
      int64_t j = part * 32 + lane;
      for (; j + (U - 1) * step < n4; j += U * step) {
        float4 v[U], w[NMAT == 2 ? U : 1];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          v[u] = ld_na4(ar + j + u * step);
          if (NMAT == 2) w[u] = ld_na4(br + j + u * step);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const float4 xv = x4[j + u * step];
          acc = fmaf(v[u].x, xv.x, acc);
          acc = fmaf(v[u].y, xv.y, acc);
          acc = fmaf(v[u].z, xv.z, acc);
          acc = fmaf(v[u].w, xv.w, acc);
          if (NMAT == 2) {
            acc2 = fmaf(w[u].x, xv.x, acc2);
            acc2 = fmaf(w[u].y, xv.y, acc2);
            acc2 = fmaf(w[u].z, xv.z, acc2);
            acc2 = fmaf(w[u].w, xv.w, acc2);
          }
        }
      }
      for (; j < n4; j += step) {
        const float4 v = ld_na4(ar + j), xv = x4[j];
        acc = fmaf(v.x, xv.x, acc);
        acc = fmaf(v.y, xv.y, acc);
        acc = fmaf(v.z, xv.z, acc);
        acc = fmaf(v.w, xv.w, acc);
        if (NMAT == 2) {
          const float4 w = ld_na4(br + j);
          acc2 = fmaf(w.x, xv.x, acc2);
          acc2 = fmaf(w.y, xv.y, acc2);
          acc2 = fmaf(w.z, xv.z, acc2);
          acc2 = fmaf(w.w, xv.w, acc2);
        }
      }
    } else {
      const float* ar = a.A + i * N;
      const float* br = NMAT == 2 ? a.B + i * N : a.A;
#pragma unroll 4
      for (int64_t j = part * 32 + lane; j < N; j += 32 * S) {
        const float xv = a.x[j];
        acc = fmaf(ld_na(ar + j), xv, acc);
        if (NMAT == 2) acc2 = fmaf(ld_na(br + j), xv, acc2);
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      acc += __shfl_xor_sync(0xffffffffu, acc, o);
      if (NMAT == 2) acc2 += __shfl_xor_sync(0xffffffffu, acc2, o);
    }
  });
  if (S > 1) {
    if (lane == 0) {
      red[0][warp] = acc;
      red[1][warp] = acc2;
    }
    __syncthreads();
    if (part == 0 && lane == 0) {
      for (int p = 1; p < S; ++p) {
        acc += red[0][warp + p];
        acc2 += red[1][warp + p];
      }
    }
  }
  if (part == 0 && lane == 0 && i < a.M) {
    if (EPI == EPI_ACCUM) acc = a.y[i] + acc;
    row_epilogue<NMAT, EPI>(a, i, acc, acc2);
  }
  cta_exit(a.t);
}

// ---------------------------------------------------------------- column, thread per column
template <int EPI, bool VEC>
__global__ void __launch_bounds__(1024, 2) col_thread_kernel(ColArgs a) {
  __shared__ int slots;
  gate_init(&slots, a.t);
  __syncthreads();
  cta_enter(a.t);
  const int64_t j = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  throttled(a.t, &slots, [&]() {
    const int64_t N = a.N, M = a.M;
    const float* __restrict__ A = a.A;
    const float* __restrict__ v = a.v;
    if (!VEC) {
      if (j >= N) return;
      float acc = (EPI == EPI_ACCUM) ? a.y[j] : 0.0f;
      const float* p = A + j;
#pragma unroll 2
      for (int64_t i = 0; i < M; ++i, p += N) acc = fmaf(*p, v[i], acc);
      a.y[j] = acc;
    } else {
      if (4 * j >= N) return;
      const int64_t n4 = N >> 2;
      const float4* p = reinterpret_cast<const float4*>(A) + j;
      float4 acc = (EPI == EPI_ACCUM) ? reinterpret_cast<const float4*>(a.y)[j] : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll 1
      for (int64_t i = 0; i < M; ++i, p += n4) {
        const float4 av = *p;
        const float vi = v[i];
        acc.x = fmaf(av.x, vi, acc.x);
        acc.y = fmaf(av.y, vi, acc.y);
        acc.z = fmaf(av.z, vi, acc.z);
        acc.w = fmaf(av.w, vi, acc.w);
      }
      reinterpret_cast<float4*>(a.y)[j] = acc;
    }
  });
  cta_exit(a.t);
}

// ---------------------------------------------------------------- ATAX in one literal kernel
// Both ATAX loops in ONE kernel with a throttle per loop (throttling
// "even within a kernel", applied "to individual loops"; PF#1's loops
// get different factors): loop 1 (thread per row: tmp[i] = sum_j A[i][j]
// x[j], memory-divergent) under warp gate t1, a grid barrier (cooperative
// launch), loop 2 (thread per column: y[j] = sum_i A[i][j] tmp[i],
// coalesced) under warp gate t2. The CTA-level cap is one decision for the
// whole kernel, entered and left around each loop. Results are the
// literal loops' (bit-exact to seq-fmaf).
__global__ void __launch_bounds__(1024, 2) atax_onekernel_kernel(RowArgs r, Throttle t2) {
  namespace cg = cooperative_groups;
  __shared__ int slots;
  gate_init(&slots, r.t);
  __syncthreads();
  const int64_t g = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  cta_enter(r.t);
  throttled(r.t, &slots, [&]() {
    if (g >= r.M) return;
    const int64_t N = r.N;
    const float* __restrict__ ar = r.A + g * N;
    float acc = 0.0f;
#pragma unroll 2
    for (int64_t j = 0; j < N; ++j) acc = fmaf(ar[j], r.x[j], acc);
    r.y[g] = acc;                                             // tmp
  });
  cta_exit(r.t);
  __threadfence();
  cg::this_grid().sync();
  gate_init(&slots, t2);
  __syncthreads();
  cta_enter(t2);
  throttled(t2, &slots, [&]() {
    if (g >= r.N) return;
    const int64_t N = r.N, M = r.M;
    const float* __restrict__ tmp = r.y;
    float acc = 0.0f;
    const float* p = r.A + g;
#pragma unroll 2
    for (int64_t i = 0; i < M; ++i, p += N) acc = fmaf(*p, tmp[i], acc);
    r.tmp[g] = acc;                                           // y
  });
  cta_exit(t2);
}

// ---------------------------------------------------------------- column, CTA per 32-column block (COOP)
// Lane l owns column c0 + l; warp w sums rows w, w + NW, ...; the NW partial
// sums are then added in warp order (deterministic).
template <int EPI>
__global__ void __launch_bounds__(1024, 1) col_warp_kernel(ColArgs a) {
  __shared__ int slots;
  __shared__ float red[32][33];
  gate_init(&slots, a.t);
  __syncthreads();
  cta_enter(a.t);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, NW = blockDim.x >> 5;
  const int64_t j = int64_t(blockIdx.x) * 32 + lane;
  float acc = 0.0f;
  throttled(a.t, &slots, [&]() {
    if (j >= a.N) return;
    const int64_t N = a.N, M = a.M;
    const float* col = a.A + j;
    int64_t i = warp;
    for (; i + 7 * NW < M; i += 8 * NW) {
      float w[8], vv[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        w[u] = ld_na(col + (i + int64_t(u) * NW) * N);
        vv[u] = a.v[i + int64_t(u) * NW];
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) acc = fmaf(w[u], vv[u], acc);
    }
    for (; i < M; i += NW) acc = fmaf(ld_na(col + i * N), a.v[i], acc);
  });
  red[warp][lane] = acc;
  __syncthreads();
  if (warp == 0 && j < a.N) {
    float s = red[0][lane];
    for (int w = 1; w < NW; ++w) s += red[w][lane];
    if (EPI == EPI_ACCUM) s = a.y[j] + s;
    a.y[j] = s;
  }
  cta_exit(a.t);
}

// ---------------------------------------------------------------- column, cluster of CTAs per 128-column block (COOP)
// Lane l owns 16-byte column chunk c0 + l (4 columns); the R CTAs of a
// cluster split the rows; warp w of CTA r sums rows r*Mr + w + 8*t. Warp
// partials are added in warp order in shared memory, then CTA 0 adds the R
// CTA partials in rank order through distributed shared memory.
template <int EPI>
__global__ void __launch_bounds__(256) col_cluster_kernel(ColArgs a) {
  namespace cg = cooperative_groups;
  constexpr int U = 8, NW = 8;
  __shared__ int slots;
  __shared__ float4 red[NW][32];
  __shared__ float4 partial[32];
  cg::cluster_group cluster = cg::this_cluster();
  const int R = int(cluster.num_blocks()), rank = int(cluster.block_rank());
  gate_init(&slots, a.t);
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t n4 = a.N >> 2;
  const int64_t jq = int64_t(blockIdx.x) * 32 + lane;
  const int64_t Mr = (a.M + R - 1) / R;
  const int64_t r0 = rank * Mr, r1 = imin64(a.M, r0 + Mr);
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
  throttled(a.t, &slots, [&]() {
    if (jq >= n4) return;
    const float4* col = reinterpret_cast<const float4*>(a.A) + jq;
    int64_t i = r0 + warp;
    for (; i + (U - 1) * NW < r1; i += U * NW) {
      float4 w[U];
      float vv[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        w[u] = ld_na4(col + (i + int64_t(u) * NW) * n4);
        vv[u] = a.v[i + int64_t(u) * NW];
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        acc.x = fmaf(w[u].x, vv[u], acc.x);
        acc.y = fmaf(w[u].y, vv[u], acc.y);
        acc.z = fmaf(w[u].z, vv[u], acc.z);
        acc.w = fmaf(w[u].w, vv[u], acc.w);
      }
    }
    for (; i < r1; i += NW) {
      const float4 w = ld_na4(col + i * n4);
      const float vi = a.v[i];
      acc.x = fmaf(w.x, vi, acc.x);
      acc.y = fmaf(w.y, vi, acc.y);
      acc.z = fmaf(w.z, vi, acc.z);
      acc.w = fmaf(w.w, vi, acc.w);
    }
  });
  red[warp][lane] = acc;
  __syncthreads();
  if (warp == 0) {
    float4 s = red[0][lane];
    for (int w = 1; w < NW; ++w) {
      s.x += red[w][lane].x;
      s.y += red[w][lane].y;
      s.z += red[w][lane].z;
      s.w += red[w][lane].w;
    }
    partial[lane] = s;
  }
  cluster.sync();
  if (rank == 0 && warp == 0 && jq < n4) {
    float4 s = partial[lane];
    for (int q = 1; q < R; ++q) {
      const float4 o = cluster.map_shared_rank(partial, q)[lane];
      s.x += o.x;
      s.y += o.y;
      s.z += o.z;
      s.w += o.w;
    }
    float4* y4 = reinterpret_cast<float4*>(a.y);
    if (EPI == EPI_ACCUM) {
      const float4 y0 = y4[jq];
      s = make_float4(y0.x + s.x, y0.y + s.y, y0.z + s.z, y0.w + s.w);
    }
    y4[jq] = s;
  }
  cluster.sync();
}

// ---------------------------------------------------------------- host launchers
catt_status launch_row_tma(const float* A, const float* B, const float* x, float* y, float* tmp, int64_t M, int64_t N,
                           float alpha, float beta, int epi, const catt_throttle* t, cudaStream_t s);
catt_status launch_col_tma(const float* A, const float* v, float* y, int64_t M, int64_t N, int accumulate,
                           const catt_throttle* t, cudaStream_t s);

namespace {

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

// warps per row for the COOP row loop: enough warps to fill the GPU
int coop_split(int64_t M) {
  const int64_t target = 148 * 32;
  int S = 1;
  while (S < 8 && M * S < target) S *= 2;
  return S;
}

template <int NMAT, int EPI, bool VEC>
const void* row_warp_func(int S) {
  switch (S) {
    case 1: return (const void*)row_warp_kernel<NMAT, EPI, VEC, 1>;
    case 2: return (const void*)row_warp_kernel<NMAT, EPI, VEC, 2>;
    case 4: return (const void*)row_warp_kernel<NMAT, EPI, VEC, 4>;
    default: return (const void*)row_warp_kernel<NMAT, EPI, VEC, 8>;
  }
}

template <int NMAT, int EPI, bool VEC>
void row_warp_launch(int S, unsigned grid, size_t dyn, cudaStream_t s, const RowArgs& a) {
  switch (S) {
    case 1: row_warp_kernel<NMAT, EPI, VEC, 1><<<grid, 256, dyn, s>>>(a); break;
    case 2: row_warp_kernel<NMAT, EPI, VEC, 2><<<grid, 256, dyn, s>>>(a); break;
    case 4: row_warp_kernel<NMAT, EPI, VEC, 4><<<grid, 256, dyn, s>>>(a); break;
    default: row_warp_kernel<NMAT, EPI, VEC, 8><<<grid, 256, dyn, s>>>(a); break;
  }
}

// the 3-matrix row loop (CATT_ROWS_SUM3): literal only, for the decision-rule
// studies (three divergent streams per thread)
catt_status launch_row3(RowArgs a, const catt_throttle* t, cudaStream_t s) {
  if (a.M == 0) return CATT_OK;
  if (variant_of(t) != CATT_VAR_LITERAL) return CATT_EINVAL;
  const int threads = cta_threads_or(t, 256);
  const void* f = (const void*)row_thread_kernel<3, EPI_SUM3, 0>;
  size_t dyn = 0;
  catt_status st = prepare_launch(f, t, threads, 0, true, &a.t, &dyn);
  if (st != CATT_OK) return st;
  row_thread_kernel<3, EPI_SUM3, 0><<<dim3(unsigned((a.M + threads - 1) / threads)), threads, dyn, s>>>(a);
  return after_launch();
}

template <int NMAT, int EPI>
catt_status launch_row_t(RowArgs a, const catt_throttle* t, cudaStream_t s) {
  const int var = variant_of(t);
  if (a.M == 0) return CATT_OK;
  const bool vec_ok = (a.N % 4 == 0) && aligned16(a.A) && aligned16(a.x) && (NMAT == 1 || aligned16(a.B));
  if (var == CATT_VAR_LITERAL || var == CATT_VAR_VEC4 || var == CATT_VAR_BYPASS) {
    const int threads = cta_threads_or(t, 256);
    if (var == CATT_VAR_VEC4 && !vec_ok) return CATT_EINVAL;
    const void* f = var == CATT_VAR_VEC4     ? (const void*)row_thread_kernel<NMAT, EPI, 1>
                    : var == CATT_VAR_BYPASS ? (const void*)row_thread_kernel<NMAT, EPI, 2>
                                             : (const void*)row_thread_kernel<NMAT, EPI, 0>;
    size_t dyn = 0;
    catt_status st = prepare_launch(f, t, threads, 0, true, &a.t, &dyn);
    if (st != CATT_OK) return st;
    const int64_t grid = (a.M + threads - 1) / threads;
    if (var == CATT_VAR_VEC4)
      row_thread_kernel<NMAT, EPI, 1><<<dim3(unsigned(grid)), threads, dyn, s>>>(a);
    else if (var == CATT_VAR_BYPASS)
      row_thread_kernel<NMAT, EPI, 2><<<dim3(unsigned(grid)), threads, dyn, s>>>(a);
    else
      row_thread_kernel<NMAT, EPI, 0><<<dim3(unsigned(grid)), threads, dyn, s>>>(a);
    return after_launch();
  }
  if (var == CATT_VAR_COOP) {
    if (t && t->cta_threads != 0 && t->cta_threads != 256) return CATT_EINVAL;
    const int S = coop_split(a.M);
    const void* f = vec_ok ? row_warp_func<NMAT, EPI, true>(S) : row_warp_func<NMAT, EPI, false>(S);
    size_t dyn = 0;
    catt_status st = prepare_launch(f, t, 256, 0, true, &a.t, &dyn);
    if (st != CATT_OK) return st;
    const unsigned grid = unsigned((a.M + (8 / S) - 1) / (8 / S));
    if (vec_ok)
      row_warp_launch<NMAT, EPI, true>(S, grid, dyn, s, a);
    else
      row_warp_launch<NMAT, EPI, false>(S, grid, dyn, s, a);
    return after_launch();
  }
  if (var == CATT_VAR_STAGED)
    return launch_row_tma(a.A, a.B, a.x, a.y, a.tmp, a.M, a.N, a.alpha, a.beta, EPI, t, s);
  return CATT_EINVAL;
}

template <int EPI>
catt_status launch_col_t(ColArgs a, const catt_throttle* t, cudaStream_t s) {
  const int var = variant_of(t);
  if (a.N == 0) return CATT_OK;
  if (var == CATT_VAR_LITERAL || var == CATT_VAR_VEC4) {
    const int threads = cta_threads_or(t, 256);
    const bool vec = var == CATT_VAR_VEC4;
    if (vec && !((a.N % 4 == 0) && aligned16(a.A) && aligned16(a.y))) return CATT_EINVAL;
    const void* f = vec ? (const void*)col_thread_kernel<EPI, true> : (const void*)col_thread_kernel<EPI, false>;
    size_t dyn = 0;
    catt_status st = prepare_launch(f, t, threads, 0, true, &a.t, &dyn);
    if (st != CATT_OK) return st;
    const int64_t cols = vec ? a.N / 4 : a.N;
    const int64_t grid = (cols + threads - 1) / threads;
    if (vec)
      col_thread_kernel<EPI, true><<<dim3(unsigned(grid)), threads, dyn, s>>>(a);
    else
      col_thread_kernel<EPI, false><<<dim3(unsigned(grid)), threads, dyn, s>>>(a);
    return after_launch();
  }
  if (var == CATT_VAR_COOP) {
    // The cluster/DSMEM form measured slower than the 1024-thread CTA per
    // 32-column block on B200 (profiles/round1_explore_*.txt); kept for
    // CATT_COOP_CLUSTER=1 experiments only.
    const bool vec = (a.N % 4 == 0) && aligned16(a.A) && aligned16(a.y);
    const bool capped = t && t->active_ctas > 0;
    const char* want_cluster = getenv("CATT_COOP_CLUSTER");
    if (vec && !capped && want_cluster && want_cluster[0] == '1') {
      if (t && t->cta_threads != 0 && t->cta_threads != 256) return CATT_EINVAL;
      const void* f = (const void*)col_cluster_kernel<EPI>;
      size_t dyn = 0;
      catt_status st = prepare_launch(f, t, 256, 0, true, &a.t, &dyn);
      if (st != CATT_OK) return st;
      const int64_t nblk = (a.N / 4 + 31) / 32;
      int R = 1;
      while (R < 8 && nblk * R < 2 * 148) R *= 2;
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(unsigned(nblk), unsigned(R), 1);
      cfg.blockDim = dim3(256, 1, 1);
      cfg.dynamicSmemBytes = dyn;
      cfg.stream = s;
      cudaLaunchAttribute attr[1];
      attr[0].id = cudaLaunchAttributeClusterDimension;
      attr[0].val.clusterDim.x = 1;
      attr[0].val.clusterDim.y = unsigned(R);
      attr[0].val.clusterDim.z = 1;
      cfg.attrs = attr;
      cfg.numAttrs = 1;
      cudaError_t e = cudaLaunchKernelEx(&cfg, col_cluster_kernel<EPI>, a);
      if (e != cudaSuccess) {
        record_cuda_error(e);
        return CATT_ECUDA;
      }
      return after_launch();
    }
    const int threads = cta_threads_or(t, 1024);
    const void* f = (const void*)col_warp_kernel<EPI>;
    size_t dyn = 0;
    catt_status st = prepare_launch(f, t, threads, 0, true, &a.t, &dyn);
    if (st != CATT_OK) return st;
    const int64_t grid = (a.N + 31) / 32;
    col_warp_kernel<EPI><<<dim3(unsigned(grid)), threads, dyn, s>>>(a);
    return after_launch();
  }
  if (var == CATT_VAR_STAGED) return launch_col_tma(a.A, a.v, a.y, a.M, a.N, EPI == EPI_ACCUM, t, s);
  return CATT_EINVAL;
}

catt_status check_common(int64_t m, int64_t n) {
  if (m < 0 || n < 0) return CATT_EINVAL;
  if (m > (int64_t(1) << 40) || n > (int64_t(1) << 40)) return CATT_EINVAL;
  return CATT_OK;
}

}  // namespace

const void* row_tma_func(int nmat);
const void* col_tma_func();

// Kernel instance a loop + variant launches (for attributes / descriptors).
const void* gemv_func(int loop, int variant, bool vec_ok) {
  if (loop == CATT_K_ROWS3) return (const void*)row_thread_kernel<3, EPI_SUM3, 0>;
  const bool row = loop == CATT_K_ATAX_1 || loop == CATT_K_BICG_2 || loop == CATT_K_MVT_1 || loop == CATT_K_GESUMMV;
  if (row) {
    const int nmat = loop == CATT_K_GESUMMV ? 2 : 1;
    if (variant == CATT_VAR_STAGED) return row_tma_func(nmat);
    const int vm = variant == CATT_VAR_VEC4 ? 1 : variant == CATT_VAR_BYPASS ? 2 : 0;
    if (loop == CATT_K_GESUMMV) {
      if (variant == CATT_VAR_COOP)
        return vec_ok ? row_warp_func<2, EPI_GESUMMV, true>(1) : row_warp_func<2, EPI_GESUMMV, false>(1);
      return vm == 1 ? (const void*)row_thread_kernel<2, EPI_GESUMMV, 1>
                     : vm == 2 ? (const void*)row_thread_kernel<2, EPI_GESUMMV, 2>
                               : (const void*)row_thread_kernel<2, EPI_GESUMMV, 0>;
    }
    if (loop == CATT_K_MVT_1) {
      if (variant == CATT_VAR_COOP)
        return vec_ok ? row_warp_func<1, EPI_ACCUM, true>(1) : row_warp_func<1, EPI_ACCUM, false>(1);
      return vm == 1 ? (const void*)row_thread_kernel<1, EPI_ACCUM, 1>
                     : vm == 2 ? (const void*)row_thread_kernel<1, EPI_ACCUM, 2>
                               : (const void*)row_thread_kernel<1, EPI_ACCUM, 0>;
    }
    if (variant == CATT_VAR_COOP)
      return vec_ok ? row_warp_func<1, EPI_STORE, true>(1) : row_warp_func<1, EPI_STORE, false>(1);
    return vm == 1 ? (const void*)row_thread_kernel<1, EPI_STORE, 1>
                   : vm == 2 ? (const void*)row_thread_kernel<1, EPI_STORE, 2>
                             : (const void*)row_thread_kernel<1, EPI_STORE, 0>;
  }
  const bool acc = loop == CATT_K_MVT_2;
  if (variant == CATT_VAR_STAGED) return col_tma_func();
  if (variant == CATT_VAR_VEC4) return acc ? (const void*)col_thread_kernel<EPI_ACCUM, true> : (const void*)col_thread_kernel<EPI_STORE, true>;
  if (variant == CATT_VAR_COOP) return acc ? (const void*)col_warp_kernel<EPI_ACCUM> : (const void*)col_warp_kernel<EPI_STORE>;
  return acc ? (const void*)col_thread_kernel<EPI_ACCUM, false> : (const void*)col_thread_kernel<EPI_STORE, false>;
}

catt_status launch_row(const float* A, const float* B, const float* x, float* y, float* tmp, int64_t M, int64_t N,
                       float alpha, float beta, int epi, const catt_throttle* t, cudaStream_t s) {
  RowArgs a{A, B, x, y, tmp, M, N, alpha, beta, Throttle{}};
  if (epi == EPI_SUM3) return launch_row3(a, t, s);
  if (epi == EPI_GESUMMV) return launch_row_t<2, EPI_GESUMMV>(a, t, s);
  if (epi == EPI_ACCUM) return launch_row_t<1, EPI_ACCUM>(a, t, s);
  return launch_row_t<1, EPI_STORE>(a, t, s);
}

catt_status launch_col(const float* A, const float* v, float* y, int64_t M, int64_t N, int epi,
                       const catt_throttle* t, cudaStream_t s) {
  ColArgs a{A, v, y, M, N, Throttle{}};
  if (epi == EPI_ACCUM) return launch_col_t<EPI_ACCUM>(a, t, s);
  return launch_col_t<EPI_STORE>(a, t, s);
}

catt_status launch_fused(bool dep, const float* A, const float* xr, const float* xc, float* yr, float* yc, int64_t M,
                         int64_t N, int row_acc, int col_acc, const catt_throttle* t, cudaStream_t s);

}  // namespace catt

namespace {
bool fused(const catt_throttle* k1, int64_t m, int64_t n) {
  return k1 && k1->variant == CATT_VAR_FUSED && m > 0 && n > 0;
}
catt_throttle coop_of(const catt_throttle* t) {
  catt_throttle c{};
  c.variant = CATT_VAR_COOP;
  (void)t;
  return c;
}
}  // namespace

using namespace catt;

extern "C" catt_status catt_atax(const float* A, const float* x, float* tmp, float* y, int64_t m, int64_t n,
                                 const catt_throttle* k1, const catt_throttle* k2, void* stream) {
  if (check_common(m, n) != CATT_OK || (m * n > 0 && !A) || (n > 0 && (!x || !y)) || (m > 0 && !tmp))
    return CATT_EINVAL;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (fused(k1, m, n)) return launch_fused(true, A, x, nullptr, tmp, y, m, n, 0, 0, k1, s);
  if (k1 && k1->variant == CATT_VAR_FUSED) {   // empty shapes: the per-loop path
    const catt_throttle c = coop_of(k1);
    catt_status st0 = launch_row(A, nullptr, x, tmp, nullptr, m, n, 0.f, 0.f, EPI_STORE, &c, s);
    return st0 != CATT_OK ? st0 : launch_col(A, tmp, y, m, n, EPI_STORE, &c, s);
  }
  catt_status st = launch_row(A, nullptr, x, tmp, nullptr, m, n, 0.f, 0.f, EPI_STORE, k1, s);  // tmp = A x
  if (st != CATT_OK) return st;
  return launch_col(A, tmp, y, m, n, EPI_STORE, k2, s);                                        // y = A^T tmp
}

extern "C" catt_status catt_atax_onekernel(const float* A, const float* x, float* tmp, float* y, int64_t m, int64_t n,
                                           const catt_throttle* k1, const catt_throttle* k2, void* stream) {
  if (check_common(m, n) != CATT_OK || m < 1 || n < 1 || !A || !x || !tmp || !y) return CATT_EINVAL;
  if ((k1 && k1->variant != CATT_VAR_LITERAL) || (k2 && k2->variant != CATT_VAR_LITERAL)) return CATT_EINVAL;
  const int threads = cta_threads_or(k1, 256);
  // one launch: k2 may only choose its warp gate; CTA size, carveout, CTA
  // cap and probe are the kernel's (k1's)
  catt_throttle c2 = k1 ? *k1 : catt_throttle{};
  if (!k1) {
    c2.carveout_kb = -1;
  }
  if (k2) {
    if ((k2->cta_threads && k2->cta_threads != threads) || (k2->active_ctas && k2->active_ctas != c2.active_ctas))
      return CATT_EINVAL;
    c2.active_warps = k2->active_warps;
    c2.gate = k2->gate;
  } else {
    c2.active_warps = 0;
  }
  c2.probe = nullptr;
  const void* f = (const void*)atax_onekernel_kernel;
  RowArgs r{A, nullptr, x, tmp, y, m, n, 0.f, 0.f, Throttle{}};
  Throttle t2{};
  size_t dyn = 0, dyn2 = 0;
  catt_status st = prepare_launch(f, k1, threads, 0, true, &r.t, &dyn);
  if (st != CATT_OK) return st;
  st = prepare_launch(f, &c2, threads, 0, true, &t2, &dyn2);
  if (st != CATT_OK) return st;
  int occ = 0;
  cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, f, threads, dyn);
  DevCtx* ctx = nullptr;
  if ((st = dev_ctx(&ctx)) != CATT_OK) return st;
  const int64_t grid = (std::max(m, n) + threads - 1) / threads;
  if (e != cudaSuccess || occ < 1) {
    record_cuda_error(e == cudaSuccess ? cudaErrorInvalidConfiguration : e);
    return CATT_ECUDA;
  }
  if (grid > int64_t(occ) * ctx->hw.num_sms) return CATT_EUNSUPPORTED;  // the grid barrier needs every CTA resident
  void* args[] = {&r, &t2};
  e = cudaLaunchCooperativeKernel(f, dim3(unsigned(grid)), dim3(unsigned(threads)), args, dyn,
                                  static_cast<cudaStream_t>(stream));
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  return after_launch();
}

extern "C" catt_status catt_bicg(const float* A, const float* p, const float* r, float* q, float* s_out,
                                 int64_t nx, int64_t ny, const catt_throttle* k1, const catt_throttle* k2,
                                 void* stream) {
  if (check_common(nx, ny) != CATT_OK || (nx * ny > 0 && !A) || (ny > 0 && (!p || !s_out)) ||
      (nx > 0 && (!r || !q)))
    return CATT_EINVAL;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (fused(k1, nx, ny)) return launch_fused(false, A, p, r, q, s_out, nx, ny, 0, 0, k1, s);
  if (k1 && k1->variant == CATT_VAR_FUSED) {
    const catt_throttle c = coop_of(k1);
    catt_status st0 = launch_col(A, r, s_out, nx, ny, EPI_STORE, &c, s);
    return st0 != CATT_OK ? st0 : launch_row(A, nullptr, p, q, nullptr, nx, ny, 0.f, 0.f, EPI_STORE, &c, s);
  }
  catt_status st = launch_col(A, r, s_out, nx, ny, EPI_STORE, k1, s);                          // s = A^T r
  if (st != CATT_OK) return st;
  return launch_row(A, nullptr, p, q, nullptr, nx, ny, 0.f, 0.f, EPI_STORE, k2, s);          // q = A p
}

extern "C" catt_status catt_mvt(const float* A, const float* y1, const float* y2, float* x1, float* x2, int64_t n,
                                const catt_throttle* k1, const catt_throttle* k2, void* stream) {
  if (check_common(n, n) != CATT_OK || (n > 0 && (!A || !y1 || !y2 || !x1 || !x2))) return CATT_EINVAL;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (fused(k1, n, n)) return launch_fused(false, A, y1, y2, x1, x2, n, n, 1, 1, k1, s);
  catt_status st = launch_row(A, nullptr, y1, x1, nullptr, n, n, 0.f, 0.f, EPI_ACCUM, k1, s);   // x1 += A y1
  if (st != CATT_OK) return st;
  return launch_col(A, y2, x2, n, n, EPI_ACCUM, k2, s);                                        // x2 += A^T y2
}

extern "C" catt_status catt_gesummv(const float* A, const float* B, const float* x, float* y, float* tmp, int64_t n,
                                    float alpha, float beta, const catt_throttle* t, void* stream) {
  if (check_common(n, n) != CATT_OK || (n > 0 && (!A || !B || !x || !y || !tmp))) return CATT_EINVAL;
  return launch_row(A, B, x, y, tmp, n, n, alpha, beta, EPI_GESUMMV, t, static_cast<cudaStream_t>(stream));
}

extern "C" catt_status catt_rows(const float* A, const float* B, const float* x, float* y, float* tmp, int64_t m,
                                 int64_t n, float alpha, float beta, int32_t mode, const catt_throttle* t,
                                 void* stream) {
  if (check_common(m, n) != CATT_OK || mode < CATT_ROWS_STORE || mode > CATT_ROWS_SUM3) return CATT_EINVAL;
  if ((m * n > 0 && !A) || (n > 0 && !x) || (m > 0 && !y)) return CATT_EINVAL;
  if (mode == CATT_ROWS_GESUMMV && ((m * n > 0 && !B) || (m > 0 && !tmp))) return CATT_EINVAL;
  if (mode == CATT_ROWS_SUM3 && m * n > 0 && !B) return CATT_EINVAL;
  return launch_row(A, B, x, y, tmp, m, n, alpha, beta, mode, t, static_cast<cudaStream_t>(stream));
}

extern "C" catt_status catt_cols(const float* A, const float* v, float* y, int64_t m, int64_t n, int32_t accumulate,
                                 const catt_throttle* t, void* stream) {
  if (check_common(m, n) != CATT_OK || (m * n > 0 && !A) || (m > 0 && !v) || (n > 0 && !y)) return CATT_EINVAL;
  return launch_col(A, v, y, m, n, accumulate ? EPI_ACCUM : EPI_STORE, t, static_cast<cudaStream_t>(stream));
}
