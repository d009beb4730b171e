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

#include "internal.h"

namespace catt {

enum { EPI_STORE = 0, EPI_ACCUM = 1, EPI_GESUMMV = 2 };

struct RowArgs {
  const float* A;
  const float* B;   // second matrix (GESUMMV) or nullptr
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
__device__ __forceinline__ void row_epilogue(const RowArgs& a, int64_t i, float acc, float acc2) {
  if (EPI == EPI_GESUMMV) {
    a.tmp[i] = acc;
    a.y[i] = __fmaf_rn(a.alpha, acc, __fmul_rn(a.beta, acc2));
  } else {
    a.y[i] = acc;
  }
}

// ---------------------------------------------------------------- row, thread per row
template <int NMAT, int EPI, bool VEC>
__global__ void __launch_bounds__(1024, (NMAT == 2 && VEC) ? 1 : 2) row_thread_kernel(RowArgs a) {
  __shared__ int slots;
  gate_init(&slots, a.t);
  __syncthreads();
  cta_enter(a.t);
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  throttled(a.t, &slots, [&]() {
    if (i >= a.M) return;
    const int64_t N = a.N;
    const float* __restrict__ ar = a.A + i * N;
    const float* __restrict__ br = (NMAT == 2) ? a.B + i * N : nullptr;
    const float* __restrict__ x = a.x;
    float acc = (EPI == EPI_ACCUM) ? a.y[i] : 0.0f;
    float acc2 = 0.0f;
    if (!VEC) {
#pragma unroll 2
      for (int64_t j = 0; j < N; ++j) {
        const float xv = x[j];
        acc = fmaf(ar[j], xv, acc);
        if (NMAT == 2) acc2 = fmaf(br[j], xv, acc2);
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
    row_epilogue<NMAT, EPI>(a, i, acc, acc2);
  });
  cta_exit(a.t);
}

// ---------------------------------------------------------------- row, warp per row (COOP)
template <int NMAT, int EPI, bool VEC>
__global__ void __launch_bounds__(1024) row_warp_kernel(RowArgs a) {
  __shared__ int slots;
  gate_init(&slots, a.t);
  __syncthreads();
  cta_enter(a.t);
  const int lane = threadIdx.x & 31;
  const int64_t i = int64_t(blockIdx.x) * (blockDim.x >> 5) + (threadIdx.x >> 5);
  throttled(a.t, &slots, [&]() {
    if (i >= a.M) return;  // warp-uniform
    const int64_t N = a.N;
    float acc = 0.0f, acc2 = 0.0f;
    if (VEC) {
      const float4* ar = reinterpret_cast<const float4*>(a.A + i * N);
      const float4* br = reinterpret_cast<const float4*>(NMAT == 2 ? a.B + i * N : a.A);
      const float4* x4 = reinterpret_cast<const float4*>(a.x);
      const int64_t n4 = N >> 2;
      int64_t j = lane;
      for (; j + 96 < n4; j += 128) {
        float4 v[4], w[4], xv[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          v[u] = ld_na4(ar + j + 32 * u);
          if (NMAT == 2) w[u] = ld_na4(br + j + 32 * u);
          xv[u] = x4[j + 32 * u];
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          acc = fmaf(v[u].x, xv[u].x, acc);
          acc = fmaf(v[u].y, xv[u].y, acc);
          acc = fmaf(v[u].z, xv[u].z, acc);
          acc = fmaf(v[u].w, xv[u].w, acc);
          if (NMAT == 2) {
            acc2 = fmaf(w[u].x, xv[u].x, acc2);
            acc2 = fmaf(w[u].y, xv[u].y, acc2);
            acc2 = fmaf(w[u].z, xv[u].z, acc2);
            acc2 = fmaf(w[u].w, xv[u].w, acc2);
          }
        }
      }
      for (; j < n4; j += 32) {
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
      for (int64_t j = lane; j < N; j += 32) {
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
    if (lane == 0) {
      if (EPI == EPI_ACCUM) acc = a.y[i] + acc;
      row_epilogue<NMAT, EPI>(a, i, acc, acc2);
    }
  });
  cta_exit(a.t);
}

// ---------------------------------------------------------------- row, staged (cp.async.bulk + mbarrier)
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "LAB_WAIT:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@P1 bra DONE;\n"
      "bra LAB_WAIT;\n"
      "DONE:\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

constexpr int kStageKT = 128;               // columns per stage (512 B per row segment)
constexpr int kStagePitch = kStageKT + 4;   // +16 B per row: conflict-free float4 column reads

// One thread per row; each thread copies its own row segment of every stage
// into shared memory (one bulk copy per stage) and consumes it in order, so
// the per-row order of operations is the literal loop's.
template <int NMAT, int EPI>
__global__ void __launch_bounds__(256) row_staged_kernel(RowArgs a, int stages) {
  extern __shared__ __align__(128) unsigned char dyn[];
  uint64_t* bar = reinterpret_cast<uint64_t*>(dyn);
  float* tiles = reinterpret_cast<float*>(dyn + 128);
  const int R = blockDim.x;
  const int t = threadIdx.x;
  const int64_t row0 = int64_t(blockIdx.x) * R;
  const int64_t i = row0 + t;
  const int64_t N = a.N;
  const int nvalid = int(imin64(R, a.M - row0));
  const int64_t ntiles = (N + kStageKT - 1) / kStageKT;
  const int64_t stage_floats = int64_t(NMAT) * R * kStagePitch;

  if (t == 0) {
    for (int s = 0; s < stages; ++s) mbar_init(&bar[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  cta_enter(a.t);
  if (i < a.M) {
    auto issue = [&](int64_t c) {
      const int s = int(c % stages);
      const int64_t j0 = c * kStageKT;
      const int len = int(imin64(kStageKT, N - j0));
      const uint32_t bytes = uint32_t(len) * 4u;
      if (t == 0) mbar_arrive_expect_tx(&bar[s], bytes * uint32_t(nvalid) * NMAT);
      float* dst = tiles + s * stage_floats + int64_t(t) * kStagePitch;
      bulk_g2s(dst, a.A + i * N + j0, bytes, &bar[s]);
      if (NMAT == 2) bulk_g2s(dst + int64_t(R) * kStagePitch, a.B + i * N + j0, bytes, &bar[s]);
    };
    const int64_t pro = imin64(stages, ntiles);
    for (int64_t c = 0; c < pro; ++c) issue(c);
    float acc = (EPI == EPI_ACCUM) ? a.y[i] : 0.0f;
    float acc2 = 0.0f;
    const float4* x4 = reinterpret_cast<const float4*>(a.x);
    for (int64_t c = 0; c < ntiles; ++c) {
      const int s = int(c % stages);
      mbar_wait(&bar[s], uint32_t((c / stages) & 1));
      const float4* ra = reinterpret_cast<const float4*>(tiles + s * stage_floats + int64_t(t) * kStagePitch);
      const float4* rb = ra + R * kStagePitch / 4;
      const int64_t j0 = c * kStageKT;
      const int len4 = int(imin64(kStageKT, N - j0)) >> 2;
#pragma unroll 8
      for (int q = 0; q < len4; ++q) {
        const float4 xv = x4[(j0 >> 2) + q];
        const float4 v = ra[q];
        acc = fmaf(v.x, xv.x, acc);
        acc = fmaf(v.y, xv.y, acc);
        acc = fmaf(v.z, xv.z, acc);
        acc = fmaf(v.w, xv.w, acc);
        if (NMAT == 2) {
          const float4 w = rb[q];
          acc2 = fmaf(w.x, xv.x, acc2);
          acc2 = fmaf(w.y, xv.y, acc2);
          acc2 = fmaf(w.z, xv.z, acc2);
          acc2 = fmaf(w.w, xv.w, acc2);
        }
      }
      if (c + stages < ntiles) {
        // this thread's generic reads of its slot are done before the async
        // proxy overwrites it
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        issue(c + stages);
      }
    }
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

// ---------------------------------------------------------------- host launchers
namespace {

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

template <int NMAT, int EPI>
catt_status launch_row_t(RowArgs a, const catt_throttle* t, cudaStream_t s) {
  const int var = variant_of(t);
  if (a.M == 0) return CATT_OK;
  const bool vec_ok = (a.N % 4 == 0) && aligned16(a.A) && aligned16(a.x) && (NMAT == 1 || aligned16(a.B));
  if (var == CATT_VAR_LITERAL || var == CATT_VAR_VEC4) {
    const int threads = cta_threads_or(t, 256);
    if (var == CATT_VAR_VEC4 && !vec_ok) return CATT_EINVAL;
    const void* f = (var == CATT_VAR_VEC4) ? (const void*)row_thread_kernel<NMAT, EPI, true>
                                           : (const void*)row_thread_kernel<NMAT, EPI, false>;
    size_t dyn = 0;
    catt_status st = prepare_launch(f, t, threads, 0, true, &a.t, &dyn);
    if (st != CATT_OK) return st;
    const int64_t grid = (a.M + threads - 1) / threads;
    if (var == CATT_VAR_VEC4)
      row_thread_kernel<NMAT, EPI, true><<<dim3(unsigned(grid)), threads, dyn, s>>>(a);
    else
      row_thread_kernel<NMAT, EPI, false><<<dim3(unsigned(grid)), threads, dyn, s>>>(a);
    return after_launch();
  }
  if (var == CATT_VAR_COOP) {
    const int threads = cta_threads_or(t, 256);
    const void* f = vec_ok ? (const void*)row_warp_kernel<NMAT, EPI, true>
                           : (const void*)row_warp_kernel<NMAT, EPI, false>;
    size_t dyn = 0;
    catt_status st = prepare_launch(f, t, threads, 0, true, &a.t, &dyn);
    if (st != CATT_OK) return st;
    const int64_t grid = (a.M + threads / 32 - 1) / (threads / 32);
    if (vec_ok)
      row_warp_kernel<NMAT, EPI, true><<<dim3(unsigned(grid)), threads, dyn, s>>>(a);
    else
      row_warp_kernel<NMAT, EPI, false><<<dim3(unsigned(grid)), threads, dyn, s>>>(a);
    return after_launch();
  }
  if (var == CATT_VAR_STAGED) {
    if (!vec_ok) return CATT_EINVAL;
    const int R = cta_threads_or(t, 32);
    if (R > 256) return CATT_EINVAL;
    const int64_t stage_bytes = int64_t(NMAT) * R * kStagePitch * 4;
    const int stages = int(std::min<int64_t>(16, (200 * 1024) / stage_bytes));
    if (stages < 2) return CATT_EINVAL;
    const size_t dyn = 128 + size_t(stages) * size_t(stage_bytes);
    const void* f = (const void*)row_staged_kernel<NMAT, EPI>;
    if (cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, int(dyn)) != cudaSuccess)
      return after_launch();
    size_t dyn_total = 0;
    catt_status st = prepare_launch(f, t, R, dyn, false, &a.t, &dyn_total);
    if (st != CATT_OK) return st;
    const int64_t grid = (a.M + R - 1) / R;
    row_staged_kernel<NMAT, EPI><<<dim3(unsigned(grid)), R, dyn_total, s>>>(a, stages);
    return after_launch();
  }
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
    const int threads = cta_threads_or(t, 1024);
    const void* f = (const void*)col_warp_kernel<EPI>;
    size_t dyn = 0;
    catt_status st = prepare_launch(f, t, threads, 0, true, &a.t, &dyn);
    if (st != CATT_OK) return st;
    const int64_t grid = (a.N + 31) / 32;
    col_warp_kernel<EPI><<<dim3(unsigned(grid)), threads, dyn, s>>>(a);
    return after_launch();
  }
  return CATT_EINVAL;
}

catt_status check_common(int64_t m, int64_t n) {
  if (m < 0 || n < 0) return CATT_EINVAL;
  if (m > (int64_t(1) << 40) || n > (int64_t(1) << 40)) return CATT_EINVAL;
  return CATT_OK;
}

}  // namespace

// Kernel instance a loop + variant launches (for attributes / descriptors).
const void* gemv_func(int loop, int variant, bool vec_ok) {
  const bool row = loop == CATT_K_ATAX_1 || loop == CATT_K_BICG_2 || loop == CATT_K_MVT_1 || loop == CATT_K_GESUMMV;
  if (row) {
    if (loop == CATT_K_GESUMMV) {
      if (variant == CATT_VAR_VEC4) return (const void*)row_thread_kernel<2, EPI_GESUMMV, true>;
      if (variant == CATT_VAR_COOP)
        return vec_ok ? (const void*)row_warp_kernel<2, EPI_GESUMMV, true> : (const void*)row_warp_kernel<2, EPI_GESUMMV, false>;
      if (variant == CATT_VAR_STAGED) return (const void*)row_staged_kernel<2, EPI_GESUMMV>;
      return (const void*)row_thread_kernel<2, EPI_GESUMMV, false>;
    }
    if (loop == CATT_K_MVT_1) {
      if (variant == CATT_VAR_VEC4) return (const void*)row_thread_kernel<1, EPI_ACCUM, true>;
      if (variant == CATT_VAR_COOP)
        return vec_ok ? (const void*)row_warp_kernel<1, EPI_ACCUM, true> : (const void*)row_warp_kernel<1, EPI_ACCUM, false>;
      if (variant == CATT_VAR_STAGED) return (const void*)row_staged_kernel<1, EPI_ACCUM>;
      return (const void*)row_thread_kernel<1, EPI_ACCUM, false>;
    }
    if (variant == CATT_VAR_VEC4) return (const void*)row_thread_kernel<1, EPI_STORE, true>;
    if (variant == CATT_VAR_COOP)
      return vec_ok ? (const void*)row_warp_kernel<1, EPI_STORE, true> : (const void*)row_warp_kernel<1, EPI_STORE, false>;
    if (variant == CATT_VAR_STAGED) return (const void*)row_staged_kernel<1, EPI_STORE>;
    return (const void*)row_thread_kernel<1, EPI_STORE, false>;
  }
  const bool acc = loop == CATT_K_MVT_2;
  if (variant == CATT_VAR_VEC4) return acc ? (const void*)col_thread_kernel<EPI_ACCUM, true> : (const void*)col_thread_kernel<EPI_STORE, true>;
  if (variant == CATT_VAR_COOP) return acc ? (const void*)col_warp_kernel<EPI_ACCUM> : (const void*)col_warp_kernel<EPI_STORE>;
  return acc ? (const void*)col_thread_kernel<EPI_ACCUM, false> : (const void*)col_thread_kernel<EPI_STORE, false>;
}

int staged_stages(int nmat, int rows) {
  const int64_t stage_bytes = int64_t(nmat) * rows * kStagePitch * 4;
  return int(std::min<int64_t>(16, (200 * 1024) / stage_bytes));
}

catt_status launch_row(const float* A, const float* B, const float* x, float* y, float* tmp, int64_t M, int64_t N,
                       float alpha, float beta, int epi, const catt_throttle* t, cudaStream_t s) {
  RowArgs a{A, B, x, y, tmp, M, N, alpha, beta, Throttle{}};
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

}  // namespace catt

using namespace catt;

extern "C" catt_status catt_atax(const float* A, const float* x, float* tmp, float* y, int64_t m, int64_t n,
                                 const catt_throttle* k1, const catt_throttle* k2, void* stream) {
  if (check_common(m, n) != CATT_OK || (m * n > 0 && !A) || (n > 0 && (!x || !y)) || (m > 0 && !tmp))
    return CATT_EINVAL;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  catt_status st = launch_row(A, nullptr, x, tmp, nullptr, m, n, 0.f, 0.f, EPI_STORE, k1, s);  // tmp = A x
  if (st != CATT_OK) return st;
  return launch_col(A, tmp, y, m, n, EPI_STORE, k2, s);                                        // y = A^T tmp
}

extern "C" catt_status catt_bicg(const float* A, const float* p, const float* r, float* q, float* s_out,
                                 int64_t nx, int64_t ny, const catt_throttle* k1, const catt_throttle* k2,
                                 void* stream) {
  if (check_common(nx, ny) != CATT_OK || (nx * ny > 0 && !A) || (ny > 0 && (!p || !s_out)) ||
      (nx > 0 && (!r || !q)))
    return CATT_EINVAL;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  catt_status st = launch_col(A, r, s_out, nx, ny, EPI_STORE, k1, s);                          // s = A^T r
  if (st != CATT_OK) return st;
  return launch_row(A, nullptr, p, q, nullptr, nx, ny, 0.f, 0.f, EPI_STORE, k2, s);          // q = A p
}

extern "C" catt_status catt_mvt(const float* A, const float* y1, const float* y2, float* x1, float* x2, int64_t n,
                                const catt_throttle* k1, const catt_throttle* k2, void* stream) {
  if (check_common(n, n) != CATT_OK || (n > 0 && (!A || !y1 || !y2 || !x1 || !x2))) return CATT_EINVAL;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
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
  if (check_common(m, n) != CATT_OK || mode < CATT_ROWS_STORE || mode > CATT_ROWS_GESUMMV) return CATT_EINVAL;
  if ((m * n > 0 && !A) || (n > 0 && !x) || (m > 0 && !y)) return CATT_EINVAL;
  if (mode == CATT_ROWS_GESUMMV && ((m * n > 0 && !B) || (m > 0 && !tmp))) return CATT_EINVAL;
  return launch_row(A, B, x, y, tmp, m, n, alpha, beta, mode, t, static_cast<cudaStream_t>(stream));
}

extern "C" catt_status catt_cols(const float* A, const float* v, float* y, int64_t m, int64_t n, int32_t accumulate,
                                 const catt_throttle* t, void* stream) {
  if (check_common(m, n) != CATT_OK || (m * n > 0 && !A) || (m > 0 && !v) || (n > 0 && !y)) return CATT_EINVAL;
  return launch_col(A, v, y, m, n, accumulate ? EPI_ACCUM : EPI_STORE, t, static_cast<cudaStream_t>(stream));
}
