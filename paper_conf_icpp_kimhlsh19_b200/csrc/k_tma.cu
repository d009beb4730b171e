// k_tma.cu — STAGED variants: the literal per-output sequential loops fed by
// 2-D TMA tensor copies (cp.async.bulk.tensor) into a shared-memory ring.
//
// The paper keeps the row-per-thread loop and protects its L1 reuse by
// throttling. On B200 the same loop can instead take its operands
// from shared memory: one elected thread issues TMA box copies (a box is up to
// 256 rows x 128 B, one request) into an S-stage ring guarded by full/empty
// mbarriers, and every thread still accumulates its own output in the literal
// order (bit-exact to the sequential oracle). No L1 reuse is needed, so there
// is nothing to throttle (descriptor refs are CATT_REF_NOT_L1).
//
// Row loop: CTA = R threads = R rows; a stage is B boxes of {32 columns x R
// rows} with the 128-byte swizzle (16-byte chunk k of row r lands at chunk
// k ^ (r & 7)), so thread t reading float4 chunks of its own row is
// bank-conflict free.
// Column loop: CTA = CB threads = CB columns; a stage is one box of {CB
// columns x RB rows}, unswizzled: thread t reads column t of each row, a
// contiguous 4-byte access across the warp.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdint>
#include <mutex>

#include "internal.h"
#include "tma.cuh"

namespace catt {


struct TmaRowArgs {
  const float* x;
  float* y;
  float* tmp;
  int64_t M, N;
  float alpha, beta;
  int stages, boxes, epi;
  Throttle t;
};

// NMAT = 1: y[i] (=|+=) sum_j A[i][j] x[j];  NMAT = 2: GESUMMV.
template <int NMAT>
__global__ void __launch_bounds__(256) row_tma_kernel(const __grid_constant__ CUtensorMap mapA,
                                                      const __grid_constant__ CUtensorMap mapB, TmaRowArgs a) {
  extern __shared__ __align__(1024) unsigned char dyn[];
  const int R = blockDim.x, t = threadIdx.x, lane = t & 31, nw = R >> 5;
  const int S = a.stages, B = a.boxes;
  uint64_t* full = reinterpret_cast<uint64_t*>(dyn);
  uint64_t* empty = full + S;
  unsigned char* tiles = dyn + 1024;
  const int box_bytes = R * 128;
  const int KT = 32 * B;
  const int x_off = NMAT * B * box_bytes;                    // x segment follows the boxes
  const int stage_bytes = (x_off + KT * 4 + 1023) / 1024 * 1024;
  const int64_t row0 = int64_t(blockIdx.x) * R;
  const int64_t i = row0 + t;
  const int64_t N = a.N;
  const int64_t ntiles = (N + KT - 1) / KT;
  if (t == 0) {
    for (int s = 0; s < S; ++s) {
      bar_init(&full[s], 1);
      bar_init(&empty[s], nw);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  cta_enter(a.t);
  auto issue = [&](int64_t c) {  // thread 0 only
    const int s = int(c % S);
    if (c >= S) bar_wait(&empty[s], uint32_t(((c / S) - 1) & 1));
    const int64_t j0 = c * KT;
    const uint32_t xbytes = uint32_t(imin64(KT, N - j0)) * 4u;
    bar_expect_tx(&full[s], uint32_t(NMAT * B * box_bytes) + xbytes);
    unsigned char* st = tiles + int64_t(s) * stage_bytes;
    for (int b = 0; b < B; ++b) {
      const int32_t col = int32_t(j0 + 32 * b), row = int32_t(row0);
      tma_2d(st + b * box_bytes, &mapA, col, row, &full[s]);
      if (NMAT == 2) tma_2d(st + (B + b) * box_bytes, &mapB, col, row, &full[s]);
    }
    bulk_1d(st + x_off, a.x + j0, xbytes, &full[s]);
  };
  if (t == 0)
    for (int64_t c = 0; c < imin64(S, ntiles); ++c) issue(c);
  const bool valid = i < a.M;
  float acc = (valid && a.epi == 1) ? a.y[i] : 0.0f;
  float acc2 = 0.0f;
  const int sw = t & 7;
  for (int64_t c = 0; c < ntiles; ++c) {
    const int s = int(c % S);
    bar_wait(&full[s], uint32_t((c / S) & 1));
    if (valid) {
      const int64_t j0 = c * KT;
      const int len = int(imin64(KT, N - j0));  // multiple of 4 (N % 4 == 0)
      const unsigned char* st = tiles + int64_t(s) * stage_bytes;
      const unsigned char* rowp = st + t * 128;
      const float4* xs = reinterpret_cast<const float4*>(st + x_off);
      if (len == KT) {
        // full tile: software-pipelined one box (8 chunks) ahead, so the
        // shared-memory latency overlaps the previous box's FMA chain
        float4 v[8], w[NMAT == 2 ? 8 : 1], xv[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          v[k] = *reinterpret_cast<const float4*>(rowp + ((k ^ sw) << 4));
          if (NMAT == 2) w[k] = *reinterpret_cast<const float4*>(rowp + B * box_bytes + ((k ^ sw) << 4));
          xv[k] = xs[k];
        }
        for (int b = 0; b < B; ++b) {
          float4 vn[8], wn[NMAT == 2 ? 8 : 1], xn[8];
          if (b + 1 < B) {
            const unsigned char* bp = rowp + (b + 1) * box_bytes;
#pragma unroll
            for (int k = 0; k < 8; ++k) {
              vn[k] = *reinterpret_cast<const float4*>(bp + ((k ^ sw) << 4));
              if (NMAT == 2) wn[k] = *reinterpret_cast<const float4*>(bp + B * box_bytes + ((k ^ sw) << 4));
              xn[k] = xs[(b + 1) * 8 + k];
            }
          }
#pragma unroll
          for (int k = 0; k < 8; ++k) {
            acc = fmaf(v[k].x, xv[k].x, acc);
            acc = fmaf(v[k].y, xv[k].y, acc);
            acc = fmaf(v[k].z, xv[k].z, acc);
            acc = fmaf(v[k].w, xv[k].w, acc);
            if (NMAT == 2) {
              acc2 = fmaf(w[k].x, xv[k].x, acc2);
              acc2 = fmaf(w[k].y, xv[k].y, acc2);
              acc2 = fmaf(w[k].z, xv[k].z, acc2);
              acc2 = fmaf(w[k].w, xv[k].w, acc2);
            }
          }
          if (b + 1 < B) {
#pragma unroll
            for (int k = 0; k < 8; ++k) {
              v[k] = vn[k];
              if (NMAT == 2) w[k] = wn[k];
              xv[k] = xn[k];
            }
          }
        }
      } else {
        for (int q = 0; q < (len >> 2); ++q) {
          const int b = q >> 3, k = q & 7;
          const unsigned char* bp = rowp + b * box_bytes;
          const float4 v = *reinterpret_cast<const float4*>(bp + ((k ^ sw) << 4));
          const float4 xv = xs[q];
          acc = fmaf(v.x, xv.x, acc);
          acc = fmaf(v.y, xv.y, acc);
          acc = fmaf(v.z, xv.z, acc);
          acc = fmaf(v.w, xv.w, acc);
          if (NMAT == 2) {
            const float4 w = *reinterpret_cast<const float4*>(bp + B * box_bytes + ((k ^ sw) << 4));
            acc2 = fmaf(w.x, xv.x, acc2);
            acc2 = fmaf(w.y, xv.y, acc2);
            acc2 = fmaf(w.z, xv.z, acc2);
            acc2 = fmaf(w.w, xv.w, acc2);
          }
        }
      }
    }
    __syncwarp();
    if (lane == 0) bar_arrive(&empty[s]);
    if (t == 0 && c + S < ntiles) issue(c + S);
  }
  if (valid) {
    if (NMAT == 2) {
      a.tmp[i] = acc;
      a.y[i] = __fmaf_rn(a.alpha, acc, __fmul_rn(a.beta, acc2));
    } else {
      a.y[i] = acc;
    }
  }
  cta_exit(a.t);
}

struct TmaColArgs {
  const float* v;
  float* y;
  int64_t M, N;
  int stages, rows_per_stage, accumulate;
  Throttle t;
};

__global__ void __launch_bounds__(256) col_tma_kernel(const __grid_constant__ CUtensorMap mapA, TmaColArgs a) {
  extern __shared__ __align__(1024) unsigned char dyn[];
  const int CB = blockDim.x, t = threadIdx.x, lane = t & 31, nw = CB >> 5;
  const int S = a.stages, RB = a.rows_per_stage;
  uint64_t* full = reinterpret_cast<uint64_t*>(dyn);
  uint64_t* empty = full + S;
  unsigned char* tiles = dyn + 1024;
  const int tile_bytes = CB * RB * 4;
  const int stage_bytes = (tile_bytes + RB * 4 + 1023) / 1024 * 1024;   // tile + v segment
  const int64_t col0 = int64_t(blockIdx.x) * CB, j = col0 + t;
  const int64_t M = a.M;
  const int64_t ntiles = (M + RB - 1) / RB;
  if (t == 0) {
    for (int s = 0; s < S; ++s) {
      bar_init(&full[s], 1);
      bar_init(&empty[s], nw);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  cta_enter(a.t);
  auto issue = [&](int64_t c) {
    const int s = int(c % S);
    if (c >= S) bar_wait(&empty[s], uint32_t(((c / S) - 1) & 1));
    const uint32_t vbytes = uint32_t(imin64(RB, M - c * RB)) * 4u;
    const uint32_t vcopy = (vbytes + 15u) & ~15u;         // bulk copies move multiples of 16 B
    bar_expect_tx(&full[s], uint32_t(tile_bytes) + vcopy);
    unsigned char* st = tiles + int64_t(s) * stage_bytes;
    tma_2d(st, &mapA, int32_t(col0), int32_t(c * RB), &full[s]);
    bulk_1d(st + tile_bytes, a.v + c * RB, vcopy, &full[s]);
  };
  if (t == 0)
    for (int64_t c = 0; c < imin64(S, ntiles); ++c) issue(c);
  const bool valid = j < a.N;
  float acc = (valid && a.accumulate) ? a.y[j] : 0.0f;
  for (int64_t c = 0; c < ntiles; ++c) {
    const int s = int(c % S);
    bar_wait(&full[s], uint32_t((c / S) & 1));
    if (valid) {
      const int rows = int(imin64(RB, M - c * RB));
      const unsigned char* st = tiles + int64_t(s) * stage_bytes;
      const float* tp = reinterpret_cast<const float*>(st) + t;
      const float* vs = reinterpret_cast<const float*>(st + tile_bytes);
      if (rows == RB) {
        // pipelined 16 rows ahead of the FMA chain
        float w[16], vv[16];
#pragma unroll
        for (int u = 0; u < 16; ++u) {
          w[u] = tp[u * CB];
          vv[u] = vs[u];
        }
        for (int r0 = 0; r0 < RB; r0 += 16) {
          float wn[16], vn[16];
          if (r0 + 16 < RB) {
#pragma unroll
            for (int u = 0; u < 16; ++u) {
              wn[u] = tp[(r0 + 16 + u) * CB];
              vn[u] = vs[r0 + 16 + u];
            }
          }
#pragma unroll
          for (int u = 0; u < 16; ++u) acc = fmaf(w[u], vv[u], acc);
          if (r0 + 16 < RB) {
#pragma unroll
            for (int u = 0; u < 16; ++u) {
              w[u] = wn[u];
              vv[u] = vn[u];
            }
          }
        }
      } else {
        for (int r = 0; r < rows; ++r) acc = fmaf(tp[r * CB], vs[r], acc);
      }
    }
    __syncwarp();
    if (lane == 0) bar_arrive(&empty[s]);
    if (t == 0 && c + S < ntiles) issue(c + S);
  }
  if (valid) a.y[j] = acc;
  cta_exit(a.t);
}

// ---------------------------------------------------------------- host side
namespace {

// Row-major rows x cols fp32 matrix, box {box_cols, box_rows}.
catt_status make_map(CUtensorMap* m, const float* base, int64_t rows, int64_t cols, int box_cols, int box_rows,
                     bool swizzle128) {
  auto fn = encode_fn();
  if (!fn) return CATT_ECUDA;
  const cuuint64_t dims[2] = {cuuint64_t(cols), cuuint64_t(rows)};
  const cuuint64_t strides[1] = {cuuint64_t(cols) * 4};
  const cuuint32_t box[2] = {cuuint32_t(box_cols), cuuint32_t(box_rows)};
  const cuuint32_t estr[2] = {1, 1};
  CUresult r = fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, swizzle128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? CATT_OK : CATT_EINVAL;
}

bool tma_ok(const void* p, int64_t cols) {
  return (reinterpret_cast<uintptr_t>(p) & 15u) == 0 && cols % 4 == 0 && cols < (int64_t(1) << 31);
}

constexpr int kSmemBudget = 200 * 1024;

}  // namespace

int row_tma_stage_bytes(int nmat, int rows, int boxes) {
  return (nmat * boxes * rows * 128 + 32 * boxes * 4 + 1023) / 1024 * 1024;
}
int col_tma_stage_bytes(int cols, int rows_per_stage) {
  return (cols * rows_per_stage * 4 + rows_per_stage * 4 + 1023) / 1024 * 1024;
}
int row_tma_stages(int nmat, int rows, int boxes) {
  return std::max(2, std::min(16, (kSmemBudget - 1024) / row_tma_stage_bytes(nmat, rows, boxes)));
}
int col_tma_stages(int cols, int rows_per_stage) {
  return std::max(2, std::min(16, (kSmemBudget - 1024) / col_tma_stage_bytes(cols, rows_per_stage)));
}

const void* row_tma_func(int nmat) {
  return nmat == 2 ? (const void*)row_tma_kernel<2> : (const void*)row_tma_kernel<1>;
}
const void* col_tma_func() { return (const void*)col_tma_kernel; }

// epi: 0 store, 1 accumulate, 2 GESUMMV
catt_status launch_row_tma(const float* A, const float* Bm, const float* x, float* y, float* tmp, int64_t M,
                           int64_t N, float alpha, float beta, int epi, const catt_throttle* t, cudaStream_t s) {
  if (M == 0) return CATT_OK;
  const int nmat = epi == 2 ? 2 : 1;
  if (!tma_ok(A, N) || (nmat == 2 && !tma_ok(Bm, N)) || (reinterpret_cast<uintptr_t>(x) & 15u)) return CATT_EINVAL;
  const int R = cta_threads_or(t, 32);
  if (R > 256 || R % 32) return CATT_EINVAL;
  const int boxes = std::max(1, std::min(8, 16384 / (nmat * R * 128)));   // ~16 KB per stage
  const int stages = row_tma_stages(nmat, R, boxes);
  const size_t dyn = 1024 + size_t(stages) * row_tma_stage_bytes(nmat, R, boxes);
  CUtensorMap ma, mb;
  catt_status st = make_map(&ma, A, M, N, 32, R, true);
  if (st == CATT_OK) st = make_map(&mb, nmat == 2 ? Bm : A, M, N, 32, R, true);
  if (st != CATT_OK) return st;
  const void* f = row_tma_func(nmat);
  if (cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, int(dyn)) != cudaSuccess)
    return after_launch();
  TmaRowArgs a{x, y, tmp, M, N, alpha, beta, stages, boxes, epi, Throttle{}};
  size_t dyn_total = 0;
  st = prepare_launch(f, t, R, dyn, false, &a.t, &dyn_total);
  if (st != CATT_OK) return st;
  const unsigned grid = unsigned((M + R - 1) / R);
  if (nmat == 2)
    row_tma_kernel<2><<<grid, R, dyn_total, s>>>(ma, mb, a);
  else
    row_tma_kernel<1><<<grid, R, dyn_total, s>>>(ma, mb, a);
  return after_launch();
}

catt_status launch_col_tma(const float* A, const float* v, float* y, int64_t M, int64_t N, int accumulate,
                           const catt_throttle* t, cudaStream_t s) {
  if (N == 0) return CATT_OK;
  if (!tma_ok(A, N) || (reinterpret_cast<uintptr_t>(v) & 15u)) return CATT_EINVAL;
  const int CB = cta_threads_or(t, 32);
  if (CB > 256 || CB % 32) return CATT_EINVAL;
  const int RB = std::max(16, std::min(256, 16384 / (CB * 4))) / 16 * 16;  // ~16 KB per stage, multiple of 16
  const int stages = col_tma_stages(CB, RB);
  const size_t dyn = 1024 + size_t(stages) * col_tma_stage_bytes(CB, RB);
  CUtensorMap ma;
  catt_status st = make_map(&ma, A, M > 0 ? M : 1, N, CB, RB, false);
  if (st != CATT_OK) return st;
  const void* f = col_tma_func();
  if (cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, int(dyn)) != cudaSuccess)
    return after_launch();
  TmaColArgs a{v, y, M, N, stages, RB, accumulate, Throttle{}};
  size_t dyn_total = 0;
  st = prepare_launch(f, t, CB, dyn, false, &a.t, &dyn_total);
  if (st != CATT_OK) return st;
  col_tma_kernel<<<unsigned((N + CB - 1) / CB), CB, dyn_total, s>>>(ma, a);
  return after_launch();
}

}  // namespace catt
