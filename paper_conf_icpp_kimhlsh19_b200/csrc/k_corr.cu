// k_corr.cu — CORR, PolyBench/GPU correlation (Table 2; the CORR row of
// Table 3; the case where thread throttling gives up).
//
// data (n rows = observations x m columns = variables) is centred and scaled
// in place; per column j, i ascending (R22):
//   mean[j] = (sum data[i][j]) / fn;  std[j] = sqrtf(sum fmaf(d, d, .) / fn),
//   std = 1 if <= eps;  data[i][j] = (data[i][j] - mean[j]) / (sqrtf(fn) * std[j])
//   symmat[j1][j1] = 1;  j2 > j1: s = sum_i fmaf(data[i][j1], data[i][j2], s)
// fn = (float)n, eps = 0.005f.
// LITERAL: the paper's loops. The column statistics run thread per column
// (coalesced). The correlation loop is thread per j1 (CATT_K_CORR): for each
// j2 the thread re-reads its whole column j1 (n rows apart), so the line it
// reuses comes back only after n lines of its own: no throttle makes that fit
// (the paper's "give up"), and the analyser reports CATT_FIT_UNRESOLVABLE.
// STAGED: the columns transposed (32 x 32 tiles), the statistics a warp per
// column (the same sequential order, lane 0), the centred data transposed
// back, and symmat = D^T D by the tiled SYRK kernel with alpha = 1, beta = 0
// over the upper tiles, mirrored into the lower triangle: each element is the
// same fmaf chain over i (fmaf is commutative),
// so the result is bit-identical to LITERAL; the diagonal is then set to 1.
#include <cmath>
#include <cstdint>

#include "internal.h"
#include "tma.cuh"

namespace catt {

struct CorrStatsArgs {
  float* data;
  float* mean;
  float* stdv;
  int64_t n, m;
};

__global__ void __launch_bounds__(256) corr_stats_kernel(CorrStatsArgs a) {
  const int64_t j = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (j >= a.m) return;
  const float fn = float(a.n), eps = 0.005f;
  float* col = a.data + j;
  const int64_t m = a.m;
  float mu = 0.0f;
  for (int64_t i = 0; i < a.n; ++i) mu = __fadd_rn(mu, col[i * m]);
  mu = __fdiv_rn(mu, fn);
  float sd = 0.0f;
  for (int64_t i = 0; i < a.n; ++i) {
    const float d = __fsub_rn(col[i * m], mu);
    sd = fmaf(d, d, sd);
  }
  sd = __fsqrt_rn(__fdiv_rn(sd, fn));
  if (sd <= eps) sd = 1.0f;
  const float scale = __fmul_rn(__fsqrt_rn(fn), sd);
  for (int64_t i = 0; i < a.n; ++i) col[i * m] = __fdiv_rn(__fsub_rn(col[i * m], mu), scale);
  a.mean[j] = mu;
  a.stdv[j] = sd;
}

struct CorrArgs {
  const float* data;
  float* symmat;
  int64_t n, m;
  Throttle t;
};

__global__ void __launch_bounds__(1024, 2) corr_thread_kernel(CorrArgs a) {
  __shared__ int slots;
  gate_init(&slots, a.t);
  __syncthreads();
  cta_enter(a.t);
  const int64_t j1 = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  throttled(a.t, &slots, [&]() {
    if (j1 >= a.m) return;
    const int64_t m = a.m;
    a.symmat[j1 * m + j1] = 1.0f;
    for (int64_t j2 = j1 + 1; j2 < m; ++j2) {
      float s = 0.0f;
#pragma unroll 2
      for (int64_t i = 0; i < a.n; ++i) s = fmaf(a.data[i * m + j1], a.data[i * m + j2], s);
      a.symmat[j1 * m + j2] = s;
      a.symmat[j2 * m + j1] = s;
    }
  });
  cta_exit(a.t);
}

// out (m x n) = in (n x m)^T through 32 x 32 shared-memory tiles (pitch 33)
__global__ void __launch_bounds__(256) transpose32_kernel(const float* __restrict__ in, float* __restrict__ out,
                                                          int64_t n, int64_t m) {
  __shared__ float tile[32][33];
  const int64_t i0 = int64_t(blockIdx.y) * 32, j0 = int64_t(blockIdx.x) * 32;
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;  // 8 rows of 32
  for (int r = ty; r < 32; r += 8) {
    const int64_t i = i0 + r, j = j0 + tx;
    if (i < n && j < m) tile[r][tx] = in[i * m + j];
  }
  __syncthreads();
  for (int r = ty; r < 32; r += 8) {
    const int64_t j = j0 + r, i = i0 + tx;
    if (j < m && i < n) out[j * n + i] = tile[tx][r];
  }
}

// STAGED statistics on the transposed data (row j = column j, contiguous):
// a warp per column stages the row in shared memory (coalesced), lane 0 runs
// the two sequential sums in the same order and rounding as corr_stats_kernel,
// then the whole warp writes the centred and scaled row back.
constexpr int kStatWarps = 8;
__global__ void __launch_bounds__(kStatWarps * 32) corr_stats_rows_kernel(float* rowsT, float* mean, float* stdv,
                                                                         int64_t n, int64_t m) {
  extern __shared__ float s_row[];  // [kStatWarps][n]
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int64_t j = int64_t(blockIdx.x) * kStatWarps + w;
  if (j >= m) return;
  float* buf = s_row + int64_t(w) * n;
  float* row = rowsT + j * n;
  {
    // the row into shared memory with 16 loads in flight per lane
    int64_t i = lane;
    for (; i + 32 * 15 < n; i += 32 * 16) {
      float v[16];
#pragma unroll
      for (int u = 0; u < 16; ++u) v[u] = row[i + 32 * u];
#pragma unroll
      for (int u = 0; u < 16; ++u) buf[i + 32 * u] = v[u];
    }
    for (; i < n; i += 32) buf[i] = row[i];
  }
  __syncwarp();
  const float fn = float(n), eps = 0.005f;
  float mu = 0.0f, sd = 0.0f;
  if (lane == 0) {
    // the same two sequential chains; the loads go 32 values ahead of the
    // adds (8 x LDS.128 per batch when the rows are 16-byte aligned), so each
    // chain runs at the add latency rather than the load latency
    int64_t i = 0;
    if ((n & 3) == 0) {
      const float4* b4 = reinterpret_cast<const float4*>(buf);
      for (; i + 32 <= n; i += 32) {
        float4 v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) v[u] = b4[i / 4 + u];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          mu = __fadd_rn(mu, v[u].x);
          mu = __fadd_rn(mu, v[u].y);
          mu = __fadd_rn(mu, v[u].z);
          mu = __fadd_rn(mu, v[u].w);
        }
      }
    }
    for (; i < n; ++i) mu = __fadd_rn(mu, buf[i]);
    mu = __fdiv_rn(mu, fn);
    i = 0;
    if ((n & 3) == 0) {
      const float4* b4 = reinterpret_cast<const float4*>(buf);
      for (; i + 32 <= n; i += 32) {
        float4 v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) v[u] = b4[i / 4 + u];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          float d = __fsub_rn(v[u].x, mu);
          sd = fmaf(d, d, sd);
          d = __fsub_rn(v[u].y, mu);
          sd = fmaf(d, d, sd);
          d = __fsub_rn(v[u].z, mu);
          sd = fmaf(d, d, sd);
          d = __fsub_rn(v[u].w, mu);
          sd = fmaf(d, d, sd);
        }
      }
    }
    for (; i < n; ++i) {
      const float d = __fsub_rn(buf[i], mu);
      sd = fmaf(d, d, sd);
    }
    sd = __fsqrt_rn(__fdiv_rn(sd, fn));
    if (sd <= eps) sd = 1.0f;
    mean[j] = mu;
    stdv[j] = sd;
  }
  mu = __shfl_sync(0xffffffffu, mu, 0);
  sd = __shfl_sync(0xffffffffu, sd, 0);
  const float scale = __fmul_rn(__fsqrt_rn(fn), sd);
  for (int64_t i = lane; i < n; i += 32) row[i] = __fdiv_rn(__fsub_rn(buf[i], mu), scale);
}

// STAGED statistics straight on the row-major data (round 2): a CTA owns a
// strip of kStripCols columns and stages all n rows of it in shared memory by
// TMA boxes of 256 rows (one mbarrier per box); lane c of warp 0 runs
// column c's two
// sequential chains (the order and rounding of corr_stats_kernel, loads a
// batch ahead of the adds), and the whole CTA writes the centred and scaled
// strip back in place. No transposes: the centred data is then the k-major
// operand of the SYRK (syrk_upper_kmajor).
constexpr int kStripCols = 8, kStripBox = 256, kStripMaxBoxes = 16;  // 8 columns: 25 us at 2048 (16: 28, 4: 31)
__global__ void __launch_bounds__(256) corr_stats_strip_kernel(const __grid_constant__ CUtensorMap map, float* data,
                                                               float* mean, float* stdv, int64_t n, int64_t m) {
  asm volatile("griddepcontrol.launch_dependents;");  // the symmat tile kernel may become resident early
  extern __shared__ __align__(128) float s_strip[];  // [n rounded to boxes][kStripCols]
  __shared__ float s_mu[kStripCols], s_scale[kStripCols];
  __shared__ __align__(8) uint64_t s_bar[kStripMaxBoxes];
  const int t = threadIdx.x;
  const int64_t j0 = int64_t(blockIdx.x) * kStripCols;
  const int nc = int(imin64(kStripCols, m - j0));
  const int nbox = int((n + kStripBox - 1) / kStripBox);
  if (t == 0) {
    for (int b = 0; b < nbox; ++b) bar_init(&s_bar[b], 1);
    fence_barrier_init();
    for (int b = 0; b < nbox; ++b) {
      bar_expect_tx(&s_bar[b], uint32_t(kStripBox * kStripCols * 4));
      tma_2d(s_strip + int64_t(b) * kStripBox * kStripCols, &map, int32_t(j0), int32_t(b * kStripBox), &s_bar[b]);
    }
  }
  __syncthreads();
  const float fn = float(n), eps = 0.005f;
  if (t < nc) {
    // the mean chain starts on the first box while the others land (a
    // register double buffer of the next batch measured slower: 33 vs 28 us)
    const float* col = s_strip + t;
    constexpr int B = 16;
    float mu = 0.0f;
    int64_t i = 0;
    for (int b = 0; b < nbox; ++b) {
      bar_wait(&s_bar[b], 0u);
      const int64_t hi = imin64(n, int64_t(b + 1) * kStripBox);
      for (; i + B <= hi; i += B) {
        float v[B];
#pragma unroll
        for (int u = 0; u < B; ++u) v[u] = col[(i + u) * kStripCols];
#pragma unroll
        for (int u = 0; u < B; ++u) mu = __fadd_rn(mu, v[u]);
      }
      for (; i < hi; ++i) mu = __fadd_rn(mu, col[i * kStripCols]);
    }
    mu = __fdiv_rn(mu, fn);
    float sd = 0.0f;
    i = 0;
    for (; i + B <= n; i += B) {
      float v[B];
#pragma unroll
      for (int u = 0; u < B; ++u) v[u] = col[(i + u) * kStripCols];
#pragma unroll
      for (int u = 0; u < B; ++u) {
        const float d = __fsub_rn(v[u], mu);
        sd = fmaf(d, d, sd);
      }
    }
    for (; i < n; ++i) {
      const float d = __fsub_rn(col[i * kStripCols], mu);
      sd = fmaf(d, d, sd);
    }
    sd = __fsqrt_rn(__fdiv_rn(sd, fn));
    if (sd <= eps) sd = 1.0f;
    mean[j0 + t] = mu;
    stdv[j0 + t] = sd;
    s_mu[t] = mu;
    s_scale[t] = __fmul_rn(__fsqrt_rn(fn), sd);
  } else if (t < kStripCols) {
    for (int b = 0; b < nbox; ++b) bar_wait(&s_bar[b], 0u);  // every box landed before the write-back reads it
  }
  __syncthreads();
  // write-back: float4 of 4 columns per thread (m % 4 == 0 on this path)
  const int q4 = (nc + 3) / 4;
  constexpr int R4 = kStripCols / 4;  // float4 per strip row
  for (int64_t e = t; e < n * R4; e += 256) {
    const int64_t i = e / R4;
    const int c4 = int(e % R4);
    if (c4 < q4) {
      const float4 v = *reinterpret_cast<const float4*>(s_strip + i * kStripCols + 4 * c4);
      float4 o;
      o.x = __fdiv_rn(__fsub_rn(v.x, s_mu[4 * c4]), s_scale[4 * c4]);
      o.y = __fdiv_rn(__fsub_rn(v.y, s_mu[4 * c4 + 1]), s_scale[4 * c4 + 1]);
      o.z = __fdiv_rn(__fsub_rn(v.z, s_mu[4 * c4 + 2]), s_scale[4 * c4 + 2]);
      o.w = __fdiv_rn(__fsub_rn(v.w, s_mu[4 * c4 + 3]), s_scale[4 * c4 + 3]);
      *reinterpret_cast<float4*>(data + i * m + j0 + 4 * c4) = o;
    }
  }
}

// symmat[i][j] = symmat[j][i] for i > j, through 32 x 32 tiles (the lower
// triangle from the computed upper one)
__global__ void __launch_bounds__(256) mirror_lower_kernel(float* symmat, int64_t m) {
  if (blockIdx.x > blockIdx.y) return;  // destination tile (by, bx) must be on or below the diagonal
  __shared__ float tile[32][33];
  const int64_t di = int64_t(blockIdx.y) * 32, dj = int64_t(blockIdx.x) * 32;  // destination rows, columns
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
  for (int r = ty; r < 32; r += 8) {  // source tile (dj, di): rows dj.., columns di..
    const int64_t i = dj + r, j = di + tx;
    if (i < m && j < m) tile[r][tx] = symmat[i * m + j];
  }
  __syncthreads();
  for (int r = ty; r < 32; r += 8) {
    const int64_t i = di + r, j = dj + tx;
    if (i < m && j < m && i > j) symmat[i * m + j] = tile[tx][r];
  }
}

__global__ void corr_diag_kernel(float* symmat, int64_t m) {
  const int64_t j = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (j < m) symmat[j * m + j] = 1.0f;
}

const void* syrk_func(int variant, int64_t n, bool tri);

const void* corr_func(int variant, int64_t m) {
  return variant == CATT_VAR_STAGED ? syrk_func(CATT_VAR_STAGED, m, true) : (const void*)corr_thread_kernel;
}

// data (n x m, row-major) as a TMA map with boxes {kStripCols columns, kStripBox rows}
static bool strip_map(CUtensorMap* mp, const float* data, int64_t n, int64_t m) {
  auto fn = encode_fn();
  if (!fn) return false;
  const cuuint64_t dims[2] = {cuuint64_t(m), cuuint64_t(n)};
  const cuuint64_t strides[1] = {cuuint64_t(m) * 4};
  const cuuint32_t box[2] = {cuuint32_t(kStripCols), cuuint32_t(kStripBox)};
  const cuuint32_t estr[2] = {1, 1};
  return fn(mp, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(data), dims, strides, box, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

}  // namespace catt

using namespace catt;

extern "C" catt_status catt_corr(float* data, int64_t n, int64_t m, float* mean, float* stdv, float* symmat,
                                 float* work, const catt_throttle* t, void* stream) {
  if (n < 1 || m < 1 || n > (int64_t(1) << 31) || m > (int64_t(1) << 31)) return CATT_EINVAL;
  if (!data || !mean || !stdv || !symmat) return CATT_EINVAL;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  const int var = variant_of(t);
  if (var != CATT_VAR_LITERAL && var != CATT_VAR_STAGED) return CATT_EINVAL;
  if (var == CATT_VAR_STAGED && !work) return CATT_EINVAL;
  catt_status st = CATT_OK;
  if (var == CATT_VAR_LITERAL) {
    corr_stats_kernel<<<dim3(unsigned((m + 255) / 256)), 256, 0, s>>>(CorrStatsArgs{data, mean, stdv, n, m});
    if ((st = after_launch()) != CATT_OK) return st;
    CorrArgs a{data, symmat, n, m, Throttle{}};
    const int threads = cta_threads_or(t, 256);
    size_t dyn = 0;
    st = prepare_launch((const void*)corr_thread_kernel, t, threads, 0, true, &a.t, &dyn);
    if (st != CATT_OK) return st;
    corr_thread_kernel<<<dim3(unsigned((m + threads - 1) / threads)), threads, dyn, s>>>(a);
    return after_launch();
  }
  const int64_t gy = (n + 31) / 32, gx = (m + 31) / 32;
  if (gy > 65535 || gx > 65535) return CATT_EINVAL;
  // STAGED, direct form (round 2): statistics on column strips of the data in
  // place, then symmat = D^T D by T2 straight from the centred data (its
  // k-major operand) over the upper tiles; mirrored; diagonal 1. Used when
  // the strip fits shared memory and T2 can read D (16-byte rows).
  const int64_t nbox = (n + kStripBox - 1) / kStripBox;
  const size_t sstrip = size_t(nbox) * kStripBox * kStripCols * 4;
  CUtensorMap smap;
  if (nbox <= kStripMaxBoxes && sstrip <= 200 * 1024 && syrk_kmajor_ok(data, m) && strip_map(&smap, data, n, m)) {
    if (cudaFuncSetAttribute((const void*)corr_stats_strip_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             int(sstrip)) != cudaSuccess)
      return after_launch();
    corr_stats_strip_kernel<<<dim3(unsigned((m + kStripCols - 1) / kStripCols)), 256, sstrip, s>>>(smap, data, mean, stdv,
                                                                                                  n, m);
    if ((st = after_launch()) != CATT_OK) return st;
    // the whole symmat in one launch: upper tiles, their mirror, diagonal 1
    return syrk_upper_kmajor(data, nullptr, symmat, m, n, s, true);
  }
  // STAGED, transposed form: work = data^T (m x n); statistics and scaling on
  // its rows; data = work^T (the centred data, as LITERAL leaves it); symmat
  // = work work^T by the tiled SYRK (alpha 1, beta 0); diagonal 1
  const size_t srow = size_t(kStatWarps) * size_t(n) * 4;
  if (srow > 200 * 1024) return CATT_EUNSUPPORTED;  // n > 6400 rows: use LITERAL
  transpose32_kernel<<<dim3(unsigned(gx), unsigned(gy)), 256, 0, s>>>(data, work, n, m);
  if ((st = after_launch()) != CATT_OK) return st;
  if (srow > 48 * 1024 && cudaFuncSetAttribute((const void*)corr_stats_rows_kernel,
                                               cudaFuncAttributeMaxDynamicSharedMemorySize, int(srow)) != cudaSuccess)
    return after_launch();
  corr_stats_rows_kernel<<<dim3(unsigned((m + kStatWarps - 1) / kStatWarps)), kStatWarps * 32, srow, s>>>(
      work, mean, stdv, n, m);
  if ((st = after_launch()) != CATT_OK) return st;
  transpose32_kernel<<<dim3(unsigned(gy), unsigned(gx)), 256, 0, s>>>(work, data, m, n);
  if ((st = after_launch()) != CATT_OK) return st;
  st = syrk_upper_kmajor(data, work, symmat, m, n, s);  // upper tiles only: symmat is symmetric
  if (st != CATT_OK) return st;
  mirror_lower_kernel<<<dim3(unsigned(gx), unsigned(gx)), 256, 0, s>>>(symmat, m);
  if ((st = after_launch()) != CATT_OK) return st;
  corr_diag_kernel<<<dim3(unsigned((m + 255) / 256)), 256, 0, s>>>(symmat, m);
  return after_launch();
}
