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
// STAGED: the same statistics kernel, then the columns transposed (32 x 32
// tiles) and symmat = D^T D by the tiled SYRK kernel with alpha = 1, beta = 0:
// each element is the same fmaf chain over i (fmaf is commutative),
// so the result is bit-identical to LITERAL; the diagonal is then set to 1.
#include <cmath>
#include <cstdint>

#include "internal.h"

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

__global__ void corr_diag_kernel(float* symmat, int64_t m) {
  const int64_t j = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (j < m) symmat[j * m + j] = 1.0f;
}

const void* syrk_func(int variant);

const void* corr_func(int variant) {
  return variant == CATT_VAR_STAGED ? syrk_func(CATT_VAR_STAGED) : (const void*)corr_thread_kernel;
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
  corr_stats_kernel<<<dim3(unsigned((m + 255) / 256)), 256, 0, s>>>(CorrStatsArgs{data, mean, stdv, n, m});
  catt_status st = after_launch();
  if (st != CATT_OK) return st;
  if (var == CATT_VAR_LITERAL) {
    CorrArgs a{data, symmat, n, m, Throttle{}};
    const int threads = cta_threads_or(t, 256);
    size_t dyn = 0;
    st = prepare_launch((const void*)corr_thread_kernel, t, threads, 0, true, &a.t, &dyn);
    if (st != CATT_OK) return st;
    corr_thread_kernel<<<dim3(unsigned((m + threads - 1) / threads)), threads, dyn, s>>>(a);
    return after_launch();
  }
  // STAGED: work = data^T (m x n), symmat = work work^T (alpha 1, beta 0), diagonal 1
  const int64_t gy = (n + 31) / 32;
  if (gy > 65535) return CATT_EINVAL;
  transpose32_kernel<<<dim3(unsigned((m + 31) / 32), unsigned(gy)), 256, 0, s>>>(data, work, n, m);
  st = after_launch();
  if (st != CATT_OK) return st;
  if (cudaMemsetAsync(symmat, 0, size_t(m) * size_t(m) * 4, s) != cudaSuccess) return after_launch();
  catt_throttle staged{};
  staged.variant = CATT_VAR_STAGED;
  st = catt_syrk(work, symmat, m, n, 1.0f, 0.0f, &staged, stream);
  if (st != CATT_OK) return st;
  corr_diag_kernel<<<dim3(unsigned((m + 255) / 256)), 256, 0, s>>>(symmat, m);
  return after_launch();
}
