// launch.cu — device context, throttle validation and application, the
// descriptors of this library's own kernels, catt_plan, and helper kernels
// (seeded generator, Fig 3-style L1D probe).
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <mutex>
#include <vector>

#include <cuda.h>

#include "internal.h"

namespace catt {

const void* gemv_func(int loop, int variant, bool vec_ok);
int row_tma_stages(int nmat, int rows, int boxes);
int col_tma_stages(int cols, int rows_per_stage);
int row_tma_stage_bytes(int nmat, int rows, int boxes);
int col_tma_stage_bytes(int cols, int rows_per_stage);
const void* syrk_func(int variant, int64_t n, bool tri);
const void* syr2k_func(int variant, int64_t n);
int64_t syr2k_staged_dyn(int64_t n);
int64_t syrk_staged_dyn(int64_t n, bool tri);
const void* kmeans_func(int variant, int nf);
int64_t kmeans_tma_smem(int nf, int k);
const void* kmeans_t_func(int variant);
const void* corr_func(int variant, int64_t m);
const void* gemm_func(int variant);
const void* fused_func(bool dep);

namespace {
std::mutex g_mu;
DevCtx g_ctx[64];
thread_local int g_last_err = 0;
}  // namespace

void record_cuda_error(cudaError_t e) { g_last_err = int(e); }

catt_status after_launch() {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  return CATT_OK;
}

catt_status dev_ctx(DevCtx** out) {
  int dev = -1;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess || dev < 0 || dev >= 64) {
    record_cuda_error(e);
    return CATT_ENODEV;
  }
  std::lock_guard<std::mutex> lk(g_mu);
  DevCtx& c = g_ctx[dev];
  if (c.device < 0) {
    catt_status st = catt_hw_query(dev, &c.hw);
    if (st != CATT_OK) return st;
    void* p = nullptr;
    e = cudaMalloc(&p, size_t(c.hw.num_sms) * sizeof(int) + 256);
    if (e != cudaSuccess) {
      record_cuda_error(e);
      return CATT_ENOMEM;
    }
    e = cudaMemset(p, 0, size_t(c.hw.num_sms) * sizeof(int) + 256);
    if (e != cudaSuccess) {
      record_cuda_error(e);
      return CATT_ECUDA;
    }
    c.sm_counter = static_cast<int*>(p);
    c.gbar = reinterpret_cast<unsigned*>(static_cast<char*>(p) + ((size_t(c.hw.num_sms) * sizeof(int) + 127) / 128) * 128);
    c.device = dev;
  }
  *out = &c;
  return CATT_OK;
}

catt_status dev_workspace(size_t bytes, float** out, unsigned** gbar) {
  DevCtx* c = nullptr;
  catt_status st = dev_ctx(&c);
  if (st != CATT_OK) return st;
  std::lock_guard<std::mutex> lk(g_mu);
  if (c->work_bytes < bytes) {
    if (c->work) cudaFree(c->work);
    c->work = nullptr;
    c->work_bytes = 0;
    void* p = nullptr;
    cudaError_t e = cudaMalloc(&p, bytes);
    if (e != cudaSuccess) {
      record_cuda_error(e);
      return CATT_ENOMEM;
    }
    c->work = static_cast<float*>(p);
    c->work_bytes = bytes;
  }
  *out = c->work;
  *gbar = c->gbar;
  return CATT_OK;
}

catt_status prepare_launch(const void* func, const catt_throttle* t, int threads, size_t dyn_smem,
                           bool allow_warp_gate, Throttle* kt, size_t* dyn_total) {
  if (threads < 32 || threads > 1024 || threads % 32) return CATT_EINVAL;
  const int W = threads / 32;
  DevCtx* ctx = nullptr;
  catt_status st = dev_ctx(&ctx);
  if (st != CATT_OK) return st;
  kt->active_warps = W;
  kt->gate = CATT_GATE_SEMAPHORE;
  kt->cta_cap = 0;
  kt->sm_counter = ctx->sm_counter;
  kt->probe = nullptr;
  *dyn_total = dyn_smem;
  if (!t) return CATT_OK;
  if (t->active_warps < 0 || t->active_warps > W || t->active_ctas < 0 || t->active_ctas > 32) return CATT_EINVAL;
  if (t->gate != CATT_GATE_SEMAPHORE && t->gate != CATT_GATE_BARRIER) return CATT_EINVAL;
  if (t->cap != CATT_CAP_SM_COUNTER && t->cap != CATT_CAP_SMEM_PAD) return CATT_EINVAL;
  const int aw = t->active_warps == 0 ? W : t->active_warps;
  if (aw < W && !allow_warp_gate) return CATT_EINVAL;
  kt->active_warps = aw;
  kt->gate = t->gate;
  kt->probe = reinterpret_cast<unsigned long long*>(t->probe);
  int64_t carve_bytes = -1;
  if (t->carveout_kb >= 0) {
    int idx = -1;
    for (int i = 0; i < ctx->hw.n_carveouts; ++i)
      if (ctx->hw.carveout_kb[i] == t->carveout_kb) idx = i;
    if (idx < 0) return CATT_EINVAL;
    cudaError_t e = cudaFuncSetAttribute(func, cudaFuncAttributePreferredSharedMemoryCarveout, ctx->hw.carveout_pct[idx]);
    if (e != cudaSuccess) {
      record_cuda_error(e);
      return CATT_ECUDA;
    }
    carve_bytes = int64_t(ctx->hw.carveout_kb[idx]) * 1024;
  }
  if (t->active_ctas > 0) {
    int occ = 0;
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, func, threads, dyn_smem);
    if (e != cudaSuccess) {
      record_cuda_error(e);
      return CATT_ECUDA;
    }
    if (t->active_ctas < occ || t->cap == CATT_CAP_SMEM_PAD) {
      if (t->cap == CATT_CAP_SM_COUNTER) {
        kt->cta_cap = t->active_ctas;
      } else {
        // Fig 5: pad dynamic shared memory so that exactly
        // active_ctas CTAs fit in the requested carveout.
        if (carve_bytes <= 0) return CATT_EINVAL;
        cudaFuncAttributes fa;
        e = cudaFuncGetAttributes(&fa, func);
        if (e != cudaSuccess) {
          record_cuda_error(e);
          return CATT_ECUDA;
        }
        const int64_t unit = ctx->hw.smem_alloc_unit, rsv = ctx->hw.reserved_smem_cta;
        const int64_t budget = (carve_bytes / t->active_ctas) / unit * unit;   // per-CTA allocation
        int64_t pad = budget - rsv - int64_t(fa.sharedSizeBytes) - int64_t(dyn_smem);
        pad = pad / unit * unit;
        if (pad < 0) return CATT_EINVAL;
        const int64_t per = ((int64_t(fa.sharedSizeBytes) + int64_t(dyn_smem) + pad + rsv + unit - 1) / unit) * unit;
        if (per * t->active_ctas > carve_bytes || per * (t->active_ctas + 1) <= carve_bytes) return CATT_EINVAL;
        *dyn_total = dyn_smem + size_t(pad);
        if (*dyn_total > 48 * 1024) {
          e = cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, int(*dyn_total));
          if (e != cudaSuccess) {
            record_cuda_error(e);
            return CATT_ECUDA;
          }
        }
      }
    }
  }
  return CATT_OK;
}

// ---------------------------------------------------------------- helper kernels
__device__ __forceinline__ uint32_t fmix32_d(uint32_t h) {
  h ^= h >> 16;
  h *= 0x85EBCA6Bu;
  h ^= h >> 13;
  h *= 0xC2B2AE35u;
  h ^= h >> 16;
  return h;
}

// The counter-based generator of seeded_inputs.py, in device code.
__global__ void fill_hash_kernel(float* dst, int64_t n, uint32_t seed, uint64_t offset, int mode) {
  for (int64_t k = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; k < n; k += int64_t(gridDim.x) * blockDim.x) {
    const uint64_t idx = offset + uint64_t(k);
    const uint32_t lo = uint32_t(idx & 0xFFFFFFFFull), hi = uint32_t(idx >> 32);
    const uint32_t key = fmix32_d(seed * 0x9E3779B9u + hi * 0x632BE5ABu + 0x7F4A7C15u);
    const uint32_t h = fmix32_d((lo * 0x85EBCA77u) ^ key);
    dst[k] = (mode == 1) ? float(h & 15u) * (1.0f / 16.0f) : float(h >> 8) * (1.0f / 16777216.0f);
  }
}

__global__ void chase_kernel(const int* __restrict__ next, int nlines, int passes, long long* out_cyc, int* sink) {
  int cur = 0;
  for (int i = 0; i < nlines; ++i) cur = __ldca(next + cur);
  const long long t0 = clock64();
  for (int p = 0; p < passes; ++p)
    for (int i = 0; i < nlines; ++i) cur = __ldca(next + cur);
  out_cyc[0] = clock64() - t0;
  sink[0] = cur;
}

// ---------------------------------------------------------------- kernel descriptors
namespace {

catt_ref mkref(int64_t cx, int64_t cy, int64_t c0, int64_t c1, int32_t e, int32_t arr, int32_t flags) {
  catt_ref r;
  std::memset(&r, 0, sizeof(r));
  r.c_gid[0] = cx;
  r.c_gid[1] = cy;
  r.c_iter[0] = c0;
  r.c_iter[1] = c1;
  r.elem_bytes = e;
  r.array_id = arr;
  r.flags = flags;
  return r;
}

int default_threads(int loop, int variant) {
  if (variant == CATT_VAR_STAGED)
    return (loop == CATT_K_SYRK || loop == CATT_K_SYR2K || loop == CATT_K_GEMM || loop == CATT_K_CORR) ? 256 : 32;
  if (variant == CATT_VAR_COOP && (loop == CATT_K_ATAX_2 || loop == CATT_K_BICG_1 || loop == CATT_K_MVT_2)) return 1024;
  return 256;
}

bool is_row(int loop) {
  return loop == CATT_K_ATAX_1 || loop == CATT_K_BICG_2 || loop == CATT_K_MVT_1 || loop == CATT_K_GESUMMV ||
         loop == CATT_K_ROWS3;
}
bool is_col(int loop) { return loop == CATT_K_ATAX_2 || loop == CATT_K_BICG_1 || loop == CATT_K_MVT_2; }

const void* loop_func(const catt_problem& p, int variant) {
  if (variant == CATT_VAR_FUSED && (is_row(p.loop) || is_col(p.loop))) return fused_func(p.loop == CATT_K_ATAX_1 || p.loop == CATT_K_ATAX_2);
  if (is_row(p.loop) || is_col(p.loop)) return gemv_func(p.loop, variant, true);
  if (p.loop == CATT_K_SYRK) return syrk_func(variant, p.n, false);
  if (p.loop == CATT_K_SYR2K) return syr2k_func(variant, p.n);
  if (p.loop == CATT_K_KMEANS_T) return kmeans_t_func(variant);
  if (p.loop == CATT_K_CORR) return corr_func(variant, p.n);
  if (p.loop == CATT_K_GEMM) return gemm_func(variant);
  return kmeans_func(variant, int(p.n));
}

}  // namespace
}  // namespace catt

using namespace catt;

extern "C" catt_status catt_kernel_attrs(const catt_problem* prob, const catt_throttle* t, int32_t* regs,
                                         int32_t* static_smem) {
  if (!prob || prob->loop < 0 || prob->loop >= CATT_K_COUNT) return CATT_EINVAL;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return CATT_ENODEV;
  cudaFuncAttributes fa;
  cudaError_t e = cudaFuncGetAttributes(&fa, loop_func(*prob, variant_of(t)));
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  if (regs) *regs = fa.numRegs;
  if (static_smem) *static_smem = int32_t(fa.sharedSizeBytes);
  return CATT_OK;
}

extern "C" catt_status catt_kernel_occupancy(const catt_problem* prob, const catt_throttle* t, int64_t extra_dyn_smem,
                                             int32_t* ctas_per_sm, int64_t* dyn_smem) {
  if (!prob || !ctas_per_sm || extra_dyn_smem < 0) return CATT_EINVAL;
  catt_ref refs[8];
  catt_loop_desc d;
  catt_status st = catt_kernel_desc(prob, t, CATT_MODE_UNION, &d, refs, 8);
  if (st != CATT_OK) return st;
  const void* func = loop_func(*prob, variant_of(t));
  cudaFuncAttributes fa;
  cudaError_t e = cudaFuncGetAttributes(&fa, func);
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  const int64_t dyn = int64_t(d.smem_per_cta) - int64_t(fa.sharedSizeBytes) + extra_dyn_smem;
  if (dyn < 0) return CATT_EINVAL;
  const int threads = d.block[0] * d.block[1] * d.block[2];
  if (dyn > fa.maxDynamicSharedSizeBytes) {
    e = cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, int(dyn));
    if (e != cudaSuccess) {
      record_cuda_error(e);
      return CATT_ECUDA;
    }
  }
  e = cudaFuncSetAttribute(func, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
  int n = 0;
  if (e == cudaSuccess)
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessorWithFlags(&n, func, threads, size_t(dyn),
                                                               cudaOccupancyDisableCachingOverride);
  const cudaError_t e2 = cudaFuncSetAttribute(func, cudaFuncAttributePreferredSharedMemoryCarveout,
                                              fa.preferredShmemCarveout);
  if (e == cudaSuccess) e = e2;
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  *ctas_per_sm = n;
  if (dyn_smem) *dyn_smem = dyn;
  return CATT_OK;
}

extern "C" catt_status catt_kernel_desc(const catt_problem* prob, const catt_throttle* t, int32_t mode,
                                        catt_loop_desc* out, catt_ref* refs, int32_t cap) {
  if (!prob || !out || !refs || cap < 8) return CATT_EINVAL;
  if (mode != CATT_MODE_UNION && mode != CATT_MODE_PAPER) return CATT_EINVAL;
  const int loop = prob->loop;
  if (loop < 0 || loop >= CATT_K_COUNT) return CATT_EINVAL;
  const int var = variant_of(t);
  const int threads = (t && t->cta_threads > 0) ? t->cta_threads : default_threads(loop, var);
  if (threads < 32 || threads > 1024 || threads % 32) return CATT_EINVAL;
  std::memset(out, 0, sizeof(*out));
  out->mode = mode;
  out->force_carveout_kb = -1;
  out->refs = refs;
  for (int k = 0; k < 3; ++k) out->block[k] = 1, out->grid[k] = 1, out->extent[k] = 0;
  out->block[0] = threads;
  int n = 0;
  int64_t dyn = 0;
  const int NL = CATT_REF_NOT_L1;
  if (is_row(loop)) {
    const int64_t M = (loop == CATT_K_MVT_1 || loop == CATT_K_GESUMMV) ? prob->n : prob->m;
    const int64_t N = prob->n;
    if (M < 1 || N < 1) return CATT_EINVAL;
    const bool two = loop == CATT_K_GESUMMV, three = loop == CATT_K_ROWS3;
    if (three && var != CATT_VAR_LITERAL) return CATT_EINVAL;
    out->n_loops = 1;
    out->extent[0] = M;
    if (var == CATT_VAR_LITERAL || var == CATT_VAR_BYPASS) {
      const int32_t fa = var == CATT_VAR_BYPASS ? CATT_REF_NOT_L1 : 0;  // BYPASS: the rows skip L1
      refs[n++] = mkref(N, 0, 1, 0, 4, 1, fa);                    // A[i*N + j]
      refs[n++] = mkref(0, 0, 1, 0, 4, 2, 0);                     // x[j]
      if (two || three) refs[n++] = mkref(N, 0, 1, 0, 4, 3, fa);  // B[i*N + j]
      if (three) refs[n++] = mkref(N, 0, 1, 0, 4, 4, fa);         // C[i*N + j]
      out->trip[0] = N;
      out->grid[0] = (M + threads - 1) / threads;
    } else if (var == CATT_VAR_VEC4) {
      if (N % 4) return CATT_EINVAL;
      refs[n++] = mkref(N / 4, 0, 1, 0, 16, 1, 0);
      refs[n++] = mkref(0, 0, 1, 0, 16, 2, 0);
      if (two) refs[n++] = mkref(N / 4, 0, 1, 0, 16, 3, 0);
      out->trip[0] = N / 4;
      out->grid[0] = (M + threads - 1) / threads;
    } else if (var == CATT_VAR_STAGED) {
      if (N % 4) return CATT_EINVAL;
      refs[n++] = mkref(N / 4, 0, 1, 0, 16, 1, NL);                // tiles arrive by bulk copy
      refs[n++] = mkref(0, 0, 1, 0, 16, 2, 0);
      if (two) refs[n++] = mkref(N / 4, 0, 1, 0, 16, 3, NL);
      out->trip[0] = N / 4;
      out->grid[0] = (M + threads - 1) / threads;
      const int nmat = two ? 2 : 1;
      const int boxes = std::max(1, std::min(8, 16384 / (nmat * threads * 128)));
      dyn = 1024 + int64_t(row_tma_stages(nmat, threads, boxes)) * row_tma_stage_bytes(nmat, threads, boxes);
    } else if (var == CATT_VAR_COOP || var == CATT_VAR_FUSED) {
      // warp per row: lane = gid_x (block 32 x W), row = gid_y
      const int64_t C4 = (N % 4 == 0) ? N / 4 : N;
      const int32_t e = (N % 4 == 0) ? 16 : 4;
      out->block[0] = 32;
      out->block[1] = threads / 32;
      out->grid[1] = (M + threads / 32 - 1) / (threads / 32);
      out->extent[0] = 32;
      out->extent[1] = M;
      refs[n++] = mkref(1, C4, 32, 0, e, 1, NL);
      refs[n++] = mkref(1, 0, 32, 0, e, 2, 0);
      if (two) refs[n++] = mkref(1, C4, 32, 0, e, 3, NL);
      out->trip[0] = (C4 + 31) / 32;
    } else {
      return CATT_EINVAL;
    }
  } else if (is_col(loop)) {
    const int64_t M = (loop == CATT_K_MVT_2) ? prob->n : prob->m;
    const int64_t N = prob->n;
    if (M < 1 || N < 1) return CATT_EINVAL;
    out->n_loops = 1;
    if (var == CATT_VAR_LITERAL) {
      refs[n++] = mkref(1, 0, N, 0, 4, 1, 0);                      // A[i*N + j]
      refs[n++] = mkref(0, 0, 1, 0, 4, 2, 0);                      // v[i]
      out->trip[0] = M;
      out->grid[0] = (N + threads - 1) / threads;
      out->extent[0] = N;
    } else if (var == CATT_VAR_VEC4) {
      if (N % 4) return CATT_EINVAL;
      refs[n++] = mkref(1, 0, N / 4, 0, 16, 1, 0);
      refs[n++] = mkref(0, 0, 1, 0, 4, 2, 0);
      out->trip[0] = M;
      out->grid[0] = (N / 4 + threads - 1) / threads;
      out->extent[0] = N / 4;
    } else if (var == CATT_VAR_COOP || var == CATT_VAR_FUSED) {
      const int NW = threads / 32;
      out->block[0] = 32;
      out->block[1] = NW;
      out->grid[0] = (N + 31) / 32;
      out->extent[0] = N;
      refs[n++] = mkref(1, N, int64_t(NW) * N, 0, 4, 1, NL);
      refs[n++] = mkref(0, 1, NW, 0, 4, 2, 0);
      out->trip[0] = (M + NW - 1) / NW;
    } else if (var == CATT_VAR_STAGED) {
      if (N % 4) return CATT_EINVAL;
      const int RB = std::max(16, std::min(256, 16384 / (threads * 4))) / 16 * 16;
      refs[n++] = mkref(1, 0, N, 0, 4, 1, NL);                     // tiles arrive by TMA
      refs[n++] = mkref(0, 0, 1, 0, 4, 2, 0);                      // v[i] broadcast
      out->trip[0] = M;
      out->grid[0] = (N + threads - 1) / threads;
      out->extent[0] = N;
      dyn = 1024 + int64_t(col_tma_stages(threads, RB)) * col_tma_stage_bytes(threads, RB);
    } else {
      return CATT_EINVAL;
    }
  } else if (loop == CATT_K_SYRK) {
    const int64_t N = prob->n, Mk = prob->k;
    if (N < 1 || Mk < 1) return CATT_EINVAL;
    out->n_loops = 1;
    out->trip[0] = Mk;
    if (var == CATT_VAR_LITERAL) {
      const int by = threads / 32;
      out->block[0] = 32;
      out->block[1] = by;
      out->grid[0] = (N + 31) / 32;
      out->grid[1] = (N + by - 1) / by;
      out->extent[0] = N;
      out->extent[1] = N;
      refs[n++] = mkref(0, Mk, 1, 0, 4, 1, 0);                     // a[i*M + k] (i = gid_y)
      refs[n++] = mkref(Mk, 0, 1, 0, 4, 1, 0);                     // a[j*M + k] (j = gid_x)
    } else if (var == CATT_VAR_STAGED) {
      out->block[0] = 256;
      out->grid[0] = (N + 127) / 128;
      out->grid[1] = (N + 127) / 128;
      refs[n++] = mkref(0, 0, 1, 0, 4, 1, NL);                     // staged through shared memory
      dyn = syrk_staged_dyn(N, false);                             // the T2 stage ring (dynamic shared memory)
    } else {
      return CATT_EINVAL;
    }
  } else if (loop == CATT_K_SYR2K) {
    const int64_t N = prob->n, Mk = prob->k;
    if (N < 1 || Mk < 1) return CATT_EINVAL;
    out->n_loops = 1;
    out->trip[0] = Mk;
    if (var == CATT_VAR_LITERAL) {
      const int by = threads / 32;
      out->block[0] = 32;
      out->block[1] = by;
      out->grid[0] = (N + 31) / 32;
      out->grid[1] = (N + by - 1) / by;
      out->extent[0] = N;
      out->extent[1] = N;
      refs[n++] = mkref(0, Mk, 1, 0, 4, 1, 0);                     // a[i*M + k]
      refs[n++] = mkref(0, Mk, 1, 0, 4, 2, 0);                     // b[i*M + k]
      refs[n++] = mkref(Mk, 0, 1, 0, 4, 1, 0);                     // a[j*M + k]
      refs[n++] = mkref(Mk, 0, 1, 0, 4, 2, 0);                     // b[j*M + k]
    } else if (var == CATT_VAR_STAGED) {
      out->block[0] = 256;
      out->grid[0] = (N + 127) / 128;
      out->grid[1] = (N + 127) / 128;
      refs[n++] = mkref(0, 0, 1, 0, 4, 1, NL);
      dyn = syr2k_staged_dyn(N);                                    // the DEEP stages (dynamic shared memory)
    } else {
      return CATT_EINVAL;
    }
  } else if (loop == CATT_K_CORR) {
    const int64_t Mc = prob->n, Nr = prob->k;  // Mc columns (threads), Nr rows (inner trip)
    if (Mc < 1 || Nr < 1) return CATT_EINVAL;
    if (var == CATT_VAR_STAGED) {                                  // the tiled SYRK of the transposed columns
      out->n_loops = 1;
      out->trip[0] = Nr;
      out->block[0] = 256;
      out->grid[0] = (Mc + 127) / 128;
      out->grid[1] = (Mc + 127) / 128;
      refs[n++] = mkref(0, 0, 1, 0, 4, 1, NL);
      dyn = syrk_staged_dyn(Mc, true);
      goto done_refs;
    }
    if (var != CATT_VAR_LITERAL) return CATT_EINVAL;
    out->grid[0] = (Mc + threads - 1) / threads;
    out->extent[0] = Mc;
    out->n_loops = 2;
    out->trip[0] = Mc;                                             // j2 (up to m - j1 - 1 iterations)
    out->trip[1] = Nr;                                             // i
    refs[n++] = mkref(1, 0, 0, Mc, 4, 1, 0);                     // data[i*m + j1]: reused only across j2
    refs[n++] = mkref(0, 0, 1, Mc, 4, 1, 0);                     // data[i*m + j2]: broadcast
    refs[n++] = mkref(Mc, 0, 1, 0, 4, 2, CATT_REF_STORE);        // symmat[j1*m + j2]
  } else if (loop == CATT_K_GEMM) {
    const int64_t Ni = prob->m, Nj = prob->n, Nk = prob->k;
    if (Ni < 1 || Nj < 1 || Nk < 1) return CATT_EINVAL;
    out->n_loops = 1;
    out->trip[0] = Nk;
    if (var == CATT_VAR_LITERAL) {
      const int by = threads / 32;
      out->block[0] = 32;
      out->block[1] = by;
      out->grid[0] = (Nj + 31) / 32;
      out->grid[1] = (Ni + by - 1) / by;
      out->extent[0] = Nj;
      out->extent[1] = Ni;
      refs[n++] = mkref(0, Nk, 1, 0, 4, 1, 0);                   // a[i*nk + k]: broadcast in the warp
      refs[n++] = mkref(1, 0, Nj, 0, 4, 2, 0);                   // b[k*nj + j]: coalesced
    } else if (var == CATT_VAR_STAGED) {
      out->block[0] = 256;
      out->grid[0] = (Nj + 127) / 128;
      out->grid[1] = (Ni + 127) / 128;
      refs[n++] = mkref(0, 0, 1, 0, 4, 1, NL);
    } else {
      return CATT_EINVAL;
    }
  } else if (loop == CATT_K_KMEANS_T) {
    const int64_t np = prob->m, nf = prob->n, ld = prob->ld;
    if (np < 1 || nf < 1 || ld < np) return CATT_EINVAL;
    out->grid[0] = (np + threads - 1) / threads;
    out->extent[0] = np;
    out->n_loops = 1;
    out->trip[0] = nf;
    if (var == CATT_VAR_LITERAL) {
      refs[n++] = mkref(nf, 0, 1, 0, 4, 1, 0);                     // in[p*nf + f]: divergent, reused over f
      refs[n++] = mkref(1, 0, ld, 0, 4, 2, CATT_REF_STORE);        // out[f*ld + p]
    } else if (var == CATT_VAR_COOP) {
      dyn = 256 * (nf | 1) * 4;
      refs[n++] = mkref(0, 0, 1, 0, 4, 1, CATT_REF_NOT_L1);        // shared-memory tile
    } else {
      return CATT_EINVAL;
    }
  } else {  // KMEANS
    const int64_t np = prob->m, nf = prob->n, k = prob->k, ld = prob->ld;
    if (np < 1 || nf < 1 || k < 1 || ld < np) return CATT_EINVAL;
    out->grid[0] = (np + threads - 1) / threads;
    out->extent[0] = np;
    dyn = nf * k * 4;
    if (var == CATT_VAR_LITERAL) {
      out->n_loops = 2;
      out->trip[0] = k;
      out->trip[1] = nf;
      refs[n++] = mkref(1, 0, 0, ld, 4, 1, 0);                     // feat[f*ld + p], reused across c
    } else if (var == CATT_VAR_REGS) {
      out->n_loops = 1;
      out->trip[0] = nf;
      refs[n++] = mkref(1, 0, ld, 0, 4, 1, 0);                     // streamed once
    } else if (var == CATT_VAR_STAGED) {
      out->n_loops = 1;
      out->trip[0] = nf;
      refs[n++] = mkref(1, 0, ld, 0, 4, 1, CATT_REF_NOT_L1);       // TMA tiles in shared memory
      dyn = kmeans_tma_smem(int(nf), int(k));                       // centres + the tile ring (Eq 4 sizes the carveout)
      out->grid[0] = std::min<int64_t>((np + 255) / 256, 2 * 148);  // persistent: at most 2 CTAs per SM
    } else if (var == CATT_VAR_COOP) {
      out->grid[0] = (np + 4 * threads - 1) / (4 * threads);       // a lane = 4 points
      out->extent[0] = (np + 3) / 4;
      out->n_loops = 1;
      out->trip[0] = nf;
      refs[n++] = mkref(4, 0, ld, 0, 4, 1, CATT_REF_NOT_L1);       // 16-byte L1::no_allocate loads
      dyn = nf * ((k + 1) & ~1) * 8;                               // centre pairs (c, c)
    } else {
      return CATT_EINVAL;
    }
  }
done_refs:
  out->n_refs = n;
  int32_t regs = 0, ssm = 16;  // without a device: the 4-byte gate slot, 16-byte aligned
  int32_t r2 = 0, s2 = 0;
  if (catt_kernel_attrs(prob, t, &r2, &s2) == CATT_OK) {
    regs = r2;
    ssm = s2;
  } else {
    cudaGetLastError();
  }
  out->regs_per_thread = regs;
  out->smem_per_cta = int32_t(ssm + dyn);
  return CATT_OK;
}

extern "C" catt_status catt_plan(const catt_problem* prob, const catt_throttle* launch, const catt_hw* hw,
                                 int32_t mode, catt_throttle* out, catt_footprint_result* res) {
  if (!prob || !hw || !out || !res) return CATT_EINVAL;
  catt_ref refs[8];
  catt_loop_desc d;
  catt_status st = catt_kernel_desc(prob, launch, mode, &d, refs, 8);
  if (st != CATT_OK) return st;
  if (launch && launch->carveout_kb > 0) d.force_carveout_kb = launch->carveout_kb;
  st = catt_footprint(&d, hw, res);
  if (st != CATT_OK) return st;
  catt_throttle o;
  std::memset(&o, 0, sizeof(o));
  if (launch) o = *launch;
  o.cta_threads = (launch && launch->cta_threads > 0) ? launch->cta_threads
                                                      : default_threads(prob->loop, variant_of(launch));
  o.active_warps = (res->flags & (CATT_FIT_WARP | CATT_FIT_CTA)) ? res->active_warps : 0;
  o.active_ctas = (res->flags & CATT_FIT_CTA) ? res->active_ctas : 0;
  o.carveout_kb = res->carveout_kb;
  *out = o;
  return CATT_OK;
}

extern "C" catt_status catt_hw_query(int device, catt_hw* out) {
  if (!out) return CATT_EINVAL;
  cudaDeviceProp p;
  cudaError_t e = cudaGetDeviceProperties(&p, device);
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ENODEV;
  }
  catt_hw_b200(out);  // measured L1D table (sm_100); props below override the counts
  out->num_sms = p.multiProcessorCount;
  out->max_warps_sm = p.maxThreadsPerMultiProcessor / p.warpSize;
  out->max_ctas_sm = p.maxBlocksPerMultiProcessor;
  out->regs_sm = p.regsPerMultiprocessor;
  out->warp_size = p.warpSize;
  out->reserved_smem_cta = int32_t(p.reservedSharedMemPerBlock);
  if (!(p.major == 10 && p.minor == 0)) {
    // not a B200: one option, nominal L1D = unified size - max shared memory
    const int32_t smax = int32_t(p.sharedMemPerMultiprocessor / 1024);
    out->n_carveouts = 1;
    out->carveout_kb[0] = smax;
    out->carveout_pct[0] = 100;
    out->l1d_bytes[0] = 32 * 1024;
  }
  return CATT_OK;
}

extern "C" catt_status catt_fill_hash(float* dst, int64_t n, uint32_t seed, uint64_t offset, int32_t mode,
                                      void* stream) {
  if (n < 0 || (n > 0 && !dst) || (mode != 0 && mode != 1)) return CATT_EINVAL;
  if (n == 0) return CATT_OK;
  const int64_t blocks = std::min<int64_t>((n + 255) / 256, 148 * 32);
  fill_hash_kernel<<<unsigned(blocks), 256, 0, static_cast<cudaStream_t>(stream)>>>(dst, n, seed, offset, mode);
  return after_launch();
}

extern "C" catt_status catt_calibrate_l1(int device, int32_t pct, const int32_t* kb, int32_t n, float* cycles_out) {
  if (!kb || !cycles_out || n < 1 || pct < 0 || pct > 100) return CATT_EINVAL;
  if (cudaSetDevice(device) != cudaSuccess) return CATT_ENODEV;
  int32_t maxkb = 0;
  for (int i = 0; i < n; ++i) {
    if (kb[i] < 1 || kb[i] > 4096) return CATT_EINVAL;
    maxkb = std::max(maxkb, kb[i]);
  }
  const int64_t max_lines = int64_t(maxkb) * 1024 / 128;
  int *d_next = nullptr, *d_sink = nullptr;
  long long* d_cyc = nullptr;
  catt_status st = CATT_OK;
  int* h = new int[size_t(max_lines) * 32]();
  cudaError_t e = cudaMalloc(&d_next, size_t(max_lines) * 32 * sizeof(int));
  if (e == cudaSuccess) e = cudaMalloc(&d_sink, sizeof(int));
  if (e == cudaSuccess) e = cudaMalloc(&d_cyc, sizeof(long long));
  if (e == cudaSuccess) e = cudaFuncSetAttribute((const void*)chase_kernel, cudaFuncAttributePreferredSharedMemoryCarveout, pct);
  for (int i = 0; i < n && e == cudaSuccess; ++i) {
    const int nl = int(int64_t(kb[i]) * 1024 / 128);
    for (int l = 0; l < nl; ++l) h[size_t(l) * 32] = ((l + 1) % nl) * 32;
    e = cudaMemcpy(d_next, h, size_t(nl) * 32 * sizeof(int), cudaMemcpyHostToDevice);
    if (e != cudaSuccess) break;
    chase_kernel<<<1, 1>>>(d_next, nl, 4, d_cyc, d_sink);
    e = cudaDeviceSynchronize();
    long long cyc = 0;
    if (e == cudaSuccess) e = cudaMemcpy(&cyc, d_cyc, sizeof(long long), cudaMemcpyDeviceToHost);
    cycles_out[i] = float(double(cyc) / (4.0 * nl));
  }
  if (e != cudaSuccess) {
    record_cuda_error(e);
    st = CATT_ECUDA;
  }
  delete[] h;
  cudaFree(d_next);
  cudaFree(d_sink);
  cudaFree(d_cyc);
  return st;
}

extern "C" const char* catt_status_str(catt_status s) {
  switch (s) {
    case CATT_OK: return "ok";
    case CATT_EINVAL: return "invalid argument";
    case CATT_ECUDA: return "CUDA error";
    case CATT_EUNSUPPORTED: return "unsupported";
    case CATT_ENOMEM: return "out of memory";
    case CATT_ENODEV: return "no CUDA device";
    case CATT_EINEXACT: return "inexact: a KMEANS feature value outside the exact fixed-point range";
  }
  return "unknown status";
}

extern "C" int catt_last_cuda_error(void) { return g_last_err; }
extern "C" int catt_abi_version(void) { return 6; }

// ------------------------------------------------------------ SM partition
// Green context of >= min_sms SMs and a non-blocking stream in it (catt.h).
// Driver entry points through the runtime (no -lcuda link).
namespace {
struct GreenApi {
  bool ok = false;
  CUresult (*devGet)(CUdevice*, int) = nullptr;
  CUresult (*getRes)(CUdevice, CUdevResource*, CUdevResourceType) = nullptr;
  CUresult (*split)(CUdevResource*, unsigned*, const CUdevResource*, CUdevResource*, unsigned, unsigned) = nullptr;
  CUresult (*genDesc)(CUdevResourceDesc*, CUdevResource*, unsigned) = nullptr;
  CUresult (*create)(CUgreenCtx*, CUdevResourceDesc, CUdevice, unsigned) = nullptr;
  CUresult (*destroy)(CUgreenCtx) = nullptr;
  CUresult (*streamCreate)(CUstream*, CUgreenCtx, unsigned, int) = nullptr;
  CUresult (*streamDestroy)(CUstream) = nullptr;
};
template <typename F>
bool entry(const char* name, F* out) {
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess) {
    cudaGetLastError();
    return false;
  }
  *out = reinterpret_cast<F>(p);
  return true;
}
const GreenApi& green_api() {
  static GreenApi g = [] {
    GreenApi a;
    a.ok = entry("cuDeviceGet", &a.devGet) && entry("cuDeviceGetDevResource", &a.getRes) &&
           entry("cuDevSmResourceSplitByCount", &a.split) && entry("cuDevResourceGenerateDesc", &a.genDesc) &&
           entry("cuGreenCtxCreate", &a.create) && entry("cuGreenCtxDestroy", &a.destroy) &&
           entry("cuGreenCtxStreamCreate", &a.streamCreate) && entry("cuStreamDestroy", &a.streamDestroy);
    return a;
  }();
  return g;
}
std::mutex g_green_mu;
std::vector<std::pair<CUstream, CUgreenCtx>> g_green;
}  // namespace

extern "C" catt_status catt_sm_partition_create(int device, int32_t min_sms, void** stream_out, int32_t* sms_out) {
  if (!stream_out || !sms_out || min_sms < 1) return CATT_EINVAL;
  const GreenApi& g = green_api();
  if (!g.ok) return CATT_EUNSUPPORTED;
  int nsm = 0;
  cudaError_t e = cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, device);
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  if (min_sms > nsm) return CATT_EINVAL;
  e = cudaFree(nullptr);  // the primary context is active before the green one (cuGreenCtxCreate note)
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  CUdevice dev;
  CUdevResource all{}, part{};
  CUdevResourceDesc desc;
  CUgreenCtx gc = nullptr;
  CUstream st = nullptr;
  unsigned ngroups = 1;
  if (g.devGet(&dev, device) != CUDA_SUCCESS || g.getRes(dev, &all, CU_DEV_RESOURCE_TYPE_SM) != CUDA_SUCCESS ||
      g.split(&part, &ngroups, &all, nullptr, 0, unsigned(min_sms)) != CUDA_SUCCESS || ngroups < 1 ||
      g.genDesc(&desc, &part, 1) != CUDA_SUCCESS || g.create(&gc, desc, dev, CU_GREEN_CTX_DEFAULT_STREAM) != CUDA_SUCCESS)
    return CATT_ECUDA;
  if (g.streamCreate(&st, gc, CU_STREAM_NON_BLOCKING, 0) != CUDA_SUCCESS) {
    g.destroy(gc);
    return CATT_ECUDA;
  }
  {
    std::lock_guard<std::mutex> lk(g_green_mu);
    g_green.push_back({st, gc});
  }
  *stream_out = reinterpret_cast<void*>(st);
  *sms_out = int32_t(part.sm.smCount);
  return CATT_OK;
}

extern "C" catt_status catt_sm_partition_destroy(void* stream) {
  const GreenApi& g = green_api();
  if (!g.ok) return CATT_EUNSUPPORTED;
  CUgreenCtx gc = nullptr;
  {
    std::lock_guard<std::mutex> lk(g_green_mu);
    for (size_t i = 0; i < g_green.size(); ++i)
      if (reinterpret_cast<void*>(g_green[i].first) == stream) {
        gc = g_green[i].second;
        g_green.erase(g_green.begin() + long(i));
        break;
      }
  }
  if (!gc) return CATT_EINVAL;
  const bool ok = g.streamDestroy(reinterpret_cast<CUstream>(stream)) == CUDA_SUCCESS;
  return (g.destroy(gc) == CUDA_SUCCESS && ok) ? CATT_OK : CATT_ECUDA;
}
