// k_fused.cu — FUSED variant: both loops of BICG / MVT / ATAX in one pass over A.
//
// The two loops of each application read the same matrix (ATAX's
// divergent phase and its coalesced phase; BICG and MVT likewise), so on B200
// the HBM-bound choice is to read A once:
//   BICG  q[i]  = sum_j A[i][j] p[j]          s[j]  = sum_i r[i] A[i][j]
//   MVT   x1[i] = x1[i] + sum_j A[i][j] y1[j]  x2[j] = x2[j] + sum_i A[i][j] y2[i]
//   ATAX  tmp[i] = sum_j A[i][j] x[j]          y[j]  = sum_i A[i][j] tmp[i]
// Grid = row bands (one or two CTAs per SM, cooperative launch). A CTA of NW
// warps covers all columns: warp w owns the 16-byte column chunks
// w*32 + lane + 32*NW*t (t < T). Rows are streamed U at a time with 16-byte
// L1-bypassing loads, U*T chunks in flight per lane. For each row the warp
// partial dots (fixed xor tree) are added in warp order in shared memory; ATAX
// then uses tmp[i] with the row still in registers, so A is never re-read.
// Each CTA writes its column partials to a workspace; after a grid barrier the
// partials are added in band order (deterministic). Results match the
// sequential oracle within 1e-5 of fp64 and bit-exactly on exact-dyadic input.
#include <algorithm>
#include <cstdint>
#include <cstdlib>

#include <cooperative_groups.h>

#include "internal.h"
#include "tma.cuh"

namespace catt {

constexpr int kMaxDual = 4;

// Up to kMaxDual independent problems with the same column count N share one
// launch (a grouped pass): CTAs [cta0[p], cta0[p+1]) stream problem p.
struct FusedArgs {
  const float* A[kMaxDual];
  const float* xr[kMaxDual];  // row-loop vector (p, y1, x)
  const float* xc[kMaxDual];  // column-loop vector (r, y2); ATAX: unused (tmp)
  float* yr[kMaxDual];        // row outputs (q, x1 in/out, tmp)
  float* yc[kMaxDual];        // column outputs (s, x2 in/out, y)
  float* part[kMaxDual];      // workspace: (CTAs of p) x N column partials
  int64_t M[kMaxDual];
  int64_t band[kMaxDual];     // rows per CTA
  int cta0[kMaxDual + 1];
  int row_acc[kMaxDual], col_acc[kMaxDual];
  int nprob;
  unsigned* gbar;             // grid barrier {count, generation}
  int64_t N;
};

__device__ __forceinline__ float4 ld_stream4(const float4* p) {
  float4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
  return r;
}

__device__ __forceinline__ void grid_barrier(unsigned* bar, unsigned nblocks) {
  __syncthreads();
  if (threadIdx.x == 0) {
    volatile unsigned* vb = bar;
    const unsigned gen = vb[1];
    __threadfence();
    if (atomicAdd(&bar[0], 1u) == nblocks - 1) {
      bar[0] = 0;
      __threadfence();
      atomicAdd(&bar[1], 1u);
    } else {
      while (vb[1] == gen) __nanosleep(64);
    }
    __threadfence();
  }
  __syncthreads();
}

// DEP = true: ATAX (the column loop's vector is the row loop's result).
// NW warps per CTA, T 16-byte chunks per lane per row. A stage holds RPS
// whole rows (contiguous in memory: one bulk copy), S stages in a ring.
template <bool DEP, int NW, int T>
__global__ void __launch_bounds__(NW * 32, 1) fused_kernel(FusedArgs a, int RPS, int S) {
  extern __shared__ __align__(1024) unsigned char dyn[];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint64_t* full = reinterpret_cast<uint64_t*>(dyn);
  uint64_t* empty = full + S;
  float* rowbuf = reinterpret_cast<float*>(dyn + 512);         // [RPS][NW] warp partials
  float* rowval = rowbuf + RPS * NW;                            // [RPS] finished row values
  unsigned char* ring = dyn + 1024 + ((RPS * (NW + 1) * 4 + 1023) / 1024) * 1024;
  int pi = 0;
  while (pi + 1 < a.nprob && int(blockIdx.x) >= a.cta0[pi + 1]) ++pi;
  const float* __restrict__ Ap = a.A[pi];
  const int lb = int(blockIdx.x) - a.cta0[pi];                  // CTA index within its problem
  const int64_t N = a.N, n4 = N >> 2, M = a.M[pi];
  const int64_t stage_bytes = int64_t(RPS) * N * 4;
  const int64_t r0 = int64_t(lb) * a.band[pi], r1 = imin64(M, r0 + a.band[pi]);
  const int64_t nst = (r1 - r0 + RPS - 1) / RPS;               // stages of this band
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      bar_init(&full[s], 1);
      bar_init(&empty[s], NW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  auto issue = [&](int64_t c) {                                 // thread 0 only
    const int s = int(c % S);
    if (c >= S) bar_wait(&empty[s], uint32_t(((c / S) - 1) & 1));
    const int64_t rows = imin64(RPS, r1 - (r0 + c * RPS));
    const uint32_t bytes = uint32_t(rows * N * 4);
    bar_expect_tx(&full[s], bytes);
    bulk_1d(ring + int64_t(s) * stage_bytes, Ap + (r0 + c * RPS) * N, bytes, &full[s]);
  };
  if (threadIdx.x == 0)
    for (int64_t c = 0; c < imin64(S, nst); ++c) issue(c);
  const float4* x4 = reinterpret_cast<const float4*>(a.xr[pi]);
  float4 xr[T], acc[T];
#pragma unroll
  for (int t = 0; t < T; ++t) {
    const int64_t c = warp * 32 + lane + int64_t(32) * NW * t;
    xr[t] = c < n4 ? x4[c] : make_float4(0.f, 0.f, 0.f, 0.f);
    acc[t] = make_float4(0.f, 0.f, 0.f, 0.f);
  }
  for (int64_t c = 0; c < nst; ++c) {
    const int s = int(c % S);
    const int64_t i0 = r0 + c * RPS;
    const int rows = int(imin64(RPS, r1 - i0));
    bar_wait(&full[s], uint32_t((c / S) & 1));
    const float4* st = reinterpret_cast<const float4*>(ring + int64_t(s) * stage_bytes);
    // row dots: lane partial in chunk order, xor tree, warp partials to smem
    for (int u = 0; u < rows; ++u) {
      const float4* row = st + int64_t(u) * n4;
      float d = 0.0f;
#pragma unroll
      for (int t = 0; t < T; ++t) {
        const int64_t cc = warp * 32 + lane + int64_t(32) * NW * t;
        if (cc < n4) {
          const float4 v = row[cc];
          d = fmaf(v.x, xr[t].x, d);
          d = fmaf(v.y, xr[t].y, d);
          d = fmaf(v.z, xr[t].z, d);
          d = fmaf(v.w, xr[t].w, d);
        }
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) d += __shfl_xor_sync(0xffffffffu, d, o);
      if (lane == 0) rowbuf[u * NW + warp] = d;
    }
    __syncthreads();
    if (threadIdx.x < rows) {
      const int u = threadIdx.x;
      float sum = rowbuf[u * NW];
      for (int w = 1; w < NW; ++w) sum += rowbuf[u * NW + w];
      if (a.row_acc[pi]) sum = a.yr[pi][i0 + u] + sum;
      a.yr[pi][i0 + u] = sum;
      rowval[u] = sum;
    }
    __syncthreads();
    // column partials in row order, the row still in shared memory
    for (int u = 0; u < rows; ++u) {
      const float4* row = st + int64_t(u) * n4;
      const float w = DEP ? rowval[u] : a.xc[pi][i0 + u];
#pragma unroll
      for (int t = 0; t < T; ++t) {
        const int64_t cc = warp * 32 + lane + int64_t(32) * NW * t;
        if (cc < n4) {
          const float4 v = row[cc];
          acc[t].x = fmaf(v.x, w, acc[t].x);
          acc[t].y = fmaf(v.y, w, acc[t].y);
          acc[t].z = fmaf(v.z, w, acc[t].z);
          acc[t].w = fmaf(v.w, w, acc[t].w);
        }
      }
    }
    __syncwarp();
    if (lane == 0) bar_arrive(&empty[s]);
    if (threadIdx.x == 0 && c + S < nst) issue(c + S);
  }
  // column partials: first summed over the CL CTAs of this cluster through
  // distributed shared memory (rank order), so only G / CL partial vectors go
  // through global memory and the grid barrier
  namespace cg = cooperative_groups;
  cg::cluster_group cluster = cg::this_cluster();
  const int CL = int(cluster.num_blocks()), rank = int(cluster.block_rank());
  const int64_t cid = int64_t(lb) / CL;
  float* cpart = reinterpret_cast<float*>(ring);               // the ring is drained: reuse it
  {
    float4* c4 = reinterpret_cast<float4*>(cpart);
#pragma unroll
    for (int t = 0; t < T; ++t) {
      const int64_t cc = warp * 32 + lane + int64_t(32) * NW * t;
      if (cc < n4) c4[cc] = acc[t];
    }
  }
  cluster.sync();
  {
    const int64_t per = (N + CL - 1) / CL;
    const int64_t j0 = rank * per, j1 = imin64(N, j0 + per);
    for (int64_t j = j0 + threadIdx.x; j < j1; j += blockDim.x) {
      float sum = cluster.map_shared_rank(cpart, 0)[j];
      for (int q = 1; q < CL; ++q) sum += cluster.map_shared_rank(cpart, q)[j];
      a.part[pi][cid * N + j] = sum;
    }
  }
  cluster.sync();
  __threadfence();
  grid_barrier(a.gbar, gridDim.x);
  // column outputs: a fixed tree over each problem's band partials. The
  // 32-column chunks of all problems are dealt to the CTAs round robin; warp
  // w sums bands [w*gpw, (w+1)*gpw) in order (independent loads in flight),
  // the NW warp sums are added in warp order, then the initial value (MVT).
  {
    __shared__ float red[NW][32];
    const int64_t chunks = (N + 31) / 32;
    for (int64_t gch = blockIdx.x; gch < chunks * a.nprob; gch += gridDim.x) {
      const int q = int(gch / chunks);
      const int64_t ch = gch % chunks;
      const int64_t G = (a.cta0[q + 1] - a.cta0[q]) / CL;          // partial vectors of problem q
      const int64_t gpw = (G + NW - 1) / NW;
      const int64_t b0 = warp * gpw, b1 = imin64(G, b0 + gpw);
      const float* pq = a.part[q];
      const int64_t j = ch * 32 + lane;
      float sum = 0.0f;
      if (j < N) {
        int64_t b = b0;
        for (; b + 8 <= b1; b += 8) {
          float v[8];
#pragma unroll
          for (int k = 0; k < 8; ++k) v[k] = pq[(b + k) * N + j];
#pragma unroll
          for (int k = 0; k < 8; ++k) sum += v[k];
        }
        for (; b < b1; ++b) sum += pq[b * N + j];
      }
      red[warp][lane] = sum;
      __syncthreads();
      if (warp == 0 && j < N) {
        float tot = red[0][lane];
        for (int w = 1; w < NW; ++w) tot += red[w][lane];
        if (a.col_acc[q]) tot = a.yc[q][j] + tot;
        a.yc[q][j] = tot;
      }
      __syncthreads();
    }
  }
}

namespace {

template <bool DEP>
const void* fused_fn(int NW, int T) {
  if (NW == 16) {
    if (T == 2) return (const void*)fused_kernel<DEP, 16, 2>;
    if (T == 4) return (const void*)fused_kernel<DEP, 16, 4>;
    return (const void*)fused_kernel<DEP, 16, 8>;
  }
  if (T == 1) return (const void*)fused_kernel<DEP, 8, 1>;
  return (const void*)fused_kernel<DEP, 8, 2>;
}

}  // namespace

// Workspace (column partials) owned by the device context; grown on demand.
catt_status dev_workspace(size_t bytes, float** out, unsigned** gbar);

struct DualProblem {
  const float* A;
  const float* xr;
  const float* xc;
  float* yr;
  float* yc;
  int64_t M;
  int row_acc, col_acc;
};

catt_status launch_fused_group(bool dep, const DualProblem* pr, int np, int64_t N, const catt_throttle* t,
                               cudaStream_t s) {
  if (np < 1 || np > kMaxDual || N <= 0 || N % 4) return CATT_EINVAL;
  int64_t Mtot = 0;
  for (int i = 0; i < np; ++i) {
    if (pr[i].M <= 0) return CATT_EINVAL;
    if ((reinterpret_cast<uintptr_t>(pr[i].A) & 15u) || (reinterpret_cast<uintptr_t>(pr[i].xr) & 15u))
      return CATT_EINVAL;
    Mtot += pr[i].M;
  }
  if (t && (t->active_warps || t->active_ctas)) return CATT_EINVAL;  // nothing to throttle (no L1 reuse)
  const int64_t n4 = N / 4;
  // 8 warps for short rows (T <= 2 chunks per lane), else 16 warps with
  // T = 2, 4 or 8 chunks per lane (N <= 16384)
  const int NW = n4 <= 512 ? 8 : 16;
  const int64_t T64 = (n4 + 32 * NW - 1) / (32 * NW);
  if (T64 > 8) return CATT_EUNSUPPORTED;  // N > 16384
  const int T = T64 <= 1 ? 1 : (T64 <= 2 ? 2 : (T64 <= 4 ? 4 : 8));
  const int threads = NW * 32;
  const void* f = dep ? fused_fn<true>(NW, T) : fused_fn<false>(NW, T);
  // stage = RPS whole rows (~64 KB: several independent row chains per warp
  // and few barriers per byte), S stages within ~200 KB of shared memory
  const int64_t row_bytes = N * 4;
  const char* rps_env = getenv("CATT_FUSED_STAGE_KB");
  const int64_t stage_target = (rps_env ? atoi(rps_env) : 64) * 1024;
  const int RPS = int(std::max<int64_t>(1, std::min<int64_t>(16, stage_target / row_bytes)));
  const int64_t head = 1024 + ((int64_t(RPS) * (NW + 1) * 4 + 1023) / 1024) * 1024;
  const char* budget_env = getenv("CATT_FUSED_SMEM_KB");
  const int64_t budget = (budget_env ? atoi(budget_env) : 200) * 1024;
  const int S = int(std::min<int64_t>(16, (budget - head) / (RPS * row_bytes)));
  if (S < 2) return CATT_EUNSUPPORTED;
  const size_t smem = size_t(head + int64_t(S) * RPS * row_bytes);
  cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, f, threads, smem);
  if (e != cudaSuccess || occ < 1) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  DevCtx* ctx = nullptr;
  catt_status st = dev_ctx(&ctx);
  if (st != CATT_OK) return st;
  // cluster of CL CTAs for the DSMEM pre-reduction (single problem only;
  // default 1: no measured gain at 4096^2, and clustered cooperative launches
  // cannot be replayed by ncu)
  const char* cl_env = getenv("CATT_FUSED_CLUSTER");
  const int64_t slots = int64_t(ctx->hw.num_sms) * occ;
  int CL = 1;
  int64_t Gall = std::min<int64_t>(slots, Mtot);
  for (int cand = (cl_env && np == 1) ? atoi(cl_env) : 1; cand >= 2; cand /= 2) {
    if (S * RPS * row_bytes < N * 4) break;
    cudaLaunchConfig_t qc = {};
    qc.gridDim = dim3(unsigned(Gall / cand * cand), 1, 1);
    qc.blockDim = dim3(unsigned(threads), 1, 1);
    qc.dynamicSmemBytes = smem;
    cudaLaunchAttribute qa[1];
    qa[0].id = cudaLaunchAttributeClusterDimension;
    qa[0].val.clusterDim.x = unsigned(cand);
    qa[0].val.clusterDim.y = 1;
    qa[0].val.clusterDim.z = 1;
    qc.attrs = qa;
    qc.numAttrs = 1;
    int nclusters = 0;
    if (cudaOccupancyMaxActiveClusters(&nclusters, f, &qc) != cudaSuccess) {
      cudaGetLastError();
      continue;
    }
    const int64_t g = std::min<int64_t>(int64_t(nclusters) * cand, Gall / cand * cand);
    if (g >= 2 * cand && g * 100 >= Gall * 95) {
      CL = cand;
      Gall = g;
      break;
    }
  }
  // CTAs per problem proportional to its rows (each at least CL), multiples of CL
  FusedArgs args{};
  args.nprob = np;
  args.N = N;
  int64_t given = 0;
  int cta = 0;
  for (int i = 0; i < np; ++i) {
    int64_t g = (i == np - 1) ? Gall - given : (Gall * pr[i].M) / Mtot;
    g = std::max<int64_t>(CL, g / CL * CL);
    g = std::min<int64_t>(g, std::max<int64_t>(CL, (pr[i].M + CL - 1) / CL * CL));
    given += g;
    args.A[i] = pr[i].A;
    args.xr[i] = pr[i].xr;
    args.xc[i] = pr[i].xc;
    args.yr[i] = pr[i].yr;
    args.yc[i] = pr[i].yc;
    args.M[i] = pr[i].M;
    args.band[i] = (pr[i].M + g - 1) / g;
    args.row_acc[i] = pr[i].row_acc;
    args.col_acc[i] = pr[i].col_acc;
    args.cta0[i] = cta;
    cta += int(g);
  }
  args.cta0[np] = cta;
  if (cta > slots) return CATT_EUNSUPPORTED;                 // cannot be co-resident for the grid barrier
  float* work = nullptr;
  unsigned* gbar = nullptr;
  size_t need = 0;
  for (int i = 0; i < np; ++i) need += size_t((args.cta0[i + 1] - args.cta0[i]) / CL) * size_t(N);
  st = dev_workspace(need * sizeof(float), &work, &gbar);
  if (st != CATT_OK) return st;
  size_t off = 0;
  for (int i = 0; i < np; ++i) {
    args.part[i] = work + off;
    off += size_t((args.cta0[i + 1] - args.cta0[i]) / CL) * size_t(N);
  }
  args.gbar = gbar;
  int rps = RPS, stages = S;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(unsigned(cta), 1, 1);
  cfg.blockDim = dim3(unsigned(threads), 1, 1);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeCooperative;
  attr[0].val.cooperative = 1;
  attr[1].id = cudaLaunchAttributeClusterDimension;
  attr[1].val.clusterDim.x = unsigned(CL);
  attr[1].val.clusterDim.y = 1;
  attr[1].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 2;
  void* params[] = {&args, &rps, &stages};
  e = cudaLaunchKernelExC(&cfg, f, params);
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  return after_launch();
}

catt_status launch_fused(bool dep, const float* A, const float* xr, const float* xc, float* yr, float* yc, int64_t M,
                         int64_t N, int row_acc, int col_acc, const catt_throttle* t, cudaStream_t s) {
  if (M == 0 || N == 0) return CATT_EINVAL;  // callers route empty shapes to the per-loop path
  DualProblem p{A, xr, xc, yr, yc, M, row_acc, col_acc};
  return launch_fused_group(dep, &p, 1, N, t, s);
}

const void* fused_func(bool dep) { return dep ? fused_fn<true>(16, 2) : fused_fn<false>(16, 2); }

}  // namespace catt

using namespace catt;

extern "C" catt_status catt_dual_group(const catt_dual_problem* probs, int32_t count, int32_t dependent,
                                       const catt_throttle* t, void* stream) {
  if (!probs || count < 1 || count > kMaxDual) return CATT_EINVAL;
  DualProblem pr[kMaxDual];
  const int64_t N = probs[0].n;
  for (int i = 0; i < count; ++i) {
    const catt_dual_problem& q = probs[i];
    if (q.n != N || q.m < 1 || !q.A || !q.xr || !q.yr || !q.yc || (!dependent && !q.xc)) return CATT_EINVAL;
    if (dependent && q.row_accumulate) return CATT_EINVAL;
    pr[i] = DualProblem{q.A, q.xr, q.xc, q.yr, q.yc, q.m, q.row_accumulate != 0, q.col_accumulate != 0};
  }
  return launch_fused_group(dependent != 0, pr, count, N, t, static_cast<cudaStream_t>(stream));
}

extern "C" catt_status catt_dual(const float* A, const float* xr, const float* xc, float* yr, float* yc, int64_t m,
                                 int64_t n, int32_t row_accumulate, int32_t col_accumulate, int32_t dependent,
                                 const catt_throttle* t, void* stream) {
  if (m < 1 || n < 1 || !A || !xr || !yr || !yc || (!dependent && !xc)) return CATT_EINVAL;
  if (dependent && row_accumulate) return CATT_EINVAL;
  return launch_fused(dependent != 0, A, xr, xc, yr, yc, m, n, row_accumulate != 0, col_accumulate != 0, t,
                      static_cast<cudaStream_t>(stream));
}
