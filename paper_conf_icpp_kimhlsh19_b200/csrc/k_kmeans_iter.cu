// k_kmeans_iter.cu — the KMEANS full iteration around the assignment step
// (Rodinia kmeans, the KM workload of Table 2 P:84 whose two
// loops are the KM rows of Table 3).
//
// TRANSPOSE (KM's other loop, Rodinia invert_mapping): out[f*ld + p] =
//   in[p*nf + f]. LITERAL = thread per point, for f < nf: the load is
//   memory-divergent (lanes nf*4 B apart) and each line is re-used by the same
//   thread for the next features: a CATT loop (CATT_K_KMEANS_T). COOP = 256
//   points per CTA through shared memory, coalesced on both sides.
// ACCUMULATE: assignment (decisions identical to catt_kmeans_assign: f
//   ascending with fmaf, strict <) fused with exact centroid sums. Each feature
//   value becomes the two's-complement 128-bit integer x*2^64; integer sums do
//   not depend on order, so the result is the same for any CTA count, tile
//   order or number of GPUs (R21). Per 256-point tile: phase 1,
//   thread per point, streams the point's features from HBM once into a
//   shared-memory tile and decides its centre; the tile's points are then
//   counting-sorted by centre; phase 2, lane per feature, walks the sorted
//   points of each centre (a warp-uniform segment) and adds into 128-bit
//   registers. At the end each CTA sums its warps exactly and adds the four
//   32-bit chunks of each sum into int64 limbs in HBM (atomics, exact).
// FINALIZE: centre = round-to-nearest-even(sum / count) in integer arithmetic.
#include <algorithm>
#include <cfloat>
#include <cstdint>

#include "internal.h"

namespace catt {

// ------------------------------------------------------------------ transpose
struct TrArgs {
  const float* in;
  float* out;
  int64_t npoints, ld;
  int nf;
  Throttle t;
};

__global__ void __launch_bounds__(1024, 2) km_transpose_thread_kernel(TrArgs a) {
  __shared__ int slots;
  gate_init(&slots, a.t);
  __syncthreads();
  cta_enter(a.t);
  const int64_t p = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  throttled(a.t, &slots, [&]() {
    if (p >= a.npoints) return;
    const float* src = a.in + p * a.nf;
#pragma unroll 4
    for (int f = 0; f < a.nf; ++f) a.out[int64_t(f) * a.ld + p] = src[f];
  });
  cta_exit(a.t);
}

// 256 points per CTA: the tile's 256*nf contiguous floats are read coalesced
// into shared memory (row pitch nf|1, so the column reads below do not
// conflict), then written one feature row at a time.
__global__ void __launch_bounds__(256) km_transpose_tile_kernel(TrArgs a) {
  extern __shared__ float s_tile[];
  cta_enter(a.t);
  const int nf = a.nf, pitch = nf | 1;
  const int64_t p0 = int64_t(blockIdx.x) * 256;
  const int np = int(imin64(256, a.npoints - p0));
  const float* src = a.in + p0 * nf;
  const int total = np * nf;
  for (int j = threadIdx.x; j < total; j += 256) {
    const int pl = j / nf, f = j - pl * nf;
    s_tile[pl * pitch + f] = __ldg(src + j);
  }
  __syncthreads();
  if (int(threadIdx.x) < np)
    for (int f = 0; f < nf; ++f) a.out[int64_t(f) * a.ld + p0 + threadIdx.x] = s_tile[threadIdx.x * pitch + f];
  cta_exit(a.t);
}

const void* kmeans_t_func(int variant) {
  return variant == CATT_VAR_COOP ? (const void*)km_transpose_tile_kernel : (const void*)km_transpose_thread_kernel;
}

// ------------------------------------------------------------------ exact sums
typedef unsigned __int128 u128;

// x * 2^64 as a two's-complement 128-bit integer. Exact for x = 0 and for
// 2^-64 <= ulp(x), |x| < 2^31; anything else (non-zero bits below 2^-64,
// |x| >= 2^31, subnormal, inf, NaN) counts in `inexact`.
__device__ __forceinline__ u128 to_fixed(float x, int& inexact) {
  const uint32_t b = __float_as_uint(x);
  const int e = int((b >> 23) & 0xffu);
  uint32_t m = b & 0x7fffffu;
  if (e == 0) {
    inexact += (m != 0u);
    return 0;
  }
  if (e >= 158) {
    ++inexact;
    return 0;
  }
  m |= 0x800000u;
  const int sh = e - 86;  // x = m * 2^(e-150); x * 2^64 = m * 2^(e-86)
  u128 u;
  if (sh >= 0) {
    u = u128(m) << sh;
  } else {
    const int r = -sh;
    inexact += (r >= 24) || (m & ((1u << r) - 1u)) != 0u;
    u = r >= 24 ? u128(0) : u128(m >> r);
  }
  return (b >> 31) ? u128(0) - u : u;
}

constexpr int KT = 256;      // points per tile = threads per CTA
constexpr int KTP = KT + 1;  // tile row pitch: column reads across features hit distinct banks

struct AccArgs {
  const float* feat;
  const float* clusters;
  int32_t* memb;
  unsigned long long* acc;
  const long long* done;  // nullable: skip the pass when *done != 0
  int64_t ld, npoints;
  int nf, k;
};

template <int KMAX, int FB>
__global__ void __launch_bounds__(KT, 2) km_accumulate_kernel(AccArgs a) {
  if (a.done && *a.done) return;
  extern __shared__ __align__(16) unsigned char dyn[];
  const int nf = a.nf, k = a.k;
  float* s_ct = reinterpret_cast<float*>(dyn);                         // [nf][k]
  float* tile = s_ct + ((nf * k + 3) & ~3);                             // [nf][KTP]
  __shared__ int s_cnt[KMAX], s_start[KMAX + 1], s_tot[KMAX];
  __shared__ unsigned short s_idx[KT];
  const int t = threadIdx.x, lane = t & 31, w = t >> 5;
  for (int q = t; q < nf * k; q += KT) s_ct[(q % nf) * k + q / nf] = a.clusters[q];
  if (t < KMAX) s_tot[t] = 0;
  long long delta = 0;
  int inexact = 0;
  u128 acc[FB][KMAX];
#pragma unroll
  for (int fb = 0; fb < FB; ++fb)
#pragma unroll
    for (int c = 0; c < KMAX; ++c) acc[fb][c] = 0;

  const int64_t ntiles = (a.npoints + KT - 1) / KT;
  for (int64_t tl = blockIdx.x; tl < ntiles; tl += gridDim.x) {
    if (t < KMAX) s_cnt[t] = 0;
    __syncthreads();  // s_ct ready; the previous tile's phase 2 is done with `tile`
    const int64_t p = tl * KT + t;
    int c = -1, rank = 0, changed = 0;
    if (p < a.npoints) {
      const float* f0 = a.feat + p;
      float d[KMAX];
#pragma unroll
      for (int cc = 0; cc < KMAX; ++cc) d[cc] = 0.0f;
      int f = 0;
      for (; f + 8 <= nf; f += 8) {
        float v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u)
          asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v[u]) : "l"(f0 + int64_t(f + u) * a.ld));
#pragma unroll
        for (int u = 0; u < 8; ++u) {
          tile[(f + u) * KTP + t] = v[u];
          const float* cf = s_ct + (f + u) * k;
#pragma unroll
          for (int cc = 0; cc < KMAX; ++cc)
            if (cc < k) {
              const float diff = v[u] - cf[cc];
              d[cc] = fmaf(diff, diff, d[cc]);
            }
        }
      }
      for (; f < nf; ++f) {
        const float v = f0[int64_t(f) * a.ld];
        tile[f * KTP + t] = v;
        const float* cf = s_ct + f * k;
#pragma unroll
        for (int cc = 0; cc < KMAX; ++cc)
          if (cc < k) {
            const float diff = v - cf[cc];
            d[cc] = fmaf(diff, diff, d[cc]);
          }
      }
      float best = FLT_MAX;
#pragma unroll
      for (int cc = 0; cc < KMAX; ++cc)
        if (cc < k && d[cc] < best) {
          best = d[cc];
          c = cc;
        }
      if (c >= 0) {
        changed = a.memb[p] != c;
        a.memb[p] = c;
        rank = atomicAdd(&s_cnt[c], 1);
      } else {  // every distance is NaN or >= FLT_MAX: no centre (as catt_kmeans_assign)
        changed = a.memb[p] != -1;
        a.memb[p] = -1;
      }
    }
    const int nchg = __syncthreads_count(changed);
    if (t == 0) {
      delta += nchg;
      s_start[0] = 0;
      for (int cc = 0; cc < k; ++cc) {
        s_start[cc + 1] = s_start[cc] + s_cnt[cc];
        s_tot[cc] += s_cnt[cc];
      }
    }
    __syncthreads();
    if (c >= 0) s_idx[s_start[c] + rank] = static_cast<unsigned short>(t);
    __syncthreads();
    // phase 2: warp w owns sorted entries [32w, 32w + 32); lane = feature
    const int lo_w = w * 32, hi_w = lo_w + 32;
#pragma unroll
    for (int fb = 0; fb < FB; ++fb) {
      const int f = lane + 32 * fb;
      if (f < nf) {
        const float* row = tile + f * KTP;
#pragma unroll
        for (int cc = 0; cc < KMAX; ++cc) {
          if (cc < k) {
            const int lo = max(s_start[cc], lo_w), hi = min(s_start[cc + 1], hi_w);
            u128 sum = 0;
            for (int i = lo; i < hi; ++i) sum += to_fixed(row[s_idx[i]], inexact);
            acc[fb][cc] += sum;
          }
        }
      }
    }
  }
  __syncthreads();
  // epilogue: per centre, the CTA's warps summed exactly, then four 32-bit
  // chunks of the 128-bit sum added into the int64 limbs (exact, any order)
  u128* red = reinterpret_cast<u128*>(tile);  // [8 warps][FB*32]
  const int K4 = k * nf * 4;
#pragma unroll
  for (int cc = 0; cc < KMAX; ++cc) {
    if (cc < k) {
#pragma unroll
      for (int fb = 0; fb < FB; ++fb) red[w * (FB * 32) + fb * 32 + lane] = acc[fb][cc];
      __syncthreads();
      if (t < nf) {
        u128 s = 0;
        for (int ww = 0; ww < KT / 32; ++ww) s += red[ww * (FB * 32) + t];
        unsigned long long* limb = a.acc + (int64_t(cc) * nf + t) * 4;
        const uint32_t c0 = uint32_t(s), c1 = uint32_t(s >> 32), c2 = uint32_t(s >> 64);
        const int32_t c3 = int32_t(uint32_t(s >> 96));
        if (s != 0) {
          atomicAdd(limb + 0, (unsigned long long)c0);
          atomicAdd(limb + 1, (unsigned long long)c1);
          atomicAdd(limb + 2, (unsigned long long)c2);
          atomicAdd(limb + 3, (unsigned long long)(long long)c3);
        }
      }
      __syncthreads();
    }
  }
  if (t < k && s_tot[t]) atomicAdd(a.acc + K4 + t, (unsigned long long)s_tot[t]);
  if (t == 0 && delta) atomicAdd(a.acc + K4 + k, (unsigned long long)delta);
  if (inexact) atomicAdd(a.acc + K4 + k + 1, (unsigned long long)inexact);
}

// round-to-nearest-even of (S * 2^-64) / cnt, S a signed 128-bit integer
__device__ float mean_rne(__int128 S, long long cnt) {
  if (S == 0) return 0.0f;
  const bool neg = S < 0;
  u128 U = neg ? u128(0) - u128(S) : u128(S);
  int L = 0;
  {
    const unsigned long long hi = (unsigned long long)(U >> 64), lo = (unsigned long long)U;
    L = hi ? 128 - __clzll(hi) : 64 - __clzll(lo);
  }
  const int s = 127 - L;  // U << s < 2^127
  U <<= s;
  const u128 Q = U / u128(cnt);
  const bool sticky = (U % u128(cnt)) != 0;
  int lq;
  {
    const unsigned long long hi = (unsigned long long)(Q >> 64), lo = (unsigned long long)Q;
    lq = hi ? 128 - __clzll(hi) : 64 - __clzll(lo);
  }
  int drop = lq - 24;  // >= 72 here: Q has >= 95 significant bits
  u128 mant = Q >> drop;
  const u128 rem = Q & ((u128(1) << drop) - 1);
  const u128 half = u128(1) << (drop - 1);
  if (rem > half || (rem == half && (sticky || (mant & 1)))) mant += 1;
  if (mant == (u128(1) << 24)) {
    mant >>= 1;
    ++drop;
  }
  const float v = ldexpf(float(uint32_t(mant)), drop - 64 - s);
  return neg ? -v : v;
}

// ctrl (nullable): {done, iterations, last delta, inexact total}
__global__ void __launch_bounds__(1024) km_finalize_kernel(unsigned long long* acc, int k, int nf, float* clusters,
                                                           long long* stats, int zero, long long* ctrl, int max_iter,
                                                           long long max_changes) {
  if (ctrl && ctrl[0]) return;
  const int K4 = k * nf * 4, t = threadIdx.x;
  for (int q = t; q < k * nf; q += blockDim.x) {
    const int c = q / nf;
    const long long cnt = (long long)acc[K4 + c];
    if (cnt <= 0) continue;  // a centre without points keeps its value
    const unsigned long long* l = acc + int64_t(q) * 4;
    const __int128 S = __int128((long long)l[0]) + (__int128((long long)l[1]) << 32) +
                       (__int128((long long)l[2]) << 64) + (__int128((long long)l[3]) << 96);
    clusters[q] = mean_rne(S, cnt);
  }
  __syncthreads();
  if (t == 0) {
    const long long delta = (long long)acc[K4 + k], inexact = (long long)acc[K4 + k + 1];
    long long total = 0;
    for (int c = 0; c < k; ++c) total += (long long)acc[K4 + c];
    if (stats) {
      stats[0] = delta;
      stats[1] = inexact;
      stats[2] = total;
    }
    if (ctrl) {
      ctrl[1] += 1;
      ctrl[2] = delta;
      ctrl[3] += inexact;
      if (delta <= max_changes || ctrl[1] >= max_iter) ctrl[0] = 1;
    }
  }
  __syncthreads();
  if (zero)
    for (int q = t; q < K4 + k + 2; q += blockDim.x) acc[q] = 0;
}

}  // namespace catt

using namespace catt;

namespace {

struct AccLaunch {
  const void* func;
  size_t smem;
  int grid;
};

template <int KMAX, int FB>
const void* acc_fn() {
  return (const void*)km_accumulate_kernel<KMAX, FB>;
}

catt_status acc_launch(const float* feat, int64_t ld, int64_t npoints, int32_t nf, const float* clusters, int32_t k,
                       int32_t* memb, int64_t* acc, const long long* done, cudaStream_t s) {
  const int FB = nf <= 32 ? 1 : 2;
  const int KMAX = k <= 8 ? 8 : 16;
  const void* f = KMAX == 8 ? (FB == 1 ? acc_fn<8, 1>() : acc_fn<8, 2>()) : (FB == 1 ? acc_fn<16, 1>() : acc_fn<16, 2>());
  const size_t tile_bytes = std::max<size_t>(size_t(nf) * KTP * 4, size_t(8) * FB * 32 * 16);
  const size_t smem = size_t((nf * k + 3) & ~3) * 4 + tile_bytes;
  cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  DevCtx* ctx = nullptr;
  catt_status st = dev_ctx(&ctx);
  if (st != CATT_OK) return st;
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, f, KT, smem);
  if (e != cudaSuccess || per_sm < 1) {
    record_cuda_error(e == cudaSuccess ? cudaErrorInvalidConfiguration : e);
    return CATT_ECUDA;
  }
  const int64_t tiles = (npoints + KT - 1) / KT;
  const int grid = int(std::min<int64_t>(tiles, int64_t(per_sm) * ctx->hw.num_sms));
  AccArgs a{feat, clusters, memb, reinterpret_cast<unsigned long long*>(acc), done, ld, npoints, nf, k};
  void* args[] = {&a};
  e = cudaLaunchKernel(f, dim3(unsigned(grid)), dim3(KT), args, smem, s);
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  return CATT_OK;
}

bool acc_args_ok(int64_t ld, int64_t npoints, int32_t nf, int32_t k) {
  return npoints >= 0 && nf >= 1 && nf <= 64 && k >= 1 && k <= 16 && ld >= npoints && npoints < (int64_t(1) << 31);
}

}  // namespace

extern "C" int64_t catt_kmeans_acc_words(int32_t k, int32_t nf) {
  if (k < 1 || nf < 1) return 0;
  return int64_t(k) * nf * 4 + k + 2;
}

extern "C" catt_status catt_kmeans_transpose(const float* in, float* out, int64_t npoints, int32_t nf, int64_t ld,
                                             const catt_throttle* t, void* stream) {
  if (npoints < 0 || nf < 1 || ld < npoints || nf > 4096) return CATT_EINVAL;
  if (npoints > 0 && (!in || !out)) return CATT_EINVAL;
  if (npoints == 0) return CATT_OK;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  TrArgs a{in, out, npoints, ld, nf, Throttle{}};
  const int var = variant_of(t);
  if (var == CATT_VAR_LITERAL) {
    const int threads = cta_threads_or(t, 256);
    size_t dyn = 0;
    catt_status st = prepare_launch((const void*)km_transpose_thread_kernel, t, threads, 0, true, &a.t, &dyn);
    if (st != CATT_OK) return st;
    km_transpose_thread_kernel<<<dim3(unsigned((npoints + threads - 1) / threads)), threads, dyn, s>>>(a);
    return after_launch();
  }
  if (var == CATT_VAR_COOP) {
    if (t && t->cta_threads != 0 && t->cta_threads != 256) return CATT_EINVAL;
    const size_t smem = size_t(256) * size_t(nf | 1) * 4;
    if (smem > 200 * 1024) return CATT_EUNSUPPORTED;
    if (smem > 48 * 1024 &&
        cudaFuncSetAttribute((const void*)km_transpose_tile_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             int(smem)) != cudaSuccess)
      return after_launch();
    size_t dyn = 0;
    catt_status st = prepare_launch((const void*)km_transpose_tile_kernel, t, 256, smem, false, &a.t, &dyn);
    if (st != CATT_OK) return st;
    km_transpose_tile_kernel<<<dim3(unsigned((npoints + 255) / 256)), 256, dyn, s>>>(a);
    return after_launch();
  }
  return CATT_EINVAL;
}

extern "C" catt_status catt_kmeans_accumulate(const float* feat, int64_t ld, int64_t npoints, int32_t nf,
                                              const float* clusters, int32_t k, int32_t* membership, int64_t* acc,
                                              void* stream) {
  if (!acc_args_ok(ld, npoints, nf, k) || !acc) return CATT_EINVAL;
  if (npoints > 0 && (!feat || !clusters || !membership)) return CATT_EINVAL;
  if (npoints == 0) return CATT_OK;
  return acc_launch(feat, ld, npoints, nf, clusters, k, membership, acc, nullptr, static_cast<cudaStream_t>(stream));
}

extern "C" catt_status catt_kmeans_finalize(int64_t* acc, int32_t k, int32_t nf, float* clusters, int64_t* stats,
                                            int32_t zero_acc, void* stream) {
  if (!acc || !clusters || k < 1 || nf < 1 || k > 16 || nf > 64) return CATT_EINVAL;
  km_finalize_kernel<<<1, 1024, 0, static_cast<cudaStream_t>(stream)>>>(
      reinterpret_cast<unsigned long long*>(acc), k, nf, clusters, reinterpret_cast<long long*>(stats), zero_acc,
      nullptr, 0, 0);
  return after_launch();
}

extern "C" catt_status catt_kmeans(const float* feat, int64_t ld, int64_t npoints, int32_t nf, float* clusters,
                                   int32_t k, int32_t* membership, int32_t max_iter, int64_t max_changes, int64_t* ws,
                                   int32_t* iterations, void* stream) {
  if (!acc_args_ok(ld, npoints, nf, k) || !ws || !clusters || !membership || max_iter < 1 || max_changes < 0)
    return CATT_EINVAL;
  if (npoints > 0 && !feat) return CATT_EINVAL;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  const int64_t W = catt_kmeans_acc_words(k, nf);
  long long* ctrl = reinterpret_cast<long long*>(ws + W);
  cudaError_t e = cudaMemsetAsync(ws, 0, size_t(W + 4) * 8, s);
  if (e == cudaSuccess && npoints > 0) e = cudaMemsetAsync(membership, 0xff, size_t(npoints) * 4, s);  // -1
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  long long host_ctrl[4] = {0, 0, 0, 0};
  constexpr int kBatch = 4;  // iterations queued between host checks of the device-side done flag
  for (int it = 0; it < max_iter; it += kBatch) {
    for (int j = 0; j < kBatch && it + j < max_iter; ++j) {
      if (npoints > 0) {
        catt_status st = acc_launch(feat, ld, npoints, nf, clusters, k, membership, ws, ctrl, s);
        if (st != CATT_OK) return st;
      }
      km_finalize_kernel<<<1, 1024, 0, s>>>(reinterpret_cast<unsigned long long*>(ws), k, nf, clusters, nullptr, 1,
                                            ctrl, max_iter, max_changes);
      if (after_launch() != CATT_OK) return CATT_ECUDA;
    }
    e = cudaMemcpyAsync(host_ctrl, ctrl, sizeof(host_ctrl), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) {
      record_cuda_error(e);
      return CATT_ECUDA;
    }
    if (host_ctrl[0]) break;
  }
  if (iterations) *iterations = int32_t(host_ctrl[1]);
  return host_ctrl[3] ? CATT_EINEXACT : CATT_OK;
}
