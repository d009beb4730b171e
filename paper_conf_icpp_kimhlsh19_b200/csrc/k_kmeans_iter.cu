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
#include <cstdlib>
#include <cstring>

#include "f32x2.cuh"
#include "internal.h"
#include "tma.cuh"

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

// PTX shifts clamp amounts >= 64 (as unsigned) to 64: the result is 0. That
// makes the conversion below branch-free.
__device__ __forceinline__ uint64_t shl64(uint64_t x, uint32_t n) {
  uint64_t r;
  asm("shl.b64 %0, %1, %2;" : "=l"(r) : "l"(x), "r"(n));
  return r;
}
__device__ __forceinline__ uint64_t shr64(uint64_t x, uint32_t n) {
  uint64_t r;
  asm("shr.b64 %0, %1, %2;" : "=l"(r) : "l"(x), "r"(n));
  return r;
}

// x * 2^64 as a two's-complement 128-bit integer. Exact for x = 0 and for
// 2^-64 <= ulp(x), |x| < 2^31; anything else (non-zero bits below 2^-64,
// |x| >= 2^31, subnormal, inf, NaN) counts in `inexact` (and converts to
// the truncated value, or 0 when |x| >= 2^31).
__device__ __forceinline__ u128 to_fixed(float x, int& inexact) {
  const uint32_t b = __float_as_uint(x);
  const uint32_t e = (b >> 23) & 0xffu, mant = b & 0x7fffffu;
  const bool big = e >= 158u;
  const uint64_t m = (e == 0u || big) ? 0ull : uint64_t(mant | 0x800000u);
  const uint32_t sh = e - 86u;  // x * 2^64 = m * 2^(e-86); "negative" values wrap to huge amounts
  const uint64_t lo = shl64(m, sh) | shr64(m, 0u - sh);
  const uint64_t hi = shr64(m, 64u - sh) | shl64(m, sh - 64u);
  const uint64_t lost = shl64(m, 64u + sh);  // the bits shifted out when e < 86 (0 otherwise)
  inexact += int(big | (e == 0u && mant != 0u) | (e != 0u && e < 63u) | (lost != 0ull));
  const uint64_t neg = 0ull - uint64_t(b >> 31);  // all ones for negative x
  const u128 u = (u128(hi ^ neg) << 64) | u128(lo ^ neg);
  return u + u128(neg & 1ull);  // ones' complement + 1 = two's complement negation
}

// An fp64 value that is a multiple of 2^-64 with |s| < 2^63, as the
// two's-complement 128-bit integer s * 2^64 (exact).
__device__ __forceinline__ u128 d_to_fixed(double s) {
  const uint64_t b = uint64_t(__double_as_longlong(s));
  const uint32_t e = uint32_t(b >> 52) & 0x7ffu;
  const uint64_t m = e ? ((b & 0xfffffffffffffull) | 0x10000000000000ull) : 0ull;
  const uint32_t sh = e - 1011u;  // s * 2^64 = m * 2^(e - 1075 + 64)
  const uint64_t lo = shl64(m, sh) | shr64(m, 0u - sh);
  const uint64_t hi = shr64(m, 64u - sh) | shl64(m, sh - 64u);
  const uint64_t neg = 0ull - (b >> 63);
  const u128 u = (u128(hi ^ neg) << 64) | u128(lo ^ neg);
  return u + u128(neg & 1ull);
}

// Exact sum of row[idx[i]], i in [lo, hi), as a 128-bit fixed-point value.
// Fast path: the values are summed in fp64 and the sum is provably exact when
// every value is a multiple of u = 2^(emin-150) (emin = smallest exponent
// field of the non-zero values) and sum |x| <= 2^52 u: every partial sum is
// then an integer multiple of u below 2^53 u. u >= 2^-64 and |x| < 2^31 keep
// the result inside the fixed-point contract. Otherwise: value by value.
__device__ __forceinline__ u128 segment_sum(const float* __restrict__ row, const unsigned short* __restrict__ idx,
                                            int lo, int hi, int& inexact) {
  double sum = 0.0, bnd = 0.0;
  uint32_t amin = 0xffffffffu;  // min over non-zero x of |x|'s bits - 1 (zeros wrap to the max)
  for (int i = lo; i < hi; ++i) {
    const float x = row[idx[i]];
    amin = min(amin, (__float_as_uint(x) & 0x7fffffffu) - 1u);
    const double xd = double(x);
    sum += xd;
    bnd += fabs(xd);
  }
  const int emin = amin == 0xffffffffu ? 255 : int((amin + 1u) >> 23);
  // bnd < 2^31 bounds every |x| (and rejects inf/NaN); emin >= 86: u >= 2^-64
  if (emin >= 86 && bnd < 2147483648.0 && bnd <= ldexp(1.0, emin - 98)) return d_to_fixed(sum);
  u128 v = 0;
  for (int i = lo; i < hi; ++i) v += to_fixed(row[idx[i]], inexact);
  return v;
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
  // fused finalize (catt_kmeans_step, the single-GPU loop): the last CTA to
  // finish rounds the new centres; fin_ctr = nullptr: accumulate only
  unsigned* fin_ctr;
  float* clusters_out;
  long long* stats;
  long long* ctrl;
  int max_iter;
  long long max_changes;
  int fence_all;  // every thread fences before the arrival (CATT_KM_FENCE_ALL; the earlier form)
};

__device__ void finalize_body(unsigned long long* acc, int k, int nf, float* clusters, long long* stats, int zero,
                              long long* ctrl, int max_iter, long long max_changes);

// Dynamic shared memory: {mbarrier | centres [nf][KP] | TMA stage [nf][256]
// (TMA only) | tile [nf][KTP] | 128-bit accumulators}.
struct AccSmem {
  int ct, stage, tile, acc, total;
  __host__ __device__ AccSmem(int nf, int k, int KP, int FB, bool tma) {
    ct = 128;
    stage = ((ct + nf * KP * 4 + 127) / 128) * 128;
    tile = stage + (tma ? nf * KT * 4 : 0);
    acc = ((tile + nf * KTP * 4 + 15) / 16) * 16;
    total = acc + (KT / 32) * FB * k * 32 * 16;
  }
};

// TMA = true: the tile {256 points x nf} arrives by one 2-D tensor copy into
// the stage while the previous tile's sort and phase 2 run (map over feat:
// dims {npoints, nf}, row stride ld*4 bytes; out-of-range points read 0).
template <int KMAX, int FB, bool TMA>
__global__ void __launch_bounds__(KT, 2) km_accumulate_kernel(const __grid_constant__ CUtensorMap map, AccArgs a) {
  if (a.done && *a.done) return;
  extern __shared__ __align__(128) unsigned char dyn[];
  const int nf = a.nf, k = a.k;
  constexpr int KP = (KMAX + 3) & ~3;                                   // centre pitch (float4 reads)
  const AccSmem L(nf, k, KP, FB, TMA);
  uint64_t* full = reinterpret_cast<uint64_t*>(dyn);
  float* s_ct = reinterpret_cast<float*>(dyn + L.ct);                  // [nf][KP], padding = +inf
  float* stage = reinterpret_cast<float*>(dyn + L.stage);              // [nf][256] (TMA)
  float* tile = reinterpret_cast<float*>(dyn + L.tile);                // [nf][KTP]
  __shared__ int s_cnt[KMAX], s_start[KMAX + 1], s_tot[KMAX];
  __shared__ unsigned short s_idx[KT];
  __shared__ unsigned char s_cid[KT];                                    // centre of each sorted entry
  const int t = threadIdx.x, lane = t & 31, w = t >> 5;
  // a padded centre at +inf is never strictly nearer than FLT_MAX: same decisions
  for (int q = t; q < nf * KP; q += KT) {
    const int f = q / KP, cc = q - f * KP;
    s_ct[q] = cc < k ? a.clusters[cc * nf + f] : __int_as_float(0x7f800000);
  }
  if (t < KMAX) s_tot[t] = 0;
  long long delta = 0;
  int inexact = 0;
  // per-lane private 128-bit accumulators: s_acc[((w*FB + g)*k + c)*32 + lane]
  u128* s_acc = reinterpret_cast<u128*>(dyn + L.acc);
  for (int q = t; q < (KT / 32) * FB * k * 32; q += KT) s_acc[q] = 0;

  const int64_t ntiles = (a.npoints + KT - 1) / KT;
  const uint32_t tile_bytes = uint32_t(nf) * KT * 4u;
  if (TMA && t == 0) {
    bar_init(full, 1);
    fence_barrier_init();
    if (int64_t(blockIdx.x) < ntiles) {
      bar_expect_tx(full, tile_bytes);
      tma_2d(stage, &map, int32_t(blockIdx.x) * KT, 0, full);
    }
  }
  uint32_t parity = 0;
  for (int64_t tl = blockIdx.x; tl < ntiles; tl += gridDim.x) {
    if (t < KMAX) s_cnt[t] = 0;
    const int64_t p = tl * KT + t;
    const int old = p < a.npoints ? a.memb[p] : -1;
    __syncthreads();  // s_ct / barrier ready; the previous tile's phase 2 is done with `tile`
    if (TMA) {
      bar_wait(full, parity);
      parity ^= 1u;
    }
    int c = -1, rank = 0, changed = 0;
    if (p < a.npoints) {
      const float* f0 = a.feat + p;
      // partial distances as packed pairs of centres (d[2p], d[2p+1]): one
      // FADD2 + one FFMA2 per pair, the point's value broadcast; each half is
      // the scalar IEEE operation (same order, bit-identical decisions)
      constexpr int KH = (KMAX + 1) / 2;
      uint64_t dp[KH];
#pragma unroll
      for (int h = 0; h < KH; ++h) dp[h] = 0ull;
      auto feature = [&](int f, float v) {
        tile[f * KTP + t] = v;
        const float4* cf = reinterpret_cast<const float4*>(s_ct + f * KP);
        const uint64_t vv = f2_pack(v, v);
#pragma unroll
        for (int q = 0; q < KP / 4; ++q) {
          const float4 c4 = cf[q];
#pragma unroll
          for (int j = 0; j < 4; j += 2)
            if (4 * q + j < KMAX) {
              const uint64_t e = f2_sub(vv, j == 0 ? f2_pack(c4.x, c4.y) : f2_pack(c4.z, c4.w));
              dp[(4 * q + j) / 2] = f2_fma(e, e, dp[(4 * q + j) / 2]);
            }
        }
      };
      int f = 0;
      if (TMA) {
#pragma unroll 8
        for (; f < nf; ++f) feature(f, stage[f * KT + t]);
      }
      for (; f + 32 <= nf; f += 32) {  // 32 loads in flight per thread
        float v[32];
#pragma unroll
        for (int u = 0; u < 32; ++u)
          asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v[u]) : "l"(f0 + int64_t(f + u) * a.ld));
#pragma unroll
        for (int u = 0; u < 32; ++u) feature(f + u, v[u]);
      }
      for (; f < nf; f += 8) {
        float v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u)
          if (f + u < nf)
            asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v[u]) : "l"(f0 + int64_t(f + u) * a.ld));
#pragma unroll
        for (int u = 0; u < 8; ++u)
          if (f + u < nf) feature(f + u, v[u]);
      }
      float best = FLT_MAX;
#pragma unroll
      for (int cc = 0; cc < KMAX; ++cc) {
        const float dc = (cc & 1) ? f2_hi(dp[cc / 2]) : f2_lo(dp[cc / 2]);
        if (dc < best) {
          best = dc;
          c = cc;
        }
      }
      changed = old != c;  // c = -1: every distance NaN or >= FLT_MAX (as catt_kmeans_assign)
      a.memb[p] = c;
      if (c >= 0) rank = atomicAdd(&s_cnt[c], 1);
    }
    const int nchg = __syncthreads_count(changed);  // every thread is done with the stage
    if (TMA && t == 0 && tl + gridDim.x < ntiles) {  // prefetch the next tile during sort + phase 2
      bar_expect_tx(full, tile_bytes);
      tma_2d(stage, &map, int32_t((tl + gridDim.x) * KT), 0, full);
    }
    if (t == 0) {
      delta += nchg;
      s_start[0] = 0;
      for (int cc = 0; cc < k; ++cc) {
        s_start[cc + 1] = s_start[cc] + s_cnt[cc];
        s_tot[cc] += s_cnt[cc];
      }
    }
    __syncthreads();
    if (c >= 0) {
      s_idx[s_start[c] + rank] = static_cast<unsigned short>(t);
      s_cid[s_start[c] + rank] = static_cast<unsigned char>(c);
    }
    __syncthreads();
    // phase 2: warp w owns sorted entries [32w, 32w + 32). Group g holds
    // features [32g, 32g + 32); a group with fg < 32 features (the last one)
    // spreads its lanes as fg features x (32/fg) sub-chunks of fg entries.
    // The centres met by a lane's range are consecutive in the sorted order
    // (s_cid of its first and last entry bound them).
#pragma unroll
    for (int g = 0; g < FB; ++g) {
      const int rem = nf - 32 * g;
      if (rem > 0) {
        const int fg = rem >= 32 ? 32 : (rem > 16 ? 32 : rem > 8 ? 16 : rem > 4 ? 8 : rem > 2 ? 4 : rem);
        const int fl = lane & (fg - 1), h = lane / fg;
        const int s_lo = w * 32 + h * fg, s_hi = s_lo + fg;
        const bool fok = fl < rem;
        const float* row = tile + (32 * g + fl) * KTP;
        u128* mine = s_acc + (w * FB + g) * k * 32 + lane;
        // only the centres whose segments meet [s_lo, s_hi) (usually one or two)
        const int e1 = min(s_hi, s_start[k]);
        const int c0 = s_lo < e1 ? int(s_cid[s_lo]) : k, c1 = s_lo < e1 ? int(s_cid[e1 - 1]) : -1;
        for (int cc = c0; cc <= c1; ++cc) {
          const int lo = max(s_start[cc], s_lo), hi = fok ? min(s_start[cc + 1], s_hi) : lo;
          if (lo < hi) mine[cc * 32] += segment_sum(row, s_idx, lo, hi, inexact);
        }
      }
    }
  }
  __syncthreads();
  // epilogue: per (centre, feature) the CTA's lanes summed exactly, then the
  // four 32-bit chunks of the 128-bit sum added into the int64 limbs
  const int K4 = k * nf * 4;
  for (int q = t; q < k * nf; q += KT) {
    const int cc = q / nf, f = q - cc * nf;
    const int g = f >> 5, fl = f & 31, rem = nf - 32 * g;
    const int fg = rem >= 32 ? 32 : (rem > 16 ? 32 : rem > 8 ? 16 : rem > 4 ? 8 : rem > 2 ? 4 : rem);
    u128 s = 0;
    for (int ww = 0; ww < KT / 32; ++ww)
      for (int l = fl; l < 32; l += fg) s += s_acc[((ww * FB + g) * k + cc) * 32 + l];
    if (s != 0) {
      // only the non-zero chunks: the 296 CTAs add into the same k * nf * 4
      // words at the end, so every atomic saved shortens the contended tail
      // (values in [2^-9, 1) leave chunk 0 and chunk 3 zero)
      unsigned long long* limb = a.acc + int64_t(q) * 4;
      const uint32_t c0 = uint32_t(s), c1 = uint32_t(s >> 32), c2 = uint32_t(s >> 64), c3 = uint32_t(s >> 96);
      if (c0) atomicAdd(limb + 0, (unsigned long long)c0);
      if (c1) atomicAdd(limb + 1, (unsigned long long)c1);
      if (c2) atomicAdd(limb + 2, (unsigned long long)c2);
      if (c3) atomicAdd(limb + 3, (unsigned long long)(long long)int32_t(c3));
    }
  }
  if (t < k && s_tot[t]) atomicAdd(a.acc + K4 + t, (unsigned long long)s_tot[t]);
  if (t == 0 && delta) atomicAdd(a.acc + K4 + k, (unsigned long long)delta);
  if (inexact) atomicAdd(a.acc + K4 + k + 1, (unsigned long long)inexact);
  if (a.fin_ctr) {
    // last-CTA finalize: this CTA's sums are published before its arrival
    // (the barrier orders every thread's atomics before thread 0's fence and
    // acq_rel arrival, the cooperative-groups grid-sync pattern); the CTA
    // that arrives last sees every CTA's sums (acq_rel)
    __shared__ int s_last;
    if (a.fence_all) __threadfence();
    __syncthreads();
    if (t == 0) {
      __threadfence();
      unsigned prev;
      asm volatile("atom.add.acq_rel.gpu.u32 %0, [%1], 1;" : "=r"(prev) : "l"(a.fin_ctr) : "memory");
      s_last = prev == gridDim.x - 1;
    }
    __syncthreads();
    if (s_last) {
      __threadfence();
      finalize_body(a.acc, k, nf, a.clusters_out, a.stats, 1, a.ctrl, a.max_iter, a.max_changes);
      if (t == 0) *a.fin_ctr = 0u;                               // ready for the next launch
    }
  }
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
  finalize_body(acc, k, nf, clusters, stats, zero, ctrl, max_iter, max_changes);
}

// the finalize of one CTA (any block size): new centres, stats, loop control, zeroing
__device__ void finalize_body(unsigned long long* acc, int k, int nf, float* clusters, long long* stats, int zero,
                              long long* ctrl, int max_iter, long long max_changes) {
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

template <int KMAX, int FB, bool TMA>
const void* acc_fn() {
  return (const void*)km_accumulate_kernel<KMAX, FB, TMA>;
}

struct FinArgs {
  float* clusters;
  long long* stats;
  long long* ctrl;
  int max_iter;
  long long max_changes;
};

catt_status acc_launch(const float* feat, int64_t ld, int64_t npoints, int32_t nf, const float* clusters, int32_t k,
                       int32_t* memb, int64_t* acc, const long long* done, cudaStream_t s,
                       const FinArgs* fin = nullptr) {
  // TMA needs a 16-B aligned base and a row stride that is a multiple of 16 B;
  // otherwise the general form (per-thread loads, centres padded to 16)
  const bool tma = (reinterpret_cast<uintptr_t>(feat) & 15u) == 0 && ld % 4 == 0 && encode_fn() != nullptr;
  const int FB = nf <= 32 ? 1 : 2;
  const int KMAX = !tma ? 16 : k <= 4 ? 4 : k == 5 ? 5 : k <= 8 ? 8 : 16;
  const int FBx = tma ? FB : 2;
  const void* f = nullptr;
  switch (KMAX * 4 + FBx) {
    case 17: f = acc_fn<4, 1, true>(); break;
    case 18: f = acc_fn<4, 2, true>(); break;
    case 21: f = acc_fn<5, 1, true>(); break;
    case 22: f = acc_fn<5, 2, true>(); break;
    case 33: f = acc_fn<8, 1, true>(); break;
    case 34: f = acc_fn<8, 2, true>(); break;
    case 65: f = acc_fn<16, 1, true>(); break;
    default: f = tma ? acc_fn<16, 2, true>() : acc_fn<16, 2, false>(); break;
  }
  const AccSmem L(nf, k, (KMAX + 3) & ~3, FBx, tma);
  const size_t smem = size_t(L.total);
  CUtensorMap map;
  memset(&map, 0, sizeof(map));
  if (tma) {
    const cuuint64_t dims[2] = {cuuint64_t(npoints), cuuint64_t(nf)};
    const cuuint64_t strides[1] = {cuuint64_t(ld) * 4};
    const cuuint32_t box[2] = {cuuint32_t(KT), cuuint32_t(nf)};
    const cuuint32_t es[2] = {1, 1};
    if (encode_fn()(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(feat), dims, strides, box, es,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
      return CATT_EINVAL;
  }
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
  AccArgs a{feat, clusters, memb, reinterpret_cast<unsigned long long*>(acc), done, ld, npoints, nf, k,
            nullptr, nullptr, nullptr, nullptr, 0, 0, getenv("CATT_KM_FENCE_ALL") != nullptr};
  if (fin) {
    // the arrival counter is the last word of the caller's acc (catt.h), so
    // steps on different acc arrays never share it
    a.fin_ctr = reinterpret_cast<unsigned*>(acc + catt_kmeans_acc_words(k, nf) - 1);
    a.clusters_out = fin->clusters;
    a.stats = fin->stats;
    a.ctrl = fin->ctrl;
    a.max_iter = fin->max_iter;
    a.max_changes = fin->max_changes;
  }
  void* args[] = {&map, &a};
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
  return int64_t(k) * nf * 4 + k + 3;
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

extern "C" catt_status catt_kmeans_step(const float* feat, int64_t ld, int64_t npoints, int32_t nf, float* clusters,
                                        int32_t k, int32_t* membership, int64_t* acc, int64_t* stats, void* stream) {
  if (!acc_args_ok(ld, npoints, nf, k) || !acc || !clusters) return CATT_EINVAL;
  if (npoints > 0 && (!feat || !membership)) return CATT_EINVAL;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (npoints == 0) {
    km_finalize_kernel<<<1, 1024, 0, s>>>(reinterpret_cast<unsigned long long*>(acc), k, nf, clusters,
                                          reinterpret_cast<long long*>(stats), 1, nullptr, 0, 0);
    return after_launch();
  }
  FinArgs fin{clusters, reinterpret_cast<long long*>(stats), nullptr, 0, 0};
  return acc_launch(feat, ld, npoints, nf, clusters, k, membership, acc, nullptr, s, &fin);
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
      if (npoints > 0) {                                           // one launch per iteration
        FinArgs fin{clusters, nullptr, ctrl, max_iter, max_changes};
        catt_status st = acc_launch(feat, ld, npoints, nf, clusters, k, membership, ws, ctrl, s, &fin);
        if (st != CATT_OK) return st;
      } else {
        km_finalize_kernel<<<1, 1024, 0, s>>>(reinterpret_cast<unsigned long long*>(ws), k, nf, clusters, nullptr, 1,
                                              ctrl, max_iter, max_changes);
        if (after_launch() != CATT_OK) return CATT_ECUDA;
      }
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
