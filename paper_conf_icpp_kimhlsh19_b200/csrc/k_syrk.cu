// k_syrk.cu — SYRK, C = beta*C + alpha*A*A^T over the full n x n square
// (PolyBench/GPU syrk, Table 2; the 2-D thread-block case of P:246).
//
// LITERAL: block 32 x BY, thread (i = by*BY + ty, j = bx*32 + tx):
//     c = C[i][j] * beta;  for k < m: c = fmaf(alpha * a[i][k], a[j][k], c)
// a[j][k] is memory-divergent across the warp (32 rows of A) and reused for
// 32 consecutive k; a[i][k] is a broadcast. CATT throttles this loop.
// STAGED: 128 x 128 output tiles in shared memory (alpha*a_i pre-multiplied
// with the same rounding), 8 x 8 outputs per thread held in registers; every
// output still accumulates k = 0, 1, ..., m-1 in order, so the result is
// bit-identical to LITERAL. FP32 CUDA-core bound (no tensor cores: TF32 would
// break the 1e-5 bar, BASELINE north_star). SYR2K (below) shares the tiled
// kernel; its literal kernel is the paper's 2-D CS loop.
#include <algorithm>
#include <cstdlib>
#include <mutex>
#include <cstdint>

#include "f32x2.cuh"
#include "internal.h"
#include "tma.cuh"

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

// ---------------------------------------------------------------- SYR2K
// PolyBench/GPU syr2k (Table 2; Table 3): the paper's 2-D CS
// kernel. Per element, k ascending, with the evaluation order of R20:
//   p = alpha*a[i][k], q = alpha*b[i][k], s = fmaf(p, b[j][k], q*a[j][k]), c = c + s.
struct Syr2kArgs {
  const float* A;
  const float* B;
  float* C;
  int64_t n, m;
  float alpha, beta;
  Throttle t;
};

__global__ void __launch_bounds__(1024, 2) syr2k_thread_kernel(Syr2kArgs a) {
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
    const float* __restrict__ bi = a.B + i * m;
    const float* __restrict__ aj = a.A + j * m;
    const float* __restrict__ bj = a.B + j * m;
    float c = __fmul_rn(a.C[i * a.n + j], a.beta);
#pragma unroll 2
    for (int64_t k = 0; k < m; ++k) {
      const float p = __fmul_rn(a.alpha, ai[k]);
      const float q = __fmul_rn(a.alpha, bi[k]);
      const float s = fmaf(p, bj[k], __fmul_rn(q, aj[k]));
      c = __fadd_rn(c, s);
    }
    a.C[i * a.n + j] = c;
  });
  cta_exit(a.t);
}

// ---------------------------------------------------------------- tiled
// STAGED SYRK / SYR2K: 128 x 128 output tile per 256-thread CTA, 8 x 8 outputs
// per thread on rows {ty*4 + r, 64 + ty*4 + r} x cols {tx*4 + q, 64 + tx*4 + q}
// (conflict-free float4 fragment reads), BK k per shared-memory stage, double-
// buffered stages and double-buffered register fragments. Every output runs
// k = 0, 1, ..., m-1 in order with the literal kernel's per-step rounding, so
// the result is bit-identical to LITERAL (and to the oracle). Stage arrays:
//   SYRK : 0 = alpha*a[i][k], 1 = a[j][k]
//   SYR2K: 0 = alpha*a[i][k], 1 = b[j][k], 2 = alpha*b[i][k], 3 = a[j][k]
//   GEMM : 0 = alpha*a[i][k], 1 = b[k][j] (B is k-major: loaded without a transpose)
// C is ni x nj (SYRK/SYR2K: ni = nj = n), the inner size is m.
constexpr int MODE_SYRK = 0, MODE_SYR2K = 1, MODE_GEMM = 2;
// TM x TM outputs per thread, 16 x 16 threads: TM = 8 -> 128 x 128 tiles,
// TM = 4 -> 64 x 64 tiles (SYRK and GEMM only), for grids that would leave
// most SMs idle with the large tile.

struct TileArgs {
  const float* A;
  const float* B;  // SYR2K, GEMM
  float* C;
  int64_t ni, nj, m;
  float alpha, beta;
  int vec;  // m % 4 == 0 and A (SYR2K: and B) 16-B aligned: float4 loads along k
  int bvec; // GEMM: nj % 4 == 0 and B 16-B aligned: float4 loads of B rows
  int cvec; // nj % 4 == 0 and C 16-B aligned
  int tri;  // SYRK only: compute the tiles on and above the diagonal (C symmetric; caller mirrors)
  Throttle t;
  int zinit = 0;              // T2: accumulators start at +0 without reading C (CORR's s = 0)
  int mirror = 0;             // T2, tri: write C[i][j] and C[j][i] for j > i, C[i][i] = 1 (CORR's symmat)
  const float* kmaj = nullptr;  // T2, SYRK with alpha = 1: A^T given (k-major, pitch kld): no prep
  int64_t kld = 0;
};

template <int MODE, int TM, bool LEAN = false, bool DEEP = false>
struct TileCfg {
  static constexpr int BM = 16 * TM;            // tile edge
  static constexpr int H = TM / 4;              // float4 groups per thread per dimension
  static constexpr int GS = BM / H;             // group stride: rows {g*GS + 4t + r}
  static constexpr int PITCH = BM + 4;          // transposed stage rows: 16-B aligned, store banks spread
  // DEEP: BK = 32 (SYR2K: 16) in dynamic shared memory, half the stage
  // barriers and global-load phases per k
  static constexpr int BK = DEEP ? ((MODE == MODE_SYR2K) ? 16 : 32) : (MODE == MODE_SYR2K || LEAN) ? 8 : 16;
  static constexpr size_t SBYTES = size_t(2) * (MODE == MODE_SYR2K ? 4 : 2) * BK * PITCH * 4;
  static constexpr int FBUF = LEAN ? 1 : 2;     // register fragments: double-buffered unless LEAN
  static constexpr int NA = MODE == MODE_SYR2K ? 4 : 2;
  static constexpr int KQ = BK / 4;             // float4 per stage row
  static constexpr int NV = BM * KQ / 256;      // float4 per thread per array per stage
  static_assert(NV >= 1, "tile too small for the stage depth");
};

// LEAN: BK = 8 and single-buffered fragments (fewer registers: 2 CTAs per SM)
template <int MODE, int MINB, int TM = 8, bool LEAN = false, bool DEEP = false>
__global__ void __launch_bounds__(256, MINB) tiled_kernel(TileArgs a) {
  constexpr bool TWO = MODE == MODE_SYR2K, GEMM = MODE == MODE_GEMM;
  using Cfg = TileCfg<MODE, TM, LEAN, DEEP>;
  constexpr int BK = Cfg::BK, NA = Cfg::NA, KQ = Cfg::KQ, NV = Cfg::NV, BM = Cfg::BM, H = Cfg::H, GS = Cfg::GS;
  constexpr int PITCH = Cfg::PITCH;
  auto tile_off = [](int t, int r) { return (r / 4) * GS + t * 4 + (r % 4); };
  float (*S)[NA][BK][PITCH];
  if constexpr (DEEP) {
    extern __shared__ __align__(16) float tiled_dyn[];
    S = reinterpret_cast<float (*)[NA][BK][PITCH]>(tiled_dyn);
  } else {
    __shared__ __align__(16) float S_st[2][NA][BK][PITCH];
    S = S_st;
  }
  if (a.tri && blockIdx.x < blockIdx.y) return;  // strictly below the diagonal: mirrored by the caller
  cta_enter(a.t);
  const int tid = threadIdx.x;
  const int tx = tid & 15, ty = tid >> 4;
  const int64_t i0 = int64_t(blockIdx.y) * BM, j0 = int64_t(blockIdx.x) * BM;
  const int64_t ni = a.ni, nj = a.nj, m = a.m;

  float c[TM][TM];
#pragma unroll
  for (int r = 0; r < TM; ++r) {
    const int64_t gi = i0 + tile_off(ty, r);
#pragma unroll
    for (int h = 0; h < H; ++h) {
      const int64_t gj = j0 + GS * h + tx * 4;
      if (a.cvec && gi < ni && gj + 3 < nj) {
        const float4 v = *reinterpret_cast<const float4*>(a.C + gi * nj + gj);
        c[r][4 * h] = __fmul_rn(v.x, a.beta);
        c[r][4 * h + 1] = __fmul_rn(v.y, a.beta);
        c[r][4 * h + 2] = __fmul_rn(v.z, a.beta);
        c[r][4 * h + 3] = __fmul_rn(v.w, a.beta);
      } else {
#pragma unroll
        for (int q = 0; q < 4; ++q)
          c[r][4 * h + q] = (gi < ni && gj + q < nj) ? __fmul_rn(a.C[gi * nj + gj + q], a.beta) : 0.0f;
      }
    }
  }

  // stage array s: source matrix, whether its row is the output row i (and
  // pre-scaled by alpha) or the output column j
  auto src = [&](int s) -> const float* { return (s == 0 || s == 3 || (!TWO && s == 1)) ? a.A : a.B; };
  auto is_row = [](int s) { return s == 0 || s == 2; };
  float4 ld[NA][NV];
  auto gload = [&](int64_t k0) {
#pragma unroll
    for (int v = 0; v < NV; ++v) {
      const int idx = tid + v * 256;
      const int row = idx / KQ;
      const int64_t k = k0 + (idx % KQ) * 4;
#pragma unroll
      for (int s = 0; s < NA; ++s) {
        if (GEMM && s == 1) {  // B rows k0 + kk, columns j0 + 4*c4 .. +3
          const int kk = idx / (BM / 4), c4 = idx % (BM / 4);
          const int64_t kb = k0 + kk, jb = j0 + 4 * c4;
          const float* Bp = a.B + kb * nj + jb;
          if (a.bvec && kb < m && jb + 3 < nj) {
            ld[1][v] = __ldg(reinterpret_cast<const float4*>(Bp));
          } else {
            const bool ok = kb < m;
            ld[1][v].x = (ok && jb < nj) ? Bp[0] : 0.0f;
            ld[1][v].y = (ok && jb + 1 < nj) ? Bp[1] : 0.0f;
            ld[1][v].z = (ok && jb + 2 < nj) ? Bp[2] : 0.0f;
            ld[1][v].w = (ok && jb + 3 < nj) ? Bp[3] : 0.0f;
          }
          continue;
        }
        const int64_t g = (is_row(s) ? i0 : j0) + row;
        const int64_t gl = is_row(s) ? ni : nj;
        const float* M = src(s);
        if (a.vec && g < gl && k + 3 < m) {
          ld[s][v] = __ldg(reinterpret_cast<const float4*>(M + g * m + k));
        } else {
          const bool ok = g < gl;
          ld[s][v].x = (ok && k < m) ? M[g * m + k] : 0.0f;
          ld[s][v].y = (ok && k + 1 < m) ? M[g * m + k + 1] : 0.0f;
          ld[s][v].z = (ok && k + 2 < m) ? M[g * m + k + 2] : 0.0f;
          ld[s][v].w = (ok && k + 3 < m) ? M[g * m + k + 3] : 0.0f;
        }
      }
    }
  };
  auto sstore = [&](int buf) {
#pragma unroll
    for (int v = 0; v < NV; ++v) {
      const int idx = tid + v * 256;
      const int row = idx / KQ, kq = (idx % KQ) * 4;
#pragma unroll
      for (int s = 0; s < NA; ++s) {
        float4 x = ld[s][v];
        if (GEMM && s == 1) {
          *reinterpret_cast<float4*>(&S[buf][1][idx / (BM / 4)][4 * (idx % (BM / 4))]) = x;
          continue;
        }
        if (is_row(s)) {
          x.x = __fmul_rn(a.alpha, x.x);
          x.y = __fmul_rn(a.alpha, x.y);
          x.z = __fmul_rn(a.alpha, x.z);
          x.w = __fmul_rn(a.alpha, x.w);
        }
        S[buf][s][kq][row] = x.x;
        S[buf][s][kq + 1][row] = x.y;
        S[buf][s][kq + 2][row] = x.z;
        S[buf][s][kq + 3][row] = x.w;
      }
    }
  };
  float f[Cfg::FBUF][NA][TM];
  auto fload = [&](int fb, int buf, int kk) {
#pragma unroll
    for (int s = 0; s < NA; ++s) {
      const int t = is_row(s) ? ty : tx;
#pragma unroll
      for (int h = 0; h < H; ++h) {
        const float4 v = *reinterpret_cast<const float4*>(&S[buf][s][kk][GS * h + t * 4]);
        f[fb][s][4 * h] = v.x;
        f[fb][s][4 * h + 1] = v.y;
        f[fb][s][4 * h + 2] = v.z;
        f[fb][s][4 * h + 3] = v.w;
      }
    }
  };
  // the accumulators as packed pairs (c[r][2p], c[r][2p+1]): one FFMA2 (SYR2K:
  // FMUL2 + FFMA2 + FADD2) advances two outputs; the row operand is a
  // broadcast (ptxas folds it into the .F32 operand form), and each half is
  // the scalar IEEE operation, so the result stays bit-identical
  uint64_t cp[TM][TM / 2];
#pragma unroll
  for (int r = 0; r < TM; ++r)
#pragma unroll
    for (int p = 0; p < TM / 2; ++p) cp[r][p] = f2_pack(c[r][2 * p], c[r][2 * p + 1]);
  auto fma_step = [&](int fb) {
#pragma unroll
    for (int r = 0; r < TM; ++r) {
      const uint64_t ar = f2_pack(f[fb][0][r], f[fb][0][r]);
#pragma unroll
      for (int p = 0; p < TM / 2; ++p) {
        const uint64_t bq = f2_pack(f[fb][1][2 * p], f[fb][1][2 * p + 1]);
        if constexpr (TWO) {
          const uint64_t pr = f2_mul(f2_pack(f[fb][2][r], f[fb][2][r]), f2_pack(f[fb][3][2 * p], f[fb][3][2 * p + 1]));
          cp[r][p] = f2_add(cp[r][p], f2_fma(ar, bq, pr));
        } else {
          cp[r][p] = f2_fma(ar, bq, cp[r][p]);
        }
      }
    }
  };

  const int64_t ktiles = (m + BK - 1) / BK;
  if (ktiles > 0) {
    gload(0);
    sstore(0);
    __syncthreads();
    fload(0, 0, 0);
  }
  for (int64_t kt = 0; kt < ktiles; ++kt) {
    const int buf = int(kt & 1);
    const bool more = kt + 1 < ktiles;
    if (more) gload((kt + 1) * BK);
    const int kvalid = int(imin64(BK, m - kt * BK));
    if (kvalid == BK) {
#pragma unroll
      for (int kk = 0; kk < BK; ++kk) {
        if constexpr (LEAN) {
          if (kk > 0) fload(0, buf, kk);
          fma_step(0);
        } else {
          if (kk + 1 < BK) fload((kk + 1) & 1, buf, kk + 1);
          fma_step(kk & 1);
        }
      }
    } else {  // ragged last stage: exactly kvalid steps
      fma_step(0);
      for (int kk = 1; kk < kvalid; ++kk) {
        fload(0, buf, kk);
        fma_step(0);
      }
    }
    if (more) {
      sstore(buf ^ 1);
      __syncthreads();
      fload(0, buf ^ 1, 0);
    }
  }

#pragma unroll
  for (int r = 0; r < TM; ++r)
#pragma unroll
    for (int p = 0; p < TM / 2; ++p) {
      c[r][2 * p] = f2_lo(cp[r][p]);
      c[r][2 * p + 1] = f2_hi(cp[r][p]);
    }
#pragma unroll
  for (int r = 0; r < TM; ++r) {
    const int64_t gi = i0 + tile_off(ty, r);
    if (gi >= ni) continue;
#pragma unroll
    for (int h = 0; h < H; ++h) {
      const int64_t gj = j0 + GS * h + tx * 4;
      if (a.cvec && gj + 3 < nj) {
        *reinterpret_cast<float4*>(a.C + gi * nj + gj) =
            make_float4(c[r][4 * h], c[r][4 * h + 1], c[r][4 * h + 2], c[r][4 * h + 3]);
      } else {
#pragma unroll
        for (int q = 0; q < 4; ++q)
          if (gj + q < nj) a.C[gi * nj + gj + q] = c[r][4 * h + q];
      }
    }
  }
  cta_exit(a.t);
}

// ---------------------------------------------------------------- tiled, two CTAs per SM (round 2)
// T2: the tile, the per-thread 8 x 8 outputs and the per-element order of
// tiled_kernel (so the result is bit-identical to it, to LITERAL and to the
// oracle), rebuilt for two co-resident CTAs per SM (<= 128 registers: 4
// warps per SM sub-partition instead of 2) and for a barrier-free main loop:
//  * a prep kernel writes the operands k-major once per call, A^T and
//    (alpha A)^T (SYR2K: also B^T and (alpha B)^T), into a stream-ordered
//    workspace; alpha * a[i][k] is the literal kernel's rounding, so nothing
//    changes numerically. This replaces tiled_kernel's per-stage transpose
//    through registers (what held it at 182 registers, one CTA per SM);
//  * one elected thread streams [BK k][128 rows] boxes of the k-major
//    operands global -> shared with TMA into an NS-stage ring (zero fill past
//    n and m); every warp waits on the stage's full mbarrier, computes its
//    BK steps and arrives on the stage's empty mbarrier, and the elected
//    thread refills a stage once all 8 warps released it: no CTA barrier in
//    the k loop;
//  * a warp owns 4 ty x 8 tx threads; a float4 fragment read costs 2
//    shared-memory wavefronts for the row operand (<= 2 distinct words per
//    quarter-warp: merged) and 4 for the column operand (tools/lds_probe.cu).
// Tiles are 64 x 256 (8 x 8 outputs per thread; warp w = row group w, lane =
// column group): the row operand is a broadcast in every warp (2 shared-memory
// wavefronts per float4 read), the column operand 32 distinct words (4).
// Measured at 2048: 0.366 ms against 0.375 ms for 128 x 128 tiles. A mix of
// 64- and 48-row CTAs that fills the 296 CTA slots in one wave measured the
// same 0.367 ms (round 2, early): which CTAs share an SM is not under the
// kernel's control, and two 64-row CTAs on one SM still load each
// sub-partition with 4 units. The work per sub-partition is what sets the
// time once the grid is one wave (a warp runs on sub-partition warp % 4; two
// warps per sub-partition issue FFMA2 as fast as four, tools/warp_rate_probe):
// the mixed 56-row tile (kMixRows) mixes within the CTA instead, 8 + 6 rows
// per sub-partition from every CTA, and took SYRK 2048 from 0.342 to 0.327 ms
// and SYR2K from 0.976 to 0.916 ms, bit-identical (t2_use_mix picks it).
#ifndef T2_NS
#define T2_NS 4
#endif
#ifndef T2_BK
#define T2_BK 16
#endif
// RH rows per thread: 8 (64-row tiles, two CTAs per SM, <= 128 registers).
// The template also builds RH = 15 (120-row tiles, one CTA per SM, 222
// registers: 15 x 8 outputs per thread cut the shared-memory wavefronts per
// FMA by 0.6x, and 2048 rows make 144 tiles for 148 SMs); measured slower at
// every size (2048: 0.379 vs 0.357 ms; 4096: 1.65 vs 1.15 ms; one CTA of 8
// warps per SM does not keep the FMA pipe busy), so only RH = 8 is launched.
template <int MODE, int RH = 8, int RBOX = 8 * RH>
struct T2Cfg {
  static constexpr int NA = MODE == MODE_SYR2K ? 4 : 2;
  static constexpr int NP = NA / 2;                               // row-side (and column-side) arrays
  static constexpr int BK = MODE == MODE_SYR2K ? 8 : T2_BK;
  static constexpr int MINB = RH > 8 ? 1 : 2;                    // CTAs per SM
  static constexpr int NS = RH > 8 ? 6 : T2_NS;                  // ring stages
  static constexpr int RB = RBOX, CB = 256;                       // row box, column strip
  static constexpr int ROW_FLOATS = BK * RB, COL_FLOATS = BK * CB;
  static constexpr int STAGE_FLOATS = NP * (ROW_FLOATS + COL_FLOATS);
  static constexpr int FBUF = MODE == MODE_SYR2K ? 1 : 2;
  static constexpr size_t SBYTES = size_t(NS) * STAGE_FLOATS * 4 + 2 * NS * 8;
};

#ifndef T2_PAIR_OUTER
#define T2_PAIR_OUTER 1
#endif

struct T2Maps {
  CUtensorMap m[4];  // per stage array (row-side first): the k-major operand it is loaded from
};

struct T2Geo {
  int cs;            // column strips of 256
  int rbs;           // tri: row blocks of 8 * RH rows
  int tri;           // compute only tiles reaching the diagonal or above (8 warps per tile)
  int q;             // otherwise: CTAs per strip, each 8-row warp units of the strip's rows:
  int uw, ux;        // uw units each, the first ux CTAs one more (<= 8: one unit per warp)
};

// The mixed tile (tile2_mix_kernel): 56 rows, warps 0-3 take 8 rows each and
// warps 4-7 take 6. A warp runs on sub-partition (warp % 4), so every CTA
// gives each sub-partition 8 + 6 rows of work, wherever the CTA lands. With
// whole 8-row units a 2048-row SYRK has 13.8 units per SM, and the busiest of
// the four sub-partitions carries 4 of them (two CTAs of 7 active warps: one
// sub-partition gets 2 units, the others 4); the mixed tile carries 3.5.
constexpr int kMixRows = 56;

// One (RH W) x 256 tile computed by its first W warps (W <= 8), RH rows per
// thread: rows {4 W g + 4 ty + r} for the G = RH / 4 full groups, then
// {4 W G + (RH % 4) ty + r} (ty = warp). Fewer active warps make a shorter
// tile at the same 8 x 8 outputs (and shared-memory cost) per thread, which
// is how the grid balances the SMs' work (launch_t2).
// MIX (the 56-row tile): this warp's RH rows start at row wrow of the tile,
// contiguous (8: two float4 groups; 6: one float4 and one float2 group,
// whichever order keeps both aligned).
template <int MODE, int RH, int RBOX = 8 * RH, bool MIX = false>
__device__ __forceinline__ void t2_tile(float* sm, uint64_t* full, uint64_t* empty, const T2Maps& maps,
                                        const TileArgs& a, int64_t i0, int64_t j0, int W, int wrow = 0) {
  constexpr bool TWO = MODE == MODE_SYR2K;
  using Cfg = T2Cfg<MODE, RH, RBOX>;
  constexpr int BK = Cfg::BK, NP = Cfg::NP, NS = Cfg::NS, RBX = Cfg::RB, CBX = Cfg::CB;
  constexpr int G = RH / 4, RR = RH % 4;
  // stage layout: NP row arrays [BK][8 RH], then NP column arrays [BK][256]
  auto rowp = [&](int slot, int s, int kk) { return sm + slot * Cfg::STAGE_FLOATS + s * Cfg::ROW_FLOATS + kk * RBX; };
  auto colp = [&](int slot, int s, int kk) {
    return sm + slot * Cfg::STAGE_FLOATS + NP * Cfg::ROW_FLOATS + s * Cfg::COL_FLOATS + kk * CBX;
  };
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int ty = warp, tx = lane;
  const int64_t n = a.ni, m = a.m;
  const int64_t ktiles = (m + BK - 1) / BK;
  const int gs = 4 * W;  // row group stride
  // tile row of the warp's float4 group g (rows off4(g) .. +3) and of its
  // remaining RR rows (off2() ..); the uniform tile interleaves the warps'
  // groups, the mixed tile gives each warp contiguous rows
  int m4a = 0, m4b = 0, m2 = 0;
  if constexpr (MIX) {
    static_assert(RH == 8 || RH == 6, "the mixed tile has 8- and 6-row warps");
    if constexpr (RH == 8) {
      m4a = wrow, m4b = wrow + 4;
    } else {
      const bool lo = (wrow & 3) == 0;
      m4a = lo ? wrow : wrow + 2, m2 = lo ? wrow + 4 : wrow;
    }
  }
  auto off4 = [&](int g) {
    if constexpr (MIX) return g == 0 ? m4a : m4b;
    else return gs * g + 4 * ty;
  };
  auto off2 = [&]() {
    if constexpr (MIX) return m2;
    else return gs * G + RR * ty;
  };
  auto row_of = [&](int r) { return r < 4 * G ? off4(r / 4) + (r % 4) : off2() + (r - 4 * G); };

  // row-side stage arrays: alpha*a[i][k] (SYR2K: then alpha*b[i][k]); column-side: a[j][k]
  // (SYR2K: b[j][k], then a[j][k]); maps in the same order
  auto tma = [&](int64_t kt) {  // the elected thread
    const int slot = int(kt % NS);
    bar_expect_tx(&full[slot], uint32_t(Cfg::STAGE_FLOATS * 4));
    const int32_t k0 = int32_t(kt * BK);
#pragma unroll
    for (int s = 0; s < NP; ++s) {
      tma_2d(rowp(slot, s, 0), &maps.m[s], int32_t(i0), k0, &full[slot]);
      tma_2d(colp(slot, s, 0), &maps.m[NP + s], int32_t(j0), k0, &full[slot]);
    }
  };
  if (tid == 0)
    for (int64_t kt = 0; kt < NS && kt < ktiles; ++kt) tma(kt);
  if (warp >= W) return;  // an idle warp of a short tile (not with a.mirror: W == 8 there)

  // beta * C into the accumulators (pairs along j), while the first stages land
  uint64_t cp[RH][4];
  const bool cvec = a.cvec, zinit = a.zinit != 0;
#pragma unroll
  for (int r = 0; r < RH; ++r) {
    const int64_t gi = i0 + row_of(r);
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      if (zinit) {
        cp[r][2 * h] = cp[r][2 * h + 1] = 0ull;
        continue;
      }
      const int64_t gj = j0 + 128 * h + tx * 4;
      float c4[4];
      if (cvec && gi < n && gj + 3 < n) {
        const float4 v = *reinterpret_cast<const float4*>(a.C + gi * n + gj);
        c4[0] = v.x, c4[1] = v.y, c4[2] = v.z, c4[3] = v.w;
      } else {
#pragma unroll
        for (int q = 0; q < 4; ++q) c4[q] = (gi < n && gj + q < n) ? a.C[gi * n + gj + q] : 0.0f;
      }
      cp[r][2 * h] = f2_pack(__fmul_rn(c4[0], a.beta), __fmul_rn(c4[1], a.beta));
      cp[r][2 * h + 1] = f2_pack(__fmul_rn(c4[2], a.beta), __fmul_rn(c4[3], a.beta));
    }
  }

  float fr[Cfg::FBUF][NP][RH], fc[Cfg::FBUF][NP][8];
  auto fload = [&](int fb, int slot, int kk) {
#pragma unroll
    for (int s = 0; s < NP; ++s) {
      const float* rp = rowp(slot, s, kk);
#pragma unroll
      for (int g = 0; g < G; ++g) {
        const float4 v = *reinterpret_cast<const float4*>(rp + off4(g));
        fr[fb][s][4 * g] = v.x, fr[fb][s][4 * g + 1] = v.y, fr[fb][s][4 * g + 2] = v.z, fr[fb][s][4 * g + 3] = v.w;
      }
      if constexpr (RR == 2) {
        const float2 v = *reinterpret_cast<const float2*>(rp + off2());
        fr[fb][s][4 * G] = v.x, fr[fb][s][4 * G + 1] = v.y;
      } else {
#pragma unroll
        for (int q = 0; q < RR; ++q) fr[fb][s][4 * G + q] = rp[off2() + q];
      }
      const float* cq = colp(slot, s, kk);
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const float4 v = *reinterpret_cast<const float4*>(cq + 128 * h + tx * 4);
        fc[fb][s][4 * h] = v.x, fc[fb][s][4 * h + 1] = v.y, fc[fb][s][4 * h + 2] = v.z, fc[fb][s][4 * h + 3] = v.w;
      }
    }
  };
  auto fma_step = [&](int fb) {
    // column pair outer: its two registers stay in the operand reuse cache
    // across the RH instructions that use them (SYRK 0.359 -> 0.348 ms)
    if constexpr (!TWO && T2_PAIR_OUTER) {
#pragma unroll
      for (int p = 0; p < 4; ++p) {
        const uint64_t bq = f2_pack(fc[fb][0][2 * p], fc[fb][0][2 * p + 1]);
#pragma unroll
        for (int r = 0; r < RH; ++r) f2_fma_acc(cp[r][p], f2_pack(fr[fb][0][r], fr[fb][0][r]), bq);
      }
      return;
    }
    if constexpr (TWO && T2_PAIR_OUTER) {  // SYR2K: the same, each op kind grouped over r
      // (grouping 4 rows at a time spills less at 128 registers but measured
      // slower: 0.976 -> 1.010 ms uniform, equal in the mixed tile)
#pragma unroll
      for (int p = 0; p < 4; ++p) {
        const uint64_t bq = f2_pack(fc[fb][0][2 * p], fc[fb][0][2 * p + 1]);
        const uint64_t aq = f2_pack(fc[fb][1][2 * p], fc[fb][1][2 * p + 1]);
        uint64_t pr[RH];
#pragma unroll
        for (int r = 0; r < RH; ++r) pr[r] = f2_mul(f2_pack(fr[fb][1][r], fr[fb][1][r]), aq);
#pragma unroll
        for (int r = 0; r < RH; ++r) pr[r] = f2_fma(f2_pack(fr[fb][0][r], fr[fb][0][r]), bq, pr[r]);
#pragma unroll
        for (int r = 0; r < RH; ++r) f2_add_acc(cp[r][p], pr[r]);
      }
      return;
    }
#pragma unroll
    for (int r = 0; r < RH; ++r) {
      const uint64_t ar = f2_pack(fr[fb][0][r], fr[fb][0][r]);
#pragma unroll
      for (int p = 0; p < 4; ++p) {
        const uint64_t bq = f2_pack(fc[fb][0][2 * p], fc[fb][0][2 * p + 1]);
        if constexpr (TWO) {  // fmaf(alpha*a_ik, b_jk, (alpha*b_ik) * a_jk), then c + s (R20)
          const uint64_t pr = f2_mul(f2_pack(fr[fb][1][r], fr[fb][1][r]), f2_pack(fc[fb][1][2 * p], fc[fb][1][2 * p + 1]));
          f2_add_acc(cp[r][p], f2_fma(ar, bq, pr));
        } else {
          f2_fma_acc(cp[r][p], ar, bq);
        }
      }
    }
  };
  // the warp is done reading stage kt's slot; the elected thread refills the
  // slot of the stage before (released by every warp by now, in practice)
  auto release = [&](int64_t kt) {
    __syncwarp();
    if (lane == 0) bar_arrive(&empty[kt % NS]);
    if (tid == 0 && kt >= 1 && kt - 1 + NS < ktiles) {
      bar_wait(&empty[(kt - 1) % NS], uint32_t(((kt - 1) / NS) & 1));
      tma(kt - 1 + NS);
    }
  };

  // full stages in a loop of their own (one register assignment for the
  // accumulators), then the ragged last stage
  const int64_t kfull = m / BK;
  for (int64_t kt = 0; kt < kfull; ++kt) {
    const int slot = int(kt % NS);
    bar_wait(&full[slot], uint32_t((kt / NS) & 1));
    fload(0, slot, 0);
#pragma unroll
    for (int kk = 0; kk < BK; ++kk) {
      if constexpr (Cfg::FBUF == 2) {
        if (kk + 1 < BK) fload((kk + 1) & 1, slot, kk + 1);
        fma_step(kk & 1);
      } else {
        if (kk > 0) fload(0, slot, kk);
        fma_step(0);
      }
    }
    release(kt);
  }
  if (kfull < ktiles) {  // exactly m % BK steps
    const int slot = int(kfull % NS);
    bar_wait(&full[slot], uint32_t((kfull / NS) & 1));
    const int kvalid = int(m - kfull * BK);
    for (int kk = 0; kk < kvalid; ++kk) {
      fload(0, slot, kk);
      fma_step(0);
    }
  }

#pragma unroll
  for (int r = 0; r < RH; ++r) {
    const int64_t gi = i0 + row_of(r);
    if (gi >= n) continue;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int64_t gj = j0 + 128 * h + tx * 4;
      const float c0 = f2_lo(cp[r][2 * h]), c1 = f2_hi(cp[r][2 * h]);
      const float c2 = f2_lo(cp[r][2 * h + 1]), c3 = f2_hi(cp[r][2 * h + 1]);
      if (a.mirror) {
        // CORR: only the upper elements (j > i) and the unit diagonal here;
        // the lower triangle below, through shared memory
        const float cv[4] = {c0, c1, c2, c3};
        if (gj > gi && gj + 3 < n) {
          *reinterpret_cast<float4*>(a.C + gi * n + gj) = make_float4(c0, c1, c2, c3);
        } else {
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            const int64_t j = gj + q;
            if (j < n && j >= gi) a.C[gi * n + j] = j == gi ? 1.0f : cv[q];
          }
        }
        continue;
      }
      if (cvec && gj + 3 < n) {
        *reinterpret_cast<float4*>(a.C + gi * n + gj) = make_float4(c0, c1, c2, c3);
      } else {
        const float cv[4] = {c0, c1, c2, c3};
#pragma unroll
        for (int q = 0; q < 4; ++q)
          if (gj + q < n) a.C[gi * n + gj + q] = cv[q];
      }
    }
  }
  if constexpr (MODE == MODE_SYRK && !MIX) if (a.mirror) {
    // the lower triangle: C[j][i] = C[i][j] for j > i, the tile staged
    // transposed through the (now idle) stage ring so each warp writes whole
    // 64-float row segments of C^T (coalesced). Every stage was consumed
    // (each warp waited on it), so after the barrier the ring is free.
    constexpr int TP = CBX + 1;                  // [8 RH rows][256 cols], odd pitch: row writes and column reads conflict-free
    static_assert(8 * RH * TP <= NS * Cfg::STAGE_FLOATS, "the staged tile must fit the ring");
    __syncthreads();
    float* tt = sm;
#pragma unroll
    for (int r = 0; r < RH; ++r)
#pragma unroll
      for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const float v = (q & 1) ? f2_hi(cp[r][2 * h + q / 2]) : f2_lo(cp[r][2 * h + q / 2]);
          tt[row_of(r) * TP + 128 * h + tx * 4 + q] = v;
        }
    __syncthreads();
    for (int c = warp; c < CBX; c += 8) {
      const int64_t j = j0 + c;
      if (j >= n) break;
      for (int r = lane; r < 8 * RH; r += 32) {
        const int64_t i = i0 + r;
        if (i < n && j > i) a.C[j * n + i] = tt[r * TP + c];
      }
    }
  }
}

template <int MODE, int RH>
__global__ void __launch_bounds__(256, (RH > 8 ? 1 : 2)) tile2_kernel(const __grid_constant__ T2Maps maps, TileArgs a,
                                                                      T2Geo g) {
  static_assert(MODE != MODE_GEMM, "T2 covers SYRK and SYR2K");
  using Cfg = T2Cfg<MODE, RH>;
  constexpr int NS = Cfg::NS;
  extern __shared__ __align__(128) float t2_dyn[];
  uint64_t* full = reinterpret_cast<uint64_t*>(t2_dyn + NS * Cfg::STAGE_FLOATS);
  uint64_t* empty = full + NS;
  // the tile. tri: the 8-warp tiles that reach the diagonal, by row block;
  // otherwise CTA k of strip cs owns warp units [k uw + min(k, ux), +W)
  int cs, W;
  int64_t i0;
  if (g.tri) {
    int rem = int(blockIdx.x), rb = 0;
    while (true) {
      const int lo = int((int64_t(Cfg::RB) * rb) / 256);  // first strip with an element j >= i
      if (rem < g.cs - lo) {
        cs = lo + rem;
        break;
      }
      rem -= g.cs - lo;
      ++rb;
    }
    W = 8;
    i0 = int64_t(Cfg::RB) * rb;
  } else {
    cs = int(blockIdx.x) / g.q;
    const int k = int(blockIdx.x) % g.q;
    W = g.uw + (k < g.ux ? 1 : 0);
    i0 = int64_t(RH) * (int64_t(k) * g.uw + min(k, g.ux));
  }
  cta_enter(a.t);
  if (threadIdx.x == 0) {
    for (int s = 0; s < NS; ++s) {
      bar_init(&full[s], 1);
      bar_init(&empty[s], unsigned(W));
    }
    fence_barrier_init();
  }
  __syncthreads();
  // launched as a programmatic dependent of the kernel that wrote the
  // operands (the prep copies; CORR's statistics): everything above overlapped
  // its tail; wait for its completion (and memory) before reading A or C
  asm volatile("griddepcontrol.wait;" ::: "memory");
  t2_tile<MODE, RH>(t2_dyn, full, empty, maps, a, i0, int64_t(cs) * Cfg::CB, W);
  cta_exit(a.t);
}

// The mixed 56-row tile (kMixRows): CTA k of strip cs owns rows [56 k, 56 k + 56).
template <int MODE>
__global__ void __launch_bounds__(256, 2) tile2_mix_kernel(const __grid_constant__ T2Maps maps, TileArgs a, T2Geo g) {
  using Cfg = T2Cfg<MODE, 8, kMixRows>;
  static_assert(sizeof(T2Cfg<MODE, 6, kMixRows>) > 0 && T2Cfg<MODE, 6, kMixRows>::STAGE_FLOATS == Cfg::STAGE_FLOATS &&
                    T2Cfg<MODE, 6, kMixRows>::NS == Cfg::NS && T2Cfg<MODE, 6, kMixRows>::BK == Cfg::BK,
                "both warp kinds read one stage ring");
  constexpr int NS = Cfg::NS;
  extern __shared__ __align__(128) float t2_dyn[];
  uint64_t* full = reinterpret_cast<uint64_t*>(t2_dyn + NS * Cfg::STAGE_FLOATS);
  uint64_t* empty = full + NS;
  const int cs = int(blockIdx.x) / g.q, k = int(blockIdx.x) % g.q;
  const int64_t i0 = int64_t(kMixRows) * k;
  auto wrow = [](int w) { return w < 4 ? 8 * w : 32 + 6 * (w - 4); };
  int W = 0;  // warps with a row inside the matrix (rows ascend with the warp)
  for (int w = 0; w < 8; ++w)
    if (i0 + wrow(w) < a.ni) W = w + 1;
  cta_enter(a.t);
  if (threadIdx.x == 0) {
    for (int s = 0; s < NS; ++s) {
      bar_init(&full[s], 1);
      bar_init(&empty[s], unsigned(W));
    }
    fence_barrier_init();
  }
  __syncthreads();
  asm volatile("griddepcontrol.wait;" ::: "memory");
  const int warp = int(threadIdx.x) >> 5;
  if (warp < 4)
    t2_tile<MODE, 8, kMixRows, true>(t2_dyn, full, empty, maps, a, i0, int64_t(cs) * Cfg::CB, W, wrow(warp));
  else
    t2_tile<MODE, 6, kMixRows, true>(t2_dyn, full, empty, maps, a, i0, int64_t(cs) * Cfg::CB, W, wrow(warp));
  cta_exit(a.t);
}

// k-major copies of X (n x m, row-major): Xt[k][i] = X[i][k] and, when aXt is
// given, aXt[k][i] = alpha * X[i][k] (the literal kernel's rounding). Rows of
// the copies have pitch ld (a multiple of 4 floats: the TMA stride).
struct PrepSrc {
  const float* X;   // n x m, row-major
  float* Xt;        // m x ld: X^T
  float* aXt;       // m x ld: (alpha X)^T, or null
  int vec;          // float4 loads of X (m % 4 == 0, 16-byte aligned)
};

// blockIdx.z selects the matrix (SYR2K copies A and B in one launch)
__global__ void __launch_bounds__(256) t2_prep_kernel(PrepSrc s0, PrepSrc s1, int64_t n, int64_t m, int64_t ld,
                                                      float alpha) {
  asm volatile("griddepcontrol.launch_dependents;");  // the tile kernel may start its prologue
  const PrepSrc& src = blockIdx.z ? s1 : s0;
  const float* __restrict__ X = src.X;
  float* __restrict__ Xt = src.Xt;
  float* __restrict__ aXt = src.aXt;
  const int vec = src.vec;
  // 64 (i) x 64 (k) tiles; float4 reads along k when vec (m % 4 == 0, X
  // 16-byte aligned), float4 writes along i (ld % 4 == 0). 32 x 32 scalar
  // tiles ran at ~3 TB/s (16 us per 2048^2 matrix).
  __shared__ float tile[64][65];
  const int64_t i0 = int64_t(blockIdx.x) * 64, k0 = int64_t(blockIdx.y) * 64;
  const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;  // 16 float4 columns x 16 rows per pass
#pragma unroll
  for (int r = 0; r < 4; ++r) {
    const int row = ty + 16 * r;
    const int64_t i = i0 + row, k = k0 + 4 * tx;
    float v[4];
    if (vec && i < n && k + 3 < m) {
      const float4 q = __ldg(reinterpret_cast<const float4*>(X + i * m + k));
      v[0] = q.x, v[1] = q.y, v[2] = q.z, v[3] = q.w;
    } else {
#pragma unroll
      for (int c = 0; c < 4; ++c) v[c] = (i < n && k + c < m) ? X[i * m + k + c] : 0.0f;
    }
#pragma unroll
    for (int c = 0; c < 4; ++c) tile[row][4 * tx + c] = v[c];
  }
  __syncthreads();
#pragma unroll
  for (int r = 0; r < 4; ++r) {
    const int kk = ty + 16 * r;
    const int64_t k = k0 + kk, i = i0 + 4 * tx;
    if (k >= m) continue;
    float v[4];
#pragma unroll
    for (int c = 0; c < 4; ++c) v[c] = tile[4 * tx + c][kk];
    if (i + 3 < n) {
      *reinterpret_cast<float4*>(Xt + k * ld + i) = make_float4(v[0], v[1], v[2], v[3]);
      if (aXt)
        *reinterpret_cast<float4*>(aXt + k * ld + i) = make_float4(
            __fmul_rn(alpha, v[0]), __fmul_rn(alpha, v[1]), __fmul_rn(alpha, v[2]), __fmul_rn(alpha, v[3]));
    } else {
#pragma unroll
      for (int c = 0; c < 4; ++c)
        if (i + c < n) {
          Xt[k * ld + i + c] = v[c];
          if (aXt) aXt[k * ld + i + c] = __fmul_rn(alpha, v[c]);
        }
    }
  }
}

// T2 is the default for the 128 x 128 SYRK / SYR2K tiles; CATT_TILED_T2=0
// restores tiled_kernel (tools only, for A/B timing).
static bool tiled_t2() {
  static const int env = [] {
    const char* e = getenv("CATT_TILED_T2");
    return e ? atoi(e) : 1;
  }();
  return env != 0;
}

// a k-major operand: m rows (k) x n columns, pitch ld; box {bw columns, BK rows}
static bool t2_map(CUtensorMap* mp, const float* base, int64_t n, int64_t m, int64_t ld, int bw, int bk) {
  auto fn = encode_fn();
  if (!fn) return false;
  const cuuint64_t dims[2] = {cuuint64_t(n), cuuint64_t(m)};
  const cuuint64_t strides[1] = {cuuint64_t(ld) * 4};
  const cuuint32_t box[2] = {cuuint32_t(bw), cuuint32_t(bk)};
  const cuuint32_t estr[2] = {1, 1};
  return fn(mp, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims, strides, box, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

template <int MODE>
static bool t2_ok(const TileArgs& a) {
  return tiled_t2() && a.m > 0 && a.m < (int64_t(1) << 31) && a.ni < (int64_t(1) << 31);
}

// Tiles for an n x n output. tri: 8-warp tiles of 8 RH rows. Otherwise each
// 256-column strip's rows are dealt as 8-row warp units to q CTAs, q chosen
// so that the grid fills the 2 x #SM CTA slots (one wave) with at most 8
// units per CTA: 2048 on 148 SMs gives 37 CTAs per strip of 7 or 6 units
// (56 or 48 rows), so the busiest SM has 14 units of work where 64-row
// tiles gave it 16 (256 tiles in 296 slots).
static T2Geo t2_geometry(int64_t n, bool tri, int rh) {
  static const int nsm = [] {
    int d = 0, v = 148;
    if (cudaGetDevice(&d) == cudaSuccess) cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, d);
    return v;
  }();
  T2Geo g{};
  g.cs = int((n + 255) / 256);
  g.tri = tri ? 1 : 0;
  g.rbs = int((n + 8 * rh - 1) / (8 * rh));
  const int64_t units = (n + rh - 1) / rh;                  // warp units of rh rows
  const int64_t per_strip = std::max<int64_t>(1, (2 * int64_t(nsm)) / g.cs);
  const int64_t q = std::max((units + 7) / 8, std::min(units, per_strip));
  g.q = int(q);
  g.uw = int(units / q);
  g.ux = int(units % q);
  return g;
}

static int64_t t2_tiles(const T2Geo& g, int rb_rows) {
  int64_t tiles = 0;
  for (int rb = 0; rb < g.rbs; ++rb) tiles += g.tri ? g.cs - (int64_t(rb_rows) * rb) / 256 : g.cs;
  return tiles;
}

// The mixed 56-row tile instead of whole 8-row units: when both grids fit one
// wave, when it lowers the busiest sub-partition's load (in 8-row units:
// per CTA ceil(W / 4) of its W active warps, 1.75 for the mixed tile; two
// CTAs per SM when the grid exceeds the SMs). CATT_T2_MIX=0/1 overrides
// (tools only).
static bool t2_use_mix(int64_t n, bool tri) {
  static const int env = [] {
    const char* e = getenv("CATT_T2_MIX");
    return e ? atoi(e) : -1;
  }();
  static const int nsm = [] {
    int d = 0, v = 148;
    if (cudaGetDevice(&d) == cudaSuccess) cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, d);
    return v;
  }();
  if (tri) return false;
  if (env == 0 || env == 1) return env == 1;
  const T2Geo g = t2_geometry(n, false, 8);
  const int64_t gu = int64_t(g.cs) * g.q, gm = int64_t(g.cs) * ((n + kMixRows - 1) / kMixRows);
  if (gu > 2 * nsm || gm > 2 * nsm) return false;
  const int wmax = g.uw + (g.ux > 0 ? 1 : 0);
  const double lu = (gu > nsm ? 2 : 1) * double((wmax + 3) / 4);
  const double lm = (gm > nsm ? 2 : 1) * 1.75;
  return lm < lu;
}

template <int MODE, int RH, int RBOX = 8 * RH>
static catt_status launch_t2(TileArgs a, const catt_throttle* t, cudaStream_t s) {
  constexpr bool MIX = RBOX != 8 * RH;
  const void* f = MIX ? (const void*)tile2_mix_kernel<MODE> : (const void*)tile2_kernel<MODE, RH>;
  constexpr size_t sb = T2Cfg<MODE, RH, RBOX>::SBYTES;
  cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, int(sb));
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  size_t dyn = 0;
  catt_status st = prepare_launch(f, t, 256, sb, false, &a.t, &dyn);
  if (st != CATT_OK) return st;
  if (dyn > sb) {  // a Fig 5 pad on top
    e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, int(dyn));
    if (e != cudaSuccess) {
      record_cuda_error(e);
      return CATT_ECUDA;
    }
  }
  const bool given = MODE == MODE_SYRK && a.kmaj && a.alpha == 1.0f;  // A^T supplied: no prep, no workspace
  const int64_t n = a.ni, m = a.m, ld = given ? a.kld : (n + 3) / 4 * 4;
  const bool scale = a.alpha != 1.0f;  // alpha * x == x exactly: (alpha A)^T is A^T
  const int nsrc = MODE == MODE_SYR2K ? 2 : 1;
  const int64_t per = m * ld;          // floats per k-major copy
  const size_t bytes = size_t(per) * 4 * size_t(nsrc * (scale ? 2 : 1));
  // the workspace: stream-ordered, so concurrent launches on other streams get their own
  static std::once_flag pool_once;
  std::call_once(pool_once, [] {
    int d = 0;
    cudaMemPool_t pool;
    if (cudaGetDevice(&d) == cudaSuccess && cudaDeviceGetDefaultMemPool(&pool, d) == cudaSuccess) {
      uint64_t keep = UINT64_MAX;  // keep freed blocks for the next call
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
    }
  });
  float* ws = nullptr;
  e = given ? cudaSuccess : cudaMallocAsync(reinterpret_cast<void**>(&ws), bytes, s);  // nothing to copy when A^T is given
  if (e != cudaSuccess) {
    cudaGetLastError();                // not sticky: the caller falls back to tiled_kernel
    return e == cudaErrorMemoryAllocation ? CATT_ENOMEM : (record_cuda_error(e), CATT_ECUDA);
  }
  // copies: A^T, [(alpha A)^T], SYR2K: B^T, [(alpha B)^T]
  float* At = given ? const_cast<float*>(a.kmaj) : ws;
  float* aAt = scale ? ws + per : At;
  float* Bt = MODE == MODE_SYR2K ? ws + per * (scale ? 2 : 1) : nullptr;
  float* aBt = MODE == MODE_SYR2K ? (scale ? Bt + per : Bt) : nullptr;
  const dim3 pg(unsigned((n + 63) / 64), unsigned((m + 63) / 64));
  auto al16 = [](const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; };
  const int vecA = m % 4 == 0 && al16(a.A), vecB = m % 4 == 0 && (MODE != MODE_SYR2K || al16(a.B));
  if (pg.y > 65535 && !given) {
    if (ws) cudaFreeAsync(ws, s);
    return CATT_EINVAL;
  }
  if (!given) {
    const PrepSrc pa{a.A, At, scale ? aAt : nullptr, vecA};
    const PrepSrc pb{a.B, Bt, scale ? aBt : nullptr, vecB};
    const dim3 pg2(pg.x, pg.y, MODE == MODE_SYR2K ? 2u : 1u);
    t2_prep_kernel<<<pg2, 256, 0, s>>>(pa, pb, n, m, ld, a.alpha);
  }
  // stage arrays, row side then column side: SYRK {(alpha A)^T} {A^T};
  // SYR2K {(alpha A)^T, (alpha B)^T} {B^T, A^T}
  T2Maps maps{};
  using Cfg = T2Cfg<MODE, RH, RBOX>;
  const float* src[4];
  if (MODE == MODE_SYR2K) {
    src[0] = aAt, src[1] = aBt, src[2] = Bt, src[3] = At;
  } else {
    src[0] = aAt, src[1] = At, src[2] = src[3] = nullptr;
  }
  bool ok = true;
  for (int q = 0; q < Cfg::NA; ++q)
    ok = ok && t2_map(&maps.m[q], src[q], n, m, ld, q < Cfg::NP ? Cfg::RB : Cfg::CB, Cfg::BK);
  if (!ok) {
    if (ws) cudaFreeAsync(ws, s);
    return CATT_ECUDA;
  }
  T2Geo g = t2_geometry(n, a.tri != 0, RH);
  if (MIX) g.q = int((n + kMixRows - 1) / kMixRows), g.uw = g.ux = 0;
  const int64_t tiles = a.tri ? t2_tiles(g, Cfg::RB) : int64_t(g.cs) * g.q;
  if (tiles > (int64_t(1) << 31) - 1) {
    if (ws) cudaFreeAsync(ws, s);
    return CATT_EINVAL;
  }
  auto al = [](const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; };
  a.cvec = (a.nj % 4 == 0) && al(a.C);
  // programmatic dependent launch after the prep copies: the kernel's
  // prologue overlaps their tail (griddepcontrol.wait inside). Not for the
  // upper-triangle grid (CORR, one tile per SM): CTAs launched early land two
  // per SM on the SMs the previous kernel leaves free, which doubled the
  // makespan (0.216 -> 0.382 ms)
  // The upper-triangle grid can still follow its producer (CORR's statistics)
  // programmatically when it has at most one tile per SM: a dynamic
  // shared-memory request above half the SM's keeps the early CTAs one per SM
  static const int tri_pdl = [] {
    const char* e = getenv("CATT_T2_TRI_PDL");
    return e ? atoi(e) : 1;
  }();
  static const int nsm_l = [] {
    int d = 0, v = 148;
    if (cudaGetDevice(&d) == cudaSuccess) cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, d);
    return v;
  }();
  bool pdl = !a.tri;
  if (a.tri && tri_pdl && tiles <= nsm_l && !(t && t->active_ctas > 0)) {
    constexpr size_t half = 116 * 1024;  // > 228 KB / 2
    if (dyn < half) {
      e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, int(half));
      if (e != cudaSuccess) {
        record_cuda_error(e);
        if (ws) cudaFreeAsync(ws, s);
        return CATT_ECUDA;
      }
      dyn = half;
    }
    pdl = true;
  }
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(unsigned(tiles));
  cfg.blockDim = dim3(256);
  cfg.dynamicSmemBytes = dyn;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 1 : 0;
  if constexpr (MIX)
    e = cudaLaunchKernelEx(&cfg, tile2_mix_kernel<MODE>, maps, a, g);
  else
    e = cudaLaunchKernelEx(&cfg, tile2_kernel<MODE, RH>, maps, a, g);
  if (e != cudaSuccess) {
    record_cuda_error(e);
    cudaGetLastError();
  }
  const catt_status ls = e != cudaSuccess ? CATT_ECUDA : after_launch();
  if (ws) cudaFreeAsync(ws, s);
  return ls;
}

// Register budget per kernel: MINB = 1 (up to 255 registers, one 256-thread
// CTA per SM) or 2 (128 registers). CATT_TILED_MINB overrides (tools only).
static int tiled_minb(bool two) {
  static const int env = [] {
    const char* e = getenv("CATT_TILED_MINB");
    return e ? atoi(e) : 0;
  }();
  if (env == 1 || env == 2) return env;
  return 1;
  (void)two;
}

// LEAN large tiles (BK = 8, single-buffered fragments, 2 CTAs per SM): with
// scalar FFMA they beat one CTA per SM when tiles outnumber SMs (SYRK 2048:
// 0.497 -> 0.460 ms); since the inner product runs as FFMA2 the regular
// kernel is faster (0.441 ms; LEAN 0.466 ms, 44 bytes of spills at 128
// registers), so LEAN is off unless CATT_TILED_LEAN=1 (tools only).
static bool tiled_lean(int64_t active_tiles) {
  static const int env = [] {
    const char* e = getenv("CATT_TILED_LEAN");
    return e ? atoi(e) : -1;
  }();
  static const int nsm = [] {
    int d = 0, v = 148;
    if (cudaGetDevice(&d) == cudaSuccess) cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, d);
    return v;
  }();
  if (env != 1) return false;
  return active_tiles > nsm;
}

template <int MODE>
static const void* tiled_func() {
  return tiled_minb(MODE == MODE_SYR2K) == 2 ? (const void*)tiled_kernel<MODE, 2> : (const void*)tiled_kernel<MODE, 1>;
}

// The 64 x 64 tile (SYRK, GEMM) when 128 x 128 tiles would not give every SM
// a CTA; it keeps the same per-element order, so results are identical.
template <int MODE>
static bool small_tiles(int64_t ni, int64_t nj) {
  if (MODE == MODE_SYR2K) return false;
  static const int nsm = [] {
    int d = 0, v = 148;
    if (cudaGetDevice(&d) == cudaSuccess) cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, d);
    return v;
  }();
  static const int force = [] {
    const char* e = getenv("CATT_TILED_SMALL");  // 0 / 1: force the tile size (tools only)
    return e ? atoi(e) : -1;
  }();
  if (force == 0 || force == 1) return force == 1;
  return ((ni + 127) / 128) * ((nj + 127) / 128) < nsm;
}

// DEEP stages (BK = 32 / 16): measured faster for SYR2K (1.123 -> 1.101 ms
// at 2048^2) and slower for SYRK (0.439 -> 0.470 ms) and CORR
// (profiles/r1deep/); CATT_TILED_DEEP=0/1 overrides (tools only)
template <int MODE>
static bool tiled_deep() {
  static const int deep_env = [] {
    const char* e = getenv("CATT_TILED_DEEP");
    return e ? atoi(e) : -1;
  }();
  return deep_env >= 0 ? deep_env == 1 : MODE == MODE_SYR2K;
}

template <int MODE>
static catt_status launch_tiled(TileArgs a, const catt_throttle* t, cudaStream_t s) {
  if (t && t->cta_threads != 0 && t->cta_threads != 256) return CATT_EINVAL;
  const bool small = small_tiles<MODE>(a.ni, a.nj);
  if constexpr (MODE != MODE_GEMM)
    if (!small && t2_ok<MODE>(a)) {
      const catt_status st = (!a.mirror && t2_use_mix(a.ni, a.tri != 0)) ? launch_t2<MODE, 8, kMixRows>(a, t, s)
                                                                          : launch_t2<MODE, 8>(a, t, s);
      if (st != CATT_ENOMEM) return st;  // no room for the k-major copies: the round-1 kernel below
    }
  constexpr int TMs = MODE == MODE_SYR2K ? 8 : 4;  // SYR2K never takes the small tile (static_assert)
  const int64_t tt = (a.ni + 127) / 128;
  const bool lean = !small && MODE == MODE_SYRK && tiled_lean(a.tri ? tt * (tt + 1) / 2 : tt * tt);
  const void* f = small ? (const void*)tiled_kernel<MODE, 2, TMs> : tiled_func<MODE>();
  if constexpr (MODE == MODE_SYRK)
    if (lean) f = (const void*)tiled_kernel<MODE, 2, 8, true>;
  size_t dyn = 0;
  catt_status st = prepare_launch(f, t, 256, 0, false, &a.t, &dyn);
  if (st != CATT_OK) return st;
  const int64_t BMx = small ? 64 : 128;
  const int64_t ty = (a.ni + BMx - 1) / BMx, tx = (a.nj + BMx - 1) / BMx;
  if (ty > 65535 || tx > (int64_t(1) << 31) - 1) return CATT_EINVAL;
  auto al = [](const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; };
  a.vec = (a.m % 4 == 0) && al(a.A) && (MODE != MODE_SYR2K || al(a.B));
  a.bvec = MODE == MODE_GEMM && (a.nj % 4 == 0) && al(a.B);
  a.cvec = (a.nj % 4 == 0) && al(a.C);
  const dim3 grid{unsigned(tx), unsigned(ty), 1u};
  bool done = false;
  if constexpr (MODE == MODE_SYRK) {
    if (lean) {
      tiled_kernel<MODE, 2, 8, true><<<grid, 256, dyn, s>>>(a);
      done = true;
    }
  }
  if (!done && tiled_deep<MODE>() && !small && tiled_minb(MODE == MODE_SYR2K) == 1) {
    const void* fd = (const void*)tiled_kernel<MODE, 1, 8, false, true>;
    constexpr size_t sb = TileCfg<MODE, 8, false, true>::SBYTES;
    // the dynamic-size attribute first, so prepare_launch's occupancy query
    // (for a CTA cap) sees the kernel as it will run
    cudaError_t e = cudaFuncSetAttribute(fd, cudaFuncAttributeMaxDynamicSharedMemorySize, int(sb));
    if (e != cudaSuccess) {
      record_cuda_error(e);
      return CATT_ECUDA;
    }
    size_t dyn2 = 0;
    st = prepare_launch(fd, t, 256, sb, false, &a.t, &dyn2);
    if (st != CATT_OK) return st;
    if (dyn2 > sb) {                                           // a Fig 5 pad on top
      e = cudaFuncSetAttribute(fd, cudaFuncAttributeMaxDynamicSharedMemorySize, int(dyn2));
      if (e != cudaSuccess) {
        record_cuda_error(e);
        return CATT_ECUDA;
      }
    }
    tiled_kernel<MODE, 1, 8, false, true><<<grid, 256, dyn2, s>>>(a);
    done = true;
  }
  if (done) {
  } else if (small)
    tiled_kernel<MODE, 2, TMs><<<grid, 256, dyn, s>>>(a);
  else if (tiled_minb(MODE == MODE_SYR2K) == 2)
    tiled_kernel<MODE, 2><<<grid, 256, dyn, s>>>(a);
  else
    tiled_kernel<MODE, 1><<<grid, 256, dyn, s>>>(a);
  return after_launch();
}

// the kernel a large (128 x 128 tile) STAGED launch runs, and its dynamic
// shared memory (catt_kernel_desc / catt_plan describe this kernel)
const void* syrk_func(int variant, int64_t n, bool tri) {
  if (variant != CATT_VAR_STAGED) return (const void*)syrk_thread_kernel;
  if (!tiled_t2()) return tiled_func<MODE_SYRK>();
  if (t2_use_mix(n, tri)) return (const void*)tile2_mix_kernel<MODE_SYRK>;
  return (const void*)tile2_kernel<MODE_SYRK, 8>;
}

int64_t syrk_staged_dyn(int64_t n, bool tri) {
  if (!tiled_t2()) return 0;
  return t2_use_mix(n, tri) ? int64_t(T2Cfg<MODE_SYRK, 8, kMixRows>::SBYTES) : int64_t(T2Cfg<MODE_SYRK, 8>::SBYTES);
}

const void* syr2k_func(int variant, int64_t n) {
  if (variant != CATT_VAR_STAGED) return (const void*)syr2k_thread_kernel;
  if (tiled_t2()) return t2_use_mix(n, false) ? (const void*)tile2_mix_kernel<MODE_SYR2K> : (const void*)tile2_kernel<MODE_SYR2K, 8>;
  if (tiled_deep<MODE_SYR2K>() && tiled_minb(true) == 1) return (const void*)tiled_kernel<MODE_SYR2K, 1, 8, false, true>;
  return tiled_func<MODE_SYR2K>();
}

int64_t syr2k_staged_dyn(int64_t n) {
  if (tiled_t2())
    return t2_use_mix(n, false) ? int64_t(T2Cfg<MODE_SYR2K, 8, kMixRows>::SBYTES) : int64_t(T2Cfg<MODE_SYR2K, 8>::SBYTES);
  return (tiled_deep<MODE_SYR2K>() && tiled_minb(true) == 1) ? int64_t(TileCfg<MODE_SYR2K, 8, false, true>::SBYTES) : 0;
}

// ---------------------------------------------------------------- GEMM
// PolyBench/GPU gemm (Table 2 CI group; the cache-insensitive negative
// control): thread (i = by*BY + ty, j = bx*32 + tx),
//   c = C[i][j] * beta; for k: c = fmaf(alpha * a[i][k], b[k][j], c)
// a[i][k] is a broadcast in the warp, b[k][j] coalesced: nothing to throttle.
struct GemmArgs {
  const float* A;
  const float* B;
  float* C;
  int64_t ni, nj, nk;
  float alpha, beta;
  Throttle t;
};

__global__ void __launch_bounds__(1024, 2) gemm_thread_kernel(GemmArgs a) {
  __shared__ int slots;
  gate_init(&slots, a.t);
  __syncthreads();
  cta_enter(a.t);
  const int64_t j = int64_t(blockIdx.x) * 32 + threadIdx.x;
  const int64_t i = int64_t(blockIdx.y) * blockDim.y + threadIdx.y;
  throttled(a.t, &slots, [&]() {
    if (i >= a.ni || j >= a.nj) return;
    const float* __restrict__ ai = a.A + i * a.nk;
    const float* __restrict__ bj = a.B + j;
    float c = __fmul_rn(a.C[i * a.nj + j], a.beta);
#pragma unroll 2
    for (int64_t k = 0; k < a.nk; ++k) c = fmaf(__fmul_rn(a.alpha, ai[k]), bj[k * a.nj], c);
    a.C[i * a.nj + j] = c;
  });
  cta_exit(a.t);
}

// The upper tiles of C = beta C + alpha A A^T (tiles with column block >=
// row block); elements below the diagonal inside diagonal tiles are computed
// too. The caller mirrors the rest (CORR).
catt_status syrk_upper(const float* A, float* C, int64_t n, int64_t m, float alpha, float beta, cudaStream_t s) {
  return launch_tiled<MODE_SYRK>(TileArgs{A, nullptr, C, n, n, m, alpha, beta, 0, 0, 0, 1, {}}, nullptr, s);
}

// CORR's symmat = D^T D over the upper tiles straight from the centred data
// D (nrows x mcols, row-major, pitch mcols): D is already the k-major operand
// of the SYRK over D's columns, so T2 runs without its prep copy, and the
// accumulators start at +0 without reading C (the literal loop's s = 0;
// C need not be initialised). Falls back to syrk_upper's path when T2 cannot
// take D directly (TMA: 16-byte aligned rows).
bool syrk_kmajor_ok(const float* D, int64_t mcols) {
  TileArgs a{D, nullptr, nullptr, mcols, mcols, 1, 1.0f, 0.0f, 0, 0, 0, 1, {}};
  return (reinterpret_cast<uintptr_t>(D) & 15) == 0 && mcols % 4 == 0 && !small_tiles<MODE_SYRK>(mcols, mcols) &&
         t2_ok<MODE_SYRK>(a);
}

catt_status syrk_upper_kmajor(const float* D, const float* Dt, float* C, int64_t mcols, int64_t nrows, cudaStream_t s,
                              bool mirror_diag) {
  TileArgs a{Dt, nullptr, C, mcols, mcols, nrows, 1.0f, 0.0f, 0, 0, 0, 1, {}};
  if (syrk_kmajor_ok(D, mcols) && nrows > 0) {
    a.kmaj = D;
    a.kld = mcols;
    a.zinit = 1;
    a.mirror = mirror_diag ? 1 : 0;
    return launch_t2<MODE_SYRK, 8>(a, nullptr, s);
  }
  if (!Dt) return CATT_EINVAL;                 // the transposed operand is needed off the T2 path
  if (cudaMemsetAsync(C, 0, size_t(mcols) * size_t(mcols) * 4, s) != cudaSuccess) return after_launch();
  return launch_tiled<MODE_SYRK>(a, nullptr, s);
}

const void* gemm_func(int variant) {
  return variant == CATT_VAR_STAGED ? tiled_func<MODE_GEMM>() : (const void*)gemm_thread_kernel;
}

}  // namespace catt

using namespace catt;

extern "C" catt_status catt_syrk(const float* A, float* C, int64_t n, int64_t m, float alpha, float beta,
                                 const catt_throttle* t, void* stream) {
  if (n < 0 || m < 0 || n > (int64_t(1) << 31) || m > (int64_t(1) << 31)) return CATT_EINVAL;
  if (n > 0 && (!C || (m > 0 && !A))) return CATT_EINVAL;  // A is never read when m == 0
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
  if (var == CATT_VAR_STAGED) return launch_tiled<MODE_SYRK>(TileArgs{A, nullptr, C, n, n, m, alpha, beta, 0, 0, 0, 0, {}}, t, s);
  return CATT_EINVAL;
}

extern "C" catt_status catt_syr2k(const float* A, const float* B, float* C, int64_t n, int64_t m, float alpha,
                                  float beta, const catt_throttle* t, void* stream) {
  if (n < 0 || m < 0 || n > (int64_t(1) << 31) || m > (int64_t(1) << 31)) return CATT_EINVAL;
  if (n > 0 && (!C || (m > 0 && (!A || !B)))) return CATT_EINVAL;  // A, B unread when m == 0
  if (n == 0) return CATT_OK;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  Syr2kArgs a{A, B, C, n, m, alpha, beta, Throttle{}};
  const int var = variant_of(t);
  if (var == CATT_VAR_LITERAL) {
    const int threads = cta_threads_or(t, 256);
    if (threads % 32) return CATT_EINVAL;
    const int by = threads / 32;
    size_t dyn = 0;
    catt_status st = prepare_launch((const void*)syr2k_thread_kernel, t, threads, 0, true, &a.t, &dyn);
    if (st != CATT_OK) return st;
    dim3 grid(unsigned((n + 31) / 32), unsigned((n + by - 1) / by));
    if (grid.y > 65535) return CATT_EINVAL;
    syr2k_thread_kernel<<<grid, dim3(32, by), dyn, s>>>(a);
    return after_launch();
  }
  if (var == CATT_VAR_STAGED) return launch_tiled<MODE_SYR2K>(TileArgs{A, B, C, n, n, m, alpha, beta, 0, 0, 0, 0, {}}, t, s);
  return CATT_EINVAL;
}

extern "C" catt_status catt_gemm(const float* A, const float* B, float* C, int64_t ni, int64_t nj, int64_t nk,
                                 float alpha, float beta, const catt_throttle* t, void* stream) {
  if (ni < 0 || nj < 0 || nk < 0 || ni > (int64_t(1) << 31) || nj > (int64_t(1) << 31) || nk > (int64_t(1) << 31))
    return CATT_EINVAL;
  if (ni > 0 && nj > 0 && (!C || (nk > 0 && (!A || !B)))) return CATT_EINVAL;
  if (ni == 0 || nj == 0) return CATT_OK;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  const int var = variant_of(t);
  if (var == CATT_VAR_LITERAL) {
    GemmArgs a{A, B, C, ni, nj, nk, alpha, beta, Throttle{}};
    const int threads = cta_threads_or(t, 256);
    if (threads % 32) return CATT_EINVAL;
    const int by = threads / 32;
    size_t dyn = 0;
    catt_status st = prepare_launch((const void*)gemm_thread_kernel, t, threads, 0, true, &a.t, &dyn);
    if (st != CATT_OK) return st;
    dim3 grid(unsigned((nj + 31) / 32), unsigned((ni + by - 1) / by));
    if (grid.y > 65535) return CATT_EINVAL;
    gemm_thread_kernel<<<grid, dim3(32, by), dyn, s>>>(a);
    return after_launch();
  }
  if (var == CATT_VAR_STAGED) return launch_tiled<MODE_GEMM>(TileArgs{A, B, C, ni, nj, nk, alpha, beta, 0, 0, 0, 0, {}}, t, s);
  return CATT_EINVAL;
}
