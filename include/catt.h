/*
 * catt.h — C ABI of the B200-native CATT hot path.
 *
 * CATT = Compiler-Assisted Thread Throttling (Kim, Hong, Lee, Seo, Han,
 * ICPP 2019). Citations "P:N" are lines of the paper text.
 *
 * Three parts sit behind this boundary:
 *   1. the footprint analyser (host only): occupancy and carveout (Eq 1-4,
 *      P:183-208), locality and lines per warp (Eq 5-7), footprint
 *      and throttle factors (Eq 8-9);
 *   2. hand-written sm_100a kernels for the loop families of Table 2/3
 *      (ATAX, BICG, MVT, GESUMMV, SYRK, KMEANS-assign), each with an explicit
 *      throttle: a per-CTA warp-gating semaphore in shared memory (the B200
 *      form of Fig 4's warp-level throttling) and a per-SM CTA cap
 *      (the B200 form of Fig 5's TB-level throttling);
 *   3. helpers for measurement: the seeded input generator, the L1D capacity
 *      probe (Fig 3 analog).
 *
 * Conventions (all entry points):
 *   - extern "C", plain pointers and sizes; no exceptions cross the boundary.
 *   - Device pointers are owned by the caller (the Python layer allocates them
 *     with PyTorch). The library never frees caller memory. Its only state is
 *     a per-device cache (hardware table, kernel attributes), a per-device
 *     array of num_sms int32 counters for the per-SM CTA cap plus a grid
 *     barrier word (allocated on first use, left zero by every kernel that
 *     uses them), and a grow-only workspace for the FUSED variant's partials.
 *   - Kernel entry points are asynchronous on `stream` (a cudaStream_t passed
 *     as void*; NULL = legacy default stream). Nothing synchronises.
 *   - Arguments are validated synchronously before any launch; invalid input
 *     returns CATT_EINVAL and launches nothing. A launch failure returns
 *     CATT_ECUDA (catt_last_cuda_error() gives the cudaError_t value).
 *   - An unresolvable footprint is a result flag, not an error.
 *   - fp32 row-major matrices; inputs and outputs must not alias.
 *   - CTA caps that use the per-SM counters assume capped kernels on one
 *     device do not run concurrently on different streams. The same holds
 *     for FUSED launches (catt_dual*, catt_atax_peer): they share the
 *     device's workspace and its grid-barrier / arrival-counter words, whose
 *     expected values the library tracks per device in launch order (a
 *     stream-captured single-read launch uses the self-resetting barrier
 *     instead, so CUDA graphs replay correctly).
 */
#ifndef CATT_H
#define CATT_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  CATT_OK = 0,
  CATT_EINVAL = -1,       /* bad argument or throttle (nothing launched)   */
  CATT_ECUDA = -2,        /* CUDA runtime error (see catt_last_cuda_error)  */
  CATT_EUNSUPPORTED = -3, /* valid but not supported (e.g. window too big)  */
  CATT_ENOMEM = -4,       /* library workspace allocation failed            */
  CATT_ENODEV = -5,       /* no CUDA device                                 */
  CATT_EINEXACT = -6      /* KMEANS sums: a value outside the exact range   */
} catt_status;

enum { CATT_MAX_LOOPS = 4, CATT_MAX_CARVEOUTS = 16 };

/* catt_ref.flags */
enum {
  CATT_REF_IRREGULAR = 1, /* indirect access: C_tid := 1                      */
  CATT_REF_STORE = 2,     /* store: counted in paper mode, not in union mode          */
  CATT_REF_NOT_L1 = 4     /* register / shared memory / L1-bypassing: not counted     */
};

/* catt_loop_desc.mode */
enum {
  CATT_MODE_UNION = 0, /* B200 default: exact distinct lines of co-resident warps */
  CATT_MODE_PAPER = 1  /* Eq 7-9 as printed: per-warp sum of REQ_warp            */
};

/* catt_footprint_result.flags */
enum {
  CATT_FIT_NONE_NEEDED = 1, /* fits at full TLP, or the loop has no locality */
  CATT_FIT_WARP = 2,        /* warp-level throttle (N of Eq 9)                         */
  CATT_FIT_CTA = 4,         /* TB-level throttle (M of Eq 9), one warp per CTA          */
  CATT_FIT_UNRESOLVABLE = 8, /* nothing fits even at (1,1): left unthrottled    */
  CATT_FIT_GUARDED = 16      /* a B200 guard (divergence / TLP floor) limited the throttle */
};

/* One memory instruction in the loop (Eq 5):
 *   element index = base + sum_d c_gid[d] * gid_d + sum_k c_iter[k] * i_k
 * gid_d = blockIdx_d * blockDim_d + threadIdx_d (the paper's C_tid is c_gid[0]
 * for 1-D blocks); i_k are the loop induction variables, outer to inner
 * (C_i). Arrays are assumed to start on a line boundary; refs with the same
 * array_id address the same array (their lines are shared). */
typedef struct {
  int64_t c_gid[3];
  int64_t c_iter[CATT_MAX_LOOPS];
  int64_t base;
  int32_t elem_bytes;
  int32_t flags;
  int32_t array_id;
  int32_t reserved_;
} catt_ref;

/* A loop and its launch. trip[k] = iterations of loop k (outer to inner).
 * extent[d] > 0 bounds gid_d (threads with gid_d >= extent[d] do not access,
 * the usual `if (i < N)` guard). regs_per_thread / smem_per_cta come from the
 * compiled kernel (0 = no limit). force_carveout_kb >= 0 pins the shared
 * memory option ("we configured the L1D to 32KB"); < 0 chooses it by
 * Eq 4. */
typedef struct {
  int32_t n_refs;
  int32_t n_loops;
  const catt_ref* refs;
  int64_t trip[CATT_MAX_LOOPS];
  int32_t block[3];
  int32_t mode;
  int64_t grid[3];
  int64_t extent[3];
  int32_t regs_per_thread;
  int32_t smem_per_cta;
  int32_t force_carveout_kb;
  int32_t reserved_;
} catt_loop_desc;

/* Hardware parameters. carveout_kb[i] are the configurable shared-memory
 * sizes per SM (ascending); l1d_bytes[i] the L1D capacity that option leaves
 * (measured on B200, see catt_hw_b200); carveout_pct[i] the
 * cudaFuncAttributePreferredSharedMemoryCarveout value that selects it.
 * min_warps_sm / divergent_lines / min_retouch / min_reuse_trip are the B200
 * guards of union mode (0 = off; readings R18, R23): a loop is
 * throttled only if one of its reused references touches >= divergent_lines
 * lines per warp request, re-touches its line >= min_retouch times per thread
 * (line / (|C_i| * elem_bytes), capped by the trip count; an outer-level reuse
 * counts its trip count) and reuses in a loop of >= min_reuse_trip
 * iterations; and never to fewer than min_warps_sm active warps per SM.
 * max_stream_pct (R24; 0 = off, <= 100): no throttle when more than that
 * percentage of a lane's bytes per iteration are streams L1 cannot serve
 * again (stores, loads without reuse). cta_fallback (R27; 0 = off): when
 * nothing at or above min_warps_sm fits and an SM holds several CTAs (T >= 2),
 * cap whole CTAs -- (W, m) with the smallest m such that min_warps_sm <= W m
 * <= 2 min_warps_sm -- instead of gating warps down to the floor.
 * stream_floor (R29; 0 = off): with one CTA per SM (T = 1) and S >= 2
 * memory-divergent reused loads (each meeting the divergent_lines /
 * min_retouch / min_reuse_trip terms), the floor is ceil(min_warps_sm / S):
 * S streams per warp keep as many lines in flight as S times the warps.
 * private_streams (R32; 0 = off): a memory-divergent reused load whose first
 * warp request touches the same lines in warp 1 as in warp 0 of CTA 0 (the
 * lines are shared by the CTA's warps, e.g. SYRK's a[j][k] in a 32 x 8 block)
 * counts neither as divergent nor as a stream.
 * Paper mode ignores them. */
typedef struct {
  int32_t num_sms, max_warps_sm, max_ctas_sm, regs_sm, reg_alloc_unit, warp_size;
  int32_t smem_alloc_unit, reserved_smem_cta, line_bytes, n_carveouts;
  int32_t min_warps_sm, divergent_lines;
  int32_t min_retouch, min_reuse_trip, max_stream_pct, cta_fallback;
  int32_t stream_floor, private_streams;
  int32_t carveout_kb[CATT_MAX_CARVEOUTS];
  int32_t carveout_pct[CATT_MAX_CARVEOUTS];
  int64_t l1d_bytes[CATT_MAX_CARVEOUTS];
} catt_hw;

typedef struct {
  int64_t lines_per_warp_iter; /* sum over refs of lines warp 0 touches in iteration 0 (Eq 7) */
  int64_t reuse_span;          /* lines warp 0 retains until reuse                             */
  int64_t footprint_lines_full;/* F(#Warps_TB, #TB_SM), Eq 8                                    */
  int64_t footprint_lines;     /* F at the chosen (active_warps, active_ctas), Eq 9            */
  int64_t footprint_bytes;     /* footprint_lines * line_bytes                                  */
  int64_t l1d_bytes;           /* L1D left by the chosen carveout                               */
  int32_t base_warps, base_ctas;     /* (#Warps_TB, #TB_SM) at full TLP, Eq 1-3                */
  int32_t active_warps, active_ctas; /* the throttle: warps per CTA, CTAs per SM                */
  int32_t carveout_kb;               /* Eq 4 (or forced)                                        */
  int32_t flags;                     /* CATT_FIT_*                                              */
} catt_footprint_result;

/* Kernel variants (all compute the same loop):
 *   LITERAL  the paper's loop: one thread per output, scalar loads through L1,
 *            sequential order (bit-exact to the sequential-fmaf oracle).
 *   VEC4     one thread per output, 16-byte loads, same sequential order.
 *   STAGED   one thread per output, tiles moved to shared memory by
 *            cp.async.bulk (TMA bulk copies), same sequential order; does not
 *            rely on L1 reuse.
 *   COOP     warp-cooperative coalesced loads with shuffle/split reductions:
 *            the HBM-roofline variant; summation order differs (fp64-oracle
 *            tolerance, bit-exact on exact-dyadic inputs).
 *   REGS     (KMEANS) the point's features are loaded once into registers.
 *   BYPASS   (row loops) the literal loop with L2-only (ld.global.cg) matrix
 *            loads: the divergent rows never occupy L1, nothing to throttle
 *            (the bypass alternative of P:137).
 *   FUSED    (ATAX/BICG/MVT, set on k1) both loops in one pass over A: each
 *            row is read once, its dot product finished in the CTA, its A^T
 *            contribution accumulated; A^T partials reduced in band order
 *            after a grid barrier (cooperative launch). Same bar as COOP.  */
enum { CATT_VAR_LITERAL = 0, CATT_VAR_VEC4 = 1, CATT_VAR_STAGED = 2, CATT_VAR_COOP = 3, CATT_VAR_REGS = 4,
       CATT_VAR_FUSED = 5, CATT_VAR_BYPASS = 6 };

/* Warp-level mechanism: SEMAPHORE = per-CTA counting semaphore in shared
 * memory (a finished warp's slot goes to the next waiting warp);
 * BARRIER = Fig 4 literally (warp groups run in turn between __syncthreads). */
enum { CATT_GATE_SEMAPHORE = 0, CATT_GATE_BARRIER = 1 };
/* CTA-level mechanism: SM_COUNTER = per-SM counter in global memory (exact
 * cap whatever the driver's carveout choice); SMEM_PAD = Fig 5 literally
 * (dynamic shared memory pad sized so only active_ctas fit the carveout). */
enum { CATT_CAP_SM_COUNTER = 0, CATT_CAP_SMEM_PAD = 1 };

/* Launch + throttle of one loop. Zero-initialised = default launch (256
 * threads, LITERAL, no throttle, carveout preference 0 %). */
typedef struct {
  int32_t cta_threads;  /* threads per CTA (multiple of 32, <= 1024); 0 = 256; SYRK: 2-D 32 x (cta_threads/32) */
  int32_t active_warps; /* warps of a CTA allowed in the loop at once; 0 = all (#Warps_TB)                   */
  int32_t active_ctas;  /* CTAs of an SM allowed in the loop at once; 0 = no cap                            */
  int32_t carveout_kb;  /* shared-memory option to request; 0 = max L1D; < 0 = leave the driver default      */
  int32_t variant;      /* CATT_VAR_*                                                                          */
  int32_t gate;         /* CATT_GATE_*                                                                         */
  int32_t cap;          /* CATT_CAP_*                                                                          */
  int32_t reserved_;
  uint64_t* probe;      /* optional device buffer: per warp {smid, t_start_ns, t_end_ns} around the loop,
                           indexed by (linear CTA id * warps per CTA + warp) * 3; NULL = off             */
} catt_throttle;

/* Loop identifiers for catt_kernel_desc / catt_plan: one per loop of Table 3. */
enum {
  CATT_K_ATAX_1 = 0,  /* tmp = A x        (row per thread, memory-divergent)  */
  CATT_K_ATAX_2 = 1,  /* y = A^T tmp      (column per thread, coalesced)      */
  CATT_K_BICG_1 = 2,  /* s = A^T r        (column per thread)                 */
  CATT_K_BICG_2 = 3,  /* q = A p          (row per thread)                    */
  CATT_K_MVT_1 = 4,   /* x1 += A y1       (row per thread)                    */
  CATT_K_MVT_2 = 5,   /* x2 += A^T y2     (column per thread)                 */
  CATT_K_GESUMMV = 6, /* y = alpha A x + beta B x (row per thread, 2 matrices)*/
  CATT_K_SYRK = 7,    /* C = beta C + alpha A A^T (2-D block 32 x 8)          */
  CATT_K_KMEANS = 8,  /* membership = argmin_c |f_p - c|^2, feature-major     */
  CATT_K_SYR2K = 9,   /* C = beta C + alpha (A B^T + B A^T), 2-D block 32 x 8 */
  CATT_K_KMEANS_T = 10, /* KM transpose: out[f*ld + p] = in[p*nf + f]          */
  CATT_K_CORR = 11,   /* CORR loop: symmat[j1][j2] = sum_i d[i][j1] d[i][j2]   */
  CATT_K_GEMM = 12,   /* C = beta C + alpha A B, 2-D block 32 x 8 (CI control) */
  CATT_K_ROWS3 = 13,  /* y = A x + B x + C x, thread per row (three divergent streams; rule studies) */
  CATT_K_COUNT = 14
};

/* Problem sizes: ATAX/BICG m x n (rows, cols); MVT/GESUMMV n (m ignored);
 * SYRK/SYR2K n x n output, k = inner size m; GEMM m = ni, n = nj, k = nk;
 * CORR n = columns m, k = rows n; KMEANS m = npoints, n = nfeatures,
 * k = clusters, ld = feature-major leading dimension. */
typedef struct {
  int32_t loop;
  int32_t reserved_;
  int64_t m, n, k, ld;
} catt_problem;

/* ------------------------------------------------------------------ hardware */
/* Device properties + the L1D table of catt_hw_b200 (CATT_ENODEV without a GPU). */
catt_status catt_hw_query(int device, catt_hw* out);
/* B200 (sm_100a, 148 SMs) with the L1D capacities measured per carveout option
 * by the Fig 3-style footprint sweep (profiles/round1_probe_hw.txt), and the
 * B200 rule on: min_warps_sm 8, divergent_lines 8, min_retouch 16,
 * min_reuse_trip 0, max_stream_pct 25, cta_fallback 1, stream_floor 1,
 * private_streams 1 (R18-R32). No GPU needed. */
catt_status catt_hw_b200(catt_hw* out);
/* Titan V, the paper's GPU: Table 1, 64 warps/SM, shared
 * memory options 0/8/16/32/64/96 KB with L1D = 128 KB - option. */
catt_status catt_hw_titanv(catt_hw* out);

/* ------------------------------------------------------------------ analyser */
/* Steps a1-a5 (Eq 1-9). Host only, no device work; deterministic. */
catt_status catt_footprint(const catt_loop_desc* desc, const catt_hw* hw, catt_footprint_result* out);

/* The descriptor of this library's kernel for one loop of `prob` under the
 * launch in `t` (cta_threads, variant; throttle fields ignored). refs_buf must
 * hold `cap` refs (8 is enough for every loop). regs_per_thread comes from
 * cudaFuncGetAttributes when a device is present, else 0 (unknown). */
catt_status catt_kernel_desc(const catt_problem* prob, const catt_throttle* t, int32_t mode,
                             catt_loop_desc* out, catt_ref* refs_buf, int32_t cap);

/* catt_kernel_desc + catt_footprint, and the throttle to launch with: `out` =
 * `launch` with active_warps / active_ctas / carveout_kb set to the CATT pick. */
catt_status catt_plan(const catt_problem* prob, const catt_throttle* launch, const catt_hw* hw, int32_t mode,
                      catt_throttle* out, catt_footprint_result* res);

/* ------------------------------------------------------------------ kernels */
/* ATAX (Table 3): tmp = A x (loop 1, throttle k1), then
 * y = A^T tmp (loop 2, throttle k2). A is m x n; x[n], tmp[m], y[n] device
 * pointers; tmp and y are overwritten. For a row shard, y is the shard's
 * partial A_g^T tmp_g (the caller all-reduces). */
catt_status catt_atax(const float* A, const float* x, float* tmp, float* y, int64_t m, int64_t n,
                      const catt_throttle* k1, const catt_throttle* k2, void* stream);

/* ATAX's two literal loops in ONE kernel with a warp-level throttle per loop
 * (throttling applied "to individual loops in a kernel"; PF#1's
 * loops take different factors): loop 1 (thread per row, tmp = A x) runs
 * under k1->active_warps, then a grid barrier, then loop 2 (thread per
 * column, y = A^T tmp) under k2->active_warps. The CTA size, carveout, CTA
 * cap (one decision for the whole kernel; applied around each loop)
 * and probe come from k1; k2 may only set active_warps and gate (a k2
 * cta_threads or active_ctas that differs from k1's is CATT_EINVAL). LITERAL
 * only; cooperative launch of ceil(max(m, n) / cta_threads) CTAs, which must
 * all be resident (CATT_EUNSUPPORTED otherwise). Results bit-exact to the
 * sequential oracle, as catt_atax's literal loops. */
catt_status catt_atax_onekernel(const float* A, const float* x, float* tmp, float* y, int64_t m, int64_t n,
                                const catt_throttle* k1, const catt_throttle* k2, void* stream);

/* BICG (Table 2, Table 3): s = A^T r (loop 1, k1) and q = A p
 * (loop 2, k2). A is nx x ny; p[ny], r[nx], q[nx], s[ny]; q, s overwritten. */
catt_status catt_bicg(const float* A, const float* p, const float* r, float* q, float* s, int64_t nx, int64_t ny,
                      const catt_throttle* k1, const catt_throttle* k2, void* stream);

/* MVT (Table 2, Table 3): x1 += A y1 (loop 1, k1) and
 * x2 += A^T y2 (loop 2, k2). A is n x n; x1, x2 in/out. */
catt_status catt_mvt(const float* A, const float* y1, const float* y2, float* x1, float* x2, int64_t n,
                     const catt_throttle* k1, const catt_throttle* k2, void* stream);

/* GESUMMV (Table 2, Table 3): tmp = A x, y = alpha*tmp + beta*(B x)
 * in one loop over j. A, B n x n; x[n]; y[n], tmp[n] overwritten. */
catt_status catt_gesummv(const float* A, const float* B, const float* x, float* y, float* tmp, int64_t n,
                         float alpha, float beta, const catt_throttle* t, void* stream);

/* SYRK (Table 2): C = beta*C + alpha*A*A^T over the full n x n square.
 * A is n x m; C in/out. LITERAL = 2-D block 32 x (cta_threads/32), one thread
 * per C element; STAGED = shared-memory tiles, register blocking, same k order.
 * STAGED with at least one tile per SM (T2) first writes A^T
 * and (alpha*A)^T (one copy when alpha == 1) into a workspace taken from the
 * device's default memory pool, stream-ordered on `stream` (cudaMallocAsync,
 * released by cudaFreeAsync after the launch; the pool keeps it for reuse):
 * 2*n*m floats. If that allocation fails the library runs its round-1 tiled
 * kernel instead, which needs no workspace (same results, slower). */
catt_status catt_syrk(const float* A, float* C, int64_t n, int64_t m, float alpha, float beta,
                      const catt_throttle* t, void* stream);

/* SYR2K (Table 2, Table 3; the paper's 2-D cache-sensitive kernel):
 * C = beta*C + alpha*(A B^T + B A^T) over the full square, A and B n x m,
 * C in/out. Per element, k ascending: p = alpha*a_ik, q = alpha*b_ik,
 * s = fmaf(p, b_jk, q*a_jk), c = c + s (every intermediate rounded; DESIGN.md
 * R20). LITERAL = 2-D block 32 x (cta_threads/32); STAGED = shared-memory
 * tiles with the same order; its workspace as catt_syrk's with B too:
 * 4*n*m floats (2*n*m when alpha == 1). */
catt_status catt_syr2k(const float* A, const float* B, float* C, int64_t n, int64_t m, float alpha, float beta,
                       const catt_throttle* t, void* stream);

/* GEMM (Table 2 CI group; the cache-insensitive negative control):
 * C (ni x nj, in/out) = beta*C + alpha*A*B, A ni x nk, B nk x nj, row-major.
 * Per element, k ascending: c = fmaf(alpha*a_ik, b_kj, c) (alpha*a_ik rounded).
 * LITERAL = 2-D block 32 x (cta_threads/32); STAGED = the tiled kernel. */
catt_status catt_gemm(const float* A, const float* B, float* C, int64_t ni, int64_t nj, int64_t nk, float alpha,
                      float beta, const catt_throttle* t, void* stream);

/* CORR (Table 2; Table 3; the give-up case of P:244):
 * Pearson correlation of the m columns of data (n x m, row-major). data is
 * centred and scaled in place; mean[m], stdv[m] and symmat[m x m] are
 * outputs (R22 gives the per-column order, fn = n, eps = 0.005).
 * LITERAL: thread per column for the statistics, then the paper's loop
 * (thread per j1; the throttle applies to it, CATT_K_CORR). STAGED: work is
 * a device buffer of m*n floats (the transposed columns) and symmat is
 * computed by the tiled SYRK kernel: bit-identical to LITERAL. */
catt_status catt_corr(float* data, int64_t n, int64_t m, float* mean, float* stdv, float* symmat, float* work,
                      const catt_throttle* t, void* stream);

/* KMEANS assignment (Table 2, Table 3): feat is feature-major,
 * feat[f*ld + p] for f < nf, p < npoints (ld >= npoints); clusters is k x nf;
 * membership[npoints] int32 overwritten with the lowest-index nearest centre.
 * Requires nf * k <= 4096 (the centres are staged in shared memory). */
catt_status catt_kmeans_assign(const float* feat, int64_t ld, int64_t npoints, int32_t nf, const float* clusters,
                               int32_t k, int32_t* membership, const catt_throttle* t, void* stream);

/* ------------------------------------------------------------------ KMEANS iteration
 * the steps around the assignment (Rodinia kmeans; the KM
 * rows of Table 3 P:338-339 are its two loops). DESIGN.md reading R21.
 *
 * Transpose (KM's other loop): out[f*ld + p] = in[p*nf + f] for p < npoints,
 * f < nf; in is point-major (npoints x nf), out feature-major with ld >=
 * npoints (columns >= npoints untouched). Variants: LITERAL (thread per
 * point, the divergent CATT loop CATT_K_KMEANS_T, throttle honoured) and COOP
 * (256-point shared-memory tiles, coalesced; no throttle). Bit-exact copy.
 *
 * Exact centroid sums. acc is a device int64 array of
 * catt_kmeans_acc_words(k, nf) = 4*k*nf + k + 3 words:
 *   acc[(c*nf + f)*4 + l], l < 4  limbs of the sum, over the points assigned to
 *                                 c, of feature f as the two's-complement
 *                                 128-bit integer v = x * 2^64. Each 128-bit
 *                                 partial is split v = l0 + l1*2^32 + l2*2^64 +
 *                                 l3*2^96 (l0..l2 unsigned 32-bit chunks, l3 a
 *                                 signed 32-bit chunk) and chunk l is added to
 *                                 limb l. The sum is S = sum_l acc[..+l]*2^(32l).
 *   acc[4*k*nf + c]               points assigned to c
 *   acc[4*k*nf + k]               delta: points whose membership changed
 *   acc[4*k*nf + k + 1]           inexact: feature values not representable
 *                                 (non-zero bits below 2^-64, |x| >= 2^31,
 *                                 subnormal, inf, NaN); 0 means S is exact
 *   acc[4*k*nf + k + 2]           arrival counter of catt_kmeans_step's last-CTA
 *                                 finalize (0 between launches; the launch that
 *                                 uses it resets it). Kept in the caller's acc
 *                                 so concurrent steps on different acc arrays
 *                                 (streams) never share a counter.
 * All limbs are integer sums, so adding acc arrays (e.g. an integer
 * all-reduce across GPUs, each holding a shard of the points) gives exactly
 * the acc of the whole point set. Limits: nf <= 64, k <= 16, npoints < 2^31. */
int64_t catt_kmeans_acc_words(int32_t k, int32_t nf);
catt_status catt_kmeans_transpose(const float* in, float* out, int64_t npoints, int32_t nf, int64_t ld,
                                  const catt_throttle* t, void* stream);

/* One pass over the points: assignment exactly as catt_kmeans_assign (reading
 * membership's previous value first: -1 = none), then acc += the point's
 * features into its centre's sums, counts and delta. acc is accumulated into
 * (zero it before the first pass). */
catt_status catt_kmeans_accumulate(const float* feat, int64_t ld, int64_t npoints, int32_t nf,
                                   const float* clusters, int32_t k, int32_t* membership, int64_t* acc,
                                   void* stream);

/* clusters[c][f] = round-to-nearest-even fp32 of (S * 2^-64) / count[c] when
 * count[c] > 0, else unchanged (a centre without points keeps its value).
 * stats (device int64[3], may be NULL) receives {delta, inexact, sum of
 * counts}. zero_acc != 0 zeroes acc afterwards (ready for the next pass). */
catt_status catt_kmeans_finalize(int64_t* acc, int32_t k, int32_t nf, float* clusters, int64_t* stats,
                                 int32_t zero_acc, void* stream);

/* One k-means iteration on one GPU in ONE launch: catt_kmeans_accumulate,
 * then (the last CTA to finish, after every CTA's exact sums are in acc) the
 * work of catt_kmeans_finalize with zero_acc = 1. Bit-identical to the two
 * calls. stats (device int64[3], may be NULL) as in catt_kmeans_finalize.
 * Not for sharded runs: there the sums are all-reduced between the two.
 * Concurrent steps (different streams) must use different acc arrays. */
catt_status catt_kmeans_step(const float* feat, int64_t ld, int64_t npoints, int32_t nf, float* clusters, int32_t k,
                             int32_t* membership, int64_t* acc, int64_t* stats, void* stream);

/* The k-means loop on one GPU: membership := -1, then up to max_iter
 * iterations of catt_kmeans_step (one launch each); stops after the first iteration whose
 * delta <= max_changes. clusters (k x nf, in: initial centres, out: final).
 * ws: device int64 workspace of catt_kmeans_acc_words(k, nf) + 4 words.
 * Iterations are queued without host round trips (a device-side done flag
 * turns the remaining queued passes into no-ops); the call synchronizes the
 * stream and writes the iteration count to *iterations (host, may be NULL).
 * Returns CATT_EINEXACT when any sum was not exact. */
catt_status catt_kmeans(const float* feat, int64_t ld, int64_t npoints, int32_t nf, float* clusters, int32_t k,
                        int32_t* membership, int32_t max_iter, int64_t max_changes, int64_t* ws,
                        int32_t* iterations, void* stream);

/* ------------------------------------------------------------------ single loops
 * CATT throttles per loop: these run one loop each and
 * are what the application entry points above are made of.
 *
 * Row loop (ATAX#1, BICG#2, MVT#1, GESUMMV; memory-divergent): for i < m,
 *   mode CATT_ROWS_STORE:   y[i] = sum_j A[i*n + j] * x[j]
 *   mode CATT_ROWS_ACCUM:   y[i] = y[i] + sum_j A[i*n + j] * x[j]   (y in/out)
 *   mode CATT_ROWS_GESUMMV: tmp[i] = sum_j A[i*n+j] x[j];
 *                           y[i] = alpha*tmp[i] + beta*sum_j B[i*n+j] x[j]
 *   mode CATT_ROWS_SUM3:    y[i] = (sA + sB) + sC, sX = sum_j X[i*n + j] * x[j]
 *                           each by fmaf in j order; B holds the m x n matrices
 *                           B and C back to back (2 m n floats); LITERAL only.
 *                           Three memory-divergent streams per thread: the
 *                           loop the decision-rule studies use (DESIGN R29).
 * B and tmp are used only by CATT_ROWS_GESUMMV (B also by CATT_ROWS_SUM3;
 * else may be NULL).
 * Column loop (ATAX#2, BICG#1, MVT#2; coalesced): for j < n,
 *   y[j] = (accumulate ? y[j] : 0) + sum_i A[i*n + j] * v[i].
 * A is m x n row-major in both. */
enum { CATT_ROWS_STORE = 0, CATT_ROWS_ACCUM = 1, CATT_ROWS_GESUMMV = 2, CATT_ROWS_SUM3 = 3 };
catt_status catt_rows(const float* A, const float* B, const float* x, float* y, float* tmp, int64_t m, int64_t n,
                      float alpha, float beta, int32_t mode, const catt_throttle* t, void* stream);
catt_status catt_cols(const float* A, const float* v, float* y, int64_t m, int64_t n, int32_t accumulate,
                      const catt_throttle* t, void* stream);

/* Both loops of an application in one pass over A (the FUSED variant; SURVEY
 * 8(f) f4): yr (+)= A xr (row loop) and yc (+)= A^T v with v = xc, or v = the
 * finished yr when `dependent` (ATAX: y = A^T (A x)). row_/col_accumulate make
 * yr / yc in/out. A is m x n row-major, n % 4 == 0, n <= 16384, 16-B aligned
 * A and xr. Uses the library's per-device workspace (grid x n floats) and a
 * cooperative launch; t must not request a throttle (CATT_EINVAL). */
catt_status catt_dual(const float* A, const float* xr, const float* xc, float* yr, float* yc, int64_t m, int64_t n,
                      int32_t row_accumulate, int32_t col_accumulate, int32_t dependent, const catt_throttle* t,
                      void* stream);

/* Several independent dual problems with the same n in one grouped launch
 * (up to 4; e.g. BICG and MVT of one step): one longer stream instead of
 * several short ones. Semantics per problem as catt_dual; `dependent` applies
 * to all of them. */
typedef struct {
  const float* A;
  const float* xr;
  const float* xc;
  float* yr;
  float* yc;
  int64_t m, n;
  int32_t row_accumulate, col_accumulate;
} catt_dual_problem;
catt_status catt_dual_group(const catt_dual_problem* probs, int32_t count, int32_t dependent, const catt_throttle* t,
                            void* stream);

/* ------------------------------------------------------------------ helpers */
/* dst[i] = value(seed, offset + i): the counter-based generator of
 * seeded_inputs.py (mode 0 uniform [0,1), 1 dyadic k/16). Device pointer. */
catt_status catt_fill_hash(float* dst, int64_t n, uint32_t seed, uint64_t offset, int32_t mode, void* stream);

/* Fig 3 analog: one thread chases a cyclic chain of `kb` KiB (one
 * load per 128-B line) under carveout preference `pct`, 4 passes; writes the
 * mean cycles per load for each size. Synchronous. */
catt_status catt_calibrate_l1(int device, int32_t pct, const int32_t* kb, int32_t n, float* cycles_out);

/* Number of registers / static shared bytes of the kernel a loop+launch uses. */
catt_status catt_kernel_attrs(const catt_problem* prob, const catt_throttle* t, int32_t* regs, int32_t* static_smem);

/* Eq 1-3 as the CUDA runtime computes it, for pinning the
 * analyser's a1 step: cudaOccupancyMaxActiveBlocksPerMultiprocessor for the
 * kernel a loop+launch uses, with that launch's CTA size and dynamic shared
 * memory plus `extra_dyn_smem` bytes (a Fig 5 style pad), evaluated at the
 * largest shared-memory carveout (Eq 1 divides the maximum shared memory; the
 * function's carveout preference is restored afterwards). No grid bound.
 * *ctas_per_sm receives the count; *dyn_smem (may be NULL) the dynamic bytes
 * used. Synchronous, no launch. EINVAL on bad arguments, ECUDA on a runtime
 * error. */
catt_status catt_kernel_occupancy(const catt_problem* prob, const catt_throttle* t, int64_t extra_dyn_smem,
                                  int32_t* ctas_per_sm, int64_t* dyn_smem);

const char* catt_status_str(catt_status s);
int catt_last_cuda_error(void);
/* ------------------------------------------------------------ multi-GPU
 * Row-sharded ATAX with the A^T partial sums all-reduced inside the fused
 * kernel through peer memory (the row-sharded step of 8(e)
 * with NCCL's all-reduce replaced by stores into the other ranks' buffers
 * over NVLink). One process per GPU; world <= 8 ranks of one NVLink domain.
 *
 * catt_peer_create allocates this rank's buffer (receive slots and flags for
 * n columns, cudaMalloc, owned by the object) and writes its CUDA IPC handle
 * (CATT_PEER_HANDLE_BYTES bytes) to host memory `handle`. The caller ships
 * the handles between ranks (e.g. all_gather_object) and calls
 * catt_peer_open once per other rank. catt_atax_peer then computes, on every
 * rank g, tmp_g = A_g x (rows of this shard, m x n row-major) and the full
 * y = sum over ranks of A_g^T tmp_g, summed in rank order in the kernel, so
 * every rank holds bit-identical y. All ranks must call it in the same order
 * with equal shapes (equal shards give equal grids); each call is one launch
 * on `stream`, asynchronous. A wait for a peer longer than 10 s makes the
 * kernel give up; a peer whose launch has another grid size (shards of
 * different row counts below the co-resident CTA count) is detected at its
 * first flag and the kernel gives up too (its column outputs are then
 * undefined). catt_peer_check (synchronous) reports the error word:
 * *timed_out = 0 (none), 1 (a wait timed out), 2 (grid mismatch between
 * ranks); the word stays set until the peer object is destroyed. Results: within
 * 1e-5 of fp64, bit-exact on exact-dyadic inputs (the FUSED bar). Errors: CATT_EINVAL (arguments, a peer not opened, grids over
 * 1024 CTAs), CATT_ECUDA (IPC or launch), CATT_EUNSUPPORTED (n > 16384). */
enum { CATT_PEER_HANDLE_BYTES = 64 };
typedef struct catt_peer catt_peer;
catt_status catt_peer_create(int32_t world, int32_t rank, int64_t n, catt_peer** out, void* handle);
catt_status catt_peer_open(catt_peer* p, int32_t peer_rank, const void* handle);
catt_status catt_peer_check(catt_peer* p, int32_t* timed_out);
catt_status catt_peer_destroy(catt_peer* p);
catt_status catt_atax_peer(const float* A, const float* x, float* tmp, float* y, int64_t m, int64_t n, catt_peer* p,
                           void* stream);

/* The same peer state over memory the caller maps (the
 * NVSwitch form): symmetric memory in which every rank's buffer is mapped
 * into every process (e.g. torch.distributed._symmetric_memory
 * `buffer_ptrs`), optionally with a multicast alias of those buffers bound
 * to an NVLS multicast object (`multicast_ptr`). bases[r] is rank r's buffer
 * as mapped in this process, each catt_peer_bytes(world, n) bytes, 256-byte
 * aligned and zero-filled before the first launch; the caller keeps them
 * mapped until catt_peer_destroy (the library frees nothing of them).
 * mc_base: the multicast alias (256-byte aligned) or NULL. With mc_base
 * each column partial and each flag is one multimem.st (the NVSwitch
 * replicates it to every rank) instead of one store per rank; without it
 * the kernel stores to every rank through bases[] as with CUDA IPC. The sums
 * are read from this rank's own buffer in rank order either way, so results
 * are the same bits as catt_peer_create's. catt_peer_open is not used
 * (CATT_EINVAL). Errors: CATT_EINVAL (arguments, misaligned bases). */
int64_t catt_peer_bytes(int32_t world, int64_t n);
catt_status catt_peer_create_mapped(int32_t world, int32_t rank, int64_t n, void* const* bases, void* mc_base,
                                    catt_peer** out);

/* ------------------------------------------------------------ SM partition
 * A stream whose kernels run on a partition of the device's SMs (a CUDA green
 * context, driver 12.4+). SURVEY 8(d) [3]: CTA-level throttling (Fig 5,
 * P:295-322) needs several co-resident CTAs per SM, which GESUMMV 8192's 32
 * CTAs of 256 threads only get on a few SMs; the partition reproduces the
 * paper's #TB_SM > 1 regime (Eq 3) on B200. `min_sms` is rounded up by
 * the driver to its partition granularity; *sms_out receives the partition's
 * SM count (plan with catt_hw.num_sms = *sms_out). The stream is owned by the
 * library until catt_sm_partition_destroy; device memory of the primary
 * context is usable on it. Errors: CATT_EINVAL (min_sms < 1 or above the
 * device's count, null outputs), CATT_EUNSUPPORTED (driver without green
 * contexts), CATT_ECUDA (driver call failed). */
catt_status catt_sm_partition_create(int device, int32_t min_sms, void** stream_out, int32_t* sms_out);
catt_status catt_sm_partition_destroy(void* stream);

/* Row-sharded BICG / MVT (any group of independent single-read problems, as
 * catt_dual_group with dependent = 0) with every problem's column outputs
 * all-reduced across ranks inside the kernel through the same peer memory
 * (s = sum over ranks of A_g^T r_g, x2 = x2 + sum over ranks of
 * A_g^T y2_g). On rank g each problem holds the rank's rows A_g (m x n); row
 * outputs (q, x1) stay rank-local; column outputs are summed over ranks in
 * rank order and then, for col_accumulate, added to the initial value (which
 * must be the same on every rank), so every rank holds bit-identical columns.
 * `p` must have been created with n = problems' n x count. Same calling rules,
 * asynchrony, give-up and error codes as catt_atax_peer. */
catt_status catt_dual_group_peer(const catt_dual_problem* probs, int32_t count, catt_peer* p, void* stream);

/* Diagnostics: the FUSED single-read kernel records, when the environment
 * variable CATT_FUSED_TRACE is set at launch, six %globaltimer stamps per CTA
 * (start, first stage landed, last stage consumed, column partials written,
 * after the grid barrier, end) for CTAs < 1024. Copies the first n of the
 * 6144 u64 values (CTA-major) to host memory `out` (synchronous). */
catt_status catt_fused_trace(uint64_t* out, int32_t n);
/* ABI revision of this header: 6 (catt_hw.reserved_ became private_streams);
 * 5 (catt_hw.stream_floor + reserved_,
 * CATT_K_ROWS3, CATT_ROWS_SUM3; 4 added catt_kernel_occupancy; 3: catt_hw's
 * last reserved word became cta_fallback; 2 added min_retouch,
 * min_reuse_trip, max_stream_pct). */
int catt_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* CATT_H */
