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
#include <cstring>

#include <cooperative_groups.h>

#include "internal.h"
#include "tma.cuh"

namespace catt {

constexpr int kMaxDual = 4;
constexpr int kMaxPeers = 8;      // ranks of one NVLink / NVSwitch domain
constexpr int kPeerCtas = 1024;   // flag slots per (parity, source rank)
constexpr int kTraceCtas = 1024, kTracePhases = 6;
// per-CTA %globaltimer at: start, first stage landed, last stage consumed,
// partials written, after the grid barrier, end (diagnostics only)
__device__ unsigned long long g_fused_trace[kTraceCtas * kTracePhases];
constexpr int kBandMax = 2048;  // rows per CTA whose xc / yr are staged in shared memory

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
  int bandcap;                // rows per CTA whose xc / yr fit the shared-memory band buffer (nd kernel)
  int inter;                  // nd kernel: stage chunks dealt round robin over the problem's CTAs
  int trace;                  // nd kernel: record phase timestamps per CTA (catt_fused_trace)
  int fastbar;                // nd kernel: grid barrier by ordered atomics (grid_barrier_ordered)
  int redpf;                  // nd kernel: column reduction issues a warp's band loads together
  unsigned* arrive;           // nd kernel, fastbar 2: per-problem monotonic arrival counters
  unsigned arrive_target[kMaxDual];  // counter value once every CTA of problem p has arrived
  unsigned* gbar;             // grid barrier {count, generation}
  int64_t N;
  // DEP kernel, row-sharded ATAX (catt_atax_peer): the column outputs are
  // all-reduced across ranks through peer memory inside this kernel
  float* peer_recv[kMaxPeers];       // rank p's receive buffer [2 parities][world][N] (IPC-mapped)
  unsigned* peer_flag[kMaxPeers];    // rank p's flags [2][world][kPeerCtas]
  float* mc_recv;                    // multicast alias of every rank's receive buffer (NVLS), or null
  unsigned* mc_flag;                 // multicast alias of every rank's flags, or null
  unsigned* peer_err;                // this rank's error word (a wait timed out)
  int world, rank;                   // world = 0: no peer reduction
  unsigned epoch;                    // launch number, equal on every rank
  int fence_all;                     // peer_flags: every thread fences (diagnostics)
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

// The same barrier with ordered atomics instead of separate fences: the
// arrival is one acq_rel add (it publishes this CTA's earlier writes, which
// __syncthreads made visible to thread 0), the last arriver resets the count
// and bumps the generation with one release add, the others poll the
// generation with acquire loads (no sleep: 148 pollers on one L2 line).
__device__ __forceinline__ void grid_barrier_ordered(unsigned* bar, unsigned nblocks) {
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned gen, old;
    asm volatile("ld.relaxed.gpu.u32 %0, [%1];" : "=r"(gen) : "l"(bar + 1) : "memory");
    asm volatile("atom.add.acq_rel.gpu.u32 %0, [%1], 1;" : "=r"(old) : "l"(bar) : "memory");
    if (old == nblocks - 1) {
      asm volatile("st.relaxed.gpu.u32 [%0], 0;" ::"l"(bar) : "memory");
      asm volatile("red.release.gpu.add.u32 [%0], 1;" ::"l"(bar + 1) : "memory");
    } else {
      unsigned cur;
      do {
        asm volatile("ld.acquire.gpu.u32 %0, [%1];" : "=r"(cur) : "l"(bar + 1) : "memory");
      } while (cur == gen);
    }
  }
  __syncthreads();
}

// Peer-memory all-reduce of the column outputs (row-sharded ATAX): every CTA
// has stored its columns' partials into slot [par][rank] of every rank's
// receive buffer (plain stores through the IPC-mapped pointers, over NVLink
// between GPUs). Then: system-scope fence, and thread 0 publishes epoch in
// flag [par][rank][cta] of every rank (release). The CTA waits for flag
// [par][g][cta] == epoch from every source g (acquire; the chunk -> CTA map
// is the same on every rank: equal shards, equal grids), and sums the slots
// in rank order: every rank gets bit-identical outputs. par = epoch & 1
// double-buffers slots and flags, so a rank one launch ahead never
// overwrites data still being read (it cannot get two launches ahead: its
// next wait needs this rank's next flags). A wait longer than 10 s sets
// *peer_err (1) and gives up instead of hanging the GPU; a source rank that
// launched another grid (unequal shards) sets it to 2 at once.
// The flag half of it: publish this CTA's partials, wait for the same CTA
// index of every rank. Returns false (every thread) after a 10 s give-up.
// One store that lands in every rank's copy of a buffer bound to a multicast
// object (NVSwitch NVLS): replaces the world per-peer stores.
__device__ __forceinline__ void mc_st_f32(float* p, float v) {
  asm volatile("multimem.st.relaxed.sys.global.f32 [%0], %1;" ::"l"(p), "f"(v) : "memory");
}
__device__ __forceinline__ void mc_st_release_u32(unsigned* p, unsigned v) {
  asm volatile("multimem.st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// this rank's partial of one column into slot `slot` of every rank's receive buffer
__device__ __forceinline__ void peer_put(const FusedArgs& a, int64_t slot, float v) {
  if (a.mc_recv) {
    mc_st_f32(a.mc_recv + slot, v);
  } else {
    for (int p = 0; p < a.world; ++p) a.peer_recv[p][slot] = v;
  }
}

__device__ bool peer_flags(const FusedArgs& a) {
  const unsigned par = a.epoch & 1u;
  // the flag carries the launch's grid size beside the epoch: the chunk ->
  // CTA map is a function of the grid, so a rank whose grid differs (unequal
  // shards of fewer rows than CTAs) is detected instead of summed silently
  const unsigned tag = (a.epoch << 11) | (gridDim.x & 0x7FFu);
  // the CTA's partial stores are ordered before thread 0's system-scope fence
  // by the barrier (release cumulativity), so one fence per CTA publishes
  // them (CATT_PEER_FENCE_ALL: every thread fences, the earlier form)
  if (a.fence_all) __threadfence_system();
  __syncthreads();
  __shared__ int s_ok;
  if (threadIdx.x == 0) {
    if (!a.fence_all) __threadfence_system();
    const int64_t fo = (int64_t(par) * a.world + a.rank) * kPeerCtas + blockIdx.x;
    if (a.mc_flag) {
      mc_st_release_u32(a.mc_flag + fo, tag);
    } else {
      for (int p = 0; p < a.world; ++p)
        asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(a.peer_flag[p] + fo), "r"(tag) : "memory");
    }
    int ok = 1;
    const unsigned long long t0 = gtimer();
    unsigned* mine = a.peer_flag[a.rank];
    for (int g = 0; g < a.world && ok; ++g) {
      const unsigned* f = mine + (int64_t(par) * a.world + g) * kPeerCtas + blockIdx.x;
      unsigned v;
      while (true) {
        asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(f) : "memory");
        if (v == tag) break;
        if ((v >> 11) == (tag >> 11)) {                 // this launch, another grid
          atomicExch(a.peer_err, 2u);
          ok = 0;
          break;
        }
        if (*reinterpret_cast<volatile unsigned*>(a.peer_err) != 0u || gtimer() - t0 > 10000000000ull) {
          atomicCAS(a.peer_err, 0u, 1u);                // another CTA's verdict stands
          ok = 0;
          break;
        }
        __nanosleep(100);
      }
    }
    s_ok = ok;
  }
  __syncthreads();
  return s_ok != 0;
}

template <int NW>
__device__ void peer_allreduce(const FusedArgs& a) {
  const int64_t N = a.N;
  const unsigned par = a.epoch & 1u;
  if (!peer_flags(a)) return;
  const float* recv = a.peer_recv[a.rank] + int64_t(par) * a.world * N;
  const int64_t chunks = (N + 31) / 32;
  for (int64_t ch = blockIdx.x; ch < chunks; ch += gridDim.x) {
    const int64_t j = ch * 32 + (threadIdx.x & 31);
    if ((threadIdx.x >> 5) == 0 && j < N) {
      float tot = __ldcg(recv + j);
      for (int g = 1; g < a.world; ++g) tot += __ldcg(recv + int64_t(g) * N + j);
      if (a.col_acc[0]) tot = a.yc[0][j] + tot;
      a.yc[0][j] = tot;
    }
  }
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
        if (a.world > 0) {
          // this rank's partial of column j, stored into every rank's slot [par][rank]
          const int64_t slot = (int64_t(a.epoch & 1u) * a.world + a.rank) * N + j;
          peer_put(a, slot, tot);
        } else {
          if (a.col_acc[q]) tot = a.yc[q][j] + tot;
          a.yc[q][j] = tot;
        }
      }
      __syncthreads();
    }
  }
  if (a.world > 0) peer_allreduce<NW>(a);
}

// Independent pair (BICG, MVT: the column weights xc are inputs), one read
// of each element: every float4 of a row feeds the row dot and the column
// partial. Warp roles: NW consumer warps own 16-byte column chunks (as in
// fused_kernel) and do only the streaming math; one producer warp issues the
// stage copies and adds the row partials, so neither sits on the consumers'
// path. Rows go 4 at a time (4 independent dot chains); the 4 lane partials
// are reduced by a fixed butterfly (offset 16 halves the rows per lane, 8
// again, then 4, 2, 1: 6 shuffles for 4 rows) and written to a row-partial
// ring of 2S slots. Per stage c: consumers wait full[c%S], compute, publish
// partials (part_full[c%2S]) and release the stage (empty[c%S]); the producer
// waits part_full, adds the NW partials of each row with a fixed xor tree,
// writes the row outputs, then refills slot c%S with stage c+S. Slot c%2S is
// rewritten only at stage c+2S, whose copy is issued after totals(c+S).
template <int NW, int T>
__global__ void __launch_bounds__((NW + 1) * 32, 1) fused_nd_kernel(FusedArgs a, int RPS, int S) {
  extern __shared__ __align__(1024) unsigned char dyn[];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const bool producer = warp == NW;
  uint64_t* full = reinterpret_cast<uint64_t*>(dyn);
  uint64_t* empty = full + S;
  uint64_t* part_full = empty + S;                                // [2S]
  float* rowbuf = reinterpret_cast<float*>(dyn + 1024);          // [2S][RPS][NW] warp partials
  float* bandbuf = rowbuf + 2 * S * RPS * NW;                   // [2][bandcap] xc and yr of the band
  const int BC = a.bandcap;
  unsigned char* ring = dyn + 1024 + ((int64_t(2 * S) * RPS * NW * 4 + 2 * int64_t(BC) * 4 + 1023) / 1024) * 1024;
  int pi = 0;
  while (pi + 1 < a.nprob && int(blockIdx.x) >= a.cta0[pi + 1]) ++pi;
  const float* __restrict__ Ap = a.A[pi];
  const float* __restrict__ xc = a.xc[pi];
  float* __restrict__ yr = a.yr[pi];
  const int lb = int(blockIdx.x) - a.cta0[pi];
  const int64_t N = a.N, n4 = N >> 2, M = a.M[pi];
  const int64_t stage_bytes = int64_t(RPS) * N * 4;
  // rows of stage c: a.inter = 0: the CTA's band [r0, r1) in order; a.inter = 1:
  // chunks of RPS rows dealt round robin (chunk lb + c * Gp), so at any time
  // all CTAs stream one narrow window of A
  const int64_t Gp = a.cta0[pi + 1] - a.cta0[pi];
  const int64_t r0 = a.inter ? 0 : int64_t(lb) * a.band[pi], r1 = a.inter ? M : imin64(M, r0 + a.band[pi]);
  const int64_t nch = (M + RPS - 1) / RPS;
  const int64_t nst = a.inter ? (nch > lb ? (nch - lb + Gp - 1) / Gp : 0) : (r1 > r0 ? (r1 - r0 + RPS - 1) / RPS : 0);
  auto row0 = [&](int64_t c) { return a.inter ? (int64_t(lb) + c * Gp) * RPS : r0 + c * RPS; };
  const bool racc = a.row_acc[pi] != 0;
  const bool tr = a.trace && blockIdx.x < kTraceCtas;
  unsigned long long* trp = g_fused_trace + blockIdx.x * kTracePhases;
  if (tr && threadIdx.x == 0) trp[0] = gtimer();
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      bar_init(&full[s], 1);
      bar_init(&empty[s], NW);
    }
    // every lane that writes a row partial (lanes 0, 8, 16, 24 of each
    // consumer warp) arrives itself: its write is ordered before the
    // producer's read by its own release-arrive / the producer's acquire-wait
    for (int s = 0; s < 2 * S; ++s) bar_init(&part_full[s], NW * 4);
    fence_barrier_init();
  }
  auto issue = [&](int64_t c) {                                 // producer lane 0
    const int s = int(c % S);
    const int64_t rows = imin64(RPS, r1 - row0(c));
    const uint32_t bytes = uint32_t(rows * N * 4);
    bar_expect_tx(&full[s], bytes);
    bulk_1d(ring + int64_t(s) * stage_bytes, Ap + row0(c) * N, bytes, &full[s]);
  };
  __syncthreads();
  if (producer && lane == 0)
    for (int64_t c = 0; c < imin64(S, nst); ++c) issue(c);
  // the band's column weights and initial row values, all loads in flight at once
  // the CTA's column weights and initial row values (local row c * RPS + u),
  // all loads in flight at once
  const bool inband = nst * RPS <= BC;
  if (inband) {
    for (int64_t i = threadIdx.x; i < nst * RPS; i += blockDim.x) {
      const int64_t g = row0(i / RPS) + i % RPS;
      bandbuf[i] = g < M ? xc[g] : 0.0f;
      bandbuf[BC + i] = (racc && g < M) ? yr[g] : 0.0f;
    }
  }
  __syncthreads();
  float4 acc[T];
#pragma unroll
  for (int t = 0; t < T; ++t) acc[t] = make_float4(0.f, 0.f, 0.f, 0.f);

  if (producer) {
    // row totals, then refill the consumed slot
    constexpr int RPP = 32 / NW;
    for (int64_t c = 0; c < nst; ++c) {
      const int64_t i0 = row0(c);
      const int rows = int(imin64(RPS, r1 - i0));
      const int q = int(c % (2 * S));
      const float* rb = rowbuf + int64_t(q) * RPS * NW;
      bar_wait(&part_full[q], uint32_t((c / (2 * S)) & 1));
      for (int u0 = 0; u0 < rows; u0 += RPP) {
        const int u = u0 + lane / NW;
        float v = u < rows ? rb[u * NW + (lane % NW)] : 0.0f;
#pragma unroll
        for (int o = NW / 2; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if (lane % NW == 0 && u < rows) {
          const float y0 = racc ? (inband ? bandbuf[BC + c * RPS + u] : yr[i0 + u]) : 0.0f;
          yr[i0 + u] = racc ? y0 + v : v;
        }
      }
      if (lane == 0 && c + S < nst) {
        bar_wait(&empty[c % S], uint32_t((c / S) & 1));
        issue(c + S);
      }
      __syncwarp();
    }
  } else {
    const float4* x4 = reinterpret_cast<const float4*>(a.xr[pi]);
    float4 xr[T];
    bool ok[T];
    int64_t col[T];
#pragma unroll
    for (int t = 0; t < T; ++t) {
      col[t] = warp * 32 + lane + int64_t(32) * NW * t;
      ok[t] = col[t] < n4;
      xr[t] = ok[t] ? x4[col[t]] : make_float4(0.f, 0.f, 0.f, 0.f);
    }
    const bool b4 = (lane & 16) != 0, b3 = (lane & 8) != 0;
    for (int64_t c = 0; c < nst; ++c) {
      const int s = int(c % S);
      const int q = int(c % (2 * S));
      const int64_t i0 = row0(c);
      const int rows = int(imin64(RPS, r1 - i0));
      const float wl = lane < rows ? (inband ? bandbuf[c * RPS + lane] : xc[i0 + lane]) : 0.0f;
      bar_wait(&full[s], uint32_t((c / S) & 1));
      if (tr && c == 0 && threadIdx.x == 0) trp[1] = gtimer();
      const float4* st = reinterpret_cast<const float4*>(ring + int64_t(s) * stage_bytes);
      float* rb = rowbuf + int64_t(q) * RPS * NW;
      for (int u0 = 0; u0 < rows; u0 += 4) {
        float d[4] = {0.f, 0.f, 0.f, 0.f};
        float w[4];
#pragma unroll
        for (int r = 0; r < 4; ++r) w[r] = __shfl_sync(0xffffffffu, wl, (u0 + r) & 31);
        const float4* g = st + int64_t(u0) * n4;
        auto row4 = [&](int r, int t) {
          const float4 v = g[int64_t(r) * n4 + col[t]];
          d[r] = fmaf(v.x, xr[t].x, d[r]);
          d[r] = fmaf(v.y, xr[t].y, d[r]);
          d[r] = fmaf(v.z, xr[t].z, d[r]);
          d[r] = fmaf(v.w, xr[t].w, d[r]);
          acc[t].x = fmaf(v.x, w[r], acc[t].x);
          acc[t].y = fmaf(v.y, w[r], acc[t].y);
          acc[t].z = fmaf(v.z, w[r], acc[t].z);
          acc[t].w = fmaf(v.w, w[r], acc[t].w);
        };
        if (u0 + 4 <= rows) {   // full group: no per-row guards
#pragma unroll
          for (int t = 0; t < T; ++t)
            if (ok[t]) {
#pragma unroll
              for (int r = 0; r < 4; ++r) row4(r, t);
            }
        } else {
#pragma unroll
          for (int t = 0; t < T; ++t)
            if (ok[t]) {
#pragma unroll
              for (int r = 0; r < 4; ++r)
                if (u0 + r < rows) row4(r, t);
            }
        }
        // butterfly: after offset 16 a lane holds rows {2*b4, 2*b4+1}, after 8 row 2*b4+b3
        const float s0 = b4 ? d[0] : d[2], s1 = b4 ? d[1] : d[3];
        const float k0 = b4 ? d[2] : d[0], k1 = b4 ? d[3] : d[1];
        const float e0 = k0 + __shfl_xor_sync(0xffffffffu, s0, 16);
        const float e1 = k1 + __shfl_xor_sync(0xffffffffu, s1, 16);
        float f = (b3 ? e1 : e0) + __shfl_xor_sync(0xffffffffu, b3 ? e0 : e1, 8);
        f += __shfl_xor_sync(0xffffffffu, f, 4);
        f += __shfl_xor_sync(0xffffffffu, f, 2);
        f += __shfl_xor_sync(0xffffffffu, f, 1);
        const int r = lane >> 3;
        if ((lane & 7) == 0 && u0 + r < rows) rb[(u0 + r) * NW + warp] = f;
      }
      if ((lane & 7) == 0) bar_arrive(&part_full[q]);
      __syncwarp();
      if (lane == 0) bar_arrive(&empty[s]);
    }
  }
  // column partials -> workspace (the producer's acc is zero and unused);
  // grid barrier; fixed-tree column outputs
  float* part = a.part[pi] + int64_t(lb) * N;
  if (tr && threadIdx.x == 0) trp[2] = gtimer();
  if (!producer) {
#pragma unroll
    for (int t = 0; t < T; ++t) {
      const int64_t cc = warp * 32 + lane + int64_t(32) * NW * t;
      if (cc < n4) reinterpret_cast<float4*>(part)[cc] = acc[t];
    }
  }
  if (a.fastbar == 2) {
    // split arrival: one release add on this problem's counter, no last
    // arriver; a CTA waits below only for the problem whose columns it sums
    __syncthreads();
    if (tr && threadIdx.x == 0) trp[3] = gtimer();
    if (threadIdx.x == 0) asm volatile("red.release.gpu.add.u32 [%0], 1;" ::"l"(a.arrive + pi) : "memory");
  } else if (a.fastbar) {
    if (tr && threadIdx.x == 0) trp[3] = gtimer();
    grid_barrier_ordered(a.gbar, gridDim.x);
  } else {
    __threadfence();
    if (tr && threadIdx.x == 0) trp[3] = gtimer();
    grid_barrier(a.gbar, gridDim.x);
  }
  if (tr && threadIdx.x == 0) trp[4] = gtimer();
  // column outputs in one round: chunks of CW = 32*L columns (L per lane,
  // chosen so every problem's chunks fit the grid); consumer warp w sums band
  // partials [w*gpw, (w+1)*gpw) in order, then the NW warp sums in warp order
  {
    constexpr int LMAX = 4;
    __shared__ float red[NW][32 * LMAX];
    const int64_t per_cta = (N * a.nprob + gridDim.x - 1) / gridDim.x;
    const int L = per_cta <= 32 ? 1 : per_cta <= 64 ? 2 : per_cta <= 96 ? 3 : 4;
    const int64_t CW = 32 * L;
    const int64_t chunks = (N + CW - 1) / CW;
    for (int64_t gch = blockIdx.x; gch < chunks * a.nprob; gch += gridDim.x) {
      const int q = int(gch / chunks);
      const int64_t ch = gch % chunks;
      const int64_t G = a.cta0[q + 1] - a.cta0[q];
      const int64_t gpw = (G + NW - 1) / NW;
      const int64_t b0 = warp * gpw, b1 = imin64(G, b0 + gpw);
      const float* pq = a.part[q];
      // MVT's x2 (in/out) is an input until this chunk writes it: fetch it
      // before waiting
      float y0[LMAX];
#pragma unroll
      for (int l = 0; l < LMAX; ++l) {
        const int64_t j = ch * CW + l * 32 + lane;
        y0[l] = (warp == 0 && a.col_acc[q] && l < L && j < N) ? a.yc[q][j] : 0.0f;
      }
      if (a.fastbar == 2) {
        if (threadIdx.x == 0) {
          unsigned cur;
          do {
            asm volatile("ld.acquire.gpu.u32 %0, [%1];" : "=r"(cur) : "l"(a.arrive + q) : "memory");
          } while (int(cur - a.arrive_target[q]) < 0);
          if (tr && gch == blockIdx.x) trp[4] = gtimer();
        }
        __syncthreads();
      }
      if (!producer) {
        float sum[LMAX];
#pragma unroll
        for (int l = 0; l < LMAX; ++l) sum[l] = 0.0f;
        if (a.redpf) {
          // all of the warp's band partials in flight at once (one L2 round
          // trip instead of gpw), then added in band order as before
          constexpr int BP = 8;
          for (int64_t bb = b0; bb < b1; bb += BP) {
            float v[BP][LMAX];
#pragma unroll
            for (int u = 0; u < BP; ++u)
#pragma unroll
              for (int l = 0; l < LMAX; ++l) {
                const int64_t j = ch * CW + l * 32 + lane;
                v[u][l] = (bb + u < b1 && l < L && j < N) ? pq[(bb + u) * N + j] : 0.0f;
              }
#pragma unroll
            for (int u = 0; u < BP; ++u)
#pragma unroll
              for (int l = 0; l < LMAX; ++l)
                if (bb + u < b1) sum[l] += v[u][l];
          }
        } else {
          for (int64_t b = b0; b < b1; ++b) {
#pragma unroll
            for (int l = 0; l < LMAX; ++l) {
              const int64_t j = ch * CW + l * 32 + lane;
              if (l < L && j < N) sum[l] += pq[b * N + j];
            }
          }
        }
#pragma unroll
        for (int l = 0; l < LMAX; ++l) red[warp][l * 32 + lane] = sum[l];
      }
      __syncthreads();
      if (warp == 0) {
        for (int l = 0; l < L; ++l) {
          const int64_t j = ch * CW + l * 32 + lane;
          if (j < N) {
            float tot = red[0][l * 32 + lane];
            for (int w = 1; w < NW; ++w) tot += red[w][l * 32 + lane];
            if (a.world > 0) {
              // row-sharded (catt_dual_group_peer): this rank's partial of
              // column j of problem q into slot [par][rank] of every rank
              const int64_t slot = (int64_t(a.epoch & 1u) * a.world + a.rank) * (N * a.nprob) + int64_t(q) * N + j;
              peer_put(a, slot, tot);
            } else {
              if (a.col_acc[q]) tot = y0[l] + tot;
              a.yc[q][j] = tot;
            }
          }
        }
      }
      __syncthreads();
    }
    if (a.world > 0 && peer_flags(a)) {
      // the same chunks again: every rank's partials in rank order, then the
      // initial value (MVT's x2, replicated on every rank): bit-identical
      // outputs on every rank
      const int64_t NP = N * a.nprob;
      const float* recv = a.peer_recv[a.rank] + int64_t(a.epoch & 1u) * a.world * NP;
      for (int64_t gch = blockIdx.x; gch < chunks * a.nprob; gch += gridDim.x) {
        const int q = int(gch / chunks);
        const int64_t ch = gch % chunks;
        if (warp == 0)
          for (int l = 0; l < L; ++l) {
            const int64_t j = ch * CW + l * 32 + lane;
            if (j < N) {
              const int64_t c = int64_t(q) * N + j;
              float tot = __ldcg(recv + c);
              for (int g = 1; g < a.world; ++g) tot += __ldcg(recv + int64_t(g) * NP + c);
              if (a.col_acc[q]) tot = a.yc[q][j] + tot;
              a.yc[q][j] = tot;
            }
          }
      }
    }
  }
  if (tr && threadIdx.x == 0) trp[5] = gtimer();
}

namespace {

template <bool DEP>
const void* fused_fn(int NW, int T) {
  if (!DEP && getenv("CATT_FUSED_ND") == nullptr) {  // the single-read kernel (CATT_FUSED_ND set: old form)
    if (NW == 16) {
      if (T == 2) return (const void*)fused_nd_kernel<16, 2>;
      if (T == 4) return (const void*)fused_nd_kernel<16, 4>;
      return (const void*)fused_nd_kernel<16, 8>;
    }
    if (T == 1) return (const void*)fused_nd_kernel<8, 1>;
    return (const void*)fused_nd_kernel<8, 2>;
  }
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

// Small ATAX (N <= 1024, A <= 4 MB; configs[0]'s 256^2): the row-serial
// fused kernel spends its time in per-row CTA barriers, so here every warp
// owns whole rows (warp w of CTA c: rows c*8 + w, + 8G, ...). A lane holds NV
// 16-byte chunks of the row (lane + 32v), the row dot is a warp xor tree
// (tmp_i in every lane), and the lane adds tmp_i * row into its NV column
// accumulators, with the next row's loads already in flight. The G <= 8
// CTAs form one cluster: the 8 G warp partials of each column are added in
// (CTA rank, warp) order through distributed shared memory, so no workspace,
// grid barrier or cooperative launch is needed. ≤ 1e-5 of fp64 (the FUSED bar).
template <int NV>
__global__ void __launch_bounds__(256, 1) atax_small_kernel(const float* __restrict__ A, const float* __restrict__ x,
                                                            float* __restrict__ tmp, float* __restrict__ y, int64_t M,
                                                            int64_t N) {
  namespace cg = cooperative_groups;
  cg::cluster_group cluster = cg::this_cluster();
  __shared__ __align__(16) float part[8][NV * 128];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int G = int(cluster.num_blocks()), rank = int(cluster.block_rank());
  const int64_t n4 = N >> 2;
  const float4* x4 = reinterpret_cast<const float4*>(x);
  float4 xv[NV], acc[NV], cur[NV], nxt[NV];
#pragma unroll
  for (int v = 0; v < NV; ++v) {
    const int64_t c = lane + 32 * v;
    xv[v] = c < n4 ? x4[c] : make_float4(0.f, 0.f, 0.f, 0.f);
    acc[v] = make_float4(0.f, 0.f, 0.f, 0.f);
  }
  const int64_t step = int64_t(G) * 8;
  auto load = [&](int64_t i, float4 (&r)[NV]) {
    const float4* row = reinterpret_cast<const float4*>(A + i * N);
#pragma unroll
    for (int v = 0; v < NV; ++v) {
      const int64_t c = lane + 32 * v;
      r[v] = (i < M && c < n4) ? ld_stream4(row + c) : make_float4(0.f, 0.f, 0.f, 0.f);
    }
  };
  int64_t i = int64_t(rank) * 8 + warp;
  load(i, cur);
  for (; i < M; i += step) {
    load(i + step, nxt);
    float d = 0.0f;
#pragma unroll
    for (int v = 0; v < NV; ++v) {
      d = fmaf(cur[v].x, xv[v].x, d);
      d = fmaf(cur[v].y, xv[v].y, d);
      d = fmaf(cur[v].z, xv[v].z, d);
      d = fmaf(cur[v].w, xv[v].w, d);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) d += __shfl_xor_sync(0xffffffffu, d, o);
    if (lane == 0) tmp[i] = d;
#pragma unroll
    for (int v = 0; v < NV; ++v) {
      acc[v].x = fmaf(cur[v].x, d, acc[v].x);
      acc[v].y = fmaf(cur[v].y, d, acc[v].y);
      acc[v].z = fmaf(cur[v].z, d, acc[v].z);
      acc[v].w = fmaf(cur[v].w, d, acc[v].w);
    }
#pragma unroll
    for (int v = 0; v < NV; ++v) cur[v] = nxt[v];
  }
#pragma unroll
  for (int v = 0; v < NV; ++v) reinterpret_cast<float4*>(part[warp])[lane + 32 * v] = acc[v];
  cluster.sync();
  const int64_t per = (N + G - 1) / G;
  const int64_t j0 = rank * per, j1 = imin64(N, j0 + per);
  for (int64_t j = j0 + threadIdx.x; j < j1; j += blockDim.x) {
    float sum = 0.0f;
    for (int q = 0; q < G; ++q) {
      const float* pq = cluster.map_shared_rank(&part[0][0], q);
#pragma unroll
      for (int w = 0; w < 8; ++w) sum += pq[w * NV * 128 + j];
    }
    y[j] = sum;
  }
  cluster.sync();  // no CTA leaves while its partials are read
}

catt_status launch_atax_small(const DualProblem& p, int64_t N, cudaStream_t s) {
  const int64_t n4 = N / 4;
  const int NV = n4 <= 32 ? 1 : n4 <= 64 ? 2 : n4 <= 128 ? 4 : 8;
  const int G = int(std::max<int64_t>(1, std::min<int64_t>(8, (p.M + 31) / 32)));  // >= 4 rows per warp
  const void* f = NV == 1 ? (const void*)atax_small_kernel<1>
                : NV == 2 ? (const void*)atax_small_kernel<2>
                : NV == 4 ? (const void*)atax_small_kernel<4> : (const void*)atax_small_kernel<8>;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(unsigned(G), 1, 1);
  cfg.blockDim = dim3(256, 1, 1);
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = unsigned(G);
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  const float* A = p.A;
  const float* x = p.xr;
  float* tmp = p.yr;
  float* y = p.yc;
  int64_t M = p.M, NN = N;
  void* params[] = {&A, &x, &tmp, &y, &M, &NN};
  cudaError_t e = cudaLaunchKernelExC(&cfg, f, params);
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  return after_launch();
}

}  // namespace catt

// A rank's peer-reduction state (catt_peer_*): one cudaMalloc holding
// [receive slots: 2 x world x n floats][flags: 2 x world x kPeerCtas u32][error word],
// exported by a CUDA IPC handle; the peers' buffers opened from theirs.
struct catt_peer {
  int world = 0, rank = 0;
  int64_t n = 0;
  void* base = nullptr;              // own allocation (catt_peer_create), else null
  size_t bytes = 0;
  float* mc_recv = nullptr;          // catt_peer_create_mapped with a multicast alias
  unsigned* mc_flag = nullptr;
  float* recv[catt::kMaxPeers] = {};
  unsigned* flag[catt::kMaxPeers] = {};
  void* opened[catt::kMaxPeers] = {};
  unsigned epoch = 0;
  unsigned* err = nullptr;
};

namespace catt {

struct PeerLaunch {
  catt_peer* p;
};

catt_status launch_fused_group(bool dep, const DualProblem* pr, int np, int64_t N, const catt_throttle* t,
                               cudaStream_t s, const PeerLaunch* peer = nullptr) {
  if (np < 1 || np > kMaxDual || N <= 0 || N % 4) return CATT_EINVAL;
  int64_t Mtot = 0;
  for (int i = 0; i < np; ++i) {
    if (pr[i].M <= 0) return CATT_EINVAL;
    if ((reinterpret_cast<uintptr_t>(pr[i].A) & 15u) || (reinterpret_cast<uintptr_t>(pr[i].xr) & 15u))
      return CATT_EINVAL;
    Mtot += pr[i].M;
  }
  if (t && (t->active_warps || t->active_ctas)) return CATT_EINVAL;  // nothing to throttle (no L1 reuse)
  if (dep && np == 1 && !peer && !pr[0].col_acc && N <= 1024 && pr[0].M * N * 4 <= (int64_t(4) << 20) &&
      getenv("CATT_FUSED_NO_SMALL") == nullptr)
    return launch_atax_small(pr[0], N, s);
  const int64_t n4 = N / 4;
  // 8 warps for short rows (T <= 2 chunks per lane), else 16 warps with
  // T = 2, 4 or 8 chunks per lane (N <= 16384)
  const int NW = n4 <= 512 ? 8 : 16;
  const int64_t T64 = (n4 + 32 * NW - 1) / (32 * NW);
  if (T64 > 8) return CATT_EUNSUPPORTED;  // N > 16384
  const int T = T64 <= 1 ? 1 : (T64 <= 2 ? 2 : (T64 <= 4 ? 4 : 8));
  const bool nd = !dep && getenv("CATT_FUSED_ND") == nullptr;  // single-read kernel (+1 producer warp)
  const int threads = (NW + (nd ? 1 : 0)) * 32;
  const void* f = dep ? fused_fn<true>(NW, T) : fused_fn<false>(NW, T);
  // stage = RPS whole rows (~64 KB: several independent row chains per warp
  // and few barriers per byte), S stages within ~200 KB of shared memory
  const int64_t row_bytes = N * 4;
  const char* rps_env = getenv("CATT_FUSED_STAGE_KB");
  const int64_t stage_target = (rps_env ? atoi(rps_env) : 64) * 1024;
  const int RPS = int(std::max<int64_t>(1, std::min<int64_t>(16, stage_target / row_bytes)));
  const char* budget_env = getenv("CATT_FUSED_SMEM_KB");
  const int64_t budget = (budget_env ? atoi(budget_env) : 220) * 1024;
  // head: barriers in the first 1 KB, then the row partials (DEP: [RPS][NW+1];
  // single-read kernel: [S][RPS][NW], sized for up to 16 stages)
  DevCtx* ctx = nullptr;
  catt_status st = dev_ctx(&ctx);
  if (st != CATT_OK) return st;
  int64_t Mmax = 0;
  for (int i = 0; i < np; ++i) Mmax = std::max<int64_t>(Mmax, pr[i].M);
  // ~2x the expected band (one CTA per SM, CTAs split by rows): larger bands
  // fall back to loading xc / yr per stage
  const int bandcap = dep ? 0 : int(std::min<int64_t>(kBandMax, (2 * Mmax * np) / ctx->hw.num_sms + 64));
  const int64_t head =
      1024 + ((int64_t(RPS) * (NW + 1) * 4 * (dep ? 1 : 32) + 2 * int64_t(bandcap) * 4 + 1023) / 1024) * 1024;
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
  // cluster of CL CTAs for the DSMEM pre-reduction (single problem only;
  // default 1: no measured gain at 4096^2, and clustered cooperative launches
  // cannot be replayed by ncu)
  const char* cl_env = getenv("CATT_FUSED_CLUSTER");
  const int64_t slots = int64_t(ctx->hw.num_sms) * occ;
  int CL = 1;
  int64_t Gall = std::min<int64_t>(slots, Mtot);
  // the single-read kernel has no cluster pre-reduction
  for (int cand = (cl_env && np == 1 && !nd) ? atoi(cl_env) : 1; cand >= 2; cand /= 2) {
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
  args.bandcap = bandcap;
  {
    const char* ie = getenv("CATT_FUSED_INTERLEAVE");
    args.inter = nd ? (ie ? atoi(ie) != 0 : 1) : 0;
    args.trace = nd && getenv("CATT_FUSED_TRACE") != nullptr;
    const char* fb = getenv("CATT_FUSED_BARRIER");
    args.fastbar = fb ? atoi(fb) : 2;
    const char* rp = getenv("CATT_FUSED_REDPF");
    args.redpf = rp ? atoi(rp) != 0 : 1;
  }
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
  if (peer) {
    catt_peer* P = peer->p;
    // ATAX (DEP): one problem; the single-read kernel: any group, the peer
    // buffer holding every problem's columns
    if ((dep && np != 1) || (!dep && !nd) || CL != 1 || cta > kPeerCtas || P->n != N * np) return CATT_EINVAL;
    for (int r = 0; r < P->world; ++r)
      if (!P->recv[r] || !P->flag[r]) return CATT_EINVAL;       // a peer not opened yet
    args.world = P->world;
    args.rank = P->rank;
    args.epoch = ++P->epoch;
    args.fence_all = getenv("CATT_PEER_FENCE_ALL") != nullptr;
    args.peer_err = P->err;
    args.mc_recv = P->mc_recv;
    args.mc_flag = P->mc_flag;
    for (int r = 0; r < P->world; ++r) {
      args.peer_recv[r] = P->recv[r];
      args.peer_flag[r] = P->flag[r];
    }
  }
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
  // per-problem arrival counters (fastbar 2) live after the {count,
  // generation} pair, on their own 128-byte line; the host tracks their
  // running totals and commits them only when the launch went in
  args.arrive = gbar + 32;
  {
    // a captured launch would replay stale targets: graphs get the
    // self-resetting barrier
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    if (args.fastbar == 2 && (cudaStreamIsCapturing(s, &cs) != cudaSuccess || cs != cudaStreamCaptureStatusNone)) {
      cudaGetLastError();
      args.fastbar = 1;
    }
  }
  for (int i = 0; i < np; ++i) args.arrive_target[i] = ctx->arrive_total[i] + unsigned(args.cta0[i + 1] - args.cta0[i]);
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
  st = after_launch();
  if (st == CATT_OK && nd && args.fastbar == 2)
    for (int i = 0; i < np; ++i) ctx->arrive_total[i] = args.arrive_target[i];
  return st;
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

namespace {
size_t peer_layout(int world, int64_t n, size_t* flag_off, size_t* err_off) {
  *flag_off = ((size_t(2) * world * size_t(n) * sizeof(float) + 255) / 256) * 256;
  *err_off = *flag_off + size_t(2) * world * kPeerCtas * sizeof(unsigned);
  return *err_off + 256;
}
}  // namespace

extern "C" catt_status catt_peer_create(int32_t world, int32_t rank, int64_t n, catt_peer** out, void* handle) {
  if (!out || !handle || world < 1 || world > kMaxPeers || rank < 0 || rank >= world || n < 1) return CATT_EINVAL;
  catt_peer* p = new catt_peer();
  p->world = world;
  p->rank = rank;
  p->n = n;
  size_t foff = 0, eoff = 0;
  p->bytes = peer_layout(world, n, &foff, &eoff);
  cudaError_t e = cudaMalloc(&p->base, p->bytes);
  if (e == cudaSuccess) e = cudaMemset(p->base, 0, p->bytes);
  if (e == cudaSuccess) e = cudaIpcGetMemHandle(static_cast<cudaIpcMemHandle_t*>(handle), p->base);
  if (e != cudaSuccess) {
    record_cuda_error(e);
    if (p->base) cudaFree(p->base);
    delete p;
    return e == cudaErrorMemoryAllocation ? CATT_ENOMEM : CATT_ECUDA;
  }
  char* b = static_cast<char*>(p->base);
  p->recv[rank] = reinterpret_cast<float*>(b);
  p->flag[rank] = reinterpret_cast<unsigned*>(b + foff);
  p->err = reinterpret_cast<unsigned*>(b + eoff);
  *out = p;
  return CATT_OK;
}

extern "C" int64_t catt_peer_bytes(int32_t world, int64_t n) {
  if (world < 1 || world > kMaxPeers || n < 1) return -1;
  size_t foff = 0, eoff = 0;
  return int64_t(peer_layout(world, n, &foff, &eoff));
}

extern "C" catt_status catt_peer_create_mapped(int32_t world, int32_t rank, int64_t n, void* const* bases, void* mc_base,
                                               catt_peer** out) {
  if (!out || !bases || world < 1 || world > kMaxPeers || rank < 0 || rank >= world || n < 1) return CATT_EINVAL;
  for (int r = 0; r < world; ++r)
    if (!bases[r] || (reinterpret_cast<uintptr_t>(bases[r]) & 255u)) return CATT_EINVAL;
  if (reinterpret_cast<uintptr_t>(mc_base) & 255u) return CATT_EINVAL;
  catt_peer* p = new catt_peer();
  p->world = world;
  p->rank = rank;
  p->n = n;
  size_t foff = 0, eoff = 0;
  p->bytes = peer_layout(world, n, &foff, &eoff);
  for (int r = 0; r < world; ++r) {
    char* b = static_cast<char*>(bases[r]);
    p->recv[r] = reinterpret_cast<float*>(b);
    p->flag[r] = reinterpret_cast<unsigned*>(b + foff);
  }
  p->err = reinterpret_cast<unsigned*>(static_cast<char*>(bases[rank]) + eoff);
  if (mc_base) {
    p->mc_recv = static_cast<float*>(mc_base);
    p->mc_flag = reinterpret_cast<unsigned*>(static_cast<char*>(mc_base) + foff);
  }
  *out = p;
  return CATT_OK;
}

extern "C" catt_status catt_peer_open(catt_peer* p, int32_t peer_rank, const void* handle) {
  if (!p || !handle || peer_rank < 0 || peer_rank >= p->world) return CATT_EINVAL;
  if (peer_rank == p->rank) return CATT_OK;                  // own buffer: nothing to open
  if (!p->base) return CATT_EINVAL;                          // mapped by the caller (catt_peer_create_mapped)
  if (p->opened[peer_rank]) return CATT_EINVAL;
  cudaIpcMemHandle_t h;
  std::memcpy(&h, handle, sizeof(h));
  void* q = nullptr;
  cudaError_t e = cudaIpcOpenMemHandle(&q, h, cudaIpcMemLazyEnablePeerAccess);
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  size_t foff = 0, eoff = 0;
  peer_layout(p->world, p->n, &foff, &eoff);
  p->opened[peer_rank] = q;
  p->recv[peer_rank] = static_cast<float*>(q);
  p->flag[peer_rank] = reinterpret_cast<unsigned*>(static_cast<char*>(q) + foff);
  return CATT_OK;
}

extern "C" catt_status catt_peer_check(catt_peer* p, int32_t* timed_out) {
  if (!p || !timed_out) return CATT_EINVAL;
  unsigned v = 0;
  cudaError_t e = cudaMemcpy(&v, p->err, sizeof(v), cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  *timed_out = int32_t(v);
  return CATT_OK;
}

extern "C" catt_status catt_peer_destroy(catt_peer* p) {
  if (!p) return CATT_EINVAL;
  for (int r = 0; r < kMaxPeers; ++r)
    if (p->opened[r]) cudaIpcCloseMemHandle(p->opened[r]);
  if (p->base) cudaFree(p->base);
  delete p;
  return CATT_OK;
}

extern "C" catt_status catt_atax_peer(const float* A, const float* x, float* tmp, float* y, int64_t m, int64_t n,
                                      catt_peer* p, void* stream) {
  if (!A || !x || !tmp || !y || !p || m < 1 || n < 1) return CATT_EINVAL;
  DualProblem pr{A, x, nullptr, tmp, y, m, 0, 0};
  PeerLaunch pl{p};
  return launch_fused_group(true, &pr, 1, n, nullptr, static_cast<cudaStream_t>(stream), &pl);
}

extern "C" catt_status catt_fused_trace(uint64_t* out, int32_t n) {
  if (!out || n < 0) return CATT_EINVAL;
  const size_t bytes = size_t(std::min(n, kTraceCtas * kTracePhases)) * sizeof(uint64_t);
  cudaError_t e = cudaMemcpyFromSymbol(out, g_fused_trace, bytes);
  if (e != cudaSuccess) {
    record_cuda_error(e);
    return CATT_ECUDA;
  }
  return CATT_OK;
}

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

extern "C" catt_status catt_dual_group_peer(const catt_dual_problem* probs, int32_t count, catt_peer* p,
                                            void* stream) {
  if (!probs || !p || count < 1 || count > kMaxDual) return CATT_EINVAL;
  DualProblem pr[kMaxDual];
  const int64_t N = probs[0].n;
  for (int i = 0; i < count; ++i) {
    const catt_dual_problem& q = probs[i];
    if (q.n != N || q.m < 1 || !q.A || !q.xr || !q.xc || !q.yr || !q.yc) return CATT_EINVAL;
    pr[i] = DualProblem{q.A, q.xr, q.xc, q.yr, q.yc, q.m, q.row_accumulate != 0, q.col_accumulate != 0};
  }
  if (getenv("CATT_FUSED_ND") != nullptr) return CATT_EINVAL;  // the peer form is the single-read kernel's
  PeerLaunch pl{p};
  return launch_fused_group(false, pr, count, N, nullptr, static_cast<cudaStream_t>(stream), &pl);
}

extern "C" catt_status catt_dual(const float* A, const float* xr, const float* xc, float* yr, float* yc, int64_t m,
                                 int64_t n, int32_t row_accumulate, int32_t col_accumulate, int32_t dependent,
                                 const catt_throttle* t, void* stream) {
  if (m < 1 || n < 1 || !A || !xr || !yr || !yc || (!dependent && !xc)) return CATT_EINVAL;
  if (dependent && row_accumulate) return CATT_EINVAL;
  return launch_fused(dependent != 0, A, xr, xc, yr, yc, m, n, row_accumulate != 0, col_accumulate != 0, t,
                      static_cast<cudaStream_t>(stream));
}
