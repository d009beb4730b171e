// common.cuh — device-side throttle mechanisms shared by every CATT kernel.
//
// Warp level (Fig 4): the paper splits the loop into N sequential
// warp groups separated by __syncthreads(). On B200 the default is a per-CTA
// counting semaphore in shared memory: at most `active_warps` warps of a CTA
// are inside the loop at once and a finishing warp hands its slot to the next
// waiting one (no idle group tail). CATT_GATE_BARRIER reproduces Fig 4.
//
// CTA level (Fig 5): the paper pads shared memory so only M TBs
// fit. On B200 the carveout is only a hint (the driver may pick a larger
// shared-memory configuration, profiles/round1_probe_hw.txt), so the default
// cap is a per-SM counter in global memory: a CTA enters the loop only when
// fewer than `active_ctas` CTAs of its SM are inside. CATT_CAP_SMEM_PAD
// reproduces Fig 5 (the pad is chosen on the host).
#pragma once
#include <cstdint>

#include <cuda_runtime.h>

namespace catt {

struct Throttle {
  int active_warps;          // warps per CTA allowed in the loop (>= 1)
  int gate;                  // CATT_GATE_*
  int cta_cap;               // CTAs per SM allowed in the loop; 0 = no cap
  int* sm_counter;           // num_sms counters (zero outside capped kernels)
  unsigned long long* probe; // per-warp {smid, t0, t1} or nullptr
};

__host__ __device__ __forceinline__ int64_t imin64(int64_t a, int64_t b) { return a < b ? a : b; }

__device__ __forceinline__ unsigned smid() {
  unsigned r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long r;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(r));
  return r;
}

__device__ __forceinline__ int linear_tid() {
  return threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
}

__device__ __forceinline__ long long linear_cta() {
  return blockIdx.x + (long long)gridDim.x * (blockIdx.y + (long long)gridDim.y * blockIdx.z);
}

// The SM counter a CTA took in cta_enter, kept for cta_exit: %smid may change
// during execution (e.g. after preemption), so cta_exit must not read it again.
__device__ __forceinline__ unsigned& cta_slot() {
  __shared__ unsigned slot;
  return slot;
}

// CTA-level entry: one thread waits for a slot on its SM's counter.
__device__ __forceinline__ void cta_enter(const Throttle& t) {
  if (t.cta_cap <= 0) return;
  if (linear_tid() == 0) {
    const unsigned sm = smid();
    cta_slot() = sm;
    int* c = t.sm_counter + sm;
    unsigned ns = 64;
    while (true) {
      int v = atomicAdd(c, 1);
      if (v < t.cta_cap) break;
      atomicSub(c, 1);
      __nanosleep(ns);
      ns = ns < 2048 ? ns * 2 : ns;
    }
    __threadfence();
  }
  __syncthreads();
}

__device__ __forceinline__ void cta_exit(const Throttle& t) {
  if (t.cta_cap <= 0) return;
  __syncthreads();
  if (linear_tid() == 0) {
    __threadfence();
    atomicSub(t.sm_counter + cta_slot(), 1);
  }
}

// Warp-level semaphore. `slots` lives in shared memory; initialise with
// gate_init before the first __syncthreads of the kernel.
__device__ __forceinline__ void gate_init(int* slots, const Throttle& t) {
  if (linear_tid() == 0) *slots = t.active_warps;
}

__device__ __forceinline__ void warp_acquire(int* slots) {
  if ((linear_tid() & 31) == 0) {
    unsigned ns = 32;
    while (true) {
      int v = atomicSub(slots, 1);
      if (v > 0) break;
      atomicAdd(slots, 1);
      __nanosleep(ns);
      ns = ns < 1024 ? ns * 2 : ns;
    }
  }
  __syncwarp();
}

__device__ __forceinline__ void warp_release(int* slots) {
  __syncwarp();
  if ((linear_tid() & 31) == 0) atomicAdd(slots, 1);
}

// Residency probe: {smid, t_start, t_end} per warp around the loop. The start
// stamp is stored before the loop so no register stays live across it.
__device__ __forceinline__ long long probe_index() {
  const int W = (blockDim.x * blockDim.y * blockDim.z + 31) / 32;
  return (linear_cta() * W + linear_tid() / 32) * 3;
}
__device__ __forceinline__ void probe_begin(const Throttle& t) {
  if (t.probe && (linear_tid() & 31) == 0) {
    const long long idx = probe_index();
    t.probe[idx + 0] = smid();
    t.probe[idx + 1] = gtimer();
  }
}
__device__ __forceinline__ void probe_end(const Throttle& t) {
  if (t.probe && (linear_tid() & 31) == 0) t.probe[probe_index() + 2] = gtimer();
}

// Runs body() (the per-thread loop) under the warp-level throttle. Every
// thread of the CTA must call this exactly once (threads with nothing to do
// pass a body that returns immediately): the barrier form needs all of them.
template <class Body>
__device__ __forceinline__ void throttled(const Throttle& t, int* slots, Body&& body) {
  const int W = (blockDim.x * blockDim.y * blockDim.z + 31) / 32;
  if (t.active_warps >= W) {
    probe_begin(t);
    body();
    probe_end(t);
  } else if (t.gate == 1) {  // CATT_GATE_BARRIER: Fig 4
    const int groups = (W + t.active_warps - 1) / t.active_warps;
    for (int g = 0; g < groups; ++g) {
      if ((linear_tid() / 32) / t.active_warps == g) {
        probe_begin(t);
        body();
        probe_end(t);
      }
      __syncthreads();
    }
  } else {  // CATT_GATE_SEMAPHORE
    warp_acquire(slots);
    probe_begin(t);
    body();
    probe_end(t);
    warp_release(slots);
  }
}

}  // namespace catt
