// internal.h — host-side launch plumbing shared by the kernel files.
#pragma once
#include <cstddef>
#include <cstdint>

#include <cuda_runtime.h>

#include "../../include/catt.h"
#include "common.cuh"

namespace catt {

struct DevCtx {
  int device = -1;
  catt_hw hw{};
  int* sm_counter = nullptr;  // hw.num_sms int32, zero between capped launches
  unsigned* gbar = nullptr;   // grid barrier {count, generation} of the fused kernels (inside the same allocation)
  float* work = nullptr;      // fused kernels' column partials, grown on demand
  size_t work_bytes = 0;
  unsigned arrive_total[4] = {};  // FUSED single-read kernel: expected per-problem arrival counts (gbar + 32)
};

// Per-device context of the current device (hardware table, CTA-cap counters).
catt_status dev_ctx(DevCtx** out);

// Validates the throttle for a kernel with `threads` threads per CTA, applies
// the carveout preference to `func`, and fills the device-side Throttle.
// dyn_smem is the kernel's own dynamic shared memory; *dyn_total receives it
// plus the Fig 5 pad when cap == CATT_CAP_SMEM_PAD. allow_warp_gate=false
// rejects active_warps < #warps (pipelined variants cannot gate warps).
catt_status prepare_launch(const void* func, const catt_throttle* t, int threads, size_t dyn_smem,
                           bool allow_warp_gate, Throttle* kt, size_t* dyn_total);

// cudaGetLastError after a launch -> CATT_OK / CATT_ECUDA (and records it).
catt_status after_launch();
void record_cuda_error(cudaError_t e);

inline int cta_threads_or(const catt_throttle* t, int def) {
  return (t && t->cta_threads > 0) ? t->cta_threads : def;
}
inline int variant_of(const catt_throttle* t) { return t ? t->variant : CATT_VAR_LITERAL; }

// Tiled SYRK over the tiles on and above the diagonal only (k_syrk.cu).
catt_status syrk_upper(const float* A, float* C, int64_t n, int64_t m, float alpha, float beta, cudaStream_t s);
// CORR: symmat = D^T D (upper tiles, accumulators from +0) with D (nrows x
// mcols) the centred data and Dt = D^T (mcols x nrows) its transpose (only
// read when syrk_kmajor_ok(D, mcols) is false; may be null otherwise).
bool syrk_kmajor_ok(const float* D, int64_t mcols);
// mirror_diag (T2 path only): the kernel also writes the lower triangle and
// a unit diagonal (CORR's symmat in one pass); the caller checks
// syrk_kmajor_ok first and otherwise mirrors itself.
catt_status syrk_upper_kmajor(const float* D, const float* Dt, float* C, int64_t mcols, int64_t nrows, cudaStream_t s,
                              bool mirror_diag = false);

}  // namespace catt
