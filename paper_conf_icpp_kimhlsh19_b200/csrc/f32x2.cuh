// f32x2.cuh — packed fp32 pairs (sm_100a FFMA2 / FADD2). Each half is an
// ordinary IEEE round-to-nearest fp32 operation, so a kernel that pairs two
// independent chains computes bit-for-bit what two scalar chains compute.
#pragma once
#include <cstdint>

namespace catt {

__device__ __forceinline__ uint64_t f2_pack(float lo, float hi) {
  uint64_t r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(lo), "f"(hi));
  return r;
}
__device__ __forceinline__ float f2_lo(uint64_t v) { return __uint_as_float(unsigned(v)); }
__device__ __forceinline__ float f2_hi(uint64_t v) { return __uint_as_float(unsigned(v >> 32)); }
// a - b per half
__device__ __forceinline__ uint64_t f2_sub(uint64_t a, uint64_t b) {
  uint64_t d;
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
// a + b per half
__device__ __forceinline__ uint64_t f2_add(uint64_t a, uint64_t b) {
  uint64_t d;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
// a * b per half
__device__ __forceinline__ uint64_t f2_mul(uint64_t a, uint64_t b) {
  uint64_t d;
  asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
// fmaf(a, b, c) per half
__device__ __forceinline__ uint64_t f2_fma(uint64_t a, uint64_t b, uint64_t c) {
  uint64_t d;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
  return d;
}

// c = fmaf(a, b, c) per half, accumulating in place: the tied operand keeps
// the accumulator in one register pair across an unrolled loop (with separate
// in/out operands ptxas rotated accumulators between pairs and paid ~50
// IMAD.MOV / MOV per stage, on the FMA pipe, to restore them)
__device__ __forceinline__ void f2_fma_acc(uint64_t& c, uint64_t a, uint64_t b) {
  asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(c) : "l"(a), "l"(b));
}
// c = c + a per half, in place
__device__ __forceinline__ void f2_add_acc(uint64_t& c, uint64_t a) {
  asm("add.rn.f32x2 %0, %0, %1;" : "+l"(c) : "l"(a));
}

}  // namespace catt
