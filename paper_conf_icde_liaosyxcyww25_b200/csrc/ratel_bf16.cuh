// ratel_bf16.cuh -- bf16 bit helpers shared by the update kernel and the
// GPU-side RNE test hook (so the hook tests exactly the P16 conversion).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

namespace ratel {

__device__ __forceinline__ float bf16_bits_to_f32(uint32_t b) { return __uint_as_float(b << 16); }

// RNE fp32 -> bf16 of two values, packed (lo in bits 0-15): cvt.rn.bf16x2.f32.
__device__ __forceinline__ uint32_t pack_bf16x2_rn(float lo, float hi) {
  uint32_t r;
  asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
  return r;
}

}  // namespace ratel
