// common.cuh -- shared device helpers for libsbr (sm_100a only).
#pragma once
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <stdint.h>
#include <algorithm>

#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ < 1000)
#error "libsbr targets sm_100a only"
#endif

#define SBR_DEV __device__ __forceinline__

namespace sbr {

SBR_DEV float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

SBR_DEV float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// Round-to-nearest-away TF32 (cvt.rna.tf32.f32), returned as an fp32 bit pattern
// with the low 13 mantissa bits cleared (reading C11).
SBR_DEV float tf32_rna(float x) {
  uint32_t r;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
  return __uint_as_float(r & 0xffffe000u);
}

SBR_DEV int lane_id() { return threadIdx.x & 31; }
SBR_DEV int warp_id() { return threadIdx.x >> 5; }

}  // namespace sbr
