// common.cuh -- shared device helpers for libsbr (sm_100a only).
#pragma once
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <utility>

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

// 16-bit tensor-core operand format of the reduction: IEEE fp16 (SBR_FP16_FP32ACC, the paper's
// P:348) or bfloat16 (SBR_BF16_FP32ACC, the ablation of SURVEY 8(f) f4) in the same 2-byte
// storage.  One __constant__ flag per translation unit, set from the host in stream order before
// a reduction's first kernel (set_op16_all, sbr_api.cu); read by every float -> 16-bit operand
// conversion and by the kind::f16 instruction descriptors (a/b format bits: 0 f16, 1 bf16).
static __constant__ int g_op16_bf16;
SBR_DEV __half cvt16(float x) {
  if (g_op16_bf16) return __ushort_as_half(__bfloat16_as_ushort(__float2bfloat16_rn(x)));
  return __float2half_rn(x);
}
SBR_DEV float from16(__half h) {
  if (g_op16_bf16) return __bfloat162float(__ushort_as_bfloat16(__half_as_ushort(h)));
  return __half2float(h);
}
SBR_DEV uint32_t op16_fmt() { return g_op16_bf16 ? ((1u << 7) | (1u << 10)) : 0u; }
#define SBR_OP16_SETTER(name)                                                                   \
  cudaError_t set_op16_##name(int bf16, cudaStream_t st) {                                        \
    return cudaMemcpyToSymbolAsync(g_op16_bf16, &bf16, sizeof(int), 0, cudaMemcpyHostToDevice, st); \
  }

SBR_DEV int lane_id() { return threadIdx.x & 31; }
SBR_DEV int warp_id() { return threadIdx.x >> 5; }

}  // namespace sbr

namespace sbr {

// Programmatic dependent launch (PDL).  Every kernel of the per-panel chain triggers its
// dependents at entry and waits for its predecessor (griddepcontrol.wait: full completion
// and memory flush of the prerequisite grid) before its first global-memory access, so the
// next kernel's launch, barrier init, TMEM allocation and descriptor prefetch overlap the
// tail of the previous one.  Without the launch attribute both are no-ops.
SBR_DEV void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
SBR_DEV void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

bool pdl_enabled();   // SBR_PDL=0 disables (ablation)

// cudaFuncSetAttribute is per device context: set (fn, attr) = value once per device
// (cached under a mutex keyed by the current device), so a handle on a second device in
// the same process gets its own attributes.  k_misc.cu.
cudaError_t func_attr(const void* fn, cudaFuncAttribute attr, int value);
// occupancy-derived co-resident CTAs per SM of (fn, threads, smem) on the current device (cached)
int func_blocks_per_sm(const void* fn, int threads, size_t smem);
int current_device_sms();

// test-only experiment knobs (sbr_testing.h sbr_test_set_knob); 0 unless a test set them
enum Knob { KNOB_PASS_EXPER = 0, KNOB_TF32_SIMT_PASS = 1, KNOB_SYR2K_BAND = 2, KNOB_SYR2K_MC = 3, KNOB_COUNT = 8 };
int knob(Knob k);

// A plain launch of a kernel that also calls pdl_trigger / pdl_wait (no-ops then): used where an
// early-launched dependent grid measured slower (config 5's b = 64 SIMT merge: 726 -> 868 ms on PDL,
// its 64-wide gemm_tn and in-place update park resident CTAs beside their predecessors).
template <typename... KArgs, typename... Args>
inline cudaError_t launch_plain(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                                Args&&... args) {
  kern<<<grid, block, smem, st>>>(std::forward<Args>(args)...);
  return cudaGetLastError();
}

template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                              Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

}  // namespace sbr
