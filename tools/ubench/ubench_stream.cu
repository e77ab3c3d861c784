// Micro-benchmark: TMA streaming rate of the pass's lower-tile walk (128x128 fp16 tiles, the
// PassWalk order, one CTA per SM, NS-stage ring, consumer releases each slot at once) for
// three shadow layouts:
//   0: column-major fp16 n x n, ld = ldsh (the production layout): 2 boxes of 64 rows x 128 cols
//   1: tile-contiguous (each 128x128 tile = 32 KB, column-major inside): 3-D map, same boxes
//   2: tile-contiguous, one 1-D bulk copy of 32 KB per tile (no swizzle)
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr -lcuda \
//      -I paper_conf_ppopp_zhangsoyw23_b200/csrc -I include tools/ubench/ubench_stream.cu -o /tmp/ubench_stream
#include <cuda.h>
#include <cstdio>
#include <vector>
#include "../../paper_conf_ppopp_zhangsoyw23_b200/csrc/k_pass_tc.cu"

namespace sbr { bool pdl_enabled() { return false; } }
using namespace sbr;

SBR_DEV void tma_load_3d(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1, int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];" ::
          "r"(smem_u32(dst)), "l"(map), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2)
      : "memory");
}
SBR_DEV void bulk_load(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}

template <int NS>
__global__ void __launch_bounds__(128, 1) stream_kernel(const __grid_constant__ CUtensorMap map, int mode,
                                                        const __half* tiles, int NT, int NTg, int C, int64_t T) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint64_t* full = (uint64_t*)(smem + NS * 32768);
  uint64_t* empty = full + NS;
  const int64_t t_beg = (int64_t)blockIdx.x * T / gridDim.x, t_end = (int64_t)(blockIdx.x + 1) * T / gridDim.x;
  if (threadIdx.x == 0) {
    for (int i = 0; i < NS; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    mbar_fence_init();
  }
  __syncthreads();
  PassWalk w;
  if (threadIdx.x == 0) {
    int st = 0; uint32_t ph = 0;
    for (w.start(NT, C, t_beg, t_end - t_beg); w.valid(); w.next()) {
      mbar_wait(&empty[st], ph ^ 1);
      mbar_expect_tx(&full[st], 32768);
      uint8_t* dst = smem + st * 32768;
      const int gi = w.I + 1, gj = w.J + 1;   // block-0-like origin one tile in
      if (mode == 0) {
        for (int rb = 0; rb < 2; ++rb) tma_load_2d(dst + rb * 16384, &map, &full[st], 96 + gi * 128 + rb * 64, 96 + gj * 128);
      } else if (mode == 1) {
        for (int rb = 0; rb < 2; ++rb) tma_load_3d(dst + rb * 16384, &map, &full[st], rb * 64, 0, gi + gj * NTg);
      } else {
        bulk_load(dst, tiles + ((int64_t)gi + (int64_t)gj * NTg) * 16384, 32768, &full[st]);
      }
      if (++st == NS) { st = 0; ph ^= 1; }
    }
  } else if (threadIdx.x == 32) {
    int st = 0; uint32_t ph = 0;
    for (w.start(NT, C, t_beg, t_end - t_beg); w.valid(); w.next()) {
      mbar_wait(&full[st], ph);
      mbar_arrive(&empty[st]);
      if (++st == NS) { st = 0; ph ^= 1; }
    }
  }
  __syncthreads();
}

typedef CUresult (*EncFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                          const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                          CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  const int n = 32768, NTg = 257;
  const int64_t ldsh = 32896;
  EncFn enc = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q);
  const size_t bytes_cm = sizeof(__half) * ldsh * (n + 128);
  const size_t bytes_t = sizeof(__half) * (size_t)NTg * NTg * 16384;
  __half *cm, *tl;
  cudaMalloc(&cm, bytes_cm);
  cudaMalloc(&tl, bytes_t);
  cudaMemset(cm, 0, bytes_cm);
  cudaMemset(tl, 0, bytes_t);
  CUtensorMap m2, m3;
  {
    cuuint64_t dims[2] = {(cuuint64_t)n + 128, (cuuint64_t)n + 128};
    cuuint64_t str[1] = {(cuuint64_t)ldsh * 2};
    cuuint32_t box[2] = {64, 128}, es[2] = {1, 1};
    CUresult r = enc(&m2, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, cm, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r) printf("enc2 %d\n", (int)r);
  }
  {
    cuuint64_t dims[3] = {128, 128, (cuuint64_t)NTg * NTg};
    cuuint64_t str[2] = {256, 32768};
    cuuint32_t box[3] = {64, 128, 1}, es[3] = {1, 1, 1};
    CUresult r = enc(&m3, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 3, tl, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r) printf("enc3 %d\n", (int)r);
  }
  int nsm = 0;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (int NT : {255, 128, 64}) {
    for (int C : {8}) {
      const int64_t T = pass_total_tiles(NT, C);
      for (int NSv : {4, 6}) {
        for (int mode = 0; mode < 3; ++mode) {
          auto kern = NSv == 4 ? stream_kernel<4> : stream_kernel<6>;
          const int smem = NSv * 32768 + 1024 + 256;
          cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
          const CUtensorMap& mp = mode == 1 ? m3 : m2;
          for (int it = 0; it < 3; ++it) kern<<<nsm, 128, smem>>>(mp, mode, tl, NT, NTg, C, T);
          const int reps = 20;
          cudaEventRecord(e0);
          for (int it = 0; it < reps; ++it) kern<<<nsm, 128, smem>>>(mp, mode, tl, NT, NTg, C, T);
          cudaEventRecord(e1);
          cudaEventSynchronize(e1);
          float ms = 0;
          cudaEventElapsedTime(&ms, e0, e1);
          const double us = 1e3 * ms / reps;
          printf("NT=%3d C=%d NS=%d mode=%d: %8.1f us/launch  %7.1f GB/s  (%s)\n", NT, C, NSv, mode, us,
                 T * 32768.0 / us * 1e-3, cudaGetErrorString(cudaGetLastError()));
        }
      }
    }
  }
  return 0;
}
