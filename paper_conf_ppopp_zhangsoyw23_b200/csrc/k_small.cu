// k_small.cu -- fp32 SIMT kernels for the small (k x b, b x b) corrections of the WY steps,
// written for parallelism (split-K with fp32 reductions) since they sit on the serial
// per-panel chain:
//   small_gemm : D (+)= alpha * A op(B) + beta * op(C)   (m, n <= a few thousand, K split)
//     * P = W^T R = X(c,:)^T - (W^T X) Y_c^T          (lazy update)
//     * W^T X_t (rows < k) = H - (W^T X) G            (symmetry of OA)
//   tn_small   : D[b x b] += A^T B over many rows      (W_t^T X_t)
#include "common.cuh"
#include "kernels.h"

namespace sbr {

constexpr int SG_T = 64, SG_KC = 16, SG_SPLIT = 128;

__global__ void __launch_bounds__(256) small_gemm_kernel(int m, int n, int K, float alpha, const float* __restrict__ A,
                                                         int64_t lda, const float* __restrict__ B, int64_t ldb,
                                                         int transB, float beta, const float* __restrict__ C,
                                                         int64_t ldc, int transC, float* D, int64_t ldd) {
  pdl_trigger();   // 3xTF32 / SIMT chain: launched with PDL (launch_pdl), waits before any access
  pdl_wait();
  __shared__ float As[SG_KC][SG_T + 1];
  __shared__ float Bs[SG_KC][SG_T + 1];
  const int i0 = blockIdx.x * SG_T, j0 = blockIdx.y * SG_T;
  const int k0 = blockIdx.z * SG_SPLIT, k1 = min(K, k0 + SG_SPLIT);
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  float acc[4][4] = {};
  for (int kb = k0; kb < k1; kb += SG_KC) {
    for (int e = threadIdx.x; e < SG_KC * SG_T; e += 256) {
      const int ii = e % SG_T, kk = e / SG_T;
      const int k = kb + kk;
      As[kk][ii] = (i0 + ii < m && k < k1) ? A[(i0 + ii) + (int64_t)k * lda] : 0.f;
      if (transB) {
        const int jj = e % SG_T;
        Bs[kk][jj] = (j0 + jj < n && k < k1) ? B[(j0 + jj) + (int64_t)k * ldb] : 0.f;
      } else {
        const int kk2 = e % SG_KC, jj = e / SG_KC;
        Bs[kk2][jj] = (j0 + jj < n && kb + kk2 < k1) ? B[(kb + kk2) + (int64_t)(j0 + jj) * ldb] : 0.f;
      }
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < SG_KC; ++kk) {
      float a[4], bb[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) { a[u] = As[kk][ty + 16 * u]; bb[u] = Bs[kk][tx + 16 * u]; }
#pragma unroll
      for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4; ++v) acc[u][v] = fmaf(a[u], bb[v], acc[u][v]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int u = 0; u < 4; ++u)
#pragma unroll
    for (int v = 0; v < 4; ++v) {
      const int i = i0 + ty + 16 * u, j = j0 + tx + 16 * v;
      if (i < m && j < n) {
        float val = alpha * acc[u][v];
        if (blockIdx.z == 0 && beta != 0.f) val += beta * (transC ? C[j + (int64_t)i * ldc] : C[i + (int64_t)j * ldc]);
        atomicAdd(&D[i + (int64_t)j * ldd], val);
      }
    }
}

cudaError_t small_gemm(int m, int n, int K, float alpha, const float* A, int64_t lda, const float* B, int64_t ldb,
                       bool transB, float beta, const float* C, int64_t ldc, bool transC, float* D, int64_t ldd,
                       cudaStream_t st) {
  if (m <= 0 || n <= 0) return cudaSuccess;
  cudaError_t e = zero_matrix(m, n, D, ldd, st);
  if (e != cudaSuccess) return e;
  dim3 grid((m + SG_T - 1) / SG_T, (n + SG_T - 1) / SG_T, std::max(1, (K + SG_SPLIT - 1) / SG_SPLIT));
  return launch_pdl(small_gemm_kernel, grid, dim3(256), 0, st, m, n, K, alpha, A, lda, B, ldb, transB ? 1 : 0, beta, C,
                    ldc, transC ? 1 : 0, D, ldd);
}

// D[b x b] += A[rows x b]^T B[rows x b]   (fp32, column-major; D zeroed here)
constexpr int TS_R = 64;
__global__ void __launch_bounds__(256) tn_small_kernel(int64_t rows, int b, const float* __restrict__ A, int64_t lda,
                                                       const float* __restrict__ B, int64_t ldb, float* D,
                                                       int64_t ldd) {
  __shared__ float As[TS_R][65];
  __shared__ float Bs[TS_R][65];
  const int64_t r0 = (int64_t)blockIdx.x * TS_R;
  const int nr = (int)std::min<int64_t>(TS_R, rows - r0);
  for (int e = threadIdx.x; e < TS_R * b; e += 256) {
    const int r = e % TS_R, c = e / TS_R;
    As[r][c] = r < nr ? A[(r0 + r) + (int64_t)c * lda] : 0.f;
    Bs[r][c] = r < nr ? B[(r0 + r) + (int64_t)c * ldb] : 0.f;
  }
  __syncthreads();
  for (int o = threadIdx.x; o < b * b; o += 256) {
    const int i = o % b, j = o / b;
    float acc = 0.f;
#pragma unroll 8
    for (int r = 0; r < TS_R; ++r) acc = fmaf(As[r][i], Bs[r][j], acc);
    atomicAdd(&D[i + (int64_t)j * ldd], acc);
  }
}

cudaError_t tn_small(int64_t rows, int b, const float* A, int64_t lda, const float* B, int64_t ldb, float* D,
                     int64_t ldd, cudaStream_t st) {
  cudaError_t e = zero_matrix(b, b, D, ldd, st);
  if (e != cudaSuccess || rows <= 0) return e;
  tn_small_kernel<<<(unsigned)((rows + TS_R - 1) / TS_R), 256, 0, st>>>(rows, b, A, lda, B, ldb, D, ldd);
  return cudaGetLastError();
}

}  // namespace sbr
