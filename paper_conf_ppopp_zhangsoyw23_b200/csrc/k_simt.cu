// k_simt.cu -- fp32 SIMT building blocks for the skinny WY steps (a3, a5) and the
// first (pre-tensor-core) versions of the pass (a4) and trailing SYR2K (a6).
#include "common.cuh"
#include "kernels.h"

namespace sbr {

// ---------------------------------------------------------------- gemm_tn
// C[m1 x n2] += alpha * A^T B over `rows` rows; each CTA: 64x64 output tile over a
// row chunk, atomically accumulated (C zeroed by the caller).
constexpr int TN_T = 64, TN_KC = 32;

__global__ void __launch_bounds__(256) gemm_tn_kernel(int64_t rows, int64_t chunk, int m1, int n2, float alpha,
                                                      const float* __restrict__ A, int64_t lda,
                                                      const float* __restrict__ B, int64_t ldb, float* C,
                                                      int64_t ldc) {
  pdl_trigger();   // 3xTF32 / SIMT chain: launched with PDL (launch_pdl), waits before any access
  pdl_wait();
  __shared__ float As[TN_KC][TN_T + 1];
  __shared__ float Bs[TN_KC][TN_T + 1];
  const int i0 = blockIdx.x * TN_T, j0 = blockIdx.y * TN_T;
  const int64_t r_beg = (int64_t)blockIdx.z * chunk;
  const int64_t r_end = min(rows, r_beg + chunk);
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  float acc[4][4] = {};
  for (int64_t r0 = r_beg; r0 < r_end; r0 += TN_KC) {
    for (int e = threadIdx.x; e < TN_KC * TN_T; e += 256) {
      const int rr = e % TN_KC, cc = e / TN_KC;
      const int64_t r = r0 + rr;
      const bool ok = r < r_end;
      As[rr][cc] = (ok && i0 + cc < m1) ? A[r + (int64_t)(i0 + cc) * lda] : 0.f;
      Bs[rr][cc] = (ok && j0 + cc < n2) ? B[r + (int64_t)(j0 + cc) * ldb] : 0.f;
    }
    __syncthreads();
#pragma unroll 8
    for (int rr = 0; rr < TN_KC; ++rr) {
      float a[4], bb[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) { a[u] = As[rr][ty * 4 + u]; bb[u] = Bs[rr][tx * 4 + u]; }
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
      const int i = i0 + ty * 4 + u, j = j0 + tx * 4 + v;
      if (i < m1 && j < n2) atomicAdd(&C[i + (int64_t)j * ldc], alpha * acc[u][v]);
    }
}

// Skinny reduction C[m1 x n2] += alpha * A^T B over `rows` (n2 <= 32): the 3xTF32 chain's
// G = Y^T W0 and W^T X_t.  64 x 32 output tiles (no half-empty 64 x 64 tile at n2 = b = 32),
// rows split to fill every SM twice, register prefetch of the next 64-row chunk, fp32 atomics.
__global__ void __launch_bounds__(256) skinny_tn32_kernel(int64_t rows, int64_t chunk, int m1, int n2, float alpha,
                                                          const float* __restrict__ A, int64_t lda,
                                                          const float* __restrict__ B, int64_t ldb, float* C,
                                                          int64_t ldc) {
  pdl_trigger();   // 3xTF32 / SIMT chain: launched with PDL (launch_pdl), waits before any access
  pdl_wait();
  constexpr int KC = 64, TI = 64, TJ = 32;
  __shared__ float As[TI][KC + 1];
  __shared__ float Bs[TJ][KC + 1];
  const int i0 = blockIdx.x * TI;
  const int64_t r_beg = (int64_t)blockIdx.z * chunk, r_end = min(rows, r_beg + chunk);
  const int ti = threadIdx.x & 15, tj = threadIdx.x >> 4;   // outputs i = ti*4 .. +3, j = tj*2 .. +1
  float acc[4][2] = {};
  float ra[16], rb[8];
  auto load = [&](int64_t r0) {
#pragma unroll
    for (int q = 0; q < 16; ++q) {   // A: 64 rows (contiguous) x 64 columns
      const int e = threadIdx.x + q * 256, rr = e & (KC - 1), ii = e >> 6;
      const int64_t r = r0 + rr;
      ra[q] = (r < r_end && i0 + ii < m1) ? __ldg(A + r + (int64_t)(i0 + ii) * lda) : 0.f;
    }
#pragma unroll
    for (int q = 0; q < 8; ++q) {    // B: 64 rows x 32 columns
      const int e = threadIdx.x + q * 256, rr = e & (KC - 1), jj = e >> 6;
      const int64_t r = r0 + rr;
      rb[q] = (r < r_end && jj < n2) ? __ldg(B + r + (int64_t)jj * ldb) : 0.f;
    }
  };
  if (r_beg < r_end) load(r_beg);
  for (int64_t r0 = r_beg; r0 < r_end; r0 += KC) {
    __syncthreads();
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      const int e = threadIdx.x + q * 256;
      As[e >> 6][e & (KC - 1)] = ra[q];
    }
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const int e = threadIdx.x + q * 256;
      Bs[e >> 6][e & (KC - 1)] = rb[q];
    }
    __syncthreads();
    if (r0 + KC < r_end) load(r0 + KC);
#pragma unroll 16
    for (int rr = 0; rr < KC; ++rr) {
      float a[4], bb[2];
#pragma unroll
      for (int u = 0; u < 4; ++u) a[u] = As[ti * 4 + u][rr];
      bb[0] = Bs[tj * 2][rr];
      bb[1] = Bs[tj * 2 + 1][rr];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        acc[u][0] = fmaf(a[u], bb[0], acc[u][0]);
        acc[u][1] = fmaf(a[u], bb[1], acc[u][1]);
      }
    }
  }
#pragma unroll
  for (int u = 0; u < 4; ++u)
#pragma unroll
    for (int v = 0; v < 2; ++v) {
      const int i = i0 + ti * 4 + u, j = tj * 2 + v;
      if (i < m1 && j < n2) atomicAdd(&C[i + (int64_t)j * ldc], alpha * acc[u][v]);
    }
}

cudaError_t gemm_tn(int64_t rows, int m1, int n2, float alpha, const float* A, int64_t lda, const float* B,
                    int64_t ldb, float* C, int64_t ldc, cudaStream_t st) {
  if (rows <= 0 || m1 <= 0 || n2 <= 0) return cudaSuccess;
  if (n2 <= 32) {
    // ~8 CTAs per SM (126 registers, 25 KB smem: 2 resident, the rest hides the tail): measured
    // 2 per SM left 18% of the warp slots active (ncu, config 3) with a half-empty second wave
    const int gx = (m1 + 63) / 64;
    int64_t want = std::max<int64_t>(1, (8 * 148 + gx - 1) / gx);
    int64_t chunk = std::max<int64_t>((rows + want - 1) / want, 64);
    chunk = (chunk + 63) / 64 * 64;
    const int gz = (int)((rows + chunk - 1) / chunk);
    return launch_pdl(skinny_tn32_kernel, dim3(gx, 1, gz), dim3(256), 0, st, rows, chunk, m1, n2, alpha, A, lda, B, ldb,
                      C, ldc);
  }
  const int gx = (m1 + TN_T - 1) / TN_T, gy = (n2 + TN_T - 1) / TN_T;
  int64_t want = std::max<int64_t>(1, 296 / (gx * gy));
  int64_t chunk = (rows + want - 1) / want;
  chunk = std::max<int64_t>(chunk, 256);
  chunk = (chunk + TN_KC - 1) / TN_KC * TN_KC;
  const int gz = (int)((rows + chunk - 1) / chunk);
  return launch_plain(gemm_tn_kernel, dim3(gx, gy, gz), dim3(256), 0, st, rows, chunk, m1, n2, alpha, A, lda, B, ldb, C,
                    ldc);
}

// ---------------------------------------------------------------- gemm_nn
// D = beta*C + alpha*A*op(B); 64x64 tiles, K in chunks of 32; C/D may alias.
constexpr int NN_T = 64, NN_KC = 32;

__global__ void __launch_bounds__(256) gemm_nn_kernel(int64_t M, int N, int K, float alpha,
                                                      const float* __restrict__ A, int64_t lda,
                                                      const float* __restrict__ B, int64_t ldb, bool transB,
                                                      float beta, const float* C, int64_t ldc, float* D,
                                                      int64_t ldd) {
  pdl_trigger();   // 3xTF32 / SIMT chain: launched with PDL (launch_pdl), waits before any access
  pdl_wait();
  __shared__ float As[NN_KC][NN_T + 1];
  __shared__ float Bs[NN_KC][NN_T + 1];
  const int64_t i0 = (int64_t)blockIdx.x * NN_T;
  const int j0 = blockIdx.y * NN_T;
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  float acc[4][4] = {};
  for (int k0 = 0; k0 < K; k0 += NN_KC) {
    for (int e = threadIdx.x; e < NN_KC * NN_T; e += 256) {
      {  // A tile: rows i0.., k k0..; coalesce along rows
        const int ii = e % NN_T, kk = e / NN_T;
        const int64_t i = i0 + ii;
        const int k = k0 + kk;
        As[kk][ii] = (i < M && k < K) ? A[i + (int64_t)k * lda] : 0.f;
      }
      if (!transB) {  // B(k, j) at B[k + j ldb]; coalesce along k
        const int kk = e % NN_KC, jj = e / NN_KC;
        const int k = k0 + kk, j = j0 + jj;
        Bs[kk][jj] = (k < K && j < N) ? B[k + (int64_t)j * ldb] : 0.f;
      } else {        // op(B)(k, j) = B[j + k ldb]; coalesce along j
        const int jj = e % NN_T, kk = e / NN_T;
        const int k = k0 + kk, j = j0 + jj;
        Bs[kk][jj] = (k < K && j < N) ? B[j + (int64_t)k * ldb] : 0.f;
      }
    }
    __syncthreads();
#pragma unroll 8
    for (int kk = 0; kk < NN_KC; ++kk) {
      float a[4], bb[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) { a[u] = As[kk][ty + 16 * u]; bb[u] = Bs[kk][tx * 4 + u]; }
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
      const int64_t i = i0 + ty + 16 * u;
      const int j = j0 + tx * 4 + v;
      if (i < M && j < N) {
        const float c = (beta != 0.f) ? beta * C[i + (int64_t)j * ldc] : 0.f;
        D[i + (int64_t)j * ldd] = c + alpha * acc[u][v];
      }
    }
}

// ---------------------------------------------------------------- skinny in-place update (3xTF32 chain)
// D[M x N] += alpha * A[M x K] op(B), N <= 64, fp32 SIMT: the skinny steps a3/a5 of the 3xTF32
// mode (X Y_c^T, Y P, W G).  Bound by fp32 FMA issue (8 FMA per A byte at N = 32), so the grid
// is 128-row blocks x a K split sized to fill every SM twice; partial sums go to D with fp32
// atomics (D = C in place, beta = 1).  Per thread 4 rows x NG*4 columns; A / B chunks of 32 K
// staged through shared memory with a register prefetch of the next chunk.
// A second segment (K1 > 0) appends A1 op(B1) along K: D += alpha (A op(B) + A1 op(B1)) in one
// launch (the 3xTF32 lazy update X Y_c^T + Y P).
template <int NG>   // NG = N / 32 rounded up (1 or 2)
__global__ void __launch_bounds__(256) skinny_upd_kernel(int64_t M, int N, int K, int kper, float alpha,
                                                         const float* __restrict__ A, int64_t lda,
                                                         const float* __restrict__ B, int64_t ldb, bool transB,
                                                         float* D, int64_t ldd, int K0,
                                                         const float* __restrict__ A1, int64_t lda1,
                                                         const float* __restrict__ B1, int64_t ldb1, bool transB1) {
  pdl_trigger();   // 3xTF32 / SIMT chain: launched with PDL (launch_pdl), waits before any access
  pdl_wait();
  constexpr int RB = 128, KC = 32, NC = 32 * NG;
  __shared__ __align__(16) float As[KC][RB];
  __shared__ __align__(16) float Bs[KC][NC];
  const int64_t i0 = (int64_t)blockIdx.x * RB;
  const int kb = blockIdx.y * kper, ke = min(K, kb + kper);
  const int tr = threadIdx.x & 31, tc = threadIdx.x >> 5;   // rows tr*4.., cols tc*4*NG..
  float acc[4][4 * NG];
#pragma unroll
  for (int u = 0; u < 4; ++u)
#pragma unroll
    for (int v = 0; v < 4 * NG; ++v) acc[u][v] = 0.f;
  float ra[16], rbv[4 * NG];
  auto load = [&](int k0) {
#pragma unroll
    for (int q = 0; q < 16; ++q) {   // A: 32 k x 128 rows, rows contiguous
      const int e = threadIdx.x + q * 256, ii = e & (RB - 1), kk = e >> 7;
      const int64_t i = i0 + ii;
      const int k = k0 + kk;
      ra[q] = (i < M && k < ke) ? __ldg(k < K0 ? A + i + (int64_t)k * lda : A1 + i + (int64_t)(k - K0) * lda1) : 0.f;
    }
#pragma unroll
    for (int q = 0; q < 4 * NG; ++q) {   // B: 32 k x NC columns (the layout of the chunk's first segment)
      const int e = threadIdx.x + q * 256;
      const bool tb = (k0 < K0) ? transB : transB1;
      int kk, jj;
      if (tb) { jj = e % NC; kk = e / NC; } else { kk = e % KC; jj = e / KC; }
      const int k = k0 + kk;
      const float* bp = k < K0 ? (transB ? B + jj + (int64_t)k * ldb : B + k + (int64_t)jj * ldb)
                               : (transB1 ? B1 + jj + (int64_t)(k - K0) * ldb1 : B1 + (k - K0) + (int64_t)jj * ldb1);
      rbv[q] = (k < ke && jj < N) ? __ldg(bp) : 0.f;
    }
  };
  bool tbs = transB;   // B layout of the chunk whose loads are in rbv
  auto store = [&]() {
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      const int e = threadIdx.x + q * 256;
      As[e >> 7][e & (RB - 1)] = ra[q];
    }
#pragma unroll
    for (int q = 0; q < 4 * NG; ++q) {
      const int e = threadIdx.x + q * 256;
      if (tbs) Bs[e / NC][e % NC] = rbv[q];
      else Bs[e % KC][e / KC] = rbv[q];
    }
  };
  if (kb < ke) load(kb);
  for (int k0 = kb; k0 < ke; k0 += KC) {
    __syncthreads();
    tbs = (k0 < K0) ? transB : transB1;
    store();
    __syncthreads();
    if (k0 + KC < ke) load(k0 + KC);   // next chunk's loads in flight during this chunk's FMAs
#pragma unroll 8
    for (int kk = 0; kk < KC; ++kk) {
      const float4 a4 = *reinterpret_cast<const float4*>(&As[kk][tr * 4]);
      const float a[4] = {a4.x, a4.y, a4.z, a4.w};
      float bb[4 * NG];
#pragma unroll
      for (int g = 0; g < NG; ++g) {
        const float4 b4 = *reinterpret_cast<const float4*>(&Bs[kk][tc * 4 + 32 * g]);
        bb[4 * g] = b4.x; bb[4 * g + 1] = b4.y; bb[4 * g + 2] = b4.z; bb[4 * g + 3] = b4.w;
      }
#pragma unroll
      for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4 * NG; ++v) acc[u][v] = fmaf(a[u], bb[v], acc[u][v]);
    }
  }
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    const int64_t i = i0 + tr * 4 + u;
    if (i >= M) continue;
#pragma unroll
    for (int g = 0; g < NG; ++g)
#pragma unroll
      for (int v = 0; v < 4; ++v) {
        const int j = tc * 4 + 32 * g + v;
        if (j < N) atomicAdd(D + i + (int64_t)j * ldd, alpha * acc[u][4 * g + v]);
      }
  }
}

cudaError_t gemm_nn(int64_t M, int N, int K, float alpha, const float* A, int64_t lda, const float* B,
                    int64_t ldb, bool transB, float beta, const float* C, int64_t ldc, float* D, int64_t ldd,
                    cudaStream_t st) {
  if (M <= 0 || N <= 0) return cudaSuccess;
  if (N <= 64 && beta == 1.f && C == D && ldc == ldd && K > 0) {   // in-place skinny update
    const int gx = (int)((M + 127) / 128);
    // N <= 32: ~8 CTAs per SM (64 registers: 4 resident; ncu at config 3 saw 25% of the warp slots at
    // 2 per SM); N = 64 keeps 2 per SM (config 5: more K splits doubled the 128 x 64 atomic flushes)
    const int per = N <= 32 ? 8 : 2;
    int ks = std::max(1, std::min((K + 63) / 64, (per * 148 + gx - 1) / gx));
    const int kper = ((K + ks - 1) / ks + 31) / 32 * 32;
    ks = (K + kper - 1) / kper;
    if (N <= 32)
      return launch_pdl(skinny_upd_kernel<1>, dim3(gx, ks), dim3(256), 0, st, M, N, K, kper, alpha, A, lda, B, ldb,
                        transB, D, ldd, K, (const float*)nullptr, (int64_t)0, (const float*)nullptr, (int64_t)0, false);
    return launch_plain(skinny_upd_kernel<2>, dim3(gx, ks), dim3(256), 0, st, M, N, K, kper, alpha, A, lda, B, ldb,
                      transB, D, ldd, K, (const float*)nullptr, (int64_t)0, (const float*)nullptr, (int64_t)0, false);
  }
  dim3 grid((unsigned)((M + NN_T - 1) / NN_T), (N + NN_T - 1) / NN_T);
  return launch_pdl(gemm_nn_kernel, grid, dim3(256), 0, st, M, N, K, alpha, A, lda, B, ldb, transB, beta, C, ldc, D,
                    ldd);
}

// D += alpha (A0 op(B0) + A1 op(B1)), N <= 64, K0 + K1 along K, D in place (fp32 atomics)
cudaError_t skinny_upd2(int64_t M, int N, int K0, const float* A0, int64_t lda0, const float* B0, int64_t ldb0,
                        bool transB0, int K1, const float* A1, int64_t lda1, const float* B1, int64_t ldb1,
                        bool transB1, float alpha, float* D, int64_t ldd, cudaStream_t st) {
  const int K = K0 + K1;
  if (M <= 0 || N <= 0 || K <= 0) return cudaSuccess;
  const int gx = (int)((M + 127) / 128);
  const int per = 8;   // the two-segment lazy update: K = 2k, ~8 CTAs per SM helped at b = 32 and 64
  int ks = std::max(1, std::min((K + 63) / 64, (per * 148 + gx - 1) / gx));
  const int kper = ((K + ks - 1) / ks + 31) / 32 * 32;
  ks = (K + kper - 1) / kper;
  if (N <= 32)
    return launch_pdl(skinny_upd_kernel<1>, dim3(gx, ks), dim3(256), 0, st, M, N, K, kper, alpha, A0, lda0, B0, ldb0,
                      transB0, D, ldd, K0, A1, lda1, B1, ldb1, transB1);
  return launch_pdl(skinny_upd_kernel<2>, dim3(gx, ks), dim3(256), 0, st, M, N, K, kper, alpha, A0, lda0, B0, ldb0,
                    transB0, D, ldd, K0, A1, lda1, B1, ldb1, transB1);
}

// ---------------------------------------------------------------- sym_pass (SIMT v1)
// X = OA * W, OA symmetric (lower storage).  CTA = 64-row block x a range of 64-col
// tiles; tiles above the diagonal are read transposed from the lower triangle.
constexpr int SP_T = 64;

template <int BW>
__global__ void __launch_bounds__(256) sym_pass_kernel(int64_t M, int b, int tiles_per_cta,
                                                       const float* __restrict__ OA, int64_t ld,
                                                       const float* __restrict__ S, int64_t lds, int sw,
                                                       const float* __restrict__ W, int64_t ldw, float* X,
                                                       int64_t ldx) {
  __shared__ float Ts[SP_T][SP_T + 1];
  __shared__ float Ws[SP_T][BW + 1];
  const int64_t I0 = (int64_t)blockIdx.x * SP_T;
  const int64_t nt = (M + SP_T - 1) / SP_T;
  const int64_t jt0 = (int64_t)blockIdx.y * tiles_per_cta;
  const int64_t jt1 = min(nt, jt0 + tiles_per_cta);
  constexpr int OPT = SP_T * BW / 256;  // outputs per thread
  float acc[OPT];
#pragma unroll
  for (int u = 0; u < OPT; ++u) acc[u] = 0.f;
  const int ri = threadIdx.x % SP_T;          // output row within block
  const int cgrp = threadIdx.x / SP_T;        // 4 column groups
  for (int64_t jt = jt0; jt < jt1; ++jt) {
    const int64_t J0 = jt * SP_T;
    for (int e = threadIdx.x; e < SP_T * SP_T; e += 256) {
      const int a = e % SP_T, c = e / SP_T;
      // coalesced index a runs along the stored-contiguous dimension
      int64_t i, j;
      if (J0 <= I0) { i = I0 + a; j = J0 + c; }   // lower (or diagonal) tile: rows contiguous
      else { j = J0 + a; i = I0 + c; }            // upper tile: read (j, i) from lower storage
      float v = 0.f;
      if (i < M && j < M) {
        const int64_t hi = i >= j ? i : j, lo = i >= j ? j : i;
        v = (lo < sw) ? S[hi + lo * lds] : OA[hi + lo * ld];
      }
      if (J0 <= I0) Ts[a][c] = v; else Ts[c][a] = v;
    }
    for (int e = threadIdx.x; e < SP_T * BW; e += 256) {
      const int jj = e % SP_T, c = e / SP_T;
      const int64_t j = J0 + jj;
      Ws[jj][c] = (j < M && c < b) ? W[j + c * ldw] : 0.f;
    }
    __syncthreads();
#pragma unroll 4
    for (int jj = 0; jj < SP_T; ++jj) {
      const float t = Ts[ri][jj];
#pragma unroll
      for (int u = 0; u < OPT; ++u) acc[u] = fmaf(t, Ws[jj][cgrp + 4 * u], acc[u]);
    }
    __syncthreads();
  }
  const int64_t i = I0 + ri;
  if (i < M) {
#pragma unroll
    for (int u = 0; u < OPT; ++u) {
      const int c = cgrp + 4 * u;
      if (c < b) atomicAdd(&X[i + c * ldx], acc[u]);
    }
  }
}

cudaError_t sym_pass(int64_t M, int b, const float* OA, int64_t ldoa, const float* S, int64_t lds, int sw,
                     const float* W, int64_t ldw, float* X, int64_t ldx, cudaStream_t st) {
  cudaError_t e = zero_matrix(M, b, X, ldx, st);
  if (e != cudaSuccess) return e;
  const int64_t nt = (M + SP_T - 1) / SP_T;
  const int tpc = 16;
  dim3 grid((unsigned)nt, (unsigned)((nt + tpc - 1) / tpc));
  if (b <= 16) sym_pass_kernel<16><<<grid, 256, 0, st>>>(M, b, tpc, OA, ldoa, S, lds, sw, W, ldw, X, ldx);
  else if (b <= 32) sym_pass_kernel<32><<<grid, 256, 0, st>>>(M, b, tpc, OA, ldoa, S, lds, sw, W, ldw, X, ldx);
  else sym_pass_kernel<64><<<grid, 256, 0, st>>>(M, b, tpc, OA, ldoa, S, lds, sw, W, ldw, X, ldx);
  return cudaGetLastError();
}

// ---------------------------------------------------------------- syr2k_lower (SIMT v1)
constexpr int SY_T = 64, SY_KC = 16;

__global__ void __launch_bounds__(256) syr2k_lower_kernel(int64_t M, int K, const float* __restrict__ Y,
                                                          int64_t ldy, const float* __restrict__ Z, int64_t ldz,
                                                          float* C, int64_t ldc) {
  __shared__ float Yi[SY_KC][SY_T + 1], Zi[SY_KC][SY_T + 1], Yj[SY_KC][SY_T + 1], Zj[SY_KC][SY_T + 1];
  // linear lower-tile index -> (I, J), I >= J
  const int64_t t = blockIdx.x;
  int64_t I = (int64_t)((sqrt(8.0 * (double)t + 1.0) - 1.0) * 0.5);
  while (I * (I + 1) / 2 > t) --I;
  while ((I + 1) * (I + 2) / 2 <= t) ++I;
  const int64_t J = t - I * (I + 1) / 2;
  const int64_t i0 = I * SY_T, j0 = J * SY_T;
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  float acc[4][4] = {};
  for (int k0 = 0; k0 < K; k0 += SY_KC) {
    for (int e = threadIdx.x; e < SY_KC * SY_T; e += 256) {
      const int rr = e % SY_T, kk = e / SY_T;
      const int k = k0 + kk;
      const int64_t ri = i0 + rr, rj = j0 + rr;
      const bool okk = k < K;
      Yi[kk][rr] = (okk && ri < M) ? Y[ri + (int64_t)k * ldy] : 0.f;
      Zi[kk][rr] = (okk && ri < M) ? Z[ri + (int64_t)k * ldz] : 0.f;
      Yj[kk][rr] = (okk && rj < M) ? Y[rj + (int64_t)k * ldy] : 0.f;
      Zj[kk][rr] = (okk && rj < M) ? Z[rj + (int64_t)k * ldz] : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < SY_KC; ++kk) {
      float yi[4], zi[4], yj[4], zj[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        yi[u] = Yi[kk][ty + 16 * u]; zi[u] = Zi[kk][ty + 16 * u];
        yj[u] = Yj[kk][tx * 4 + u]; zj[u] = Zj[kk][tx * 4 + u];
      }
#pragma unroll
      for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4; ++v) acc[u][v] = fmaf(yi[u], zj[v], fmaf(zi[u], yj[v], acc[u][v]));
    }
    __syncthreads();
  }
#pragma unroll
  for (int u = 0; u < 4; ++u)
#pragma unroll
    for (int v = 0; v < 4; ++v) {
      const int64_t i = i0 + ty + 16 * u, j = j0 + tx * 4 + v;
      if (i < M && j < M && i >= j) C[i + j * ldc] -= acc[u][v];
    }
}

cudaError_t syr2k_lower(int64_t M, int K, const float* Y, int64_t ldy, const float* Z, int64_t ldz, float* C,
                        int64_t ldc, cudaStream_t st) {
  if (M <= 0) return cudaSuccess;
  const int64_t nt = (M + SY_T - 1) / SY_T;
  const int64_t ntiles = nt * (nt + 1) / 2;
  syr2k_lower_kernel<<<(unsigned)ntiles, 256, 0, st>>>(M, K, Y, ldy, Z, ldz, C, ldc);
  return cudaGetLastError();
}

}  // namespace sbr
