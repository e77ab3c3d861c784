// kernels.h -- internal launch interface between the driver (sbr_api.cu) and the kernels.
#pragma once
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <stdint.h>

namespace sbr {

constexpr int kPanelMaxLev = 8;

struct PanelArgs {
  // panel: m x b, column-major in A (rows = OA rows row0 .. row0+m-1)
  float* P;
  int64_t ldp;
  int m, b;
  // block buffers: explicit Y and W columns of this panel, OA row 0 .. M-1
  float* Y;
  int64_t ldy;
  float* W;
  int64_t ldw;
  int64_t row0, M;
  // workspace
  float* ws_v;
  float* ws_tau;
  float* ws_r;
  float* ws_q;
  float* ws_misc;
  // tree (filled by launch_panel)
  int nlev, arity;
  int nodes[kPanelMaxLev];
  int64_t voff[kPanelMaxLev], roff[kPanelMaxLev], toff[kPanelMaxLev], qoff[kPanelMaxLev];
};

struct PanelWs {
  size_t v, tau, r, q, misc;  // floats
};
PanelWs panel_ws_sizes(int64_t m_max, int b);
cudaError_t launch_panel(PanelArgs& a, int max_ctas, cudaStream_t st);
int panel_max_ctas(int b);

// ---- SIMT building blocks (fp32) ----
// C[m1 x n2] (+)= alpha * A[rows x m1]^T B[rows x n2]   (accumulate=1: atomics into C)
cudaError_t gemm_tn(int64_t rows, int m1, int n2, float alpha, const float* A, int64_t lda,
                    const float* B, int64_t ldb, float* C, int64_t ldc, cudaStream_t st);
// D[M x N] = beta*C + alpha * A[M x K] op(B)  ; op(B) = B (K x N, ld) or B^T (B is N x K)
// C and D may alias (in place).
cudaError_t gemm_nn(int64_t M, int N, int K, float alpha, const float* A, int64_t lda,
                    const float* B, int64_t ldb, bool transB, float beta, const float* C, int64_t ldc,
                    float* D, int64_t ldd, cudaStream_t st);

// ---- misc ----
cudaError_t gen_symmetric(uint64_t seed, int64_t n, float* A, int64_t lda, cudaStream_t st);
cudaError_t check_finite(int64_t n, const float* A, int64_t lda, unsigned* flag, cudaStream_t st);
cudaError_t extract_band(int64_t n, int b, const float* A, int64_t lda, float* AB, int64_t ldab,
                         cudaStream_t st);
cudaError_t mirror_lower_block(int b, float* A, int64_t lda, cudaStream_t st);
cudaError_t lazy_small_p(int k, int b, const float* Xc, int64_t ldx, const float* WtX, int64_t ldwx,
                         const float* Yc, int64_t ldy, float* P, cudaStream_t st);
cudaError_t mirror_wtx(int k, int b, float* WtX, int64_t ld, cudaStream_t st);
cudaError_t zero_matrix(int64_t rows, int64_t cols, float* A, int64_t lda, cudaStream_t st);

// ---- the two large contractions ----
// X[:, 0:b] = OA (M x M symmetric, lower referenced) * W (M x b).  OA columns < sw are
// read from the frozen strip copy S (ld lds), the rest from OA.
cudaError_t sym_pass(int64_t M, int b, const float* OA, int64_t ldoa, const float* S, int64_t lds, int sw,
                     const float* W, int64_t ldw, float* X, int64_t ldx, cudaStream_t st);
// C (M x M, lower) -= Y Z^T + Z Y^T, Y, Z: M x K
cudaError_t syr2k_lower(int64_t M, int K, const float* Y, int64_t ldy, const float* Z, int64_t ldz,
                        float* C, int64_t ldc, cudaStream_t st);

}  // namespace sbr
