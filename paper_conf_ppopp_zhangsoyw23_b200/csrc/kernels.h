// kernels.h -- internal launch interface between the driver (sbr_api.cu) and the kernels.
#pragma once
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <stdint.h>
#include <cuda.h>

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
  __half* Yh;     // optional fp16 row-major copy of Y (row r, column c at Yh[r*ldyh + c])
  int64_t ldyh;
  __half* Wh;     // optional fp16 column-major copy of W^0 (Wh[r + c*ldwh]), rows 0 .. M-1
  int64_t ldwh;
  __half* Wrh;    // optional fp16 row-major copy of W^0 (Wrh[r*ldwrh + c]), rows 0 .. M-1
  int64_t ldwrh;
  int64_t row0, M;
  // workspace
  float* ws_v;
  float* ws_tau;
  float* ws_r;
  float* ws_q;
  float* ws_misc;
  int64_t* trace;  // optional: CTA 0 phase timestamps (globaltimer ns), 10 entries
  const int* run_if;  // TSQR only: if non-NULL, do nothing unless *run_if != 0 (CholQR fallback)
  double orth_tol;    // CholeskyQR acceptance: max|Q^T Q - I| (fp64) <= orth_tol (0: default 1e-9)
  int over_capacity;  // set by launch_panel: the TSQR tree needs more co-resident CTAs than exist (no launch)
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
// CholeskyQR panel (k_panel_chol.cu): b in {8,16,32,64}; returns cudaErrorNotSupported when it
// does not apply (then run TSQR).  A declined panel (rank deficient / not orthonormal after
// three rounds) is factored by Householder QR in the same launch.  ws: panel_chol_ws_bytes()
// bytes, zeroed once at allocation; launch: per-handle launch counter (buffers are
// double-buffered by its parity).
size_t panel_chol_ws_bytes();
int* panel_chol_fail(void* ws);
unsigned* panel_chol_declines(void* ws);   // count of declined CholeskyQR panels (device)
cudaError_t launch_panel_chol(PanelArgs& a, void* ws, unsigned launch, cudaStream_t st);

// ---- SIMT building blocks (fp32) ----
// C[m1 x n2] (+)= alpha * A[rows x m1]^T B[rows x n2]   (accumulate=1: atomics into C)
cudaError_t gemm_tn(int64_t rows, int m1, int n2, float alpha, const float* A, int64_t lda,
                    const float* B, int64_t ldb, float* C, int64_t ldc, cudaStream_t st);
// D[M x N] = beta*C + alpha * A[M x K] op(B)  ; op(B) = B (K x N, ld) or B^T (B is N x K)
// C and D may alias (in place).
cudaError_t skinny_upd2(int64_t M, int N, int K0, const float* A0, int64_t lda0, const float* B0, int64_t ldb0,
                        bool transB0, int K1, const float* A1, int64_t lda1, const float* B1, int64_t ldb1,
                        bool transB1, float alpha, float* D, int64_t ldd, cudaStream_t st);
cudaError_t gemm_nn(int64_t M, int N, int K, float alpha, const float* A, int64_t lda,
                    const float* B, int64_t ldb, bool transB, float beta, const float* C, int64_t ldc,
                    float* D, int64_t ldd, cudaStream_t st);

// ---- small split-K SIMT kernels (k_small.cu); D is zeroed and accumulated atomically ----
// D = alpha * A op(B) + beta * op(C); op(B) = B^T (B stored n x K) if transB; op(C) = C^T if transC
cudaError_t small_gemm(int m, int n, int K, float alpha, const float* A, int64_t lda, const float* B, int64_t ldb,
                       bool transB, float beta, const float* C, int64_t ldc, bool transC, float* D, int64_t ldd,
                       cudaStream_t st);
// D[b x b] = A^T B over `rows` rows
cudaError_t tn_small(int64_t rows, int b, const float* A, int64_t lda, const float* B, int64_t ldb, float* D,
                     int64_t ldd, cudaStream_t st);

// ---- misc ----
cudaError_t gen_symmetric(uint64_t seed, int64_t n, float* A, int64_t lda, cudaStream_t st);
// Local -> global column map of a rank's 1D block-cyclic storage (sbr_reduce_dist): local column
// lc holds global column ((lc / nbo) P + rank) nbo + lc % nbo.  P = 1: identity.
struct ColMap {
  int P = 1, rank = 0;
  int64_t nbo = 1;
  __host__ __device__ int64_t g(int64_t lc) const { return P <= 1 ? lc : ((lc / nbo) * P + rank) * nbo + lc % nbo; }
};
// a0: scan[0] = ||A_lower||_F^2 over the local columns, scan[1] = count of non-finite entries (2
// doubles, summed over ranks by the caller if distributed); then choose_scale: flag[0] = 1 if any
// Inf/NaN (k = a sentinel: the matrix is zeroed), else *kexp = k of 2^k with ||A||_F 2^k in
// [2^12, 2^13)
cudaError_t prep_scan(int64_t n, int64_t ncols, const float* A, int64_t lda, ColMap cm, double* scan,
                      cudaStream_t st);
cudaError_t choose_scale(const double* scan, unsigned* flag, int* kexp, cudaStream_t st);
// 3xTF32 mode: A's lower triangle *= 2^k in place (the FP16 mode does it in shadow_init)
cudaError_t scale_lower(int64_t n, int64_t ncols, float* A, int64_t lda, ColMap cm, const int* kexp, cudaStream_t st);
cudaError_t note_unhandled(const int* fail, unsigned* sticky, cudaStream_t st);
// band out, unscaled by 2^-k (kexp may be NULL: k = 0); A's band rewritten unscaled; a non-finite
// band entry sets flag[2] (flag may be NULL)
cudaError_t extract_band(int64_t n, int b, float* A, int64_t lda, float* AB, int64_t ldab, const int* kexp,
                         unsigned* flag, cudaStream_t st, int64_t ncols = -1, ColMap cm = ColMap());
cudaError_t mirror_lower_block(int b, float* A, int64_t lda, cudaStream_t st);
cudaError_t lazy_small_p(int k, int b, const float* Xc, int64_t ldx, const float* WtX, int64_t ldwx,
                         const float* Yc, int64_t ldy, float* P, cudaStream_t st);
cudaError_t mirror_wtx(int k, int b, float* WtX, int64_t ld, cudaStream_t st);
cudaError_t zero_matrix(int64_t rows, int64_t cols, float* A, int64_t lda, cudaStream_t st);
// Wo[:, c] = W[:, c] for rows r >= (c / nb) nb + b, 0 above (columns c < n - b)
cudaError_t copy_block_w(int64_t n, int b, int nb, const float* W, int64_t ldw, float* Wo, int64_t ldwo, cudaStream_t st);

// ---- the two large contractions ----
// X[:, 0:b] = OA (M x M symmetric, lower referenced) * W (M x b).  OA columns < sw are
// read from the frozen strip copy S (ld lds), the rest from OA.
cudaError_t sym_pass(int64_t M, int b, const float* OA, int64_t ldoa, const float* S, int64_t lds, int sw,
                     const float* W, int64_t ldw, float* X, int64_t ldx, cudaStream_t st);
// C (M x M, lower) -= Y Z^T + Z Y^T, Y, Z: M x K
cudaError_t syr2k_lower(int64_t M, int K, const float* Y, int64_t ldy, const float* Z, int64_t ldz,
                        float* C, int64_t ldc, cudaStream_t st);

// ---- tcgen05 / TMA path (FP16 mode) ----
cudaError_t make_tmap_2d(CUtensorMap* map, const void* base, bool fp16, uint64_t inner, uint64_t outer, uint64_t ld,
                         uint32_t box_inner, uint32_t box_outer, int l2_promo = 256);

struct PassLaunch {
  const __half* shadow;  // n x n fp16 shadow of the trailing matrix (strict lower, half diag, zero upper)
  int64_t n, ld_shadow;
  const __half* Wh;      // M x BN fp16, column-major, ld_wh >= M (multiple of 8)
  int64_t M, ld_wh;
  int64_t r0;            // OA origin (global row/col of OA(0,0))
  int b;
  float* X;              // M x b fp32 output (zeroed by the caller), column-major
  int64_t ldx;
  int num_sms;
  int seg_rows;
  int rank = 0, nranks = 1;   // tile share of this launch: [T*rank/nranks, T*(rank+1)/nranks) of the walked tiles
  // multi-GPU column ownership (sbr_reduce_dist): the shadow holds the columns of blocks J % own_P
  // == own_rank only (shadow_cols of them, local column = (g / nbo / own_P) nbo + g % nbo); r0 is
  // then the 128-aligned origin of the tile grid and `off` the OA row of its first row (W stored
  // with `off` zero rows in front, X rows = tile rows - off)
  int own_P = 1, own_rank = 0;
  int64_t nbo = 0, shadow_cols = 0;
  int off = 0;
};
cudaError_t launch_pass_tc(const PassLaunch& p, cudaStream_t st);
// host mirror of the pass's tile order (k_pass_tc.cu PassWalk): share of `rank`, and the (I, J) list
void pass_partition(int64_t M, int b, int rank, int nranks, int64_t* t0, int64_t* t1, int64_t* total);
void pass_tiles(int64_t M, int b, int64_t t0, int64_t t1, int* IJ);
int pass_bn(int b);
int pass_dist_align(int b);
int64_t pass_owned_tiles(int64_t M, int b, int64_t r0g, int off, int64_t nbo, int P, int rank, int* IJ, int64_t cap);   // column-block width multiple the distributed pass needs (128 x tile columns per group)

// 3xTF32 pass (k_pass_tf32.cu): X (M x b, b <= 32, column-major, zeroed by the caller) +=
// OA WS with OA = A[r0:, r0:] (fp32 master, lower referenced, lda % 4 == 0) except tile
// columns J < ceil(sw/128), read from the strip S (M x >= min(128 ceil(sw/128), M), ld lds).
// WS: M x 64 column-major [W_hi (32 cols) | W_lo (32 cols)] from split_tf32_w (bn = 32).
struct PassTf32Launch {
  const float* A; int64_t n, lda, r0;   // OA = A[r0:, r0:] (global rows / columns)
  const float* S; int64_t lds; int64_t sw;
  const float* WS; int64_t ldws;
  int64_t M;
  int b;
  float* X; int64_t ldx;
  int num_sms;
  // sbr_reduce_dist: the 128-aligned tile grid starts `off` rows / columns before OA (at the
  // block start); only tile columns of this rank's nb-blocks are visited; A holds `ncols` local
  // columns (1D block-cyclic, nb = nbo)
  int off = 0;
  int own_P = 1, own_rank = 0;
  int64_t nbo = 0, ncols = 0;
};
cudaError_t launch_pass_tf32(const PassTf32Launch& p, cudaStream_t st);
int64_t pass_tf32_tiles(int64_t M);

struct GemmTcLaunch {
  // fp16 row-major operands (K contiguous): A rows = output rows, B rows = output cols
  const __half *A0, *A1, *B0, *B1;  // SYR2K: A=[Y|Z] (A0=Yh, A1=Zh), B=[Z|Y]; ZFORM: A0=Yh, B0=WtXh
  int64_t K;                        // K per half (columns of the operand arrays used)
  int64_t a_rows, ld_a, b_rows, ld_b;
  int64_t arow0, brow0;             // first operand row of output row/col 0
  int64_t Mrows, Ncols;             // output size
  float* C; int64_t ldc;            // SYR2K: fp32 master (lower), column-major
  __half* shadow; int64_t ld_shadow;
  const float* X; int64_t ldx;      // ZFORM: X (column-major fp32)
  __half* Zh; int64_t ldz;          // ZFORM: Z out (row-major fp16)
  int num_sms;
  // 3xTF32 (launch_*_tf32): A0..B1 point at fp32 row-major [hi | lo] arrays (cast), lo at
  // column lo_off >= round_up(K, 32); hi columns [K, lo_off) must be zero.  ZFORM writes Zs
  // (fp32 row-major, ld ldz) in the same split layout.
  int64_t lo_off = 0;
  float* Zs = nullptr;
  int64_t zlo_off = -1;   // lo offset of the Zs output (default lo_off)
  // SYR2K column ownership (sbr_reduce_dist): output column rel is global column own_org + rel,
  // updated only if ((own_org + rel) / nbo) % own_P == own_rank, at LOCAL column
  // (g / nbo / own_P) nbo + g % nbo of C / shadow (which then point at the region's first row,
  // column 0).  own_P = 1: every tile; C / shadow point at the region's origin.
  int own_P = 1, own_rank = 0;
  int64_t own_org = 0, nbo = 1;
};
cudaError_t launch_syr2k_tc(const GemmTcLaunch& p, cudaStream_t st);
cudaError_t launch_zform_tc(const GemmTcLaunch& p, cudaStream_t st);
cudaError_t launch_syr2k_tf32(const GemmTcLaunch& p, cudaStream_t st);
cudaError_t launch_zform_tf32(const GemmTcLaunch& p, cudaStream_t st);
// general 3xTF32 products (sbr_form_q): Zs = split(A B^T) (row-major [hi | lo], Mrows x Ncols),
// and C (column-major fp32, Mrows x Ncols) -= A B^T
cudaError_t launch_gemm_split_tf32(const GemmTcLaunch& p, cudaStream_t st);
cudaError_t launch_gemm_sub_tf32(const GemmTcLaunch& p, cudaStream_t st);
// column-major src (rows x cols) -> dst row c = split of column c: dst[c*ldd + r] = rna_tf32(a),
// dst[c*ldd + lo_off + r] = rna_tf32(a - hi), zeros in [rows, lo_off).  unit_y: src is the Y of
// sbr_reduce's output (column c: zero above row c, 1 at row c, the stored tail below).
cudaError_t split_tf32_cm(int64_t rows, int cols, const float* src, int64_t lds, bool unit_y, float* dst,
                          int64_t ldd, int64_t lo_off, cudaStream_t st);
cudaError_t set_identity(int64_t n, float* Q, int64_t ldq, cudaStream_t st);
// fp32 column-major src (rows x cols) -> row-major split dst: dst[r*ldd + c] = rna_tf32(a),
// dst[r*ldd + lo_off + c] = rna_tf32(a - hi), zeros in hi columns [cols, lo_off)
cudaError_t split_tf32_rm(int64_t rows, int cols, const float* src, int64_t lds, float* dst, int64_t ldd,
                          int64_t lo_off, cudaStream_t st);
// fp32 column-major W (rows x b) -> column-major [W_hi | W_lo] (rows x 2*bn, hi cols [0,bn), lo [bn, 2bn);
// pad columns b..bn-1 zero), the B operand of the 3xTF32 pass
// inverse of split_tf32_rm (tests): dst[r + c*ldd] = src[r*lds + c] + src[r*lds + lo_off + c]
cudaError_t splitsum_rm_to_cm(int64_t rows, int cols, const float* src, int64_t lds, int64_t lo_off, float* dst,
                              int64_t ldd, cudaStream_t st);
cudaError_t split_tf32_w(int64_t rows, int b, int bn, const float* W, int64_t ldw, float* dst, int64_t ldd,
                         cudaStream_t st);

// skinny tcgen05 GEMMs (k_skinny_tc.cu)
struct SkinnyNN {                 // D[rows x b] = C - [A0 | A1] [B0 | B1]^T
  const __half *A0, *A1;          // row-major fp16, K0 / K1 columns used, a_rows x lda
  int64_t K0, K1, a_rows, lda, arow0;
  const __half* B0;               // row-major fp16 (K-major), rows brow0 .. brow0+b-1 of b0_rows, K0 columns
  int64_t ldb0, b0_rows, brow0;
  const __half* B1;               // row-major fp16 b x K1 (may be NULL if K1 == 0)
  int64_t ldb1;
  int64_t rows;
  int b;
  const float* C; int64_t ldc;    // column-major fp32 (may alias D)
  float* D; int64_t ldd;
  __half* Hcm; int64_t ldhc;      // optional fp16 column-major copy of D
  __half* Hrm; int64_t ldhr;      // optional fp16 row-major copy of D
};
cudaError_t launch_skinny_nn(const SkinnyNN& p, cudaStream_t st);
struct SkinnyTN {                 // D0 += A0[rows]^T B[rows], D1 += A1[rows]^T B[rows] (fp32 reductions)
  const __half *A0, *A1;          // row-major fp16 (a_rows x lda), K1 columns; A1 may be NULL
  int64_t K1, a_rows, lda;
  const __half* B;                // column-major fp16 (b_rows x b), ld ldb
  int64_t b_rows, ldb;
  int64_t row0, rows;             // reduction rows [row0, row0+rows)
  int b;
  float *D0, *D1; int64_t ldd;    // K1 x b, column-major, pre-zeroed
  int num_sms;
};
cudaError_t launch_skinny_tn(const SkinnyTN& p, cudaStream_t st);

// per-panel chain helpers (k_chain.cu)
// kxb: D[q, p] = C(q, p) - sum_r WtX[q + r*ldwx] B(r, p),  q < k, p < b, r < k.
//   LAZY  (a5): B(r,p) = Y[(c+p) + r*ldy], C(q,p) = X[(c+p) + q*ldx]  -> Ph[p*ldph + q] = fp16(D)  (P^T)
//               also mirrors the b x b diagonal block of the master at Adiag.
//   MERGE (a3): B(r,p) = G[r + p*ldg],     C(q,p) = H[q + p*ldg]    -> WtX[q + (k+p)*ldwx] = D and its
//               mirror WtX[(k+p) + q*ldwx]; also Gh[r + p*ldgh] = fp16(G(r, p)).
struct KxbArgs {
  int mode;                       // 0 = LAZY, 1 = MERGE
  int k, b;
  float* WtX; int64_t ldwx;
  const float* Y; int64_t ldy; const float* X; int64_t ldx; int64_t c;   // LAZY
  __half* Ph; int64_t ldph;      // fp16 P^T (FP16 chain) ...
  float* P32 = nullptr; int64_t ldp32 = 0;   // ... and/or fp32 P[q + p*ldp32] (3xTF32 / SIMT chain)
  float* Adiag; int64_t lda;
  const float* G; const float* H; int64_t ldg;                           // MERGE
  __half* Gh; int64_t ldgh;
};
cudaError_t launch_kxb(const KxbArgs& a, cudaStream_t st);
// after the pass: Xh[r*ldxh + p] = fp16(X[r + p*ldx]) and WtXtt[i + j*ldw] += sum_r W[r,i] X[r,j]
cudaError_t launch_postpass(int64_t M, int b, const float* X, int64_t ldx, const float* W, int64_t ldw, __half* Xh,
                            int64_t ldxh, float* WtXtt, int64_t ldwtx, cudaStream_t st);
// the postpass and the MERGE kxb's W^T X_t column block (a.Gh unused) as ONE launch of 8-CTA
// clusters (independent work, one dependent step fewer on the per-panel chain); b > 32: two launches
cudaError_t launch_postpass_merge(int64_t M, int b, const float* X, int64_t ldx, const float* W, int64_t ldw,
                                  __half* Xh, int64_t ldxh, float* WtXtt, int64_t ldwtx, const KxbArgs& a,
                                  cudaStream_t st);
// Gh[r + p*ldgh] = fp16(G[r + p*ldg]), r < k, p < b (PDL; the merge GEMM's B operand)
cudaError_t launch_g_to_half(int k, int b, const float* G, int64_t ldg, __half* Gh, int64_t ldgh, cudaStream_t st);

// The fused per-panel chain of the FP16 mode (k_chain_fused.cu): ONE cooperative launch per
// panel t does the previous pass's tail (Xh, W^T X diagonal block), the lazy update, the panel
// QR (CholeskyQR + reconstruction, Householder fallback), and the W merge.  b = 32 only.
struct ChainFusedLaunch {
  int t, k;                        // panel index in the block, k = t b
  int64_t M, tb;                   // block-local order, t b
  float* A; int64_t lda, r0;       // master, OA origin r0
  float* Yb; int64_t ldy;          // block Y fp32 (OA rows)
  float* Wt; int64_t ldw;          // this panel's W columns (OA rows)
  const float* Xb; int64_t ldx;    // X (M x p b)
  __half* Xh;                      // fp16 row-major X (ld ldk)
  float* WtX; int64_t ldwx;
  float* Gf; float* Hf;            // k x 32 fp32 scratch each
  __half* Ph; __half* Yh; __half* Wrh; int64_t ldk;
  __half* Wh; int64_t ldwh;        // fp16 column-major W_t (pass operand)
  void* ws; unsigned launch;       // chain_fused_ws_bytes(), zeroed once; launch counter (parity)
  unsigned* declines;
  double orth_tol;
  int grid;                        // CTAs (= SMs; all co-resident)
  int64_t* trace;                  // optional phase stamps (16 int64, CTA 0)
};
size_t chain_fused_ws_bytes();
bool chain_fused_supported(int b, int64_t M, int num_sms);
cudaError_t launch_chain_fused(const ChainFusedLaunch& L, cudaStream_t st);

// fp16 conversions
cudaError_t f32cm_to_f16rm(int64_t rows, int cols, const float* src, int64_t lds, __half* dst, int64_t ldd,
                           cudaStream_t st);
cudaError_t build_lazy_b(int k, int b, const __half* Yh, int64_t ldyh, int64_t c, const float* P, __half* Bl,
                         int64_t ldbl, cudaStream_t st);
// fp16 shadow of 2^k A (lower; half diagonal; zero upper); with k != 0 also scales A's lower
// triangle in place (kexp may be NULL: k = 0)
cudaError_t shadow_init(int64_t n, float* A, int64_t lda, __half* Sh, int64_t ldsh, const int* kexp,
                        cudaStream_t st, int64_t ncols = -1, ColMap cm = ColMap());
cudaError_t to_half_cm(int64_t rows, int cols, int cols_pad, const float* src, int64_t lds, __half* dst,
                       int64_t ldd, cudaStream_t st);

// stage two (k_stage2.cu): band (fp32, LAPACK lower band storage) -> tridiagonal
// (d, e fp64) by Householder bulge chasing; eigenvalues of tridiag(d, e) by Sturm bisection
size_t stage2_ws_bytes(int64_t n, int b);
cudaError_t band_to_tridiag(int64_t n, int b, const float* AB, int64_t ldab, void* ws, double* d, double* e,
                            cudaStream_t st);
size_t tridiag_eig_ws_bytes(int64_t n);
cudaError_t tridiag_eigenvalues(int64_t n, const double* d, const double* e, void* ws, double* lam, cudaStream_t st);

// 16-bit operand format (fp16 / bf16) of each translation unit's conversions and kind::f16
// descriptors (common.cuh g_op16_bf16); set_op16_all (sbr_api.cu) calls them all in stream order.
cudaError_t set_op16_chain(int bf16, cudaStream_t st);
cudaError_t set_op16_gemm(int bf16, cudaStream_t st);
cudaError_t set_op16_misc(int bf16, cudaStream_t st);
cudaError_t set_op16_panel(int bf16, cudaStream_t st);
cudaError_t set_op16_chol(int bf16, cudaStream_t st);
cudaError_t set_op16_skinny(int bf16, cudaStream_t st);
cudaError_t set_op16_pass(int bf16, cudaStream_t st);
cudaError_t set_op16_api(int bf16, cudaStream_t st);
cudaError_t set_op16_all(int bf16, cudaStream_t st);

}  // namespace sbr
