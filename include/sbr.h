/*
 * sbr.h -- C ABI of libsbr: stage-one successive band reduction (SBR) of a dense
 * symmetric matrix to band form with the WY formulation, on NVIDIA B200 (sm_100a).
 *
 * Method: Zhang, Shah, Ootomo, Yokota, Wu, "Fast Symmetric Eigenvalue
 * Decomposition via WY Representation on Tensor Core", PPoPP'23.  "P:n" below is
 * line n of the paper text (/root/reference/PAPER.md at authoring time).
 *
 *   A = Q B Q^T,  Q = H_1 H_2 ... H_{n-b},  B symmetric with bandwidth b
 *   (Sec. 3.1; reading C2 of DESIGN.md for the product order).
 *
 * The reduction is Algorithm 1: b-wide panels are factored by a
 * tall-skinny QR (TSQR) whose explicit Q is turned back into
 * Householder vectors (Alg. 3 + sign matrix S); inside an nb-wide
 * block every panel is updated lazily from the block's original trailing matrix
 * OA and the accumulated (W, Y); the trailing matrix is
 * updated once per block, A <- (I - W Y^T)^T A (I - W Y^T) (Eq. 1),
 * evaluated as the lower-triangular rank-2nb update A - Y Z^T - Z Y^T with
 * Z = X - 1/2 Y (W^T X), X = OA W (Eq. 2-3; reading C5).
 *
 * Conventions (all arrays column-major, 64-bit leading dimensions, fp32):
 *   - Householder convention: LAPACK dlarfg (reading C1).  Entry for entry the
 *     result equals LAPACK dsytrd_sy2sb(UPLO='L') up to rounding, except that a
 *     panel whose column needs no reduction may yield H = I - 2 e e^T instead of
 *     H = I (B -> D B D with D = diag(+-1)).
 *   - Only the lower triangle of A is referenced (reading C14).
 *
 * Threading / streams: a handle is bound to one device and one CUDA stream; all
 * calls on it are stream-ordered and return after enqueueing device work (no
 * host synchronisation) unless stated.  A handle must not be used by two host
 * threads at once.  Device pointers are plain CUDA device addresses.
 *
 * Errors: 0 = OK; -i = argument i invalid (LAPACK style); positive values:
 */
#ifndef SBR_H_
#define SBR_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SBR_OK 0
#define SBR_ERR_NONFINITE 1  /* input holds Inf/NaN, or the band overflowed fp32   */
#define SBR_ERR_CUDA 2       /* CUDA runtime/driver error; see sbr_status_string    */
#define SBR_ERR_NCCL 3       /* reserved for the multi-GPU path                     */
#define SBR_ERR_NOMEM 4      /* device workspace allocation failed                  */
#define SBR_ERR_UNSUPPORTED 5 /* valid arguments this build does not support        */

typedef struct sbr_ctx* sbr_handle_t;

/* Arithmetic of the GEMM-shaped steps (Sec. 5.3).  The panel QR,
 * reconstruction and all accumulations are fp32 in every mode.
 *   SBR_FP16_FP32ACC : operands rounded to fp16 (RN), fp32 accumulate on tcgen05
 *                      (kind::f16) -- the paper's Tensor Core mode.
 *   SBR_3XTF32       : FP32-accurate "EC-TCGEMM" mode (reading C11):
 *                      a = hi + lo with hi = rna_tf32(a), lo = rna_tf32(a - hi);
 *                      C = hi*hi' + (hi*lo' + lo*hi').
 *   SBR_BF16_FP32ACC : the FP16 path with bfloat16 operands (RN) instead of fp16 -- an ablation
 *                      (SURVEY 8(f) f4): same kernels and speed, 8 bits less mantissa (2^-9 vs
 *                      2^-12 unit roundoff), so its errors are ~8x the FP16 mode's and exceed
 *                      the 5e-3 FP16 gates; its wider range needs no scaling (a0 still applies).
 *                      The operand format is a per-device setting written in stream order at the
 *                      start of each reduction: do not run FP16 and BF16 reductions concurrently
 *                      on one device.  Not supported by the opt-in fused chain (SBR_FUSED=1). */
typedef enum { SBR_FP16_FP32ACC = 0, SBR_3XTF32 = 1, SBR_BF16_FP32ACC = 2 } sbr_precision_t;

/* Create a handle on CUDA device `device`, bound to `stream` (a cudaStream_t;
 * NULL = the legacy default stream).  Allocates nothing large.
 * Returns SBR_OK, -1 (h NULL), -2 (bad device) or SBR_ERR_CUDA. */
int sbr_create(sbr_handle_t* h, int device, void* stream);

/* Rebind the handle to another stream on the same device. */
int sbr_set_stream(sbr_handle_t h, void* stream);

/* Free the handle and its workspace (synchronises the handle's stream). */
int sbr_destroy(sbr_handle_t h);

/* Device workspace sbr_reduce needs for (n, b, nb, mode), in bytes.  The handle
 * allocates and owns it (grown on demand, kept between calls). */
int sbr_workspace_query(sbr_handle_t h, int64_t n, int b, int nb, int mode, size_t* bytes);

/* Reduce the symmetric n x n matrix A (device, fp32, lower triangle referenced)
 * to bandwidth b with outer block nb (Alg. 1).
 *   mode  : sbr_precision_t.
 *   n     : order, n >= 1.                                   (arg 3)
 *   b     : bandwidth, 1 <= b <= 64.                          (arg 4)
 *   nb    : outer block, nb >= b, nb % b == 0, nb <= 4096.    (arg 5)
 *   A     : in: symmetric matrix (lower).  out: LAPACK dsytrd_sy2sb layout --
 *           the band (diagonal blocks and the upper-triangular R factors) in the
 *           lower band, and the Householder vector of reflector column c
 *           (0 <= c < n-b; unit at row c+b, implicit) in A[c+b+1:n, c].
 *           Entries above the diagonal are left unspecified.           (arg 6)
 *   lda   : >= max(1, n).                                     (arg 7)
 *   AB    : out: band in LAPACK lower band storage, AB[d + j*ldab] = B[j+d, j],
 *           0 <= d <= b; may alias nothing else.             (arg 8)
 *   ldab  : >= b + 1.                                         (arg 9)
 *   W     : out (may be NULL): per-block W factors: for block J
 *           (columns c0 = J*nb .. c0+k_J-1), Q_J = I - W_J Y_J^T acting on
 *           rows/cols c0+b .. n-1, W_J stored in W[c0+b : n, c0 : c0+k_J];
 *           Q = Q_0 Q_1 ... .  Other entries are not referenced.  n x (n-b).
 *           If NULL, W lives in handle workspace (per block) and is dropped. (arg 10)
 *   ldw   : >= n if W != NULL.                                (arg 11)
 * Trivial case n <= b+1: AB = band of A, W untouched, no reflectors.
 * FP16 mode range handling (a0, reading C10): the reduction runs on 2^k A with the
 * exact power of two 2^k chosen on the device so that ||A||_F 2^k lies in [2^12, 2^13) -- every
 * fp16 operand then stays below 2^15 and typical entries far from fp16's subnormals.  The
 * fp32 master (A's lower triangle) is scaled in place; on exit the band (in A and in AB) is
 * unscaled by 2^-k, Y and W are scale free.  The 3xTF32 mode takes the same scale (its fp32
 * panel norms and products would under/overflow near the ends of the fp32 range).
 * Returns (argument checks, enqueue failures) 0, -i, SBR_ERR_CUDA, SBR_ERR_NOMEM, or an error
 * LATCHED by an earlier call on this handle.  The call never synchronises the host: errors
 * detected on the device -- SBR_ERR_NONFINITE (Inf/NaN in the referenced input, or a
 * non-finite band entry, i.e. fp16 range exceeded after scaling) -- are latched and returned
 * by sbr_sync or by the next call on the handle; the outputs of that reduction are then
 * invalid.  A panel that CholeskyQR declines (numerically rank deficient) is factored by
 * Householder QR inside the same kernel, at any height: rank deficiency is not an error. */
int sbr_reduce(sbr_handle_t h, int mode, int64_t n, int b, int nb,
               float* A, int64_t lda, float* AB, int64_t ldab, float* W, int64_t ldw);

/* End-to-end variant with HOST buffers (pinned or pageable): copies A to the
 * device, reduces, copies the band AB back and, as selected by `outputs`
 * (bitmask of SBR_OUT_*), A (holding Y) and W; all on the handle's stream,
 * returning after the results are on the host.  The band alone is what the
 * paper's eigenvalue pipeline moves to the host.  Same arguments and
 * errors as sbr_reduce (outputs is argument 12).  Device copies are owned by the
 * handle (grown on demand). */
#define SBR_OUT_BAND 1
#define SBR_OUT_Y 2
#define SBR_OUT_W 4
int sbr_reduce_host(sbr_handle_t h, int mode, int64_t n, int b, int nb,
                    float* A, int64_t lda, float* AB, int64_t ldab, float* W, int64_t ldw,
                    int outputs);

/* Explicit Q of a reduction ("Q = I - W Y^T", P:115 A = Q B Q^T):
 *   Q = prod_J (I - W_J Y_J^T), block J (c0 = J nb, k_J = min(nb, n-b-c0) reflector columns)
 *   acting on rows/cols c0+b .. n-1, with Y_J and W_J read from sbr_reduce's outputs (same
 *   n, b, nb): Y_J column jj = unit at row c0+jj+b, tail A[c0+jj+b+1 : n, c0+jj], zero above;
 *   W_J = W[c0+b : n, c0 : c0+k_J].
 *   A   : device fp32, column-major, lda >= n (read only).               (args 5, 6)
 *   W   : device fp32, column-major, ldw >= n (read only).               (args 7, 8)
 *   Q   : device fp32, column-major n x n, ldq >= n; overwritten.        (args 9, 10)
 * Backward accumulation, last block first: Q[r0:, r0:] -= W_J (Y_J^T Q[r0:, r0:]), both
 * products on tcgen05 in 3xTF32 (FP32-accurate) whatever the reduction's mode: Q feeds the
 * eigenvector back-transformation, where FP32 accuracy is what the paper targets.
 * The split operands (about 8 (n-b)^2 + 24 n nb bytes) live in handle-owned device memory,
 * grown on demand and freed by sbr_destroy; the call is stream-ordered and returns after enqueue.
 * Returns 0, -1 (h), -2 (n < 1), -3 (b not in 1..64), -4 (nb), -5 (A NULL), -6 (lda),
 * -7 (W NULL), -8 (ldw), -9 (Q NULL), -10 (ldq), SBR_ERR_NOMEM, SBR_ERR_CUDA. */
int sbr_form_q(sbr_handle_t h, int64_t n, int b, int nb, const float* A, int64_t lda, const float* W, int64_t ldw,
               float* Q, int64_t ldq);

/* Back-transformation (Sec. 4.4), both on tcgen05 3xTF32 like sbr_form_q.
 * sbr_form_w: Alg. 2 -- the per-block W_J of sbr_reduce merged recursively (left half,
 *   right half, then W_R <- W_R - W_L (Y_L^T W_R)) into ONE n x (n-b) W with Q = I - W Y^T, Y the
 *   unit lower staircase of sbr_reduce's output (column c: unit at row c+b, tail in A below).
 *   A (Y), W: sbr_reduce's outputs (same n, b, nb), read only.  Wo: device fp32, n x (n-b),
 *   column-major, ldwo >= n, overwritten (zeros above each column's first touched row).
 *   Returns 0, -1 (h), -2 (n), -3 (b), -4 (nb), -5 (A), -6 (lda), -7 (W), -8 (ldw), -9 (Wo),
 *   -10 (ldwo), SBR_ERR_NOMEM, SBR_ERR_CUDA.
 * sbr_apply_q: X <- Q X for the n x kx block X (device fp32, column-major, ldx >= n): the eigenvector
 *   back-transformation of the band's eigenvectors.  Applies the per-block factors last
 *   block first, X[r0:] -= W_J (Y_J^T X[r0:]).  Returns as sbr_form_w with -9 (X), -10 (ldx),
 *   -11 (kx < 0).
 * Both are stream-ordered; their split operands live in handle-owned device memory. */
int sbr_form_w(sbr_handle_t h, int64_t n, int b, int nb, const float* A, int64_t lda, const float* W, int64_t ldw,
               float* Wo, int64_t ldwo);
int sbr_apply_q(sbr_handle_t h, int64_t n, int b, int nb, const float* A, int64_t lda, const float* W, int64_t ldw,
                float* X, int64_t ldx, int64_t kx);

/* ---- Stage two: band -> tridiagonal -> eigenvalues on the GPU ----
 * The paper's two-stage EVD (Fig. 1) runs stage two on the CPU (MAGMA, after a
 * device->host copy of the band) and names a GPU stage two as future work.
 * These calls run it on the device, in fp64, stream-ordered (return after enqueue):
 *
 * sbr_band_to_tridiag: T = Q2^T B Q2 tridiagonal, by Householder bulge chasing (SBR with target
 *   bandwidth 1, Fig. 2; sweep s annihilates column s and chases the bulge in b-row
 *   steps; sweeps run pipelined, one warp each).  Q2 is not formed.
 *   AB : device fp32 band in LAPACK lower band storage, AB[d + j ldab] = B[j+d, j], 0 <= d <= b
 *        (sbr_reduce's AB output), ldab >= b+1; read only.  Entries with j+d >= n are ignored.
 *   d  : device fp64, n entries: diag(T).  e: device fp64, n-1 entries: subdiag(T) (signs are
 *        not normalised: T is unique up to D T D, D = diag(+-1)).
 *   Returns 0, -1 (h), -2 (n < 0), -3 (b not in 1..64), -4 (AB), -5 (ldab), -6 (d), -7 (e),
 *   SBR_ERR_NOMEM, SBR_ERR_CUDA.
 * sbr_tridiag_eigenvalues: all eigenvalues of tridiag(d, e), ascending, into lam (device fp64,
 *   n), by bisection on Sturm counts: eigenvalue k is the smallest x with more than k
 *   negative pivots in the LDL^T factorisation of T - x I, each interval halved from the
 *   Gershgorin bounds until its width is <= 2 eps max(|lo|, |hi|) (pivots below
 *   DBL_MIN max(1, max(|d|,|e|)^2) in magnitude replaced by -that).  One thread per eigenvalue.
 *   Returns 0, -1 (h), -2 (n), -3 (d), -4 (e), -5 (lam), SBR_ERR_NOMEM, SBR_ERR_CUDA.
 * sbr_band_eigenvalues: both steps (d, e in handle-owned memory).  Arguments as
 *   sbr_band_to_tridiag, lam = argument 6.
 * sbr_eigenvalues: the whole two-stage pipeline on one GPU -- sbr_reduce (W not kept; A is
 *   overwritten as by sbr_reduce) then sbr_band_eigenvalues into lam (device fp64, n).  Argument
 *   errors 1-7 as sbr_reduce, -8 (lam NULL); latched reduction errors as sbr_reduce.
 * Workspace: about (16 b + 28) n bytes (plus the band for sbr_eigenvalues), handle-owned, grown
 * on demand and freed by sbr_destroy. */
int sbr_band_to_tridiag(sbr_handle_t h, int64_t n, int b, const float* AB, int64_t ldab, double* d, double* e);
int sbr_tridiag_eigenvalues(sbr_handle_t h, int64_t n, const double* d, const double* e, double* lam);
int sbr_band_eigenvalues(sbr_handle_t h, int64_t n, int b, const float* AB, int64_t ldab, double* lam);
int sbr_eigenvalues(sbr_handle_t h, int mode, int64_t n, int b, int nb, float* A, int64_t lda, double* lam);

/* ---- Multi-GPU (north star: 1D block-cyclic columns) ----
 *
 * Data distribution: the columns of A are split into nb-wide blocks J (global columns
 * [J nb, (J+1) nb)); rank r holds the blocks with J % nranks == r, in order, as an n x ncols_loc
 * column-major array A_local (local column of global column g: (J / nranks) nb + (g - J nb));
 * ncols_loc = sbr_local_cols(n, nb, r, nranks).  The fp16 shadow of the trailing matrix is
 * sharded the same way, so device memory per rank is about 6 n^2 / nranks bytes plus the
 * replicated block buffers (Y, X, Z: n x nb each).
 *
 * sbr_get_unique_id: rank 0 creates the 128-byte NCCL unique id (host call, no device work)
 *   and distributes it to the other ranks out of band (e.g. torch.distributed).  Returns 0
 *   or SBR_ERR_NCCL (libnccl.so.2 not loadable; it is dlopen'ed, the single-GPU path never
 *   needs it).
 * sbr_create_dist: like sbr_create, plus an NCCL communicator of `nranks` ranks built from
 *   `unique_id` (collective: every rank must call it; one process per GPU).  Returns 0, -1 (h
 *   NULL), -2 (device), -4 (unique_id NULL), -5 (rank), -6 (nranks), SBR_ERR_CUDA, SBR_ERR_NCCL.
 * sbr_create_dist_local: the same reduction with `nranks` handles in ONE process (one host
 *   thread per rank, any devices, the same one included), exchanging through device memory
 *   with host barriers instead of NCCL: every rank passes the same `group` key.  It runs the
 *   same kernels and call sequence as NCCL ranks (used to test the sharded reduction on one
 *   GPU).  1 <= nranks <= 16.  Same returns as sbr_create_dist.
 * sbr_local_cols: ncols_loc of `rank` (host only); -1 on invalid arguments.
 * sbr_reduce_dist: the reduction of ONE matrix across the ranks (strong scaling), collective:
 *   every rank calls it with the same n, b, nb, mode and its A_local (lda >= n).  The owner of
 *   block J (J % nranks) factors that block's panels (its columns only: the lazy panel
 *   updates, TSQR/CholeskyQR + reconstruction and W merges) and broadcasts W_t
 *   (fp16) per panel; every rank streams the pass tiles of ITS column blocks and the partial
 *   X_t = OA W_t are summed by an all-reduce (M x b fp32); per block the owner broadcasts Y
 *   (fp16) and W^T X and every rank applies the trailing SYR2K to its own columns (Eq. 1-3).
 *   On return: A_local holds the owned columns in sbr_reduce's output layout (band + Y below
 *   it), W_local (may be NULL, ldw >= n) the owned blocks' W columns (same local columns), and
 *   AB (rank 0; may be NULL elsewhere) the whole band, assembled over the ranks.  With
 *   nranks > 1: FP16 mode with b % 8 == 0 and nb a multiple of 128 x the pass's tile columns
 *   per group (1024 for b <= 32, 512 for b = 64), or 3xTF32 mode with b % 4 == 0, nb a
 *   multiple of 256 and A_local 16-byte aligned with lda % 4 == 0 (3xTF32 broadcasts W_t and Y
 *   in fp32 and every rank splits them); else SBR_ERR_UNSUPPORTED.  Same argument
 *   errors as sbr_reduce; SBR_ERR_NCCL on a communication error (a failing rank can leave
 *   the others blocked in a collective: treat it as fatal for the group).
 * With nranks == 1, sbr_reduce_dist is sbr_reduce. */
int sbr_get_unique_id(void* unique_id_128_bytes);
int sbr_create_dist(sbr_handle_t* h, int device, void* stream, const void* unique_id, int rank, int nranks);
int sbr_create_dist_local(sbr_handle_t* h, int device, void* stream, int group, int rank, int nranks);
int64_t sbr_local_cols(int64_t n, int nb, int rank, int nranks);
int sbr_reduce_dist(sbr_handle_t h, int mode, int64_t n, int b, int nb,
                    float* A_local, int64_t lda, float* AB, int64_t ldab, float* W_local, int64_t ldw);
int sbr_rank(sbr_handle_t h);     /* 0 for sbr_create handles; -1 if h is NULL */
int sbr_nranks(sbr_handle_t h);   /* 1 for sbr_create handles; -1 if h is NULL */

/* Wait for all work enqueued on the handle's stream; returns the first error latched by a
 * finished reduction (SBR_ERR_NONFINITE / SBR_ERR_UNSUPPORTED, see sbr_reduce) or 0. */
int sbr_sync(sbr_handle_t h);

/* Human-readable text for a status code (static storage; includes the last
 * CUDA error seen by any handle when status == SBR_ERR_CUDA). */
const char* sbr_status_string(int status);

/* Seeded input generator, bit-identical to workloads.random_symmetric (host):
 * A[i + j*lda] = U[-1,1) from splitmix64(seed ^ (max(i,j) << 32 | min(i,j))),
 * top 24 bits u -> (u - 2^23) * 2^-23.  Full (both triangles) n x n.  Not part
 * of the method; used to create large inputs without a host copy. */
int sbr_generate_symmetric(sbr_handle_t h, uint64_t seed, int64_t n, float* A, int64_t lda);

/* Per-kernel timing for roofline reporting.  When enabled, sbr_reduce records a
 * CUDA event pair (on the handle's stream) around every launch of each kernel
 * class; sbr_kernel_stats returns, for class `kid` (see SBR_K_*), the number of
 * launches, their summed device time (ms, elapsed between each pair) and the
 * summed algorithmic bytes and flops since the last
 * reset.  sbr_kernel_stats synchronises the stream. */
#define SBR_K_PANEL 0   /* TSQR + reconstruction (a1, a2)          */
#define SBR_K_LAZY 1    /* lazy next-panel update (a5)             */
#define SBR_K_WMERGE 2  /* W merge + W^T X (a3)                    */
#define SBR_K_PASS 3    /* X_t = OA W_t (a4)                       */
#define SBR_K_SYR2K 4   /* trailing update (a6, with Z formation)  */
#define SBR_K_OTHER 5   /* setup, band extraction                  */
#define SBR_K_STAGE2 6  /* stage two: bulge chase, bisection (f2)  */
#define SBR_K_COUNT 7
int sbr_set_kernel_timing(sbr_handle_t h, int enable);
int sbr_reset_kernel_stats(sbr_handle_t h);
int sbr_kernel_stats(sbr_handle_t h, int kid, int64_t* launches, double* ms,
                     double* bytes, double* flops);

/* Number of kernels libsbr launched since the handle was created (a counter
 * incremented on every launch, including those replayed from graphs). */
int64_t sbr_launch_count(sbr_handle_t h);

/* Build identification, e.g. "libsbr 0.1 sm_100a". */
const char* sbr_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SBR_H_ */
