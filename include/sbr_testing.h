/*
 * sbr_testing.h -- kernel-level test hooks of libsbr (not part of the product API).
 *
 * Each call runs ONE of the tensor-core kernels sbr_reduce uses, on device buffers,
 * with the same operand preparation as the driver (fp16 rounding, shadow layout), so
 * tests can compare it against fp64 products of the same rounded operands.  All
 * arrays are fp32, column-major, on the handle's device; calls synchronise.
 * Returns 0 or an sbr.h status code.
 */
#ifndef SBR_TESTING_H_
#define SBR_TESTING_H_

#include <stdint.h>

#include "sbr.h"

#ifdef __cplusplus
extern "C" {
#endif

/* X (M x b) = OA W with OA (M x M, lower referenced) symmetric -- step a4 on tcgen05
 * (OA and W rounded to fp16; fp32 accumulation). */
int sbr_test_pass_fp16(sbr_handle_t h, int64_t M, int b, const float* OA, int64_t ldoa, const float* W,
                       int64_t ldw, float* X, int64_t ldx);

/* C_low (M x M) -= Y Z^T + Z Y^T (Y, Z: M x K, rounded to fp16) -- step a6 on tcgen05.
 * Also writes the fp16 shadow of the result to S (M x M fp32 copy of the fp16 values,
 * strict lower, half diagonal) if S != NULL. */
int sbr_test_syr2k_fp16(sbr_handle_t h, int64_t M, int K, const float* Y, int64_t ldy, const float* Z,
                        int64_t ldz, float* C, int64_t ldc, float* S, int64_t lds);

/* Z (M x K) = X - 1/2 Y G with G (K x K) symmetric (Y, G rounded to fp16) -- Z formation
 * on tcgen05; Z is returned as fp32 (of the fp16 values). */
int sbr_test_zform_fp16(sbr_handle_t h, int64_t M, int K, const float* Y, int64_t ldy, const float* G, int64_t ldg,
                        const float* X, int64_t ldx, float* Z, int64_t ldz);

/* One panel factorisation (steps a1-a2: CholeskyQR + reconstruction with the in-kernel
 * Householder fallback for m > 512, the paper's TSQR for m <= 512 or SBR_PANEL=tsqr) of the m x b panel P
 * (overwritten with the compact form); explicit Y and W = Y T (m x b, ld ldyw).  If
 * trace != NULL it receives 16 int64 globaltimer stamps (ns) of the kernel's phases. */
int sbr_test_panel(sbr_handle_t h, int64_t m, int b, float* P, int64_t ldp, float* Y, float* W, int64_t ldyw,
                   int64_t* trace);

/* Diagnostic: per-panel phase stamps inside sbr_reduce (the CholeskyQR panel kernel, or the
 * fused chain kernel of the FP16 mode).  cap > 0 arms recording for the next cap panels
 * (device buffer owned by the handle, 32 int64 globaltimer slots in ns per panel, CTA 0's
 * view, stamp 0 taken before the PDL wait); host != NULL copies the stamps recorded so far
 * (count * 32 int64) after synchronising the handle's stream and stores the panel count in
 * *count (NULL count with non-NULL host: -4). */
int sbr_test_panel_trace(sbr_handle_t h, int cap, int64_t* host, int* count);

/* Same as sbr_test_pass_fp16 but only the share of `rank` of `nranks` (the tiles
 * sbr_test_pass_partition assigns): summing the X of all ranks gives the full pass. */
int sbr_test_pass_fp16_part(sbr_handle_t h, int64_t M, int b, int rank, int nranks, const float* OA, int64_t ldoa,
                            const float* W, int64_t ldw, float* X, int64_t ldx);

/* Host only (no device work): the share of the per-panel pass (a4) that `rank` of `nranks`
 * streams under sbr_reduce_dist, for an M x M block-local OA and bandwidth b: tiles
 * [*t0, *t1) of *total 128 x 128 lower tiles, in the order of sbr_test_pass_tiles.
 * Returns 0, -1 (M < 1), -2 (b), -3 (rank / nranks), -5 (NULL output). */
int sbr_test_pass_partition(int64_t M, int b, int rank, int nranks, int64_t* t0, int64_t* t1, int64_t* total);

/* Host only: tile coordinates of tiles [t0, t1) of the pass order -- tile k is the lower
 * tile (row block I, column block J), I >= J, of OA, IJ[2k] = I, IJ[2k+1] = J (caller
 * allocates 2*(t1-t0) ints).  Each rank's contribution is X_I += L_IJ W_J and, for I > J,
 * X_J += L_IJ^T W_I (a diagonal tile holds the strict lower part plus half the diagonal). */
int sbr_test_pass_tiles(int64_t M, int b, int64_t t0, int64_t t1, int* IJ);

/* 3xTF32 mode (reading C11 / R4): X (M x b) = OA W on tcgen05 kind::tf32 from the fp32 OA
 * (ldoa % 4 == 0; lower referenced; the upper triangle is ignored).  If S != NULL, the
 * 128-column tiles covering OA columns [0, sw) are read from S (M x >= min(128 ceil(sw/128), M),
 * ld lds) instead -- the frozen-strip path of sbr_reduce.  W is split rna hi/lo. */
int sbr_test_pass_tf32(sbr_handle_t h, int64_t M, int b, const float* OA, int64_t ldoa, const float* S,
                       int64_t lds, int64_t sw, const float* W, int64_t ldw, float* X, int64_t ldx);

/* 3xTF32: C_low (M x M) -= Y Z^T + Z Y^T (hi/lo split Y, Z; 6 tf32 products per pair). */
int sbr_test_syr2k_tf32(sbr_handle_t h, int64_t M, int K, const float* Y, int64_t ldy, const float* Z,
                        int64_t ldz, float* C, int64_t ldc);

/* 3xTF32: Z (M x K) = X - 1/2 Y G (G K x K symmetric); Z returned as hi + lo in fp32. */
int sbr_test_zform_tf32(sbr_handle_t h, int64_t M, int K, const float* Y, int64_t ldy, const float* G, int64_t ldg,
                        const float* X, int64_t ldx, float* Z, int64_t ldz);

/* Host only: the pass tiles rank `rank` of `nranks` streams under sbr_reduce_dist for the block
 * at column c0 (n, b, nb as the reduction): the 128-aligned tile grid with origin c0 (global
 * rows / columns c0 + 128 I ..; OA rows start b rows into tile 0), column-block ownership
 * (J % nranks), lower tiles I >= J.  Writes up to cap pairs IJ[2k] = I, IJ[2k+1] = J in walk
 * order and returns the count (-1: invalid arguments / unsupported nb). */
int64_t sbr_test_pass_owned_tiles(int64_t n, int b, int nb, int64_t c0, int rank, int nranks, int* IJ, int64_t cap);

/* Number of CholeskyQR panels that declined (rank deficient / not orthonormal after three
 * rounds, so the kernel's Householder QR fallback factored them) since the handle's workspace was allocated or
 * the last call with reset != 0.  Synchronises.  Returns 0, -1 (h), -3 (count NULL). */
int sbr_test_panel_declines(sbr_handle_t h, int reset, int64_t* count);

/* Experiment knobs (timing experiments only; process-wide, 0 = production behaviour):
 *   knob 0 (pass experiment bits): 1 = skip the pass's L W MMAs, 2 = skip its L^T W MMAs,
 *     8 = skip its X reductions (row and column accumulators), 16 = skip the column ones only
 *   (results are WRONG: for timing the stream alone), 4 = normal L2 policy for the OA stream.
 * Returns 0, or -1 for an unknown knob. */
int sbr_test_set_knob(int knob, int value);

#ifdef __cplusplus
}
#endif
#endif /* SBR_TESTING_H_ */
