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

/* One panel factorisation (TSQR + reconstruction, steps a1-a2) of the m x b panel P
 * (overwritten with the compact form); explicit Y and W = Y T (m x b, ld ldyw).  If
 * trace != NULL it receives 16 int64 globaltimer stamps (ns) of the kernel's phases. */
int sbr_test_panel(sbr_handle_t h, int64_t m, int b, float* P, int64_t ldp, float* Y, float* W, int64_t ldyw,
                   int64_t* trace);

#ifdef __cplusplus
}
#endif
#endif /* SBR_TESTING_H_ */
