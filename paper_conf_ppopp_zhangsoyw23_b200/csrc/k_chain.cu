// k_chain.cu -- the small steps of the per-panel chain (FP16 mode), fused so that each
// b-panel costs few dependent launches (the chain is sequential over all n/b panels).
//
//   kxb (LAZY,  a5):  P = W^T R = X(c,:)^T - (W^T X) Y_c^T            (k x b; Alg.1 l.8-10)
//                     -> fp16 P^T, the second B operand of the lazy skinny GEMM; plus the mirror
//                        of the b x b diagonal block of the fp32 master (upper <- lower, C14).
//   kxb (MERGE, a3):  W_{<t}^T X_t = H - (W^T X) G,  H = X^T W^0, G = Y^T W^0   (reading R2)
//                     -> WtX column block and its mirror (WtX is symmetric); plus G -> fp16 for
//                        the merge GEMM W_t = W^0 - W G.
//   postpass (a4 tail): X_t -> fp16 row-major (operand of later lazy updates) and the diagonal
//                     block W_t^T X_t of W^T X, one read of X_t and W_t.
// All three are fp32 SIMT: k x k x b is tiny and the operands (W^T X, b rows of X and Y) sit in L2.
// The K dimension is split over the 8 warps of a CTA so that every warp has its loads in flight
// at once (these kernels are latency-, not bandwidth-bound), reduced through shared memory.
#include "common.cuh"
#include "kernels.h"

namespace sbr {

constexpr int KXB_QT = 8;   // output rows (q) per CTA

template <int NG>  // NG = 32-column groups of b (1: b <= 32, 2: b <= 64)
__global__ void __launch_bounds__(256) kxb_kernel(KxbArgs a) {
  __shared__ float red[8][KXB_QT][64];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int k = a.k, b = a.b;
  const int q0 = blockIdx.x * KXB_QT;
  const int r0 = (int)((int64_t)warp * k / 8), r1 = (int)((int64_t)(warp + 1) * k / 8);
  float* __restrict__ WtX = a.WtX;
  const int64_t ldwx = a.ldwx;
  float acc[KXB_QT][NG];
#pragma unroll
  for (int i = 0; i < KXB_QT; ++i)
#pragma unroll
    for (int g = 0; g < NG; ++g) acc[i][g] = 0.f;
  const bool lazy = a.mode == 0;
#pragma unroll 4
  for (int r = r0; r < r1; ++r) {
    float bv[NG];
#pragma unroll
    for (int g = 0; g < NG; ++g) {
      const int p = lane + 32 * g;
      bv[g] = 0.f;
      if (p < b) bv[g] = lazy ? __ldg(a.Y + (a.c + p) + (int64_t)r * a.ldy) : __ldcg(a.G + (int64_t)r * b + p);
    }
    const float* col = WtX + (int64_t)r * ldwx + q0;
#pragma unroll
    for (int i = 0; i < KXB_QT; ++i) {
      const float av = (q0 + i < k) ? __ldcg(col + i) : 0.f;
#pragma unroll
      for (int g = 0; g < NG; ++g) acc[i][g] = fmaf(av, bv[g], acc[i][g]);
    }
  }
#pragma unroll
  for (int i = 0; i < KXB_QT; ++i)
#pragma unroll
    for (int g = 0; g < NG; ++g) red[warp][i][lane + 32 * g] = acc[i][g];
  __syncthreads();
  for (int e = threadIdx.x; e < KXB_QT * b; e += blockDim.x) {
    const int i = e / b, p = e % b;
    const int q = q0 + i;
    if (q >= k) continue;
    float s = 0.f;
#pragma unroll
    for (int w = 0; w < 8; ++w) s += red[w][i][p];
    if (lazy) {
      const float d = a.X[(a.c + p) + (int64_t)q * a.ldx] - s;
      a.Ph[(int64_t)p * a.ldph + q] = __float2half_rn(d);
    } else {
      const float d = __ldcg(a.H + (int64_t)q * b + p) - s;
      WtX[q + (int64_t)(k + p) * ldwx] = d;
      WtX[(k + p) + (int64_t)q * ldwx] = d;
    }
  }
  if (lazy) {
    if (blockIdx.x == 0) {   // upper <- lower on the b x b diagonal block of the panel's columns
      for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
        const int i = e % b, j = e / b;
        if (i < j) a.Adiag[i + (int64_t)j * a.lda] = a.Adiag[j + (int64_t)i * a.lda];
      }
    }
  } else {   // G -> fp16, column-major (k contiguous): B operand of the merge GEMM
    const int64_t tot = (int64_t)k * b;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < tot; e += (int64_t)gridDim.x * blockDim.x) {
      const int r = (int)(e / b), p = (int)(e % b);
      a.Gh[r + (int64_t)p * a.ldgh] = __float2half_rn(__ldcg(a.G + e));
    }
  }
}

cudaError_t launch_kxb(const KxbArgs& a, cudaStream_t st) {
  if (a.k <= 0 || a.b <= 0) return cudaSuccess;
  const int grid = (a.k + KXB_QT - 1) / KXB_QT;
  if (a.b <= 32)
    kxb_kernel<1><<<grid, 256, 0, st>>>(a);
  else
    kxb_kernel<2><<<grid, 256, 0, st>>>(a);
  return cudaGetLastError();
}

// ------------------------------------------------------------------ postpass
template <int BB>  // BB >= b, multiple of 8; rows per CTA sized for 48 KB of static smem
constexpr int pp_rows() { return BB <= 16 ? 256 : BB <= 32 ? 128 : 64; }

template <int BB>
__global__ void __launch_bounds__(256) postpass_kernel(int64_t M, int b, const float* __restrict__ X, int64_t ldx,
                                                       const float* __restrict__ W, int64_t ldw, __half* Xh,
                                                       int64_t ldxh, float* WtXtt, int64_t ldwtx) {
  constexpr int PP_ROWS = pp_rows<BB>();
  __shared__ float Xs[PP_ROWS][BB + 1];
  __shared__ float Ws[PP_ROWS][BB + 1];
  const int64_t rbeg = (int64_t)blockIdx.x * PP_ROWS;
  const int nr = (int)(M - rbeg < PP_ROWS ? M - rbeg : PP_ROWS);
  for (int e = threadIdx.x; e < PP_ROWS * b; e += blockDim.x) {
    const int r = e % PP_ROWS, c = e / PP_ROWS;
    float xv = 0.f, wv = 0.f;
    if (r < nr) {
      xv = __ldcg(X + (rbeg + r) + (int64_t)c * ldx);
      wv = W[(rbeg + r) + (int64_t)c * ldw];
    }
    Xs[r][c] = xv;
    Ws[r][c] = wv;
  }
  __syncthreads();
  // X_t rows -> fp16 row-major
  const bool vec = (b % 8 == 0) && (ldxh % 8 == 0) && ((reinterpret_cast<uintptr_t>(Xh) & 15) == 0);
  const int groups = (b + 7) / 8;
  for (int e = threadIdx.x; e < nr * groups; e += blockDim.x) {
    const int r = e / groups, g = e % groups;
    __half* dst = Xh + (rbeg + r) * ldxh + g * 8;
    if (vec) {
      __align__(16) __half hv[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) hv[u] = __float2half_rn(Xs[r][g * 8 + u]);
      *reinterpret_cast<uint4*>(dst) = *reinterpret_cast<const uint4*>(hv);
    } else {
      for (int u = 0; u < 8 && g * 8 + u < b; ++u) dst[u] = __float2half_rn(Xs[r][g * 8 + u]);
    }
  }
  // partial W_t^T X_t over this CTA's rows
  for (int o = threadIdx.x; o < b * b; o += blockDim.x) {
    const int i = o % b, j = o / b;
    float acc = 0.f;
#pragma unroll 8
    for (int r = 0; r < nr; ++r) acc = fmaf(Ws[r][i], Xs[r][j], acc);
    atomicAdd(WtXtt + i + (int64_t)j * ldwtx, acc);
  }
}

cudaError_t launch_postpass(int64_t M, int b, const float* X, int64_t ldx, const float* W, int64_t ldw, __half* Xh,
                            int64_t ldxh, float* WtXtt, int64_t ldwtx, cudaStream_t st) {
  if (M <= 0) return cudaSuccess;
  auto grid = [&](int rows) { return (unsigned)((M + rows - 1) / rows); };
  if (b <= 16)
    postpass_kernel<16><<<grid(pp_rows<16>()), 256, 0, st>>>(M, b, X, ldx, W, ldw, Xh, ldxh, WtXtt, ldwtx);
  else if (b <= 32)
    postpass_kernel<32><<<grid(pp_rows<32>()), 256, 0, st>>>(M, b, X, ldx, W, ldw, Xh, ldxh, WtXtt, ldwtx);
  else
    postpass_kernel<64><<<grid(pp_rows<64>()), 256, 0, st>>>(M, b, X, ldx, W, ldw, Xh, ldxh, WtXtt, ldwtx);
  return cudaGetLastError();
}

}  // namespace sbr
