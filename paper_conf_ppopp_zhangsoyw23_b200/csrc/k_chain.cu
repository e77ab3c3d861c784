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
// All three are fp32 SIMT: k x k x b is tiny and the operands (W^T X, b rows of X and Y) sit in
// L2, so these kernels are latency-bound.  Design for latency:
//   * every CTA issues all of its global loads before the first use (one round trip);
//   * the reduction dimension is split over the 8 CTAs of a thread-block cluster and the
//     partial results are summed through distributed shared memory -- no global atomics on
//     the hot addresses, no pre-zeroed outputs, no second launch.
#include <cooperative_groups.h>

#include "common.cuh"
#include "kernels.h"

namespace cg = cooperative_groups;

namespace sbr {

constexpr int KXB_QT = 32;   // output rows (q) per cluster
constexpr int KXB_CL = 8;    // CTAs per cluster (split of the reduction dimension r)
template <int NG>            // r-chunk staged in shared memory (48 KB static)
constexpr int kxb_rc() { return NG == 1 ? 128 : 96; }

template <int NG>  // NG = 32-column groups of b (1: b <= 32, 2: b <= 64)
__global__ void __cluster_dims__(1, KXB_CL, 1) __launch_bounds__(256) kxb_kernel(KxbArgs a) {
  constexpr int KXB_RC = kxb_rc<NG>();
  __shared__ __align__(16) float As[KXB_RC][KXB_QT];   // As[r][q] = WtX[q0+q, r]; reused for partials
  __shared__ float Bs[KXB_RC][32 * NG + 1];            // Bs[r][p] = B(r, p)
  cg::cluster_group cluster = cg::this_cluster();
  pdl_trigger();
  pdl_wait();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int k = a.k, b = a.b;
  const bool lazy = a.mode == 0;
  const int q0 = blockIdx.x * KXB_QT;
  const int rank = (int)cluster.block_rank();
  const int rper = (k + KXB_CL - 1) / KXB_CL;
  const int rb = rank * rper, re = min(k, rb + rper);
  float* __restrict__ WtX = a.WtX;
  const int64_t ldwx = a.ldwx;
  float acc[4][NG];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int g = 0; g < NG; ++g) acc[i][g] = 0.f;
  for (int r0 = rb; r0 < re; r0 += KXB_RC) {
    const int nr = min(KXB_RC, re - r0);
    // stage: all loads issued before any use
    for (int e = threadIdx.x; e < KXB_RC * KXB_QT; e += blockDim.x) {
      const int q = e % KXB_QT, r = e / KXB_QT;
      As[r][q] = (r < nr && q0 + q < k) ? __ldcg(WtX + (q0 + q) + (int64_t)(r0 + r) * ldwx) : 0.f;
    }
    if (lazy) {
      for (int e = threadIdx.x; e < KXB_RC * 32 * NG; e += blockDim.x) {
        const int p = e % (32 * NG), r = e / (32 * NG);
        Bs[r][p] = (r < nr && p < b) ? __ldcg(a.Y + (a.c + p) + (int64_t)(r0 + r) * a.ldy) : 0.f;
      }
    } else {
      for (int e = threadIdx.x; e < KXB_RC * 32 * NG; e += blockDim.x) {
        const int r = e % KXB_RC, p = e / KXB_RC;
        Bs[r][p] = (r < nr && p < b) ? __ldcg(a.G + (r0 + r) + (int64_t)p * a.ldg) : 0.f;
      }
    }
    __syncthreads();
#pragma unroll 4
    for (int r = 0; r < nr; ++r) {
      const float4 av = *reinterpret_cast<const float4*>(&As[r][warp * 4]);
      const float aa[4] = {av.x, av.y, av.z, av.w};
#pragma unroll
      for (int g = 0; g < NG; ++g) {
        const float bv = Bs[r][lane + 32 * g];
#pragma unroll
        for (int i = 0; i < 4; ++i) acc[i][g] = fmaf(aa[i], bv, acc[i][g]);
      }
    }
    __syncthreads();
  }
  // partials -> shared (As reused as Ps[q][p], p < 32*NG), then the cluster reduction:
  // CTA `rank` finalises rows q in [rank*4, rank*4 + 4) of the cluster's 32.
  static_assert(KXB_RC * KXB_QT >= KXB_QT * 64, "partials fit in As");
  float* Ps = &As[0][0];
  constexpr int LDP = 32 * NG;
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int g = 0; g < NG; ++g) Ps[(warp * 4 + i) * LDP + lane + 32 * g] = acc[i][g];
  cluster.sync();
  for (int e = threadIdx.x; e < 4 * b; e += blockDim.x) {
    const int qi = rank * 4 + e / b, p = e % b;
    const int q = q0 + qi;
    float s = 0.f;
#pragma unroll
    for (int j = 0; j < KXB_CL; ++j) s += cluster.map_shared_rank(Ps, j)[qi * LDP + p];
    if (q < k) {
      if (lazy) {
        const float d = __ldcg(a.X + (a.c + p) + (int64_t)q * a.ldx) - s;
        a.Ph[(int64_t)p * a.ldph + q] = __float2half_rn(d);
      } else {
        const float d = __ldcg(a.H + q + (int64_t)p * a.ldg) - s;
        WtX[q + (int64_t)(k + p) * ldwx] = d;
        WtX[(k + p) + (int64_t)q * ldwx] = d;
      }
    }
  }
  if (lazy) {
    if (blockIdx.x == 0 && rank == 0) {   // upper <- lower on the b x b diagonal block of the panel's columns
      for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
        const int i = e % b, j = e / b;
        if (i < j) a.Adiag[i + (int64_t)j * a.lda] = a.Adiag[j + (int64_t)i * a.lda];
      }
    }
  } else {   // G -> fp16, column-major (k contiguous): B operand of the merge GEMM
    const int64_t nth = (int64_t)gridDim.x * gridDim.y * blockDim.x;
    const int64_t tid = ((int64_t)blockIdx.y * gridDim.x + blockIdx.x) * blockDim.x + threadIdx.x;
    for (int64_t e = tid; e < (int64_t)k * b; e += nth) {
      const int r = (int)(e % k), p = (int)(e / k);
      a.Gh[r + (int64_t)p * a.ldgh] = __float2half_rn(__ldcg(a.G + r + (int64_t)p * a.ldg));
    }
  }
  cluster.sync();   // keep this CTA's partials alive until every reader is done
}

cudaError_t launch_kxb(const KxbArgs& a, cudaStream_t st) {
  if (a.k <= 0 || a.b <= 0) return cudaSuccess;
  const dim3 grid((a.k + KXB_QT - 1) / KXB_QT, KXB_CL);
  if (a.b <= 32)
    return launch_pdl(kxb_kernel<1>, grid, dim3(256), 0, st, a);
  return launch_pdl(kxb_kernel<2>, grid, dim3(256), 0, st, a);
}

// ------------------------------------------------------------------ postpass
constexpr int PP_CL = 8;

template <int BB>  // BB >= b, multiple of 16; rows per CTA sized for 48 KB of static smem
constexpr int pp_rows() { return BB <= 16 ? 256 : BB <= 32 ? 128 : 64; }

template <int BB>
__global__ void __cluster_dims__(PP_CL, 1, 1) __launch_bounds__(256)
    postpass_kernel(int64_t M, int b, const float* __restrict__ X, int64_t ldx, const float* __restrict__ W,
                    int64_t ldw, __half* Xh, int64_t ldxh, float* WtXtt, int64_t ldwtx) {
  constexpr int PP_ROWS = pp_rows<BB>();
  constexpr int BI = BB / 16;   // register block BI x BI per thread (16 x 16 thread grid)
  __shared__ float Xs[PP_ROWS][BB + 1];
  __shared__ float Ws[PP_ROWS][BB + 1];
  static_assert(PP_ROWS * (BB + 1) >= BB * BB, "partial fits in Xs");
  cg::cluster_group cluster = cg::this_cluster();
  pdl_trigger();
  pdl_wait();
  const int64_t rbeg = (int64_t)blockIdx.x * PP_ROWS;
  const int nr = (int)(M - rbeg < PP_ROWS ? (M - rbeg > 0 ? M - rbeg : 0) : PP_ROWS);
  for (int e = threadIdx.x; e < PP_ROWS * BB; e += blockDim.x) {
    const int r = e % PP_ROWS, c = e / PP_ROWS;
    float xv = 0.f, wv = 0.f;
    if (r < nr && c < b) {
      xv = __ldcg(X + (rbeg + r) + (int64_t)c * ldx);
      wv = __ldcg(W + (rbeg + r) + (int64_t)c * ldw);
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
  // partial W_t^T X_t over this CTA's rows: thread (ti, tj) owns rows i = ti*BI+u, cols j = tj*BI+v
  const int ti = threadIdx.x % 16, tj = threadIdx.x / 16;
  float acc[BI][BI];
#pragma unroll
  for (int u = 0; u < BI; ++u)
#pragma unroll
    for (int v = 0; v < BI; ++v) acc[u][v] = 0.f;
#pragma unroll 4
  for (int r = 0; r < nr; ++r) {
    float wv[BI], xv[BI];
#pragma unroll
    for (int u = 0; u < BI; ++u) {
      wv[u] = Ws[r][ti * BI + u];
      xv[u] = Xs[r][tj * BI + u];
    }
#pragma unroll
    for (int u = 0; u < BI; ++u)
#pragma unroll
      for (int v = 0; v < BI; ++v) acc[u][v] = fmaf(wv[u], xv[v], acc[u][v]);
  }
  __syncthreads();   // Xs is reused for the partial
  float* Ps = &Xs[0][0];
#pragma unroll
  for (int u = 0; u < BI; ++u)
#pragma unroll
    for (int v = 0; v < BI; ++v) Ps[(ti * BI + u) + (tj * BI + v) * BB] = acc[u][v];
  cluster.sync();
  // cluster reduction: CTA `rank` sums 1/PP_CL of the b x b block and adds it to WtX(t,t)
  const int rank = (int)cluster.block_rank();
  const int per = (b * b + PP_CL - 1) / PP_CL;
  for (int e = rank * per + threadIdx.x; e < min(b * b, (rank + 1) * per); e += blockDim.x) {
    const int i = e % b, j = e / b;
    float s = 0.f;
#pragma unroll
    for (int q = 0; q < PP_CL; ++q) s += cluster.map_shared_rank(Ps, q)[i + j * BB];
    atomicAdd(WtXtt + i + (int64_t)j * ldwtx, s);
  }
  cluster.sync();
}

cudaError_t launch_postpass(int64_t M, int b, const float* X, int64_t ldx, const float* W, int64_t ldw, __half* Xh,
                            int64_t ldxh, float* WtXtt, int64_t ldwtx, cudaStream_t st) {
  if (M <= 0) return cudaSuccess;
  auto grid = [&](int rows) {
    const int64_t g = (M + rows - 1) / rows;
    return (unsigned)((g + PP_CL - 1) / PP_CL * PP_CL);
  };
  if (b <= 16)
    return launch_pdl(postpass_kernel<16>, dim3(grid(pp_rows<16>())), dim3(256), 0, st, M, b, X, ldx, W, ldw, Xh,
                      ldxh, WtXtt, ldwtx);
  if (b <= 32)
    return launch_pdl(postpass_kernel<32>, dim3(grid(pp_rows<32>())), dim3(256), 0, st, M, b, X, ldx, W, ldw, Xh,
                      ldxh, WtXtt, ldwtx);
  return launch_pdl(postpass_kernel<64>, dim3(grid(pp_rows<64>())), dim3(256), 0, st, M, b, X, ldx, W, ldw, Xh,
                    ldxh, WtXtt, ldwtx);
}

}  // namespace sbr
