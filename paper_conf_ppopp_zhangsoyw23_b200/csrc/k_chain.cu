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
//   * the reduction dimension is split over the 16 CTAs of a thread-block cluster (kxb; 8 for
//     the postpass) and the partial results are summed through distributed shared memory -- no global atomics on
//     the hot addresses, no pre-zeroed outputs, no second launch.
#include <cooperative_groups.h>

#include "common.cuh"
#include "kernels.h"

namespace cg = cooperative_groups;

namespace sbr {

constexpr int KXB_QT = 32;   // output rows (q) per cluster
constexpr int KXB_RC = 64;   // r-chunk staged in shared memory per iteration

// CL = CTAs per cluster (split of the reduction dimension r): 16 (non-portable cluster size,
// halves each warp's dependent chain and doubles the resident warps), 8 if that launch fails.
// NG = 32-column groups of b (1: b <= 32, 2: b <= 64).
template <int CL, int NG>
SBR_DEV void kxb_body(const KxbArgs& a, int qblk) {
  constexpr int NB = 32 * NG;
  constexpr int LA = KXB_RC * KXB_QT / 256;   // A elements staged per thread per chunk
  constexpr int LB = KXB_RC * NB / 256;       // B elements staged per thread per chunk
  __shared__ __align__(16) float As[KXB_RC][KXB_QT];   // As[r][q] = WtX[q0+q, r]; reused for partials
  __shared__ float Bs[KXB_RC][NB + 1];                  // Bs[r][p] = B(r, p)
  cg::cluster_group cluster = cg::this_cluster();
  pdl_trigger();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int k = a.k, b = a.b;
  const bool lazy = a.mode == 0;
  const int q0 = qblk * KXB_QT;
  const int rank = (int)cluster.block_rank();
  const int rper = (k + CL - 1) / CL;
  const int rb = rank * rper, re = min(k, rb + rper);
  float* __restrict__ WtX = a.WtX;
  const int64_t ldwx = a.ldwx;
  float acc[4][NG];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int g = 0; g < NG; ++g) acc[i][g] = 0.f;
  pdl_wait();
  for (int r0 = rb; r0 < re; r0 += KXB_RC) {
    const int nr = min(KXB_RC, re - r0);
    // stage: every load of the chunk issued (into registers) before the first shared store
    float av[LA], bv[LB];
#pragma unroll
    for (int u = 0; u < LA; ++u) {
      const int e = threadIdx.x + u * 256;
      const int q = e % KXB_QT, r = e / KXB_QT;
      av[u] = (r < nr && q0 + q < k) ? __ldcg(WtX + (q0 + q) + (int64_t)(r0 + r) * ldwx) : 0.f;
    }
    if (lazy) {
#pragma unroll
      for (int u = 0; u < LB; ++u) {
        const int e = threadIdx.x + u * 256;
        const int p = e % NB, r = e / NB;
        bv[u] = (r < nr && p < b) ? __ldcg(a.Y + (a.c + p) + (int64_t)(r0 + r) * a.ldy) : 0.f;
      }
    } else {
#pragma unroll
      for (int u = 0; u < LB; ++u) {
        const int e = threadIdx.x + u * 256;
        const int r = e % KXB_RC, p = e / KXB_RC;
        bv[u] = (r < nr && p < b) ? __ldcg(a.G + (r0 + r) + (int64_t)p * a.ldg) : 0.f;
      }
    }
#pragma unroll
    for (int u = 0; u < LA; ++u) {
      const int e = threadIdx.x + u * 256;
      As[e / KXB_QT][e % KXB_QT] = av[u];
    }
#pragma unroll
    for (int u = 0; u < LB; ++u) {
      const int e = threadIdx.x + u * 256;
      if (lazy) Bs[e / NB][e % NB] = bv[u];
      else Bs[e % KXB_RC][e / KXB_RC] = bv[u];
    }
    __syncthreads();
#pragma unroll 4
    for (int r = 0; r < nr; ++r) {
      const float4 a4 = *reinterpret_cast<const float4*>(&As[r][warp * 4]);
      const float aa[4] = {a4.x, a4.y, a4.z, a4.w};
#pragma unroll
      for (int g = 0; g < NG; ++g) {
        const float bb = Bs[r][lane + 32 * g];
#pragma unroll
        for (int i = 0; i < 4; ++i) acc[i][g] = fmaf(aa[i], bb, acc[i][g]);
      }
    }
    __syncthreads();
  }
  // partials -> shared (As reused as Ps[q][p], p < NB), then the cluster reduction:
  // CTA `rank` finalises rows q in [rank*QPC, rank*QPC + QPC) of the cluster's 32.
  constexpr int QPC = KXB_QT / CL;
  static_assert(KXB_RC * KXB_QT >= KXB_QT * 64, "partials fit in As");
  float* Ps = &As[0][0];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int g = 0; g < NG; ++g) Ps[(warp * 4 + i) * NB + lane + 32 * g] = acc[i][g];
  cluster.sync();
  for (int e = threadIdx.x; e < QPC * b; e += blockDim.x) {
    const int qi = rank * QPC + e / b, p = e % b;
    const int q = q0 + qi;
    float part[CL];
#pragma unroll
    for (int j = 0; j < CL; ++j) part[j] = cluster.map_shared_rank(Ps, j)[qi * NB + p];
    float s = 0.f;
#pragma unroll
    for (int j = 0; j < CL; ++j) s += part[j];
    if (q < k) {
      if (lazy) {
        const float d = __ldcg(a.X + (a.c + p) + (int64_t)q * a.ldx) - s;
        if (a.Ph) a.Ph[(int64_t)p * a.ldph + q] = cvt16(d);
        if (a.P32) a.P32[q + (int64_t)p * a.ldp32] = d;
      } else {
        const float d = __ldcg(a.H + q + (int64_t)p * a.ldg) - s;
        WtX[q + (int64_t)(k + p) * ldwx] = d;
        WtX[(k + p) + (int64_t)q * ldwx] = d;
      }
    }
  }
  if (lazy) {
    if (qblk == 0 && rank == 0) {   // upper <- lower on the b x b diagonal block of the panel's columns
      for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
        const int i = e % b, j = e / b;
        if (i < j) a.Adiag[i + (int64_t)j * a.lda] = a.Adiag[j + (int64_t)i * a.lda];
      }
    }
  } else if (a.Gh) {   // G -> fp16, column-major (k contiguous): B operand of the merge GEMM
    const int64_t nth = (int64_t)gridDim.x * gridDim.y * blockDim.x;
    const int64_t tid = ((int64_t)blockIdx.y * gridDim.x + blockIdx.x) * blockDim.x + threadIdx.x;
    for (int64_t e = tid; e < (int64_t)k * b; e += nth) {
      const int r = (int)(e % k), p = (int)(e / k);
      a.Gh[r + (int64_t)p * a.ldgh] = cvt16(__ldcg(a.G + r + (int64_t)p * a.ldg));
    }
  }
  cluster.sync();   // keep this CTA's partials alive until every reader is done
}

template <int CL, int NG>
__global__ void __launch_bounds__(256) kxb_kernel(KxbArgs a) {
  kxb_body<CL, NG>(a, blockIdx.x);
}

template <int CL, int NG>
static cudaError_t launch_kxb_t(const KxbArgs& a, cudaStream_t st) {
  auto kern = kxb_kernel<CL, NG>;
  if (CL > 8) {
    const cudaError_t e = func_attr((const void*)kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    if (e != cudaSuccess) return e;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((a.k + KXB_QT - 1) / KXB_QT, CL);
  cfg.blockDim = dim3(256);
  cfg.dynamicSmemBytes = 0;
  cfg.stream = st;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = 1;
  at[0].val.clusterDim.y = CL;
  at[0].val.clusterDim.z = 1;
  at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl_enabled() ? 2 : 1;
  return cudaLaunchKernelEx(&cfg, kern, a);
}

static int kxb_cluster() {   // SBR_KXB_CL=8 forces the portable cluster size (ablation)
  static int cl = [] {
    const char* e = std::getenv("SBR_KXB_CL");
    return (e && std::atoi(e) == 8) ? 8 : 16;
  }();
  return cl;
}

cudaError_t launch_kxb(const KxbArgs& a, cudaStream_t st) {
  if (a.k <= 0 || a.b <= 0) return cudaSuccess;
  static bool cl16_ok = true;
  if (cl16_ok && kxb_cluster() == 16) {
    const cudaError_t e = a.b <= 32 ? launch_kxb_t<16, 1>(a, st) : launch_kxb_t<16, 2>(a, st);
    if (e == cudaSuccess) return e;
    cudaGetLastError();   // cluster of 16 not schedulable here: portable size from now on
    cl16_ok = false;
  }
  return a.b <= 32 ? launch_kxb_t<8, 1>(a, st) : launch_kxb_t<8, 2>(a, st);
}

// ------------------------------------------------------------------ postpass
constexpr int PP_CL = 8;

template <int BB>  // BB >= b, multiple of 16; rows per CTA sized for 48 KB of static smem
constexpr int pp_rows() { return BB <= 16 ? 128 : 64; }   // 8-16 loads per thread and array, ~3 CTAs per SM

template <int BB>
SBR_DEV void postpass_body(int64_t M, int b, const float* __restrict__ X, int64_t ldx, const float* __restrict__ W,
                           int64_t ldw, __half* Xh, int64_t ldxh, float* WtXtt, int64_t ldwtx, int vblk) {
  constexpr int PP_ROWS = pp_rows<BB>();
  constexpr int BI = BB / 16;   // register block BI x BI per thread (16 x 16 thread grid)
  __shared__ float Xs[PP_ROWS][BB + 1];
  __shared__ float Ws[PP_ROWS][BB + 1];
  static_assert(PP_ROWS * (BB + 1) >= BB * BB, "partial fits in Xs");
  cg::cluster_group cluster = cg::this_cluster();
  pdl_trigger();
  pdl_wait();
  const int64_t rbeg = (int64_t)vblk * PP_ROWS;
  const int nr = (int)(M - rbeg < PP_ROWS ? (M - rbeg > 0 ? M - rbeg : 0) : PP_ROWS);
  constexpr int LU = PP_ROWS * BB / 256;   // elements per thread and array, all loads issued before any store
  float xv[LU], wv[LU];
#pragma unroll
  for (int u = 0; u < LU; ++u) {
    const int e = threadIdx.x + u * 256;
    const int r = e % PP_ROWS, c = e / PP_ROWS;
    const bool in = r < nr && c < b;
    xv[u] = in ? __ldcg(X + (rbeg + r) + (int64_t)c * ldx) : 0.f;
    wv[u] = in ? __ldcg(W + (rbeg + r) + (int64_t)c * ldw) : 0.f;
  }
#pragma unroll
  for (int u = 0; u < LU; ++u) {
    const int e = threadIdx.x + u * 256;
    Xs[e % PP_ROWS][e / PP_ROWS] = xv[u];
    Ws[e % PP_ROWS][e / PP_ROWS] = wv[u];
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
      for (int u = 0; u < 8; ++u) hv[u] = cvt16(Xs[r][g * 8 + u]);
      *reinterpret_cast<uint4*>(dst) = *reinterpret_cast<const uint4*>(hv);
    } else {
      for (int u = 0; u < 8 && g * 8 + u < b; ++u) dst[u] = cvt16(Xs[r][g * 8 + u]);
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

template <int BB>
__global__ void __cluster_dims__(PP_CL, 1, 1) __launch_bounds__(256)
    postpass_kernel(int64_t M, int b, const float* __restrict__ X, int64_t ldx, const float* __restrict__ W,
                    int64_t ldw, __half* Xh, int64_t ldxh, float* WtXtt, int64_t ldwtx) {
  postpass_body<BB>(M, b, X, ldx, W, ldw, Xh, ldxh, WtXtt, ldwtx, blockIdx.x);
}

// The postpass of panel t and the MERGE kxb of panel t (W^T X_t = H - (W^T X) G; G -> fp16 is a
// separate small launch before the merge GEMM) in ONE launch: CTAs [0, npp) are the postpass's,
// the rest form the kxb's 8-CTA clusters.  Both read only what the pass and the merge left
// behind and write disjoint parts of W^T X (diagonal block / column + row block).
template <int BB, int NG>
__global__ void __cluster_dims__(PP_CL, 1, 1) __launch_bounds__(256)
    postpass_merge_kernel(int64_t M, int b, const float* __restrict__ X, int64_t ldx, const float* __restrict__ W,
                          int64_t ldw, __half* Xh, int64_t ldxh, float* WtXtt, int64_t ldwtx, KxbArgs a, int npp) {
  if ((int)blockIdx.x < npp)
    postpass_body<BB>(M, b, X, ldx, W, ldw, Xh, ldxh, WtXtt, ldwtx, blockIdx.x);
  else
    kxb_body<PP_CL, NG>(a, ((int)blockIdx.x - npp) / PP_CL);
}

cudaError_t launch_postpass_merge(int64_t M, int b, const float* X, int64_t ldx, const float* W, int64_t ldw,
                                  __half* Xh, int64_t ldxh, float* WtXtt, int64_t ldwtx, const KxbArgs& a,
                                  cudaStream_t st) {
  if (M <= 0) return cudaSuccess;
  KxbArgs m = a;
  m.mode = 1;
  m.Gh = nullptr;
  if (b > 32) {   // both kernels' static shared memory together exceeds 48 KB: two launches
    const cudaError_t e = launch_kxb(m, st);
    if (e != cudaSuccess) return e;
    return launch_postpass(M, b, X, ldx, W, ldw, Xh, ldxh, WtXtt, ldwtx, st);
  }
  const int rows = b <= 16 ? pp_rows<16>() : pp_rows<32>();
  const int64_t g = (M + rows - 1) / rows;
  const int npp = (int)((g + PP_CL - 1) / PP_CL * PP_CL);
  const int nk = a.k > 0 ? (a.k + KXB_QT - 1) / KXB_QT : 0;
  const dim3 grid((unsigned)(npp + nk * PP_CL));
  if (b <= 16)
    return launch_pdl(postpass_merge_kernel<16, 1>, grid, dim3(256), 0, st, M, b, X, ldx, W, ldw, Xh, ldxh, WtXtt,
                      ldwtx, m, npp);
  return launch_pdl(postpass_merge_kernel<32, 1>, grid, dim3(256), 0, st, M, b, X, ldx, W, ldw, Xh, ldxh, WtXtt,
                    ldwtx, m, npp);
}

__global__ void __launch_bounds__(256) g_to_half_kernel(int k, int b, const float* __restrict__ G, int64_t ldg,
                                                        __half* Gh, int64_t ldgh) {
  pdl_trigger();
  pdl_wait();
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  if (e < k * b) {
    const int r = e % k, p = e / k;
    Gh[r + (int64_t)p * ldgh] = cvt16(__ldcg(G + r + (int64_t)p * ldg));
  }
}

cudaError_t launch_g_to_half(int k, int b, const float* G, int64_t ldg, __half* Gh, int64_t ldgh, cudaStream_t st) {
  if (k <= 0 || b <= 0) return cudaSuccess;
  return launch_pdl(g_to_half_kernel, dim3((unsigned)((k * b + 255) / 256)), dim3(256), 0, st, k, b, G, ldg, Gh,
                    ldgh);
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

SBR_OP16_SETTER(chain)

}  // namespace sbr
