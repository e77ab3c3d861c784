// k_panel.cu -- panel factorisation: TSQR + Householder reconstruction (steps a1, a2).
//
// PAPER.md Sec. 5.1: the m x b panel is factored by Tall-Skinny QR, a
// reduction tree of local Householder QRs ("Householder transformation rather than
// modified Gram-Schmidt on each small block", "each warp is in charge of one
// column").  Sec. 5.2 (Alg. 3 + Ballard's sign matrix S, reading
// C7): the explicit Q of the tree is turned back into Householder vectors by the
// non-pivoted LU  Q_1 - S = L U  (s_j = -sign(d_j) chosen on the fly),
// Y = [L; Q_2 U^-1],  T = -U S L^-T,  W = Y T,  R = S R_tree.
//
// One cooperative kernel does the whole panel (grid barriers between tree levels):
//   up sweep   : leaves (<= 512 rows, b <= 32) and inner nodes (stacked child R's)
//                are QR-factored in registers, one warp per column; V, tau, R -> ws.
//   down sweep : explicit Q = H_node [C; 0] from the root down; leaves write their
//                Q rows over the panel.
//   reconstruct: CTA 0 runs the modified LU on Q's top b x b block and forms
//                T = -U S L^-T; every row i >= b then solves y_i U = q_i and
//                w_i = y_i T (thread per row).
// A panel that fits one leaf (m <= 32*S rows) is factored directly (exact LAPACK
// dgeqr2 convention, T by the dlarft recurrence), without tree or reconstruction.
//
// Outputs: the panel in A is overwritten in LAPACK compact form (R on and above
// the diagonal, Y's tail strictly below); explicit Y and W^0 = Y T columns
// (with zero rows above row0) go to the block's Y and W buffers.
#include <cooperative_groups.h>

#include "common.cuh"
#include "kernels.h"

namespace cg = cooperative_groups;

namespace sbr {

// Householder QR of a register-resident node (rows x b), warp w owns columns
// w, w+32, ... (slot j), lane l owns rows l, l+32, ... (slot s).  Writes the
// reflectors (unit diagonal, zeros above) to Vs (ld RS), taus, and R (b x b, ld b).
template <int CPW, int S>
SBR_DEV void cta_qr(float (&x)[CPW][S], int rows, int b, float* Vs, float* Rs, float* taus) {
  constexpr int NW = 32, RS = 32 * S;
  const int lane = lane_id(), warp = warp_id();
  const int kr = min(rows, b);
  for (int jc = 0; jc < kr; ++jc) {
    const int ow = jc % NW, oslot = jc / NW;
    if (warp == ow) {
#pragma unroll
      for (int j = 0; j < CPW; ++j) {
        if (j != oslot) continue;
        float a_l = 0.f, s2 = 0.f;
#pragma unroll
        for (int s = 0; s < S; ++s) {
          const int i = lane + 32 * s;
          const float v = x[j][s];
          if (i == jc) a_l = v;
          else if (i > jc) s2 = fmaf(v, v, s2);
        }
        const float alpha = warp_sum(a_l);
        const float sig2 = warp_sum(s2);
        float beta, tau, scal;
        if (sig2 == 0.f) {            // dlarfg: x(2:) == 0 -> H = I
          beta = alpha; tau = 0.f; scal = 0.f;
        } else {
          const float nrm = sqrtf(fmaf(alpha, alpha, sig2));
          beta = alpha >= 0.f ? -nrm : nrm;
          tau = (beta - alpha) / beta;
          scal = 1.f / (alpha - beta);
        }
#pragma unroll
        for (int s = 0; s < S; ++s) {
          const int i = lane + 32 * s;
          const float v = (i == jc) ? 1.f : (i > jc ? x[j][s] * scal : 0.f);
          Vs[i + jc * RS] = v;
          if (i < b) Rs[i + jc * b] = (i < jc) ? x[j][s] : (i == jc ? beta : 0.f);
        }
        if (lane == 0) taus[jc] = tau;
      }
    }
    __syncthreads();
    const float tau = taus[jc];
    if (tau != 0.f) {
#pragma unroll
      for (int j = 0; j < CPW; ++j) {
        const int c = warp + j * NW;
        if (c > jc && c < b) {
          float d = 0.f;
#pragma unroll
          for (int s = 0; s < S; ++s) d = fmaf(Vs[lane + 32 * s + jc * RS], x[j][s], d);
          d = warp_sum(d) * tau;
#pragma unroll
          for (int s = 0; s < S; ++s) x[j][s] = fmaf(-d, Vs[lane + 32 * s + jc * RS], x[j][s]);
        }
      }
    }
  }
  // wide node (rows < b): the remaining columns are all R
#pragma unroll
  for (int j = 0; j < CPW; ++j) {
    const int c = warp + j * NW;
    if (c >= kr && c < b) {
#pragma unroll
      for (int s = 0; s < S; ++s) {
        const int i = lane + 32 * s;
        if (i < b) Rs[i + c * b] = (i < rows) ? x[j][s] : 0.f;
      }
    }
  }
  for (int e = threadIdx.x; e < RS * b; e += blockDim.x) {
    const int c = e / RS;
    if (c >= kr) Vs[e] = 0.f;
  }
  if (threadIdx.x < b && threadIdx.x >= kr) taus[threadIdx.x] = 0.f;
  __syncthreads();
}

// x <- H_1 ... H_kr x   (explicit-Q formation, reflectors read from smem).
template <int CPW, int S>
SBR_DEV void cta_apply_q(float (&x)[CPW][S], int kr, int b, const float* Vs, const float* taus) {
  constexpr int NW = 32, RS = 32 * S;
  const int lane = lane_id(), warp = warp_id();
  for (int jc = kr - 1; jc >= 0; --jc) {
    const float tau = taus[jc];
    if (tau == 0.f) continue;
#pragma unroll
    for (int j = 0; j < CPW; ++j) {
      const int c = warp + j * NW;
      if (c < b) {
        float d = 0.f;
#pragma unroll
        for (int s = 0; s < S; ++s) d = fmaf(Vs[lane + 32 * s + jc * RS], x[j][s], d);
        d = warp_sum(d) * tau;
#pragma unroll
        for (int s = 0; s < S; ++s) x[j][s] = fmaf(-d, Vs[lane + 32 * s + jc * RS], x[j][s]);
      }
    }
  }
}

struct NodeInfo {
  int rows;
  int64_t start;  // level 0: first panel row
};

SBR_DEV NodeInfo node_info(const PanelArgs& a, int lev, int k) {
  NodeInfo ni;
  if (lev == 0) {
    const int64_t L = a.nodes[0];
    const int64_t s0 = (int64_t)k * a.m / L, s1 = (int64_t)(k + 1) * a.m / L;
    ni.start = s0;
    ni.rows = (int)(s1 - s0);
  } else {
    const int c0 = k * a.arity;
    const int nch = min(a.arity, a.nodes[lev - 1] - c0);
    ni.start = 0;
    ni.rows = nch * a.b;
  }
  return ni;
}

SBR_DEV float* node_v(const PanelArgs& a, int lev, int k, const NodeInfo& ni) {
  return a.ws_v + a.voff[lev] + (lev == 0 ? ni.start * a.b : (int64_t)k * a.arity * a.b * a.b);
}

template <int B, int CPW, int S>
__global__ void __launch_bounds__(1024, 1) panel_tsqr_kernel(PanelArgs a) {
  constexpr int NW = 32, RS = 32 * S;
  extern __shared__ __align__(16) float smem[];
  float* Vs = smem;               // RS x B
  float* Rs = Vs + RS * B;        // B x B
  float* taus = Rs + B * B;       // B (padded to 64)
  float* Us = taus + 64;          // B x B  (LU's U; later kept for the row solves)
  float* Ts = Us + B * B;         // B x B  (T)
  float* Ls = Ts + B * B;         // B x B  (L1, then scratch)
  float* Ss = Ls + B * B;         // B      (signs)
  const int b = a.b;
  const int lane = lane_id(), warp = warp_id();
  cg::grid_group grid = cg::this_grid();
  float x[CPW][S];

  // ---------------- up sweep ----------------
  for (int lev = 0; lev < a.nlev; ++lev) {
    for (int k = blockIdx.x; k < a.nodes[lev]; k += gridDim.x) {
      const NodeInfo ni = node_info(a, lev, k);
#pragma unroll
      for (int j = 0; j < CPW; ++j) {
        const int c = warp + j * NW;
#pragma unroll
        for (int s = 0; s < S; ++s) {
          const int i = lane + 32 * s;
          float v = 0.f;
          if (c < b && i < ni.rows) {
            if (lev == 0) {
              v = a.P[(ni.start + i) + (int64_t)c * a.ldp];
            } else {
              const int ch = k * a.arity + i / b, ii = i % b;
              v = a.ws_r[a.roff[lev - 1] + (int64_t)ch * b * b + ii + c * b];
            }
          }
          x[j][s] = v;
        }
      }
      cta_qr<CPW, S>(x, ni.rows, b, Vs, Rs, taus);
      if (a.nlev == 1) break;  // single leaf: keep V, R, tau in smem
      float* vd = node_v(a, lev, k, ni);
      for (int e = threadIdx.x; e < ni.rows * b; e += blockDim.x) {
        const int i = e % ni.rows, c = e / ni.rows;
        vd[e] = Vs[i + c * RS];
      }
      if (threadIdx.x < b) a.ws_tau[a.toff[lev] + (int64_t)k * b + threadIdx.x] = taus[threadIdx.x];
      for (int e = threadIdx.x; e < b * b; e += blockDim.x) a.ws_r[a.roff[lev] + (int64_t)k * b * b + e] = Rs[e];
      __syncthreads();
    }
    if (a.nlev > 1) grid.sync();
  }

  const int64_t M = a.M;
  const int64_t row0 = a.row0;
  if (a.nlev == 1) {
    // --------- single leaf: LAPACK-exact V, T (dlarft), R ---------
    const int rows = a.m, kr = min(rows, b);
    // T[0:j, j] = -tau_j T[0:j,0:j] (V^T v_j)[0:j]; first G[p][j] = v_p . v_j (p < j) by warps
    for (int pair = warp; pair < b * b; pair += NW) {
      const int p = pair % b, j = pair / b;
      if (p >= j) continue;
      float d = 0.f;
      for (int i = lane; i < rows; i += 32) d = fmaf(Vs[i + p * RS], Vs[i + j * RS], d);
      d = warp_sum(d);
      if (lane == 0) Ls[p + j * B] = d;
    }
    __syncthreads();
    for (int j = 0; j < b; ++j) {     // dlarft recurrence, one column per step
      const float tj = (j < kr) ? taus[j] : 0.f;
      if (threadIdx.x < b) {
        const int p = threadIdx.x;
        float val = (p == j) ? tj : 0.f;
        if (p < j) {
          float acc = 0.f;
          for (int q = p; q < j; ++q) acc = fmaf(Ts[p + q * B], Ls[q + j * B], acc);
          val = -tj * acc;
        }
        Ts[p + j * B] = val;
      }
      __syncthreads();
    }
    // rows: y = v, w = y T; compact panel: strictly lower = v, upper = R
    for (int64_t i = threadIdx.x; i < M; i += blockDim.x) {
      if (i < row0) {
        for (int c = 0; c < b; ++c) { a.Y[i + c * a.ldy] = 0.f; a.W[i + c * a.ldw] = 0.f; }
        if (a.Yh) for (int c = 0; c < b; ++c) a.Yh[i * a.ldyh + c] = __float2half_rn(0.f);
        continue;
      }
      const int64_t il = i - row0;
      for (int c = 0; c < b; ++c) {
        const float y = Vs[il + c * RS];
        a.Y[i + c * a.ldy] = y;
        if (a.Yh) a.Yh[i * a.ldyh + c] = __float2half_rn(y);
        a.P[il + c * a.ldp] = (il > c) ? y : (il < b ? Rs[il + c * b] : 0.f);
        float w = 0.f;
        for (int k = 0; k <= c; ++k) w = fmaf(Vs[il + k * RS], Ts[k + c * B], w);
        a.W[i + c * a.ldw] = w;
      }
    }
    return;
  }

  // ---------------- down sweep: explicit Q ----------------
  for (int lev = a.nlev - 1; lev >= 0; --lev) {
    for (int k = blockIdx.x; k < a.nodes[lev]; k += gridDim.x) {
      const NodeInfo ni = node_info(a, lev, k);
      const float* vs = node_v(a, lev, k, ni);
      for (int e = threadIdx.x; e < RS * b; e += blockDim.x) {   // rows >= ni.rows must read 0
        const int i = e % RS, c = e / RS;
        Vs[e] = (i < ni.rows) ? vs[i + c * ni.rows] : 0.f;
      }
      if (threadIdx.x < b) taus[threadIdx.x] = a.ws_tau[a.toff[lev] + (int64_t)k * b + threadIdx.x];
      __syncthreads();
      const float* cpar = nullptr;
      int ldc = 0;
      if (lev < a.nlev - 1) {
        const int parent = k / a.arity, idx = k % a.arity;
        const NodeInfo pi = node_info(a, lev + 1, parent);
        cpar = a.ws_q + a.qoff[lev + 1] + (int64_t)parent * a.arity * b * b + idx * b;
        ldc = pi.rows;
      }
#pragma unroll
      for (int j = 0; j < CPW; ++j) {
        const int c = warp + j * NW;
#pragma unroll
        for (int s = 0; s < S; ++s) {
          const int i = lane + 32 * s;
          float v = 0.f;
          if (c < b && i < b) v = cpar ? cpar[i + (int64_t)c * ldc] : (i == c ? 1.f : 0.f);
          x[j][s] = v;
        }
      }
      cta_apply_q<CPW, S>(x, min(ni.rows, b), b, Vs, taus);
#pragma unroll
      for (int j = 0; j < CPW; ++j) {
        const int c = warp + j * NW;
#pragma unroll
        for (int s = 0; s < S; ++s) {
          const int i = lane + 32 * s;
          if (c < b && i < ni.rows) {
            if (lev == 0) a.P[(ni.start + i) + (int64_t)c * a.ldp] = x[j][s];
            else a.ws_q[a.qoff[lev] + (int64_t)k * a.arity * b * b + i + (int64_t)c * ni.rows] = x[j][s];
          }
        }
      }
      __syncthreads();
    }
    grid.sync();
  }

  // ---------------- reconstruction (Alg. 3 + S) ----------------
  if (blockIdx.x == 0) {
    // Q_1 = top b x b of the explicit Q (written by this CTA: leaf 0)
    for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
      const int i = e % b, c = e / b;
      Us[i + c * B] = a.P[i + (int64_t)c * a.ldp];
      Ts[i + c * B] = Us[i + c * B];   // keep Q_1 for W_top
    }
    __syncthreads();
    for (int j = 0; j < b; ++j) {      // non-pivoted LU of Q_1 - S
      if (threadIdx.x == 0) {
        const float d = Us[j + j * B];
        const float sj = (d >= 0.f) ? -1.f : 1.f;   // s_j = -sign(d_j)
        Ss[j] = sj;
        Us[j + j * B] = d - sj;
      }
      __syncthreads();
      const float piv = Us[j + j * B];
      for (int i = j + 1 + threadIdx.x; i < b; i += blockDim.x) Us[i + j * B] /= piv;
      __syncthreads();
      const int nt = b - j - 1;
      for (int e = threadIdx.x; e < nt * nt; e += blockDim.x) {
        const int i = j + 1 + e % nt, c = j + 1 + e / nt;
        Us[i + c * B] = fmaf(-Us[i + j * B], Us[j + c * B], Us[i + c * B]);
      }
      __syncthreads();
    }
    // L1 (unit lower) -> Ls;  L1^-1 by column forward substitution (thread per column) -> scratch in Rs? keep R!
    for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
      const int i = e % b, c = e / b;
      Ls[i + c * B] = (i > c) ? Us[i + c * B] : (i == c ? 1.f : 0.f);
    }
    __syncthreads();
    // Linv (lower unit) into Vs scratch (Vs is free now): Linv[:, c] solves L1 x = e_c
    float* Linv = Vs;
    if (threadIdx.x < b) {
      const int c = threadIdx.x;
      for (int i = 0; i < b; ++i) {
        float v = (i == c) ? 1.f : 0.f;
        for (int k = c; k < i; ++k) v = fmaf(-Ls[i + k * B], Linv[k + c * B], v);
        Linv[i + c * B] = (i < c) ? 0.f : v;
      }
    }
    __syncthreads();
    // T = -U S L1^-T : T[r][c] = -sum_k U[r][k] s_k Linv[c][k], k in [r, c]
    float* Tn = Vs + B * B;
    for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
      const int r = e % b, c = e / b;
      float acc = 0.f;
      for (int k = r; k <= c; ++k) acc = fmaf(Us[r + k * B] * Ss[k], Linv[c + k * B], acc);
      Tn[r + c * B] = (r <= c) ? -acc : 0.f;
    }
    __syncthreads();
    // R = S R_root ; publish U, T for the row solves
    const float* rroot = a.ws_r + a.roff[a.nlev - 1];
    for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
      const int i = e % b, c = e / b;
      a.ws_misc[e] = (i <= c) ? Us[i + c * B] : 0.f;              // U
      a.ws_misc[b * b + e] = Tn[i + c * B];                          // T
      // top b rows of the panel: Y_top = L1, W_top = L1 T, compact = L1 (strict) / S R
      const float rfin = Ss[i] * rroot[i + c * b];
      a.P[i + (int64_t)c * a.ldp] = (i > c) ? Ls[i + c * B] : rfin;
      a.Y[(row0 + i) + c * a.ldy] = Ls[i + c * B];
      if (a.Yh) a.Yh[(row0 + i) * a.ldyh + c] = __float2half_rn(Ls[i + c * B]);
      float w = 0.f;
      for (int k = 0; k <= min(i, c); ++k) w = fmaf(Ls[i + k * B], Tn[k + c * B], w);
      a.W[(row0 + i) + c * a.ldw] = w;
    }
  }
  grid.sync();
  // rows i >= b of the panel:  y_i U = q_i  ;  w_i = y_i T   (thread per row)
  for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
    Us[e % b + (e / b) * B] = a.ws_misc[e];
    Ts[e % b + (e / b) * B] = a.ws_misc[b * b + e];
  }
  __syncthreads();
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t nth = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid; i < row0; i += nth) {
    for (int c = 0; c < b; ++c) { a.Y[i + c * a.ldy] = 0.f; a.W[i + c * a.ldw] = 0.f; }
    if (a.Yh) for (int c = 0; c < b; ++c) a.Yh[i * a.ldyh + c] = __float2half_rn(0.f);
  }
  for (int64_t il = b + tid; il < a.m; il += nth) {
    float q[B];
#pragma unroll
    for (int c = 0; c < B; ++c) q[c] = (c < b) ? a.P[il + (int64_t)c * a.ldp] : 0.f;
#pragma unroll
    for (int c = 0; c < B; ++c) {
      if (c < b) {
        float v = q[c];
#pragma unroll
        for (int k = 0; k < c; ++k) v = fmaf(-q[k], Us[k + c * B], v);
        q[c] = v / Us[c + c * B];
      }
    }
#pragma unroll
    for (int c = 0; c < B; ++c) {
      if (c < b) {
        a.P[il + (int64_t)c * a.ldp] = q[c];
        a.Y[(row0 + il) + c * a.ldy] = q[c];
        if (a.Yh) a.Yh[(row0 + il) * a.ldyh + c] = __float2half_rn(q[c]);
      }
    }
#pragma unroll
    for (int c = B - 1; c >= 0; --c) {
      if (c < b) {
        float w = 0.f;
#pragma unroll
        for (int k = 0; k <= c; ++k) w = fmaf(q[k], Ts[k + c * B], w);
        q[c] = w;
      }
    }
#pragma unroll
    for (int c = 0; c < B; ++c)
      if (c < b) a.W[(row0 + il) + c * a.ldw] = q[c];
  }
}

// ---------------------------------------------------------------- host side
template <int B, int CPW, int S>
static cudaError_t launch_panel_t(PanelArgs& a, int max_ctas, cudaStream_t st) {
  constexpr int RS = 32 * S;
  const size_t smem = sizeof(float) * (RS * B + B * B + 64 + 4 * B * B + B);
  auto kern = panel_tsqr_kernel<B, CPW, S>;
  static bool attr_set = false;
  if (!attr_set) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    attr_set = true;
  }
  // tree shape
  const int cap = RS;
  int L = (a.m <= cap) ? 1 : (a.m + cap - 1) / cap;
  a.arity = max(2, cap / a.b);
  a.nlev = 0;
  int nodes = L;
  int64_t voff = 0, roff = 0, toff = 0, qoff = 0;
  while (true) {
    a.nodes[a.nlev] = nodes;
    a.voff[a.nlev] = voff;
    a.roff[a.nlev] = roff;
    a.toff[a.nlev] = toff;
    a.qoff[a.nlev] = qoff;
    if (a.nlev == 0) voff += (int64_t)a.m * a.b;
    else { voff += (int64_t)nodes * a.arity * a.b * a.b; qoff += (int64_t)nodes * a.arity * a.b * a.b; }
    roff += (int64_t)nodes * a.b * a.b;
    toff += (int64_t)nodes * a.b;
    a.nlev++;
    if (nodes == 1) break;
    nodes = (nodes + a.arity - 1) / a.arity;
    if (a.nlev >= kPanelMaxLev) return cudaErrorInvalidValue;
  }
  const int grid = (L == 1) ? 1 : min(L, max_ctas);
  void* args[] = {&a};
  return cudaLaunchCooperativeKernel((const void*)kern, dim3(grid), dim3(1024), args, smem, st);
}

cudaError_t launch_panel(PanelArgs& a, int max_ctas, cudaStream_t st) {
  if (a.b <= 8) return launch_panel_t<8, 1, 16>(a, max_ctas, st);
  if (a.b <= 16) return launch_panel_t<16, 1, 16>(a, max_ctas, st);
  if (a.b <= 32) return launch_panel_t<32, 1, 16>(a, max_ctas, st);
  return launch_panel_t<64, 2, 8>(a, max_ctas, st);
}

PanelWs panel_ws_sizes(int64_t m_max, int b) {
  // leaves hold >= 256/2 rows, so #nodes over all levels <= 2*(m/128 + 1) + 2
  const int64_t nodes = 2 * (m_max / 128 + 2) + 2;
  const int64_t arity_rows = 64 * 64 * 2;  // generous: inner node rows x b bound
  PanelWs w;
  w.v = (size_t)(m_max * b + nodes * arity_rows + 4096);
  w.q = (size_t)(nodes * arity_rows + 4096);
  w.r = (size_t)(nodes * b * b + 4096);
  w.tau = (size_t)(nodes * b + 256);
  w.misc = (size_t)(2 * 64 * 64 + 256);
  return w;
}

int panel_max_ctas(int b) {
  int dev = 0, nsm = 0, per = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  const void* k;
  size_t smem;
  if (b <= 8) { k = (const void*)panel_tsqr_kernel<8, 1, 16>; smem = sizeof(float) * (512 * 8 + 5 * 64 + 64 + 8); }
  else if (b <= 16) { k = (const void*)panel_tsqr_kernel<16, 1, 16>; smem = sizeof(float) * (512 * 16 + 5 * 256 + 64 + 16); }
  else if (b <= 32) { k = (const void*)panel_tsqr_kernel<32, 1, 16>; smem = sizeof(float) * (512 * 32 + 5 * 1024 + 64 + 32); }
  else { k = (const void*)panel_tsqr_kernel<64, 2, 8>; smem = sizeof(float) * (256 * 64 + 5 * 4096 + 64 + 64); }
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k, 1024, smem);
  return max(1, per) * nsm;
}

}  // namespace sbr
