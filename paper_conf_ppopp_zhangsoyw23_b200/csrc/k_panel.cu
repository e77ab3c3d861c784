// k_panel.cu -- panel factorisation: TSQR + Householder reconstruction (steps a1, a2).
//
// PAPER.md Sec. 5.1: the m x b panel is factored by Tall-Skinny QR, a
// reduction tree of local Householder QRs ("Householder transformation rather than
// modified Gram-Schmidt on each small block", "each warp is in charge of one
// column").  Sec. 5.2 (Alg. 3 + Ballard's sign matrix S, reading
// C7): the explicit Q of the tree is turned back into Householder vectors by the
// non-pivoted LU  Q_1 - S = L U  (s_j = -sign(d_j) chosen on the fly):
//     Y = [L; Q_2 U^-1],   W = Y T = (E - Q S) L^-T,   R = S R_tree.
// Each row of Y and W is obtained by two b x b triangular solves (with U and with L),
// so the T factor is never formed.
//
// One cooperative kernel per panel, one CTA (16 warps, each owning b/16 columns) per
// leaf of <= 256 rows, inner tree nodes of <= 512 rows (16 stacked R factors for b=32):
//   up    : node QR in registers; the reflector of column j is broadcast through shared
//           memory and read ONCE into registers by every warp; V -> ws; grid barrier
//           per level; the root CTA factors the root and forms its explicit Q directly.
//   down  : each node forms H_node [C; 0] from its parent's block C; a leaf keeps its
//           Q rows in shared memory.  CTA 0 (leaf 0 holds Q's top b rows) runs the
//           modified LU in one warp (columns in registers) and publishes L, U, S.
//   rows  : after one more grid barrier every CTA solves its own rows from shared
//           memory and writes Y (fp32 + fp16 row-major), W^0 and the compact panel.
// A panel of <= 512 rows is factored directly by one CTA (LAPACK dgeqr2 convention,
// T by the dlarft recurrence) -- no tree and no reconstruction.
#include <cooperative_groups.h>

#include "common.cuh"
#include "kernels.h"

namespace cg = cooperative_groups;

namespace sbr {

constexpr int P_NW = 32;   // warps per CTA (one column per warp for b <= 32)
constexpr int P_SL = 8;    // leaf rows per lane  (256-row leaves)
constexpr int P_SN = 16;   // inner-node rows per lane (512-row nodes)

SBR_DEV int64_t gtimer() {
  int64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define PTRACE(k) \
  if (a.trace && blockIdx.x == 0 && threadIdx.x == 0) a.trace[k] = gtimer();

// Householder QR of a register-resident node (rows x b, rows <= 32*S): warp w owns columns
// w, w+NW, .. (slot j), lane l owns rows l, l+32, .. (slot s).  Reflector jc (unit diagonal,
// zeros above) goes to Vs[:, jc] (ld 32*S), tau to taus[jc], R (b x b, ld b) to Rs.
// Reflector of column jc from alpha = x[jc] and sig2 = ||x[jc+1:]||^2 (dlarfg), written to
// Vs[:, jc], Rs[:, jc] and taus[jc] by the owning warp (column values in xs[0..S)).
template <int S, int SM>
SBR_DEV void make_reflector(const float (&xs)[SM], int jc, int b, float alpha, float sig2, float* Vs, float* Rs,
                            float* taus) {
  constexpr int RS = 32 * S;
  const int lane = lane_id();
  float beta, tau, scal;
  if (sig2 <= 0.f) {               // dlarfg: x(2:) == 0 -> H = I
    beta = alpha; tau = 0.f; scal = 0.f;
  } else {
    const float nrm = sqrtf(fmaf(alpha, alpha, sig2));
    beta = alpha >= 0.f ? -nrm : nrm;
    tau = __fdividef(beta - alpha, beta);
    scal = __frcp_rn(alpha - beta);
  }
#pragma unroll
  for (int s = 0; s < S; ++s) {
    const int i = lane + 32 * s;
    Vs[i + jc * RS] = (i == jc) ? 1.f : (i > jc ? xs[s] * scal : 0.f);
    if (i < b) Rs[i + jc * b] = (i < jc) ? xs[s] : (i == jc ? beta : 0.f);
  }
  if (lane == 0) taus[jc] = tau;
}

// alpha = x[jc], sig2 = sum_{i > jc} x_i^2 by a plain warp reduction
template <int S, int SM>
SBR_DEV void col_norm(const float (&xs)[SM], int jc, float& alpha, float& sig2) {
  const int lane = lane_id();
  float a_own = 0.f, s2 = 0.f;
#pragma unroll
  for (int s = 0; s < S; ++s) {
    const int i = lane + 32 * s;
    if (i == jc) a_own = xs[s];
    if (i > jc) s2 = fmaf(xs[s], xs[s], s2);
  }
  alpha = __shfl_sync(0xffffffffu, a_own, jc & 31);
  sig2 = warp_sum(s2);
}

// Householder QR of a register-resident node (rows x b, rows <= 32*S): warp w owns columns
// w, w+NW, .. (slot j), lane l owns rows l, l+32, .. (slot s).  Reflector jc (unit diagonal,
// zeros above) goes to Vs[:, jc] (ld 32*S), tau to taus[jc], R (b x b, ld b) to Rs.
// The warp owning column jc+1 fuses, into the single reduction of its update with
// reflector jc, the sums it needs for reflector jc+1 (norm downdate
//   ||x - d v||^2 = xx - 2 d xv + d^2 vv  over rows > jc+1),
// and recomputes the norm directly when the downdate cancels (< 1/64 of xx).
template <int CPW, int S, int SM>
SBR_DEV void cta_qr(float (&x)[CPW][SM], int rows, int b, float* Vs, float* Rs, float* taus,
                    long long* dbg = nullptr) {
  constexpr int RS = 32 * S;
  const int lane = lane_id(), warp = warp_id();
  const int kr = min(rows, b);
  const int wmax = warp + (CPW - 1) * P_NW;  // this warp's last column
  if (warp == 0 && kr > 0) {
    float alpha, sig2;
    col_norm<S, SM>(x[0], 0, alpha, sig2);
    make_reflector<S, SM>(x[0], 0, b, alpha, sig2, Vs, Rs, taus);
  }
  long long t_a = 0, t_b = 0, t_c = 0, t_d = 0;
  for (int jc = 0; jc < kr; ++jc) {
    const long long c0 = clock64();
    __syncthreads();                                  // reflector jc published
    const long long c1 = clock64();
    const float tau = taus[jc];
    if (wmax <= jc) continue;
    float v[S];
#pragma unroll
    for (int s = 0; s < S; ++s) v[s] = Vs[lane + 32 * s + jc * RS];
#pragma unroll
    for (int j = 0; j < CPW; ++j) {
      const int c = warp + j * P_NW;
      if (c <= jc || c >= b) continue;
      const int nx = jc + 1;
      if (c == nx && nx < kr) {                       // next owner: fused reduction
        t_a += c1 - c0;
        float d0 = 0.f, xx = 0.f, xv = 0.f, vv = 0.f, xo = 0.f, vo = 0.f;
#pragma unroll
        for (int s = 0; s < S; ++s) {
          const int i = lane + 32 * s;
          d0 = fmaf(v[s], x[j][s], d0);
          if (i > nx) {
            xx = fmaf(x[j][s], x[j][s], xx);
            xv = fmaf(x[j][s], v[s], xv);
            vv = fmaf(v[s], v[s], vv);
          }
          if (i == nx) { xo = x[j][s]; vo = v[s]; }
        }
        const long long c2 = clock64();
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
          d0 += __shfl_xor_sync(0xffffffffu, d0, o);
          xx += __shfl_xor_sync(0xffffffffu, xx, o);
          xv += __shfl_xor_sync(0xffffffffu, xv, o);
          vv += __shfl_xor_sync(0xffffffffu, vv, o);
        }
        const long long c3 = clock64();
        t_b += c2 - c1;
        t_c += c3 - c2;
        const float d = d0 * tau;
#pragma unroll
        for (int s = 0; s < S; ++s) x[j][s] = fmaf(-d, v[s], x[j][s]);
        const float xo_b = __shfl_sync(0xffffffffu, xo, nx & 31);
        const float vo_b = __shfl_sync(0xffffffffu, vo, nx & 31);
        const float alpha = fmaf(-d, vo_b, xo_b);
        float sig2 = fmaf(d * d, vv, fmaf(-2.f * d, xv, xx));
        if (!(sig2 > xx * (1.f / 64.f))) {            // cancellation: recompute directly
          float a2;
          col_norm<S, SM>(x[j], nx, a2, sig2);
        }
        make_reflector<S, SM>(x[j], nx, b, alpha, sig2, Vs, Rs, taus);
        t_d += clock64() - c3;
      } else if (tau != 0.f) {
        float d0 = 0.f, d1 = 0.f;
#pragma unroll
        for (int s = 0; s < S; s += 2) {
          d0 = fmaf(v[s], x[j][s], d0);
          if (s + 1 < S) d1 = fmaf(v[s + 1], x[j][s + 1], d1);
        }
        const float d = warp_sum(d0 + d1) * tau;
#pragma unroll
        for (int s = 0; s < S; ++s) x[j][s] = fmaf(-d, v[s], x[j][s]);
      }
    }
  }
#pragma unroll
  if (dbg && lane == 0 && blockIdx.x == 0) {
    atomicAdd((unsigned long long*)&dbg[0], (unsigned long long)t_a);
    atomicAdd((unsigned long long*)&dbg[1], (unsigned long long)t_b);
    atomicAdd((unsigned long long*)&dbg[2], (unsigned long long)t_c);
    atomicAdd((unsigned long long*)&dbg[3], (unsigned long long)t_d);
  }
  for (int j = 0; j < CPW; ++j) {  // wide node (rows < b): the remaining columns are all R
    const int c = warp + j * P_NW;
    if (c >= kr && c < b) {
#pragma unroll
      for (int s = 0; s < S; ++s) {
        const int i = lane + 32 * s;
        if (i < b) Rs[i + c * b] = (i < rows) ? x[j][s] : 0.f;
      }
    }
  }
  for (int e = threadIdx.x; e < RS * b; e += blockDim.x)
    if (e / RS >= kr) Vs[e] = 0.f;
  if (threadIdx.x < b && threadIdx.x >= kr) taus[threadIdx.x] = 0.f;
  __syncthreads();
}

// x <- H_1 ... H_kr x   (explicit-Q formation; reflectors read from smem, no barriers).
template <int CPW, int S, int SM>
SBR_DEV void cta_apply_q(float (&x)[CPW][SM], int kr, int b, const float* Vs, const float* taus) {
  constexpr int RS = 32 * S;
  const int lane = lane_id(), warp = warp_id();
  if (warp >= b) return;
  for (int jc = kr - 1; jc >= 0; --jc) {
    const float tau = taus[jc];
    if (tau == 0.f) continue;
    float v[S];
#pragma unroll
    for (int s = 0; s < S; ++s) v[s] = Vs[lane + 32 * s + jc * RS];
#pragma unroll
    for (int j = 0; j < CPW; ++j) {
      const int c = warp + j * P_NW;
      if (c < b) {
        float d0 = 0.f, d1 = 0.f;
#pragma unroll
        for (int s = 0; s < S; s += 2) {
          d0 = fmaf(v[s], x[j][s], d0);
          if (s + 1 < S) d1 = fmaf(v[s + 1], x[j][s + 1], d1);
        }
        const float d = warp_sum(d0 + d1) * tau;
#pragma unroll
        for (int s = 0; s < S; ++s) x[j][s] = fmaf(-d, v[s], x[j][s]);
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

template <int CPW, int S, int SM>
SBR_DEV void load_node(const PanelArgs& a, int lev, int k, const NodeInfo& ni, float (&x)[CPW][SM]) {
  const int lane = lane_id(), warp = warp_id(), b = a.b;
#pragma unroll
  for (int j = 0; j < CPW; ++j) {
    const int c = warp + j * P_NW;
#pragma unroll
    for (int s = 0; s < SM; ++s) {
      const int i = lane + 32 * s;
      float v = 0.f;
      if (s < S && c < b && i < ni.rows) {
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
}

template <int S>
SBR_DEV void store_v(const PanelArgs& a, int lev, int k, const NodeInfo& ni, const float* Vs, const float* taus,
                     const float* Rs) {
  constexpr int RS = 32 * S;
  const int b = a.b;
  float* vd = node_v(a, lev, k, ni);
  for (int e = threadIdx.x; e < ni.rows * b; e += blockDim.x) vd[e] = Vs[(e % ni.rows) + (e / ni.rows) * RS];
  if (threadIdx.x < b) a.ws_tau[a.toff[lev] + (int64_t)k * b + threadIdx.x] = taus[threadIdx.x];
  for (int e = threadIdx.x; e < b * b; e += blockDim.x) a.ws_r[a.roff[lev] + (int64_t)k * b * b + e] = Rs[e];
}

// x = [C; 0] with C = the node's b x b block of its parent's explicit Q (or I at the root)
template <int CPW, int SM>
SBR_DEV void load_c(const PanelArgs& a, int lev, int k, float (&x)[CPW][SM]) {
  const int lane = lane_id(), warp = warp_id(), b = a.b;
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
    const int c = warp + j * P_NW;
#pragma unroll
    for (int s = 0; s < SM; ++s) {
      const int i = lane + 32 * s;
      float v = 0.f;
      if (c < b && i < b) v = cpar ? cpar[i + (int64_t)c * ldc] : (i == c ? 1.f : 0.f);
      x[j][s] = v;
    }
  }
}

template <int CPW, int S, int SM>
SBR_DEV void store_q_ws(const PanelArgs& a, int lev, int k, const NodeInfo& ni, const float (&x)[CPW][SM]) {
  const int lane = lane_id(), warp = warp_id(), b = a.b;
#pragma unroll
  for (int j = 0; j < CPW; ++j) {
    const int c = warp + j * P_NW;
#pragma unroll
    for (int s = 0; s < S; ++s) {
      const int i = lane + 32 * s;
      if (c < b && i < ni.rows) a.ws_q[a.qoff[lev] + (int64_t)k * a.arity * b * b + i + (int64_t)c * ni.rows] = x[j][s];
    }
  }
}

template <int S>
SBR_DEV void stage_v(const PanelArgs& a, int lev, int k, const NodeInfo& ni, float* Vs, float* taus) {
  constexpr int RS = 32 * S;
  const int b = a.b;
  const float* vs = node_v(a, lev, k, ni);
  for (int e = threadIdx.x; e < RS * b; e += blockDim.x) {   // rows >= ni.rows must read 0
    const int i = e % RS, c = e / RS;
    Vs[e] = (i < ni.rows) ? vs[i + c * ni.rows] : 0.f;
  }
  if (threadIdx.x < b) taus[threadIdx.x] = a.ws_tau[a.toff[lev] + (int64_t)k * b + threadIdx.x];
  __syncthreads();
}

// modified LU of Q_1 - S (s_j = -sign(d_j)), one warp, lane c holds column c in
// registers (b <= 32).  Writes U (upper, incl. diagonal) and L (unit lower) to Us / Ls.
template <int LDU>
SBR_DEV void warp_lu32(int b, const float* Q1, int ldq, float* Us, float* Ls, float* Ss) {
  const int lane = lane_id();
  float col[32];
#pragma unroll
  for (int i = 0; i < 32; ++i) col[i] = (lane < b && i < b) ? Q1[i + lane * ldq] : 0.f;
  float sgn = 0.f;
#pragma unroll
  for (int j = 0; j < 32; ++j) {
    if (j < b) {
      const float d = __shfl_sync(0xffffffffu, col[j], j);
      const float sj = (d >= 0.f) ? -1.f : 1.f;   // s_j = -sign(d_j)
      const float piv = d - sj;
      if (lane == j) { col[j] = piv; sgn = sj; }
      const float inv = 1.f / piv;
      if (lane == j) {
#pragma unroll
        for (int i = j + 1; i < 32; ++i) col[i] *= inv;
      }
      // broadcast L[:, j] (rows > j) and update columns c > j
#pragma unroll
      for (int i = j + 1; i < 32; ++i) {
        const float lij = __shfl_sync(0xffffffffu, col[i], j);
        if (lane > j) col[i] = fmaf(-lij, col[j], col[i]);
      }
    }
  }
  if (lane < b) {
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      if (i < b) {
        Us[i + lane * LDU] = (i <= lane) ? col[i] : 0.f;
        Ls[i + lane * LDU] = (i > lane) ? col[i] : (i == lane ? 1.f : 0.f);
      }
    }
    Ss[lane] = sgn;
  }
}

template <int B, int CPW>
__global__ void __launch_bounds__(P_NW * 32, 1) panel_tsqr_kernel(PanelArgs a) {
  pdl_trigger();   // the successor may launch early; it waits (griddepcontrol.wait) before reading
  constexpr int RSL = 32 * P_SL, RSN = 32 * P_SN;
  constexpr int LDU = B + 1;                 // padded ld for the b x b factors
  extern __shared__ __align__(16) float smem[];
  float* Vs = smem;                          // RSN x B (reflectors; later the leaf's explicit Q)
  float* Rs = Vs + RSN * B;                  // B x B
  float* taus = Rs + B * B;                  // 64
  float* Us = taus + 64;                     // B x LDU : U (upper) / LU work
  float* Ls = Us + B * LDU;                  // B x LDU : L_1 (unit lower) ; T in the single-leaf path
  float* Ss = Ls + B * LDU;                  // B signs
  const int b = a.b;
  const int lane = lane_id(), warp = warp_id();
  cg::grid_group grid = cg::this_grid();
  pdl_wait();                                 // launched with PDL: predecessor complete
  if (a.run_if && *a.run_if == 0) return;    // CholeskyQR already factored this panel
  float x[CPW][P_SN];
  PTRACE(0);
  if (a.trace && blockIdx.x == 0 && threadIdx.x == 0) a.trace[10] = clock64();
  const int64_t M = a.M, row0 = a.row0;

  // ================= single node: LAPACK-exact V, T (dlarft), R; W = V T =================
  if (a.nlev == 1) {
    const NodeInfo ni = node_info(a, 0, 0);
    load_node<CPW, P_SN, P_SN>(a, 0, 0, ni, x);
    cta_qr<CPW, P_SN, P_SN>(x, ni.rows, b, Vs, Rs, taus);
    const int rows = a.m, kr = min(rows, b);
    float* G = Us;  // G[p][j] = v_p . v_j, p < j
    for (int pair = warp; pair < b * b; pair += P_NW) {
      const int p = pair % b, j = pair / b;
      if (p >= j) continue;
      float d = 0.f;
      for (int i = lane; i < rows; i += 32) d = fmaf(Vs[i + p * RSN], Vs[i + j * RSN], d);
      d = warp_sum(d);
      if (lane == 0) G[p + j * LDU] = d;
    }
    __syncthreads();
    float* T = Ls;
    for (int j = 0; j < b; ++j) {  // dlarft recurrence: T[0:j, j] = -tau_j T[0:j,0:j] G[0:j, j]
      const float tj = (j < kr) ? taus[j] : 0.f;
      if (threadIdx.x < b) {
        const int p = threadIdx.x;
        float val = (p == j) ? tj : 0.f;
        if (p < j) {
          float acc = 0.f;
          for (int q = p; q < j; ++q) acc = fmaf(T[p + q * LDU], G[q + j * LDU], acc);
          val = -tj * acc;
        }
        T[p + j * LDU] = val;
      }
      __syncthreads();
    }
    for (int64_t i = threadIdx.x; i < M; i += blockDim.x) {
      if (i < row0) {
        for (int c = 0; c < b; ++c) { a.Y[i + c * a.ldy] = 0.f; a.W[i + c * a.ldw] = 0.f; }
        if (a.Yh) for (int c = 0; c < b; ++c) a.Yh[i * a.ldyh + c] = cvt16(0.f);
        if (a.Wh) for (int c = 0; c < b; ++c) a.Wh[i + c * a.ldwh] = cvt16(0.f);
        if (a.Wrh) for (int c = 0; c < b; ++c) a.Wrh[i * a.ldwrh + c] = cvt16(0.f);
        continue;
      }
      const int64_t il = i - row0;
      for (int c = 0; c < b; ++c) {
        const float y = Vs[il + c * RSN];
        a.Y[i + c * a.ldy] = y;
        if (a.Yh) a.Yh[i * a.ldyh + c] = cvt16(y);
        a.P[il + c * a.ldp] = (il > c) ? y : (il < b ? Rs[il + c * b] : 0.f);
        float w = 0.f;
        for (int k = 0; k <= c; ++k) w = fmaf(Vs[il + k * RSN], T[k + c * LDU], w);
        a.W[i + c * a.ldw] = w;
        if (a.Wh) a.Wh[i + c * a.ldwh] = cvt16(w);
        if (a.Wrh) a.Wrh[i * a.ldwrh + c] = cvt16(w);
      }
    }
    return;
  }

  // ================= up sweep =================
  const int top = a.nlev - 1;
  for (int lev = 0; lev < top; ++lev) {
    const int k = blockIdx.x;
    if (k < a.nodes[lev]) {
      const NodeInfo ni = node_info(a, lev, k);
      if (lev == 0) {
        load_node<CPW, P_SL, P_SN>(a, lev, k, ni, x);
        cta_qr<CPW, P_SL, P_SN>(x, ni.rows, b, Vs, Rs, taus, a.trace ? (long long*)(a.trace + 12) : nullptr);
        PTRACE(1);
        if (a.trace && blockIdx.x == 0 && threadIdx.x == 0) a.trace[11] = clock64();
        store_v<P_SL>(a, lev, k, ni, Vs, taus, Rs);
      } else {
        load_node<CPW, P_SN, P_SN>(a, lev, k, ni, x);
        cta_qr<CPW, P_SN, P_SN>(x, ni.rows, b, Vs, Rs, taus);
        store_v<P_SN>(a, lev, k, ni, Vs, taus, Rs);
      }
    }
    grid.sync();
    if (lev == 0) PTRACE(2);
  }
  // root: QR and explicit Q = H_root [I; 0] in the same CTA
  if (blockIdx.x == 0) {
    const NodeInfo ni = node_info(a, top, 0);
    load_node<CPW, P_SN, P_SN>(a, top, 0, ni, x);
    cta_qr<CPW, P_SN, P_SN>(x, ni.rows, b, Vs, Rs, taus);
    PTRACE(3);
    for (int e = threadIdx.x; e < b * b; e += blockDim.x) a.ws_r[a.roff[top] + e] = Rs[e];
    load_c<CPW, P_SN>(a, top, 0, x);
    cta_apply_q<CPW, P_SN, P_SN>(x, min(ni.rows, b), b, Vs, taus);
    store_q_ws<CPW, P_SN, P_SN>(a, top, 0, ni, x);
    PTRACE(4);
  }
  grid.sync();
  PTRACE(5);
  // ================= down sweep =================
  for (int lev = top - 1; lev >= 1; --lev) {
    const int k = blockIdx.x;
    if (k < a.nodes[lev]) {
      const NodeInfo ni = node_info(a, lev, k);
      stage_v<P_SN>(a, lev, k, ni, Vs, taus);
      load_c<CPW, P_SN>(a, lev, k, x);
      cta_apply_q<CPW, P_SN, P_SN>(x, min(ni.rows, b), b, Vs, taus);
      store_q_ws<CPW, P_SN, P_SN>(a, lev, k, ni, x);
    }
    grid.sync();
  }
  const NodeInfo ni = node_info(a, 0, blockIdx.x);   // this CTA's leaf
  stage_v<P_SL>(a, 0, blockIdx.x, ni, Vs, taus);
  load_c<CPW, P_SN>(a, 0, blockIdx.x, x);
  cta_apply_q<CPW, P_SL, P_SN>(x, min(ni.rows, b), b, Vs, taus);
  __syncthreads();
#pragma unroll
  for (int j = 0; j < CPW; ++j) {   // leaf: keep Q in smem (Vs, ld RSL) for the row phase
    const int c = warp + j * P_NW;
#pragma unroll
    for (int s = 0; s < P_SL; ++s)
      if (c < b) Vs[lane + 32 * s + c * RSL] = x[j][s];
  }
  __syncthreads();
  PTRACE(6);
  // ================= reconstruction: modified LU of Q_1 - S (CTA 0) =================
  if (blockIdx.x == 0) {
    if (B <= 32) {
      if (warp == 0) warp_lu32<LDU>(b, Vs, RSL, Us, Ls, Ss);
    } else if (warp == 0) {            // b > 32: column-per-lane LU through shared memory
      for (int e = lane; e < b * b; e += 32) Us[(e % b) + (e / b) * LDU] = Vs[(e % b) + (e / b) * RSL];
      __syncwarp();
      for (int j = 0; j < b; ++j) {
        const float d = Us[j + j * LDU];
        const float sj = (d >= 0.f) ? -1.f : 1.f;
        const float piv = d - sj;
        __syncwarp();
        if (lane == 0) { Us[j + j * LDU] = piv; Ss[j] = sj; }
        for (int i = j + 1 + lane; i < b; i += 32) Us[i + j * LDU] /= piv;
        __syncwarp();
        for (int c = j + 1 + lane; c < b; c += 32) {
          const float ujc = Us[j + c * LDU];
          for (int i = j + 1; i < b; ++i) Us[i + c * LDU] = fmaf(-Us[i + j * LDU], ujc, Us[i + c * LDU]);
        }
        __syncwarp();
      }
      for (int e = lane; e < b * b; e += 32) {
        const int i = e % b, c = e / b;
        Ls[i + c * LDU] = (i > c) ? Us[i + c * LDU] : (i == c ? 1.f : 0.f);
        if (i > c) Us[i + c * LDU] = 0.f;
      }
    }
    __syncthreads();
    for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
      const int i = e % b, c = e / b;
      a.ws_misc[e] = Us[i + c * LDU];
      a.ws_misc[b * b + e] = Ls[i + c * LDU];
    }
    if (threadIdx.x < b) a.ws_misc[2 * b * b + threadIdx.x] = Ss[threadIdx.x];
  }
  PTRACE(7);
  grid.sync();
  PTRACE(8);
  // ================= rows of this leaf: y U = q (rows >= b), w L^T = (E - q S) =================
  if (blockIdx.x != 0) {
    for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
      const int i = e % b, c = e / b;
      Us[i + c * LDU] = a.ws_misc[e];
      Ls[i + c * LDU] = a.ws_misc[b * b + e];
    }
    if (threadIdx.x < b) Ss[threadIdx.x] = a.ws_misc[2 * b * b + threadIdx.x];
    __syncthreads();
  }
  const float* rroot = a.ws_r + a.roff[top];
  for (int il_local = threadIdx.x; il_local < ni.rows; il_local += blockDim.x) {
    const int64_t il = ni.start + il_local;           // panel row
    const int64_t gr = row0 + il;
    const float* qrow = Vs + il_local;                 // q_c = qrow[c * RSL]
    float v_[B];
    // w L_1^T = (e_il if il < b) - q S   (forward substitution, L_1 unit lower)
#pragma unroll
    for (int c = 0; c < B; ++c) {
      if (c < b) {
        float v = ((il == c) ? 1.f : 0.f) - qrow[c * RSL] * Ss[c];
#pragma unroll
        for (int k = 0; k < c; ++k) v = fmaf(-v_[k], Ls[c + k * LDU], v);
        v_[c] = v;
      } else {
        v_[c] = 0.f;
      }
    }
#pragma unroll
    for (int c = 0; c < B; ++c)
      if (c < b) {
        a.W[gr + c * a.ldw] = v_[c];
        if (a.Wh) a.Wh[gr + c * a.ldwh] = cvt16(v_[c]);
        if (a.Wrh) a.Wrh[gr * a.ldwrh + c] = cvt16(v_[c]);
      }
    // y = L_1 row (il < b)  or  y U = q
#pragma unroll
    for (int c = 0; c < B; ++c) {
      if (c < b) {
        if (il < b) {
          v_[c] = Ls[il + c * LDU];
        } else {
          float v = qrow[c * RSL];
#pragma unroll
          for (int k = 0; k < c; ++k) v = fmaf(-v_[k], Us[k + c * LDU], v);
          v_[c] = v / Us[c + c * LDU];
        }
      } else {
        v_[c] = 0.f;
      }
    }
#pragma unroll
    for (int c = 0; c < B; ++c) {
      if (c < b) {
        a.Y[gr + c * a.ldy] = v_[c];
        a.P[il + (int64_t)c * a.ldp] = (il > c) ? v_[c] : (Ss[il] * rroot[il + c * b]);   // il < b here
        if (a.Yh) a.Yh[gr * a.ldyh + c] = cvt16(v_[c]);
      }
    }
  }
  // rows above the panel: zero Y and W (and Yh)
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t nth = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid; i < row0; i += nth) {
    for (int c = 0; c < b; ++c) { a.Y[i + c * a.ldy] = 0.f; a.W[i + c * a.ldw] = 0.f; }
    if (a.Yh) for (int c = 0; c < b; ++c) a.Yh[i * a.ldyh + c] = cvt16(0.f);
    if (a.Wh) for (int c = 0; c < b; ++c) a.Wh[i + c * a.ldwh] = cvt16(0.f);
    if (a.Wrh) for (int c = 0; c < b; ++c) a.Wrh[i * a.ldwrh + c] = cvt16(0.f);
  }
  PTRACE(9);
}

// ---------------------------------------------------------------- host side
template <int B>
static constexpr size_t panel_smem() {
  return sizeof(float) * (32 * P_SN * B + B * B + 64 + 2 * B * (B + 1) + B);
}

template <int B, int CPW>
static cudaError_t launch_panel_t(PanelArgs& a, int max_ctas, cudaStream_t st) {
  constexpr size_t smem = panel_smem<B>();
  auto kern = panel_tsqr_kernel<B, CPW>;
  {
    cudaError_t e = func_attr((const void*)kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
  }
  constexpr int capN = 32 * P_SN, capL = 32 * P_SL;
  const int L = (a.m <= capN) ? 1 : (a.m + capL - 1) / capL;   // 1: single node, direct QR
  a.over_capacity = 0;
  if (L > max_ctas) {   // one CTA per leaf must be co-resident: reported through over_capacity
    a.over_capacity = 1;
    return cudaSuccess;
  }
  a.arity = std::max(2, capN / a.b);
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
  cudaLaunchConfig_t cfg = {};   // cooperative + programmatic dependent launch (see k_panel_chol.cu)
  cfg.gridDim = dim3(L);
  cfg.blockDim = dim3(P_NW * 32);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = 1;
  at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl_enabled() ? 2 : 1;
  return cudaLaunchKernelEx(&cfg, kern, a);
}

cudaError_t launch_panel(PanelArgs& a, int max_ctas, cudaStream_t st) {
  if (a.b <= 16) return launch_panel_t<16, 1>(a, max_ctas, st);
  if (a.b <= 32) return launch_panel_t<32, 1>(a, max_ctas, st);
  return launch_panel_t<64, 2>(a, max_ctas, st);
}

PanelWs panel_ws_sizes(int64_t m_max, int b) {
  const int64_t nodes = 2 * (m_max / 128 + 2) + 2;
  const int64_t node_floats = 512 * 64;  // inner node rows x b bound (rows <= 512)
  PanelWs w;
  w.v = (size_t)(m_max * b + nodes * node_floats + 4096);
  w.q = (size_t)(nodes * node_floats + 4096);
  w.r = (size_t)(nodes * b * b + 4096);
  w.tau = (size_t)(nodes * b + 256);
  w.misc = (size_t)(2 * 64 * 64 + 256);
  return w;
}

int panel_max_ctas(int b) {
  const int nsm = current_device_sms();
  const void* k;
  size_t smem;
  if (b <= 16) { k = (const void*)panel_tsqr_kernel<16, 1>; smem = panel_smem<16>(); }
  else if (b <= 32) { k = (const void*)panel_tsqr_kernel<32, 1>; smem = panel_smem<32>(); }
  else { k = (const void*)panel_tsqr_kernel<64, 2>; smem = panel_smem<64>(); }
  func_attr(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  const int per = func_blocks_per_sm(k, P_NW * 32, smem);
  return std::max(1, per) * nsm;
}

SBR_OP16_SETTER(panel)

}  // namespace sbr
