// k_panel_chol.cu -- panel QR by shifted CholeskyQR in fp64 + the paper's Householder
// reconstruction (steps a1, a2), the B200 fast path for tall panels.
//
// Why not only TSQR: on sm_100a the TSQR tree is latency-bound -- every tree
// level is b dependent Householder column steps in one CTA -- while fp64 SIMT throughput
// is ample.  Shifted CholeskyQR3 (Fukaya, Kannan, Nakatsukasa, Yamamoto, Yanagisawa 2020)
// needs grid-wide Gram reductions only and keeps all SMs busy:
//     G1 = P^T P + s I, R1 = chol(G1), Q1 = P R1^-1   (s = 11 (m b + b(b+1)) u ||P||_F^2)
//     G2 = Q1^T Q1,     R2 = chol(G2), Q2 = Q1 R2^-1
//     G3 = Q2^T Q2,     R3 = chol(G3), Q  = Q2 R3^-1,  R = R3 R2 R1
// in fp64 (u = 2^-53; panel data fp32), stable for cond(P) up to ~1e12.  A round k >= 2 is
// skipped once G_k = I to 1e-12 (Q is orthonormal to fp64 accuracy).  A panel whose
// second-round Cholesky signals (numerical) rank deficiency is left untouched and a flag
// makes the TSQR kernel (k_panel.cu), launched right after, factor it instead.
// The explicit Q then goes through the same reconstruction as TSQR's (Alg. 3 + S,
// P:315-339; reading C7): Q_1 - S = L U, Y = [L; Q_2 U^-1], W = (E - Q S) L^-T,
// R_h = S R.  The result is the LAPACK dgeqrf (V, T, R) of the panel.
// Latency design: every b x b factorisation is one warp with its columns in registers
// (fully unrolled, row broadcasts through shared memory); every triangular solve is
// right-looking so its dependency chain is b steps, not b^2/2.
#include <cooperative_groups.h>

#include "common.cuh"
#include "kernels.h"

namespace cg = cooperative_groups;

namespace sbr {

constexpr int PC_THREADS = 256;
constexpr int PC_NCOPY = 8;   // Gram accumulated into 8 copies (CTA k -> k % 8): less atomic contention
template <int B> constexpr int pc_maxr() { return B <= 32 ? 512 : 160; }   // rows per CTA
template <int B> constexpr int pc_ngrp() { return PC_THREADS / ((B / 4) * (B / 4)) > 0 ? PC_THREADS / ((B / 4) * (B / 4)) : 1; }

template <int B>
struct CholSmem {
  static constexpr int LDG = B + 1;
  static constexpr size_t OFF_Q = 0;                                            // double rows x B
  static constexpr size_t OFF_GP = OFF_Q + sizeof(double) * pc_maxr<B>() * B;  // double NGRP x B x B
  static constexpr size_t OFF_G = OFF_GP + sizeof(double) * (pc_ngrp<B>() > 2 ? pc_ngrp<B>() : 2) * B * B;   // double B x LDG
  static constexpr size_t OFF_RD = OFF_G + sizeof(double) * B * LDG;           // double B
  static constexpr size_t OFF_RR = OFF_RD + sizeof(double) * B;                // double B (row broadcast)
  static constexpr size_t OFF_U = OFF_RR + sizeof(double) * B;                 // float B x LDG
  static constexpr size_t OFF_L = OFF_U + sizeof(float) * B * LDG;             // float B x LDG
  static constexpr size_t OFF_S = OFF_L + sizeof(float) * B * LDG;             // float B (signs)
  static constexpr size_t OFF_LR = OFF_S + sizeof(float) * B;                  // float B (row broadcast)
  static constexpr size_t BYTES = OFF_LR + sizeof(float) * B + 64;
};

// In-place Cholesky (CTA, one barrier per column) -- used for b > 32.
template <int LDG>
SBR_DEV bool cta_chol(double* G, double* rd, int b, double floor_rel) {
  double dmax = 0.0;
  for (int i = 0; i < b; ++i) dmax = fmax(dmax, G[i + i * LDG]);
  bool ok = true;
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5, ny = blockDim.x >> 5;
  for (int j = 0; j < b; ++j) {
    const double gjj = G[j + j * LDG];
    if (!(gjj > floor_rel * dmax)) ok = false;
    const double inv = __drcp_rn(fmax(gjj, 1e-300));
    for (int c = j + 1 + tx; c < b; c += 32) {
      const double gjc = G[j + c * LDG] * inv;
      for (int i = j + 1 + ty; i <= c; i += ny) G[i + c * LDG] = fma(-G[j + i * LDG], gjc, G[i + c * LDG]);
    }
    __syncthreads();
  }
  for (int i = threadIdx.x; i < b; i += blockDim.x) rd[i] = rsqrt(fmax(G[i + i * LDG], 1e-300));
  __syncthreads();
  for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
    const int i = e % b, c = e / b;
    G[i + c * LDG] = (i <= c) ? G[i + c * LDG] * rd[i] : 0.0;
  }
  __syncthreads();
  return ok;
}

// Cholesky G = R^T R of a b x b (b <= 32) fp64 matrix by ONE warp: lane c holds column c
// in registers, R row j is broadcast through rrow.  G (upper) -> R (upper) in place, rd = 1/diag.
template <int LDG>
SBR_DEV bool warp_chol32(double* G, double* rd, double* rrow, int b, double floor_rel) {
  const int lane = lane_id();
  double g[32];
#pragma unroll
  for (int i = 0; i < 32; ++i) g[i] = (lane < b && i <= lane) ? G[i + lane * LDG] : 0.0;
  double dmax = (lane < b) ? G[lane + lane * LDG] : 0.0;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) dmax = fmax(dmax, __shfl_xor_sync(0xffffffffu, dmax, o));
  bool ok = true;
#pragma unroll
  for (int j = 0; j < 32; ++j) {
    if (j < b) {
      const double gjj = __shfl_sync(0xffffffffu, g[j], j);
      if (!(gjj > floor_rel * dmax)) ok = false;
      const double rjj = sqrt(fmax(gjj, 1e-300));
      const double rjc = (lane == j) ? rjj : g[j] * __drcp_rn(rjj);
      if (lane >= j) g[j] = rjc;
      rrow[lane] = (lane > j && lane < b) ? rjc : 0.0;
      __syncwarp();
#pragma unroll
      for (int i = j + 1; i < 32; ++i) {
        const double rji = rrow[i];
        if (lane >= i) g[i] = fma(-rji, rjc, g[i]);
      }
      __syncwarp();
    }
  }
  if (lane < b) {
#pragma unroll
    for (int i = 0; i < 32; ++i)
      if (i < b) G[i + lane * LDG] = (i <= lane) ? g[i] : 0.0;
  }
  __syncwarp();
  if (lane < b) rd[lane] = 1.0 / G[lane + lane * LDG];
  __syncwarp();
  return __all_sync(0xffffffffu, ok);
}

// Modified LU of Q_1 - S (s_j = -sign(d_j)) of a b x b (b <= 32) fp32 matrix by ONE
// warp: lane c holds column c; the L column is broadcast through lrow.  Writes U (with the
// pivots on its diagonal), L (unit lower) and the signs.
template <int LDG>
SBR_DEV void warp_lu32(int b, const double* Q1, int ldq_row, float* Us, float* Ls, float* Ss, float* lrow) {
  const int lane = lane_id();
  float col[32];
#pragma unroll
  for (int i = 0; i < 32; ++i) col[i] = (lane < b && i < b) ? (float)Q1[i * ldq_row + lane] : 0.f;
#pragma unroll
  for (int j = 0; j < 32; ++j) {
    if (j < b) {
      const float d = __shfl_sync(0xffffffffu, col[j], j);
      const float sj = (d >= 0.f) ? -1.f : 1.f;
      const float piv = d - sj;
      const float inv = __frcp_rn(piv);
      if (lane == j) {
        col[j] = piv;
#pragma unroll
        for (int i = j + 1; i < 32; ++i) { col[i] *= inv; lrow[i] = col[i]; }
        Ss[j] = sj;
      }
      __syncwarp();
      if (lane > j) {
        const float ujc = col[j];
#pragma unroll
        for (int i = j + 1; i < 32; ++i) col[i] = fmaf(-lrow[i], ujc, col[i]);
      }
      __syncwarp();
    }
  }
  if (lane < b) {
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      if (i < b) {
        Us[i + lane * LDG] = (i <= lane) ? col[i] : 0.f;
        Ls[i + lane * LDG] = (i > lane) ? col[i] : (i == lane ? 1.f : 0.f);
      }
    }
  }
}

// Same by the whole CTA (one barrier per column) -- used for b > 32.
template <int LDG>
SBR_DEV void cta_lu(int b, const double* Q1, int ldq_row, float* Us, float* Ls, float* Ss) {
  for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
    const int i = e % b, c = e / b;
    Us[i + c * LDG] = (float)Q1[i * ldq_row + c];
  }
  __syncthreads();
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5, ny = blockDim.x >> 5;
  for (int j = 0; j < b; ++j) {
    const float d = Us[j + j * LDG];
    const float sj = (d >= 0.f) ? -1.f : 1.f;
    const float invp = __frcp_rn(d - sj);
    for (int c = j + 1 + tx; c < b; c += 32) {
      const float ujc = Us[j + c * LDG] * invp;
      for (int i = j + 1 + ty; i < b; i += ny) Us[i + c * LDG] = fmaf(-Us[i + j * LDG], ujc, Us[i + c * LDG]);
    }
    __syncthreads();
    for (int i = j + 1 + threadIdx.x; i < b; i += blockDim.x) Ls[i + j * LDG] = Us[i + j * LDG] * invp;
    if (threadIdx.x == 0) { Ss[j] = sj; Us[j + j * LDG] = d - sj; }
    __syncthreads();
  }
  for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
    const int i = e % b, c = e / b;
    if (i > c) Us[i + c * LDG] = 0.f;
    else Ls[i + c * LDG] = (i == c) ? 1.f : 0.f;
  }
  __syncthreads();
}

template <int B>
__global__ void __launch_bounds__(PC_THREADS, 1) panel_chol_kernel(PanelArgs a, double* gram, int* fail) {
  using L = CholSmem<B>;
  constexpr int LDG = L::LDG;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  double* Qd = reinterpret_cast<double*>(smem_raw + L::OFF_Q);     // rows x B, row-major, fp64
  double* Gpart = reinterpret_cast<double*>(smem_raw + L::OFF_GP);
  double* Gk = reinterpret_cast<double*>(smem_raw + L::OFF_G);
  double* rd = reinterpret_cast<double*>(smem_raw + L::OFF_RD);
  double* rrow = reinterpret_cast<double*>(smem_raw + L::OFF_RR);
  float* Us = reinterpret_cast<float*>(smem_raw + L::OFF_U);
  float* Ls = reinterpret_cast<float*>(smem_raw + L::OFF_L);
  float* Ss = reinterpret_cast<float*>(smem_raw + L::OFF_S);
  float* lrow = reinterpret_cast<float*>(smem_raw + L::OFF_LR);
  double* Rstore = gram + 3 * PC_NCOPY * B * B;                    // R_1, R_2, R_3 (global)
  cg::grid_group grid = cg::this_grid();
  const int b = a.b;
  const int warp = warp_id(), lane = lane_id();
  const int64_t m = a.m;
  const int64_t r_beg = (int64_t)blockIdx.x * m / gridDim.x, r_end = (int64_t)(blockIdx.x + 1) * m / gridDim.x;
  const int rows = (int)(r_end - r_beg);
  auto stamp = [&](int k) {
    if (a.trace && blockIdx.x == 0 && threadIdx.x == 0) {
      int64_t t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      a.trace[k] = t;
    }
  };
  stamp(0);
  // ---- load the CTA's rows: warp w -> columns w, w+8, ..; lane -> rows (coalesced, unrolled)
  for (int c = warp; c < B; c += PC_THREADS / 32) {
    const float* src = a.P + r_beg + (int64_t)c * a.ldp;
#pragma unroll 4
    for (int r = lane; r < pc_maxr<B>(); r += 32)
      if (r < rows) Qd[r * B + c] = (c < b) ? (double)src[r] : 0.0;
  }
  __syncthreads();
  stamp(4);

  int nrounds = 3;
  for (int round = 0; round < nrounds; ++round) {
    double* Gg = gram + (size_t)round * PC_NCOPY * B * B;   // PC_NCOPY copies
    // ---- partial Gram of this CTA's rows: 4x4 register tiles, reduced over the row
    //      groups in smem, then fp64 reductions of the upper triangle into Gg
    {
      constexpr int TPB = B / 4, NTILE = TPB * TPB, NGRP = pc_ngrp<B>();
      const int grp = threadIdx.x / NTILE, tl = threadIdx.x % NTILE;
      const int ti = tl / TPB, tj = tl % TPB;
      double acc[4][4];
#pragma unroll
      for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4; ++v) acc[u][v] = 0.0;
      if (grp < NGRP && ti <= tj) {
#pragma unroll 2
        for (int r = grp; r < rows; r += NGRP) {
          const double2 a0 = *reinterpret_cast<const double2*>(Qd + r * B + 4 * ti);
          const double2 a1 = *reinterpret_cast<const double2*>(Qd + r * B + 4 * ti + 2);
          const double2 b0 = *reinterpret_cast<const double2*>(Qd + r * B + 4 * tj);
          const double2 b1 = *reinterpret_cast<const double2*>(Qd + r * B + 4 * tj + 2);
          const double aa[4] = {a0.x, a0.y, a1.x, a1.y};
          const double bb[4] = {b0.x, b0.y, b1.x, b1.y};
#pragma unroll
          for (int u = 0; u < 4; ++u)
#pragma unroll
            for (int v = 0; v < 4; ++v) acc[u][v] = fma(aa[u], bb[v], acc[u][v]);
        }
      }
      if (grp < NGRP) {
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
          for (int v = 0; v < 4; ++v) Gpart[grp * B * B + (4 * ti + u) + (4 * tj + v) * B] = acc[u][v];
      }
      __syncthreads();
      if (round == 0) stamp(8);
      for (int e = threadIdx.x; e < B * B; e += blockDim.x) {
        const int p = e % B, q = e / B;
        if (p <= q && q < b) {
          double sum = 0.0;
#pragma unroll
          for (int g = 0; g < NGRP; ++g) sum += Gpart[g * B * B + e];
          atomicAdd(&Gg[(blockIdx.x % PC_NCOPY) * B * B + p + q * B], sum);
        }
      }
    }
    stamp(1 + 4 * round);
    grid.sync();
    stamp(2 + 4 * round);
    // ---- Cholesky (redundantly in every CTA; identical input -> identical R)
    for (int e = threadIdx.x; e < B * B; e += blockDim.x) {
      const int i = e % B, c = e / B;
      double g = 0.0;
      if (i < b && c < b && i <= c)
#pragma unroll
        for (int k = 0; k < PC_NCOPY; ++k) g += Gg[k * B * B + i + c * B];
      Gk[i + c * LDG] = g;
    }
    __syncthreads();
    if (round == 0) {                          // shift s = 11 (m b + b(b+1)) u ||P||_F^2
      double tr = 0.0;
      for (int i = 0; i < b; ++i) tr += Gk[i + i * LDG];
      const double sh = 11.0 * ((double)m * b + (double)b * (b + 1)) * 1.1102230246251565e-16 * tr;
      __syncthreads();
      if (threadIdx.x < b) Gk[threadIdx.x * (LDG + 1)] += (sh > 0.0 ? sh : 1e-300);
      __syncthreads();
    } else {                                   // Q orthonormal to fp64 accuracy already: done
      double dev = 0.0;
      for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
        const int i = e % b, c = e / b;
        if (i <= c) dev = fmax(dev, fabs(Gk[i + c * LDG] - (i == c ? 1.0 : 0.0)));
      }
      const int big = __syncthreads_or(dev > 1e-12);
      if (!big) {
        if (blockIdx.x == 0)
          for (int rr = round; rr < 3; ++rr)
            for (int e = threadIdx.x; e < B * B; e += blockDim.x) Rstore[rr * B * B + e] = (e % B == e / B) ? 1.0 : 0.0;
        nrounds = round;
        break;
      }
    }
    bool ok;
    if constexpr (B <= 32) {
      __shared__ int okflag;
      if (warp == 0) {
        const bool w = warp_chol32<LDG>(Gk, rd, rrow, b, round == 0 ? 0.0 : 1e-12);
        if (lane == 0) okflag = w ? 1 : 0;
      }
      __syncthreads();
      ok = okflag != 0;
    } else {
      ok = cta_chol<LDG>(Gk, rd, b, round == 0 ? 0.0 : 1e-12);
    }
    stamp(3 + 4 * round);
    if (!ok) {                                 // rank deficient: leave the panel to TSQR
      if (blockIdx.x == 0 && threadIdx.x == 0) *fail = 1;
      return;
    }
    if (blockIdx.x == 0)
      for (int e = threadIdx.x; e < B * B; e += blockDim.x) {
        const int i = e % B, c = e / B;
        Rstore[round * B * B + e] = (i < b && c < b) ? Gk[i + c * LDG] : 0.0;
      }
    // ---- Q <- Q R_k^-1: thread per row, right-looking forward substitution (chain b)
    for (int r = threadIdx.x; r < rows; r += blockDim.x) {
      double q[B];
#pragma unroll
      for (int c = 0; c < B; ++c) q[c] = Qd[r * B + c];
#pragma unroll
      for (int c = 0; c < B; ++c) {
        if (c < b) {
          q[c] *= rd[c];
#pragma unroll
          for (int c2 = c + 1; c2 < B; ++c2)
            if (c2 < b) q[c2] = fma(-q[c], Gk[c + c2 * LDG], q[c2]);
        }
      }
#pragma unroll
      for (int c = 0; c < B; ++c) Qd[r * B + c] = (c < b) ? q[c] : 0.0;
    }
    __syncthreads();
  }
  stamp(13);
  // ---- reconstruction: LU of Q_1 - S by CTA 0 (holds Q's top b rows), published to all
  if (blockIdx.x == 0) {
    if (threadIdx.x == 0) *fail = 0;
    if constexpr (B <= 32) {
      if (warp == 0) warp_lu32<LDG>(b, Qd, B, Us, Ls, Ss, lrow);
      __syncthreads();
    } else {
      cta_lu<LDG>(b, Qd, B, Us, Ls, Ss);
    }
    stamp(12);
    for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
      const int i = e % b, c = e / b;
      a.ws_misc[e] = Us[i + c * LDG];
      a.ws_misc[b * b + e] = Ls[i + c * LDG];
    }
    if (threadIdx.x < b) a.ws_misc[2 * b * b + threadIdx.x] = Ss[threadIdx.x];
    // R = R_3 R_2 R_1 for the compact panel (rows < b): copy to smem, two triangular products
    double* R1 = Gpart;
    double* R2 = Gpart + B * B;
    double* R3 = Gk;   // ld B here
    for (int e = threadIdx.x; e < B * B; e += blockDim.x) {
      R1[e] = Rstore[e];
      R2[e] = Rstore[B * B + e];
      R3[e] = Rstore[2 * B * B + e];
    }
    __syncthreads();
    double t4[(B * B + PC_THREADS - 1) / PC_THREADS];
    for (int k = 0; k < (B * B + PC_THREADS - 1) / PC_THREADS; ++k) t4[k] = 0.0;
    int kk = 0;
    for (int e = threadIdx.x; e < b * b; e += blockDim.x, ++kk) {   // T = R2 R1
      const int i = e % b, c = e / b;
      double acc = 0.0;
      for (int k = i; k <= c; ++k) acc = fma(R2[i + k * B], R1[k + c * B], acc);
      t4[kk] = (i <= c) ? acc : 0.0;
    }
    __syncthreads();
    kk = 0;
    for (int e = threadIdx.x; e < b * b; e += blockDim.x, ++kk) R2[(e % b) + (e / b) * B] = t4[kk];
    __syncthreads();
    kk = 0;
    for (int e = threadIdx.x; e < b * b; e += blockDim.x, ++kk) {   // R = R3 T
      const int i = e % b, c = e / b;
      double acc = 0.0;
      for (int k = i; k <= c; ++k) acc = fma(R3[i + k * B], R2[k + c * B], acc);
      t4[kk] = (i <= c) ? acc : 0.0;
    }
    __syncthreads();
    kk = 0;
    for (int e = threadIdx.x; e < b * b; e += blockDim.x, ++kk) R1[(e % b) + (e / b) * B] = t4[kk];
    __syncthreads();
  }
  stamp(14);
  grid.sync();
  stamp(15);
  if (blockIdx.x != 0) {
    for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
      const int i = e % b, c = e / b;
      Us[i + c * LDG] = a.ws_misc[e];
      Ls[i + c * LDG] = a.ws_misc[b * b + e];
    }
    if (threadIdx.x < b) Ss[threadIdx.x] = a.ws_misc[2 * b * b + threadIdx.x];
    __syncthreads();
  }
  const double* Rfin = Gpart;   // CTA 0 only (ld B)
  // ---- rows (right-looking solves): w L_1^T = (e_il) - q S ;  y = L_1 row (il < b) or y U = q
  const int64_t row0 = a.row0;
  for (int r = threadIdx.x; r < rows; r += blockDim.x) {
    const int64_t il = r_beg + r;
    const int64_t gr = row0 + il;
    float v_[B];
#pragma unroll
    for (int c = 0; c < B; ++c) v_[c] = (c < b) ? ((il == c) ? 1.f : 0.f) - (float)Qd[r * B + c] * Ss[c] : 0.f;
#pragma unroll
    for (int k = 0; k < B; ++k) {
      if (k < b) {
#pragma unroll
        for (int c = k + 1; c < B; ++c)
          if (c < b) v_[c] = fmaf(-v_[k], Ls[c + k * LDG], v_[c]);
      }
    }
#pragma unroll
    for (int c = 0; c < B; ++c)
      if (c < b) a.W[gr + c * a.ldw] = v_[c];
    if (il < b) {
#pragma unroll
      for (int c = 0; c < B; ++c) v_[c] = (c < b) ? Ls[il + c * LDG] : 0.f;
    } else {
#pragma unroll
      for (int c = 0; c < B; ++c) v_[c] = (c < b) ? (float)Qd[r * B + c] : 0.f;
#pragma unroll
      for (int k = 0; k < B; ++k) {
        if (k < b) {
          v_[k] = v_[k] / Us[k + k * LDG];
#pragma unroll
          for (int c = k + 1; c < B; ++c)
            if (c < b) v_[c] = fmaf(-v_[k], Us[k + c * LDG], v_[c]);
        }
      }
    }
#pragma unroll
    for (int c = 0; c < B; ++c) {
      if (c < b) {
        a.Y[gr + c * a.ldy] = v_[c];
        // compact panel: Y tail strictly below, R_h = S R on and above the diagonal (CTA 0)
        a.P[il + (int64_t)c * a.ldp] = (il > c) ? v_[c] : (float)((double)Ss[il] * Rfin[il + c * B]);
        if (a.Yh) a.Yh[gr * a.ldyh + c] = __float2half_rn(v_[c]);
      }
    }
  }
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t nth = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid; i < row0; i += nth) {
    for (int c = 0; c < b; ++c) { a.Y[i + c * a.ldy] = 0.f; a.W[i + c * a.ldw] = 0.f; }
    if (a.Yh) for (int c = 0; c < b; ++c) a.Yh[i * a.ldyh + c] = __float2half_rn(0.f);
  }
}

template <int B>
static cudaError_t launch_chol_t(PanelArgs& a, double* gram, int* fail, cudaStream_t st) {
  auto kern = panel_chol_kernel<B>;
  constexpr size_t smem = CholSmem<B>::BYTES;
  static int per_sm = -1;
  if (per_sm < 0) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, PC_THREADS, smem);
    if (per_sm < 1) per_sm = 1;
  }
  int nsm = 0, dev = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  const int cap = per_sm * nsm;
  int G = (int)std::min<int64_t>(cap, (a.m + 127) / 128);
  if ((int64_t)G * pc_maxr<B>() < a.m) G = (int)((a.m + pc_maxr<B>() - 1) / pc_maxr<B>());
  if (G > cap) return cudaErrorNotSupported;   // too tall for one pass: caller uses TSQR
  cudaError_t e = cudaMemsetAsync(gram, 0, sizeof(double) * 3 * PC_NCOPY * B * B, st);
  if (e != cudaSuccess) return e;
  void* args[] = {&a, &gram, &fail};
  return cudaLaunchCooperativeKernel((const void*)kern, dim3(G), dim3(PC_THREADS), args, smem, st);
}

cudaError_t launch_panel_chol(PanelArgs& a, int max_ctas, double* gram, int* fail, cudaStream_t st) {
  (void)max_ctas;
  if (a.b <= 32) return launch_chol_t<32>(a, gram, fail, st);
  return launch_chol_t<64>(a, gram, fail, st);
}

}  // namespace sbr
