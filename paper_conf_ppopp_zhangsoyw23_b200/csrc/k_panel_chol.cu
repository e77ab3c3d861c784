// k_panel_chol.cu -- panel QR by CholeskyQR in fp64 + the paper's Householder
// reconstruction (steps a1, a2), the B200 fast path for tall panels.
//
// Why not only TSQR: on sm_100a the TSQR tree is latency-bound -- every tree
// level is b dependent Householder column steps in one CTA -- while fp64 SIMT throughput
// is ample.  CholeskyQR needs only grid-wide Gram reductions and keeps all SMs busy:
//     round 0:  G = P^T P,  R_0 = chol(G),  Q = P R_0^-1
//     round k:  G = Q^T Q;  if max|G - I| <= 1e-9 stop, else R_k = chol(G), Q <- Q R_k^-1
//     R = R_k ... R_1 R_0
// in fp64 (panel data fp32).  The a-posteriori test G = Q^T Q ~ I (to 1e-9, far below the
// fp32 outputs' rounding) makes the result as good as TSQR's whenever it is accepted; one
// round suffices for cond(P) up to ~1e3, two up to ~1e7 (CholeskyQR2).  A panel whose
// Cholesky breaks down (numerical rank deficiency) or that is still not orthonormal after
// three rounds is left untouched and a flag makes the TSQR kernel (k_panel.cu), launched
// right after, factor it instead.
// The explicit Q then goes through the same reconstruction as TSQR's (Alg. 3 + S,
// P:315-339; reading C7): Q_1 - S = L U, Y = [L; Q_2 U^-1], W = (E - Q S) L^-T,
// R_h = S R.  The result is the LAPACK dgeqrf (V, T, R) of the panel.
//
// Latency design (the panel is on the critical path of every b columns):
//  * one CTA per SM, rows of the panel resident in shared memory in fp64 for all rounds;
//  * Gram matrices reduced by fp64 atomics into PC_NCOPY copies, then a hand-rolled split
//    grid barrier (arrive / wait) so CTA 0 can run the LU of Q_1 - S speculatively between
//    its arrive and its wait -- the LU overlaps the barrier instead of adding one;
//  * the b x b Cholesky / LU are one warp each with columns in registers; the next pivot
//    is computed first so the dependency chain per column is shfl -> rsqrt -> fma;
//  * Gram sets, barrier counters are double-buffered by launch parity: launch L zeroes the
//    buffers of parity (L+1)&1 while using those of parity L&1 -- no memset launches.
#include <cooperative_groups.h>

#include "common.cuh"
#include "kernels.h"

namespace sbr {

constexpr int PC_THREADS = 256;
constexpr int PC_NCOPY = 8;    // Gram accumulated into 8 copies (CTA k -> k % 8): less atomic contention
constexpr int PC_NSET = 4;     // Gram sets per launch: round 0 + up to 3 checks
constexpr int PC_SETSTRIDE = 64 * 64;   // doubles per copy (max b)
constexpr double PC_ORTH_TOL = 1e-9;
template <int B> constexpr int pc_maxr() { return B <= 32 ? 512 : 128; }   // rows per CTA (smem)
template <int B> constexpr int pc_tpb() { return B / 4; }
template <int B> constexpr int pc_nt() { return pc_tpb<B>() * (pc_tpb<B>() + 1) / 2; }   // upper 4x4 tiles
template <int B> constexpr int pc_ngrp() { return PC_THREADS / pc_nt<B>() > 0 ? PC_THREADS / pc_nt<B>() : 1; }

// global workspace (bytes): [sets: 2 parities x NSET x NCOPY x 64 x 64 doubles]
//                           [ctr[2], luflag, fail]  [lu: Lcol, Urow (64x64 f32), S, dinv (64 f32)]
constexpr size_t PCW_SETS = 0;
constexpr size_t PCW_CTL = PCW_SETS + sizeof(double) * 2 * PC_NSET * PC_NCOPY * PC_SETSTRIDE;
constexpr size_t PCW_LU = PCW_CTL + 256;
constexpr size_t PCW_FB = PCW_LU + sizeof(float) * (2 * 64 * 64 + 2 * 64);   // Householder fallback:
// [64 x 64 doubles: per-column sums x_2^T p_c][64 x 64 doubles: V^T V][64 x 64 floats: R rows]
constexpr size_t PCW_BYTES = PCW_FB + sizeof(double) * 2 * 64 * 64 + sizeof(float) * 64 * 64;

size_t panel_chol_ws_bytes() { return PCW_BYTES; }
int* panel_chol_fail(void* ws) { return reinterpret_cast<int*>((char*)ws + PCW_CTL) + 3; }
unsigned* panel_chol_declines(void* ws) { return reinterpret_cast<unsigned*>((char*)ws + PCW_CTL) + 4; }

template <int B>
struct CholSmem {
  static constexpr int LDG = B + 1;
  static constexpr int LDQ = B + 2;   // Qd row stride (doubles): 4-way instead of 32-way conflicts on column stores
  static constexpr int NGRP = pc_ngrp<B>();
  static constexpr size_t OFF_Q = 0;                                              // double rows x B (row-major)
  static constexpr size_t OFF_GP = OFF_Q + sizeof(double) * pc_maxr<B>() * LDQ;  // double NGRP x B x B
  static constexpr size_t OFF_G = OFF_GP + sizeof(double) * NGRP * B * B;        // double B x LDG (chol in place)
  static constexpr size_t OFF_RRM = OFF_G + sizeof(double) * B * LDG;            // double B x B, R row-major
  static constexpr size_t OFF_RACC = OFF_RRM + sizeof(double) * B * B;           // double B x B (CTA 0: R product)
  static constexpr size_t OFF_RD = OFF_RACC + sizeof(double) * B * B;            // double B (1 / r_jj)
  static constexpr size_t OFF_RROW = OFF_RD + sizeof(double) * B;                // double 2B (row broadcast, padded)
  // L, U alias the Gram partials (Gpart is dead once a round's bulk reduction completed;
  // the LU of a round is recomputed after any later Gram)
  static constexpr size_t OFF_LC = OFF_GP;                                       // float B x B: Lcol[k*B + c] = L[c][k]
  static constexpr size_t OFF_UR = OFF_LC + sizeof(float) * B * B;               // float B x B: Urow[k*B + c] = U[k][c]
  static constexpr size_t OFF_S = OFF_RROW + sizeof(double) * 2 * B;             // float B signs
  static constexpr size_t OFF_DI = OFF_S + sizeof(float) * B;                    // float B 1/U[k][k]
  static constexpr size_t OFF_LR = OFF_DI + sizeof(float) * B;
  static constexpr size_t OFF_RDA = (OFF_LR + sizeof(float) * B + 15) / 16 * 16;   // double B: 1 / Racc_jj
  static constexpr size_t BYTES = OFF_RDA + sizeof(double) * B + 64;
};

SBR_DEV unsigned ld_acquire_u32(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
SBR_DEV void st_release_u32(unsigned* p, unsigned v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
SBR_DEV void bar_arrive(unsigned* ctr) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    atomicAdd(ctr, 1u);
  }
}
SBR_DEV void bar_wait(const unsigned* ctr, unsigned target) {
  if (threadIdx.x == 0) {
    while (ld_acquire_u32(ctr) < target) {
    }
  }
  __syncthreads();
}

// Cholesky G = R^T R of a B x B (B <= 32, power of two) fp64 matrix by ONE warp: lane c holds
// column c in registers, SHIFTED so that row j sits in slot 0 at step j; R row j is broadcast
// through shared memory, stored shifted too (rrow[i] = r_{j,j+i}, zero past B) so that every
// lane reads it with aligned 16-byte loads;
// the next pivot is computed first so the chain per column is shfl -> rsqrt -> mul -> fma.
// The step loop is unrolled (measured in the reduction: 5.6 us vs 6.9 us rolled -- one warp
// streams its straight-line code without the fetch stalls the CTA-wide phases show).  Writes R (upper, row-major) to Rrm, R (upper, ld LDG)
// to G and 1/r_jj to rd.  Returns false on breakdown (pivot <= floor_rel * max diag).
template <int B, int LDG>
SBR_DEV bool warp_chol(double* G, double* Rrm, double* rd, double* rrow, double floor_rel) {
  const int lane = lane_id();
  double g[B];
#pragma unroll
  for (int i = 0; i < B; ++i) g[i] = (lane < B && i <= lane) ? G[i + lane * LDG] : 0.0;
  double dmax = (lane < B) ? G[lane + lane * LDG] : 0.0;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) dmax = fmax(dmax, __shfl_xor_sync(0xffffffffu, dmax, o));
  bool ok = true;
  double piv = __shfl_sync(0xffffffffu, g[0], 0);
#pragma unroll
  for (int j = 0; j < B; ++j) {
    ok = ok && (piv > floor_rel * dmax);
    const double r = rsqrt(fmax(piv, 1e-300));   // 1 / r_jj
    const double rjc = (lane >= j) ? g[0] * r : 0.0;   // r_jc (lane j: r_jj)
    const double pn = __shfl_sync(0xffffffffu, fma(-rjc, rjc, g[1]), (j + 1) & 31);
    if (lane == j) rd[j] = r;
    if (lane < B) {
      rrow[(lane - j) & (B - 1)] = rjc;   // shifted: rrow[i] = r_{j, j+i} (zero past B: lanes < j)
      Rrm[j * B + lane] = rjc;
      G[j + lane * LDG] = rjc;
    }
    __syncwarp();
    const double2* rr2 = reinterpret_cast<const double2*>(rrow);
#pragma unroll
    for (int h = 0; h < B / 2; ++h) {
      const double2 rr = rr2[h];
      if (h > 0) g[2 * h - 1] = fma(-rr.x, rjc, g[2 * h]);
      g[2 * h] = fma(-rr.y, rjc, g[2 * h + 1]);
    }
    g[B - 1] = 0.0;
    piv = pn;
    __syncwarp();
  }
  return __all_sync(0xffffffffu, ok);
}

// Same by the whole CTA (one barrier per column) -- used for B > 32.
template <int B, int LDG>
SBR_DEV bool cta_chol(double* G, double* Rrm, double* rd, double floor_rel) {
  double dmax = 0.0;
  for (int i = 0; i < B; ++i) dmax = fmax(dmax, G[i + i * LDG]);
  bool ok = true;
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5, ny = blockDim.x >> 5;
  for (int j = 0; j < B; ++j) {
    const double gjj = G[j + j * LDG];
    if (!(gjj > floor_rel * dmax)) ok = false;
    const double inv = 1.0 / fmax(gjj, 1e-300);
    for (int c = j + 1 + tx; c < B; c += 32) {
      const double gjc = G[j + c * LDG] * inv;
      for (int i = j + 1 + ty; i <= c; i += ny) G[i + c * LDG] = fma(-G[j + i * LDG], gjc, G[i + c * LDG]);
    }
    __syncthreads();
  }
  for (int i = threadIdx.x; i < B; i += blockDim.x) rd[i] = rsqrt(fmax(G[i + i * LDG], 1e-300));
  __syncthreads();
  for (int e = threadIdx.x; e < B * B; e += blockDim.x) {
    const int i = e % B, c = e / B;
    const double v = (i <= c) ? G[i + c * LDG] * rd[i] : 0.0;
    G[i + c * LDG] = v;
    Rrm[i * B + c] = v;
  }
  __syncthreads();
  return ok;
}

// Modified LU of Q_1 - S (s_j = -sign(d_j)) of a B x B (B <= 32) matrix by ONE warp
// (fp32).  Lane i holds ROW i in registers, shifted so that column j sits in slot 0 at step j;
// the pivot row is broadcast through a ping-pong shared buffer with 16-byte stores / loads
// (stage, 2 x B floats), so a step is 2B/4 vector memory ops + B FMAs instead of B shuffles.
// Writes Lcol[k*B + c] = L[c][k] (unit lower), Urow[k*B + c] = U[k][c], S and dinv = 1/U[k][k].
template <int B, int LDQ>
SBR_DEV void warp_lu(const double* Q1, float* Lcol, float* Urow, float* Ss, float* dinv, float* stage) {
  const int lane = lane_id();
  float x[B];
#pragma unroll
  for (int c = 0; c < B; ++c) x[c] = (lane < B) ? (float)Q1[lane * LDQ + c] : 0.f;
#pragma unroll 1
  for (int j = 0; j < B; ++j) {
    float* st = stage + (j & 1) * B;
    if (lane == j) {
#pragma unroll
      for (int c = 0; c < B; c += 4) *reinterpret_cast<float4*>(st + c) = make_float4(x[c], x[c + 1], x[c + 2], x[c + 3]);
    }
    __syncwarp();
    float u[B];
#pragma unroll
    for (int c = 0; c < B; c += 4) {
      const float4 t = *reinterpret_cast<const float4*>(st + c);
      u[c] = t.x;
      u[c + 1] = t.y;
      u[c + 2] = t.z;
      u[c + 3] = t.w;
    }
    const float d = u[0];                      // A[j][j]
    const float sj = (d >= 0.f) ? -1.f : 1.f;
    const float piv = d - sj;
    const float inv = __fdividef(1.f, piv);
    if (lane < B) {
      Urow[j * B + lane] = (lane > j) ? st[(lane - j) & (B - 1)] : (lane == j ? piv : 0.f);
      const float l = (lane > j) ? x[0] * inv : (lane == j ? 1.f : 0.f);
      Lcol[j * B + lane] = l;
#pragma unroll
      for (int c = 1; c < B; ++c) x[c - 1] = fmaf(-l, u[c], x[c]);
      x[B - 1] = 0.f;
    }
    if (lane == j) {
      Ss[j] = sj;
      dinv[j] = inv;
    }
  }
  __syncwarp();
}

// Same by the whole CTA (one barrier per column) -- used for B > 32.
template <int B, int LDQ>
SBR_DEV void cta_lu(const double* Q1, float* Lcol, float* Urow, float* Ss, float* dinv) {
  // work in Urow as a dense row-major matrix A[i][c] = Urow[i*B + c]
  for (int e = threadIdx.x; e < B * B; e += blockDim.x) Urow[e] = (float)Q1[(e / B) * LDQ + e % B];
  __syncthreads();
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5, ny = blockDim.x >> 5;
  for (int j = 0; j < B; ++j) {
    const float d = Urow[j * B + j];
    const float sj = (d >= 0.f) ? -1.f : 1.f;
    const float invp = __frcp_rn(d - sj);
    for (int c = j + 1 + tx; c < B; c += 32) {
      const float ujc = Urow[j * B + c];
      for (int i = j + 1 + ty; i < B; i += ny) Urow[i * B + c] = fmaf(-Urow[i * B + j] * invp, ujc, Urow[i * B + c]);
    }
    __syncthreads();
    for (int i = j + 1 + threadIdx.x; i < B; i += blockDim.x) Lcol[j * B + i] = Urow[i * B + j] * invp;
    if (threadIdx.x == 0) {
      Ss[j] = sj;
      dinv[j] = invp;
      Urow[j * B + j] = d - sj;
    }
    __syncthreads();
  }
  for (int e = threadIdx.x; e < B * B; e += blockDim.x) {
    const int k = e / B, c = e % B;
    if (c < k) Urow[k * B + c] = 0.f;             // U is upper
    if (c <= k) Lcol[k * B + c] = (c == k) ? 1.f : 0.f;   // L column k: rows < k zero, unit diagonal
  }
  __syncthreads();
}

template <int B, bool STREAM>
__global__ void __launch_bounds__(PC_THREADS, 1) panel_chol_kernel(PanelArgs a, unsigned char* ws, unsigned launch) {
  pdl_trigger();   // the successor may launch early; it waits (griddepcontrol.wait) before reading
  using L = CholSmem<B>;
  constexpr int LDG = L::LDG;
  constexpr int LDQ = L::LDQ;
  constexpr int NGRP = L::NGRP;
  constexpr int TPB = pc_tpb<B>(), NT = pc_nt<B>();
  extern __shared__ __align__(16) unsigned char smem_raw[];
  double* Qd = reinterpret_cast<double*>(smem_raw + L::OFF_Q);
  double* Gpart = reinterpret_cast<double*>(smem_raw + L::OFF_GP);
  double* Gk = reinterpret_cast<double*>(smem_raw + L::OFF_G);
  double* Rrm = reinterpret_cast<double*>(smem_raw + L::OFF_RRM);
  double* Racc = reinterpret_cast<double*>(smem_raw + L::OFF_RACC);
  double* rd = reinterpret_cast<double*>(smem_raw + L::OFF_RD);
  double* rrow = reinterpret_cast<double*>(smem_raw + L::OFF_RROW);
  float* Lc = reinterpret_cast<float*>(smem_raw + L::OFF_LC);
  float* Ur = reinterpret_cast<float*>(smem_raw + L::OFF_UR);
  float* Ss = reinterpret_cast<float*>(smem_raw + L::OFF_S);
  float* Di = reinterpret_cast<float*>(smem_raw + L::OFF_DI);
  double* rda = reinterpret_cast<double*>(smem_raw + L::OFF_RDA);

  const unsigned par = launch & 1u;
  double* sets = reinterpret_cast<double*>(ws + PCW_SETS) + (size_t)par * PC_NSET * PC_NCOPY * PC_SETSTRIDE;
  unsigned* ctl = reinterpret_cast<unsigned*>(ws + PCW_CTL);
  unsigned* ctr = ctl + par;
  unsigned* luflag = ctl + 2;
  int* fail = reinterpret_cast<int*>(ctl + 3);
  float* gLc = reinterpret_cast<float*>(ws + PCW_LU);
  float* gUr = gLc + 64 * 64;
  float* gS = gUr + 64 * 64;
  float* gDi = gS + 64;

  const int warp = warp_id(), lane = lane_id();
  const int64_t m = a.m;
  const int G = gridDim.x;
  const int64_t r_beg = (int64_t)blockIdx.x * m / G, r_end = (int64_t)(blockIdx.x + 1) * m / G;
  const int rows = (int)(r_end - r_beg);
  // Panels taller than the shared-memory row capacity (148 CTAs x CH rows) are STREAMED: the CTA's
  // rows are processed in chunks of CH, and every round recomputes Q = P Racc^-1 (fp64) from the
  // fp32 panel instead of keeping Q resident.  Grid-uniform (row counts differ by at most one).
  constexpr int CH = pc_maxr<B>();
  constexpr bool stream = STREAM;   // the host picks it when (m + G - 1) / G > CH
  const int nch = STREAM ? (rows + CH - 1) / CH : 1;
  auto crows = [&](int ch) { return STREAM ? min(CH, rows - ch * CH) : rows; };
  auto stamp = [&](int k) {
    if (a.trace && blockIdx.x == 0 && threadIdx.x == 0) {
      int64_t t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      a.trace[k] = t;
    }
  };
  stamp(0);
  pdl_wait();   // launched with PDL: the predecessor (lazy update) must be complete before any read
  // ---- load rows [c0, c0 + n) of the CTA's range (column-major fp32 -> row-major fp64): all
  //      loads issued first
  auto load_rows = [&](int c0, int n) {
    constexpr int CPW = (B + 7) / 8, RPL = pc_maxr<B>() / 32;
    float v[CPW][RPL];
#pragma unroll
    for (int ci = 0; ci < CPW; ++ci) {
      const int c = warp + 8 * ci;
      const float* src = a.P + r_beg + c0 + (int64_t)c * a.ldp;
#pragma unroll
      for (int k = 0; k < RPL; ++k) {
        const int r = lane + 32 * k;
        v[ci][k] = (c < B && r < n) ? __ldg(src + r) : 0.f;
      }
    }
#pragma unroll
    for (int ci = 0; ci < CPW; ++ci) {
      const int c = warp + 8 * ci;
#pragma unroll
      for (int k = 0; k < RPL; ++k) {
        const int r = lane + 32 * k;
        if (c < B && r < n) Qd[r * LDQ + c] = (double)v[ci][k];
      }
    }
  };
  load_rows(0, crows(0));
  // ---- zero the other parity's Gram sets and barrier counter (used by the next launch)
  {
    double* other = reinterpret_cast<double*>(ws + PCW_SETS) + (size_t)(par ^ 1u) * PC_NSET * PC_NCOPY * PC_SETSTRIDE;
    // only the B x B head of each (set, copy) is ever accumulated (index p + q B)
    const int64_t tot = (int64_t)PC_NSET * PC_NCOPY * B * B;
    const int64_t per = (tot + G - 1) / G;
    const int64_t lo = (int64_t)blockIdx.x * per, hi = std::min<int64_t>(tot, lo + per);
    for (int64_t e = lo + threadIdx.x; e < hi; e += blockDim.x) other[(e / (B * B)) * PC_SETSTRIDE + e % (B * B)] = 0.0;
    if (blockIdx.x == 0 && threadIdx.x == 0) ctl[par ^ 1u] = 0u;
  }
  __syncthreads();
  stamp(1);

  // Gram tile of this thread: upper 4x4 tile (ti, tj), row group grp
  const int grp = threadIdx.x / NT, tl = threadIdx.x % NT;
  int ti = 0, tj = tl;
  while (tj >= TPB - ti) {
    tj -= TPB - ti;
    ++ti;
  }
  tj += ti;
  double acc[4][4];
  auto gram_zero = [&]() {
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
      for (int v = 0; v < 4; ++v) acc[u][v] = 0.0;
  };
  auto gram_acc = [&](int n) {   // this thread's 4x4 Gram tile over Qd rows [0, n) of its row group
    if (grp < NGRP) {
#pragma unroll 2
      for (int r = grp; r < n; r += NGRP) {
        const double2 a0 = *reinterpret_cast<const double2*>(Qd + r * LDQ + 4 * ti);
        const double2 a1 = *reinterpret_cast<const double2*>(Qd + r * LDQ + 4 * ti + 2);
        const double2 b0 = *reinterpret_cast<const double2*>(Qd + r * LDQ + 4 * tj);
        const double2 b1 = *reinterpret_cast<const double2*>(Qd + r * LDQ + 4 * tj + 2);
        const double aa[4] = {a0.x, a0.y, a1.x, a1.y};
        const double bb[4] = {b0.x, b0.y, b1.x, b1.y};
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
          for (int v = 0; v < 4; ++v) acc[u][v] = fma(aa[u], bb[v], acc[u][v]);
      }
    }
  };
  auto gram_arrive = [&](int set) {   // partial Gram tiles -> smem reduction -> set -> barrier arrive
    if (grp < NGRP) {
#pragma unroll
      for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4; ++v) Gpart[grp * B * B + (4 * ti + u) + (4 * tj + v) * B] = acc[u][v];
    }
    __syncthreads();
    // reduce the row groups in place into group 0 (lower triangle zero), then ONE bulk
    // async reduction (cp.reduce.async.bulk .add.f64) of the b x b block into the set copy
    for (int e = threadIdx.x; e < B * B; e += blockDim.x) {
      const int p = e % B, q = e / B;
      double sum = 0.0;
      if (p <= q) {
#pragma unroll 4
        for (int g2 = 0; g2 < NGRP; ++g2) sum += Gpart[g2 * B * B + e];
      }
      Gpart[e] = sum;
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    if (threadIdx.x == 0) {
      double* Gg = sets + ((size_t)set * PC_NCOPY + blockIdx.x % PC_NCOPY) * PC_SETSTRIDE;
      const unsigned sa = (unsigned)__cvta_generic_to_shared(Gpart);
      asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f64 [%0], [%1], %2;"
                   ::"l"(Gg), "r"(sa), "r"((unsigned)(B * B * sizeof(double))) : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
      asm volatile("fence.proxy.async.global;" ::: "memory");
      __threadfence();
      atomicAdd(ctr, 1u);
    }
    // Gpart is read by the bulk reduction until thread 0's wait_group: no warp may reuse it
    // (the LU's Lcol/Urow alias it) before that
    __syncthreads();
  };
  auto gram_read = [&](int set) {   // after the barrier: sum the copies into Gk (upper)
    const double* Gs = sets + (size_t)set * PC_NCOPY * PC_SETSTRIDE;
    for (int e = threadIdx.x; e < B * B; e += blockDim.x) {
      const int i = e % B, c = e / B;
      double g = 0.0;
      if (i <= c) {
#pragma unroll
        for (int k = 0; k < PC_NCOPY; ++k) g += __ldcg(Gs + (size_t)k * PC_SETSTRIDE + e);
      }
      Gk[i + c * LDG] = g;
    }
    __syncthreads();
  };
  auto chol = [&](double floor_rel) -> bool {
    if constexpr (B <= 32) {
      __shared__ int okflag;
      if (warp == 0) {
        const bool w = warp_chol<B, LDG>(Gk, Rrm, rd, rrow, floor_rel);
        if (lane == 0) okflag = w ? 1 : 0;
      }
      __syncthreads();
      return okflag != 0;
    } else {
      return cta_chol<B, LDG>(Gk, Rrm, rd, floor_rel);
    }
  };
  // Q <- Q R^-1 on Qd rows [0, n), 2 rows per thread: column-oriented forward substitution over
  // a SHIFTED copy of R (Rsh[k][i] = R[k][k+i], zero beyond B; in the Gram slot Gk, dead between
  // a round's Cholesky and the next Gram).  The k loop is rolled and the register row shifts
  // down one slot per step, so the code is a few hundred instructions: this phase runs once
  // per panel per SM, and inside the reduction (the pass's stream between panels evicts it)
  // fetching a fully unrolled triangle's code cost more than its arithmetic.
  auto solve = [&](const double* Rm, const double* rdg, int n) {
    double* Rsh = Gk;
    for (int e = threadIdx.x; e < B * B; e += blockDim.x) {
      const int k = e / B, i = e % B;
      Rsh[e] = (k + i < B) ? Rm[k * B + k + i] : 0.0;
    }
    __syncthreads();
    const int half = (n + 1) >> 1;
    for (int r = threadIdx.x; r < half; r += blockDim.x) {
      const int r2 = r + half;
      const bool two = r2 < n;
      double* qrow = Qd + r * LDQ;
      double* prow = Qd + (two ? r2 : r) * LDQ;
      double q[B], p[B];
#pragma unroll
      for (int c = 0; c < B; c += 2) {
        const double2 t = *reinterpret_cast<const double2*>(qrow + c);
        q[c] = t.x;
        q[c + 1] = t.y;
        const double2 u = *reinterpret_cast<const double2*>(prow + c);
        p[c] = u.x;
        p[c + 1] = u.y;
      }
#pragma unroll 1
      for (int k0 = 0; k0 < B; k0 += 2) {
        double qo[2], po[2];
#pragma unroll
        for (int s2 = 0; s2 < 2; ++s2) {
          const int k = k0 + s2;
          const double rk = rdg[k];
          const double qk = q[0] * rk, pk = p[0] * rk;
          qo[s2] = qk;
          po[s2] = pk;
          const double2* R2 = reinterpret_cast<const double2*>(Rsh + k * B);
#pragma unroll
          for (int h = 0; h < B / 2; ++h) {
            const double2 rr = R2[h];
            if (h > 0) {
              q[2 * h - 1] = fma(-qk, rr.x, q[2 * h]);
              p[2 * h - 1] = fma(-pk, rr.x, p[2 * h]);
            }
            q[2 * h] = fma(-qk, rr.y, q[2 * h + 1]);
            p[2 * h] = fma(-pk, rr.y, p[2 * h + 1]);
          }
          q[B - 1] = 0.0;
          p[B - 1] = 0.0;
        }
        *reinterpret_cast<double2*>(qrow + k0) = make_double2(qo[0], qo[1]);
        if (two) *reinterpret_cast<double2*>(prow + k0) = make_double2(po[0], po[1]);
      }
    }
    __syncthreads();
  };
  auto racc_update = [&](bool first) {   // Racc <- R_k Racc (upper triangular product); streaming: rda
    if (first) {
      for (int e = threadIdx.x; e < B * B; e += blockDim.x) Racc[e] = Rrm[e];
      if (threadIdx.x < B) rda[threadIdx.x] = rd[threadIdx.x];
      __syncthreads();
      return;
    }
    constexpr int PER = (B * B + PC_THREADS - 1) / PC_THREADS;
    double t4[PER];
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      const int e = threadIdx.x + k * PC_THREADS;
      double acc = 0.0;
      if (e < B * B) {
        const int i = e / B, c = e % B;
        for (int kk = i; kk <= c; ++kk) acc = fma(Rrm[i * B + kk], Racc[kk * B + c], acc);
      }
      t4[k] = acc;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      const int e = threadIdx.x + k * PC_THREADS;
      if (e < B * B) Racc[e] = t4[k];
    }
    __syncthreads();
    if (threadIdx.x < B) rda[threadIdx.x] = 1.0 / Racc[threadIdx.x * B + threadIdx.x];
    __syncthreads();
  };
  // streaming: Q rows of chunk ch = P rows Racc^-1, into Qd
  auto stream_q = [&](int ch) {
    __syncthreads();   // previous users of Qd are done
    load_rows(ch * CH, crows(ch));
    __syncthreads();
    solve(Racc, rda, crows(ch));
  };
  auto lu_publish = [&](unsigned gen) {   // CTA 0: LU of Q_1 - S, to smem and to global
    if constexpr (B <= 32) {
      if (warp == 0) warp_lu<B, LDQ>(Qd, Lc, Ur, Ss, Di, reinterpret_cast<float*>(rrow));
      __syncthreads();
    } else {
      cta_lu<B, LDQ>(Qd, Lc, Ur, Ss, Di);
    }
    for (int e = threadIdx.x; e < B * B; e += blockDim.x) {
      gLc[e] = Lc[e];
      gUr[e] = Ur[e];
    }
    if (threadIdx.x < B) {
      gS[threadIdx.x] = Ss[threadIdx.x];
      gDi[threadIdx.x] = Di[threadIdx.x];
    }
    __syncthreads();
    if (threadIdx.x == 0) {
      __threadfence();
      st_release_u32(luflag, gen);
    }
  };

  // rows of the block above the panel: Y = W = 0
  auto zero_above = [&]() {
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t nth = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = tid; i < a.row0; i += nth) {
#pragma unroll
      for (int c = 0; c < B; ++c) {
        a.Y[i + c * a.ldy] = 0.f;
        a.W[i + c * a.ldw] = 0.f;
        if (a.Wh) a.Wh[i + c * a.ldwh] = cvt16(0.f);
        if (a.Wrh) a.Wrh[i * a.ldwrh + c] = cvt16(0.f);
      }
      if (a.Yh) {   // 16-byte row stores
        const uint4 z = make_uint4(0u, 0u, 0u, 0u);
#pragma unroll
        for (int c = 0; c < B; c += 8) *reinterpret_cast<uint4*>(a.Yh + i * a.ldyh + c) = z;
      }
    }
  };

  // ---- Householder QR fallback (CholeskyQR declined: numerically rank deficient, or not
  //      orthonormal after three rounds).  dgeqr2 on the fp32 panel in global memory, fp64
  //      sums: per column j ONE grid reduction of t_c = x_2^T p_c (c >= j; x_2 = rows > j of
  //      column j), then every CTA forms dlarfg's (beta, tau) and w_c = tau (p_jc + t_c / (alpha -
  //      beta)) and updates its own rows; row j (R) goes to a side buffer so no CTA reads a row
  //      another one is writing.  Then T (dlarft) from V^T V (one more reduction) and the same
  //      outputs as the CholeskyQR path: Y = V, W^0 = V T, compact panel [R; V].
  auto hh_fallback = [&](unsigned& nb_) {
    if (blockIdx.x == 0 && threadIdx.x == 0) {
      *fail = 0;
      atomicAdd(ctl + 4, 1u);   // declines since the workspace was zeroed (sbr_test_panel_declines)
    }
    double* fsum = reinterpret_cast<double*>(ws + PCW_FB);
    double* fvv = fsum + 64 * 64;
    float* fR = reinterpret_cast<float*>(fvv + 64 * 64);
    float* P = a.P;
    const int64_t ldp = a.ldp;
    for (int e = blockIdx.x * blockDim.x + threadIdx.x; e < 2 * 64 * 64; e += G * blockDim.x) fsum[e] = 0.0;
    __syncthreads();   // Gpart (smem scratch below) is free: all Gram traffic is complete
    bar_arrive(ctr);
    bar_wait(ctr, (unsigned)G * ++nb_);
    double* wsm = Gpart;           // smem: w_c [B]
    double* taus = Gpart + 64;     // tau [B]
    double* Tm = Gpart + 128;      // T [B x B] row-major (fp64)
    float* Tf = reinterpret_cast<float*>(Tm + B * B);   // T as fp32
    const int64_t rb = r_beg, re = r_end;
    for (int j = 0; j < B; ++j) {
      const int64_t i0 = std::max<int64_t>(rb, j + 1);
      for (int c = j + warp; c < B; c += PC_THREADS / 32) {
        double sacc = 0.0;
        for (int64_t il = i0 + lane; il < re; il += 32)
          sacc = fma((double)__ldcg(P + il + (int64_t)j * ldp), (double)__ldcg(P + il + (int64_t)c * ldp), sacc);
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) sacc += __shfl_xor_sync(0xffffffffu, sacc, o);
        if (lane == 0 && sacc != 0.0) atomicAdd(fsum + j * 64 + c, sacc);
      }
      bar_arrive(ctr);
      bar_wait(ctr, (unsigned)G * ++nb_);
      const double sig2 = __ldcg(fsum + j * 64 + j);
      const double alpha = (double)__ldcg(P + j + (int64_t)j * ldp);
      double tj, bj, scal;
      if (!(sig2 > 0.0)) {   // x_2 = 0: H = I (dlarfg: tau = 0, beta = alpha)
        tj = 0.0;
        bj = alpha;
        scal = 0.0;
      } else {
        const double nrm = sqrt(fma(alpha, alpha, sig2));
        bj = alpha >= 0.0 ? -nrm : nrm;
        tj = (bj - alpha) / bj;
        scal = 1.0 / (alpha - bj);
      }
      const bool own_j = (j >= rb && j < re);
      if (threadIdx.x < B) {
        const int c = threadIdx.x;
        if (c > j) {
          const double pj = (double)__ldcg(P + j + (int64_t)c * ldp);
          const double wc = tj * (pj + scal * __ldcg(fsum + j * 64 + c));
          wsm[c] = wc;
          if (own_j) fR[j * 64 + c] = (float)(pj - wc);
        } else if (c == j) {
          taus[j] = tj;
          if (own_j) fR[j * 64 + j] = (float)bj;
        }
      }
      __syncthreads();
      for (int64_t il = i0 + threadIdx.x; il < re; il += blockDim.x) {
        const double v = (double)P[il + (int64_t)j * ldp] * scal;
        P[il + (int64_t)j * ldp] = (float)v;
        for (int c = j + 1; c < B; ++c) {
          float* pc = P + il + (int64_t)c * ldp;
          *pc = (float)fma(-v, wsm[c], (double)*pc);
        }
      }
      __syncthreads();
    }
    // V^T V (strict upper; v_i = 1 at row i, 0 above): one warp per pair, lanes over rows >= j2
    for (int e = warp; e < B * B; e += PC_THREADS / 32) {
      const int i = e / B, j2 = e % B;
      if (j2 <= i) continue;
      double sv = 0.0;
      for (int64_t il = std::max<int64_t>(rb, j2) + lane; il < re; il += 32) {
        const double vj = (il == j2) ? 1.0 : (double)P[il + (int64_t)j2 * ldp];
        sv = fma((double)P[il + (int64_t)i * ldp], vj, sv);
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) sv += __shfl_xor_sync(0xffffffffu, sv, o);
      if (lane == 0 && sv != 0.0) atomicAdd(fvv + i * 64 + j2, sv);
    }
    bar_arrive(ctr);
    bar_wait(ctr, (unsigned)G * ++nb_);
    // T (dlarft forward columnwise): T_jj = tau_j, T[0:j, j] = -tau_j T[0:j, 0:j] (V^T v_j)
    for (int e = threadIdx.x; e < B * B; e += blockDim.x) Tm[e] = 0.0;
    __syncthreads();
    if (warp == 0) {
      for (int j = 0; j < B; ++j) {
        for (int i = lane; i < j; i += 32) {
          double sacc = 0.0;
          for (int l = i; l < j; ++l) sacc = fma(Tm[i * B + l], __ldcg(fvv + l * 64 + j), sacc);
          Tm[i * B + j] = -taus[j] * sacc;
        }
        if (lane == 0) Tm[j * B + j] = taus[j];
        __syncwarp();
      }
    }
    __syncthreads();
    for (int e = threadIdx.x; e < B * B; e += blockDim.x) Tf[e] = (float)Tm[e];
    __syncthreads();
    // outputs per row: y = v, w = v T, compact panel
    for (int64_t il = rb + threadIdx.x; il < re; il += blockDim.x) {
      const int64_t gr = a.row0 + il;
      float v[B];
#pragma unroll
      for (int c = 0; c < B; ++c) v[c] = (il > c) ? P[il + (int64_t)c * ldp] : (il == c ? 1.f : 0.f);
      __align__(16) __half yh[B];
#pragma unroll
      for (int c = 0; c < B; ++c) {
        float w = 0.f;
#pragma unroll
        for (int k = 0; k <= c; ++k) w = fmaf(v[k], Tf[k * B + c], w);
        a.W[gr + (int64_t)c * a.ldw] = w;
        if (a.Wh) a.Wh[gr + (int64_t)c * a.ldwh] = cvt16(w);
        if (a.Wrh) a.Wrh[gr * a.ldwrh + c] = cvt16(w);
        a.Y[gr + (int64_t)c * a.ldy] = v[c];
        yh[c] = cvt16(v[c]);
        if (il <= c) P[il + (int64_t)c * ldp] = __ldcg(fR + il * 64 + c);   // R (il < B here)
      }
      if (a.Yh) {
#pragma unroll
        for (int c = 0; c < B; ++c) a.Yh[gr * a.ldyh + c] = yh[c];
      }
    }
  };

  // ---- round 0: G = P^T P, R_0 = chol(G), Q = P R_0^-1
  gram_zero();
  gram_acc(crows(0));
  for (int ch = 1; ch < nch; ++ch) {   // streaming only
    __syncthreads();
    load_rows(ch * CH, crows(ch));
    __syncthreads();
    gram_acc(crows(ch));
  }
  gram_arrive(0);
  stamp(2);
  bar_wait(ctr, (unsigned)G);
  unsigned nbar = 1;   // grid barriers passed (the counter target of the next is G * (nbar + 1))
  stamp(3);
  gram_read(0);
  if (!chol(0.0)) {                    // not numerically SPD: Householder QR in this launch
    hh_fallback(nbar);
    zero_above();
    return;
  }
  stamp(4);
  if (!stream) solve(Rrm, rd, rows);
  if (blockIdx.x == 0 || stream) racc_update(true);
  stamp(5);
  // ---- rounds k = 1..3: check G = Q^T Q ~ I, else one more CholeskyQR step
  unsigned gen = 0;
  bool done = false;
  for (int k = 1; k < PC_NSET; ++k) {
    gram_zero();
    if (!stream) {
      gram_acc(rows);
    } else {
      for (int ch = 0; ch < nch; ++ch) {
        stream_q(ch);
        gram_acc(crows(ch));
      }
    }
    gram_arrive(k);
    gen = launch * 4u + (unsigned)k;
    if (k == 1) stamp(6);
    if (blockIdx.x == 0) {   // speculative: valid if this round's check passes
      if (stream) stream_q(0);   // the top b rows of Q
      lu_publish(gen);
    }
    if (k == 1) stamp(7);
    bar_wait(ctr, (unsigned)G * (k + 1));
    nbar = k + 1;
    if (k == 1) stamp(8);
    gram_read(k);
    double dev = 0.0;
    for (int e = threadIdx.x; e < B * B; e += blockDim.x) {
      const int i = e % B, c = e / B;
      if (i <= c) dev = fmax(dev, fabs(Gk[i + c * LDG] - (i == c ? 1.0 : 0.0)));
    }
    if (!__syncthreads_or(!(dev <= (a.orth_tol > 0.0 ? a.orth_tol : PC_ORTH_TOL)))) {
      done = true;
      break;
    }
    if (k == PC_NSET - 1 || !chol(0.0)) break;
    if (!stream) solve(Rrm, rd, rows);
    if (blockIdx.x == 0 || stream) racc_update(false);
  }
  if (!done) {   // still not orthonormal after three rounds: Householder QR in this launch
    hh_fallback(nbar);
    zero_above();
    return;
  }
  stamp(9);
  // ---- L, U, S from CTA 0
  if (blockIdx.x != 0) {
    if (threadIdx.x == 0) {
      while (ld_acquire_u32(luflag) != gen) {
      }
    }
    __syncthreads();
    for (int e = threadIdx.x; e < B * B; e += blockDim.x) {
      Lc[e] = __ldcg(gLc + e);
      Ur[e] = __ldcg(gUr + e);
    }
    if (threadIdx.x < B) {
      Ss[threadIdx.x] = __ldcg(gS + threadIdx.x);
      Di[threadIdx.x] = __ldcg(gDi + threadIdx.x);
    }
    __syncthreads();
  } else if (threadIdx.x == 0) {
    *fail = 0;
  }
  stamp(10);
  // ---- rows: w L_1^T = e_il - q S ;  y = L_1 row (il < B) or y U = q ;  compact panel.
  //      Both triangular solves are column-oriented over SHIFTED fp32 factors (in the dead Rrm
  //      slot: Lsh[k][i] = L[k+i][k], Ush[k][i] = U[k][k+i], zero beyond B) with the k loop
  //      rolled in groups of 8 columns; each group's 8 outputs leave as coalesced fp32 / fp16
  //      column stores and one 16-byte fp16 row store (per-column 2-byte row stores measured
  //      slower inside the reduction: this phase is bound by its stores, not its arithmetic).
  const int64_t row0 = a.row0;
  float* Lsh = reinterpret_cast<float*>(Rrm);
  float* Ush = Lsh + B * B;
  for (int e = threadIdx.x; e < B * B; e += blockDim.x) {
    const int k = e / B, c = k + e % B;
    Lsh[e] = (c < B) ? Lc[k * B + c] : 0.f;
    Ush[e] = (c < B) ? Ur[k * B + c] : 0.f;
  }
  __syncthreads();
  stamp(12);
  for (int ch = 0; ch < nch; ++ch) {
  const int c0 = ch * CH, nr = crows(ch);
  if (stream) stream_q(ch);   // Q rows of this chunk (resident otherwise)
  for (int r = threadIdx.x; r < nr; r += blockDim.x) {
    const int64_t il = r_beg + c0 + r;
    const int64_t gr = row0 + il;
    const double* qrow = Qd + r * LDQ;
    float v[B];
#pragma unroll
    for (int c = 0; c < B; c += 2) {
      const double2 t = *reinterpret_cast<const double2*>(qrow + c);
      v[c] = ((il == c) ? 1.f : 0.f) - (float)t.x * Ss[c];
      v[c + 1] = ((il == c + 1) ? 1.f : 0.f) - (float)t.y * Ss[c + 1];
    }
#pragma unroll 1
    for (int k0 = 0; k0 < B; k0 += 8) {
      float wo[8];
#pragma unroll
      for (int s8 = 0; s8 < 8; ++s8) {
        const float wk = v[0];
        wo[s8] = wk;
        const float4* L4 = reinterpret_cast<const float4*>(Lsh + (k0 + s8) * B);
#pragma unroll
        for (int h = 0; h < B / 4; ++h) {
          const float4 l = L4[h];
          if (h > 0) v[4 * h - 1] = fmaf(-wk, l.x, v[4 * h]);
          v[4 * h] = fmaf(-wk, l.y, v[4 * h + 1]);
          v[4 * h + 1] = fmaf(-wk, l.z, v[4 * h + 2]);
          v[4 * h + 2] = fmaf(-wk, l.w, v[4 * h + 3]);
        }
        v[B - 1] = 0.f;
      }
      __align__(16) __half wh[8];
#pragma unroll
      for (int s8 = 0; s8 < 8; ++s8) {
        const int64_t c = k0 + s8;
        a.W[gr + c * a.ldw] = wo[s8];
        wh[s8] = cvt16(wo[s8]);
        if (a.Wh) a.Wh[gr + c * a.ldwh] = wh[s8];
      }
      if (a.Wrh) *reinterpret_cast<uint4*>(a.Wrh + gr * a.ldwrh + k0) = *reinterpret_cast<const uint4*>(wh);
    }
    if (r == 0 && ch == 0) stamp(13);
    float q[B];
#pragma unroll
    for (int c = 0; c < B; c += 2) {
      const double2 t = *reinterpret_cast<const double2*>(qrow + c);
      q[c] = (float)t.x;
      q[c + 1] = (float)t.y;
    }
#pragma unroll 1
    for (int k0 = 0; k0 < B; k0 += 8) {
      float yo[8];
      if (il >= B) {
#pragma unroll
        for (int s8 = 0; s8 < 8; ++s8) {
          const float yk = q[0] * Di[k0 + s8];
          yo[s8] = yk;
          const float4* U4 = reinterpret_cast<const float4*>(Ush + (k0 + s8) * B);
#pragma unroll
          for (int h = 0; h < B / 4; ++h) {
            const float4 u = U4[h];
            if (h > 0) q[4 * h - 1] = fmaf(-yk, u.x, q[4 * h]);
            q[4 * h] = fmaf(-yk, u.y, q[4 * h + 1]);
            q[4 * h + 1] = fmaf(-yk, u.z, q[4 * h + 2]);
            q[4 * h + 2] = fmaf(-yk, u.w, q[4 * h + 3]);
          }
          q[B - 1] = 0.f;
        }
      } else {   // top rows (CTA 0): y = row il of the unit lower L (Lsh[k][il-k] = L[il][k])
#pragma unroll
        for (int s8 = 0; s8 < 8; ++s8) {
          const int c = k0 + s8;
          yo[s8] = (c < il) ? Lsh[c * B + ((int)il - c)] : (c == il ? 1.f : 0.f);
        }
      }
      __align__(16) __half yh[8];
#pragma unroll
      for (int s8 = 0; s8 < 8; ++s8) {
        const int c = k0 + s8;
        a.Y[gr + (int64_t)c * a.ldy] = yo[s8];
        // compact panel: Y tail strictly below, R_h = S R on and above the diagonal (il < B)
        a.P[il + (int64_t)c * a.ldp] = (il > c) ? yo[s8] : (float)((double)Ss[il] * Racc[il * B + c]);
        yh[s8] = cvt16(yo[s8]);
      }
      if (a.Yh) *reinterpret_cast<uint4*>(a.Yh + gr * a.ldyh + k0) = *reinterpret_cast<const uint4*>(yh);
    }
    if (r == 0 && ch == 0) stamp(14);
  }
  }   // chunks
  stamp(15);
  zero_above();
  stamp(11);
}

template <int B>
static cudaError_t launch_chol_t(PanelArgs& a, void* ws, unsigned launch, cudaStream_t st) {
  constexpr size_t smem = CholSmem<B>::BYTES;
  cudaError_t e = func_attr((const void*)panel_chol_kernel<B, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)smem);
  if (e != cudaSuccess) return e;
  e = func_attr((const void*)panel_chol_kernel<B, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  const int per_sm = std::max(1, func_blocks_per_sm((const void*)panel_chol_kernel<B, false>, PC_THREADS, smem));
  const int nsm = current_device_sms();
  const int cap = per_sm * nsm;
  // >= 64 rows per CTA (CTA 0 must hold the b top rows); panels beyond cap x pc_maxr rows are
  // streamed in row chunks (see the kernel)
  int G = (int)std::min<int64_t>(cap, a.m / 64);
  if ((int64_t)G * pc_maxr<B>() < a.m) G = (int)std::min<int64_t>(cap, (a.m + pc_maxr<B>() - 1) / pc_maxr<B>());
  if (G < 1) return cudaErrorNotSupported;   // caller uses TSQR
  const bool stream = (a.m + G - 1) / G > pc_maxr<B>();
  auto kern = stream ? panel_chol_kernel<B, true> : panel_chol_kernel<B, false>;
  unsigned char* wsp = (unsigned char*)ws;
  // cooperative (grid-wide barriers) AND programmatic dependent launch: the launch and the
  // prologue overlap the tail of the lazy update; all CTAs are co-resident once it drains
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(G);
  cfg.blockDim = dim3(PC_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = 1;
  at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl_enabled() ? 2 : 1;
  return cudaLaunchKernelEx(&cfg, kern, a, wsp, launch);
}

cudaError_t launch_panel_chol(PanelArgs& a, void* ws, unsigned launch, cudaStream_t st) {
  if (a.m < 2 * a.b) return cudaErrorNotSupported;
  switch (a.b) {
    case 8: return launch_chol_t<8>(a, ws, launch, st);
    case 16: return launch_chol_t<16>(a, ws, launch, st);
    case 32: return launch_chol_t<32>(a, ws, launch, st);
    case 64: return launch_chol_t<64>(a, ws, launch, st);
    default: return cudaErrorNotSupported;
  }
}

SBR_OP16_SETTER(chol)

}  // namespace sbr
