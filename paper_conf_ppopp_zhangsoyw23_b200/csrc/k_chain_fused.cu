// k_chain_fused.cu -- the whole per-panel chain of the FP16 mode in ONE cooperative kernel
// (one launch per b-panel; the pass X_t = OA W_t stays a separate, HBM-streaming kernel).
//
// Per panel t of an nb-block (Alg. 1 l.5-10; readings C3-C5, R1, R2 of DESIGN.md),
// k = t b accumulated reflector columns, c = tb - b the OA column of the panel:
//   B  (t >= 1)  P = W^T R = X(c,:)^T - (W^T X) Y_c^T        k x b, fp32 -> fp16
//   C  (t >= 1)  GA = OA(:,c) - [X | Y] [Y_c ; P]^T           rows [c, M), tcgen05    (Alg.1 l.8-10)
//   D            panel QR of GA rows [tb, M): CholeskyQR in fp64 with the a-posteriori
//                orthogonality test (R1), or -- if it declines -- Householder QR (dgeqr2 in
//                fp64, dlarfg signs); the CholeskyQR Q goes through the paper's
//                reconstruction Q_1 - S = L U, Y = [L; Q_2 U^-1], W^0 = (E - Q S) L^-T
//                (Alg. 3 + S, reading C7)
//   E  (t >= 1)  G = Y_{<t}^T W^0,  H = X_{<t}^T W^0            k x b            (reading R2)
//   F  (t >= 1)  W_{<t}^T X_t = H - (W^T X) G -> W^T X column block (+ mirror)
//   G  (t >= 1)  W_t = W^0 - W_{<t} G -> fp32 W, fp16 copies for the pass / merges
//   A  (t >= 1)  tail of the previous pass: X_{t-1} -> fp16 row-major, W_{t-1}^T X_{t-1} (diagonal
//                block of W^T X)
// with grid-wide barriers between the phases that exchange data (7 per panel on the
// CholeskyQR path).
//
// One CTA per SM (cooperative launch, ~214 KB of shared memory): the panel rows a CTA
// updates in phase C are the rows it factors in phase D (kept in shared memory in fp64, no
// global round trip), the W^0 rows it writes in D are those phase E reads back through TMA.
// GEMM phases: warp 0 = TMA producer, warp 1 = MMA issuer (tcgen05 kind::f16, accumulators in
// TMEM), warps 4-7 = epilogue; SIMT phases use all 8 warps.
#include "common.cuh"
#include "kernels.h"
#include "tc.cuh"

namespace sbr {

using namespace tc;

namespace {

constexpr int CB = 32;                 // bandwidth of this kernel (b = 32: configs 2-4)
constexpr int CF_THREADS = 256;
constexpr int RING_NS = 4;
constexpr int RING_STAGE = 36864;      // phase E stage: Y slab 16 KB + X slab 16 KB + W rows 4 KB
constexpr int OFF_QD = RING_NS * RING_STAGE;   // 147456 (1024-aligned)
constexpr int LDQ = CB + 2;            // doubles per panel row in shared memory
constexpr int QD_ROWS = 256;           // panel rows per CTA (2 tiles of 128)
constexpr int OFF_BARS = OFF_QD + QD_ROWS * LDQ * 8;
constexpr int CF_SMEM = OFF_BARS + 256 + 1024;
constexpr int TPB4 = CB / 4;                       // 4x4 Gram tiles per row / column
constexpr int NT4 = TPB4 * (TPB4 + 1) / 2;        // upper 4x4 tiles (36)
constexpr int NGRP = CF_THREADS / NT4;            // row groups of the Gram (7)
constexpr int NCOPY = 8;                           // Gram copies (CTA % 8): less contention
constexpr int GSET = CB * CB;                      // doubles per Gram copy
constexpr int MAX_ROUNDS = 3;                      // CholeskyQR rounds (round 0 + checks)

// phase D scratch inside the ring (the ring is idle in phase D)
constexpr int D_GPART = 0;                                  // NGRP x B x B fp64
constexpr int D_GK = D_GPART + NGRP * CB * CB * 8;          // B x (B+1) fp64 (reduced Gram)
constexpr int D_RINV = D_GK + CB * (CB + 1) * 8;            // B x B fp64: R^-1 of the current round (row-major)
constexpr int D_RIACC = D_RINV + CB * CB * 8;               // accumulated R^-1 (Q = P RIACC)
constexpr int D_RACC = D_RIACC + CB * CB * 8;               // accumulated R (row-major)
constexpr int D_RR = D_RACC + CB * CB * 8;                  // R of the round (row-major)
constexpr int D_Q1 = D_RR + CB * CB * 8;                    // top b rows of Q (fp64 row-major)
constexpr int D_LINV = D_Q1 + CB * CB * 8;                  // fp32 L^-1 (unit lower), row-major
constexpr int D_UINV = D_LINV + CB * CB * 4;                // fp32 U^-1 (upper), row-major
constexpr int D_U = D_UINV + CB * CB * 4;                   // fp32 U row-major
constexpr int D_L = D_U + CB * CB * 4;                      // fp32 L row-major (unit lower)
constexpr int D_S = D_L + CB * CB * 4;                      // fp32 S
constexpr int D_DINV = D_S + CB * 4;                        // fp32 1/U_jj
constexpr int D_RD = D_DINV + CB * 4;                       // fp64 1/r_jj
constexpr int D_TMP = D_RD + CB * 8;                        // fp64 row / column buffers (4 x 2 x B)
constexpr int D_RINVT = D_TMP + CB * CB * 2;                // fp64 (R^-1)^T (row c = column c of R^-1)
constexpr int D_FLAG = D_RINVT + CB * CB * 8;                // ints
constexpr int D_END = D_FLAG + 64;
static_assert(D_END <= OFF_QD, "phase D scratch fits in the ring");

// per-launch workspace (double-buffered by launch parity): [counter | Gram sets | HH scratch]
constexpr size_t WS_CTR = 0;
constexpr size_t WS_GRAM = 256;
constexpr size_t WS_HH = WS_GRAM + sizeof(double) * MAX_ROUNDS * NCOPY * GSET;
constexpr size_t WS_HH_N = 2 * CB + 2 * CB * CB;                 // doubles
constexpr size_t WS_WTXP = WS_HH + sizeof(double) * WS_HH_N;     // NCOPY x B x B fp32: W^T X diag-block partials
constexpr size_t WS_PARITY = WS_WTXP + sizeof(float) * NCOPY * CB * CB;
static_assert(CF_SMEM <= 232448, "shared memory");

SBR_DEV unsigned ld_acquire(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// grid-wide barrier on a monotonic counter (wrap-safe); generic writes before it are visible to
// TMA (async proxy) reads after it
SBR_DEV void grid_barrier(unsigned* ctr, unsigned target) {
  asm volatile("fence.proxy.async.global;" ::: "memory");
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    atomicAdd(ctr, 1u);
    while ((int)(ld_acquire(ctr) - target) < 0) {
    }
    __threadfence();
    asm volatile("fence.proxy.async.global;" ::: "memory");
  }
  __syncthreads();
}

// async 16-byte global -> shared copies (LDGSTS): every copy of a staging loop in flight at once
SBR_DEV void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
SBR_DEV void cp_async_wait_all() {
  asm volatile("cp.async.commit_group;" ::: "memory");
  asm volatile("cp.async.wait_group 0;" ::: "memory");
}
SBR_DEV bool al16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; }

// stage `cols` columns of `rows` fp32 each (column j at src + j * lds, rows contiguous) into
// dst[j * ldd + i]; rows % 4 == 0 and 16-byte alignment -> cp.async, else batched loads
SBR_DEV void stage_cols(float* dst, int ldd, const float* src, int64_t lds, int rows, int cols) {
  const int tid = threadIdx.x;
  const bool vec = (rows % 4 == 0) && (ldd % 4 == 0) && (lds % 4 == 0) && al16(src) && al16(dst);
  if (vec) {
    const int q = rows / 4;
    for (int e = tid; e < q * cols; e += CF_THREADS) {
      const int j = e / q, i4 = e % q;
      cp_async16(dst + j * ldd + 4 * i4, src + j * lds + 4 * i4);
    }
    cp_async_wait_all();
  } else {
    constexpr int U = 8;
    for (int e0 = 0; e0 < rows * cols; e0 += U * CF_THREADS) {
      float v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int e = e0 + u * CF_THREADS + tid;
        v[u] = e < rows * cols ? __ldcg(src + (e / rows) * lds + e % rows) : 0.f;
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int e = e0 + u * CF_THREADS + tid;
        if (e < rows * cols) dst[(e / rows) * ldd + e % rows] = v[u];
      }
    }
  }
}

// out[qi][p] = sum_r Wc[qi * k + r] * Ys[r * B + p] for the CTA's nq (<= 8) rows qi, p < B:
// warp w sums r in its eighth of [0, k) for all rows (8 accumulators per lane; W loaded 4 r at a
// time as float4 broadcasts), then the 8 partials are summed through shared memory `red`
// (8 x 8 x B floats).  Returns the sum for (qi = warp, p = lane); k % 32 == 0.
SBR_DEV float cta_rows_dot(const float* Wc, int k, int nq, const float* Ys, float* red) {
  const int warp = warp_id(), lane = lane_id();
  const int ks = k / 8, r0 = warp * ks;
  float acc[8];
#pragma unroll
  for (int q = 0; q < 8; ++q) acc[q] = 0.f;
#pragma unroll 1
  for (int r = r0; r < r0 + ks; r += 4) {
    const float y0 = Ys[r * CB + lane], y1 = Ys[(r + 1) * CB + lane], y2 = Ys[(r + 2) * CB + lane],
                y3 = Ys[(r + 3) * CB + lane];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      if (q < nq) {
        const float4 w = *reinterpret_cast<const float4*>(Wc + q * k + r);
        acc[q] = fmaf(w.x, y0, acc[q]);
        acc[q] = fmaf(w.y, y1, acc[q]);
        acc[q] = fmaf(w.z, y2, acc[q]);
        acc[q] = fmaf(w.w, y3, acc[q]);
      }
    }
  }
#pragma unroll
  for (int q = 0; q < 8; ++q) red[(warp * 8 + q) * CB + lane] = acc[q];
  __syncthreads();
  float sacc = 0.f;
#pragma unroll
  for (int w = 0; w < 8; ++w) sacc += red[(w * 8 + warp) * CB + lane];
  __syncthreads();
  return sacc;
}

SBR_DEV void red_add_v4(float* addr, float a, float b, float c, float d) {
  asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(addr), "f"(a), "f"(b), "f"(c), "f"(d)
               : "memory");
}

// byte offset of element (row n, k) of a K-major fp16 tile (rows of 64 halves = 128 B) in the
// TMA SWIZZLE_128B layout: 16-byte chunk j of row n sits at chunk j ^ (n & 7)
SBR_DEV uint32_t sw128_off(int n, int k) {
  return (uint32_t)(n * 128 + ((((k >> 3) ^ n) & 7) << 4) + (k & 7) * 2);
}

// ---- b x b kernels on the whole CTA.  Element ownership is fixed for the whole factorisation:
// thread t owns row t / 8 (8 threads per row) and 4 consecutive columns 4 (t % 8) .. +3, in
// registers; one row is published through shared memory per elimination step (double-buffered),
// one __syncthreads per step.  (Measured on B200: one-warp versions -- lane = row, shuffles --
// took 13-50 k cycles each; per-step index arithmetic over shared memory 10-25 k.)

// Cholesky G = R^T R (fp64).  G read symmetric from Gk (upper stored, ld B+1).  Right-looking on
// the full symmetric matrix: step j: W[i][c] -= W[i][j] W[j][c] / W[j][j] (i, c > j).  R[j][c] =
// W[j][c] / sqrt(W[j][j]) for c >= j (row-major RR), rd[j] = 1 / r_jj.  rowbuf: 2 x B doubles.
// Every step loads what it needs into registers before computing or storing (shared-memory
// stores in between would serialise the loads: measured 3x).
SBR_DEV bool cta_chol64(const double* Gk, double* RR, double* rd, double floor_rel, double* rowbuf) {
  const int tid = threadIdx.x, i = tid >> 3, c0 = (tid & 7) * 4;
  double w[4];
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    const int c = c0 + u, lo = i < c ? i : c, hi = i < c ? c : i;
    w[u] = Gk[lo + hi * (CB + 1)];
  }
  double dmax = 0.0;
#pragma unroll 8
  for (int d = 0; d < CB; ++d) dmax = fmax(dmax, Gk[d * (CB + 2)]);
  bool ok = true;
#pragma unroll 1
  for (int j = 0; j < CB; ++j) {
    double* rb = rowbuf + (j & 1) * CB;
    if (i == j) {
#pragma unroll
      for (int u = 0; u < 4; ++u) rb[c0 + u] = w[u];
    }
    __syncthreads();
    double rv[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) rv[u] = rb[c0 + u];
    const double d = rb[j], wij = rb[i];
    ok = ok && (d > floor_rel * dmax) && (d < 1e300);
    const double r = rsqrt(fmax(d, 1e-300));
    if (i > j) {
      const double f = wij * (r * r);   // W[i][j] / W[j][j] (symmetric)
#pragma unroll
      for (int u = 0; u < 4; ++u)
        if (c0 + u > j) w[u] = fma(-f, rv[u], w[u]);
    } else if (i == j) {   // R row j (final)
#pragma unroll
      for (int u = 0; u < 4; ++u) RR[j * CB + c0 + u] = (c0 + u >= j) ? rv[u] * r : 0.0;
      if (c0 == 0) rd[j] = r;
    }
  }
  __syncthreads();
  return ok;
}

// X = R^-1 for R upper triangular (row-major; rdiag[j] = 1 / R[j][j]) by Gauss-Jordan from the
// bottom on [R | I], X part only: step j = B-1 .. 0: X[j] *= rdiag[j] (published), then
// X[i] -= R[i][j] X[j] for i < j.  Threads [tb0, tb0 + 8 * B / CPT) take part, CPT columns each.
// X != NULL: X row-major; XT != NULL: X^T (row c = column c of X).  rowbuf: 2 x B.
template <typename T, int CPT>
SBR_DEV void cta_inv_upper(const T* R, const T* rdiag, T* X, T* XT, T* rowbuf, int tb0) {
  constexpr int TPR = CB / CPT;   // threads per row
  const int t = threadIdx.x - tb0;
  const bool mine = t >= 0 && t < TPR * CB;
  const int i = mine ? t / TPR : 0, c0 = mine ? (t % TPR) * CPT : 0;
  T x[CPT];
#pragma unroll
  for (int u = 0; u < CPT; ++u) x[u] = (i == c0 + u) ? T(1) : T(0);
#pragma unroll 1
  for (int j = CB - 1; j >= 0; --j) {
    T* rb = rowbuf + (j & 1) * CB;
    const T dj = rdiag[j], f = R[i * CB + j];
    if (mine && i == j) {
#pragma unroll
      for (int u = 0; u < CPT; ++u) {
        x[u] *= dj;
        rb[c0 + u] = x[u];
      }
    }
    __syncthreads();
    T rv[CPT];
#pragma unroll
    for (int u = 0; u < CPT; ++u) rv[u] = rb[c0 + u];
    if (mine && i < j) {
#pragma unroll
      for (int u = 0; u < CPT; ++u) x[u] -= f * rv[u];
    }
  }
  if (mine) {
#pragma unroll
    for (int u = 0; u < CPT; ++u) {
      if (X) X[i * CB + c0 + u] = x[u];
      if (XT) XT[(c0 + u) * CB + i] = x[u];
    }
  }
  __syncthreads();
}

// U^-1 (written transposed into UT: row c = column c of U^-1) on threads 0-127 and L^-1 (L unit
// lower, row-major into LI) on threads 128-255, 8 columns per thread, sharing the 32 barriers.
SBR_DEV void cta_inv_both32(const float* U, const float* dinv, float* UT, const float* L, float* LI, float* rowbuf) {
  const int tid = threadIdx.x;
  const bool up = tid < 128;
  const int t = up ? tid : tid - 128;
  const int i = t >> 2, c0 = (t & 3) * 8;
  float x[8];
#pragma unroll
  for (int u = 0; u < 8; ++u) x[u] = (i == c0 + u) ? 1.f : 0.f;
#pragma unroll 1
  for (int s = 0; s < CB; ++s) {
    const int j = up ? CB - 1 - s : s;
    float* rb = rowbuf + ((s & 1) * 2 + (up ? 0 : 1)) * CB;
    const float dj = up ? dinv[j] : 1.f;
    const float f = up ? U[i * CB + j] : L[i * CB + j];
    if (i == j) {
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        x[u] *= dj;
        rb[c0 + u] = x[u];
      }
    }
    __syncthreads();
    float rv[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) rv[u] = rb[c0 + u];
    if (up ? (i < j) : (i > j)) {
#pragma unroll
      for (int u = 0; u < 8; ++u) x[u] = fmaf(-f, rv[u], x[u]);
    }
  }
#pragma unroll
  for (int u = 0; u < 8; ++u) {
    if (up) UT[(c0 + u) * CB + i] = x[u];
    else LI[i * CB + c0 + u] = x[u];
  }
  __syncthreads();
}

// Modified LU of Q_1 - S (s_j = -sign(d_j), pivot d_j - s_j, |pivot| >= 1), right-looking
// in fp32, element ownership as cta_chol64.  Writes L (unit lower), U (row-major), S, 1/U_jj.
SBR_DEV void cta_lu(const double* Q1, float* L, float* U, float* S, float* dinv, float* rowbuf, float* colbuf) {
  const int tid = threadIdx.x, i = tid >> 3, c0 = (tid & 7) * 4;
  float a[4];
#pragma unroll
  for (int u = 0; u < 4; ++u) a[u] = (float)Q1[i * CB + c0 + u];
#pragma unroll 1
  for (int j = 0; j < CB; ++j) {
    float* rb = rowbuf + (j & 1) * CB;
    float* cb = colbuf + (j & 1) * CB;
    if (i == j) {
#pragma unroll
      for (int u = 0; u < 4; ++u) rb[c0 + u] = a[u];
    }
    if (c0 == (j & ~3)) {   // column j of every row
      float v = a[0];
#pragma unroll
      for (int u = 1; u < 4; ++u)
        if (c0 + u == j) v = a[u];
      cb[i] = v;
    }
    __syncthreads();
    float rv[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) rv[u] = rb[c0 + u];
    const float d = rb[j], aij = cb[i];
    const float sj = (d >= 0.f) ? -1.f : 1.f;
    const float inv = 1.f / (d - sj);
    if (tid == 0) {
      S[j] = sj;
      dinv[j] = inv;
    }
    if (i > j) {
      const float l = aij * inv;
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int c = c0 + u;
        if (c > j) a[u] = fmaf(-l, rv[u], a[u]);
        else if (c == j) a[u] = l;   // L[i][j]
      }
    } else if (i == j) {
#pragma unroll
      for (int u = 0; u < 4; ++u)
        if (c0 + u == j) a[u] = d - sj;   // U[j][j] = pivot
    }
  }
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    const int c = c0 + u;
    U[i * CB + c] = (c >= i) ? a[u] : 0.f;
    L[i * CB + c] = (c < i) ? a[u] : (c == i ? 1.f : 0.f);
  }
  __syncthreads();
}

}  // namespace

struct ChainFusedArgs {
  int t, k;
  int64_t M, tb, c;        // c = tb - b (t >= 1)
  float* A;                // master; OA(i, j) = A[(r0 + i) + (r0 + j) * lda]
  int64_t lda, r0;
  float* Yb;               // block Y, fp32 column-major (OA rows), ld ldy
  int64_t ldy;
  float* Wt;               // this panel's W columns (OA rows), fp32 column-major, ld ldw
  int64_t ldw;
  const float* Xb;         // X, fp32 column-major M x (p b), ld ldx
  int64_t ldx;
  __half* Xh;              // M x ldk row-major fp16 X (phase A writes column block t-1)
  float* WtX;              // nb x nb fp32 (symmetric)
  int64_t ldwx;
  float* Gf;               // k x B row-major fp32 scratch (G), zeroed in phase B
  float* Hf;               // k x B row-major fp32 scratch (H)
  __half* Ph;              // B x ldk row-major (P^T)
  __half* Yh;              // M x ldk row-major
  __half* Wrh;             // M x ldk row-major (W, later merges)
  int64_t ldk;
  __half* Wh;              // column-major fp16 W of this panel (pass operand), ld ldwh
  int64_t ldwh;
  uint8_t* ws_cur;          // this launch's parity of the workspace (zeroed by the previous launch)
  uint8_t* ws_next;         // the next launch's parity (zeroed here)
  unsigned* declines;      // count of CholeskyQR declines (test hook)
  double orth_tol;
  int64_t* trace;          // optional: CTA 0 phase stamps (globaltimer ns), 16 entries
};

__global__ void __launch_bounds__(CF_THREADS, 1)
    chain_fused_kernel(const __grid_constant__ CUtensorMap mXc, const __grid_constant__ CUtensorMap mYc,
                       const __grid_constant__ CUtensorMap mYb, const __grid_constant__ CUtensorMap mPh,
                       const __grid_constant__ CUtensorMap mXe, const __grid_constant__ CUtensorMap mYe,
                       const __grid_constant__ CUtensorMap mWe, const __grid_constant__ CUtensorMap mWg,
                       ChainFusedArgs a) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* ring = smem;
  double* Qd = reinterpret_cast<double*>(smem + OFF_QD);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + OFF_BARS);
  uint64_t* full = bars;                 // [RING_NS]
  uint64_t* empty = bars + RING_NS;      // [RING_NS]
  uint64_t* accf = bars + 2 * RING_NS;   // [2]
  uint64_t* acce = accf + 2;             // [2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(acce + 2);
  int* sflag = reinterpret_cast<int*>(tmem_slot + 2);

  const int warp = warp_id(), lane = lane_id(), tid = threadIdx.x;
  const int G = gridDim.x, cta = blockIdx.x;
  auto stamp = [&](int i) {
    if (a.trace && cta == 0 && tid == 0) {
      int64_t tt;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tt));
      a.trace[i] = tt;
    }
  };
  stamp(0);
  const int t = a.t, k = a.k;
  const int64_t M = a.M, tb = a.tb, c = a.c;
  pdl_trigger();
  if (tid == 0) {
    for (int i = 0; i < RING_NS; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    for (int i = 0; i < 2; ++i) { mbar_init(&accf[i], 1); mbar_init(&acce[i], 128); }
    mbar_fence_init();
  }
  if (warp == 0 && lane == 0) {
    tma_prefetch(&mXc); tma_prefetch(&mYc); tma_prefetch(&mYb); tma_prefetch(&mPh);
    tma_prefetch(&mXe); tma_prefetch(&mYe); tma_prefetch(&mWe); tma_prefetch(&mWg);
  }
  if (warp == 2) tmem_alloc(tmem_slot, 128);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();
  stamp(1);

  unsigned* const ctr = reinterpret_cast<unsigned*>(a.ws_cur + WS_CTR);
  double* const gsets = reinterpret_cast<double*>(a.ws_cur + WS_GRAM);
  double* const hhs = reinterpret_cast<double*>(a.ws_cur + WS_HH);
  float* const wtxp = reinterpret_cast<float*>(a.ws_cur + WS_WTXP);
  {   // the next launch's workspace: zero it now (this launch completes before that one reads it)
    const size_t nw = WS_PARITY / sizeof(unsigned);
    unsigned* z = reinterpret_cast<unsigned*>(a.ws_next);
    for (size_t e = (size_t)cta * CF_THREADS + tid; e < nw; e += (size_t)G * CF_THREADS) z[e] = 0u;
  }
  unsigned nbar = 0;
  auto gbar = [&]() { grid_barrier(ctr, (unsigned)G * (++nbar)); };

  // persistent ring / accumulator state of the three roles (advanced identically)
  int p_st = 0; uint32_t p_ph = 0;            // producer
  int m_st = 0; uint32_t m_ph = 0;            // MMA
  int m_ab = 0; uint32_t m_aph = 0;
  int e_ab = 0; uint32_t e_aph = 0;           // epilogue

  // ---- rows of phases C / D: 128-row tiles of [c0r, M) (c0r = c for t >= 1: the diagonal block
  //      and the panel; tb = 0 for t = 0), contiguous per CTA
  const int64_t c0r = (t >= 1) ? c : 0;
  const int ntc = (int)((M - c0r + 127) / 128);
  const int tpc = (ntc + G - 1) / G;          // <= 2 (host checks the capacity)
  const int ti0 = min(ntc, cta * tpc), ti1 = min(ntc, ti0 + tpc);
  const int64_t R0 = c0r + (int64_t)ti0 * 128, R1 = std::min<int64_t>(M, c0r + (int64_t)ti1 * 128);
  const int64_t P0 = std::max<int64_t>(R0, tb);    // first panel row of this CTA (OA row)
  const int nloc = (int)std::max<int64_t>(0, R1 - P0);   // panel rows held in Qd
  const int64_t m = M - tb;                   // panel height

  // the panel's columns: global column g = c0 + tb = r0 - b + tb; Acol(i, p) = A at OA row i,
  // panel column p (OA column c + p for t >= 1)
  const int64_t gcol = a.r0 + tb - CB;
  auto Acol = [&](int64_t i, int col) -> float& { return a.A[(a.r0 + i) + (gcol + col) * a.lda]; };

  // =====================================================================================
  // Phase A (t >= 1): tail of pass t-1 -- Xh(:, tp) = fp16(X_tp) and W^T X(tp, tp) += W_tp^T X_tp
  // =====================================================================================
  if (t >= 1) {
    const int64_t tp = tb - CB;
    const int64_t per = ((M + G - 1) / G + 3) / 4 * 4;   // rows per CTA (multiple of 4: aligned staging)
    const int64_t rbeg = std::min<int64_t>(M, (int64_t)cta * per), rend = std::min<int64_t>(M, rbeg + per);
    const int nr = (int)(rend - rbeg);                  // <= 256 (host checks M <= 2 * 128 * grid)
    const int lds = ((int)per + 3) / 4 * 4 % 32 == 4 ? ((int)per + 3) / 4 * 4 : ((int)per + 3) / 32 * 32 + 36;
    float* Xs = reinterpret_cast<float*>(ring);        // column p at Xs + p * lds
    float* Ws = Xs + CB * lds;
    if (nr > 0) {
      stage_cols(Xs, lds, a.Xb + rbeg + tp * a.ldx, a.ldx, nr, CB);
      stage_cols(Ws, lds, a.Wt - CB * a.ldw + rbeg, a.ldw, nr, CB);
    }
    __syncthreads();
    stamp(25);
    for (int e = tid; e < nr * (CB / 8); e += CF_THREADS) {
      const int rr = e / (CB / 8), g8 = e % (CB / 8);
      __align__(16) __half hv[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) hv[u] = __float2half_rn(Xs[(g8 * 8 + u) * lds + rr]);
      *reinterpret_cast<uint4*>(a.Xh + (rbeg + rr) * a.ldk + tp + g8 * 8) = *reinterpret_cast<const uint4*>(hv);
    }
    {   // W_tp^T X_tp partial over the CTA's rows: thread = (i = lane, j = 4 warp .. +3); W column i
        // (bank (4 i + rr) % 32 with lds = 4 mod 32: 4-way), X columns j broadcast
      const int ii = lane, j0 = warp * 4;
      float acc[4] = {0.f, 0.f, 0.f, 0.f};
      const float* wp = Ws + ii * lds;
#pragma unroll 4
      for (int rr = 0; rr < nr; ++rr) {
        const float wv = wp[rr];
#pragma unroll
        for (int v = 0; v < 4; ++v) acc[v] = fmaf(wv, Xs[(j0 + v) * lds + rr], acc[v]);
      }
      // partial block (column-major 32 x 32) -> one bulk fp32 reduction into copy cta % NCOPY
      float* P2 = Ws + CB * lds;
      __syncthreads();
      stamp(26);
#pragma unroll
      for (int v = 0; v < 4; ++v) P2[ii + (j0 + v) * CB] = acc[v];
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncthreads();
      if (tid == 0 && nr > 0) {
        asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f32 [%0], [%1], %2;" ::"l"(
                         wtxp + (size_t)(cta % NCOPY) * CB * CB),
                     "r"(smem_u32(P2)), "r"((unsigned)(CB * CB * sizeof(float)))
                     : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
      }
    }
    gbar();   // W^T X partials of block tp complete; Xh of X_tp
    if (cta == 0) {   // W^T X(tp, tp) = sum of the copies (later phases / kernels read WtX)
      for (int e = tid; e < CB * CB; e += CF_THREADS) {
        float v = 0.f;
#pragma unroll
        for (int kk = 0; kk < NCOPY; ++kk) v += __ldcg(wtxp + kk * CB * CB + e);
        a.WtX[(tp + e % CB) + (tp + e / CB) * a.ldwx] = v;
      }
    }
  }
  stamp(2);

  // =====================================================================================
  // Phase B (t >= 1): P = X(c,:)^T - (W^T X) Y_c^T   (k x B) -> Ph (fp16, P^T row-major)
  // =====================================================================================
  if (t >= 1) {
    // zero the G / H reduction targets of phase E
    const int64_t kz = (int64_t)((k + 127) / 128) * 128 * CB;   // whole slabs (phase E reduces 128-row blocks)
    for (int64_t e = (int64_t)cta * CF_THREADS + tid; e < kz; e += (int64_t)G * CF_THREADS) {
      a.Gf[e] = 0.f;
      a.Hf[e] = 0.f;
    }
    float* Ycs = reinterpret_cast<float*>(ring);               // Ycs[r * B + p] = Y(c + p, r)
    float* Wcs = reinterpret_cast<float*>(ring) + (size_t)k * CB;   // the CTA's WtX columns (8 x k)
    const int q0 = cta * 8;
    if (q0 < k) {
      stage_cols(Ycs, CB, a.Yb + c, a.ldy, CB, k);                         // Y(c + p, r) -> Ycs[r B + p]
      stage_cols(Wcs, k, a.WtX + (int64_t)q0 * a.ldwx, a.ldwx, k, min(8, k - q0));   // WtX columns q0..
    }
    __syncthreads();
    stamp(22);
    const int64_t tp = tb - CB;
    if (q0 < k && q0 >= tp) {   // columns in block tp: its diagonal block is the sum of the phase-A copies
      for (int e = tid; e < min(8, k - q0) * CB; e += CF_THREADS) {
        const int qi = e / CB, i = e % CB;
        float v = 0.f;
#pragma unroll
        for (int kk = 0; kk < NCOPY; ++kk) v += __ldcg(wtxp + kk * CB * CB + i + (q0 + qi - tp) * CB);
        Wcs[qi * k + tp + i] = v;
      }
    }
    __syncthreads();
    {
      const int nqb = q0 < k ? min(8, k - q0) : 0;
      const float xv = (warp < nqb) ? __ldcg(a.Xb + (c + lane) + (int64_t)(q0 + warp) * a.ldx) : 0.f;
      const float dot = cta_rows_dot(Wcs, k, nqb, Ycs, reinterpret_cast<float*>(smem + 163840));   // past Ycs + Wcs (k <= 1024)
      if (warp < nqb) a.Ph[(int64_t)lane * a.ldk + q0 + warp] = __float2half_rn(xv - dot);
    }
    gbar();   // 1: P complete (TMA-readable)
  }
  stamp(3);

  // =====================================================================================
  // Phase C (t >= 1): GA = OA(:, c) - [X | Y] [Y_c ; P]^T on rows [R0, R1)  -> A, Qd (fp64)
  // Phase D input for t = 0: the panel rows straight from A.
  // =====================================================================================
  if (t >= 1) {
    const int kc0 = (k + 63) / 64;
    const int nk = 2 * kc0;
    constexpr uint32_t STAGE_BYTES = 128 * 64 * 2 + CB * 64 * 2;
    if (warp == 0 && lane == 0) {
      for (int ti = ti0; ti < ti1; ++ti) {
        const int row = (int)(c0r + (int64_t)ti * 128);
        for (int kc = 0; kc < nk; ++kc) {
          mbar_wait(&empty[p_st], p_ph ^ 1);
          mbar_expect_tx(&full[p_st], STAGE_BYTES);
          uint8_t* sa = ring + p_st * RING_STAGE;
          const bool second = kc >= kc0;
          const int kin = (second ? kc - kc0 : kc) * 64;
          tma_load_2d(sa, second ? &mYc : &mXc, &full[p_st], kin, row);
          tma_load_2d(sa + 16384, second ? &mPh : &mYb, &full[p_st], kin, second ? 0 : (int)c);
          if (++p_st == RING_NS) { p_st = 0; p_ph ^= 1; }
        }
      }
    } else if (warp == 1 && lane == 0) {
      constexpr uint32_t idesc = idesc_make(128, CB, 0, 0, 0);
      const uint32_t s0 = smem_u32(ring);
      for (int ti = ti0; ti < ti1; ++ti) {
        mbar_wait(&acce[m_ab], m_aph ^ 1);
        tc_fence_after();
        const uint32_t d = tmem + 64 * m_ab;
        for (int kc = 0; kc < nk; ++kc) {
          mbar_wait(&full[m_st], m_ph);
          tc_fence_after();
          const uint32_t sa = s0 + m_st * RING_STAGE, sb = sa + 16384;
#pragma unroll
          for (int s = 0; s < 4; ++s)
            mma_f16(d, sdesc_sw128(sa + s * 32, 16, 1024), sdesc_sw128(sb + s * 32, 16, 1024), idesc,
                    (kc > 0 || s > 0) ? 1u : 0u);
          mma_commit(&empty[m_st]);
          if (++m_st == RING_NS) { m_st = 0; m_ph ^= 1; }
        }
        mma_commit(&accf[m_ab]);
        if (++m_ab == 2) { m_ab = 0; m_aph ^= 1; }
      }
    } else if (warp >= 4) {
      const int qw = warp - 4;
      for (int ti = ti0; ti < ti1; ++ti) {
        const int64_t r = c0r + (int64_t)ti * 128 + qw * 32 + lane;
        float cv[CB];
        const bool in = r < M;
        const int64_t idg = r - c;   // row within the diagonal block (< B)
#pragma unroll
        for (int p = 0; p < CB; ++p) {
          float v = 0.f;
          if (in) v = (idg < p) ? Acol(c + p, (int)idg) : Acol(r, p);   // upper part of the block: mirror (C14)
          cv[p] = v;
        }
        mbar_wait(&accf[e_ab], e_aph);
        tc_fence_after();
        float acc[32];
        tmem_ld32(tmem + 64 * e_ab + ((uint32_t)(qw * 32) << 16), acc);
        tc_fence_before();
        mbar_arrive(&acce[e_ab]);
        if (++e_ab == 2) { e_ab = 0; e_aph ^= 1; }
        if (in) {
#pragma unroll
          for (int p = 0; p < CB; ++p) {
            const float v = cv[p] - acc[p];
            Acol(r, p) = v;
            cv[p] = v;
          }
          if (r >= P0) {
            double* q = Qd + (r - P0) * LDQ;
#pragma unroll
            for (int p = 0; p < CB; p += 2) *reinterpret_cast<double2*>(q + p) = make_double2(cv[p], cv[p + 1]);
          }
        }
      }
    }
    __syncthreads();
  } else {
    // t = 0: the panel is current in A (updated by the previous block's SYR2K)
    for (int e0 = 0; e0 < nloc * CB; e0 += 8 * CF_THREADS) {
      float v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int e = e0 + u * CF_THREADS + tid;
        v[u] = e < nloc * CB ? __ldcg(&Acol(P0 + e % nloc, e / nloc)) : 0.f;
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int e = e0 + u * CF_THREADS + tid;
        if (e < nloc * CB) Qd[(e % nloc) * LDQ + e / nloc] = (double)v[u];
      }
    }
    __syncthreads();
  }

  // =====================================================================================
  // Phase D: panel QR of the m x B panel (rows [tb, M)): CholeskyQR + reconstruction, or
  // Householder QR if CholeskyQR declines.  Outputs: Y (A below the diagonal, Yb, Yh), R_h
  // (band), W^0 (Wt fp32, Wh fp16 column-major; t = 0 also Wrh).
  // =====================================================================================
  double* Gpart = reinterpret_cast<double*>(ring + D_GPART);
  double* Gk = reinterpret_cast<double*>(ring + D_GK);
  double* Rinv = reinterpret_cast<double*>(ring + D_RINV);
  double* Riacc = reinterpret_cast<double*>(ring + D_RIACC);
  double* Racc = reinterpret_cast<double*>(ring + D_RACC);
  double* RR = reinterpret_cast<double*>(ring + D_RR);
  double* Q1 = reinterpret_cast<double*>(ring + D_Q1);
  float* Linv = reinterpret_cast<float*>(ring + D_LINV);
  float* Uinv = reinterpret_cast<float*>(ring + D_UINV);
  float* Us = reinterpret_cast<float*>(ring + D_U);
  float* Ls = reinterpret_cast<float*>(ring + D_L);
  float* Ss = reinterpret_cast<float*>(ring + D_S);
  float* Dinv = reinterpret_cast<float*>(ring + D_DINV);
  double* rd = reinterpret_cast<double*>(ring + D_RD);
  double* RinvT = reinterpret_cast<double*>(ring + D_RINVT);

  // Gram of Qd rows [0, nloc): thread = upper 4x4 tile (ti4, tj4) x row group; reduced in smem,
  // then one bulk fp64 reduction into set copy (cta % NCOPY)
  const int grp = tid / NT4, tl = tid % NT4;
  int ti4 = 0, tj4 = tl;
  while (tj4 >= TPB4 - ti4) { tj4 -= TPB4 - ti4; ++ti4; }
  tj4 += ti4;
  auto gram_arrive = [&](int set) {
    double acc[4][4];
#pragma unroll
    for (int u = 0; u < 4; ++u)
#pragma unroll
      for (int v = 0; v < 4; ++v) acc[u][v] = 0.0;
    if (grp < NGRP) {
      for (int r = grp; r < nloc; r += NGRP) {
        const double* q = Qd + r * LDQ;
        const double2 a0 = *reinterpret_cast<const double2*>(q + 4 * ti4);
        const double2 a1 = *reinterpret_cast<const double2*>(q + 4 * ti4 + 2);
        const double2 b0 = *reinterpret_cast<const double2*>(q + 4 * tj4);
        const double2 b1 = *reinterpret_cast<const double2*>(q + 4 * tj4 + 2);
        const double aa[4] = {a0.x, a0.y, a1.x, a1.y}, bb[4] = {b0.x, b0.y, b1.x, b1.y};
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
          for (int v = 0; v < 4; ++v) acc[u][v] = fma(aa[u], bb[v], acc[u][v]);
      }
#pragma unroll
      for (int u = 0; u < 4; ++u)
#pragma unroll
        for (int v = 0; v < 4; ++v) Gpart[grp * GSET + (4 * ti4 + u) + (4 * tj4 + v) * CB] = acc[u][v];
    }
    __syncthreads();
    for (int e = tid; e < GSET; e += CF_THREADS) {
      const int p = e % CB, q = e / CB;
      double s = 0.0;
      if (p <= q)
        for (int g2 = 0; g2 < NGRP; ++g2) s += Gpart[g2 * GSET + e];
      Gpart[e] = s;
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncthreads();
    if (tid == 0 && nloc > 0) {
      double* dst = gsets + ((size_t)set * NCOPY + cta % NCOPY) * GSET;
      asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f64 [%0], [%1], %2;" ::"l"(dst),
                   "r"(smem_u32(Gpart)), "r"((unsigned)(GSET * sizeof(double)))
                   : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    }
    __syncthreads();
  };
  auto gram_read = [&](int set) {   // -> Gk (upper, ld B+1)
    const double* Gs = gsets + (size_t)set * NCOPY * GSET;
    for (int e = tid; e < GSET; e += CF_THREADS) {
      const int i = e % CB, j = e / CB;
      double g = 0.0;
      if (i <= j)
#pragma unroll
        for (int kk = 0; kk < NCOPY; ++kk) g += __ldcg(Gs + (size_t)kk * GSET + e);
      Gk[i + j * (CB + 1)] = g;
    }
    __syncthreads();
  };
  // Qd rows <- Qd rows * Rinv (upper triangular, row-major fp64): q_c = sum_{k<=c} q_k Rinv[k][c]
  auto apply_rinv = [&]() {
    for (int r = tid; r < nloc; r += CF_THREADS) {
      double* q = Qd + r * LDQ;
      double x[CB];
#pragma unroll
      for (int p = 0; p < CB; p += 2) {
        const double2 v = *reinterpret_cast<const double2*>(q + p);
        x[p] = v.x;
        x[p + 1] = v.y;
      }
#pragma unroll 1
      for (int cc = 0; cc < CB; ++cc) {   // q_c = sum_{k<=c} x_k Rinv[k][c] (x: the original row)
        const double2* rt = reinterpret_cast<const double2*>(RinvT + cc * CB);
        double s0 = 0.0, s1 = 0.0;
#pragma unroll
        for (int kk = 0; kk < CB; kk += 2) {
          const double2 r2 = rt[kk / 2];   // zeros above the diagonal of R^-1: no predicate needed
          s0 = fma(x[kk], r2.x, s0);
          s1 = fma(x[kk + 1], r2.y, s1);
        }
        q[cc] = s0 + s1;
      }
    }
    __syncthreads();
  };
  // the panel's top B rows (OA rows tb .. tb+B) times Riacc -> Q1 (every CTA, from the fp32 GA in A)
  float* P1s = Linv;   // (free until the LU) top rows of the panel, fp32 B x B row-major
  auto top_rows_q1 = [&]() {
    constexpr int U = CB * CB / CF_THREADS;
    float v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int e = tid + u * CF_THREADS;
      const int i = e % CB, kk = e / CB;
      v[u] = (tb + i < M) ? __ldcg(&Acol(tb + i, kk)) : 0.f;
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int e = tid + u * CF_THREADS;
      P1s[(e % CB) * CB + e / CB] = v[u];
    }
    __syncthreads();
    {   // 4 entries per thread (rows i, i + 8, i + 16, i + 24 of column cc): 4 interleaved chains
      const int cc = tid % CB, i0 = tid / CB;
      double s4[4] = {0.0, 0.0, 0.0, 0.0};
#pragma unroll 4
      for (int kk = 0; kk < CB; ++kk) {
        const double rk = (kk <= cc) ? Riacc[kk * CB + cc] : 0.0;
#pragma unroll
        for (int u = 0; u < 4; ++u) s4[u] = fma((double)P1s[(i0 + 8 * u) * CB + kk], rk, s4[u]);
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) Q1[(i0 + 8 * u) * CB + cc] = s4[u];
    }
    __syncthreads();
  };

  stamp(4);
  bool accepted = false;
  int rounds_done = 0;
  if (m >= CB) {
    // round 0
    gram_arrive(0);
    stamp(5);
    gbar();   // 2
    stamp(6);
    gram_read(0);
    stamp(15);
    const bool ok0 = cta_chol64(Gk, RR, rd, 0.0, reinterpret_cast<double*>(ring + D_TMP));
    stamp(16);
    if (ok0) {
      cta_inv_upper<double, 4>(RR, rd, Rinv, RinvT, reinterpret_cast<double*>(ring + D_TMP), 0);
      stamp(17);
      for (int e = tid; e < CB * CB; e += CF_THREADS) {
        Riacc[e] = Rinv[e];
        Racc[e] = RR[e];
      }
      apply_rinv();
      stamp(18);
      rounds_done = 1;
      for (int rnd = 1; rnd < MAX_ROUNDS; ++rnd) {
        gram_arrive(rnd);
        if (rnd == 1) stamp(7);
        // speculative (valid if this round's check passes): Q_1 and its LU, L^-1, U^-1 -- every
        // CTA redundantly, overlapping the barrier's latency
        top_rows_q1();
        if (rnd == 1) stamp(19);
        cta_lu(Q1, Ls, Us, Ss, Dinv, reinterpret_cast<float*>(ring + D_TMP), reinterpret_cast<float*>(ring + D_TMP) + 2 * CB);
        if (rnd == 1) stamp(20);
        // U^-1 (transposed: column c contiguous) on threads 0-127, L^-1 on 128-255, same barriers
        cta_inv_both32(Us, Dinv, Uinv, Ls, Linv, reinterpret_cast<float*>(ring + D_TMP));   // Uinv holds (U^-1)^T
        if (rnd == 1) stamp(8);
        gbar();   // 3 (rnd 1)
        if (rnd == 1) stamp(9);
        gram_read(rnd);
        if (rnd == 1) stamp(21);
        double dev = 0.0;
        for (int e = tid; e < GSET; e += CF_THREADS) {
          const int i = e % CB, j = e / CB;
          if (i <= j) dev = fmax(dev, fabs(Gk[i + j * (CB + 1)] - (i == j ? 1.0 : 0.0)));
        }
        if (!__syncthreads_or(!(dev <= a.orth_tol))) {
          accepted = true;
          break;
        }
        if (rnd == MAX_ROUNDS - 1) break;
        if (!cta_chol64(Gk, RR, rd, 0.0, reinterpret_cast<double*>(ring + D_TMP))) break;
        cta_inv_upper<double, 4>(RR, rd, Rinv, RinvT, reinterpret_cast<double*>(ring + D_TMP), 0);
        // Riacc <- Riacc Rinv ; Racc <- RR Racc  (upper triangular products)
        for (int e = tid; e < CB * CB; e += CF_THREADS) {
          const int i = e / CB, j = e % CB;
          double s1 = 0.0, s2 = 0.0;
          for (int kk = i; kk <= j; ++kk) {
            s1 = fma(Riacc[i * CB + kk], Rinv[kk * CB + j], s1);
            s2 = fma(RR[i * CB + kk], Racc[kk * CB + j], s2);
          }
          Q1[e] = s1;          // temporaries
          Gpart[e] = s2;
        }
        __syncthreads();
        for (int e = tid; e < CB * CB; e += CF_THREADS) {
          Riacc[e] = Q1[e];
          Racc[e] = Gpart[e];
        }
        apply_rinv();
        rounds_done = rnd + 1;
      }
    }
  }
  (void)rounds_done;

  const int64_t ldk = a.ldk;
  if (accepted) {
    // ---- reconstruction rows: w = (e_il - q S) L^-T, y = q U^-1 (il >= B) or L row (il < B)
    float* Ystage = reinterpret_cast<float*>(ring + D_GPART);   // nloc x 33 (the Gram partials are dead)
    for (int r = tid; r < nloc; r += CF_THREADS) {
      const int64_t gr = P0 + r;         // OA row
      const int64_t il = gr - tb;        // panel row
      const double* qrow = Qd + r * LDQ;
      float q[CB], v[CB];
#pragma unroll
      for (int p = 0; p < CB; ++p) {
        q[p] = (float)qrow[p];
        v[p] = ((il == p) ? 1.f : 0.f) - q[p] * Ss[p];
      }
      __half* wr = a.Wrh + gr * ldk + tb;
      float* ys = Ystage + r * 33;
#pragma unroll 1
      for (int cc = 0; cc < CB; ++cc) {
        // w_c = sum_k v_k Linv[c][k]  (w = (e_il - q S) L^-T; Linv row c is zero beyond c)
        const float4* l4 = reinterpret_cast<const float4*>(Linv + cc * CB);
        float s0 = 0.f, s1 = 0.f;
#pragma unroll
        for (int kk = 0; kk < CB; kk += 4) {
          const float4 lv = l4[kk / 4];
          s0 = fmaf(v[kk], lv.x, s0);
          s1 = fmaf(v[kk + 1], lv.y, s1);
          s0 = fmaf(v[kk + 2], lv.z, s0);
          s1 = fmaf(v[kk + 3], lv.w, s1);
        }
        const float w = s0 + s1;
        // y_c = sum_k q_k Uinv[k][c] (il >= B; Uinv holds (U^-1)^T, zero beyond c), L[il][c] (il < B)
        float y;
        if (il < CB) {
          y = Ls[il * CB + cc];
        } else {
          const float4* u4 = reinterpret_cast<const float4*>(Uinv + cc * CB);
          float t0 = 0.f, t1 = 0.f;
#pragma unroll
          for (int kk = 0; kk < CB; kk += 4) {
            const float4 uv = u4[kk / 4];
            t0 = fmaf(q[kk], uv.x, t0);
            t1 = fmaf(q[kk + 1], uv.y, t1);
            t0 = fmaf(q[kk + 2], uv.z, t0);
            t1 = fmaf(q[kk + 3], uv.w, t1);
          }
          y = t0 + t1;
        }
        a.Wt[gr + (int64_t)cc * a.ldw] = w;
        a.Wh[gr + (int64_t)cc * a.ldwh] = __float2half_rn(w);
        a.Yb[gr + (tb + cc) * a.ldy] = y;
        ys[cc] = y;
        if (t == 0) wr[cc] = __float2half_rn(w);
        // compact panel: Y strictly below the diagonal, R_h = S R on and above (top rows)
        Acol(gr, cc) = (il > cc) ? y : (float)((double)Ss[il < CB ? il : 0] * Racc[(il < CB ? il : 0) * CB + cc]);
      }
    }
    __syncthreads();
    for (int e = tid; e < nloc * (CB / 8); e += CF_THREADS) {   // Yh rows: 16-byte stores
      const int r = e / (CB / 8), g8 = e % (CB / 8);
      __align__(16) __half hv[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) hv[u] = __float2half_rn(Ystage[r * 33 + g8 * 8 + u]);
      *reinterpret_cast<uint4*>(a.Yh + (P0 + r) * ldk + tb + g8 * 8) = *reinterpret_cast<const uint4*>(hv);
    }
  } else {
    // ---- Householder QR fallback (rank deficient / not orthonormal; or m < B): dgeqr2 in fp64
    //      over the CTA-distributed rows, 2 grid barriers per column; Y = V, W^0 = V T, R_h = R
    if (m >= CB && cta == 0 && tid == 0) atomicAdd(a.declines, 1u);   // a CholeskyQR decline (m < B: direct)
    // reload the panel (Qd may hold Q of a CholeskyQR round)
    for (int e = tid; e < nloc * CB; e += CF_THREADS) {
      const int p = e / nloc, lr = e % nloc;
      Qd[lr * LDQ + p] = (double)__ldcg(&Acol(P0 + lr, p));
    }
    __syncthreads();
    if (m < CB) gbar();                  // (no barrier yet: the scratch zeroing must be complete)
    double* hhn = hhs;                   // [B] column norms^2 ; [B] alpha ; [B x B] w rows
    double* hha = hhs + CB;
    double* hhw = hhs + 2 * CB;
    double* tau = Rinv;                  // smem: tau[B], beta[B]
    double* beta = Rinv + CB;
    const int ncols = (int)std::min<int64_t>(CB, m);
    for (int j = 0; j < CB; ++j) {
      if (j >= ncols) {   // no rows left: H = I
        if (tid == 0) { tau[j] = 0.0; beta[j] = 0.0; }
        continue;
      }
      // (1) sigma^2 = ||x[j+1:]||^2, alpha = x[j]
      double s = 0.0;
      for (int r = tid; r < nloc; r += CF_THREADS) {
        const int64_t il = P0 + r - tb;
        const double xv = Qd[r * LDQ + j];
        if (il > j) s = fma(xv, xv, s);
        if (il == j) hha[j] = xv;
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
      if (lane == 0 && s != 0.0) atomicAdd(&hhn[j], s);
      gbar();
      const double sig2 = __ldcg(&hhn[j]), alpha = __ldcg(&hha[j]);
      double tj, bj, scal;
      if (sig2 <= 0.0) { tj = 0.0; bj = alpha; scal = 0.0; }
      else {
        const double nrm = sqrt(fma(alpha, alpha, sig2));
        bj = alpha >= 0.0 ? -nrm : nrm;
        tj = (bj - alpha) / bj;
        scal = 1.0 / (alpha - bj);
      }
      if (tid == 0) { tau[j] = tj; beta[j] = bj; }
      // (2) v = x[j:] scaled (v_j = 1); partial w_c = sum_i v_i x_ic (c > j)
      for (int r = tid; r < nloc; r += CF_THREADS) {
        const int64_t il = P0 + r - tb;
        if (il > j) Qd[r * LDQ + j] *= scal;
      }
      __syncthreads();
      for (int cc = j + 1 + warp; cc < CB; cc += 8) {
        double ws = 0.0;
        for (int r = lane; r < nloc; r += 32) {
          const int64_t il = P0 + r - tb;
          if (il >= j) ws = fma(il == j ? 1.0 : Qd[r * LDQ + j], Qd[r * LDQ + cc], ws);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) ws += __shfl_xor_sync(0xffffffffu, ws, o);
        if (lane == 0 && ws != 0.0) atomicAdd(&hhw[j * CB + cc], ws);
      }
      gbar();
      // (3) x[:, c] -= tau v w_c
      for (int r = tid; r < nloc; r += CF_THREADS) {
        const int64_t il = P0 + r - tb;
        if (il < j) continue;
        const double vi = (il == j) ? 1.0 : Qd[r * LDQ + j];
        for (int cc = j + 1; cc < CB; ++cc) Qd[r * LDQ + cc] = fma(-tj * vi, __ldcg(&hhw[j * CB + cc]), Qd[r * LDQ + cc]);
      }
      __syncthreads();
    }
    // T (dlarft, forward columnwise): T_jj = tau_j, T[0:j, j] = -tau_j T[0:j,0:j] (V[:,0:j]^T v_j);
    // V^T V over all rows: one more reduction (set 0 of the Gram sets, reused: zero first)
    // R (upper, B x B): rows il < B of Qd hold R above the diagonal after elimination
    // V^T V partial (Gram of V with unit diagonal / zeros above) into hhw (reused, zeroed by host? no:
    // accumulate into the upper half region after the w rows: hh + 2B + B*B)
    double* hvv = hhs + 2 * CB + CB * CB;
    // V^T V (strict upper): thread = (i, j) pair, sum over the CTA's rows, one atomic per pair
    for (int e = tid; e < CB * CB; e += CF_THREADS) {
      const int i = e / CB, j = e % CB;
      if (j <= i) continue;
      double sv = 0.0;
      for (int r = 0; r < nloc; ++r) {
        const int64_t il = P0 + r - tb;
        if (il < j) continue;   // v_j is zero above row j
        const double vi = (il == i) ? 1.0 : (il > i ? Qd[r * LDQ + i] : 0.0);
        const double vj = (il == j) ? 1.0 : Qd[r * LDQ + j];
        sv = fma(vi, vj, sv);
      }
      if (sv != 0.0) atomicAdd(&hvv[i * CB + j], sv);
    }
    // R rows (panel rows il < B live on the CTA holding rows tb .. tb+B)
    for (int r = tid; r < nloc; r += CF_THREADS) {
      const int64_t il = P0 + r - tb;
      if (il < CB)
        for (int p = 0; p < CB; ++p) Racc[il * CB + p] = (p > il) ? Qd[r * LDQ + p] : 0.0;
    }
    gbar();
    // every CTA: T (B x B upper, dlarft) from V^T V and tau -> Riacc (reused as T, row-major);
    // column j: T[0:j, j] = -tau_j T[0:j, 0:j] (V^T v_j), lane i computes row i
    for (int e = tid; e < CB * CB; e += CF_THREADS) {
      Q1[e] = __ldcg(&hvv[e]);
      Riacc[e] = 0.0;
    }
    __syncthreads();
    if (warp == 0) {
      double* T = Riacc;
      for (int j = 0; j < CB; ++j) {
        double sacc = 0.0;
        if (lane < j)
          for (int l = lane; l < j; ++l) sacc = fma(T[lane * CB + l], Q1[l * CB + j], sacc);
        __syncwarp();
        if (lane < j) T[lane * CB + j] = -tau[j] * sacc;
        if (lane == j) T[j * CB + j] = tau[j];
        __syncwarp();
      }
    }
    __syncthreads();
    const double* T = Riacc;
    for (int r = tid; r < nloc; r += CF_THREADS) {
      const int64_t gr = P0 + r;
      const int64_t il = gr - tb;
      // Y = V (written first), then W^0 = V T in place (w_c = sum_{k<=c} v_k T[k][c], high c first)
      for (int p = 0; p < CB; ++p) {
        const double vp = (il == p) ? 1.0 : (il > p ? Qd[r * LDQ + p] : 0.0);
        const float y = (float)vp;
        a.Yb[gr + (tb + p) * a.ldy] = y;
        a.Yh[gr * ldk + tb + p] = __float2half_rn(y);
        Acol(gr, p) = (il > p) ? y : (il == p ? (float)beta[p] : 0.f);   // R above: below
      }
      for (int cc = CB - 1; cc >= 0; --cc) {
        double s = 0.0;
        for (int kk = 0; kk <= cc; ++kk) {
          const double vk = (il == kk) ? 1.0 : (il > kk ? Qd[r * LDQ + kk] : 0.0);
          s = fma(vk, T[kk * CB + cc], s);
        }
        const float w = (float)s;
        a.Wt[gr + (int64_t)cc * a.ldw] = w;
        a.Wh[gr + (int64_t)cc * a.ldwh] = __float2half_rn(w);
        if (t == 0) a.Wrh[gr * ldk + tb + cc] = __float2half_rn(w);
      }
    }
    __syncthreads();
    // R above the diagonal (rows il < B, on their CTA)
    for (int e = tid; e < nloc * CB; e += CF_THREADS) {
      const int r = e / CB, p = e % CB;
      const int64_t il = P0 + r - tb;
      if (il < CB && p > il) Acol(P0 + r, p) = (float)Racc[il * CB + p];
    }
  }

  stamp(10);
  if (t >= 1) {   // (t = 0: W_0 = W^0, nothing above the panel)
  gbar();   // W^0 (Wh) visible to every CTA's TMA
  stamp(11);

  // =====================================================================================
  // Phase E: G = Y_{<t}^T W^0, H = X_{<t}^T W^0 over rows [tb, M): CTA = (k-slab, row chunk)
  // =====================================================================================
  {
    const int nsl = (k + 127) / 128;
    const int nch = max(1, G / nsl);
    const int64_t chunk = ((m + nch - 1) / nch + 63) / 64 * 64;
    const int sl = cta % nsl, ch = cta / nsl;
    const bool active = cta < nsl * nch;
    const int64_t rb = tb + (int64_t)ch * chunk;
    const int64_t re = std::min<int64_t>(M, rb + chunk);
    const int nks = active && re > rb ? (int)((re - rb + 63) / 64) : 0;
    constexpr uint32_t BYTES = 2 * 16384 + CB * 64 * 2;
    if (warp == 0 && lane == 0) {
      for (int ks = 0; ks < nks; ++ks) {
        const int r = (int)(rb + ks * 64);
        mbar_wait(&empty[p_st], p_ph ^ 1);
        mbar_expect_tx(&full[p_st], BYTES);
        uint8_t* sa = ring + p_st * RING_STAGE;
        for (int hh2 = 0; hh2 < 2; ++hh2) {
          tma_load_2d(sa + hh2 * 8192, &mYe, &full[p_st], sl * 128 + hh2 * 64, r);
          tma_load_2d(sa + 16384 + hh2 * 8192, &mXe, &full[p_st], sl * 128 + hh2 * 64, r);
        }
        tma_load_2d(sa + 32768, &mWe, &full[p_st], r, 0);
        if (++p_st == RING_NS) { p_st = 0; p_ph ^= 1; }
      }
    } else if (warp == 1 && lane == 0) {
      if (nks > 0) {
        constexpr uint32_t idesc = idesc_make(128, CB, 0, 1, 0);
        const uint32_t s0 = smem_u32(ring);
        mbar_wait(&acce[m_ab], m_aph ^ 1);
        tc_fence_after();
        const uint32_t d0 = tmem + 64 * m_ab, d1 = d0 + 32;
        for (int ks = 0; ks < nks; ++ks) {
          mbar_wait(&full[m_st], m_ph);
          tc_fence_after();
          const uint32_t sa = s0 + m_st * RING_STAGE, sb = sa + 32768;
#pragma unroll
          for (int s = 0; s < 4; ++s) {
            const uint64_t bd = sdesc_sw128(sb + s * 32, 16, 1024);
            mma_f16(d0, sdesc_sw128(sa + s * 2048, 8192, 1024), bd, idesc, (ks > 0 || s > 0) ? 1u : 0u);
            mma_f16(d1, sdesc_sw128(sa + 16384 + s * 2048, 8192, 1024), bd, idesc, (ks > 0 || s > 0) ? 1u : 0u);
          }
          mma_commit(&empty[m_st]);
          if (++m_st == RING_NS) { m_st = 0; m_ph ^= 1; }
        }
        mma_commit(&accf[m_ab]);
        if (++m_ab == 2) { m_ab = 0; m_aph ^= 1; }
      }
    } else if (warp >= 4) {
      if (nks > 0) {
        const int qw = warp - 4;
        const int j = sl * 128 + qw * 32 + lane;
        mbar_wait(&accf[e_ab], e_aph);
        tc_fence_after();
        float g[32], hv[32];
        tmem_ld32(tmem + 64 * e_ab + ((uint32_t)(qw * 32) << 16), g);
        tmem_ld32(tmem + 64 * e_ab + 32 + ((uint32_t)(qw * 32) << 16), hv);
        tc_fence_before();
        mbar_arrive(&acce[e_ab]);
        if (++e_ab == 2) { e_ab = 0; e_aph ^= 1; }
        // the slab's 128 x B partials of G and H -> shared (row-major, as in Gf / Hf) -> two bulk
        // fp32 reductions (rows >= k are zero: their Y / X columns are TMA out-of-bounds fills)
        float* Gst = reinterpret_cast<float*>(smem + OFF_QD);
        float* Hst = Gst + 128 * CB;
        const int jl = qw * 32 + lane;
#pragma unroll
        for (int p = 0; p < CB; p += 4) {
          *reinterpret_cast<float4*>(Gst + jl * CB + p) = make_float4(g[p], g[p + 1], g[p + 2], g[p + 3]);
          *reinterpret_cast<float4*>(Hst + jl * CB + p) = make_float4(hv[p], hv[p + 1], hv[p + 2], hv[p + 3]);
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile("bar.sync 1, 128;" ::: "memory");   // the 4 epilogue warps
        if (qw == 0 && lane == 0) {
          asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f32 [%0], [%1], %2;" ::"l"(
                           a.Gf + (size_t)sl * 128 * CB),
                       "r"(smem_u32(Gst)), "r"((unsigned)(128 * CB * sizeof(float)))
                       : "memory");
          asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f32 [%0], [%1], %2;" ::"l"(
                           a.Hf + (size_t)sl * 128 * CB),
                       "r"(smem_u32(Hst)), "r"((unsigned)(128 * CB * sizeof(float)))
                       : "memory");
          asm volatile("cp.async.bulk.commit_group;" ::: "memory");
          asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
        }
        (void)j;
      }
    }
  }
  gbar();   // 5: G, H complete
  stamp(12);

  // =====================================================================================
  // Phase F: W_{<t}^T X_t = H - (W^T X) G  (column block t of W^T X and its mirror)
  // Phase G: W_t = W^0 - W_{<t} G on rows [0, M)  (+ Y, Yh zero above the panel)
  // =====================================================================================
  {
    float* Gs = reinterpret_cast<float*>(ring);                  // k x B fp32 (row-major)
    float* Wcs = reinterpret_cast<float*>(smem + OFF_QD);        // the CTA's WtX columns (8 x k)
    const int q0 = cta * 8, nq = std::max(0, std::min(8, k - q0));
    stage_cols(Gs, CB, a.Gf, CB, CB, k);
    if (nq > 0) stage_cols(Wcs, k, a.WtX + (int64_t)q0 * a.ldwx, a.ldwx, k, nq);
    __syncthreads();
    stamp(23);
    // phase F: rows q of this CTA (WtX column q is contiguous: symmetric)
    {
      const float hv = (warp < nq) ? __ldcg(a.Hf + (int64_t)(q0 + warp) * CB + lane) : 0.f;
      const float dot = cta_rows_dot(Wcs, k, nq, Gs, reinterpret_cast<float*>(smem + OFF_QD) + 8 * 1024 + 64);
      if (warp < nq) {
        const int q = q0 + warp, p = lane;
        const float v = hv - dot;
        a.WtX[q + (int64_t)(k + p) * a.ldwx] = v;
        a.WtX[(k + p) + (int64_t)q * a.ldwx] = v;
      }
    }
    __syncthreads();   // Wcs dead: Gh takes the Qd region
    stamp(24);
    // Gh (B x k, K-major, SWIZZLE_128B, 64-column chunks of 4 KB) resident in the Qd region
    uint8_t* Gh = smem + OFF_QD;
    const int kc0 = (k + 63) / 64;
    for (int e = tid; e < kc0 * 64 * CB; e += CF_THREADS) {
      const int n = e % CB, kg = e / CB;   // n fastest: conflict-free reads of Gs
      const int kc = kg / 64, kk = kg % 64;
      const float v = kg < k ? Gs[kg * CB + n] : 0.f;
      *reinterpret_cast<__half*>(Gh + kc * 4096 + sw128_off(n, kk)) = __float2half_rn(v);
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // Gh (generic writes) -> MMA reads
    __syncthreads();
    stamp(13);
    // phase G tiles: rows [0, M), <= 2 per CTA
    const int ntg = (int)((M + 127) / 128);
    const int tpg = (ntg + G - 1) / G;
    const int g0 = min(ntg, cta * tpg), g1 = min(ntg, g0 + tpg);
    if (warp == 0 && lane == 0) {
      for (int ti = g0; ti < g1; ++ti)
        for (int kc = 0; kc < kc0; ++kc) {
          mbar_wait(&empty[p_st], p_ph ^ 1);
          mbar_expect_tx(&full[p_st], 16384);
          tma_load_2d(ring + p_st * RING_STAGE, &mWg, &full[p_st], kc * 64, ti * 128);
          if (++p_st == RING_NS) { p_st = 0; p_ph ^= 1; }
        }
    } else if (warp == 1 && lane == 0) {
      constexpr uint32_t idesc = idesc_make(128, CB, 0, 0, 0);
      const uint32_t s0 = smem_u32(ring), sg = smem_u32(Gh);
      for (int ti = g0; ti < g1; ++ti) {
        mbar_wait(&acce[m_ab], m_aph ^ 1);
        tc_fence_after();
        const uint32_t d = tmem + 64 * m_ab;
        for (int kc = 0; kc < kc0; ++kc) {
          mbar_wait(&full[m_st], m_ph);
          tc_fence_after();
          const uint32_t sa = s0 + m_st * RING_STAGE, sb = sg + kc * 4096;
#pragma unroll
          for (int s = 0; s < 4; ++s)
            mma_f16(d, sdesc_sw128(sa + s * 32, 16, 1024), sdesc_sw128(sb + s * 32, 16, 1024), idesc,
                    (kc > 0 || s > 0) ? 1u : 0u);
          mma_commit(&empty[m_st]);
          if (++m_st == RING_NS) { m_st = 0; m_ph ^= 1; }
        }
        mma_commit(&accf[m_ab]);
        if (++m_ab == 2) { m_ab = 0; m_aph ^= 1; }
      }
    } else if (warp >= 4) {
      const int qw = warp - 4;
      for (int ti = g0; ti < g1; ++ti) {
        const int64_t r = (int64_t)ti * 128 + qw * 32 + lane;
        const bool in = r < M;
        float w0[CB];
#pragma unroll
        for (int p = 0; p < CB; ++p) w0[p] = (in && r >= tb) ? a.Wt[r + (int64_t)p * a.ldw] : 0.f;
        mbar_wait(&accf[e_ab], e_aph);
        tc_fence_after();
        float acc[32];
        tmem_ld32(tmem + 64 * e_ab + ((uint32_t)(qw * 32) << 16), acc);
        tc_fence_before();
        mbar_arrive(&acce[e_ab]);
        if (++e_ab == 2) { e_ab = 0; e_aph ^= 1; }
        if (in) {
          __align__(16) __half hv[CB];
#pragma unroll
          for (int p = 0; p < CB; ++p) {
            const float v = w0[p] - acc[p];
            hv[p] = __float2half_rn(v);
            a.Wt[r + (int64_t)p * a.ldw] = v;
            a.Wh[r + (int64_t)p * a.ldwh] = hv[p];
          }
#pragma unroll
          for (int p = 0; p < CB; p += 8)
            *reinterpret_cast<uint4*>(a.Wrh + r * ldk + tb + p) = *reinterpret_cast<const uint4*>(hv + p);
          if (r < tb) {   // Y_t is zero above the panel
            const __half z = __float2half_rn(0.f);
#pragma unroll
            for (int p = 0; p < CB; ++p) {
              a.Yb[r + (tb + p) * a.ldy] = 0.f;
              a.Yh[r * ldk + tb + p] = z;
            }
          }
        }
      }
    }
  }

  }   // t >= 1
  stamp(14);

  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    tc_fence_after();
    tmem_dealloc(tmem, 128);
  }
}

// ---------------------------------------------------------------------------------- host
size_t chain_fused_ws_bytes() { return 2 * WS_PARITY; }

bool chain_fused_supported(int b, int64_t M, int num_sms) {
  if (b != CB) return false;
  return (M + 127) / 128 <= 2 * (int64_t)num_sms;   // rows of phases C / D fit 2 tiles per CTA
}

cudaError_t launch_chain_fused(const ChainFusedLaunch& L, cudaStream_t st) {
  cudaError_t e = func_attr((const void*)chain_fused_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, CF_SMEM);
  if (e != cudaSuccess) return e;
  const int kk = std::max(L.k, 1);
  CUtensorMap mXc, mYc, mYb, mPh, mXe, mYe, mWe, mWg;
  if ((e = make_tmap_2d(&mXc, L.Xh, true, kk, L.M, L.ldk, 64, 128)) != cudaSuccess) return e;
  if ((e = make_tmap_2d(&mYc, L.Yh, true, kk, L.M, L.ldk, 64, 128)) != cudaSuccess) return e;
  if ((e = make_tmap_2d(&mYb, L.Yh, true, kk, L.M, L.ldk, 64, CB)) != cudaSuccess) return e;
  if ((e = make_tmap_2d(&mPh, L.Ph, true, kk, CB, L.ldk, 64, CB)) != cudaSuccess) return e;
  if ((e = make_tmap_2d(&mXe, L.Xh, true, kk, L.M, L.ldk, 64, 64)) != cudaSuccess) return e;
  if ((e = make_tmap_2d(&mYe, L.Yh, true, kk, L.M, L.ldk, 64, 64)) != cudaSuccess) return e;
  if ((e = make_tmap_2d(&mWe, L.Wh, true, L.M, CB, L.ldwh, 64, CB)) != cudaSuccess) return e;
  if ((e = make_tmap_2d(&mWg, L.Wrh, true, kk, L.M, L.ldk, 64, 128)) != cudaSuccess) return e;
  ChainFusedArgs a{};
  a.t = L.t;
  a.k = L.k;
  a.M = L.M;
  a.tb = L.tb;
  a.c = L.tb - CB;
  a.A = L.A;
  a.lda = L.lda;
  a.r0 = L.r0;
  a.Yb = L.Yb;
  a.ldy = L.ldy;
  a.Wt = L.Wt;
  a.ldw = L.ldw;
  a.Xb = L.Xb;
  a.ldx = L.ldx;
  a.WtX = L.WtX;
  a.ldwx = L.ldwx;
  a.Gf = L.Gf;
  a.Hf = L.Hf;
  a.Ph = L.Ph;
  a.Yh = L.Yh;
  a.Wrh = L.Wrh;
  a.ldk = L.ldk;
  a.Wh = L.Wh;
  a.ldwh = L.ldwh;
  a.Xh = L.Xh;
  a.ws_cur = reinterpret_cast<uint8_t*>(L.ws) + (L.launch & 1u) * WS_PARITY;
  a.ws_next = reinterpret_cast<uint8_t*>(L.ws) + ((L.launch + 1) & 1u) * WS_PARITY;
  a.declines = L.declines;
  a.trace = L.trace;
  a.orth_tol = L.orth_tol > 0 ? L.orth_tol : 1e-6;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(L.grid);
  cfg.blockDim = dim3(CF_THREADS);
  cfg.dynamicSmemBytes = CF_SMEM;
  cfg.stream = st;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = 1;
  at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl_enabled() ? 2 : 1;
  return cudaLaunchKernelEx(&cfg, chain_fused_kernel, mXc, mYc, mYb, mPh, mXe, mYe, mWe, mWg, a);
}

}  // namespace sbr
