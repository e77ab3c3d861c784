// k_stage2.cu -- stage two of the two-stage symmetric eigensolver on the GPU.
//
// The paper reduces A to a band B (stage one, this library's sbr_reduce), then runs stage two
// -- band -> tridiagonal -> eigenvalues -- on the CPU through MAGMA after a device->host copy
// of the band (Fig. 1; §6.4) and names a GPU stage two as future work
// (P:448).  Here both steps run on the device in fp64:
//
//  * band -> tridiagonal by Householder bulge chasing (the b -> 1 instance of successive band
//    reduction, Fig. 2 with b = 1).  Sweep s annihilates column s below its first
//    sub-diagonal with one reflector on the b rows R_0 = s+1 .. s+b; the reflector's right
//    application fills the block below it (the "bulge"), which step k of the same sweep removes
//    with a reflector on R_k = s+1+kb .. s+(k+1)b that annihilates the first column of the
//    bulge, pushing the rest b rows further down.  One step touches three b x b blocks:
//        west  A[R_k, R_{k-1}]  (left application; its first column is the pivot column)
//        diag  A[R_k, R_k]      (two-sided, H D H as a rank-2 update)
//        south A[R_{k+1}, R_k]  (right application: the next bulge)
//    and the working matrix never has more than 2b-1 sub-diagonals.
//  * eigenvalues by bisection on Sturm counts -- multisection, a group of lanes per
//    eigenvalue index.
//
// Parallel schedule (pipelined bulge chase): sweep s+1 step k shares with sweep s step k+2
// exactly one entry -- the pivot A[first row of R_{k+2}, first row of R_{k+1}] that step k+2
// turns into beta -- and nothing with sweep s steps >= k+3 (rows >= s+1+(k+3)b vs
// <= s+1+(k+2)b).  Each step therefore forms the NEXT step's reflector from its own south block
// (already final) and stores that beta with its results; sweep s+1 step k then only waits for
// sweep s to publish "steps <= k+1 done" on a per-sweep progress counter (release/acquire at gpu
// scope), a lag of two steps.  One CTA (4 warps) per sweep, sweeps round-robin; the launch is
// cooperative so every CTA is resident (a CTA only waits on a lower sweep held by a running
// CTA: no deadlock).  The critical path is about 2 n steps of one CTA.
//
// Layout: the working band Wk (fp64, ldw >= 2b): Wk[d + j*ldw] = A[j+d, j], 0 <= d < 2b.
#include "common.cuh"
#include "kernels.h"

namespace sbr {
namespace {

SBR_DEV int ld_acquire_s32(const int* p) {
  int v;
  asm volatile("ld.acquire.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
SBR_DEV void st_release_s32(int* p, int v) {
  asm volatile("st.release.gpu.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

SBR_DEV double warp_sum_d(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}


__global__ void s2_init_kernel(int64_t n, int b, const float* __restrict__ AB, int64_t ldab, double* __restrict__ Wk,
                               int64_t ldw, int* __restrict__ prog) {
  const int64_t total = n * ldw;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t j = e / ldw;
    const int d = (int)(e - j * ldw);
    Wk[e] = (d <= b && j + d < n) ? (double)AB[d + j * ldab] : 0.0;
    if (d == 0) prog[j] = 0;
  }
}

// Per-worker shared memory: the three b x b blocks of a step (row-major, padded rows), the
// reflector of this step and of the next one, the rank-2 vector w, and per-warp partial sums.
template <int BM>
struct S2Smem {
  double blk[3][BM][BM + 1];   // west / diag / south (west and south swap roles every step)
  double v[2][BM];             // reflector vectors (v[0] = 1), zero beyond the block's rows
  double tb[2][2];             // (tau, beta) of each reflector
  double w[BM];
  double red[3][4][BM];        // partial sums of the 4 warps: west y, diag p, south q
};

// Householder reflector of the column x (entry r = lane + 32h, length L) in the dlarfg
// convention; warp-collective.  Writes v (zero-padded to BM), (tau, beta); returns beta.
template <int BM>
SBR_DEV double householder_warp(const double (&x)[BM / 32], int L, int lane, double* v, double* tb) {
  double sig = 0.0;
#pragma unroll
  for (int h = 0; h < BM / 32; ++h) {
    const int r = lane + 32 * h;
    if (r >= 1 && r < L) sig += x[h] * x[h];
  }
  sig = warp_sum_d(sig);
  const double alpha = __shfl_sync(0xffffffffu, x[0], 0);
  double tau = 0.0, beta = alpha, scal = 0.0;
  if (sig > 0.0) {
    const double nrm = sqrt(alpha * alpha + sig);
    beta = alpha >= 0.0 ? -nrm : nrm;
    tau = (beta - alpha) / beta;
    scal = 1.0 / (alpha - beta);
  }
#pragma unroll
  for (int h = 0; h < BM / 32; ++h) {
    const int r = lane + 32 * h;
    v[r] = r == 0 ? 1.0 : (r < L ? x[h] * scal : 0.0);
  }
  if (lane == 0) {
    tb[0] = tau;
    tb[1] = beta;
  }
  return beta;
}

// One CTA (4 warps) per sweep; sweeps round-robin over the (cooperative, all-resident) grid.
// Step k of sweep s:
//   wait   until sweep s-1 finished its steps <= k+1 and stored the pivot entry of its step k+2
//          (the one entry its step k+2 shares with this step's footprint, written one step early)
//   load   diag A[R_k, R_k] (lower, mirrored) and south A[R_{k+1}, R_k] -- all loads in flight
//          before the first shared-memory write; the west block and this step's reflector are
//          already in shared memory (the previous step's south block and its first column)
//   apply  H_k: west columns 1.. from the left, diag two-sided (rank-2), south from the right
//   next   reflector H_{k+1} from the south block's first column; its (beta, 0, ..) is stored
//          with this step, so sweep s+1 can proceed while step k+1 runs
//   store  west (columns >= 1; column 0 was final one step earlier), diag lower, south; publish.
template <int BM>
__global__ void __launch_bounds__(128) s2_chase_kernel(int64_t n, int b, double* __restrict__ Wk, int64_t ldw,
                                                       int* __restrict__ prog) {
  extern __shared__ __align__(16) unsigned char s2_raw[];
  S2Smem<BM>& sm = *reinterpret_cast<S2Smem<BM>*>(s2_raw);
  constexpr int RPW = BM / 4;    // block rows (west) / columns (diag, south) per warp
  constexpr int LPT = BM / 32;   // lane slots: index lane + 32 h
  const int tid = threadIdx.x, lane = tid & 31, wp = tid >> 5;
  for (int64_t s = blockIdx.x; s < n - 2; s += gridDim.x) {
    const int64_t nst = (n - 3 - s) / b + 1;                       // steps with |R_k| >= 2
    const int64_t nprev = s > 0 ? (n - 3 - (s - 1)) / b + 1 : 0;
    int iw = 0, is = 2, cv = 0;
    for (int64_t k = 0; k < nst; ++k) {
      const int64_t r0 = s + 1 + k * b;                            // R_k = r0 .. r0+L-1
      const int L = (int)std::min<int64_t>(b, n - r0);
      const int Ls = (int)std::max<int64_t>(0, std::min<int64_t>(b, n - r0 - b));   // |R_{k+1}|
      double(*Wb)[BM + 1] = sm.blk[iw];
      double(*Dg)[BM + 1] = sm.blk[1];
      double(*Sb)[BM + 1] = sm.blk[is];
      if (s > 0) {
        if (tid == 0) {
          const int need = (int)std::min<int64_t>(k + 2, nprev);
          while (ld_acquire_s32(prog + s - 1) < need) __nanosleep(20);
        }
        __syncthreads();
      }
      {
        double td[LPT][RPW], ts[LPT][RPW], x[LPT];
        if (k == 0 && wp == 0) {   // pivot column s (rows R_0)
#pragma unroll
          for (int h = 0; h < LPT; ++h) {
            const int r = lane + 32 * h;
            x[h] = r < L ? __ldcg(Wk + (1 + r) + s * ldw) : 0.0;
          }
        }
#pragma unroll
        for (int h = 0; h < LPT; ++h)
#pragma unroll
          for (int i = 0; i < RPW; ++i) {
            const int r = lane + 32 * h, c = wp * RPW + i;
            td[h][i] = (r < L && c < L && r >= c) ? __ldcg(Wk + (r - c) + (r0 + c) * ldw) : 0.0;
            ts[h][i] = (r < Ls && c < L) ? __ldcg(Wk + (b + r - c) + (r0 + c) * ldw) : 0.0;
          }
        if (k == 0 && wp == 0) {   // the first reflector of the sweep
          const double beta = householder_warp<BM>(x, L, lane, sm.v[cv], sm.tb[cv]);
#pragma unroll
          for (int h = 0; h < LPT; ++h) {
            const int r = lane + 32 * h;
            if (r < L) Wb[r][0] = r == 0 ? beta : 0.0;
          }
        }
#pragma unroll
        for (int h = 0; h < LPT; ++h)
#pragma unroll
          for (int i = 0; i < RPW; ++i) {
            const int r = lane + 32 * h, c = wp * RPW + i;
            if (r < L && c < L && r >= c) {
              Dg[r][c] = td[h][i];
              Dg[c][r] = td[h][i];
            }
            if (r < Ls && c < L) Sb[r][c] = ts[h][i];
          }
      }
      __syncthreads();
      const double tau = sm.tb[cv][0];
      const double* v = sm.v[cv];
      if (tau != 0.0) {
        // A: partial sums over this warp's rows (west) / columns (diag, south)
#pragma unroll
        for (int h = 0; h < LPT; ++h) {
          const int c = lane + 32 * h;
          double yw = 0.0, pd = 0.0, qs = 0.0;
#pragma unroll
          for (int i = 0; i < RPW; ++i) {
            const int j = wp * RPW + i;
            if (j < L) {
              const double vj = v[j];
              if (k > 0 && c >= 1 && c < b) yw += vj * Wb[j][c];
              if (c < L) pd += Dg[c][j] * vj;
              if (c < Ls) qs += Sb[c][j] * vj;
            }
          }
          sm.red[0][wp][c] = yw;
          sm.red[1][wp][c] = pd;
          sm.red[2][wp][c] = qs;
        }
        __syncthreads();
        // B: west and south updates; warp 0 forms w = p - (tau/2)(p^T v) v, p = tau D v
#pragma unroll
        for (int h = 0; h < LPT; ++h) {
          const int c = lane + 32 * h;
          const double y = tau * (((sm.red[0][0][c] + sm.red[0][1][c]) + sm.red[0][2][c]) + sm.red[0][3][c]);
          const double q = tau * (((sm.red[2][0][c] + sm.red[2][1][c]) + sm.red[2][2][c]) + sm.red[2][3][c]);
#pragma unroll
          for (int i = 0; i < RPW; ++i) {
            const int j = wp * RPW + i;
            if (j < L) {
              if (k > 0 && c >= 1 && c < b) Wb[j][c] -= v[j] * y;
              if (c < Ls) Sb[c][j] -= q * v[j];
            }
          }
        }
        if (wp == 0) {
          double p[LPT], pv = 0.0;
#pragma unroll
          for (int h = 0; h < LPT; ++h) {
            const int i = lane + 32 * h;
            p[h] = tau * (((sm.red[1][0][i] + sm.red[1][1][i]) + sm.red[1][2][i]) + sm.red[1][3][i]);
            pv += p[h] * v[i];
          }
          const double K = 0.5 * tau * warp_sum_d(pv);
#pragma unroll
          for (int h = 0; h < LPT; ++h) sm.w[lane + 32 * h] = p[h] - K * v[lane + 32 * h];
        }
        __syncthreads();
        // C: diag D <- D - v w^T - w v^T (this warp's columns)
#pragma unroll
        for (int h = 0; h < LPT; ++h) {
          const int i = lane + 32 * h;
          if (i < L) {
            const double vi = v[i], wi = sm.w[i];
#pragma unroll
            for (int t = 0; t < RPW; ++t) {
              const int j = wp * RPW + t;
              if (j < L) Dg[i][j] -= vi * sm.w[j] + wi * v[j];
            }
          }
        }
        __syncthreads();
      }
      const bool more = k + 1 < nst;
      if (more && wp == 0) {   // reflector of step k+1 from the south block's first column
        double x[LPT];
#pragma unroll
        for (int h = 0; h < LPT; ++h) {
          const int r = lane + 32 * h;
          x[h] = r < Ls ? Sb[r][0] : 0.0;
        }
        const double beta = householder_warp<BM>(x, Ls, lane, sm.v[cv ^ 1], sm.tb[cv ^ 1]);
        __syncwarp();
#pragma unroll
        for (int h = 0; h < LPT; ++h) {
          const int r = lane + 32 * h;
          if (r < Ls) Sb[r][0] = r == 0 ? beta : 0.0;
        }
      }
      __syncthreads();
      // stores (lanes along block rows: contiguous in the band)
      if (k == 0) {
        if (tid < L) Wk[(1 + tid) + s * ldw] = Wb[tid][0];
      } else if (tau != 0.0) {
#pragma unroll
        for (int h = 0; h < LPT; ++h)
#pragma unroll
          for (int i = 0; i < RPW; ++i) {
            const int r = lane + 32 * h, c = wp * RPW + i;
            if (r < L && c >= 1 && c < b) Wk[(b + r - c) + (r0 - b + c) * ldw] = Wb[r][c];
          }
      }
#pragma unroll
      for (int h = 0; h < LPT; ++h)
#pragma unroll
        for (int i = 0; i < RPW; ++i) {
          const int r = lane + 32 * h, c = wp * RPW + i;
          if (tau != 0.0 && r < L && c < L && r >= c) Wk[(r - c) + (r0 + c) * ldw] = Dg[r][c];
          if (r < Ls && c < L && (tau != 0.0 || (more && c == 0))) Wk[(b + r - c) + (r0 + c) * ldw] = Sb[r][c];
        }
      __syncthreads();
      if (tid == 0) st_release_s32(prog + s, (int)(k + 1));   // cumulative over the CTA's stores (bar.sync)
      iw ^= 2;
      is ^= 2;
      cv ^= 1;
    }
  }
}


__global__ void s2_extract_kernel(int64_t n, const double* __restrict__ Wk, int64_t ldw, double* __restrict__ d,
                                  double* __restrict__ e) {
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    d[j] = Wk[j * ldw];
    if (j + 1 < n) e[j] = Wk[1 + j * ldw];
  }
}

// Gershgorin bounds and scale of tridiag(d, e): bnd = {lo, hi, max(|d|, |e|)}; e2 = e^2
__global__ void __launch_bounds__(1024) s2_bounds_kernel(int64_t n, const double* __restrict__ d,
                                                         const double* __restrict__ e, double* __restrict__ e2,
                                                         double* __restrict__ bnd) {
  double lo = INFINITY, hi = -INFINITY, mx = 0.0;
  for (int64_t i = threadIdx.x; i < n; i += blockDim.x) {
    const double ae = i + 1 < n ? fabs(e[i]) : 0.0, aep = i > 0 ? fabs(e[i - 1]) : 0.0;
    const double rad = ae + aep;
    lo = fmin(lo, d[i] - rad);
    hi = fmax(hi, d[i] + rad);
    mx = fmax(mx, fmax(fabs(d[i]), ae));
    if (i + 1 < n) e2[i] = e[i] * e[i];
  }
  __shared__ double sl[32], sh[32], sm[32];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    lo = fmin(lo, __shfl_xor_sync(0xffffffffu, lo, o));
    hi = fmax(hi, __shfl_xor_sync(0xffffffffu, hi, o));
    mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  }
  if ((threadIdx.x & 31) == 0) {
    sl[threadIdx.x >> 5] = lo;
    sh[threadIdx.x >> 5] = hi;
    sm[threadIdx.x >> 5] = mx;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int q = 1; q < (int)(blockDim.x >> 5); ++q) {
      lo = fmin(lo, sl[q]);
      hi = fmax(hi, sh[q]);
      mx = fmax(mx, sm[q]);
    }
    bnd[0] = lo;
    bnd[1] = hi;
    bnd[2] = mx;
  }
}

// eigenvalue k of tridiag(d, e): the smallest x with (number of negative LDL^T pivots of
// T - x I) > k.  Multisection: a group of M lanes evaluates the Sturm count at the M interior
// points lo + (hi - lo) (j+1)/(M+1) of the current interval, which shrinks to the sub-interval
// where the count first exceeds k; stop when its width is <= tol = 2 eps max(|lo|, |hi|) of the
// Gershgorin bounds.  (M = 1 is bisection.)  Pivots below pivmin = DBL_MIN max(1, scale^2) in
// magnitude are replaced by -pivmin (LAPACK dstebz).  Both ends keep count(lo) <= k < count(hi);
// the division e^2/q is a refined hardware reciprocal (a few ulps instead of IEEE rounding), so the
// count's transition points may move by a few ulps of the pivots: the result stays within a small
// multiple of tol of the oracle's IEEE bisection.
// e2 / q with a hardware reciprocal estimate refined by two Newton steps and one quotient
// correction (a few ulps; pivots are never subnormal: |q| >= pivmin >= DBL_MIN)
SBR_DEV double sturm_div(double a, double b) {
  double r;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(b));
  double t = fma(-b, r, 1.0);
  r = fma(r, t, r);
  t = fma(-b, r, 1.0);
  r = fma(r, t, r);
  const double q = a * r;
  return fma(r, fma(-b, q, a), q);
}

template <int M>
__global__ void __launch_bounds__(128) s2_multisect_kernel(int64_t n, const double* __restrict__ d,
                                                           const double* __restrict__ e2,
                                                           const double* __restrict__ bnd, double* __restrict__ lam) {
  const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t k = t / M;
  const int j = (int)(t % M);
  if (k >= n) return;   // whole groups exit together (M divides 32 and the block size)
  const unsigned gmask = M == 32 ? 0xffffffffu : (((1u << M) - 1u) << ((threadIdx.x & 31) & ~(M - 1)));
  const int gbase = (threadIdx.x & 31) & ~(M - 1);
  const double lo_b = bnd[0], hi_b = bnd[1];
  const double scale = fmax(bnd[2], 1e-300);
  const double pivmin = 2.2250738585072014e-308 * fmax(1.0, scale * scale);
  const double span = fmax(fmax(fabs(lo_b), fabs(hi_b)), 1e-300);
  const double tol = 2.0 * 2.220446049250313e-16 * span;
  double lo = lo_b - tol, hi = hi_b + tol;
  const double frac = (double)(j + 1) / (double)(M + 1);
  for (int it = 0; it < 200 && !(hi - lo <= tol); ++it) {
    const double x = M == 1 ? 0.5 * (lo + hi) : fmin(hi, fmax(lo, lo + (hi - lo) * frac));
    double q = d[0] - x;
    if (fabs(q) < pivmin) q = -pivmin;
    int64_t cnt = q < 0.0;
    for (int64_t i = 1; i < n; ++i) {
      q = __dsub_rn(__dsub_rn(d[i], x), sturm_div(e2[i - 1], q));
      if (fabs(q) < pivmin) q = -pivmin;
      cnt += q < 0.0;
    }
    if (M == 1) {
      if (cnt > k)
        hi = x;
      else
        lo = x;
    } else {
      const unsigned above = (__ballot_sync(gmask, cnt > k) & gmask) >> gbase;
      const int f = above ? __ffs(above) - 1 : M;           // first point with count > k
      const double xf = __shfl_sync(gmask, x, gbase + (f < M ? f : 0));
      const double xp = __shfl_sync(gmask, x, gbase + (f > 0 ? f - 1 : 0));
      if (f < M) hi = xf;
      if (f > 0) lo = xp;
    }
  }
  if (j == 0) lam[k] = 0.5 * (lo + hi);
}


}  // namespace

size_t stage2_ws_bytes(int64_t n, int b) {
  const int64_t ldw = 2 * (int64_t)b;
  return ((size_t)n * ldw * sizeof(double) + 255) / 256 * 256 + ((size_t)n * sizeof(int) + 255) / 256 * 256;
}

template <int BM>
cudaError_t launch_chase(int64_t n, int b, double* Wk, int64_t ldw, int* prog, int nsm, cudaStream_t st) {
  const size_t smem = sizeof(S2Smem<BM>);
  cudaError_t err = func_attr((const void*)s2_chase_kernel<BM>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (err != cudaSuccess) return err;
  const int bps = func_blocks_per_sm((const void*)s2_chase_kernel<BM>, 128, smem);
  if (bps < 1) return cudaErrorInvalidConfiguration;
  const int grid = (int)std::min<int64_t>(n - 2, (int64_t)bps * nsm);
  void* args[] = {(void*)&n, (void*)&b, (void*)&Wk, (void*)&ldw, (void*)&prog};
  return cudaLaunchCooperativeKernel((const void*)s2_chase_kernel<BM>, dim3(grid), dim3(128), args, smem, st);
}

cudaError_t band_to_tridiag(int64_t n, int b, const float* AB, int64_t ldab, void* ws, double* d, double* e,
                            cudaStream_t st) {
  const int64_t ldw = 2 * (int64_t)b;
  double* Wk = static_cast<double*>(ws);
  int* prog = reinterpret_cast<int*>(static_cast<char*>(ws) + ((size_t)n * ldw * sizeof(double) + 255) / 256 * 256);
  const int nsm = current_device_sms();
  s2_init_kernel<<<nsm * 4, 256, 0, st>>>(n, b, AB, ldab, Wk, ldw, prog);
  cudaError_t err = cudaGetLastError();
  if (err != cudaSuccess) return err;
  if (n > 2 && b > 1) {
    err = b <= 32 ? launch_chase<32>(n, b, Wk, ldw, prog, nsm, st) : launch_chase<64>(n, b, Wk, ldw, prog, nsm, st);
    if (err != cudaSuccess) return err;
  }
  s2_extract_kernel<<<(unsigned)std::min<int64_t>((n + 255) / 256, nsm * 4), 256, 0, st>>>(n, Wk, ldw, d, e);
  return cudaGetLastError();
}

size_t tridiag_eig_ws_bytes(int64_t n) { return ((size_t)std::max<int64_t>(n, 1) * sizeof(double) + 255) / 256 * 256 + 256; }

cudaError_t tridiag_eigenvalues(int64_t n, const double* d, const double* e, void* ws, double* lam, cudaStream_t st) {
  double* e2 = static_cast<double*>(ws);
  double* bnd = reinterpret_cast<double*>(static_cast<char*>(ws) +
                                          ((size_t)std::max<int64_t>(n, 1) * sizeof(double) + 255) / 256 * 256);
  s2_bounds_kernel<<<1, 1024, 0, st>>>(n, d, e, e2, bnd);
  cudaError_t err = cudaGetLastError();
  if (err != cudaSuccess) return err;
  // lanes per eigenvalue: multisection with M points costs M / log2(M+1) times bisection's work,
  // so use just enough lanes (~16 warps per SM) to cover the recurrence's latency
  const int nsm = current_device_sms();
  const int64_t want = (int64_t)nsm * 512 / std::max<int64_t>(n, 1);
  const int M = want >= 32 ? 32 : want >= 16 ? 16 : want >= 8 ? 8 : want >= 4 ? 4 : want >= 2 ? 2 : 1;
  const unsigned grid = (unsigned)((n * M + 127) / 128);
  switch (M) {
    case 32: s2_multisect_kernel<32><<<grid, 128, 0, st>>>(n, d, e2, bnd, lam); break;
    case 16: s2_multisect_kernel<16><<<grid, 128, 0, st>>>(n, d, e2, bnd, lam); break;
    case 8: s2_multisect_kernel<8><<<grid, 128, 0, st>>>(n, d, e2, bnd, lam); break;
    case 4: s2_multisect_kernel<4><<<grid, 128, 0, st>>>(n, d, e2, bnd, lam); break;
    case 2: s2_multisect_kernel<2><<<grid, 128, 0, st>>>(n, d, e2, bnd, lam); break;
    default: s2_multisect_kernel<1><<<grid, 128, 0, st>>>(n, d, e2, bnd, lam); break;
  }
  return cudaGetLastError();
}

}  // namespace sbr
