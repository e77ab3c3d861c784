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
//  * eigenvalues by bisection on Sturm counts, one thread per eigenvalue index.
//
// Parallel schedule (the standard pipelined bulge chase): sweep s+1 step k touches only
// entries that sweep s has finished with once sweep s completed its step k+2 (the footprints
// of sweep s step k+3 and of sweep s+1 step k are disjoint: rows >= s+1+(k+3)b vs
// <= s+1+(k+2)b), so each sweep is one warp-sized worker that waits on a per-sweep progress
// counter of its predecessor and publishes its own (release/acquire at gpu scope).  Workers
// take sweeps round-robin; the launch is cooperative so every worker is resident (a worker
// only ever waits on a lower sweep, held by a running worker: no deadlock).
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

// smem doubles per worker: west, diag, south (b x (b+1) each) + v + w
__host__ __device__ inline int s2_worker_doubles(int b) { return 3 * b * (b + 1) + 2 * b; }

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

// Load an L x L symmetric block (lower part read from the band, mirrored) or an Ls x L general
// block into row-major smem (stride ld).  Eight loads in flight per lane.
SBR_DEV void load_diag(double* Dg, int ld, const double* Wk, int64_t ldw, int64_t r0, int L, int lane) {
  const int total = L * L;
  for (int e0 = 0; e0 < total; e0 += 32 * 8) {
    double t[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int e = e0 + u * 32 + lane;
      const int c = e / L, r = e - c * L;
      t[u] = (e < total && r >= c) ? __ldcg(Wk + (r - c) + (r0 + c) * ldw) : 0.0;
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int e = e0 + u * 32 + lane;
      const int c = e / L, r = e - c * L;
      if (e < total && r >= c) {
        Dg[r * ld + c] = t[u];
        Dg[c * ld + r] = t[u];
      }
    }
  }
}

// block rows q0 .. q0+Lr-1, columns c0 .. c0+Lc-1 with q0 - c0 = off (>= 1): band offset off + r - c
SBR_DEV void load_block(double* S, int ld, const double* Wk, int64_t ldw, int64_t c0, int off, int Lr, int Lc,
                        int lane) {
  const int total = Lr * Lc;
  for (int e0 = 0; e0 < total; e0 += 32 * 8) {
    double t[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int e = e0 + u * 32 + lane;
      const int c = e / Lr, r = e - c * Lr;
      t[u] = e < total ? __ldcg(Wk + (off + r - c) + (c0 + c) * ldw) : 0.0;
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int e = e0 + u * 32 + lane;
      const int c = e / Lr, r = e - c * Lr;
      if (e < total) S[r * ld + c] = t[u];
    }
  }
}

SBR_DEV void store_block(const double* S, int ld, double* Wk, int64_t ldw, int64_t c0, int off, int Lr, int Lc,
                         int lane) {
  const int total = Lr * Lc;
  for (int e = lane; e < total; e += 32) {
    const int c = e / Lr, r = e - c * Lr;
    Wk[(off + r - c) + (c0 + c) * ldw] = S[r * ld + c];
  }
}

__global__ void __launch_bounds__(128) s2_chase_kernel(int64_t n, int b, double* __restrict__ Wk, int64_t ldw,
                                                       int* __restrict__ prog) {
  extern __shared__ double s2_smem[];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, wpc = blockDim.x >> 5;
  const int ld = b + 1;
  double* base = s2_smem + (size_t)wid * s2_worker_doubles(b);
  double* Wst = base;               // west  A[R_k, R_{k-1}]   (k = 0: column s only)
  double* Dg = base + b * ld;       // diag  A[R_k, R_k]       (full symmetric)
  double* So = base + 2 * b * ld;   // south A[R_{k+1}, R_k]
  double* v = base + 3 * b * ld;    // reflector H = I - tau v v^T, v[0] = 1
  double* w = v + b;
  const int64_t nsweeps = n - 2;
  const int64_t nworkers = (int64_t)gridDim.x * wpc;
  for (int64_t s = (int64_t)blockIdx.x * wpc + wid; s < nsweeps; s += nworkers) {
    const int64_t nst = (n - 3 - s) / b + 1;                       // steps with |R_k| >= 2
    const int64_t nprev = s > 0 ? (n - 3 - (s - 1)) / b + 1 : 0;
    for (int64_t k = 0; k < nst; ++k) {
      const int64_t r0 = s + 1 + k * b;                            // R_k = r0 .. r0+L-1
      const int L = (int)std::min<int64_t>(b, n - r0);
      const int wc = k == 0 ? 1 : b;                               // west columns
      const int64_t q0 = r0 + b;                                   // R_{k+1} = q0 .. q0+Ls-1
      const int Ls = (int)std::max<int64_t>(0, std::min<int64_t>(b, n - q0));
      if (s > 0) {
        if (lane == 0) {
          const int need = (int)std::min<int64_t>(k + 3, nprev);       // sweep s-1 finished step k+2
          while (ld_acquire_s32(prog + s - 1) < need) __nanosleep(40);
        }
        __syncwarp();
      }
      if (k == 0)
        for (int r = lane; r < L; r += 32) Wst[r * ld] = __ldcg(Wk + (1 + r) + s * ldw);
      load_diag(Dg, ld, Wk, ldw, r0, L, lane);
      if (Ls > 0) load_block(So, ld, Wk, ldw, r0, b, Ls, L, lane);
      __syncwarp();
      // reflector annihilating the pivot column below its first entry (dlarfg convention)
      double sig = 0.0;
      for (int r = 1 + lane; r < L; r += 32) {
        const double x = Wst[r * ld];
        sig += x * x;
      }
      sig = warp_sum_d(sig);
      const double alpha = Wst[0];
      double tau = 0.0, beta = alpha;
      if (sig > 0.0) {
        const double nrm = sqrt(alpha * alpha + sig);
        beta = alpha >= 0.0 ? -nrm : nrm;
        tau = (beta - alpha) / beta;
        const double scal = 1.0 / (alpha - beta);
        for (int r = lane; r < L; r += 32) v[r] = r == 0 ? 1.0 : Wst[r * ld] * scal;
      }
      __syncwarp();
      if (tau != 0.0) {
        for (int r = lane; r < L; r += 32) Wst[r * ld] = r == 0 ? beta : 0.0;
        // west: the other columns of R_{k-1} (left application) -- the fill later sweeps remove
        for (int c = 1 + lane; c < wc; c += 32) {
          double y = 0.0;
          for (int r = 0; r < L; ++r) y += v[r] * Wst[r * ld + c];
          y *= tau;
          for (int r = 0; r < L; ++r) Wst[r * ld + c] -= v[r] * y;
        }
        // diag: H D H = D - v w^T - w v^T, p = tau D v, w = p - (tau/2)(p^T v) v
        double pv = 0.0;
        for (int i = lane; i < L; i += 32) {
          double p = 0.0;
          for (int j = 0; j < L; ++j) p += Dg[i * ld + j] * v[j];
          p *= tau;
          w[i] = p;
          pv += p * v[i];
        }
        const double K = 0.5 * tau * warp_sum_d(pv);
        for (int i = lane; i < L; i += 32) w[i] -= K * v[i];
        __syncwarp();
        for (int i = lane; i < L; i += 32) {
          const double vi = v[i], wi = w[i];
          for (int j = 0; j < L; ++j) Dg[i * ld + j] -= vi * w[j] + wi * v[j];
        }
        // south: S H = S - tau (S v) v^T
        for (int i = lane; i < Ls; i += 32) {
          double q = 0.0;
          for (int j = 0; j < L; ++j) q += So[i * ld + j] * v[j];
          q *= tau;
          for (int j = 0; j < L; ++j) So[i * ld + j] -= q * v[j];
        }
        __syncwarp();
        // write back: west, diag (lower), south
        if (k == 0) {
          for (int r = lane; r < L; r += 32) Wk[(1 + r) + s * ldw] = Wst[r * ld];
        } else {
          store_block(Wst, ld, Wk, ldw, r0 - b, b, L, b, lane);
        }
        for (int e = lane; e < L * L; e += 32) {
          const int c = e / L, r = e - c * L;
          if (r >= c) Wk[(r - c) + (r0 + c) * ldw] = Dg[r * ld + c];
        }
        if (Ls > 0) store_block(So, ld, Wk, ldw, r0, b, Ls, L, lane);
      }
      __syncwarp();
      if (lane == 0) {
        __threadfence();
        st_release_s32(prog + s, (int)(k + 1));
      }
      // the next step's west block is this step's south block (same entries, already final
      // for sweep s-1: see the header)
      double* t = Wst;
      Wst = So;
      So = t;
      __syncwarp();
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
// T - x I) > k, by halving [lo - tol, hi + tol] until its width is <= tol = 2 eps max(|lo|,|hi|);
// a pivot below pivmin = DBL_MIN max(1, scale^2) in magnitude is replaced by -pivmin
__global__ void __launch_bounds__(128) s2_bisect_kernel(int64_t n, const double* __restrict__ d,
                                                        const double* __restrict__ e2,
                                                        const double* __restrict__ bnd, double* __restrict__ lam) {
  const int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= n) return;
  const double lo_b = bnd[0], hi_b = bnd[1];
  const double scale = fmax(bnd[2], 1e-300);
  const double pivmin = 2.2250738585072014e-308 * fmax(1.0, scale * scale);
  const double span = fmax(fmax(fabs(lo_b), fabs(hi_b)), 1e-300);
  const double tol = 2.0 * 2.220446049250313e-16 * span;
  double lo = lo_b - tol, hi = hi_b + tol;
  for (int it = 0; it < 200 && !(hi - lo <= tol); ++it) {
    const double x = 0.5 * (lo + hi);
    double q = d[0] - x;
    if (fabs(q) < pivmin) q = -pivmin;
    int64_t cnt = q < 0.0;
    for (int64_t i = 1; i < n; ++i) {
      q = __dsub_rn(__dsub_rn(d[i], x), __ddiv_rn(e2[i - 1], q));
      if (fabs(q) < pivmin) q = -pivmin;
      cnt += q < 0.0;
    }
    if (cnt > k)
      hi = x;
    else
      lo = x;
  }
  lam[k] = 0.5 * (lo + hi);
}

}  // namespace

size_t stage2_ws_bytes(int64_t n, int b) {
  const int64_t ldw = 2 * (int64_t)b;
  return ((size_t)n * ldw * sizeof(double) + 255) / 256 * 256 + ((size_t)n * sizeof(int) + 255) / 256 * 256;
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
    const size_t per = sizeof(double) * s2_worker_doubles(b);
    const int wpc = (int)std::max<size_t>(1, std::min<size_t>(4, (200u << 10) / per));
    const size_t smem = per * wpc;
    if ((err = func_attr((const void*)s2_chase_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)) !=
        cudaSuccess)
      return err;
    const int bps = func_blocks_per_sm((const void*)s2_chase_kernel, 32 * wpc, smem);
    if (bps < 1) return cudaErrorInvalidConfiguration;
    const int64_t need = (n - 2 + wpc - 1) / wpc;
    const int grid = (int)std::min<int64_t>(need, (int64_t)bps * nsm);
    void* args[] = {(void*)&n, (void*)&b, (void*)&Wk, (void*)const_cast<int64_t*>(&ldw), (void*)&prog};
    err = cudaLaunchCooperativeKernel((const void*)s2_chase_kernel, dim3(grid), dim3(32 * wpc), args, smem, st);
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
  s2_bisect_kernel<<<(unsigned)((n + 127) / 128), 128, 0, st>>>(n, d, e2, bnd, lam);
  return cudaGetLastError();
}

}  // namespace sbr
