// Micro-benchmark: one-warp b x b factorizations (Cholesky fp64, modified LU fp32) as used by
// the CholeskyQR panel kernel -- cycles per call for several code shapes.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr \
//      -I paper_conf_ppopp_zhangsoyw23_b200/csrc tools/ubench/ubench_fact.cu -o tools/ubench/ubench_fact
#include <cstdio>
#include <vector>
#include <cmath>
#include "../../paper_conf_ppopp_zhangsoyw23_b200/csrc/k_panel_chol.cu"

using namespace sbr;
constexpr int B = 32, LDG = 33;

// V2: rolled step loop, row broadcast through shared memory (double2 reads)
SBR_DEV bool chol_v2(double* G, double* Rrm, double* rd, double* rrow) {
  const int lane = lane_id();
  double g[B];
#pragma unroll
  for (int i = 0; i < B; ++i) g[i] = (i <= lane) ? G[i + lane * LDG] : 0.0;
  double piv = __shfl_sync(0xffffffffu, g[0], 0);
  bool ok = true;
#pragma unroll 1
  for (int j = 0; j < B; ++j) {
    ok = ok && piv > 0.0;
    const double r = rsqrt(fmax(piv, 1e-300));
    const double rjc = g[0] * r;
    Rrm[j * B + lane] = (lane >= j) ? rjc : 0.0;
    if (lane == j) rd[j] = r;
    const double pn = fma(-rjc, rjc, g[1]);
    piv = __shfl_sync(0xffffffffu, pn, (j + 1) & 31);
    rrow[lane] = rjc;
    __syncwarp();
    // g[k-1] = g[k] - rrow[j+k] * rjc : rrow index dynamic -> read rows j+1.. via pointer
    const double* rr = rrow + j;
#pragma unroll
    for (int k0 = 1; k0 < B; k0 += 8) {
      if (j + k0 < B) {
#pragma unroll
        for (int k = k0; k < k0 + 8 && k < B; ++k) g[k - 1] = fma(-rr[k], rjc, g[k]);
      }
    }
    g[B - 1] = 0.0;
    __syncwarp();
  }
  return __all_sync(0xffffffffu, ok);
}

// V3: fully unrolled, shuffles (the round-1 first version)
SBR_DEV bool chol_v3(double* G, double* Rrm, double* rd) {
  const int lane = lane_id();
  double g[B];
#pragma unroll
  for (int i = 0; i < B; ++i) g[i] = (i <= lane) ? G[i + lane * LDG] : 0.0;
  bool ok = true;
  double piv = __shfl_sync(0xffffffffu, g[0], 0);
  double rdl = 0.0;
#pragma unroll
  for (int j = 0; j < B; ++j) {
    ok = ok && piv > 0.0;
    const double r = rsqrt(fmax(piv, 1e-300));
    const double rjc = g[j] * r;
    g[j] = rjc;
    if (lane == j) rdl = r;
    if (j + 1 < B) piv = __shfl_sync(0xffffffffu, fma(-rjc, rjc, g[j + 1]), j + 1);
#pragma unroll
    for (int i = j + 1; i < B; ++i) g[i] = fma(-__shfl_sync(0xffffffffu, rjc, i), rjc, g[i]);
  }
  rd[lane] = rdl;
#pragma unroll
  for (int i = 0; i < B; ++i) Rrm[i * B + lane] = (i <= lane) ? g[i] : 0.0;
  return __all_sync(0xffffffffu, ok);
}

// V4: rolled, smem broadcast, but the rsqrt replaced by fp32 MUFU + 2 Newton steps
SBR_DEV double rsqrt_fast(double x) {
  double y = (double)rsqrtf((float)x);
  y = y * fma(-0.5 * x * y, y, 1.5);
  y = y * fma(-0.5 * x * y, y, 1.5);
  return y;
}
SBR_DEV bool chol_v4(double* G, double* Rrm, double* rd, double* rrow) {
  const int lane = lane_id();
  double g[B];
#pragma unroll
  for (int i = 0; i < B; ++i) g[i] = (i <= lane) ? G[i + lane * LDG] : 0.0;
  double piv = __shfl_sync(0xffffffffu, g[0], 0);
  bool ok = true;
#pragma unroll 1
  for (int j = 0; j < B; ++j) {
    ok = ok && piv > 0.0;
    const double r = rsqrt_fast(fmax(piv, 1e-300));
    const double rjc = g[0] * r;
    Rrm[j * B + lane] = (lane >= j) ? rjc : 0.0;
    if (lane == j) rd[j] = r;
    const double pn = fma(-rjc, rjc, g[1]);
    piv = __shfl_sync(0xffffffffu, pn, (j + 1) & 31);
    rrow[lane] = rjc;
    __syncwarp();
    const double* rr = rrow + j;
#pragma unroll
    for (int k0 = 1; k0 < B; k0 += 8) {
      if (j + k0 < B) {
#pragma unroll
        for (int k = k0; k < k0 + 8 && k < B; ++k) g[k - 1] = fma(-rr[k], rjc, g[k]);
      }
    }
    g[B - 1] = 0.0;
    __syncwarp();
  }
  return __all_sync(0xffffffffu, ok);
}


// V5: fully unrolled, row broadcast through shared memory, next pivot first
SBR_DEV bool chol_v5(double* G, double* Rrm, double* rd, double* rrow) {
  const int lane = lane_id();
  double g[B];
#pragma unroll
  for (int i = 0; i < B; ++i) g[i] = (i <= lane) ? G[i + lane * LDG] : 0.0;
  bool ok = true;
  double piv = __shfl_sync(0xffffffffu, g[0], 0);
#pragma unroll
  for (int j = 0; j < B; ++j) {
    ok = ok && piv > 0.0;
    const double r = rsqrt(fmax(piv, 1e-300));
    const double rjc = g[j] * r;
    g[j] = rjc;
    if (j + 1 < B) piv = __shfl_sync(0xffffffffu, fma(-rjc, rjc, g[j + 1]), j + 1);
    if (lane == j) rd[j] = r;
    rrow[lane] = rjc;
    __syncwarp();
#pragma unroll
    for (int i = j + 1; i < B; ++i) g[i] = fma(-rrow[i], rjc, g[i]);
    __syncwarp();
  }
#pragma unroll
  for (int i = 0; i < B; ++i) Rrm[i * B + lane] = (i <= lane) ? g[i] : 0.0;
  return __all_sync(0xffffffffu, ok);
}
// LU V4: fully unrolled, smem L column broadcast
SBR_DEV void lu_v4(const double* Q1, float* Lcol, float* Urow, float* Ss, float* dinv, float* lrow) {
  const int lane = lane_id();
  float col[B];
#pragma unroll
  for (int i = 0; i < B; ++i) col[i] = (float)Q1[i * 34 + lane];
  float d = __shfl_sync(0xffffffffu, col[0], 0);
#pragma unroll
  for (int j = 0; j < B; ++j) {
    const float sj = (d >= 0.f) ? -1.f : 1.f;
    const float piv = d - sj;
    const float inv = __fdividef(1.f, piv);
    if (lane == j) {
      col[j] = piv;
#pragma unroll
      for (int i = j + 1; i < B; ++i) lrow[i] = col[i] * inv;
      Ss[j] = sj; dinv[j] = inv;
    }
    if (j + 1 < B) {
      const float l1 = __shfl_sync(0xffffffffu, col[j + 1], j) * inv;
      d = __shfl_sync(0xffffffffu, fmaf(-l1, col[j], col[j + 1]), j + 1);
    }
    __syncwarp();
    if (lane > j) {
      const float ujc = col[j];
#pragma unroll
      for (int i = j + 1; i < B; ++i) col[i] = fmaf(-lrow[i], ujc, col[i]);
    }
    if (lane == j) {
#pragma unroll
      for (int i = j + 1; i < B; ++i) col[i] = lrow[i];
    }
    __syncwarp();
  }
#pragma unroll
  for (int i = 0; i < B; ++i) {
    Urow[i * B + lane] = (i <= lane) ? col[i] : 0.f;
    Lcol[lane * B + i] = (i > lane) ? col[i] : (i == lane ? 1.f : 0.f);
  }
}

__global__ void k_chol(const double* Gin, double* Rout, long long* cyc, int variant, int nwarps_active) {
  __shared__ double G[B * LDG], Rrm[B * B], rd[B], rrow[2 * B];
  for (int e = threadIdx.x; e < B * B; e += blockDim.x) G[(e % B) + (e / B) * LDG] = Gin[e];
  if (threadIdx.x < 2 * B) rrow[threadIdx.x] = 0.0;
  __syncthreads();
  bool ok = true;
  long long t0 = 0, t1 = 0;
  for (int rep = 0; rep < 2; ++rep) {   // second call: instruction cache warm
    __syncthreads();
    t0 = clock64();
    if (threadIdx.x < 32 * nwarps_active && (threadIdx.x >> 5) == 0) {
      if (variant == 1) ok = warp_chol<B, LDG>(G, Rrm, rd, 0.0);
      if (variant == 2) ok = chol_v2(G, Rrm, rd, rrow);
      if (variant == 3) ok = chol_v3(G, Rrm, rd);
      if (variant == 4) ok = chol_v4(G, Rrm, rd, rrow);
      if (variant == 5) ok = chol_v5(G, Rrm, rd, rrow);
    }
    __syncthreads();
    t1 = clock64();
    if (threadIdx.x == 0) cyc[rep] = t1 - t0;
    for (int e = threadIdx.x; e < B * B; e += blockDim.x) G[(e % B) + (e / B) * LDG] = Gin[e];
  }
  if (threadIdx.x == 0) cyc[2] = ok;
  for (int e = threadIdx.x; e < B * B; e += blockDim.x) Rout[e] = Rrm[e];
}

// LU variants
SBR_DEV void lu_v3(const double* Q1, float* Lcol, float* Urow, float* Ss, float* dinv) {   // unrolled shfl
  const int lane = lane_id();
  float col[B];
#pragma unroll
  for (int i = 0; i < B; ++i) col[i] = (float)Q1[i * 34 + lane];
  float d = __shfl_sync(0xffffffffu, col[0], 0);
  float sl = 0.f, dl = 0.f;
#pragma unroll
  for (int j = 0; j < B; ++j) {
    const float sj = (d >= 0.f) ? -1.f : 1.f;
    const float piv = d - sj;
    const float inv = __fdividef(1.f, piv);
    if (lane == j) { col[j] = piv; sl = sj; dl = inv; }
    const float ujc = col[j];
#pragma unroll
    for (int i = j + 1; i < B; ++i) {
      const float li = __shfl_sync(0xffffffffu, col[i], j) * inv;
      const float nv = fmaf(-li, ujc, col[i]);
      col[i] = (lane > j) ? nv : ((lane == j) ? li : col[i]);
      if (i == j + 1) d = __shfl_sync(0xffffffffu, col[j + 1], j + 1);
    }
  }
  Ss[lane] = sl; dinv[lane] = dl;
#pragma unroll
  for (int i = 0; i < B; ++i) {
    Urow[i * B + lane] = (i <= lane) ? col[i] : 0.f;
    Lcol[lane * B + i] = (i > lane) ? col[i] : (i == lane ? 1.f : 0.f);
  }
}
// V2: rolled, L column broadcast through smem
SBR_DEV void lu_v2(const double* Q1, float* Lcol, float* Urow, float* Ss, float* dinv, float* lrow) {
  const int lane = lane_id();
  float col[B];
#pragma unroll
  for (int i = 0; i < B; ++i) col[i] = (float)Q1[i * 34 + lane];
#pragma unroll 1
  for (int j = 0; j < B; ++j) {
    const float d = __shfl_sync(0xffffffffu, col[0], j);
    const float sj = (d >= 0.f) ? -1.f : 1.f;
    const float piv = d - sj;
    const float inv = __fdividef(1.f, piv);
    const float ujc = (lane == j) ? piv : col[0];
    Urow[j * B + lane] = (lane >= j) ? ujc : 0.f;
    Lcol[lane * B + j] = (lane < j) ? col[0] : (lane == j ? 1.f : 0.f);
    if (lane == j) { Ss[j] = sj; dinv[j] = inv; }
    if (lane == j) {
#pragma unroll
      for (int k = 1; k < B; ++k) lrow[k] = col[k] * inv;
    }
    __syncwarp();
#pragma unroll
    for (int k0 = 1; k0 < B; k0 += 8) {
      if (j + k0 < B) {
#pragma unroll
        for (int k = k0; k < k0 + 8 && k < B; ++k) {
          const float lk = lrow[k];
          col[k - 1] = (lane > j) ? fmaf(-lk, ujc, col[k]) : ((lane == j) ? lk : col[k]);
        }
      }
    }
    col[B - 1] = 0.f;
    __syncwarp();
  }
}

__global__ void k_lu(const double* Qin, float* Lout, float* Uout, long long* cyc, int variant) {
  __shared__ double Q[B * 34];
  __shared__ float Lc[B * B], Ur[B * B], Ss[B], Di[B], lrow[2 * B];
  for (int e = threadIdx.x; e < B * B; e += blockDim.x) Q[(e / B) * 34 + e % B] = Qin[e];
  if (threadIdx.x < 2 * B) lrow[threadIdx.x] = 0.f;
  __syncthreads();
  for (int rep = 0; rep < 2; ++rep) {
    __syncthreads();
    long long t0 = clock64();
    if ((threadIdx.x >> 5) == 0) {
      if (variant == 1) warp_lu<B, 34>(Q, Lc, Ur, Ss, Di);
      if (variant == 2) lu_v2(Q, Lc, Ur, Ss, Di, lrow);
      if (variant == 3) lu_v3(Q, Lc, Ur, Ss, Di);
      if (variant == 4) lu_v4(Q, Lc, Ur, Ss, Di, lrow);
    }
    __syncthreads();
    long long t1 = clock64();
    if (threadIdx.x == 0) cyc[rep] = t1 - t0;
  }
  for (int e = threadIdx.x; e < B * B; e += blockDim.x) { Lout[e] = Lc[e]; Uout[e] = Ur[e]; }
}

int main() {
  std::vector<double> X(64 * B), G(B * B), Q(B * B);
  srand(1);
  for (auto& x : X) x = (rand() / (double)RAND_MAX) - 0.5;
  for (int i = 0; i < B; ++i)
    for (int j = 0; j < B; ++j) {
      double s = 0;
      for (int r = 0; r < 64; ++r) s += X[r * B + i] * X[r * B + j];
      G[i + j * B] = s;
    }
  for (int e = 0; e < B * B; ++e) Q[e] = (rand() / (double)RAND_MAX) - 0.5;
  double *dG, *dR, *dQ;
  float *dL, *dU;
  long long* dc;
  cudaMalloc(&dG, 8 * B * B); cudaMalloc(&dR, 8 * B * B); cudaMalloc(&dQ, 8 * B * B);
  cudaMalloc(&dL, 4 * B * B); cudaMalloc(&dU, 4 * B * B); cudaMalloc(&dc, 32);
  cudaMemcpy(dG, G.data(), 8 * B * B, cudaMemcpyHostToDevice);
  cudaMemcpy(dQ, Q.data(), 8 * B * B, cudaMemcpyHostToDevice);
  std::vector<double> Rref(B * B);
  for (int v = 1; v <= 5; ++v)
    for (int threads : {256}) {
      long long c[3];
      for (int rep = 0; rep < 3; ++rep) k_chol<<<1, threads>>>(dG, dR, dc, v, 1);
      cudaDeviceSynchronize();
      cudaMemcpy(c, dc, 24, cudaMemcpyDeviceToHost);
      std::vector<double> R(B * B);
      cudaMemcpy(R.data(), dR, 8 * B * B, cudaMemcpyDeviceToHost);
      if (v == 1 && threads == 32) Rref = R;
      double err = 0;
      for (int e = 0; e < B * B; ++e) err = fmax(err, fabs(R[e] - Rref[e]));
      printf("chol v%d threads %3d: cold %6lld warm %6lld cycles ok=%lld  max|R-R_v1| %.1e  (%s)\n", v, threads, c[0], c[1], c[2], err,
             cudaGetErrorString(cudaGetLastError()));
    }
  std::vector<float> Lref(B * B), Uref(B * B);
  for (int v = 1; v <= 4; ++v) {
    long long c[2];
    for (int rep = 0; rep < 3; ++rep) k_lu<<<1, 256>>>(dQ, dL, dU, dc, v);
    cudaDeviceSynchronize();
    cudaMemcpy(c, dc, 16, cudaMemcpyDeviceToHost);
    std::vector<float> L(B * B), U(B * B);
    cudaMemcpy(L.data(), dL, 4 * B * B, cudaMemcpyDeviceToHost);
    cudaMemcpy(U.data(), dU, 4 * B * B, cudaMemcpyDeviceToHost);
    if (v == 1) { Lref = L; Uref = U; }
    double err = 0;
    for (int e = 0; e < B * B; ++e) err = fmax(err, fmax(fabs(L[e] - Lref[e]), fabs(U[e] - Uref[e])));
    printf("lu   v%d: cold %6lld warm %6lld cycles  max|LU - v1| %.1e (%s)\n", v, c[0], c[1], err, cudaGetErrorString(cudaGetLastError()));
  }
  return 0;
}
