// Microbenchmark of the b x b CTA routines of k_chain_fused.cu (cycles per call, 256 threads).
#include <cstdio>
#include <vector>
#include <cmath>
#include "../../paper_conf_ppopp_zhangsoyw23_b200/csrc/k_chain_fused.cu"

using namespace sbr;

__global__ void __launch_bounds__(256, 1) tiny_kernel(const double* Gin, double* out, long long* cyc, int reps) {
  __shared__ double Gk[CB * (CB + 1)], RR[CB * CB], rd[CB], RIT[CB * CB], buf[256];
  double* Q1 = RIT;
  __shared__ float L[CB * CB], U[CB * CB], S[CB], dinv[CB], UT[CB * CB], LI[CB * CB];
  __shared__ double Q1s[1];
  for (int e = threadIdx.x; e < CB * CB; e += blockDim.x) RIT[e] = Gin[e % (CB * (CB + 1))] * 0.01 + (e % (CB + 1) == 0 ? 0.5 : 0.0);
  for (int r = 0; r < reps; ++r) {
    for (int e = threadIdx.x; e < CB * (CB + 1); e += blockDim.x) Gk[e] = Gin[e];
    __syncthreads();
    long long t0 = clock64();
    bool ok = cta_chol64(Gk, RR, rd, 0.0, buf);
    long long t1 = clock64();
    cta_inv_upper<double, 4>(RR, rd, nullptr, RIT, buf, 0);
    long long t2 = clock64();
    cta_lu(Q1, L, U, S, dinv, reinterpret_cast<float*>(buf), reinterpret_cast<float*>(buf) + 64);
    long long t3 = clock64();
    cta_inv_both32(U, dinv, UT, L, LI, reinterpret_cast<float*>(buf));
    long long t4 = clock64();
    if (threadIdx.x == 0) {
      cyc[r * 4 + 0] = t1 - t0; cyc[r * 4 + 1] = t2 - t1; cyc[r * 4 + 2] = t3 - t2; cyc[r * 4 + 3] = t4 - t3;
      out[0] = ok ? RR[CB * CB - 1] : -1.0;
    }
    __syncthreads();
  }
  if (threadIdx.x < CB) out[1 + threadIdx.x] = RIT[threadIdx.x] + UT[threadIdx.x] + LI[threadIdx.x];
}

__global__ void __launch_bounds__(256, 1) bar_kernel(long long* cyc) {
  long long t0 = clock64();
  for (int i = 0; i < 32; ++i) __syncthreads();
  long long t1 = clock64();
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
}

int main() {
  std::vector<double> g(CB * (CB + 1), 0.0);
  for (int j = 0; j < CB; ++j)
    for (int i = 0; i <= j; ++i) g[i + j * (CB + 1)] = (i == j) ? CB : 0.3 * std::sin(i * 7 + j * 3);
  double *dg, *dout; long long* dc;
  cudaMalloc(&dg, sizeof(double) * g.size()); cudaMalloc(&dout, 64 * sizeof(double)); cudaMalloc(&dc, 4 * 8 * sizeof(long long));
  cudaMemcpy(dg, g.data(), sizeof(double) * g.size(), cudaMemcpyHostToDevice);
  tiny_kernel<<<1, 256>>>(dg, dout, dc, 8);
  cudaError_t e = cudaDeviceSynchronize();
  long long c[32]; double o[33];
  cudaMemcpy(c, dc, sizeof(c), cudaMemcpyDeviceToHost); cudaMemcpy(o, dout, sizeof(o), cudaMemcpyDeviceToHost);
  printf("err %s  R_last %g\n", cudaGetErrorString(e), o[0]);
  const char* nm[4] = {"cta_chol64", "cta_inv_upper64", "cta_lu", "cta_inv_both32"};
  for (int k = 0; k < 4; ++k) printf("%-18s first %7lld  hot %7lld cycles\n", nm[k], c[k], c[28 + k]);
  bar_kernel<<<1, 256>>>(dc);
  cudaDeviceSynchronize();
  cudaMemcpy(c, dc, 8, cudaMemcpyDeviceToHost);
  printf("32 x __syncthreads (256 thr): %lld cycles\n", c[0]);
  return 0;
}
