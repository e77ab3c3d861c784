// Micro-benchmark: cycles of small fp64/fp32 building blocks on one warp / one CTA.
#include <cstdio>
#include <cuda_runtime.h>
#define SBR_DEV __device__ __forceinline__
SBR_DEV int lane_id() { return threadIdx.x & 31; }

__global__ void k_dfma_chain(double* out, long long* cyc, int n) {
  double a = threadIdx.x * 1e-3, b = 1.0000001;
  long long t0 = clock64();
  for (int i = 0; i < n; ++i) a = fma(a, b, 1e-9);
  long long t1 = clock64();
  out[threadIdx.x] = a;
  if (threadIdx.x == 0) cyc[0] = (t1 - t0) / n;
}
__global__ void k_dfma_tput(double* out, long long* cyc, int n) {
  double a[8];
  for (int k = 0; k < 8; ++k) a[k] = threadIdx.x * 1e-3 + k;
  long long t0 = clock64();
  for (int i = 0; i < n; ++i)
#pragma unroll
    for (int k = 0; k < 8; ++k) a[k] = fma(a[k], 1.0000001, 1e-9);
  long long t1 = clock64();
  double s = 0; for (int k = 0; k < 8; ++k) s += a[k];
  out[threadIdx.x + blockIdx.x * blockDim.x] = s;
  if (threadIdx.x == 0 && blockIdx.x == 0) cyc[1] = (t1 - t0);
}
__global__ void k_ffma_tput(float* out, long long* cyc, int n) {
  float a[8];
  for (int k = 0; k < 8; ++k) a[k] = threadIdx.x * 1e-3f + k;
  long long t0 = clock64();
  for (int i = 0; i < n; ++i)
#pragma unroll
    for (int k = 0; k < 8; ++k) a[k] = fmaf(a[k], 1.0000001f, 1e-9f);
  long long t1 = clock64();
  float s = 0; for (int k = 0; k < 8; ++k) s += a[k];
  out[threadIdx.x + blockIdx.x * blockDim.x] = s;
  if (threadIdx.x == 0 && blockIdx.x == 0) cyc[2] = (t1 - t0);
}
__global__ void k_sqrt_rcp(double* out, long long* cyc, int n) {
  double a = 2.0 + threadIdx.x;
  long long t0 = clock64();
  for (int i = 0; i < n; ++i) a = sqrt(a) + 1.0;
  long long t1 = clock64();
  double c = 2.0 + threadIdx.x;
  long long t2 = clock64();
  for (int i = 0; i < n; ++i) c = __drcp_rn(c) + 1.0;
  long long t3 = clock64();
  out[threadIdx.x] = a + c;
  if (threadIdx.x == 0) { cyc[3] = (t1 - t0) / n; cyc[4] = (t3 - t2) / n; }
}
__global__ void k_bar(long long* cyc, int n) {
  long long t0 = clock64();
  for (int i = 0; i < n; ++i) __syncthreads();
  long long t1 = clock64();
  if (threadIdx.x == 0) cyc[5] = (t1 - t0) / n;
}
__global__ void k_shfl(double* out, long long* cyc, int n) {
  double v = threadIdx.x;
  long long t0 = clock64();
  for (int i = 0; i < n; ++i) v = __shfl_xor_sync(0xffffffffu, v, 1) + 1.0;
  long long t1 = clock64();
  float f = threadIdx.x;
  long long t2 = clock64();
  for (int i = 0; i < n; ++i) f = __shfl_xor_sync(0xffffffffu, f, 1) + 1.0f;
  long long t3 = clock64();
  out[threadIdx.x] = v + f;
  if (threadIdx.x == 0) { cyc[6] = (t1 - t0) / n; cyc[7] = (t3 - t2) / n; }
}
__global__ void k_lds(double* out, long long* cyc, int n) {
  __shared__ double s[1024];
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) s[i] = i;
  __syncthreads();
  int idx = threadIdx.x;
  long long t0 = clock64();
  for (int i = 0; i < n; ++i) idx = (int)s[idx & 1023] + 1;
  long long t1 = clock64();
  out[threadIdx.x] = idx;
  if (threadIdx.x == 0) cyc[8] = (t1 - t0) / n;
}
int main() {
  double* od; float* of; long long* cyc;
  cudaMalloc(&od, 1 << 24); cudaMalloc(&of, 1 << 24); cudaMallocManaged(&cyc, 64 * 8);
  const int n = 4096;
  k_dfma_chain<<<1, 32>>>(od, cyc, n);
  k_dfma_tput<<<148, 256>>>(od, cyc, n);
  k_ffma_tput<<<148, 256>>>(of, cyc, n);
  k_sqrt_rcp<<<1, 32>>>(od, cyc, 256);
  k_bar<<<1, 256>>>(cyc, n);
  k_shfl<<<1, 32>>>(od, cyc, n);
  k_lds<<<1, 32>>>(od, cyc, n);
  cudaDeviceSynchronize();
  printf("dfma latency %lld cyc\n", cyc[0]);
  printf("dfma tput: %.2f DFMA/clk/SM (256 thr x 8 chains)\n", 256.0 * 8 * n / cyc[1]);
  printf("ffma tput: %.2f FFMA/clk/SM\n", 256.0 * 8 * n / cyc[2]);
  printf("sqrt(double)+add latency %lld, drcp_rn+add %lld\n", cyc[3], cyc[4]);
  printf("syncthreads(256) %lld cyc\n", cyc[5]);
  printf("shfl f64 %lld, shfl f32 %lld (incl add)\n", cyc[6], cyc[7]);
  printf("lds f64 dependent %lld\n", cyc[8]);
  return 0;
}
