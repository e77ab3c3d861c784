// k_misc.cu -- small kernels: input generator, finiteness check, band extraction,
// symmetric mirrors, the k x b correction of the lazy panel update.
#include "common.cuh"
#include "kernels.h"

namespace sbr {

bool pdl_enabled() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("SBR_PDL");
    v = (e && strcmp(e, "0") == 0) ? 0 : 1;
  }
  return v == 1;
}

SBR_DEV uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__global__ void gen_symmetric_kernel(uint64_t seed, int64_t n, int64_t j0, float* A, int64_t lda) {
  const int64_t j = j0 + blockIdx.y;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t hi = (uint64_t)(i > j ? i : j), lo = (uint64_t)(i > j ? j : i);
    const uint64_t h = splitmix64(seed ^ ((hi << 32) | lo));
    const int64_t u = (int64_t)(h >> 40);
    A[i + j * lda] = (float)((double)(u - (1ll << 23)) * (1.0 / 8388608.0));
  }
}

cudaError_t gen_symmetric(uint64_t seed, int64_t n, float* A, int64_t lda, cudaStream_t st) {
  for (int64_t j0 = 0; j0 < n; j0 += 65535) {
    const int64_t nc = std::min<int64_t>(65535, n - j0);
    dim3 grid((unsigned)std::min<int64_t>((n + 255) / 256, 64), (unsigned)nc);
    gen_symmetric_kernel<<<grid, 256, 0, st>>>(seed, n, j0, A, lda);
  }
  return cudaGetLastError();
}

__global__ void check_finite_kernel(int64_t n, const float* A, int64_t lda, unsigned* flag) {
  const int64_t j = blockIdx.y;
  for (int64_t i = j + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    if (!isfinite(A[i + j * lda])) { atomicOr(flag, 1u); return; }
  }
}

cudaError_t check_finite(int64_t n, const float* A, int64_t lda, unsigned* flag, cudaStream_t st) {
  cudaError_t e = cudaMemsetAsync(flag, 0, sizeof(unsigned), st);
  if (e != cudaSuccess) return e;
  for (int64_t j0 = 0; j0 < n; j0 += 65535) {
    const int64_t nc = std::min<int64_t>(65535, n - j0);
    dim3 grid((unsigned)std::min<int64_t>((n + 255) / 256, 16), (unsigned)nc);
    check_finite_kernel<<<grid, 256, 0, st>>>(n - j0, A + j0 + j0 * lda, lda, flag);
  }
  return cudaGetLastError();
}

// Sticky record of a CholeskyQR panel that declined (rank deficient / not orthonormal) when the
// TSQR fallback cannot run (more leaves than co-resident CTAs): *sticky |= *fail.
__global__ void note_unhandled_kernel(const int* fail, unsigned* sticky) {
  pdl_trigger();
  pdl_wait();
  if (threadIdx.x == 0 && *fail) atomicOr(sticky, 1u);
}

cudaError_t note_unhandled(const int* fail, unsigned* sticky, cudaStream_t st) {
  return launch_pdl(note_unhandled_kernel, dim3(1), dim3(32), 0, st, fail, sticky);
}

__global__ void extract_band_kernel(int64_t n, int b, const float* A, int64_t lda, float* AB, int64_t ldab) {
  const int64_t j = (int64_t)blockIdx.x * blockDim.y + threadIdx.y;
  const int d = threadIdx.x;
  if (j >= n || d > b) return;
  AB[d + j * ldab] = (j + d < n) ? A[(j + d) + j * lda] : 0.f;
}

cudaError_t extract_band(int64_t n, int b, const float* A, int64_t lda, float* AB, int64_t ldab, cudaStream_t st) {
  const int dx = b + 1;
  const int dy = max(1, 256 / dx);
  extract_band_kernel<<<(unsigned)((n + dy - 1) / dy), dim3(dx, dy), 0, st>>>(n, b, A, lda, AB, ldab);
  return cudaGetLastError();
}

__global__ void mirror_lower_block_kernel(int b, float* A, int64_t lda) {
  for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
    const int i = e % b, j = e / b;
    if (i < j) A[i + (int64_t)j * lda] = A[j + (int64_t)i * lda];
  }
}

cudaError_t mirror_lower_block(int b, float* A, int64_t lda, cudaStream_t st) {
  mirror_lower_block_kernel<<<1, 256, 0, st>>>(b, A, lda);
  return cudaGetLastError();
}

// P[q, p] = X(c+p, q) - sum_r WtX[q, r] Y(c+p, r)   (k x b), i.e.
// W^T R = X(c,:)^T - (W^T X) Y_c^T   (reading C3/C5)
__global__ void lazy_small_p_kernel(int k, int b, const float* Xc, int64_t ldx, const float* WtX, int64_t ldwx,
                                    const float* Yc, int64_t ldy, float* P) {
  const int q = blockIdx.x * blockDim.x + threadIdx.x;
  const int p = blockIdx.y;
  if (q >= k) return;
  float acc = Xc[p + (int64_t)q * ldx];
  for (int r = 0; r < k; ++r) acc = fmaf(-WtX[q + (int64_t)r * ldwx], Yc[p + (int64_t)r * ldy], acc);
  P[q + (int64_t)p * k] = acc;
}

cudaError_t lazy_small_p(int k, int b, const float* Xc, int64_t ldx, const float* WtX, int64_t ldwx,
                         const float* Yc, int64_t ldy, float* P, cudaStream_t st) {
  dim3 grid((k + 127) / 128, b);
  lazy_small_p_kernel<<<grid, 128, 0, st>>>(k, b, Xc, ldx, WtX, ldwx, Yc, ldy, P);
  return cudaGetLastError();
}

// WtX[k+p, q] = WtX[q, k+p]  for q < k, p < b
__global__ void mirror_wtx_kernel(int k, int b, float* WtX, int64_t ld) {
  const int q = blockIdx.x * blockDim.x + threadIdx.x;
  const int p = blockIdx.y;
  if (q < k) WtX[(k + p) + (int64_t)q * ld] = WtX[q + (int64_t)(k + p) * ld];
}

cudaError_t mirror_wtx(int k, int b, float* WtX, int64_t ld, cudaStream_t st) {
  if (k <= 0) return cudaSuccess;
  mirror_wtx_kernel<<<dim3((k + 127) / 128, b), 128, 0, st>>>(k, b, WtX, ld);
  return cudaGetLastError();
}

cudaError_t zero_matrix(int64_t rows, int64_t cols, float* A, int64_t lda, cudaStream_t st) {
  if (rows <= 0 || cols <= 0) return cudaSuccess;
  return cudaMemset2DAsync(A, lda * sizeof(float), 0, rows * sizeof(float), cols, st);
}

// fp16 shadow of the lower triangle: strict lower as is, HALF the diagonal, zero above
// (so that a diagonal tile T satisfies T + T^T = L; see k_pass_tc.cu).
__global__ void shadow_init_kernel(int64_t n, int64_t j0, const float* A, int64_t lda, __half* Sh, int64_t ldsh) {
  const int64_t j = j0 + blockIdx.y;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    float v = 0.f;
    if (i > j) v = A[i + j * lda];
    else if (i == j) v = 0.5f * A[i + j * lda];
    Sh[i + j * ldsh] = __float2half_rn(v);
  }
}

cudaError_t shadow_init(int64_t n, const float* A, int64_t lda, __half* Sh, int64_t ldsh, cudaStream_t st) {
  for (int64_t j0 = 0; j0 < n; j0 += 65535) {
    const int64_t nc = std::min<int64_t>(65535, n - j0);
    dim3 grid((unsigned)std::min<int64_t>((n + 255) / 256, 32), (unsigned)nc);
    shadow_init_kernel<<<grid, 256, 0, st>>>(n, j0, A, lda, Sh, ldsh);
  }
  return cudaGetLastError();
}

__global__ void to_half_cm_kernel(int64_t rows, int cols, const float* src, int64_t lds, __half* dst, int64_t ldd) {
  const int c = blockIdx.y;
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < rows; r += (int64_t)gridDim.x * blockDim.x)
    dst[r + c * ldd] = __float2half_rn(c < cols ? src[r + c * lds] : 0.f);
}

// dst[r + c*ldd] = fp16(src[r + c*lds]) for c < cols, 0 for cols <= c < cols_pad
cudaError_t to_half_cm(int64_t rows, int cols, int cols_pad, const float* src, int64_t lds, __half* dst,
                       int64_t ldd, cudaStream_t st) {
  if (rows <= 0 || cols_pad <= 0) return cudaSuccess;
  dim3 grid((unsigned)std::min<int64_t>((rows + 255) / 256, 64), (unsigned)cols_pad);
  to_half_cm_kernel<<<grid, 256, 0, st>>>(rows, cols, src, lds, dst, ldd);
  return cudaGetLastError();
}

__global__ void f32cm_to_f16rm_kernel2(int64_t rows, int cols, const float* src, int64_t lds, __half* dst,
                                       int64_t ldd) {
  // thread per (row, 8-column group): coalesced-enough reads along rows, 16-byte row writes
  const int groups = (cols + 7) / 8;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < rows * groups;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = e % rows;
    const int g = (int)(e / rows);
    __align__(16) __half v[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const int c = g * 8 + i;
      v[i] = __float2half_rn(c < cols ? src[r + (int64_t)c * lds] : 0.f);
    }
    if (g * 8 + 8 <= cols && ((r * ldd + g * 8) & 7) == 0) {
      *reinterpret_cast<uint4*>(dst + r * ldd + g * 8) = *reinterpret_cast<const uint4*>(v);
    } else {
      for (int i = 0; i < 8 && g * 8 + i < cols; ++i) dst[r * ldd + g * 8 + i] = v[i];
    }
  }
}

cudaError_t f32cm_to_f16rm(int64_t rows, int cols, const float* src, int64_t lds, __half* dst, int64_t ldd,
                           cudaStream_t st) {
  if (rows <= 0 || cols <= 0) return cudaSuccess;
  const int64_t work = rows * ((cols + 7) / 8);
  f32cm_to_f16rm_kernel2<<<(unsigned)std::min<int64_t>((work + 255) / 256, 1184), 256, 0, st>>>(rows, cols, src, lds,
                                                                                               dst, ldd);
  return cudaGetLastError();
}

// B operand of the lazy update: row n = [ Y(c+n, 0:k) | 0 .. | P(0:k, n)^T ] with the second part
// starting at column 64*ceil(k/64) (see SkinnyNN).
__global__ void build_lazy_b_kernel(int k, int b, const __half* Yh, int64_t ldyh, int64_t c, const float* P,
                                    __half* Bl, int64_t ldbl) {
  const int kp = (k + 63) / 64 * 64;
  const int n = blockIdx.y;
  for (int j = blockIdx.x * blockDim.x + threadIdx.x; j < kp + k; j += gridDim.x * blockDim.x) {
    __half v;
    if (j < k) v = Yh[(c + n) * ldyh + j];
    else if (j < kp) v = __float2half_rn(0.f);
    else v = __float2half_rn(P[(j - kp) + (int64_t)n * k]);
    Bl[n * ldbl + j] = v;
  }
}

cudaError_t build_lazy_b(int k, int b, const __half* Yh, int64_t ldyh, int64_t c, const float* P, __half* Bl,
                         int64_t ldbl, cudaStream_t st) {
  const int kp = (k + 63) / 64 * 64;
  build_lazy_b_kernel<<<dim3((kp + k + 255) / 256, b), 256, 0, st>>>(k, b, Yh, ldyh, c, P, Bl, ldbl);
  return cudaGetLastError();
}

}  // namespace sbr
