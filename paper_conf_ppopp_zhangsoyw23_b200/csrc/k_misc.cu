// k_misc.cu -- small kernels: input generator, finiteness check, band extraction,
// symmetric mirrors, the k x b correction of the lazy panel update.
#include <map>
#include <mutex>
#include <tuple>

#include "common.cuh"
#include "kernels.h"

namespace sbr {

namespace {
std::mutex g_attr_mu;
std::map<std::tuple<const void*, int, int>, int> g_attr;   // (fn, attr, device) -> value set
std::map<std::tuple<const void*, int, size_t, int>, int> g_occ;   // (fn, threads, smem, device) -> blocks/SM
int g_knobs[KNOB_COUNT] = {};
}  // namespace

cudaError_t func_attr(const void* fn, cudaFuncAttribute attr, int value) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  std::lock_guard<std::mutex> lk(g_attr_mu);
  const auto key = std::make_tuple(fn, (int)attr, dev);
  auto it = g_attr.find(key);
  if (it != g_attr.end() && it->second == value) return cudaSuccess;
  e = cudaFuncSetAttribute(fn, attr, value);
  if (e == cudaSuccess) g_attr[key] = value;
  return e;
}

int func_blocks_per_sm(const void* fn, int threads, size_t smem) {
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> lk(g_attr_mu);
  const auto key = std::make_tuple(fn, threads, smem, dev);
  auto it = g_occ.find(key);
  if (it != g_occ.end()) return it->second;
  int per = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, threads, smem) != cudaSuccess) {
    cudaGetLastError();
    per = 0;
  }
  g_occ[key] = per;
  return per;
}

int current_device_sms() {
  int dev = 0, n = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
  return n;
}

int knob(Knob k) { return (k >= 0 && k < KNOB_COUNT) ? g_knobs[k] : 0; }
void set_knob(int k, int v) {
  if (k >= 0 && k < KNOB_COUNT) g_knobs[k] = v;
}

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

// kexp sentinel: the input held Inf/NaN; the lower triangle is zeroed instead of scaled, so the
// reduction that follows runs on finite data (its outputs are invalid; the error is latched)
constexpr int kScaleZero = -(1 << 30);

// a0 scan (reading C10): over the local columns j (global column cm.g(j)), the referenced lower
// triangle: scan[0] += ||.||_F^2 (fp64, off-diagonal entries twice), scan[1] += count of Inf/NaN.
__global__ void prep_scan_kernel(int64_t n, int64_t j0, const float* A, int64_t lda, ColMap cm, double* scan) {
  const int64_t j = j0 + blockIdx.y;
  const int64_t g = cm.g(j);
  double s = 0.0;
  bool bad = false;
  for (int64_t i = g + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const float v = A[i + j * lda];
    if (!isfinite(v)) bad = true;
    else s += (i == g ? 1.0 : 2.0) * (double)v * (double)v;
  }
  if (__syncthreads_or(bad) && threadIdx.x == 0) atomicAdd(scan + 1, 1.0);
  __shared__ double red[32];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x < 32) {
    s = threadIdx.x < (blockDim.x >> 5) ? red[threadIdx.x] : 0.0;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (threadIdx.x == 0 && s != 0.0) atomicAdd(scan, s);
  }
}

// Exact power-of-two scale (reading C10): 2^k with ||A||_F 2^k in [2^12, 2^13).  Every
// trailing matrix of the reduction is orthogonally similar to a principal part of A, so its
// entries are <= ||A||_2 <= ||A||_F; X = OA W and Z stay within a few times that: all fp16
// operands stay below 2^15 < 65504, and typical entries (||A||_F / n) far above fp16's
// subnormal range.  The 3xTF32 mode takes the same scale (tf32 has fp32's exponent range,
// but the fp32 panel norms and products of an input near the ends of that range would
// under- or overflow).  k = 0 for a zero or non-finite input.
__global__ void choose_scale_kernel(const double* scan, unsigned* flag, int* kexp) {
  int k = 0;
  const double f2 = scan[0];
  if (scan[1] != 0.0) {   // non-finite input: the reduction runs on zeros (error latched, outputs invalid)
    flag[0] = 1u;
    *kexp = kScaleZero;
    return;
  }
  if (f2 > 0.0 && isfinite(f2)) {   // both modes
    int e = 0;
    frexp(sqrt(f2), &e);   // ||A||_F in [2^(e-1), 2^e)
    k = max(-250, min(250, 13 - e));
  }
  *kexp = k;
}

// The same scan with 16-byte loads (A 16-byte aligned, lda % 4 == 0): CTAs stride over whole
// columns, the rows of a column as float4 (scalar head / tail), one atomic per CTA at the end
// (the one-CTA-per-column-segment version above issues an fp64 atomic per segment).
__global__ void __launch_bounds__(256) prep_scan_vec_kernel(int64_t n, int64_t ncols, const float* __restrict__ A,
                                                            int64_t lda, ColMap cm, double* scan) {
  double s = 0.0;
  bool bad = false;
  for (int64_t j = blockIdx.x; j < ncols; j += gridDim.x) {
    const int64_t g = cm.g(j);
    const float* col = A + j * lda;
    const int64_t h0 = min(n, (g + 3) & ~(int64_t)3), t0 = max(h0, n & ~(int64_t)3);
    for (int64_t i = g + threadIdx.x; i < h0; i += blockDim.x) {   // head (< 4 rows), incl. the diagonal
      const float v = col[i];
      if (!isfinite(v)) bad = true;
      else s += (i == g ? 1.0 : 2.0) * (double)v * (double)v;
    }
    for (int64_t i = h0 + 4 * (int64_t)threadIdx.x; i < t0; i += 4 * (int64_t)blockDim.x) {
      const float4 v = __ldcs(reinterpret_cast<const float4*>(col + i));
      bad |= !(isfinite(v.x) && isfinite(v.y) && isfinite(v.z) && isfinite(v.w));
      const double a = v.x, b = v.y, c = v.z, d = v.w;
      const double q = (a * a + b * b) + (c * c + d * d);
      s += 2.0 * q - (i == g ? a * a : 0.0);   // the diagonal (i == g: first lane entry) once
    }
    for (int64_t i = t0 + threadIdx.x; i < n; i += blockDim.x) {   // tail
      const float v = col[i];
      if (!isfinite(v)) bad = true;
      else s += (i == g ? 1.0 : 2.0) * (double)v * (double)v;
    }
  }
  if (bad) s = 0.0;
  const int anybad = __syncthreads_or(bad);
  __shared__ double red[32];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x < 32) {
    s = threadIdx.x < (blockDim.x >> 5) ? red[threadIdx.x] : 0.0;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (threadIdx.x == 0) {
      if (s != 0.0) atomicAdd(scan, s);
      if (anybad) atomicAdd(scan + 1, 1.0);
    }
  }
}

cudaError_t prep_scan(int64_t n, int64_t ncols, const float* A, int64_t lda, ColMap cm, double* scan,
                      cudaStream_t st) {
  cudaError_t e = cudaMemsetAsync(scan, 0, 2 * sizeof(double), st);
  if (e != cudaSuccess) return e;
  if (lda % 4 == 0 && ((uintptr_t)A & 15) == 0) {
    const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ncols, (int64_t)current_device_sms() * 8));
    prep_scan_vec_kernel<<<grid, 256, 0, st>>>(n, ncols, A, lda, cm, scan);
    return cudaGetLastError();
  }
  for (int64_t j0 = 0; j0 < ncols; j0 += 65535) {
    const int64_t nc = std::min<int64_t>(65535, ncols - j0);
    dim3 grid((unsigned)std::min<int64_t>((n + 255) / 256, 16), (unsigned)nc);
    prep_scan_kernel<<<grid, 256, 0, st>>>(n, j0, A, lda, cm, scan);
  }
  return cudaGetLastError();
}

cudaError_t choose_scale(const double* scan, unsigned* flag, int* kexp, cudaStream_t st) {
  choose_scale_kernel<<<1, 1, 0, st>>>(scan, flag, kexp);
  return cudaGetLastError();
}

// a * 2^k, exact whenever the result is a normal float (two factors keep each within range)
// (|k| <= 252; 2^j built from its exponent bits, j in [-126, 126])
SBR_DEV float scale_pow2(float a, int k) {
  const int k1 = k / 2, k2 = k - k1;
  return (a * __int_as_float((k1 + 127) << 23)) * __int_as_float((k2 + 127) << 23);
}

// 3xTF32 mode: the lower triangle of A scaled in place by 2^k (no-op for k = 0)
__global__ void scale_lower_kernel(int64_t n, int64_t j0, float* A, int64_t lda, ColMap cm, const int* kexp) {
  const int k = *kexp;
  if (k == 0) return;
  const int64_t j = j0 + blockIdx.y;
  const int64_t g = cm.g(j);
  for (int64_t i = g + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    A[i + j * lda] = k == kScaleZero ? 0.f : scale_pow2(A[i + j * lda], k);
}

cudaError_t scale_lower(int64_t n, int64_t ncols, float* A, int64_t lda, ColMap cm, const int* kexp, cudaStream_t st) {
  for (int64_t j0 = 0; j0 < ncols; j0 += 65535) {
    const int64_t nc = std::min<int64_t>(65535, ncols - j0);
    dim3 grid((unsigned)std::min<int64_t>((n + 255) / 256, 32), (unsigned)nc);
    scale_lower_kernel<<<grid, 256, 0, st>>>(n, j0, A, lda, cm, kexp);
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

// Band out (a7): AB = 2^-k (band of A), written back into A's band unscaled too (A's Y part is
// scale free); a non-finite band entry (fp16 range exceeded despite the scaling) latches flag[2].
// Local column lc (global cm.g(lc)) of A fills AB column cm.g(lc).
__global__ void extract_band_kernel(int64_t n, int64_t ncols, int b, float* A, int64_t lda, ColMap cm, float* AB,
                                    int64_t ldab, const int* kexp, unsigned* flag) {
  const int64_t lc = (int64_t)blockIdx.x * blockDim.y + threadIdx.y;
  const int d = threadIdx.x;
  const int k = (kexp && *kexp != kScaleZero) ? *kexp : 0;
  bool bad = false;
  if (lc < ncols && d <= b) {
    const int64_t j = cm.g(lc);
    float v = 0.f;
    if (j + d < n) {
      v = A[(j + d) + lc * lda];
      if (k != 0) {
        v = scale_pow2(v, -k);
        A[(j + d) + lc * lda] = v;
      }
      bad = !isfinite(v);
    }
    AB[d + j * ldab] = v;
  }
  if (flag && __syncthreads_or(bad) && threadIdx.x == 0 && threadIdx.y == 0) atomicOr(flag + 2, 1u);
}

cudaError_t extract_band(int64_t n, int b, float* A, int64_t lda, float* AB, int64_t ldab, const int* kexp,
                         unsigned* flag, cudaStream_t st, int64_t ncols, ColMap cm) {
  if (ncols < 0) ncols = n;
  const int dx = b + 1;
  const int dy = max(1, 256 / dx);
  extract_band_kernel<<<(unsigned)((ncols + dy - 1) / dy), dim3(dx, dy), 0, st>>>(n, ncols, b, A, lda, cm, AB, ldab,
                                                                                 kexp, flag);
  return cudaGetLastError();
}

__global__ void mirror_lower_block_kernel(int b, float* A, int64_t lda) {
  pdl_trigger();   // 3xTF32 / SIMT chain: launched with PDL (launch_pdl), waits before any access
  pdl_wait();
  for (int e = threadIdx.x; e < b * b; e += blockDim.x) {
    const int i = e % b, j = e / b;
    if (i < j) A[i + (int64_t)j * lda] = A[j + (int64_t)i * lda];
  }
}

cudaError_t mirror_lower_block(int b, float* A, int64_t lda, cudaStream_t st) {
  return launch_pdl(mirror_lower_block_kernel, dim3(1), dim3(256), 0, st, b, A, lda);
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
  pdl_trigger();   // 3xTF32 / SIMT chain: launched with PDL (launch_pdl), waits before any access
  pdl_wait();
  const int q = blockIdx.x * blockDim.x + threadIdx.x;
  const int p = blockIdx.y;
  if (q < k) WtX[(k + p) + (int64_t)q * ld] = WtX[q + (int64_t)(k + p) * ld];
}

cudaError_t mirror_wtx(int k, int b, float* WtX, int64_t ld, cudaStream_t st) {
  if (k <= 0) return cudaSuccess;
  return launch_pdl(mirror_wtx_kernel, dim3((k + 127) / 128, b), dim3(128), 0, st, k, b, WtX, ld);
}

// Wo[:, c] = W[:, c] on the rows block J = c / nb acts on (r >= J nb + b), zero above
__global__ void copy_block_w_kernel(int64_t n, int b, int nb, int64_t c0, const float* W, int64_t ldw, float* Wo,
                                    int64_t ldwo) {
  const int64_t c = c0 + blockIdx.y;
  const int64_t r0 = (c / nb) * nb + b;
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x)
    Wo[r + c * ldwo] = r >= r0 ? W[r + c * ldw] : 0.f;
}

cudaError_t copy_block_w(int64_t n, int b, int nb, const float* W, int64_t ldw, float* Wo, int64_t ldwo, cudaStream_t st) {
  const int64_t ncols = n - b;
  for (int64_t c0 = 0; c0 < ncols; c0 += 65535) {
    const int64_t nc = std::min<int64_t>(65535, ncols - c0);
    dim3 grid((unsigned)std::min<int64_t>((n + 255) / 256, 16), (unsigned)nc);
    copy_block_w_kernel<<<grid, 256, 0, st>>>(n, b, nb, c0, W, ldw, Wo, ldwo);
  }
  return cudaGetLastError();
}

// a kernel, not cudaMemset2DAsync: a memset node between two PDL launches would end the chain's
// launch overlap (the per-panel steps of the 3xTF32 / SIMT paths zero small blocks every panel)
__global__ void zero_matrix_kernel(int64_t rows, int64_t cols, float* A, int64_t lda) {
  pdl_trigger();
  pdl_wait();
  const int64_t tot = rows * cols;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < tot; e += (int64_t)gridDim.x * blockDim.x)
    A[e % rows + (e / rows) * lda] = 0.f;
}

cudaError_t zero_matrix(int64_t rows, int64_t cols, float* A, int64_t lda, cudaStream_t st) {
  if (rows <= 0 || cols <= 0) return cudaSuccess;
  const int64_t tot = rows * cols;
  if (tot > ((int64_t)1 << 22))   // block-start buffers (not on the per-panel chain): the copy engine
    return cudaMemset2DAsync(A, lda * sizeof(float), 0, rows * sizeof(float), cols, st);
  return launch_pdl(zero_matrix_kernel, dim3((unsigned)std::min<int64_t>((tot + 255) / 256, 148 * 16)), dim3(256), 0,
                    st, rows, cols, A, lda);
}

// a0: fp16 shadow of the lower triangle of 2^k A: strict lower as is, HALF the diagonal, zero
// above (so that a diagonal tile T satisfies T + T^T = L; see k_pass_tc.cu).  With k != 0 the
// fp32 master's lower triangle is scaled in place too (exact: powers of two; reading C10).
__global__ void shadow_init_kernel(int64_t n, int64_t j0, float* A, int64_t lda, __half* Sh, int64_t ldsh,
                                   const int* kexp, ColMap cm) {
  const int64_t j = j0 + blockIdx.y;
  const int64_t g = cm.g(j);
  const int k = kexp ? *kexp : 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    float v = 0.f;
    if (i >= g) {
      v = A[i + j * lda];
      if (k != 0) {
        v = k == kScaleZero ? 0.f : scale_pow2(v, k);
        A[i + j * lda] = v;
      }
      if (i == g) v *= 0.5f;
    }
    Sh[i + j * ldsh] = cvt16(v);
  }
}

// 16-byte version (A 16-byte aligned with lda % 4 == 0, shadow 8-byte aligned with ldsh % 4 == 0):
// CTAs stride over columns, 4 rows per thread step (float4 in/out, 4 halves out).
__global__ void __launch_bounds__(256) shadow_init_vec_kernel(int64_t n, int64_t ncols, float* __restrict__ A,
                                                              int64_t lda, __half* __restrict__ Sh, int64_t ldsh,
                                                              const int* kexp, ColMap cm) {
  const int k = kexp ? *kexp : 0;
  const int64_t n4 = n & ~(int64_t)3;
  for (int64_t j = blockIdx.x; j < ncols; j += gridDim.x) {
    const int64_t g = cm.g(j);
    float* col = A + j * lda;
    __half* sc = Sh + j * ldsh;
    for (int64_t i = 4 * (int64_t)threadIdx.x; i < n4; i += 4 * (int64_t)blockDim.x) {
      float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
      if (i + 3 >= g) {
        v = *reinterpret_cast<const float4*>(col + i);
        float* e = &v.x;
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          if (i + u < g) e[u] = 0.f;
          else if (k != 0) e[u] = k == kScaleZero ? 0.f : scale_pow2(e[u], k);
        }
        if (k != 0) {   // the scaled master (rows above the diagonal keep their values)
          if (i >= g) {
            *reinterpret_cast<float4*>(col + i) = v;
          } else {
#pragma unroll
            for (int u = 0; u < 4; ++u)
              if (i + u >= g) col[i + u] = e[u];
          }
        }
#pragma unroll
        for (int u = 0; u < 4; ++u)
          if (i + u == g) e[u] *= 0.5f;
      }
      __half2 h01 = __halves2half2(cvt16(v.x), cvt16(v.y)), h23 = __halves2half2(cvt16(v.z), cvt16(v.w));
      uint2 pk;
      pk.x = *reinterpret_cast<uint32_t*>(&h01);
      pk.y = *reinterpret_cast<uint32_t*>(&h23);
      *reinterpret_cast<uint2*>(sc + i) = pk;
    }
    for (int64_t i = n4 + threadIdx.x; i < n; i += blockDim.x) {   // tail rows
      float v = 0.f;
      if (i >= g) {
        v = col[i];
        if (k != 0) {
          v = k == kScaleZero ? 0.f : scale_pow2(v, k);
          col[i] = v;
        }
        if (i == g) v *= 0.5f;
      }
      sc[i] = cvt16(v);
    }
  }
}

cudaError_t shadow_init(int64_t n, float* A, int64_t lda, __half* Sh, int64_t ldsh, const int* kexp,
                        cudaStream_t st, int64_t ncols, ColMap cm) {
  if (ncols < 0) ncols = n;
  if (lda % 4 == 0 && ((uintptr_t)A & 15) == 0 && ldsh % 4 == 0 && ((uintptr_t)Sh & 7) == 0) {
    const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ncols, (int64_t)current_device_sms() * 8));
    shadow_init_vec_kernel<<<grid, 256, 0, st>>>(n, ncols, A, lda, Sh, ldsh, kexp, cm);
    return cudaGetLastError();
  }
  for (int64_t j0 = 0; j0 < ncols; j0 += 65535) {
    const int64_t nc = std::min<int64_t>(65535, ncols - j0);
    dim3 grid((unsigned)std::min<int64_t>((n + 255) / 256, 32), (unsigned)nc);
    shadow_init_kernel<<<grid, 256, 0, st>>>(n, j0, A, lda, Sh, ldsh, kexp, cm);
  }
  return cudaGetLastError();
}

__global__ void to_half_cm_kernel(int64_t rows, int cols, const float* src, int64_t lds, __half* dst, int64_t ldd) {
  const int c = blockIdx.y;
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < rows; r += (int64_t)gridDim.x * blockDim.x)
    dst[r + c * ldd] = cvt16(c < cols ? src[r + c * lds] : 0.f);
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
      v[i] = cvt16(c < cols ? src[r + (int64_t)c * lds] : 0.f);
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
    else if (j < kp) v = cvt16(0.f);
    else v = cvt16(P[(j - kp) + (int64_t)n * k]);
    Bl[n * ldbl + j] = v;
  }
}

cudaError_t build_lazy_b(int k, int b, const __half* Yh, int64_t ldyh, int64_t c, const float* P, __half* Bl,
                         int64_t ldbl, cudaStream_t st) {
  const int kp = (k + 63) / 64 * 64;
  build_lazy_b_kernel<<<dim3((kp + k + 255) / 256, b), 256, 0, st>>>(k, b, Yh, ldyh, c, P, Bl, ldbl);
  return cudaGetLastError();
}

SBR_OP16_SETTER(misc)

}  // namespace sbr
