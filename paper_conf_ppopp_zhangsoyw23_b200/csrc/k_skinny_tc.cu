// k_skinny_tc.cu -- the memory-bound "skinny" WY steps (a3, a5) on tcgen05, N = b.
//
//   skinny_nn : D[M x b] = C - A[M x K] B^T        A fp16 row-major (1 or 2 K-halves),
//               B (b x K) fp16 K-major; fp32 out (column-major, may alias C) and
//               optional fp16 copies (column-major and/or row-major).
//     * lazy panel update (Alg.1 l.8-10): GA = OA(:,c) - [X | Y] [Y_c^T ; W^T R]
//     * W merge:  W_t = W_t^0 - W (Y^T W_t^0)
//   skinny_tn : D[K1 x b] += A[rows x K1]^T B[rows x b] over a row range (split-K with
//               fp32 reductions), A fp16 row-major (MN-major operand), B fp16 column-major;
//               two A operands share one B (dual accumulators):
//     * G = Y^T W_t^0 and H = X^T W_t^0 (then W^T X_t = H - (W^T X) G by symmetry of OA)
// Both stream their big operand once through a TMA ring; the MMA is never the bound.
#include "kernels.h"
#include "tc.cuh"

namespace sbr {

using namespace tc;

// ------------------------------------------------------------------ skinny_nn
template <int BN>
struct NnCfg {
  static constexpr int NS = 4;
  static constexpr int SA = 128 * 64 * 2;   // 16 KB A tile (128 rows x 64 K)
  static constexpr int SB = BN * 64 * 2;    // B tile (BN rows x 64 K)
  static constexpr int STAGE = SA + SB;
  static constexpr int OFF_BAR = NS * STAGE;
  static constexpr int SMEM = OFF_BAR + (2 * NS + 2) * 8 + 16 + 1024;
  static constexpr int TCOLS = BN < 32 ? 32 : BN;
};

template <int BN>
__global__ void __launch_bounds__(256, 1)
    skinny_nn_kernel(const __grid_constant__ CUtensorMap mapA0, const __grid_constant__ CUtensorMap mapA1,
                     const __grid_constant__ CUtensorMap mapB0, const __grid_constant__ CUtensorMap mapB1, int kc0,
                     int kct, int arow0, int brow0, int64_t rows, int b,
                     const float* Cin, int64_t ldc, float* Dout, int64_t ldd, __half* __restrict__ Hcm, int64_t ldhc,
                     __half* __restrict__ Hrm, int64_t ldhr, int kper) {
  // split-K (gridDim.y > 1, only when D = C in place and no fp16 copies): CTA (tile, s) takes
  // k-chunks [s*kper, s*kper + kper) and subtracts its partial with fp32 reductions
  using Cfg = NnCfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint64_t* bars = (uint64_t*)(smem + Cfg::OFF_BAR);
  uint64_t* full = bars;
  uint64_t* empty = bars + Cfg::NS;
  uint64_t* acc_full = bars + 2 * Cfg::NS;
  uint32_t* tmem_slot = (uint32_t*)(bars + 2 * Cfg::NS + 2);
  const int warp = warp_id(), lane = lane_id();
  pdl_trigger();
  const int tile = blockIdx.x;
  if (threadIdx.x == 0) {
    for (int i = 0; i < Cfg::NS; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    mbar_init(acc_full, 1);
    mbar_fence_init();
  }
  if (warp == 2) tmem_alloc(tmem_slot, Cfg::TCOLS);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();
  const int kb = blockIdx.y * kper, ke = min(kct, kb + kper);
  const bool split = gridDim.y > 1;
  if (warp == 0 && lane == 0) {
    int st = 0; uint32_t ph = 0;
    for (int kc = kb; kc < ke; ++kc) {
      mbar_wait(&empty[st], ph ^ 1);
      mbar_expect_tx(&full[st], Cfg::STAGE);
      uint8_t* sa = smem + st * Cfg::STAGE;
      const bool second = kc >= kc0;
      const int kin = (second ? kc - kc0 : kc) * 64;
      tma_load_2d(sa, second ? &mapA1 : &mapA0, &full[st], kin, arow0 + tile * 128);
      tma_load_2d(sa + Cfg::SA, second ? &mapB1 : &mapB0, &full[st], kin, second ? 0 : brow0);
      if (++st == Cfg::NS) { st = 0; ph ^= 1; }
    }
  } else if (warp == 1 && lane == 0) {
    const uint32_t idesc = idesc_make(128, BN, 0, 0, 0) | op16_fmt();
    int st = 0; uint32_t ph = 0;
    const uint32_t s0 = smem_u32(smem);
    for (int kc = kb; kc < ke; ++kc) {
      mbar_wait(&full[st], ph);
      tc_fence_after();
      const uint32_t sa = s0 + st * Cfg::STAGE, sb = sa + Cfg::SA;
#pragma unroll
      for (int s = 0; s < 4; ++s)
        mma_f16(tmem, sdesc_sw128(sa + s * 32, 16, 1024), sdesc_sw128(sb + s * 32, 16, 1024), idesc,
                (kc > kb || s > 0) ? 1u : 0u);
      mma_commit(&empty[st]);
      if (++st == Cfg::NS) { st = 0; ph ^= 1; }
    }
    mma_commit(acc_full);
  } else if (warp >= 4) {
    const int q = warp - 4;
    const int64_t r = (int64_t)tile * 128 + q * 32 + lane;
    // C is independent of the accumulator: its loads are issued before the wait, so their latency
    // hides under the mainloop
    constexpr int BO = BN < 32 ? 32 : BN;
    float o[BO];
#pragma unroll
    for (int c = 0; c < BO; ++c) o[c] = (!split && r < rows && c < b) ? Cin[r + (int64_t)c * ldc] : 0.f;
    // row-major fp16 copy in 16-byte stores (8 halves) when aligned
    const bool hvec = Hrm && (b % 8 == 0) && (ldhr % 8 == 0) && ((reinterpret_cast<uintptr_t>(Hrm) & 15) == 0);
    mbar_wait(acc_full, 0);
    tc_fence_after();
#pragma unroll
    for (int c0 = 0; c0 < BN; c0 += 32) {
      float v[32];
      if (ke > kb) tmem_ld32(tmem + c0 + ((uint32_t)(q * 32) << 16), v);
      else {
#pragma unroll
        for (int c = 0; c < 32; ++c) v[c] = 0.f;
      }
      if (split) {
        if (r < rows && ke > kb) {
#pragma unroll
          for (int c = 0; c < 32; ++c)
            if (c0 + c < b) atomicAdd(Dout + r + (int64_t)(c0 + c) * ldd, -v[c]);
        }
        continue;
      }
      if (r < rows) {
        __align__(16) __half hv[32];
#pragma unroll
        for (int c = 0; c < 32; ++c) {
          const int n = c0 + c;
          const float d = o[n] - v[c];
          hv[c] = cvt16(d);
          if (n < b) {
            Dout[r + (int64_t)n * ldd] = d;
            if (Hcm) Hcm[r + (int64_t)n * ldhc] = hv[c];
            if (Hrm && !hvec) Hrm[r * ldhr + n] = hv[c];
          }
        }
        if (hvec) {
#pragma unroll
          for (int g = 0; g < 4; ++g)
            if (c0 + g * 8 < b)
              *reinterpret_cast<uint4*>(Hrm + r * ldhr + c0 + g * 8) = *reinterpret_cast<const uint4*>(hv + g * 8);
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    tc_fence_after();
    tmem_dealloc(tmem, Cfg::TCOLS);
  }
}

template <int BN>
static cudaError_t launch_nn_t(const SkinnyNN& p, cudaStream_t st) {
  using Cfg = NnCfg<BN>;
  auto kern = skinny_nn_kernel<BN>;
  {
    cudaError_t e = func_attr((const void*)kern, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM);
    if (e != cudaSuccess) return e;
  }
  CUtensorMap mA0, mA1, mB0, mB1;
  cudaError_t e;
  const int64_t K0 = std::max<int64_t>(p.K0, 1), K1 = std::max<int64_t>(p.K1, 1);
  if ((e = make_tmap_2d(&mA0, p.A0, true, K0, p.a_rows, p.lda, 64, 128)) != cudaSuccess) return e;
  if ((e = make_tmap_2d(&mA1, p.A1 ? p.A1 : p.A0, true, K1, p.a_rows, p.lda, 64, 128)) != cudaSuccess) return e;
  if ((e = make_tmap_2d(&mB0, p.B0, true, K0, p.b0_rows, p.ldb0, 64, BN)) != cudaSuccess) return e;
  if ((e = make_tmap_2d(&mB1, p.B1 ? p.B1 : p.B0, true, K1, p.B1 ? p.b : p.b0_rows, p.B1 ? p.ldb1 : p.ldb0, 64, BN)) !=
      cudaSuccess)
    return e;
  const int kc0 = (int)((p.K0 + 63) / 64);
  const int kct = kc0 + (int)((p.K1 + 63) / 64);
  const int grid = (int)((p.rows + 127) / 128);
  if (grid == 0) return cudaSuccess;
  // split-K when the update is in place without fp16 copies (the lazy update): CTAs stream shorter
  // K ranges (2 fit per SM: 80 KB smem, 32-64 TMEM columns), the split chosen to minimise the wave-quantised time ceil(grid*ns/slots)/ns with
  // at least 4 K-chunks per CTA
  int ns = 1;
  if (!p.Hcm && !p.Hrm && p.C == p.D && p.ldc == p.ldd && kct >= 8) {
    const int slots = 2 * 148;
    double best = 1e30;
    for (int s = 1; s <= std::min(8, kct / 4); ++s) {
      const double cost = (double)((grid * s + slots - 1) / slots) / s + 0.02 * s;   // + atomics / prologue per split
      if (cost < best) { best = cost; ns = s; }
    }
  }
  const int kper = (kct + ns - 1) / ns;
  ns = kct > 0 ? (kct + kper - 1) / kper : 1;
  return launch_pdl(kern, dim3(grid, ns), dim3(256), Cfg::SMEM, st, mA0, mA1, mB0, mB1, kc0, kct, (int)p.arow0,
                    (int)p.brow0, p.rows, p.b, p.C, p.ldc, p.D, p.ldd, p.Hcm, p.ldhc, p.Hrm, p.ldhr,
                    std::max(kper, 1));
}

cudaError_t launch_skinny_nn(const SkinnyNN& p, cudaStream_t st) {
  const int bn = pass_bn(p.b);
  if (bn == 16) return launch_nn_t<16>(p, st);
  if (bn == 32) return launch_nn_t<32>(p, st);
  return launch_nn_t<64>(p, st);
}

// ------------------------------------------------------------------ skinny_tn (dual)
template <int BN>
struct TnCfg {
  static constexpr int NS = 3;   // 3 x 36 KB: two CTAs per SM (one wave of 2 x 148, 216 KB in flight per SM)
  static constexpr int SA = 128 * 64 * 2;   // one A operand: 128 (K1 dim) x 64 rows, 2 boxes of 64x64
  static constexpr int SB = BN * 64 * 2;
  static constexpr int STAGE = 2 * SA + SB;
  static constexpr int OFF_BAR = NS * STAGE;
  static constexpr int SMEM = OFF_BAR + (2 * NS + 2) * 8 + 16 + 1024;
  static constexpr int TCOLS = 2 * BN < 32 ? 32 : 2 * BN;
};

template <int BN>
__global__ void __launch_bounds__(256, 1)
    skinny_tn_kernel(const __grid_constant__ CUtensorMap mapA0, const __grid_constant__ CUtensorMap mapA1,
                     const __grid_constant__ CUtensorMap mapB, int dual, int64_t row0, int64_t rows, int64_t chunk,
                     int K1, int b, float* D0, float* D1, int64_t ldd) {
  using Cfg = TnCfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint64_t* bars = (uint64_t*)(smem + Cfg::OFF_BAR);
  uint64_t* full = bars;
  uint64_t* empty = bars + Cfg::NS;
  uint64_t* acc_full = bars + 2 * Cfg::NS;
  uint32_t* tmem_slot = (uint32_t*)(bars + 2 * Cfg::NS + 2);
  const int warp = warp_id(), lane = lane_id();
  pdl_trigger();
  const int jt = blockIdx.x;                     // 128-wide slab of the K1 dimension
  const int64_t rb = row0 + (int64_t)blockIdx.y * chunk;
  const int64_t re = std::min<int64_t>(row0 + rows, rb + chunk);
  const int nks = (int)((re - rb + 63) / 64);
  if (threadIdx.x == 0) {
    for (int i = 0; i < Cfg::NS; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    mbar_init(acc_full, 1);
    mbar_fence_init();
  }
  if (warp == 2) tmem_alloc(tmem_slot, Cfg::TCOLS);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();
  const uint32_t bytes = (dual ? 2 : 1) * Cfg::SA + Cfg::SB;
  if (warp == 0 && lane == 0) {
    int st = 0; uint32_t ph = 0;
    for (int ks = 0; ks < nks; ++ks) {
      const int r = (int)(rb + ks * 64);
      mbar_wait(&empty[st], ph ^ 1);
      mbar_expect_tx(&full[st], bytes);
      uint8_t* sa = smem + st * Cfg::STAGE;
      for (int h = 0; h < 2; ++h) tma_load_2d(sa + h * 8192, &mapA0, &full[st], jt * 128 + h * 64, r);
      if (dual)
        for (int h = 0; h < 2; ++h) tma_load_2d(sa + Cfg::SA + h * 8192, &mapA1, &full[st], jt * 128 + h * 64, r);
      tma_load_2d(sa + 2 * Cfg::SA, &mapB, &full[st], r, 0);
      if (++st == Cfg::NS) { st = 0; ph ^= 1; }
    }
  } else if (warp == 1 && lane == 0) {
    // A^T is MN-major: 64-wide K1 atoms 8 KB apart (LBO), 8-row K groups 1 KB apart (SBO)
    const uint32_t idesc = idesc_make(128, BN, 0, 1, 0) | op16_fmt();
    int st = 0; uint32_t ph = 0;
    const uint32_t s0 = smem_u32(smem);
    for (int ks = 0; ks < nks; ++ks) {
      mbar_wait(&full[st], ph);
      tc_fence_after();
      const uint32_t sa = s0 + st * Cfg::STAGE, sb = sa + 2 * Cfg::SA;
#pragma unroll
      for (int s = 0; s < 4; ++s) {
        const uint64_t bd = sdesc_sw128(sb + s * 32, 16, 1024);
        mma_f16(tmem, sdesc_sw128(sa + s * 2048, 8192, 1024), bd, idesc, (ks > 0 || s > 0) ? 1u : 0u);
        if (dual)
          mma_f16(tmem + BN, sdesc_sw128(sa + Cfg::SA + s * 2048, 8192, 1024), bd, idesc,
                  (ks > 0 || s > 0) ? 1u : 0u);
      }
      mma_commit(&empty[st]);
      if (++st == Cfg::NS) { st = 0; ph ^= 1; }
    }
    mma_commit(acc_full);
  } else if (warp >= 4) {
    const int q = warp - 4;
    const int j = jt * 128 + q * 32 + lane;
    mbar_wait(acc_full, 0);
    tc_fence_after();
    if (nks > 0) {
      for (int which = 0; which < (dual ? 2 : 1); ++which) {
        float* D = which ? D1 : D0;
#pragma unroll
        for (int c0 = 0; c0 < BN; c0 += 32) {
          float v[32];
          tmem_ld32(tmem + which * BN + c0 + ((uint32_t)(q * 32) << 16), v);
          if (j < K1) {
#pragma unroll
            for (int c = 0; c < 32; ++c)
              if (c0 + c < b) atomicAdd(&D[j + (int64_t)(c0 + c) * ldd], v[c]);
          }
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    tc_fence_after();
    tmem_dealloc(tmem, Cfg::TCOLS);
  }
}

template <int BN>
static cudaError_t launch_tn_t(const SkinnyTN& p, cudaStream_t st) {
  using Cfg = TnCfg<BN>;
  auto kern = skinny_tn_kernel<BN>;
  {
    cudaError_t e = func_attr((const void*)kern, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM);
    if (e != cudaSuccess) return e;
  }
  if (p.K1 <= 0 || p.rows <= 0) return cudaSuccess;
  CUtensorMap mA0, mA1, mB;
  cudaError_t e;
  if ((e = make_tmap_2d(&mA0, p.A0, true, p.K1, p.a_rows, p.lda, 64, 64)) != cudaSuccess) return e;
  if ((e = make_tmap_2d(&mA1, p.A1 ? p.A1 : p.A0, true, p.K1, p.a_rows, p.lda, 64, 64)) != cudaSuccess) return e;
  if ((e = make_tmap_2d(&mB, p.B, true, p.b_rows, p.b, p.ldb, 64, BN)) != cudaSuccess) return e;
  const int gx = (int)((p.K1 + 127) / 128);
  int64_t want = std::max<int64_t>(1, (2 * p.num_sms) / gx);   // one wave at two CTAs per SM
  int64_t chunk = (p.rows + want - 1) / want;
  chunk = std::max<int64_t>(512, (chunk + 63) / 64 * 64);
  const int gy = (int)((p.rows + chunk - 1) / chunk);
  return launch_pdl(kern, dim3(gx, gy), dim3(256), Cfg::SMEM, st, mA0, mA1, mB, p.A1 ? 1 : 0, p.row0, p.rows, chunk,
                    (int)p.K1, p.b, p.D0, p.D1, p.ldd);
}

cudaError_t launch_skinny_tn(const SkinnyTN& p, cudaStream_t st) {
  const int bn = pass_bn(p.b);
  if (bn == 16) return launch_tn_t<16>(p, st);
  if (bn == 32) return launch_tn_t<32>(p, st);
  return launch_tn_t<64>(p, st);
}

SBR_OP16_SETTER(skinny)

}  // namespace sbr
