// k_gemm_tc.cu -- the per-block trailing update (step a6) on tcgen05 tensor cores.
//
//   ZFORM : Z = X - 1/2 Y (W^T X)                       (Eq. 2 analogue; reading C5)
//   SYR2K : A_low[s:, s:] -= Y_s Z_s^T + Z_s Y_s^T       (Eq. 3; Alg. 1 l.13)
//           computed as ONE GEMM with K = 2 nb: [Y | Z] [Z | Y]^T, lower tiles only --
//           the Tensor-Core syr2k the paper lists as future work.
//
// Operands are fp16, row-major (K contiguous = K-major for UMMA), fed by TMA with
// 128-byte swizzle into a 4-stage smem ring; 128 x 256 output tiles accumulate in TMEM
// (double-buffered: the epilogue of tile i overlaps the MMAs of tile i+1).
// SYR2K epilogue: C_new = C_old - acc on the fp32 master (lower elements only) and the
// fp16 shadow of the next block's OA (strict lower, half diagonal; see k_pass_tc.cu).
// ZFORM epilogue: Zh = fp16(X - acc/2), row-major.
//
// 3xTF32 mode (reading C11): operands are fp32 row-major arrays holding
// [hi | lo] (hi = rna_tf32(a), lo = rna_tf32(a - hi), lo at column offset `lo_off`), and
// the K loop runs over a SEGMENT TABLE: SYR2K = Yhi Zhi' + Yhi Zlo' + Ylo Zhi' + (Y <-> Z),
// ZFORM = Yhi Ghi + Yhi Glo + Ylo Ghi, all accumulated in one fp32 TMEM accumulator by
// tcgen05.mma kind::tf32 (BK = 32 fp32 = 128 B rows, the same smem bytes per stage).
// The ZFORM epilogue then writes Z split the same way; the SYR2K epilogue writes no shadow
// (the 3xTF32 pass reads the fp32 master).
#include "kernels.h"
#include "tc.cuh"

namespace sbr {

using namespace tc;

namespace {
constexpr int G_BM = 128;
constexpr int G_ROWB = 128;            // bytes of one operand row chunk (64 fp16 or 32 fp32)
constexpr int G_SA = G_BM * G_ROWB;    // 16 KB
template <bool TF> struct GCfg {
  // fp16: 128 x 256 tiles, one TMEM accumulation per tile.  3xTF32: 128 x 128 tiles and the
  // accumulator is drained every FLUSH k-chunks (128 K elements) into fp32 registers (RN adds):
  // the tensor core's own fp32 accumulation truncates, which over K = 6 nb terms would cost
  // ~K^1.5 ulps (reading R4).
  static constexpr int BN = TF ? 128 : 256;
  static constexpr int NS = TF ? 6 : 4;
  static constexpr int SB = BN * G_ROWB;
  static constexpr int STAGE = G_SA + SB;
  static constexpr int OFF_BAR = NS * STAGE;
  static constexpr int SMEM = OFF_BAR + (2 * NS + 4) * 8 + 16 + 1024;
  static constexpr int FLUSH = 4;
};
}  // namespace

// tile index -> (I, Jc).  ZFORM / GEMM modes: the full grid, row-major.  SYR2K: the lower tiles
// (Jc * BN <= I * BM + BM - 1, i.e. I >= r Jc with r = BN / BM) in an L2-friendly raster: bands of
// H tile rows, inside a band column-major (all rows I of column Jc, then Jc + 1).  The ~148 tiles
// in flight then share one or two B panels (rows Jc of [Z | Y]) and sweep the band's A panels
// (H x 128 rows of [Y | Z], which stay L2-resident), so B is read from DRAM once per band
// instead of once per tile row (the operands of a large block, 2 x M x 2nb, exceed L2).
template <int MODE, int BN, int BMU = G_BM>   // BMU: rows of one work unit (G_BM, or 2 G_BM for a CTA pair)
SBR_DEV void gemm_tile(int t, int ntn, int ntm, int& I, int& Jc, int H) {
  if (MODE != 0) {
    I = t / ntn;
    Jc = t % ntn;
    return;
  }
  constexpr int r = BN / BMU;                        // 1 or 2
  // H: band height in tile rows (A band <= ~64 MB at the default 64 / 32)
  for (int I0 = 0; I0 < ntm; I0 += H) {
    const int I1 = min(I0 + H, ntm), Hs = I1 - I0;
    const int F = I0 / r + 1;                        // columns with every band row valid
    const int D = I1 - r * F;                        // rows of column F (then D - r, D - 2r, ...)
    const int jmax = D > 0 ? (D + r - 1) / r : 0;
    const int full = F * Hs, tri = jmax * D - r * jmax * (jmax - 1) / 2;
    if (t < full) {
      Jc = t / Hs;
      I = I0 + t % Hs;
      return;
    }
    t -= full;
    if (t < tri) {   // C(j) = j D - r j (j - 1) / 2 tiles before triangular column j
      const double a = D + 0.5 * r;
      int j = (int)((a - sqrt(fmax(a * a - 2.0 * r * t, 0.0))) / r);
      j = max(0, min(j, jmax - 1));
      while (j + 1 < jmax && (j + 1) * D - r * (j + 1) * j / 2 <= t) ++j;
      while (j > 0 && j * D - r * j * (j - 1) / 2 > t) --j;
      const int u = t - (j * D - r * j * (j - 1) / 2);
      Jc = F + j;
      I = r * Jc + u;
      return;
    }
    t -= tri;
  }
  I = Jc = 0;   // not reached for t < ntiles
}

// Multi-GPU column ownership of the SYR2K output (sbr_reduce_dist): output column rel (relative to
// the trailing region) is global column org + rel, owned by rank (g / nbo) % P; the owned tiles
// (BN columns, inside one block) update C / shadow at local column (g / nbo / P) nbo + g % nbo
// (C and shadow then point at the region's first ROW, column 0).  P = 1: every tile, column rel.
struct GemmOwn {
  int P = 1, rank = 0;
  int64_t org = 0, nbo = 1;
  SBR_DEV bool owned(int64_t rel) const { return P <= 1 || ((org + rel) / nbo) % P == rank; }
  SBR_DEV int64_t lcol(int64_t rel) const {
    if (P <= 1) return rel;
    const int64_t g = org + rel;
    return (g / nbo / P) * nbo + g % nbo;
  }
};

constexpr int G_EPI_WARPS = 8;  // two warps per TMEM lane quarter, each half of the 256 columns
constexpr int G_THREADS = 128 + 32 * G_EPI_WARPS;

// K segments: segment s multiplies columns [acol[s], acol[s] + K) of A map amap[s] with
// columns [bcol[s], ...) of B map bmap[s]; all segments accumulate into the same tile.
struct GemmSegs {
  int n;
  int amap[6], acol[6], bmap[6], bcol[6];
};

// MC = 2 (FP16 SYR2K): CTA pairs (clusters of 2) take work units of two 128-row tiles with the same
// column tile Jc; each CTA loads its own A rows and HALF of the shared B tile, multicast into both
// CTAs' shared memory, so B crosses L2 -> SM once per pair (the SYR2K's operand stream per tile was
// 1.5 MB at K = 2 nb); each CTA's MMA commit frees the stage in both CTAs (empty count = 2).
template <int MODE, bool TF, int MC = 1>
__global__ void __launch_bounds__(G_THREADS, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap mapA0, const __grid_constant__ CUtensorMap mapA1,
                   const __grid_constant__ CUtensorMap mapB0, const __grid_constant__ CUtensorMap mapB1, int kpb,
                   const GemmSegs segs, int arow0, int brow0, int64_t Mrows, int64_t Ncols, int ntn, int ntiles,
                   float* C, int64_t ldc, __half* __restrict__ shadow, int64_t ldsh, const float* __restrict__ X,
                   int64_t ldx, void* __restrict__ Zout, int64_t ldz, int64_t zlo_off, const GemmOwn own, int bandH) {
  using Cfg = GCfg<TF>;
  constexpr int BK = TF ? 32 : 64;   // K elements per 128-byte row chunk
  constexpr int G_BN = Cfg::BN, G_NS = Cfg::NS, G_STAGE = Cfg::STAGE;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint64_t* bars = (uint64_t*)(smem + Cfg::OFF_BAR);
  uint64_t* full = bars;
  uint64_t* empty = bars + G_NS;
  uint64_t* acc_full = bars + 2 * G_NS;
  uint64_t* acc_empty = acc_full + 2;
  uint32_t* tmem_slot = (uint32_t*)(bars + 2 * G_NS + 4);
  const int warp = warp_id(), lane = lane_id();
  pdl_trigger();
  if (threadIdx.x == 0) {
    for (int i = 0; i < G_NS; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], MC); }
    for (int i = 0; i < 2; ++i) { mbar_init(&acc_full[i], 1); mbar_init(&acc_empty[i], 32 * G_EPI_WARPS); }
    mbar_fence_init();
  }
  const int crank = MC > 1 ? (int)cluster_ctarank() : 0;
  // work units: one tile (MC = 1) or a pair of tiles.  FP16 (128 x 256 tiles): the pair is two
  // vertically adjacent tiles sharing B (this CTA takes row I = MC Iu + crank).  3xTF32 (128 x 128
  // tiles): two horizontally adjacent tiles sharing A (column Jc = MC Jcu + crank), i.e. the unit is
  // the FP16 mode's 128 x 256 footprint.
  constexpr bool SHA = TF;
  constexpr int UBM = (MC > 1 && !SHA) ? G_BM * MC : G_BM;
  constexpr int UBN = (MC > 1 && SHA) ? G_BN * MC : G_BN;
  const int u0 = MC > 1 ? (int)blockIdx.x / MC : (int)blockIdx.x;
  const int ustride = MC > 1 ? (int)gridDim.x / MC : (int)gridDim.x;
  if (warp == 0 && lane == 0) {
    tma_prefetch(&mapA0); tma_prefetch(&mapB0); tma_prefetch(&mapA1); tma_prefetch(&mapB1);
  }
  if (warp == 2) tmem_alloc(tmem_slot, 512);
  tc_fence_before();
  __syncthreads();
  if (MC > 1) cluster_sync_all();   // the peer's barriers are initialised before any multicast / commit
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();
  const int nk = segs.n * kpb;
  const int ntm = (int)((Mrows + UBM - 1) / UBM);   // unit rows

  if (warp == 0) {
    if (lane == 0) {  // ---------------- TMA producer
      int st = 0; uint32_t ph = 0;
      for (int t = u0; t < ntiles; t += ustride) {
        int I, Jc;
        gemm_tile<MODE, UBN, UBM>(t, ntn, ntm, I, Jc, bandH);
        if (MC > 1) { if (SHA) Jc = Jc * MC + crank; else I = I * MC + crank; }
        if (!own.owned((int64_t)(Jc - (SHA && MC > 1 ? crank : 0)) * G_BN)) continue;   // per UNIT: both CTAs agree
        for (int kc = 0; kc < nk; ++kc) {
          const int sg = kc / kpb, kin = (kc % kpb) * BK;
          mbar_wait(&empty[st], ph ^ 1);
          mbar_expect_tx(&full[st], G_STAGE);
          uint8_t* sa = smem + st * G_STAGE;
          if (MC > 1 && SHA)   // this CTA's half of the shared A tile, into both CTAs (half-height box maps)
            tma_load_2d_mc(sa + crank * (G_BM / MC) * G_ROWB, segs.amap[sg] ? &mapA1 : &mapA0, &full[st],
                           segs.acol[sg] + kin, arow0 + I * G_BM + crank * (G_BM / MC), (uint16_t)((1u << MC) - 1));
          else
            tma_load_2d(sa, segs.amap[sg] ? &mapA1 : &mapA0, &full[st], segs.acol[sg] + kin, arow0 + I * G_BM);
          if (MC > 1 && !SHA)   // this CTA's half of the B tile, into both CTAs (half-height box maps)
            tma_load_2d_mc(sa + G_SA + crank * (G_BN / MC) * G_ROWB, segs.bmap[sg] ? &mapB1 : &mapB0, &full[st],
                           segs.bcol[sg] + kin, brow0 + Jc * G_BN + crank * (G_BN / MC), (uint16_t)((1u << MC) - 1));
          else
            tma_load_2d(sa + G_SA, segs.bmap[sg] ? &mapB1 : &mapB0, &full[st], segs.bcol[sg] + kin,
                        brow0 + Jc * G_BN);
          if (++st == G_NS) { st = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {  // ---------------- MMA issuer
      const uint32_t idesc = idesc_make(G_BM, G_BN, TF ? 2 : 0, 0, 0) | (TF ? 0u : op16_fmt());
      int st = 0; uint32_t ph = 0;
      int ab = 0; uint32_t aph = 0;
      const uint32_t s0 = smem_u32(smem);
      // accumulation groups: fp16 one per tile; 3xTF32 every FLUSH k-chunks (drained by the epilogue)
      const int ch = TF ? Cfg::FLUSH : nk;
      for (int t = u0; t < ntiles; t += ustride) {
        if (own.P > 1) {
          int I, Jc;
          gemm_tile<MODE, UBN, UBM>(t, ntn, ntm, I, Jc, bandH);
          if (MC > 1) { if (SHA) Jc = Jc * MC + crank; else I = I * MC + crank; }
          if (!own.owned((int64_t)(Jc - (SHA && MC > 1 ? crank : 0)) * G_BN)) continue;   // per UNIT: both CTAs agree
        }
        for (int kc = 0; kc < nk; ++kc) {
          if (kc % ch == 0) {
            mbar_wait(&acc_empty[ab], aph ^ 1);
            tc_fence_after();
          }
          const uint32_t d = tmem + ab * G_BN;
          mbar_wait(&full[st], ph);
          tc_fence_after();
          const uint32_t sa = s0 + st * G_STAGE, sb = sa + G_SA;
#pragma unroll
          for (int s = 0; s < 4; ++s) {  // 4 MMAs of 32 bytes of K (16 fp16 / 8 tf32)
            if (TF)
              mma_tf32(d, sdesc_sw128(sa + s * 32, 16, 1024), sdesc_sw128(sb + s * 32, 16, 1024), idesc,
                       (kc % ch > 0 || s > 0) ? 1u : 0u);
            else
              mma_f16(d, sdesc_sw128(sa + s * 32, 16, 1024), sdesc_sw128(sb + s * 32, 16, 1024), idesc,
                      (kc % ch > 0 || s > 0) ? 1u : 0u);
          }
          if (MC > 1) mma_commit_mc(&empty[st], (uint16_t)((1u << MC) - 1));
          else mma_commit(&empty[st]);
          if (++st == G_NS) { st = 0; ph ^= 1; }
          if (kc % ch == ch - 1 || kc == nk - 1) {
            mma_commit(&acc_full[ab]);
            if (++ab == 2) { ab = 0; aph ^= 1; }
          }
        }
      }
    }
  } else if (warp >= 4 && TF) {  // ---------------- 3xTF32 epilogue (8 warps: 32 lanes x 64 columns each)
    const int e = warp - 4;
    const int q = e & 3;
    const int chalf = e >> 2;
    const int rit = q * 32 + lane;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    const int ngroups = (nk + Cfg::FLUSH - 1) / Cfg::FLUSH;
    int ab = 0; uint32_t aph = 0;
    for (int t = u0; t < ntiles; t += ustride) {
      int I, Jc;
      gemm_tile<MODE, UBN, UBM>(t, ntn, ntm, I, Jc, bandH);
      if (MC > 1) { if (SHA) Jc = Jc * MC + crank; else I = I * MC + crank; }
      if (!own.owned((int64_t)(Jc - (SHA && MC > 1 ? crank : 0)) * G_BN)) continue;   // per UNIT: both CTAs agree
      float acc[64];
#pragma unroll
      for (int c = 0; c < 64; ++c) acc[c] = 0.f;
      for (int gi = 0; gi < ngroups; ++gi) {   // fp32 round-to-nearest sum of the partial accumulations
        mbar_wait(&acc_full[ab], aph);
        tc_fence_after();
        float v[32], u[32];
        tmem_ld32(tmem + ab * G_BN + chalf * 64 + lane_off, v);
        tmem_ld32(tmem + ab * G_BN + chalf * 64 + 32 + lane_off, u);
        tc_fence_before();
        mbar_arrive(&acc_empty[ab]);
        if (++ab == 2) { ab = 0; aph ^= 1; }
#pragma unroll
        for (int c = 0; c < 32; ++c) {
          acc[c] += v[c];
          acc[32 + c] += u[c];
        }
      }
      const int64_t row = (int64_t)I * G_BM + rit;
      if (row >= Mrows) continue;
      const int64_t col0 = (int64_t)Jc * G_BN + chalf * 64;
      if (MODE == 0 || MODE == 3) {   // SYR2K: lower elements; GEMM_SUB: all of C
        float* cp = C + row + own.lcol(col0) * ldc;
#pragma unroll
        for (int c = 0; c < 64; ++c)
          if (MODE == 0 ? (col0 + c <= row) : (col0 + c < Ncols)) __stcs(cp + c * ldc, __ldcs(cp + c * ldc) - acc[c]);
      } else {   // Z split: hi = rna_tf32(z), lo = rna_tf32(z - hi), row-major
        float* zp = (float*)Zout + row * ldz + col0;
#pragma unroll
        for (int c = 0; c < 64; ++c) {
          if (col0 + c < Ncols) {
            // ZFORM: z = X - acc/2 ; GEMM_SPLIT: z = acc
            const float z = MODE == 1 ? fmaf(-0.5f, acc[c], __ldcs(X + row + (col0 + c) * ldx)) : acc[c];
            const float hi = tf32_rna(z);
            zp[c] = hi;
            zp[c + zlo_off] = tf32_rna(z - hi);
          } else if (col0 + c < zlo_off) {
            zp[c] = 0.f;   // K padding of the hi half must read as zero in the SYR2K
          }
        }
      }
    }
  } else if (warp >= 4) {  // ---------------- epilogue (8 warps)
    const int e = warp - 4;
    const int q = e & 3;                    // TMEM lane quarter (warp % 4)
    const int chalf = e >> 2;               // which 128 of the 256 accumulator columns
    const int rit = q * 32 + lane;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    int ab = 0; uint32_t aph = 0;
    for (int t = u0; t < ntiles; t += ustride) {
      int I, Jc;
      gemm_tile<MODE, UBN, UBM>(t, ntn, ntm, I, Jc, bandH);
      if (MC > 1) { if (SHA) Jc = Jc * MC + crank; else I = I * MC + crank; }
      if (!own.owned((int64_t)(Jc - (SHA && MC > 1 ? crank : 0)) * G_BN)) continue;   // per UNIT: both CTAs agree
      mbar_wait(&acc_full[ab], aph);
      tc_fence_after();
      const int64_t row = (int64_t)I * G_BM + rit;
      const int64_t rmax = (int64_t)I * G_BM + G_BM - 1;  // last row of the tile
#pragma unroll 1
      for (int cc = chalf * 4; cc < chalf * 4 + 4; ++cc) {
        const int64_t col0 = (int64_t)Jc * G_BN + cc * 32;
        if (MODE == 0 && col0 > rmax) break;  // chunk entirely above the diagonal (warp-uniform)
        if (col0 >= Ncols) break;
        float v[32];
        tmem_ld32(tmem + ab * G_BN + cc * 32 + lane_off, v);
        if (row >= Mrows) continue;
        if (MODE == 0) {
          const int64_t lc0 = own.lcol(col0);
          float* cp = C + row + lc0 * ldc;
          __half* sp = shadow + row + lc0 * ldsh;
          float old[32];
#pragma unroll
          for (int c = 0; c < 32; ++c) old[c] = (col0 + c <= row) ? __ldcs(cp + c * ldc) : 0.f;   // all loads first
#pragma unroll
          for (int c = 0; c < 32; ++c) {
            const int64_t col = col0 + c;
            if (col <= row) {
              const float nv = old[c] - v[c];
              __stcs(cp + c * ldc, nv);
              sp[c * ldsh] = cvt16(col == row ? 0.5f * nv : nv);
            }
          }
        } else {
          float xv[32];
#pragma unroll
          for (int c = 0; c < 32; ++c) xv[c] = (col0 + c < Ncols) ? __ldcs(X + row + (col0 + c) * ldx) : 0.f;
          __half* Zh = (__half*)Zout;
          __align__(16) __half z[32];
#pragma unroll
          for (int c = 0; c < 32; ++c) z[c] = cvt16(fmaf(-0.5f, v[c], xv[c]));
          __half* zp = Zh + row * ldz + col0;
          if (col0 + 32 <= Ncols) {
#pragma unroll
            for (int c = 0; c < 32; c += 8) *reinterpret_cast<uint4*>(zp + c) = *reinterpret_cast<const uint4*>(z + c);
          } else {
            for (int c = 0; c < 32 && col0 + c < Ncols; ++c) zp[c] = z[c];
          }
        }
      }
      tc_fence_before();
      mbar_arrive(&acc_empty[ab]);
      if (++ab == 2) { ab = 0; aph ^= 1; }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (MC > 1) cluster_sync_all();   // the peer may still multicast into / commit to this CTA's smem
  if (warp == 2) {
    tc_fence_after();
    tmem_dealloc(tmem, 512);
  }
}

template <int MODE, bool TF, int MC = 1>
static cudaError_t launch_gemm_t(const GemmTcLaunch& p, cudaStream_t st) {
  auto kern = gemm_tc_kernel<MODE, TF, MC>;
  constexpr int BK = TF ? 32 : 64;
  constexpr int G_BN = GCfg<TF>::BN, G_SMEM = GCfg<TF>::SMEM;
  {
    cudaError_t e = func_attr((const void*)kern, cudaFuncAttributeMaxDynamicSharedMemorySize, G_SMEM);
    if (e != cudaSuccess) return e;
  }
  CUtensorMap mA0, mA1, mB0, mB1;
  cudaError_t e;
  // map width: the K columns (fp16) or the [hi | lo] columns (3xTF32: lo at lo_off)
  const uint64_t wid = TF ? (uint64_t)(p.lo_off + p.K) : (uint64_t)p.K;
  // MC = 2: each CTA of a pair loads half of the shared tile (B in FP16, A in 3xTF32), multicast to both
  constexpr int ABOX = (MC > 1 && TF) ? G_BM / MC : G_BM, BBOX = (MC > 1 && !TF) ? G_BN / MC : G_BN;
  if ((e = make_tmap_2d(&mA0, p.A0, !TF, wid, p.a_rows, p.ld_a, BK, ABOX)) != cudaSuccess) return e;
  if ((e = make_tmap_2d(&mB0, p.B0, !TF, wid, p.b_rows, p.ld_b, BK, BBOX)) != cudaSuccess) return e;
  if (MODE == 0) {
    if ((e = make_tmap_2d(&mA1, p.A1, !TF, wid, p.a_rows, p.ld_a, BK, ABOX)) != cudaSuccess) return e;
    if ((e = make_tmap_2d(&mB1, p.B1, !TF, wid, p.b_rows, p.ld_b, BK, BBOX)) != cudaSuccess) return e;
  } else {
    mA1 = mA0;
    mB1 = mB0;
  }
  const int kpb = (int)((p.K + BK - 1) / BK);
  GemmSegs sg{};
  const int lo = (int)p.lo_off;
  if (!TF) {        // SYR2K: [Y | Z] [Z | Y]^T ; ZFORM: Y G
    sg.n = MODE == 0 ? 2 : 1;
    sg.amap[1] = 1; sg.bmap[1] = 1;
  } else {          // hi hi' + hi lo' + lo hi' per product
    const int half = MODE == 0 ? 2 : 1;
    sg.n = 3 * half;
    for (int h = 0; h < half; ++h)
      for (int q = 0; q < 3; ++q) {
        const int s = h * 3 + q;
        sg.amap[s] = h; sg.bmap[s] = h;
        sg.acol[s] = q == 2 ? lo : 0;
        sg.bcol[s] = q == 1 ? lo : 0;
      }
  }
  constexpr int BMU = (MC > 1 && !TF) ? G_BM * MC : G_BM;   // one work unit: a tile or a CTA pair's two
  constexpr int BNU = (MC > 1 && TF) ? G_BN * MC : G_BN;
  const int ntm = (int)((p.Mrows + BMU - 1) / BMU);
  const int ntn = (int)((p.Ncols + BNU - 1) / BNU);
  int ntiles;   // work units
  if (MODE == 0) {
    ntiles = 0;
    for (int i = 0; i < ntm; ++i) ntiles += i * BMU / BNU + 1;
  } else {
    ntiles = ntm * ntn;
  }
  if (ntiles == 0) return cudaSuccess;
  const int grid = std::min(ntiles * MC, p.num_sms / MC * MC);
  GemmOwn own;
  if (p.own_P > 1) {
    // every BN-wide output tile must lie inside one column block: an nb-aligned origin (nb % BN == 0),
    // or a region that fits in one block (the ragged last block)
    const bool one_block = p.own_org / p.nbo == (p.own_org + p.Ncols - 1) / p.nbo;
    if (MODE != 0 || p.nbo % BNU != 0 || (p.own_org % p.nbo != 0 && !one_block)) return cudaErrorInvalidValue;
    own.P = p.own_P;
    own.rank = p.own_rank;
    own.org = p.own_org;
    own.nbo = p.nbo;
  }
  // raster band height in units: the same ~16K (FP16) / 4K (3xTF32) rows of A per band
  const int bandH = knob(KNOB_SYR2K_BAND) > 0 ? knob(KNOB_SYR2K_BAND) : (TF ? 32 : 64 / MC);
  if (MC == 1)
    return launch_pdl(kern, dim3(grid), dim3(G_THREADS), G_SMEM, st, mA0, mA1, mB0, mB1, kpb, sg, (int)p.arow0,
                      (int)p.brow0, p.Mrows, p.Ncols, ntn, ntiles, p.C, p.ldc, p.shadow, p.ld_shadow, p.X, p.ldx,
                      TF ? (void*)p.Zs : (void*)p.Zh, p.ldz, p.zlo_off >= 0 ? p.zlo_off : p.lo_off, own, bandH);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(G_THREADS);
  cfg.dynamicSmemBytes = G_SMEM;
  cfg.stream = st;
  cudaLaunchAttribute at[2];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = MC;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl_enabled() ? 2 : 1;
  return cudaLaunchKernelEx(&cfg, kern, mA0, mA1, mB0, mB1, kpb, sg, (int)p.arow0, (int)p.brow0, p.Mrows, p.Ncols,
                            ntn, ntiles, p.C, p.ldc, p.shadow, p.ld_shadow, p.X, p.ldx,
                            TF ? (void*)p.Zs : (void*)p.Zh, p.ldz, p.zlo_off >= 0 ? p.zlo_off : p.lo_off, own,
                            bandH);
}

// FP16 SYR2K: CTA pairs with the B tile multicast (KNOB_SYR2K_MC = 1 selects the single-CTA kernel, ablation)
cudaError_t launch_syr2k_tc(const GemmTcLaunch& p, cudaStream_t st) {
  if (knob(KNOB_SYR2K_MC) == 1) return launch_gemm_t<0, false, 1>(p, st);
  return launch_gemm_t<0, false, 2>(p, st);
}
cudaError_t launch_zform_tc(const GemmTcLaunch& p, cudaStream_t st) {   // CTA pairs sharing B (W^T X)
  if (knob(KNOB_SYR2K_MC) == 1) return launch_gemm_t<1, false, 1>(p, st);
  return launch_gemm_t<1, false, 2>(p, st);
}
// 3xTF32 SYR2K: CTA pairs sharing the A tile (KNOB_SYR2K_MC = 1: single CTAs, ablation)
cudaError_t launch_syr2k_tf32(const GemmTcLaunch& p, cudaStream_t st) {
  if (knob(KNOB_SYR2K_MC) == 1) return launch_gemm_t<0, true, 1>(p, st);
  return launch_gemm_t<0, true, 2>(p, st);
}
cudaError_t launch_zform_tf32(const GemmTcLaunch& p, cudaStream_t st) {   // CTA pairs sharing A (Y)
  if (knob(KNOB_SYR2K_MC) == 1) return launch_gemm_t<1, true, 1>(p, st);
  return launch_gemm_t<1, true, 2>(p, st);
}
cudaError_t launch_gemm_split_tf32(const GemmTcLaunch& p, cudaStream_t st) { return launch_gemm_t<2, true>(p, st); }
cudaError_t launch_gemm_sub_tf32(const GemmTcLaunch& p, cudaStream_t st) { return launch_gemm_t<3, true>(p, st); }

SBR_OP16_SETTER(gemm)

}  // namespace sbr
