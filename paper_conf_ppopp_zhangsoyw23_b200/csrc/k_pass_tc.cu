// k_pass_tc.cu -- the per-panel pass X_t = OA W_t (step a4; Alg. 1 l.9)
// on tcgen05 tensor cores, reading each lower 128x128 tile of the fp16 shadow of OA
// from HBM exactly once and using it twice:
//     X_I += L_IJ   W_J      (A = L_IJ,   MN-major view of the smem tile)
//     X_J += L_IJ^T W_I      (A = L_IJ^T, K-major view of the SAME smem bytes)
// The shadow stores the strict lower triangle, HALF the diagonal and zeros above it,
// so a diagonal tile contributes T W + T^T W = L W with no special case.
//
// Work = a balanced contiguous range of lower tiles per CTA (PassWalk).  One CTA per SM:
// TMA producer warp -> single-thread MMA warp -> 4 epilogue warps.  Row accumulators (X_I, double-buffered) and the C column accumulators (X_J)
// live in TMEM; they are flushed with fp32 reductions into the L2-resident X.
// Roofline: HBM-bound (2 bytes per stored element, 4 flops/byte at b = 32).
#include "kernels.h"
#include "tc.cuh"

namespace sbr {

using namespace tc;

template <int BN, int C, int NS>
struct PassCfg {
  static constexpr int WT = 256 * BN;          // bytes of one 128-row W tile (2 K-chunks of BN x 128 B)
  static constexpr int LT = 32768;             // one 128x128 fp16 tile (4 boxes of 64x64)
  static constexpr int OFF_WJ = 0;
  static constexpr int OFF_WI = C * WT;
  static constexpr int OFF_L = (C + 2) * WT;
  static constexpr int OFF_BAR = OFF_L + NS * LT;
  static constexpr int NBAR = 2 * NS + 4 + 4 + 4;
  // epilogue transpose buffers (one 32 x 33 fp32 block per epilogue warp) for 16-byte reductions
  // into X, when they fit next to the pipeline
  static constexpr int OFF_T = OFF_BAR + NBAR * 8 + 16;
  static constexpr int TBYTES = 4 * 32 * 33 * 4;
  static constexpr bool VT = OFF_T + TBYTES + 1024 <= 232448;
  static constexpr int SMEM = OFF_T + (VT ? TBYTES : 0) + 1024;  // + alignment slack
  static constexpr int TMEM_USED = (C + 2) * BN;
  static constexpr int TMEM_COLS = TMEM_USED <= 32 ? 32 : TMEM_USED <= 64 ? 64 : TMEM_USED <= 128 ? 128
                                   : TMEM_USED <= 256 ? 256 : 512;
};

// Work = the lower tiles of OA in the linear order (group g, tile row I, tile column J):
// group g spans tile columns [gC, gC + ceff), rows I = gC .. NT-1, row I holding
// min(ceff, I - gC + 1) tiles.  Every CTA takes an equal contiguous range of tiles
// (balanced to one tile), so a launch ends when the slowest SM has streamed T/grid tiles.
// The three roles walk the same range with this iterator.
#define SBR_HD __host__ __device__ __forceinline__
// Multi-GPU (sbr_reduce_dist, 1D block-cyclic columns): only the groups whose tile columns lie in
// this rank's column blocks are walked -- group g covers global column block blk0 + g / gpb,
// owned by rank (blk0 + g / gpb) % P (P = 1: every group).
struct PassOwn {
  int P = 1, rank = 0, blk0 = 0, gpb = 1;
  SBR_HD bool owned(int g) const { return P <= 1 || (blk0 + g / gpb) % P == rank; }
};

struct PassWalk {
  int NT, C;
  int g, J0, ceff, I, J;
  int64_t left;
  bool gfirst, rfirst;
  PassOwn own;
  SBR_HD int jend() const { return min(J0 + ceff, I + 1); }
  SBR_HD static int64_t group_tiles(int NT, int C, int g) {
    const int J0 = g * C, ce = min(C, NT - J0);
    return (int64_t)ce * (ce + 1) / 2 + (int64_t)(NT - J0 - ce) * ce;
  }
  SBR_HD int64_t owned_tiles(int g) const { return own.owned(g) ? group_tiles(NT, C, g) : 0; }
  SBR_HD void start(int NT_, int C_, int64_t t0, int64_t count, PassOwn own_ = PassOwn()) {
    NT = NT_;
    C = C_;
    own = own_;
    left = count;
    g = 0;
    gfirst = rfirst = true;
    if (count <= 0) return;   // nothing to walk (e.g. a rank that owns no column of this OA)
    for (;;) {
      if (g * C >= NT) break;
      const int64_t gt = owned_tiles(g);
      if (t0 < gt) break;
      t0 -= gt;
      ++g;
    }
    J0 = g * C;
    ceff = min(C, NT - J0);
    const int64_t tri = (int64_t)ceff * (ceff + 1) / 2;
    if (t0 < tri) {
      int d = 0;
      while ((int64_t)(d + 1) * (d + 2) / 2 <= t0) ++d;
      I = J0 + d;
      J = J0 + (int)(t0 - (int64_t)d * (d + 1) / 2);
    } else {
      const int64_t o = t0 - tri;
      I = J0 + ceff + (int)(o / ceff);
      J = J0 + (int)(o % ceff);
    }
    gfirst = rfirst = true;
  }
  SBR_HD bool valid() const { return left > 0; }
  SBR_HD bool rlast() const { return left == 1 || J + 1 == jend(); }
  SBR_HD bool glast() const { return left == 1 || (J + 1 == jend() && I + 1 == NT); }
  SBR_HD void next() {
    --left;
    gfirst = rfirst = false;
    if (J + 1 < jend()) {
      ++J;
      return;
    }
    rfirst = true;
    if (I + 1 < NT) {
      ++I;
      J = J0;
      return;
    }
    gfirst = true;
    do {
      ++g;
    } while (g * C < NT && !own.owned(g));
    J0 = g * C;
    ceff = min(C, NT - J0);
    I = J = J0;
  }
};

SBR_DEV void red_add_v4(float* addr, float a, float b, float c, float d) {
  asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(addr), "f"(a), "f"(b), "f"(c), "f"(d)
               : "memory");
}

template <int BN, int C, int NS>
__global__ void __launch_bounds__(256, 1)
    pass_tc_kernel(const __grid_constant__ CUtensorMap mapL, const __grid_constant__ CUtensorMap mapW, int r0, int M,
                   int NT, int64_t T0, int64_t T, int b, float* X, int64_t ldx, int exper, int off, PassOwn own,
                   int nbo) {
  // tile I covers shadow rows / columns r0 + 128 I .. (r0 = the first tile's origin) and OA rows
  // 128 I - off ..; W rows are stored with `off` zero rows in front (W row 128 J = OA row 128 J - off).
  // Multi-GPU: the shadow holds this rank's columns only: local column of global column g =
  // (g / nbo / P) nbo + g % nbo.
  using Cfg = PassCfg<BN, C, NS>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* sWj = smem + Cfg::OFF_WJ;
  uint8_t* sWi = smem + Cfg::OFF_WI;
  uint8_t* sL = smem + Cfg::OFF_L;
  uint64_t* bars = (uint64_t*)(smem + Cfg::OFF_BAR);
  uint64_t* l_full = bars;
  uint64_t* l_empty = bars + NS;
  uint64_t* wi_full = bars + 2 * NS;
  uint64_t* wi_empty = wi_full + 2;
  uint64_t* racc_full = wi_empty + 2;
  uint64_t* racc_empty = racc_full + 2;
  uint64_t* wj_full = racc_empty + 2;
  uint64_t* wj_empty = wj_full + 1;
  uint64_t* cacc_full = wj_empty + 1;
  uint64_t* cacc_empty = cacc_full + 1;
  uint32_t* tmem_slot = (uint32_t*)(bars + Cfg::NBAR);

  const int warp = warp_id(), lane = lane_id();
  pdl_trigger();
  // this launch covers tiles [T0, T0 + T) (a rank's share under sbr_reduce_dist); CTA share:
  const int64_t t_beg = T0 + (int64_t)blockIdx.x * T / gridDim.x;
  const int64_t t_end = T0 + (int64_t)(blockIdx.x + 1) * T / gridDim.x;
  if (threadIdx.x == 0) {
    for (int i = 0; i < NS; ++i) { mbar_init(&l_full[i], 1); mbar_init(&l_empty[i], 1); }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&wi_full[i], 1); mbar_init(&wi_empty[i], 1);
      mbar_init(&racc_full[i], 1); mbar_init(&racc_empty[i], 128);
    }
    mbar_init(wj_full, 1); mbar_init(wj_empty, 1);
    mbar_init(cacc_full, 1); mbar_init(cacc_empty, 128);
    mbar_fence_init();
  }
  if (warp == 0 && lane == 0) { tma_prefetch(&mapL); tma_prefetch(&mapW); }
  if (warp == 2) tmem_alloc(tmem_slot, Cfg::TMEM_COLS);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();
  const uint32_t t_col = tmem;                 // C column accumulators: cols [jj*BN, jj*BN+BN)
  const uint32_t t_row = tmem + C * BN;        // 2 row accumulators
  PassWalk w;
  auto lcolJ = [&](int Jt) -> int {   // shadow column coordinate of tile column Jt
    const int g = r0 + Jt * 128;
    if (own.P <= 1) return g;
    const int blk = g / nbo;
    return (blk / own.P) * nbo + g % nbo;
  };

  if (warp == 0) {
    // ------------------------------------------------ TMA producer
    if (lane == 0) {
      // OA tiles are read once per pass: evict_first (experiment knob bit 2 = normal, ablation)
      const uint64_t lpol = (exper & 4) ? l2_policy_evict_normal() : l2_policy_evict_first();
      int st = 0; uint32_t ph = 0;            // L ring
      int ws = 0; uint32_t wph = 0;           // W_I ring
      uint32_t jph = 0;
      for (w.start(NT, C, t_beg, t_end - t_beg, own); w.valid(); w.next()) {
        if (w.gfirst) {
          mbar_wait(wj_empty, jph ^ 1);
          jph ^= 1;
          mbar_expect_tx(wj_full, w.ceff * Cfg::WT);
          for (int jj = 0; jj < w.ceff; ++jj)
            for (int h = 0; h < 2; ++h)
              tma_load_2d(sWj + jj * Cfg::WT + h * (Cfg::WT / 2), &mapW, wj_full, (w.J0 + jj) * 128 + h * 64, 0);
        }
        if (w.rfirst) {
          mbar_wait(&wi_empty[ws], wph ^ 1);
          mbar_expect_tx(&wi_full[ws], Cfg::WT);
          for (int h = 0; h < 2; ++h)
            tma_load_2d(sWi + ws * Cfg::WT + h * (Cfg::WT / 2), &mapW, &wi_full[ws], w.I * 128 + h * 64, 0);
        }
        mbar_wait(&l_empty[st], ph ^ 1);
        mbar_expect_tx(&l_full[st], Cfg::LT);
        uint8_t* dst = sL + st * Cfg::LT;
        for (int rb = 0; rb < 2; ++rb)   // box = 64 rows x 128 columns (same smem image as 2 boxes of 64)
          tma_load_2d_hint(dst + rb * 16384, &mapL, &l_full[st], r0 + w.I * 128 + rb * 64, lcolJ(w.J), lpol);
        if (++st == NS) { st = 0; ph ^= 1; }
        if (w.rlast()) {
          if (++ws == 2) { ws = 0; wph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------ MMA issuer (one thread)
    if (lane == 0) {
      const uint32_t idesc_dir = idesc_make(128, BN, 0, /*a MN-major*/ 1, 0) | op16_fmt();
      const uint32_t idesc_tr = idesc_make(128, BN, 0, 0, 0) | op16_fmt();
      int st = 0; uint32_t ph = 0;
      int ws = 0; uint32_t wph = 0;
      int rb = 0; uint32_t rph = 0;
      uint32_t jph = 0, cph = 0;
      const uint32_t aL = smem_u32(sL), aWj = smem_u32(sWj), aWi = smem_u32(sWi);
      uint32_t cinit = 0;
      bool rowfirst = true;
      for (w.start(NT, C, t_beg, t_end - t_beg, own); w.valid(); w.next()) {
        if (w.gfirst) {
          mbar_wait(wj_full, jph);
          jph ^= 1;
          mbar_wait(cacc_empty, cph ^ 1);
          cph ^= 1;
          tc_fence_after();
          cinit = 0;
        }
        if (w.rfirst) {
          mbar_wait(&wi_full[ws], wph);
          mbar_wait(&racc_empty[rb], rph ^ 1);
          tc_fence_after();
          rowfirst = true;
        }
        const uint32_t d_row = t_row + rb * BN;
        const int jj = w.J - w.J0;
        mbar_wait(&l_full[st], ph);
        tc_fence_after();
        const uint32_t lt = aL + st * Cfg::LT;
        if (!(exper & 1))   // (exper: timing experiments only, test knob; 0 in production)
#pragma unroll
        for (int s = 0; s < 8; ++s) {  // X_I += L W_J : A MN-major (LBO = 16 KB between 64-row atoms)
          const uint64_t a = sdesc_sw128(lt + (s >> 2) * 8192 + (s & 3) * 2048, 16384, 1024);
          const uint64_t bd = sdesc_sw128(aWj + jj * Cfg::WT + (s >> 2) * (Cfg::WT / 2) + (s & 3) * 32, 16, 1024);
          mma_f16(d_row, a, bd, idesc_dir, (!rowfirst || s > 0) ? 1u : 0u);
        }
        const uint32_t d_col = t_col + jj * BN;
        const uint32_t acc0 = (cinit >> jj) & 1u;
        if (!(exper & 2))
#pragma unroll
        for (int s = 0; s < 8; ++s) {  // X_J += L^T W_I : A K-major (same bytes)
          const uint64_t a = sdesc_sw128(lt + (s >> 2) * 16384 + (s & 3) * 32, 16, 1024);
          const uint64_t bd = sdesc_sw128(aWi + ws * Cfg::WT + (s >> 2) * (Cfg::WT / 2) + (s & 3) * 32, 16, 1024);
          mma_f16(d_col, a, bd, idesc_tr, (acc0 || s > 0) ? 1u : 0u);
        }
        cinit |= 1u << jj;
        rowfirst = false;
        mma_commit(&l_empty[st]);
        if (++st == NS) { st = 0; ph ^= 1; }
        if (w.rlast()) {
          mma_commit(&racc_full[rb]);
          mma_commit(&wi_empty[ws]);
          if (++ws == 2) { ws = 0; wph ^= 1; }
          if (++rb == 2) { rb = 0; rph ^= 1; }
        }
        if (w.glast()) {
          mma_commit(cacc_full);
          mma_commit(wj_empty);
        }
      }
    }
  } else if (warp >= 4) {
    // ------------------------------------------------ epilogue: TMEM -> fp32 reductions into X
    const int q = warp - 4;                       // TMEM lane quarter
    const int row_in_tile = q * 32 + lane;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    int rb = 0; uint32_t rph = 0;
    uint32_t cph = 0;
    uint32_t touched = 0;
    // X += this warp's 32 rows (rows rbase + lane) x columns c0 .. c0 + 31.  Column-major X: with
    // 16-byte alignment, the block goes through shared memory so that each lane issues 8 reductions
    // of 4 consecutive rows of one column (red.global.add.v4.f32: a quarter of the L2 atomic
    // operations of per-element reductions, which cost ~8 ms per config-4 step at the launch
    // tails); otherwise per element.
    float* tb = (float*)(smem + Cfg::OFF_T) + q * (32 * 33);
    const bool vec = Cfg::VT && M % 4 == 0 && off % 4 == 0 && ldx % 4 == 0 && ((uintptr_t)X & 15) == 0;
    auto flush32 = [&](const float (&v)[32], int64_t rbase, int c0) {
      if (vec) {
#pragma unroll
        for (int c = 0; c < 32; ++c) tb[c * 33 + lane] = v[c];
        __syncwarp();
        const int r4 = 4 * (lane & 7);
        const int64_t r = rbase + r4;
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          const int c = (lane >> 3) + 4 * k;
          const float* src = tb + c * 33 + r4;
          if (c0 + c < b && r >= 0 && r < M) red_add_v4(&X[r + (int64_t)(c0 + c) * ldx], src[0], src[1], src[2], src[3]);
        }
        __syncwarp();
      } else {
        const int64_t row = rbase + lane;
        if (row >= 0 && row < M) {
#pragma unroll
          for (int c = 0; c < 32; ++c)
            if (c0 + c < b) atomicAdd(&X[row + (int64_t)(c0 + c) * ldx], v[c]);
        }
      }
    };
    for (w.start(NT, C, t_beg, t_end - t_beg, own); w.valid(); w.next()) {
      if (w.gfirst) touched = 0;
      touched |= 1u << (w.J - w.J0);
      if (w.rlast()) {
        mbar_wait(&racc_full[rb], rph);
        tc_fence_after();
        const int64_t rbase = (int64_t)w.I * 128 + q * 32 - off;
#pragma unroll
        for (int c0 = 0; c0 < BN; c0 += 32) {
          float v[32];
          tmem_ld32(t_row + rb * BN + c0 + lane_off, v);
          if (!(exper & 8)) flush32(v, rbase, c0);
        }
        tc_fence_before();
        mbar_arrive(&racc_empty[rb]);
        if (++rb == 2) { rb = 0; rph ^= 1; }
      }
      if (w.glast()) {
        mbar_wait(cacc_full, cph);
        cph ^= 1;
        tc_fence_after();
        for (int jj = 0; jj < w.ceff; ++jj) {
          if (!((touched >> jj) & 1u)) continue;
          const int64_t rbase = (int64_t)(w.J0 + jj) * 128 + q * 32 - off;
#pragma unroll
          for (int c0 = 0; c0 < BN; c0 += 32) {
            float v[32];
            tmem_ld32(t_col + jj * BN + c0 + lane_off, v);
            if (!(exper & 24)) flush32(v, rbase, c0);
          }
        }
        tc_fence_before();
        mbar_arrive(cacc_empty);
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    tc_fence_after();
    tmem_dealloc(tmem, Cfg::TMEM_COLS);
  }
}

// ---------------------------------------------------------------- host
static int64_t pass_total_tiles(int NT, int C, PassOwn own = PassOwn()) {
  int64_t T = 0;
  for (int g = 0; g * C < NT; ++g)
    if (own.owned(g)) T += PassWalk::group_tiles(NT, C, g);
  return T;
}

static int pass_variant();
static int pass_group_cols(int b) {   // C of launch_pass_tc's instantiation
  if (b <= 16) return 8;
  if (b <= 32) return pass_variant() == 1 ? 4 : pass_variant() == 2 ? 2 : 8;
  return 4;
}

void pass_partition(int64_t M, int b, int rank, int nranks, int64_t* t0, int64_t* t1, int64_t* total) {
  const int NT = (int)((M + 127) / 128);
  const int64_t T = pass_total_tiles(NT, pass_group_cols(b));
  *total = T;
  *t0 = T * rank / nranks;
  *t1 = T * (rank + 1) / nranks;
}

// multi-GPU: the tiles `rank` walks for a block with 128-aligned grid origin r0g, OA offset `off`
// (OA rows start off rows into tile 0), ownership width nbo -- host mirror of the kernel's walk
int64_t pass_owned_tiles(int64_t M, int b, int64_t r0g, int off, int64_t nbo, int P, int rank, int* IJ, int64_t cap) {
  const int C = pass_group_cols(b);
  const int NT = (int)((M + off + 127) / 128);
  PassOwn own;
  own.P = P;
  own.rank = rank;
  own.blk0 = (int)(r0g / nbo);
  own.gpb = (int)(nbo / (128 * C));
  if (P > 1 && (own.gpb < 1 || nbo % (128 * C) != 0 || r0g % 128 != 0)) return -1;
  const int64_t T = pass_total_tiles(NT, C, own);
  PassWalk w;
  int64_t k = 0;
  for (w.start(NT, C, 0, T, own); w.valid(); w.next(), ++k) {
    if (IJ && k < cap) {
      IJ[2 * k] = w.I;
      IJ[2 * k + 1] = w.J;
    }
  }
  return k;
}

void pass_tiles(int64_t M, int b, int64_t t0, int64_t t1, int* IJ) {
  const int NT = (int)((M + 127) / 128);
  PassWalk w;
  int64_t k = 0;
  for (w.start(NT, pass_group_cols(b), t0, t1 - t0); w.valid(); w.next(), ++k) {
    IJ[2 * k] = w.I;
    IJ[2 * k + 1] = w.J;
  }
}

template <int BN, int C, int NS>
static cudaError_t launch_pass_t(const PassLaunch& p, cudaStream_t st) {
  using Cfg = PassCfg<BN, C, NS>;
  auto kern = pass_tc_kernel<BN, C, NS>;
  {
    cudaError_t e = func_attr((const void*)kern, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM);
    if (e != cudaSuccess) return e;
  }
  CUtensorMap mapL, mapW;
  cudaError_t e = make_tmap_2d(&mapL, p.shadow, true, p.n, p.shadow_cols > 0 ? p.shadow_cols : p.n, p.ld_shadow, 64, 128);
  if (e != cudaSuccess) return e;
  e = make_tmap_2d(&mapW, p.Wh, true, p.M + p.off, BN, p.ld_wh, 64, BN);
  if (e != cudaSuccess) return e;
  const int NT = (int)((p.M + p.off + 127) / 128);
  PassOwn own;
  if (p.own_P > 1) {   // column-block ownership (sbr_reduce_dist): groups of C tile columns, nbo / (128 C) per block
    own.P = p.own_P;
    own.rank = p.own_rank;
    own.blk0 = (int)(p.r0 / p.nbo);
    own.gpb = (int)(p.nbo / (128 * C));
    if (own.gpb < 1 || p.nbo % (128 * C) != 0 || p.r0 % 128 != 0) return cudaErrorInvalidValue;
  }
  const int64_t Tall = pass_total_tiles(NT, C, own);
  const int64_t T0 = Tall * p.rank / p.nranks, T1 = Tall * (p.rank + 1) / p.nranks;
  const int64_t T = T1 - T0;
  if (T <= 0) return cudaSuccess;
  const int grid = (int)std::min<int64_t>(T, p.num_sms);
  const int exper = knob(KNOB_PASS_EXPER);   // timing experiments only (sbr_test_set_knob); 0 in production
  return launch_pdl(kern, dim3(grid), dim3(256), Cfg::SMEM, st, mapL, mapW, (int)p.r0, (int)p.M, NT, T0, T, p.b,
                    p.X, p.ldx, exper, p.off, own, p.nbo);
}

static int pass_variant() {   // SBR_PASS_CFG (tuning experiments only): 0 = C8/NS4, 1 = C4/NS5, 2 = C2/NS6, 3 = C12/NS3
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("SBR_PASS_CFG");
    v = e ? atoi(e) : 0;
    if (v < 0 || v > 3) v = 0;
  }
  return v;
}

cudaError_t launch_pass_tc(const PassLaunch& p, cudaStream_t st) {
  if (p.b <= 16) return launch_pass_t<16, 8, 4>(p, st);
  if (p.b <= 32) {
    switch (pass_variant()) {
      case 1: return launch_pass_t<32, 4, 5>(p, st);
      case 2: return launch_pass_t<32, 2, 6>(p, st);
      case 3: if (p.own_P <= 1) return launch_pass_t<32, 12, 3>(p, st);   // (dist: groups must tile nb)
              return launch_pass_t<32, 8, 4>(p, st);
      default: return launch_pass_t<32, 8, 4>(p, st);
    }
  }
  return launch_pass_t<64, 4, 3>(p, st);
}

int pass_bn(int b) { return b <= 16 ? 16 : b <= 32 ? 32 : 64; }

int pass_dist_align(int b) { return 128 * pass_group_cols(b); }

SBR_OP16_SETTER(pass)

}  // namespace sbr
