// k_pass_tf32.cu -- the per-panel pass X_t = OA W_t (step a4; Alg. 1 l.9) in the
// FP32-accurate 3xTF32 mode (reading C11) on tcgen05 tensor cores.
//
// OA is read in fp32 straight from the master A (tiles of the current block's first
// columns, which the panel chain rewrites, from the frozen strip copy), 4 bytes per stored
// lower element, each 128 x 128 lower tile ONCE (TMA, 128B swizzle, lines = tile columns)
// and used for both products of the symmetric pass (as k_pass_tc.cu):
//   X_J += L^T W_I : A = L^T is K-major in smem as loaded.  hi_a [hi_w | lo_w] with N = 2*32
//                    reads the RAW fp32 tile (the tensor core uses its top 19 bits, i.e.
//                    hi_a = trunc_tf32(a)); then converter warps overwrite the tile in place
//                    with lo_a = a - trunc_tf32(a) (exact) and lo_a hi_w (N = 32) follows.
//   X_I += L W_J   : A = L would be MN-major, which for 32-bit operands needs the 32-byte-atom
//                    swizzle (incompatible with the K-major view above), so the converter
//                    writes a row-major split copy of the tile into TMEM instead (thread =
//                    tile row = TMEM lane; hi = rna_tf32(a), lo = rna_tf32(a - hi)) and the
//                    MMAs take A from tensor memory: hi [hi_w | lo_w] + lo hi_w.
// W's split (rna hi, rna lo) is precomputed by split_tf32_w; each accumulator's two halves
// (a*hi_w, a*lo_w) are summed in the epilogue.  Dropped: lo_a lo_w (< 2^-20 |a w|) and, in
// X_J only, the tf32 truncation of lo_a (< 2^-20 |a|).  DESIGN.md reading R4.
// Diagonal tiles: the master's upper triangle is stale, so the converter zeroes it and halves
// the diagonal first (then L W + L^T W = OA_JJ W as with the fp16 shadow).
//
// One CTA per SM, 512 threads: warp 0 TMA producer, warp 1 MMA issuer, warp 2 TMEM allocator
// (all 512 columns: A copy hi/lo 256, row and column accumulators 2 x 64 each), warps 4-7 and
// 12-15 converter (two groups, half of the columns each), warps 8-11 epilogue (fp32 reductions
// into X).  2 stages of {L tile 64 KB, W_I
// 32 KB} + W_J 32 KB = 224 KB smem.  Work: tile columns J in order, rows I = J .. NT-1 (group
// = one tile column, W_J resident), a balanced contiguous range of tiles per CTA.
#include <cstdlib>
#include <cstring>

#include "kernels.h"
#include "tc.cuh"

namespace sbr {

using namespace tc;

namespace {
constexpr int P3_LT = 65536;                  // 128 x 128 fp32 tile: 4 boxes of 32 rows x 128 cols
constexpr int P3_WT = 32768;                  // 128 rows x [hi 32 | lo 32] fp32: 4 boxes of 32 x 64
constexpr int P3_STAGE = P3_LT + P3_WT;
constexpr int P3_NS = 2;
constexpr int P3_OFF_WJ = P3_NS * P3_STAGE;
constexpr int P3_OFF_BAR = P3_OFF_WJ + P3_WT;
constexpr int P3_NBAR = 5 * P3_NS + 2 + 4 + 4 + 2 + 1;
// TMEM columns: row-major A copy (hi, lo) for X_I, row / column accumulators (2 x 64 each)
constexpr uint32_t P3_AHI = 0, P3_ALO = 128, P3_RACC = 256, P3_CACC = 384;
constexpr int P3_SMEM = P3_OFF_BAR + P3_NBAR * 8 + 16 + 1024;
constexpr int P3_THREADS = 512;   // + converter warps 12-15 (two converter groups of 4 warps)
static_assert(P3_SMEM <= 232448, "3xTF32 pass smem");

// Tile ownership (sbr_reduce_dist, 1D block-cyclic): the tile grid starts at global column gr0
// (the block start, nb-aligned; OA begins `off` rows/columns into it), tile column J lies in the
// nb-block blk0 + J / gpb, owned by rank (block % P); P = 1: every tile.
struct PassOwnTf {
  int P = 1, rank = 0, gpb = 1;
  int64_t blk0 = 0, nbo = 1, gr0 = 0;
  SBR_DEV bool owned(int J) const { return P <= 1 || (int)((blk0 + J / gpb) % P) == rank; }
  SBR_DEV int64_t lcol(int64_t g) const {   // local column of global column g
    if (P <= 1) return g;
    const int64_t Jb = g / nbo;
    return (Jb / P) * nbo + (g - Jb * nbo);
  }
};

struct Walk1 {   // C = 1 tile walk: owned tile columns J in order, rows I = J .. NT-1
  int NT, I, J;
  int64_t left;
  bool first;   // first tile of a group (column) in this CTA's range
  PassOwnTf own;
  SBR_DEV void start(int NT_, int64_t t0, int64_t count, const PassOwnTf& o) {
    NT = NT_;
    own = o;
    left = count;
    first = true;
    I = J = 0;
    if (count <= 0) return;
    J = 0;
    for (;;) {
      if (own.owned(J)) {
        if (t0 < NT - J) break;
        t0 -= NT - J;
      }
      ++J;
    }
    I = J + (int)t0;
  }
  SBR_DEV bool valid() const { return left > 0; }
  SBR_DEV bool glast() const { return left == 1 || I + 1 == NT; }
  SBR_DEV void next() {
    --left;
    first = false;
    if (++I == NT) {
      do { ++J; } while (J < NT && !own.owned(J));
      I = J;
      first = true;
    }
  }
};
}  // namespace

SBR_DEV void fence_proxy_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

__global__ void __launch_bounds__(P3_THREADS, 1)
    pass_tf32_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapS,
                     const __grid_constant__ CUtensorMap mapW, int M, int off, int NT, int jstrip, int64_t T,
                     int b, float* X, int64_t ldx, int l2normal, PassOwnTf own) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint64_t* bars = (uint64_t*)(smem + P3_OFF_BAR);
  uint64_t* l_full = bars;                 // TMA landed (tile + W_I)
  uint64_t* l_empty = bars + P3_NS;        // lo MMAs done: stage free
  uint64_t* hi_done = bars + 2 * P3_NS;    // hi MMAs done: converter may overwrite
  uint64_t* lo_ready = bars + 3 * P3_NS;   // converter wrote lo
  uint64_t* diag_ready = bars + 4 * P3_NS; // converter fixed a diagonal tile (per stage)
  uint64_t* wj_full = bars + 5 * P3_NS;
  uint64_t* wj_empty = wj_full + 1;
  uint64_t* racc_full = wj_full + 2;       // [2]
  uint64_t* racc_empty = racc_full + 2;    // [2]
  uint64_t* cacc_full = racc_full + 4;     // [2]
  uint64_t* cacc_empty = cacc_full + 2;    // [2]
  uint64_t* ta_full = cacc_full + 4;       // converter wrote the TMEM A copy
  uint64_t* ta_empty = ta_full + 1;        // X_I MMAs done reading it
  uint32_t* tmem_slot = (uint32_t*)(bars + P3_NBAR);
  const int warp = warp_id(), lane = lane_id();
  pdl_trigger();
  const int64_t t_beg = (int64_t)blockIdx.x * T / gridDim.x;
  const int64_t t_end = (int64_t)(blockIdx.x + 1) * T / gridDim.x;
  if (threadIdx.x == 0) {
    for (int i = 0; i < P3_NS; ++i) {
      mbar_init(&l_full[i], 1); mbar_init(&l_empty[i], 1); mbar_init(&hi_done[i], 1);
      mbar_init(&lo_ready[i], 256); mbar_init(&diag_ready[i], 256);
    }
    mbar_init(wj_full, 1); mbar_init(wj_empty, 1);
    mbar_init(ta_full, 256); mbar_init(ta_empty, 1);
    for (int i = 0; i < 2; ++i) {
      mbar_init(&racc_full[i], 1); mbar_init(&racc_empty[i], 128);
      mbar_init(&cacc_full[i], 1); mbar_init(&cacc_empty[i], 128);
    }
    mbar_fence_init();
  }
  if (warp == 0 && lane == 0) { tma_prefetch(&mapA); tma_prefetch(&mapS); tma_prefetch(&mapW); }
  if (warp == 2) tmem_alloc(tmem_slot, 512);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();
  Walk1 w;

  if (warp == 0) {
    // ------------------------------------------------ TMA producer
    if (lane == 0) {
      // OA / strip tiles are read once per pass: evict_first (SBR_TF32_L2=normal: ablation)
      const uint64_t lpol = l2normal ? l2_policy_evict_normal() : l2_policy_evict_first();
      int st = 0; uint32_t ph = 0;
      uint32_t jph = 0;
      for (w.start(NT, t_beg, t_end - t_beg, own); w.valid(); w.next()) {
        if (w.first) {
          mbar_wait(wj_empty, jph ^ 1);
          jph ^= 1;
          mbar_expect_tx(wj_full, P3_WT);
          for (int rc = 0; rc < 4; ++rc)
            tma_load_2d(smem + P3_OFF_WJ + rc * 8192, &mapW, wj_full, w.J * 128 + rc * 32 - off, 0);
        }
        mbar_wait(&l_empty[st], ph ^ 1);
        mbar_expect_tx(&l_full[st], P3_STAGE);
        uint8_t* dst = smem + st * P3_STAGE;
        const bool strip = w.J < jstrip;
        // grid rows / columns from gr0; the strip and W are indexed from OA's origin (gr0 + off):
        // coordinates below 0 (the `off` rows / columns in front of OA) read as zeros (TMA OOB fill)
        const int lc = (int)own.lcol(own.gr0 + (int64_t)w.J * 128);
        for (int rc = 0; rc < 4; ++rc) {
          if (strip)
            tma_load_2d_hint(dst + rc * 16384, &mapS, &l_full[st], w.I * 128 + rc * 32 - off, w.J * 128 - off, lpol);
          else
            tma_load_2d_hint(dst + rc * 16384, &mapA, &l_full[st], (int)own.gr0 + w.I * 128 + rc * 32, lc, lpol);
        }
        for (int rc = 0; rc < 4; ++rc)
          tma_load_2d(dst + P3_LT + rc * 8192, &mapW, &l_full[st], w.I * 128 + rc * 32 - off, 0);
        if (++st == P3_NS) { st = 0; ph ^= 1; }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------ MMA issuer (one thread)
    if (lane == 0) {
      constexpr uint32_t id64 = idesc_make(128, 64, 2, 0, 0), id32 = idesc_make(128, 32, 2, 0, 0);
      const uint32_t s0 = smem_u32(smem), aWj = s0 + P3_OFF_WJ;
      int st = 0; uint32_t ph = 0;
      int rb = 0; uint32_t rph = 0;
      int cb = 0; uint32_t cph = 0;
      uint32_t jph = 0, taph = 0, dph = 0;
      for (w.start(NT, t_beg, t_end - t_beg, own); w.valid(); w.next()) {
        if (w.first) {
          mbar_wait(wj_full, jph);
          jph ^= 1;
        }
        // both accumulators are per tile (drained into fp32 registers by the epilogue: the tensor
        // core's truncating accumulation must not run over a whole tile column)
        mbar_wait(&racc_empty[rb], rph ^ 1);
        mbar_wait(&cacc_empty[cb], cph ^ 1);
        mbar_wait(&l_full[st], ph);
        if (w.I == w.J) {   // diagonal tiles only: per-stage phase bits of their own
          mbar_wait(&diag_ready[st], (dph >> st) & 1u);
          dph ^= 1u << st;
        }
        tc_fence_after();
        const uint32_t lt = s0 + st * P3_STAGE, wi = lt + P3_LT;
        const uint32_t d_row = tmem + P3_RACC + rb * 64, d_col = tmem + P3_CACC + cb * 64;
        // X_J += L^T [W_I,hi | W_I,lo]: A = raw fp32 tile (K-major; the tensor core reads trunc_tf32)
#pragma unroll
        for (int s = 0; s < 16; ++s)
          mma_tf32(d_col, sdesc_sw128(lt + (s >> 2) * 16384 + (s & 3) * 32, 16, 1024),
                   sdesc_sw128(wi + (s >> 2) * 8192 + (s & 3) * 32, 16, 1024), id64, s > 0 ? 1u : 0u);
        mma_commit(&hi_done[st]);
        // X_I += L [W_J,hi | W_J,lo] + L_lo W_J,hi: A = the converter's row-major hi / lo copy in TMEM
        mbar_wait(ta_full, taph);
        taph ^= 1;
        tc_fence_after();
#pragma unroll
        for (int s = 0; s < 16; ++s)
          mma_tf32_ts(d_row, tmem + P3_AHI + s * 8, sdesc_sw128(aWj + (s >> 2) * 8192 + (s & 3) * 32, 16, 1024),
                      id64, s > 0 ? 1u : 0u);
#pragma unroll
        for (int s = 0; s < 16; ++s)
          mma_tf32_ts(d_row, tmem + P3_ALO + s * 8, sdesc_sw128(aWj + (s >> 2) * 8192 + (s & 3) * 32, 16, 1024),
                      id32, 1u);
        mma_commit(ta_empty);
        mma_commit(&racc_full[rb]);
        // X_J += L_lo^T W_I,hi on the tile the converter rewrote in place
        mbar_wait(&lo_ready[st], ph);
        tc_fence_after();
#pragma unroll
        for (int s = 0; s < 16; ++s)
          mma_tf32(d_col, sdesc_sw128(lt + (s >> 2) * 16384 + (s & 3) * 32, 16, 1024),
                   sdesc_sw128(wi + (s >> 2) * 8192 + (s & 3) * 32, 16, 1024), id32, 1u);
        mma_commit(&l_empty[st]);
        mma_commit(&cacc_full[cb]);
        if (w.glast()) mma_commit(wj_empty);
        if (++cb == 2) { cb = 0; cph ^= 1; }
        if (++st == P3_NS) { st = 0; ph ^= 1; }
        if (++rb == 2) { rb = 0; rph ^= 1; }
      }
    }
  } else if ((warp >= 4 && warp < 8) || warp >= 12) {
    // ------------------------------------------------ converter: group cg (warps 4-7 / 12-15) takes
    // half of the columns of the TMEM copy and half of the in-place lo pass
    const int cgp = warp >= 12 ? 1 : 0;
    const int tid = threadIdx.x - (cgp ? 384 : 128);   // 0..127 within the group
    const int u = cgp * 128 + tid;                      // 0..255 over both groups
    const int q = warp & 3;                 // TMEM lane quarter = row box of the tile
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    int st = 0; uint32_t ph = 0;
    uint32_t tph = 0;
    for (w.start(NT, t_beg, t_end - t_beg, own); w.valid(); w.next()) {
      uint8_t* lt = smem + st * P3_STAGE;
      mbar_wait(&l_full[st], ph);
      if (w.I == w.J) {   // stale upper triangle -> 0, diagonal halved
        const int c = u >> 1;                 // column; rows of parity u & 1
        for (int r = u & 1; r <= c; r += 2) {
          const int rc = r >> 5, rr = r & 31;
          float* p = (float*)(lt + rc * 16384 + c * 128 + ((((rr >> 2) ^ (c & 7))) << 4) + (rr & 3) * 4);
          *p = (r == c) ? 0.5f * *p : 0.f;
        }
        fence_proxy_async_smem();
        __syncwarp();
        asm volatile("bar.sync 1, 256;" ::: "memory");   // all columns fixed before any row is read
        mbar_arrive(&diag_ready[st]);
      }
      // row-major split copy for X_I: thread = tile row 32q + lane, hi = rna_tf32(a), lo = rna_tf32(a - hi)
      mbar_wait(ta_empty, tph ^ 1);
      tph ^= 1;
      tc_fence_after();
      const uint8_t* rowbase = lt + q * 16384 + (lane & 3) * 4;
#pragma unroll 1
      for (int cc = 2 * cgp; cc < 2 * cgp + 2; ++cc) {
        float hi[32], lo[32];
#pragma unroll
        for (int j = 0; j < 32; ++j) {
          const int c = cc * 32 + j;
          const float a = *(const float*)(rowbase + c * 128 + ((((lane >> 2) ^ (c & 7))) << 4));
          hi[j] = tf32_rna(a);
          lo[j] = tf32_rna(a - hi[j]);
        }
        tmem_st32(tmem + P3_AHI + cc * 32 + lane_off, hi);
        tmem_st32(tmem + P3_ALO + cc * 32 + lane_off, lo);
      }
      tmem_wait_st();
      tc_fence_before();
      mbar_arrive(ta_full);
      // in place: lo = a - trunc_tf32(a) for X_J's correction (after its hi MMAs read the raw tile)
      mbar_wait(&hi_done[st], ph);
      float4* v = (float4*)lt;
#pragma unroll 8
      for (int i = u; i < P3_LT / 16; i += 256) {
        float4 x = v[i];
        x.x -= __uint_as_float(__float_as_uint(x.x) & 0xffffe000u);
        x.y -= __uint_as_float(__float_as_uint(x.y) & 0xffffe000u);
        x.z -= __uint_as_float(__float_as_uint(x.z) & 0xffffe000u);
        x.w -= __uint_as_float(__float_as_uint(x.w) & 0xffffe000u);
        v[i] = x;
      }
      fence_proxy_async_smem();
      mbar_arrive(&lo_ready[st]);
      if (++st == P3_NS) { st = 0; ph ^= 1; }
    }
  } else if (warp >= 8 && warp < 12) {
    // ------------------------------------------------ epilogue: TMEM -> fp32 reductions into X
    const int q = warp & 3;
    const int row_in_tile = q * 32 + lane;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    int rb = 0; uint32_t rph = 0;
    int cb = 0; uint32_t cph = 0;
    float creg[32];   // X_J of the current group, summed over its tiles in fp32 (round to nearest)
#pragma unroll
    for (int c = 0; c < 32; ++c) creg[c] = 0.f;
    for (w.start(NT, t_beg, t_end - t_beg, own); w.valid(); w.next()) {
      mbar_wait(&racc_full[rb], rph);
      tc_fence_after();
      {
        float v[32], u[32];
        tmem_ld32(tmem + P3_RACC + rb * 64 + lane_off, v);
        tmem_ld32(tmem + P3_RACC + rb * 64 + 32 + lane_off, u);
        tc_fence_before();
        mbar_arrive(&racc_empty[rb]);
        const int64_t row = (int64_t)w.I * 128 + row_in_tile - off;
        if (row >= 0 && row < M) {
#pragma unroll
          for (int c = 0; c < 32; ++c)
            if (c < b) atomicAdd(&X[row + (int64_t)c * ldx], v[c] + u[c]);
        }
      }
      if (++rb == 2) { rb = 0; rph ^= 1; }
      {
        mbar_wait(&cacc_full[cb], cph);
        tc_fence_after();
        float v[32], u[32];
        tmem_ld32(tmem + P3_CACC + cb * 64 + lane_off, v);
        tmem_ld32(tmem + P3_CACC + cb * 64 + 32 + lane_off, u);
        tc_fence_before();
        mbar_arrive(&cacc_empty[cb]);
#pragma unroll
        for (int c = 0; c < 32; ++c) creg[c] += v[c] + u[c];
        if (++cb == 2) { cb = 0; cph ^= 1; }
      }
      if (w.glast()) {
        const int64_t row = (int64_t)w.J * 128 + row_in_tile - off;
        if (row >= 0 && row < M) {
#pragma unroll
          for (int c = 0; c < 32; ++c)
            if (c < b) atomicAdd(&X[row + (int64_t)c * ldx], creg[c]);
        }
#pragma unroll
        for (int c = 0; c < 32; ++c) creg[c] = 0.f;
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    tc_fence_after();
    tmem_dealloc(tmem, 512);
  }
}

// ---------------------------------------------------------------- host
int64_t pass_tf32_tiles(int64_t M) {
  const int64_t NT = (M + 127) / 128;
  return NT * (NT + 1) / 2;
}

cudaError_t launch_pass_tf32(const PassTf32Launch& p, cudaStream_t st) {
  if (p.b < 1 || p.b > 32) return cudaErrorInvalidValue;
  auto kern = pass_tf32_kernel;
  {
    cudaError_t e = func_attr((const void*)kern, cudaFuncAttributeMaxDynamicSharedMemorySize, P3_SMEM);
    if (e != cudaSuccess) return e;
  }
  const int off = p.off;
  const int NT = (int)((p.M + off + 127) / 128);
  // tile columns J < jstrip read the frozen strip, which holds OA columns [0, 128 jstrip - off)
  const int jstrip = p.S ? (int)std::min<int64_t>((p.sw + off + 127) / 128, NT) : 0;
  PassOwnTf own;
  own.gr0 = p.r0 - off;
  if (p.own_P > 1) {
    if (p.nbo % 128 != 0 || own.gr0 % p.nbo != 0) return cudaErrorInvalidValue;
    own.P = p.own_P;
    own.rank = p.own_rank;
    own.nbo = p.nbo;
    own.gpb = (int)(p.nbo / 128);
    own.blk0 = own.gr0 / p.nbo;
  }
  CUtensorMap mapA, mapS, mapW;
  cudaError_t e = make_tmap_2d(&mapA, p.A, false, p.n, p.ncols > 0 ? p.ncols : p.n, p.lda, 32, 128);
  if (e != cudaSuccess) return e;
  if (jstrip > 0) {
    e = make_tmap_2d(&mapS, p.S, false, p.M, std::min<int64_t>((int64_t)jstrip * 128 - off, p.M), p.lds, 32, 128);
    if (e != cudaSuccess) return e;
  } else {
    mapS = mapA;
  }
  e = make_tmap_2d(&mapW, p.WS, false, p.M, 64, p.ldws, 32, 64);
  if (e != cudaSuccess) return e;
  int64_t T = 0;
  for (int J = 0; J < NT; ++J)
    if (own.P <= 1 || (int)((own.blk0 + J / own.gpb) % own.P) == own.rank) T += NT - J;
  if (T <= 0) return cudaSuccess;
  const int grid = (int)std::min<int64_t>(T, p.num_sms);
  static const int l2normal = (getenv("SBR_TF32_L2") && !strcmp(getenv("SBR_TF32_L2"), "normal")) ? 1 : 0;
  return launch_pdl(kern, dim3(grid), dim3(P3_THREADS), P3_SMEM, st, mapA, mapS, mapW, (int)p.M, off, NT, jstrip, T,
                    p.b, p.X, p.ldx, l2normal, own);
}

// ---------------------------------------------------------------- operand splits (3xTF32)
__global__ void split_tf32_rm_kernel(int64_t rows, int cols, const float* __restrict__ src, int64_t lds,
                                     float* __restrict__ dst, int64_t ldd, int64_t lo_off) {
  // thread per (row, col); consecutive threads = consecutive columns of one row (coalesced writes)
  const int64_t cpad = (cols + 31) / 32 * 32;
  const int64_t total = rows * cpad;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / cpad, c = i % cpad;
    float hi = 0.f, lo = 0.f;
    if (c < cols) {
      const float a = src[r + c * lds];
      hi = tf32_rna(a);
      lo = tf32_rna(a - hi);
    }
    dst[r * ldd + c] = hi;
    if (c < cols) dst[r * ldd + lo_off + c] = lo;
  }
}

cudaError_t split_tf32_rm(int64_t rows, int cols, const float* src, int64_t lds, float* dst, int64_t ldd,
                          int64_t lo_off, cudaStream_t st) {
  if (rows <= 0 || cols <= 0) return cudaSuccess;
  const int64_t total = rows * ((cols + 31) / 32 * 32);
  const int grid = (int)std::min<int64_t>((total + 255) / 256, 148 * 16);
  split_tf32_rm_kernel<<<grid, 256, 0, st>>>(rows, cols, src, lds, dst, ldd, lo_off);
  return cudaGetLastError();
}

__global__ void splitsum_kernel(int64_t rows, int cols, const float* __restrict__ src, int64_t lds, int64_t lo_off,
                                float* __restrict__ dst, int64_t ldd) {
  const int64_t total = rows * cols;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i % rows, c = i / rows;
    dst[r + c * ldd] = src[r * lds + c] + src[r * lds + lo_off + c];
  }
}

cudaError_t splitsum_rm_to_cm(int64_t rows, int cols, const float* src, int64_t lds, int64_t lo_off, float* dst,
                              int64_t ldd, cudaStream_t st) {
  if (rows <= 0 || cols <= 0) return cudaSuccess;
  const int grid = (int)std::min<int64_t>((rows * cols + 255) / 256, 148 * 8);
  splitsum_kernel<<<grid, 256, 0, st>>>(rows, cols, src, lds, lo_off, dst, ldd);
  return cudaGetLastError();
}

__global__ void split_tf32_cm_kernel(int64_t rows, int cols, const float* __restrict__ src, int64_t lds,
                                     bool unit_y, float* __restrict__ dst, int64_t ldd, int64_t lo_off) {
  const int64_t rpad = (rows + 31) / 32 * 32;
  for (int64_t c = blockIdx.y; c < cols; c += gridDim.y) {
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < rpad; r += (int64_t)gridDim.x * blockDim.x) {
      float a = 0.f;
      if (r < rows) a = unit_y ? (r < c ? 0.f : r == c ? 1.f : src[r + c * lds]) : src[r + c * lds];
      const float hi = tf32_rna(a);
      dst[c * ldd + r] = hi;
      if (r < rows) dst[c * ldd + lo_off + r] = tf32_rna(a - hi);
    }
  }
}

cudaError_t split_tf32_cm(int64_t rows, int cols, const float* src, int64_t lds, bool unit_y, float* dst,
                          int64_t ldd, int64_t lo_off, cudaStream_t st) {
  if (rows <= 0 || cols <= 0) return cudaSuccess;
  const int gx = (int)std::min<int64_t>((rows + 255) / 256, 64);
  const int gy = std::min(cols, 2048);
  split_tf32_cm_kernel<<<dim3(gx, gy), 256, 0, st>>>(rows, cols, src, lds, unit_y, dst, ldd, lo_off);
  return cudaGetLastError();
}

__global__ void set_identity_kernel(int64_t n, float* Q, int64_t ldq) {
  for (int64_t c = blockIdx.y; c < n; c += gridDim.y)
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x)
      Q[r + c * ldq] = r == c ? 1.f : 0.f;
}

cudaError_t set_identity(int64_t n, float* Q, int64_t ldq, cudaStream_t st) {
  if (n <= 0) return cudaSuccess;
  set_identity_kernel<<<dim3((unsigned)std::min<int64_t>((n + 255) / 256, 64), (unsigned)std::min<int64_t>(n, 4096)),
                        256, 0, st>>>(n, Q, ldq);
  return cudaGetLastError();
}

__global__ void split_tf32_w_kernel(int64_t rows, int b, int bn, const float* __restrict__ W, int64_t ldw,
                                    float* __restrict__ dst, int64_t ldd) {
  pdl_trigger();   // 3xTF32 / SIMT chain: launched with PDL (launch_pdl), waits before any access
  pdl_wait();
  const int64_t total = rows * bn;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i % rows, c = i / rows;
    float hi = 0.f, lo = 0.f;
    if (c < b) {
      const float a = W[r + c * ldw];
      hi = tf32_rna(a);
      lo = tf32_rna(a - hi);
    }
    dst[r + c * ldd] = hi;
    dst[r + (c + bn) * ldd] = lo;
  }
}

cudaError_t split_tf32_w(int64_t rows, int b, int bn, const float* W, int64_t ldw, float* dst, int64_t ldd,
                         cudaStream_t st) {
  if (rows <= 0) return cudaSuccess;
  const int64_t total = rows * bn;
  const int grid = (int)std::min<int64_t>((total + 255) / 256, 148 * 8);
  return launch_pdl(split_tf32_w_kernel, dim3(grid), dim3(256), 0, st, rows, b, bn, W, ldw, dst, ldd);
}

}  // namespace sbr
