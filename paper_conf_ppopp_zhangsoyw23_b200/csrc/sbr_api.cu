// sbr_api.cu -- C ABI and host driver of libsbr (see include/sbr.h).
//
// Host loop = Algorithm 1 of the paper in the reading of DESIGN.md:
//   for each nb-block (origin c0, OA = A[c0+b:, c0+b:] frozen at block start):
//     for each b-panel t:
//       a5 (t>=1)  lazy panel update  GA = OA(:,c) - [X | Y] [Y_c^T ; W^T R]
//       a1/a2      TSQR + reconstruction -> Y_t, W_t^0 = Y_t T_t, R    (k_panel.cu)
//       a3 (t>=1)  W merge  W_t = W_t^0 - W (Y^T W_t^0)
//       a4         pass     X_t = OA W_t ;  W^T X column block
//     a6          Z = X - 1/2 Y (W^T X);  A_trail -= Y Z^T + Z Y^T  (lower)   (Eq. 1-3)
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/sbr.h"
#include "common.cuh"
#include "common.cuh"
#include "kernels.h"
#include "comm.h"
#include "nccl_rt.h"

using namespace sbr;

namespace {

std::mutex g_err_mu;
std::string g_last_err = "";

void set_err(const char* what, cudaError_t e) {
  std::lock_guard<std::mutex> lk(g_err_mu);
  g_last_err = std::string(what) + ": " + cudaGetErrorName(e) + " (" + cudaGetErrorString(e) + ")";
}

struct Stat {
  int64_t launches = 0;
  double ms = 0, bytes = 0, flops = 0;
};

struct Pending {
  cudaEvent_t e0, e1;
  int kid;
  double bytes, flops;
};

}  // namespace

struct sbr_ctx {
  int device = 0;
  cudaStream_t stream = nullptr;
  int nsm = 0;
  // workspace
  void* ws = nullptr;
  size_t ws_bytes = 0;
  int64_t ws_n = -1;
  int ws_b = -1, ws_nb = -1, ws_mode = -1;
  int64_t ws_shcols = -1;
  float* ABd = nullptr;     // multi-GPU: (b+1) x n band assembled over the ranks
  float *Yb = nullptr, *Xb = nullptr, *Zb = nullptr, *Wws = nullptr, *Strip = nullptr, *WtX = nullptr,
        *Pb = nullptr, *Gb = nullptr;
  float *pv = nullptr, *ptau = nullptr, *pr = nullptr, *pq = nullptr, *pmisc = nullptr;
  unsigned* flag = nullptr;
  __half *Sh = nullptr, *Yh = nullptr, *Zh = nullptr, *Wh = nullptr, *WtXh = nullptr, *Xh = nullptr, *Wrh = nullptr,
         *Bl = nullptr, *Gh = nullptr;
  float* Hb = nullptr;
  // 3xTF32 tensor-core path: [hi | lo] splits (row-major, lo at column tlo) of Y, Z, W^T X, and W_t
  float *YS = nullptr, *ZS = nullptr, *GS = nullptr, *WS = nullptr;
  int64_t tlo = 0, ldts = 0, ldws = 0;
  float* GH = nullptr;     // per-block G_t / H_t (k x b, ld nb, panel t at offset t*nb*b), zeroed per block
  __half* Ph = nullptr;    // fp16 P^T (b x k, row-major) of the lazy update
  void* chol_ws = nullptr;  // CholeskyQR panel workspace (Gram sets, barrier, LU), zeroed at allocation
  void* fused_ws = nullptr; // fused chain kernel workspace (two launch parities), zeroed at allocation
  unsigned fused_launches = 0;
  bool fused = false;       // SBR_FUSED=1: the fused per-panel chain kernel (k_chain_fused.cu)
  int* pfail = nullptr;
  unsigned chol_launches = 0;
  int panel_mode = 0;      // 0: CholeskyQR3 + TSQR fallback, 1: TSQR only (SBR_PANEL=tsqr)
  int64_t ldwh = 0, ldsh = 0, ldk = 0, ldbl = 0;
  int panel_ctas = 0;
  // host-buffer (e2e) device copies
  void* e2e = nullptr;
  size_t e2e_bytes = 0;
  // sbr_form_q split operands (grown on demand, kept for the next call)
  void* fq = nullptr;
  size_t fq_bytes = 0;
  // stage two (k_stage2.cu): working band, progress counters, d/e/e^2, band of sbr_eigenvalues
  void* s2 = nullptr;
  size_t s2_bytes = 0;
  // stats
  bool timing = false;
  std::vector<cudaEvent_t> ev_pool;
  std::vector<Pending> pending;
  Stat stats[SBR_K_COUNT];
  int64_t launches = 0;
  // multi-GPU (sbr_create_dist): this process's rank in an NCCL communicator of nranks
  int rank = 0, nranks = 1;
  sbr::Comm* comm = nullptr;   // NCCL or in-process ("local") communicator (comm.h)
  bool tf32_tc = true;       // SBR_TF32_TC=0: 3xTF32 mode on the SIMT fp32 kernels (ablation)
  // latched device-detected errors (§8(b)): each sbr_reduce copies its status words (flag[0..3])
  // into a pinned slot and records an event; sbr_sync and the next calls report them
  static constexpr int kSlots = 4;
  unsigned* pinned = nullptr;          // kSlots x 4 words
  cudaEvent_t slot_ev[kSlots] = {};
  bool slot_busy[kSlots] = {};
  int slot_next = 0;
  // sbr_test_panel_trace: per-panel CholeskyQR phase stamps of the next sbr_reduce (16 int64 per panel)
  int64_t* ptrace = nullptr;
  int ptrace_cap = 0, ptrace_used = 0;
};

namespace {

cudaEvent_t get_event(sbr_ctx* h) {
  if (!h->ev_pool.empty()) {
    cudaEvent_t e = h->ev_pool.back();
    h->ev_pool.pop_back();
    return e;
  }
  cudaEvent_t e;
  cudaEventCreate(&e);
  return e;
}

struct Scope {  // per-kernel-class timing scope (CUDA events on the handle's stream)
  sbr_ctx* h;
  int kid;
  double bytes, flops;
  cudaEvent_t e0 = nullptr;
  Scope(sbr_ctx* h_, int kid_, double bytes_, double flops_) : h(h_), kid(kid_), bytes(bytes_), flops(flops_) {
    if (h->timing) {
      e0 = get_event(h);
      cudaEventRecord(e0, h->stream);
    }
  }
  ~Scope() {
    if (h->timing) {
      cudaEvent_t e1 = get_event(h);
      cudaEventRecord(e1, h->stream);
      h->pending.push_back({e0, e1, kid, bytes, flops});
    }
  }
};

void drain_stats(sbr_ctx* h) {
  if (h->pending.empty()) return;
  cudaStreamSynchronize(h->stream);
  for (auto& p : h->pending) {
    float ms = 0.f;
    cudaEventElapsedTime(&ms, p.e0, p.e1);
    Stat& s = h->stats[p.kid];
    s.launches += 1;
    s.ms += ms;
    s.bytes += p.bytes;
    s.flops += p.flops;
    h->ev_pool.push_back(p.e0);
    h->ev_pool.push_back(p.e1);
  }
  h->pending.clear();
}

// status words of a finished reduction -> sbr.h code (0 if none)
int status_of(const unsigned* w) {
  if (w[0] || w[2]) return SBR_ERR_NONFINITE;   // non-finite input / fp16 range exceeded
  if (w[1]) return SBR_ERR_UNSUPPORTED;          // declined CholeskyQR panel beyond the TSQR capacity
  return SBR_OK;
}

// Report latched errors of finished reductions (wait = block until all slots complete).
int poll_latched(sbr_ctx* h, bool wait) {
  int rc = SBR_OK;
  for (int i = 0; i < sbr_ctx::kSlots; ++i) {
    if (!h->slot_busy[i]) continue;
    const cudaError_t q = wait ? cudaEventSynchronize(h->slot_ev[i]) : cudaEventQuery(h->slot_ev[i]);
    if (q == cudaErrorNotReady) {
      cudaGetLastError();
      continue;
    }
    h->slot_busy[i] = false;
    const int r = status_of(h->pinned + 4 * i);
    if (r != SBR_OK && rc == SBR_OK) {
      rc = r;
      if (r == SBR_ERR_UNSUPPORTED) {
        std::lock_guard<std::mutex> lk(g_err_mu);
        g_last_err = "a panel taller than the TSQR capacity was rank deficient for CholeskyQR";
      }
    }
  }
  return rc;
}

// Enqueue the copy of this reduction's status words into a free pinned slot.
int latch_status(sbr_ctx* h, cudaStream_t st) {
  if (!h->pinned) {
    if (cudaHostAlloc((void**)&h->pinned, sizeof(unsigned) * 4 * sbr_ctx::kSlots, cudaHostAllocDefault) !=
        cudaSuccess) {
      cudaGetLastError();
      return SBR_ERR_NOMEM;
    }
    for (int i = 0; i < sbr_ctx::kSlots; ++i) cudaEventCreateWithFlags(&h->slot_ev[i], cudaEventDisableTiming);
  }
  const int i = h->slot_next;
  h->slot_next = (i + 1) % sbr_ctx::kSlots;
  if (h->slot_busy[i]) {   // more reductions in flight than slots: the oldest must finish first
    const int r = poll_latched(h, true);
    if (r != SBR_OK) return r;
  }
  cudaError_t e = cudaMemcpyAsync(h->pinned + 4 * i, h->flag, sizeof(unsigned) * 4, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaEventRecord(h->slot_ev[i], st);
  if (e != cudaSuccess) {
    set_err("latch status", e);
    return SBR_ERR_CUDA;
  }
  h->slot_busy[i] = true;
  return SBR_OK;
}

#define SBR_NC(expr, what)                                             \
  do {                                                                 \
    const int _r = (expr);                                             \
    if (_r != 0) {                                                     \
      std::lock_guard<std::mutex> lk(g_err_mu);                        \
      g_last_err = std::string(what) + ": " + nccl::error_string(_r);  \
      return SBR_ERR_NCCL;                                             \
    }                                                                  \
  } while (0)

#define SBR_CM(expr, what)                                                  \
  do {                                                                      \
    if ((expr) != 0) {                                                      \
      std::lock_guard<std::mutex> lk(g_err_mu);                             \
      g_last_err = std::string(what) + ": " + h->comm->err();               \
      return SBR_ERR_NCCL;                                                  \
    }                                                                       \
  } while (0)

#define SBR_CK(expr, what)                 \
  do {                                     \
    cudaError_t _e = (expr);               \
    if (_e != cudaSuccess) {               \
      set_err(what, _e);                   \
      return SBR_ERR_CUDA;                 \
    }                                      \
  } while (0)

size_t align_up(size_t x) { return (x + 255) & ~size_t(255); }

// columns of the nb-blocks J with J % P == rank (1D block-cyclic, sbr_reduce_dist)
int64_t local_cols(int64_t n, int nb, int P, int rank) {
  int64_t c = 0;
  for (int64_t c0 = (int64_t)rank * nb; c0 < n; c0 += (int64_t)P * nb) c += std::min<int64_t>(nb, n - c0);
  return c;
}

int ensure_ws(sbr_ctx* h, int64_t n, int b, int nb, int mode, size_t* bytes_out, int64_t shadow_cols = -1) {
  if (shadow_cols < 0) shadow_cols = n;
  const int64_t M = n - b;
  const PanelWs pw = panel_ws_sizes(M, b);
  size_t off = 0;
  auto take = [&](size_t floats) {
    size_t o = off;
    off += align_up(floats * sizeof(float));
    return o;
  };
  const int64_t strip_cols = (nb + 127) / 128 * 128;   // the 3xTF32 pass reads whole 128-column tiles
  const size_t oY = take((size_t)n * nb), oX = take((size_t)n * nb), oZ = take((size_t)n * nb),
               oW = take((size_t)n * nb), oS = take((size_t)n * strip_cols), oWtX = take((size_t)nb * nb),
               oP = take((size_t)nb * 64), oG = take((size_t)nb * 64), oPv = take(pw.v), oPt = take(pw.tau),
               oPr = take(pw.r), oPq = take(pw.q), oPm = take(pw.misc), oF = take(64);
  // fp16 operands of the tensor-core path (sizes in floats = halves / 2)
  // W copies: room for up to 128 zero rows in front (the multi-GPU pass's 128-aligned tile grid)
  const int64_t ldwh = (M + 128 + 7) / 8 * 8;   // TMA strides must be multiples of 16 bytes
  // fp16 shadow: ld a multiple of 128 and a row offset `shoff` chosen so that every block's OA
  // origin (row/col c0 + b, c0 = J*nb) starts on a 256-byte boundary -- the pass streams
  // 128x128 tiles of it and unaligned tiles drag in neighbouring lines (L2 256 B promotion).
  const int64_t shoff = (nb % 128 == 0 && (128 - b % 128) % 8 == 0) ? (128 - b % 128) % 128 : 0;
  const int64_t ldsh = (n + shoff + 127) / 128 * 128;
  const int64_t ldk = (nb + 7) / 8 * 8;
  const size_t oSh = take(((size_t)ldsh * shadow_cols + shoff) / 2 + 128), oYh = take((size_t)n * ldk / 2 + 8),
               oZh = take((size_t)n * ldk / 2 + 8), oWh = take((size_t)ldwh * 64 / 2 + 8),
               oWtXh = take((size_t)nb * ldk / 2 + 8), oXh = take((size_t)n * ldk / 2 + 8),
               oWrh = take((size_t)n * ldk / 2 + 8), oBl = take((size_t)64 * (2 * ldk + 128) / 2 + 8),
               oGh = take((size_t)ldk * 64 / 2 + 8), oHb = take((size_t)nb * 64), oGram = take(panel_chol_ws_bytes() / sizeof(float) + 64),
               oGH = take((size_t)2 * nb * nb), oPh = take((size_t)64 * ldk / 2 + 8),
               oFz = take(chain_fused_ws_bytes() / sizeof(float) + 64), oABd = take((size_t)(b + 1) * n + 64);
  const int64_t tlo = (nb + 31) / 32 * 32, ldts = 2 * tlo, ldws = (M + 3) / 4 * 4;
  size_t oYS = 0, oZS = 0, oGS = 0, oWS = 0;
  if (mode == SBR_3XTF32) {
    oYS = take((size_t)n * ldts);
    oZS = take((size_t)n * ldts);
    oGS = take((size_t)nb * ldts);
    oWS = take((size_t)ldws * 64);
  }
  if (bytes_out) *bytes_out = off;
  if (!h) return SBR_OK;
  if (h->ws && h->ws_bytes >= off && h->ws_n == n && h->ws_b == b && h->ws_nb == nb && h->ws_mode == mode &&
      h->ws_shcols == shadow_cols)
    return SBR_OK;
  if (h->ws) {
    cudaFree(h->ws);
    h->ws = nullptr;
    h->ws_bytes = 0;
  }
  if (cudaMalloc(&h->ws, off) != cudaSuccess) {
    cudaGetLastError();
    return SBR_ERR_NOMEM;
  }
  h->ws_bytes = off;
  h->ws_n = n;
  h->ws_b = b;
  h->ws_nb = nb;
  h->ws_mode = mode;
  h->ws_shcols = shadow_cols;
  char* base = (char*)h->ws;
  h->ABd = (float*)(base + oABd);
  h->Yb = (float*)(base + oY);
  h->Xb = (float*)(base + oX);
  h->Zb = (float*)(base + oZ);
  h->Wws = (float*)(base + oW);
  h->Strip = (float*)(base + oS);
  h->WtX = (float*)(base + oWtX);
  h->Pb = (float*)(base + oP);
  h->Gb = (float*)(base + oG);
  h->pv = (float*)(base + oPv);
  h->ptau = (float*)(base + oPt);
  h->pr = (float*)(base + oPr);
  h->pq = (float*)(base + oPq);
  h->pmisc = (float*)(base + oPm);
  h->flag = (unsigned*)(base + oF);
  h->Sh = (__half*)(base + oSh) + shoff;
  h->Yh = (__half*)(base + oYh);
  h->Zh = (__half*)(base + oZh);
  h->Wh = (__half*)(base + oWh);
  h->WtXh = (__half*)(base + oWtXh);
  h->Xh = (__half*)(base + oXh);
  h->Wrh = (__half*)(base + oWrh);
  h->Bl = (__half*)(base + oBl);
  h->Gh = (__half*)(base + oGh);
  h->Hb = (float*)(base + oHb);
  h->chol_ws = base + oGram;
  h->GH = (float*)(base + oGH);
  h->Ph = (__half*)(base + oPh);
  h->tlo = tlo;
  h->ldts = ldts;
  h->ldws = ldws;
  h->YS = mode == SBR_3XTF32 ? (float*)(base + oYS) : nullptr;
  h->ZS = mode == SBR_3XTF32 ? (float*)(base + oZS) : nullptr;
  h->GS = mode == SBR_3XTF32 ? (float*)(base + oGS) : nullptr;
  h->WS = mode == SBR_3XTF32 ? (float*)(base + oWS) : nullptr;
  h->pfail = panel_chol_fail(h->chol_ws);
  if (cudaMemset(h->chol_ws, 0, panel_chol_ws_bytes()) != cudaSuccess) return SBR_ERR_CUDA;
  h->fused_ws = base + oFz;
  h->fused_launches = 0;
  if (cudaMemset(h->fused_ws, 0, chain_fused_ws_bytes()) != cudaSuccess) return SBR_ERR_CUDA;
  h->ldbl = 2 * ldk + 128;
  h->ldwh = ldwh;
  h->ldsh = ldsh;
  h->ldk = ldk;
  h->panel_ctas = panel_max_ctas(b);
  return SBR_OK;
}

int validate(sbr_ctx* h, int mode, int64_t n, int b, int nb, const float* A, int64_t lda, const float* AB,
             int64_t ldab, const float* W, int64_t ldw) {
  if (!h) return -1;
  if (mode != SBR_FP16_FP32ACC && mode != SBR_3XTF32 && mode != SBR_BF16_FP32ACC) return -2;
  if (n < 1) return -3;
  if (b < 1 || b > 64) return -4;
  if (nb < b || nb % b != 0 || nb > 4096) return -5;
  if (!A) return -6;
  if (lda < std::max<int64_t>(1, n)) return -7;
  if (!AB) return -8;
  if (ldab < b + 1) return -9;
  if (W && ldw < n) return -11;
  return SBR_OK;
}

bool panel_mode_default(const sbr_ctx* h) { return h->panel_mode == 0; }

// Algorithm 1 on device buffers (arguments already validated).
int reduce_device(sbr_ctx* h, int mode, int64_t n, int b, int nb, float* A, int64_t lda, float* AB, int64_t ldab,
                  float* W, int64_t ldw) {
  cudaStream_t st = h->stream;
  // sbr_reduce_dist (north star): 1D block-cyclic columns -- rank r holds the
  // columns of the nb-blocks J with J % P == r (fp32 master A and fp16 shadow), local column
  // (J / P) nb + (g - J nb).  The owner of block J factors all of its panels (the chain needs
  // only its own columns) and broadcasts W_t (fp16) per panel; every rank streams the pass tiles
  // of ITS columns and the partial X_t are summed by an all-reduce; per block the owner
  // broadcasts Y (fp16) and W^T X, and every rank applies the trailing SYR2K to its own
  // columns.  The band is assembled over the ranks at the end (rank 0 returns it).
  const bool dist = h->comm != nullptr && h->nranks > 1;
  const int P = dist ? h->nranks : 1, rank = dist ? h->rank : 0;
  const bool lead = rank == 0;   // returns the band
  ColMap cm;
  cm.P = P;
  cm.rank = rank;
  cm.nbo = nb;
  const int64_t ncols_loc = dist ? local_cols(n, nb, P, rank) : n;
  auto owner = [&](int64_t c0) { return (int)((c0 / nb) % P); };
  auto blk_ptr = [&](float* base, int64_t ld, int64_t c0) -> float* {   // global column indexing inside block c0 / nb
    if (!dist || !base) return base;
    const int64_t J = c0 / nb;
    return base + ((J / P) * nb - J * nb) * ld;
  };
  {   // errors latched by earlier reductions on this handle are returned by the next call (§8(b))
    const int lr = poll_latched(h, false);
    if (lr != SBR_OK) return lr;
  }
  if (n <= b + 1 && !dist) {
    Scope sc(h, SBR_K_OTHER, 0, 0);
    SBR_CK(extract_band(n, b, A, lda, AB, ldab, nullptr, nullptr, st), "extract_band");
    h->launches++;
    return SBR_OK;
  }
  int rc = ensure_ws(h, n, b, nb, mode, nullptr, ncols_loc);
  if (rc != SBR_OK) return rc;
  // status words flag[0..3] (input non-finite, declined tall panel, non-finite band), then the
  // a0 scan: finiteness + ||A||_F -> the power-of-two scale 2^k (kexp, device)
  unsigned* flag = h->flag;
  double* scan = reinterpret_cast<double*>(h->flag + 8);
  int* kexp = reinterpret_cast<int*>(h->flag + 12);
  SBR_CK(cudaMemsetAsync(flag, 0, sizeof(unsigned) * 4, st), "zero status");
  {
    Scope sc(h, SBR_K_OTHER, 2.0 * n * ncols_loc, 2.0 * n * ncols_loc);
    SBR_CK(prep_scan(n, ncols_loc, A, lda, cm, scan, st), "prep_scan");
    if (dist) SBR_CM(h->comm->all_reduce_sum_f64(scan, 2, st), "all-reduce ||A||_F");
    SBR_CK(choose_scale(scan, flag, kexp, st), "choose_scale");
    h->launches += (ncols_loc + 65534) / 65535 + 1;
  }
  if (n <= b + 1) goto band_out;
  {
  const int64_t ncols = n - b;  // reflector columns 0 .. n-b-1
  const int64_t ldn = n;        // ld of the block buffers
  // the TMA-fed tensor-core kernels need 16-byte aligned tile origins (OA origin r0 = c0 + b):
  // FP16 operands need b, nb multiples of 8, fp32 (3xTF32) multiples of 4; other (b, nb) run on
  // the fp32 SIMT kernels (more accurate than either mode's operands)
  // tcgen05 kind::f16 path; SBR_BF16_FP32ACC is the same path with bfloat16 operands (f4 ablation)
  const bool tc16 = (mode == SBR_FP16_FP32ACC || mode == SBR_BF16_FP32ACC) && b % 8 == 0 && nb % 8 == 0;
  if (tc16) SBR_CK(set_op16_all(mode == SBR_BF16_FP32ACC, st), "operand format");
  // 3xTF32 on tcgen05 kind::tf32 (pass + Z + SYR2K); the SIMT fp32 kernels remain for A that
  // TMA cannot address (lda % 4 != 0) and for the SBR_TF32_TC=0 ablation
  const bool tc32 = mode == SBR_3XTF32 && h->tf32_tc && lda % 4 == 0 && ((uintptr_t)A & 15) == 0 && b % 4 == 0 &&
                    nb % 4 == 0;
  if (dist && !tc16 && !tc32) {   // checked by sbr_reduce_dist (the SIMT fp32 path is single-GPU)
    std::lock_guard<std::mutex> lk(g_err_mu);
    g_last_err = "sbr_reduce_dist: the tensor-core paths only (b, nb multiples of 8 / 4, A 16-byte aligned)";
    return SBR_ERR_UNSUPPORTED;
  }
  if (tc16) {  // a0: fp16 shadow of OA_0 (strict lower, half diagonal, zero upper) -- this rank's columns
    Scope sc(h, SBR_K_OTHER, 6.0 * n * ncols_loc, 0);
    SBR_CK(shadow_init(n, A, lda, h->Sh, h->ldsh, kexp, st, ncols_loc, cm), "shadow_init");
    h->launches += (ncols_loc + 65534) / 65535;
  }
  if (!tc16) {  // a0 in 3xTF32 mode: the master scaled in place (FP16: inside shadow_init)
    Scope sc(h, SBR_K_OTHER, 8.0 * n * ncols_loc / 2, 0);
    SBR_CK(scale_lower(n, ncols_loc, A, lda, cm, kexp, st), "scale_lower");
    h->launches += (ncols_loc + 65534) / 65535;
  }
  if (tc16) {  // fp16 W copies: pad columns (b < BN) and the pad rows in front must read as zero in the pass
    SBR_CK(cudaMemsetAsync(h->Wh, 0, sizeof(__half) * h->ldwh * 64, st), "zero Wh");
  }
  // multi-GPU pass grid: 128-aligned tile origin c0 (nb % 1024 == 0), OA rows start `off` = b rows
  // into it; the W copies the pass reads carry `off` zero rows in front (the chain writes Whc)
  const int off = dist ? b : 0;
  __half* const Whc = h->Wh + off;
  for (int64_t c0 = 0; c0 < ncols; c0 += nb) {
    const int64_t r0 = c0 + b, M = n - r0;
    const int kJ = (int)std::min<int64_t>(nb, ncols - c0);
    const int p = (kJ + b - 1) / b;
    const int own = owner(c0);
    const bool leadJ = own == rank;               // this rank factors block J's panels
    float* const AJ = blk_ptr(A, lda, c0);        // global column indexing inside block J (its owner only)
    float* Wb = W ? blk_ptr(W, ldw, c0) + r0 + c0 * ldw : h->Wws;
    const int64_t ldwb = W ? ldw : ldn;
    float* OA = AJ + r0 + r0 * lda;
    const int sw = std::min<int64_t>((int64_t)(p - 1) * b, M);  // OA columns rewritten during the block
    if (sw > 0 && !tc16 && leadJ) {  // tc32: whole 128-column tiles of the (offset) pass grid
      const int64_t swc = tc32 ? std::min<int64_t>((sw + off + 127) / 128 * 128 - off, M) : sw;
      Scope sc(h, SBR_K_OTHER, 8.0 * M * swc, 0);
      SBR_CK(cudaMemcpy2DAsync(h->Strip, ldn * sizeof(float), OA, lda * sizeof(float), M * sizeof(float), swc,
                               cudaMemcpyDeviceToDevice, st),
             "strip copy");
    }
    if (tc16) {  // block start: X (accumulated by the passes), W^T X (diagonal blocks accumulated), G/H
      Scope sc(h, SBR_K_OTHER, 4.0 * M * p * b + 4.0 * nb * nb * 3, 0);
      SBR_CK(zero_matrix(M, (int64_t)p * b, h->Xb, M, st), "zero X");
      SBR_CK(cudaMemsetAsync(h->WtX, 0, sizeof(float) * nb * nb, st), "zero WtX");
      SBR_CK(cudaMemsetAsync(h->GH, 0, sizeof(float) * 2 * nb * nb, st), "zero G/H");
    }
    // fused FP16 chain (k_chain_fused.cu): one cooperative launch per panel + the pass
    const bool fused = tc16 && mode == SBR_FP16_FP32ACC && h->fused && panel_mode_default(h) && nb <= 1024 && chain_fused_supported(b, M, h->nsm);
    // ---- a4 for panel t on every rank: W_t from the owner (dist), the pass over this rank's
    //      tiles (the 128-aligned grid of its column blocks when distributed), X_t summed
    auto pass_t = [&](int64_t tb) -> int {
      if (dist) SBR_CM(h->comm->broadcast(h->Wh, (size_t)h->ldwh * pass_bn(b) * sizeof(__half), own, st),
                       "broadcast W_t");
      {
        Scope sc(h, SBR_K_PASS, (1.0 * M * M + 6.0 * M * b) / P, 2.0 * M * M * b / P);
        PassLaunch pl{};
        pl.shadow = h->Sh;
        pl.n = n;
        pl.ld_shadow = h->ldsh;
        pl.Wh = h->Wh;
        pl.M = M;
        pl.ld_wh = h->ldwh;
        pl.r0 = dist ? c0 : r0;
        pl.off = off;
        pl.b = b;
        pl.X = h->Xb + tb * M;
        pl.ldx = M;
        pl.num_sms = h->nsm;
        pl.seg_rows = 8;
        if (dist) {
          pl.own_P = P;
          pl.own_rank = rank;
          pl.nbo = nb;
          pl.shadow_cols = ncols_loc;
        }
        SBR_CK(launch_pass_tc(pl, st), "pass_tc");
        h->launches += 1;
      }
      if (dist) SBR_CM(h->comm->all_reduce_sum_f32(h->Xb + tb * M, (size_t)M * b, st), "all-reduce X_t");
      return SBR_OK;
    };
    for (int t = 0; fused && t < p; ++t) {
      const int64_t tb = (int64_t)t * b;
      float* Wt = Wb + tb * ldwb;
      if (leadJ) {
        Scope sc(h, SBR_K_PANEL, 4.0 * (M - tb) * b * 4 + (t ? 8.0 * M * b + 4.0 * (M - tb) * t * b * 5 : 0),
                 4.0 * (M - tb) * b * b * 2 + (t ? 10.0 * M * t * b * b : 0));
        ChainFusedLaunch L{};
        L.t = t;
        L.k = t * b;
        L.M = M;
        L.tb = tb;
        L.A = AJ;
        L.lda = lda;
        L.r0 = r0;
        L.Yb = h->Yb;
        L.ldy = ldn;
        L.Wt = Wt;
        L.ldw = ldwb;
        L.Xb = h->Xb;
        L.ldx = M;
        L.Xh = h->Xh;
        L.WtX = h->WtX;
        L.ldwx = nb;
        L.Gf = h->GH;
        L.Hf = h->GH + (size_t)nb * nb;
        L.Ph = h->Ph;
        L.Yh = h->Yh;
        L.Wrh = h->Wrh;
        L.ldk = h->ldk;
        L.Wh = Whc;
        L.ldwh = h->ldwh;
        L.ws = h->fused_ws;
        L.launch = h->fused_launches;
        L.declines = panel_chol_declines(h->chol_ws);
        L.orth_tol = 1e-6;
        L.grid = h->nsm;
        if (h->ptrace && h->ptrace_used < h->ptrace_cap) L.trace = h->ptrace + 32 * (int64_t)h->ptrace_used++;
        const cudaError_t fe = launch_chain_fused(L, st);
        if (fe != cudaSuccess) {   // the parity chain is broken: re-zero the workspace
          cudaGetLastError();
          cudaMemsetAsync(h->fused_ws, 0, chain_fused_ws_bytes(), st);
          h->fused_launches = 0;
          SBR_CK(fe, "chain_fused");
        }
        h->fused_launches++;
        h->launches += 1;
      }
      if (int prc = pass_t(tb)) return prc;
      if (t == p - 1 && leadJ) {  // the last panel's pass tail (the next fused launch does it otherwise)
        Scope sc(h, SBR_K_WMERGE, 4.0 * M * b * 2 + 2.0 * M * b, 2.0 * M * b * b);
        SBR_CK(launch_postpass(M, b, h->Xb + tb * M, M, Wt, ldwb, h->Xh + tb, h->ldk, h->WtX + tb + tb * nb, nb, st),
               "postpass");
        h->launches += 1;
      }
    }
    for (int t = 0; !fused && t < p; ++t) {
      const int64_t g = c0 + (int64_t)t * b;
      const int64_t tb = (int64_t)t * b;
      const int64_t m = M - tb;
      const int k = t * b;
      float* Wt = Wb + tb * ldwb;  // this panel's W columns (W_t^0 from the panel, then W_t)
      float* Gt = h->GH + (size_t)t * nb * b;
      float* Ht = h->GH + (size_t)nb * nb + (size_t)t * nb * b;
      if (t >= 1) {  // ---- a5: lazy update of panel t's columns (Alg.1 l.8-10)
        const int64_t c = tb - b;  // OA column of the panel's first column
        const int64_t rows = M - c;
        float* Ablk = AJ + g + g * lda;
        if (!leadJ) {
          // not this rank's step
        } else if (tc16) {  // P = W^T R (SIMT), then GA = OA(:,c) - [X | Y] [Y_c | P^T]^T on tcgen05 (fp16 operands)
          Scope sc(h, SBR_K_LAZY, 2.0 * rows * 2.0 * k + 8.0 * rows * b, 4.0 * rows * k * b);
          KxbArgs ka{};
          ka.mode = 0;
          ka.k = k;
          ka.b = b;
          ka.WtX = h->WtX;
          ka.ldwx = nb;
          ka.Y = h->Yb;
          ka.ldy = ldn;
          ka.X = h->Xb;
          ka.ldx = M;
          ka.c = c;
          ka.Ph = h->Ph;
          ka.ldph = h->ldk;
          ka.Adiag = Ablk;
          ka.lda = lda;
          SBR_CK(launch_kxb(ka, st), "lazy P");
          SkinnyNN q{};
          q.A0 = h->Xh;
          q.A1 = h->Yh;
          q.K0 = k;
          q.K1 = k;
          q.a_rows = M;
          q.lda = h->ldk;
          q.arow0 = c;
          q.B0 = h->Yh;
          q.ldb0 = h->ldk;
          q.b0_rows = M;
          q.brow0 = c;
          q.B1 = h->Ph;
          q.ldb1 = h->ldk;
          q.rows = rows;
          q.b = b;
          q.C = Ablk;
          q.ldc = lda;
          q.D = Ablk;
          q.ldd = lda;
          SBR_CK(launch_skinny_nn(q, st), "lazy_nn");
          h->launches += 2;
        } else {
          Scope sc(h, SBR_K_LAZY, 4.0 * rows * (2.0 * k + 2 * b), 4.0 * rows * k * b);
          // P = X_c^T - (W^T X) Y_c^T (k x b, fp32) and the diagonal block's mirror: the kxb kernel of the
          // FP16 chain with an fp32 output; then A_p -= X Y_c^T + Y P as ONE two-segment skinny update
          KxbArgs ka{};
          ka.mode = 0;
          ka.k = k;
          ka.b = b;
          ka.WtX = h->WtX;
          ka.ldwx = nb;
          ka.Y = h->Yb;
          ka.ldy = ldn;
          ka.X = h->Xb;
          ka.ldx = ldn;
          ka.c = c;
          ka.Ph = nullptr;
          ka.P32 = h->Pb;
          ka.ldp32 = k;
          ka.Adiag = Ablk;
          ka.lda = lda;
          SBR_CK(launch_kxb(ka, st), "lazy P");
          SBR_CK(skinny_upd2(rows, b, k, h->Xb + c, ldn, h->Yb + c, ldn, true, k, h->Yb + c, ldn, h->Pb, k, false, -1.f,
                             Ablk, lda, st),
                 "lazy X Y_c^T + Y P");
          h->launches += 2;
        }
      }
      if (leadJ) {  // ---- a1/a2: TSQR + reconstruction
        Scope sc(h, SBR_K_PANEL, 4.0 * m * b * 4, 4.0 * m * b * b * 2);
        PanelArgs pa{};
        pa.P = AJ + (g + b) + g * lda;
        pa.ldp = lda;
        pa.m = (int)m;
        pa.b = b;
        pa.Y = h->Yb + tb * ldn;
        pa.ldy = ldn;
        pa.W = Wt;
        pa.ldw = ldwb;
        pa.row0 = tb;
        pa.M = M;
        pa.Yh = tc16 ? h->Yh + tb : nullptr;
        pa.ldyh = h->ldk;
        pa.Wh = tc16 ? Whc : nullptr;          // W^0 (fp16, column-major): pass operand / merge B
        pa.ldwh = h->ldwh;
        pa.Wrh = (tc16 && t == 0) ? h->Wrh : nullptr;   // W_0 = W^0 (row-major): later merges
        pa.ldwrh = h->ldk;
        pa.ws_v = h->pv;
        pa.ws_tau = h->ptau;
        pa.ws_r = h->pr;
        pa.ws_q = h->pq;
        pa.ws_misc = h->pmisc;
        // CholeskyQR acceptance (reading R1): Q orthonormal in fp64 to far below the rounding of the
        // mode's operands -- FP16 mode rounds every GEMM operand to fp16 (u = 4.9e-4), 3xTF32 keeps
        // fp32 (u = 6e-8)
        pa.orth_tol = tc16 ? 1e-6 : 1e-8;
        if (h->ptrace && h->ptrace_used < h->ptrace_cap) pa.trace = h->ptrace + 32 * (int64_t)h->ptrace_used++;
        bool chol = false;
        if (h->panel_mode == 0 && m > 512) {   // CholeskyQR (k_panel_chol.cu), in-kernel Householder QR if it declines
          const cudaError_t ce = launch_panel_chol(pa, h->chol_ws, h->chol_launches, st);
          if (ce == cudaSuccess) {
            h->chol_launches++;   // the Gram-set / barrier parity advances only with a launched kernel
            h->launches += 1;
            chol = true;
          } else if (ce != cudaErrorNotSupported) {
            SBR_CK(ce, "panel_chol");
          }
        }
        pa.trace = nullptr;   // the phase trace is CholeskyQR's (TSQR has its own stamps)
        if (!chol) {          // the paper's TSQR: panels of <= 512 rows, or SBR_PANEL=tsqr
          const cudaError_t te = launch_panel(pa, h->panel_ctas, st);
          SBR_CK(te, "panel");
          if (pa.over_capacity) {
            std::lock_guard<std::mutex> lk(g_err_mu);
            g_last_err = "panel of " + std::to_string(m) + " x " + std::to_string(b) +
                         " exceeds the TSQR tree's capacity (one co-resident CTA per 256-row leaf)";
            return SBR_ERR_UNSUPPORTED;
          }
          h->launches += 1;
        }
      }
      if (tc16) {
        if (t >= 1 && leadJ) {
          // ---- a3 on tcgen05: G = Y^T W0, H = X^T W0 (one pass over Y, X); W^T X_t = H - (W^T X) G;
          //      W_t = W0 - W G, written as fp32 + fp16 (column-major for the pass, row-major for later merges)
          Scope sc(h, SBR_K_WMERGE, 2.0 * (M - tb) * 2.0 * k + 2.0 * M * k + 12.0 * M * b,
                   2.0 * (2.0 * (M - tb) + M) * k * b);
          SkinnyTN q{};
          q.A0 = h->Yh;
          q.A1 = h->Xh;
          q.K1 = k;
          q.a_rows = M;
          q.lda = h->ldk;
          q.B = Whc;
          q.b_rows = M;
          q.ldb = h->ldwh;
          q.row0 = tb;
          q.rows = M - tb;
          q.b = b;
          q.D0 = Gt;
          q.D1 = Ht;
          q.ldd = nb;
          q.num_sms = h->nsm;
          SBR_CK(launch_skinny_tn(q, st), "Y^T W0, X^T W0");
          SBR_CK(launch_g_to_half(k, b, Gt, nb, h->Gh, h->ldk, st), "G -> fp16");   // merge GEMM's B operand
          SkinnyNN mq{};
          mq.A0 = h->Wrh;
          mq.A1 = nullptr;
          mq.K0 = k;
          mq.K1 = 0;
          mq.a_rows = M;
          mq.lda = h->ldk;
          mq.arow0 = 0;
          mq.B0 = h->Gh;
          mq.ldb0 = h->ldk;
          mq.b0_rows = b;
          mq.brow0 = 0;
          mq.B1 = nullptr;
          mq.rows = M;
          mq.b = b;
          mq.C = Wt;
          mq.ldc = ldwb;
          mq.D = Wt;
          mq.ldd = ldwb;
          mq.Hcm = Whc;
          mq.ldhc = h->ldwh;
          mq.Hrm = h->Wrh + tb;
          mq.ldhr = h->ldk;
          SBR_CK(launch_skinny_nn(mq, st), "W merge");
          h->launches += 3;
        }
        // ---- a4: pass X_t = OA W_t on tcgen05 (fp16 shadow of the frozen OA); X_t zeroed at block start
        if (int prc = pass_t(tb)) return prc;
        if (leadJ) {  // X_t -> fp16 row-major (operand of later lazy updates); W_t^T X_t (b x b diagonal block);
                      // t >= 1: in the same launch W_{<t}^T X_t = H - (W^T X) G (the merge's kxb, reading R2),
                      // which nothing needs before the next lazy update
          Scope sc(h, SBR_K_WMERGE, 4.0 * M * b * 2 + 2.0 * M * b, 2.0 * M * b * b);
          if (t >= 1) {
            KxbArgs ka{};
            ka.mode = 1;
            ka.k = k;
            ka.b = b;
            ka.WtX = h->WtX;
            ka.ldwx = nb;
            ka.G = Gt;
            ka.H = Ht;
            ka.ldg = nb;
            SBR_CK(launch_postpass_merge(M, b, h->Xb + tb * M, M, Wt, ldwb, h->Xh + tb, h->ldk,
                                         h->WtX + tb + tb * nb, nb, ka, st),
                   "postpass + merge kxb");
          } else {
            SBR_CK(launch_postpass(M, b, h->Xb + tb * M, M, Wt, ldwb, h->Xh + tb, h->ldk, h->WtX + tb + tb * nb, nb,
                                   st),
                   "postpass");
          }
          h->launches += 1;
        }
        continue;
      }
      if (t >= 1 && leadJ) {  // ---- a3 (SIMT fp32): W merge
        Scope sc(h, SBR_K_WMERGE, 4.0 * (M - tb) * (k + b) + 4.0 * M * (k + 2 * b), 2.0 * (2.0 * M - tb) * k * b);
        SBR_CK(zero_matrix(k, b, h->Gb, k, st), "zero G");
        SBR_CK(gemm_tn(M - tb, k, b, 1.f, h->Yb + tb, ldn, Wb + tb + tb * ldwb, ldwb, h->Gb, k, st), "Y^T W0");
        SBR_CK(gemm_nn(M, b, k, -1.f, Wb, ldwb, h->Gb, k, false, 1.f, Wb + tb * ldwb, ldwb, Wb + tb * ldwb, ldwb,
                       st),
               "W merge");
        h->launches += 2;
      }
      if (tc32 && knob(KNOB_TF32_SIMT_PASS) && !dist) {   // test knob: the SIMT fp32 pass inside the
        // 3xTF32 reduction (attributes the mode's error between the pass and the other kernels)
        Scope sc(h, SBR_K_PASS, 4.0 * M * M / 2 + 8.0 * M * b, 2.0 * M * M * b);
        SBR_CK(sym_pass(M, b, OA, lda, h->Strip, ldn, sw, Wb + tb * ldwb, ldwb, h->Xb + tb * ldn, ldn, st), "pass");
        h->launches += 1;
      } else if (tc32) {  // ---- a4 (3xTF32 on tcgen05): OA frozen = A + strip copy, 32 W columns per launch
        Scope sc(h, SBR_K_PASS, (4.0 * M * M / 2 + 12.0 * M * b) / P, 3 * 2.0 * M * M * b / P);
        // distributed: the padding rows between X_t's columns are zeroed too (the all-reduce spans them)
        SBR_CK(zero_matrix(dist ? ldn : M, b, h->Xb + tb * ldn, ldn, st), "zero X_t");
        for (int c = 0; c < b; c += 32) {
          const int bh = std::min(32, b - c);
          if (leadJ) SBR_CK(split_tf32_w(M, bh, 32, Wb + (tb + c) * ldwb, ldwb, h->WS, h->ldws, st), "split W_t");
          if (dist) SBR_CM(h->comm->broadcast(h->WS, (size_t)h->ldws * 64 * sizeof(float), own, st), "broadcast W_t");
          PassTf32Launch pl{};
          if (dist) {   // this rank's tile columns of the 128-aligned grid from the block start
            pl.off = off;
            pl.own_P = P;
            pl.own_rank = rank;
            pl.nbo = nb;
            pl.ncols = ncols_loc;
          }
          pl.A = A;
          pl.n = n;
          pl.lda = lda;
          pl.r0 = r0;
          pl.S = h->Strip;
          pl.lds = ldn;
          pl.sw = sw;
          pl.WS = h->WS;
          pl.ldws = h->ldws;
          pl.M = M;
          pl.b = bh;
          pl.X = h->Xb + (tb + c) * ldn;
          pl.ldx = ldn;
          pl.num_sms = h->nsm;
          SBR_CK(launch_pass_tf32(pl, st), "pass_tf32");
          h->launches += 2;
        }
        h->launches += 1;
        if (dist)
          SBR_CM(h->comm->all_reduce_sum_f32(h->Xb + tb * ldn, (size_t)(b - 1) * ldn + M, st), "all-reduce X_t");
      } else {  // ---- a4 (3xTF32 mode, SIMT fp32): OA frozen = A + strip copy
        Scope sc(h, SBR_K_PASS, 4.0 * M * M / 2 + 8.0 * M * b, 2.0 * M * M * b);
        SBR_CK(sym_pass(M, b, OA, lda, h->Strip, ldn, sw, Wb + tb * ldwb, ldwb, h->Xb + tb * ldn, ldn, st),
               "pass");
        h->launches += 1;
      }
      if (leadJ) {  // W^T X column block (P:223 l.9 needs W^T OA W) -> WtX[:, tb:tb+b] and mirror
        Scope sc(h, SBR_K_WMERGE, 4.0 * M * (k + 2 * b), 2.0 * M * (k + b) * b);
        SBR_CK(zero_matrix(k + b, b, h->WtX + tb * nb, nb, st), "zero wtx");
        SBR_CK(gemm_tn(M, k + b, b, 1.f, Wb, ldwb, h->Xb + tb * ldn, ldn, h->WtX + tb * nb, nb, st), "W^T X");
        SBR_CK(mirror_wtx(k, b, h->WtX, nb, st), "mirror wtx");
        h->launches += 2;
      }
    }
    // ---- a6: trailing update once per block (Alg.1 l.12-13)
    const int64_t s = (int64_t)p * b - b;
    const int64_t Mt = M - s;
    const int kk = p * b;
    if (Mt > 0 && tc16 && dist) {   // the owner's Y (fp16) and W^T X for every rank's trailing update
      SBR_CM(h->comm->broadcast(h->Yh, (size_t)M * h->ldk * sizeof(__half), own, st), "broadcast Y");
      SBR_CM(h->comm->broadcast(h->WtX, (size_t)nb * nb * sizeof(float), own, st), "broadcast W^T X");
    }
    if (Mt > 0 && tc32 && dist) {   // 3xTF32: Y in fp32 (split on every rank)
      SBR_CM(h->comm->broadcast(h->Yb, (size_t)ldn * kk * sizeof(float), own, st), "broadcast Y");
      SBR_CM(h->comm->broadcast(h->WtX, (size_t)nb * nb * sizeof(float), own, st), "broadcast W^T X");
    }
    if (Mt > 0 && tc16) {
      Scope sc(h, SBR_K_SYR2K, 10.0 * Mt * Mt / 2 + 2.0 * Mt * kk * 4 + 4.0 * Mt * kk,
               2.0 * Mt * Mt * kk + 2.0 * Mt * kk * kk);
      SBR_CK(to_half_cm(kk, kk, kk, h->WtX, nb, h->WtXh, h->ldk, st), "WtX -> fp16");
      GemmTcLaunch gz{};
      gz.A0 = gz.A1 = h->Yh;
      gz.B0 = gz.B1 = h->WtXh;
      gz.K = kk;
      gz.a_rows = M;
      gz.ld_a = h->ldk;
      gz.b_rows = kk;
      gz.ld_b = h->ldk;
      gz.arow0 = s;
      gz.brow0 = 0;
      gz.Mrows = Mt;
      gz.Ncols = kk;
      gz.X = h->Xb + s;
      gz.ldx = M;
      gz.Zh = h->Zh + s * h->ldk;
      gz.ldz = h->ldk;
      gz.num_sms = h->nsm;
      SBR_CK(launch_zform_tc(gz, st), "zform_tc");
      GemmTcLaunch gs{};
      gs.A0 = h->Yh;
      gs.A1 = h->Zh;
      gs.B0 = h->Zh;
      gs.B1 = h->Yh;
      gs.K = kk;
      gs.a_rows = gs.b_rows = M;
      gs.ld_a = gs.ld_b = h->ldk;
      gs.arow0 = gs.brow0 = s;
      gs.Mrows = gs.Ncols = Mt;
      gs.C = A + (r0 + s) + (dist ? 0 : (r0 + s) * lda);   // distributed: local columns via the ownership map
      gs.ldc = lda;
      gs.shadow = h->Sh + (r0 + s) + (dist ? 0 : (r0 + s) * h->ldsh);
      gs.ld_shadow = h->ldsh;
      gs.num_sms = h->nsm;
      if (dist) {   // this rank's columns of the trailing region only
        gs.own_P = P;
        gs.own_rank = rank;
        gs.own_org = r0 + s;
        gs.nbo = nb;
      }
      SBR_CK(launch_syr2k_tc(gs, st), "syr2k_tc");
      h->launches += 3;
    } else if (Mt > 0 && tc32) {   // a6 in 3xTF32 on tcgen05: split Y, W^T X; Z (split) ; SYR2K
      Scope sc(h, SBR_K_SYR2K, 8.0 * Mt * Mt + 4.0 * Mt * kk * 8,
               3 * (2.0 * Mt * Mt * kk + 2.0 * Mt * kk * kk));
      SBR_CK(split_tf32_rm(Mt, kk, h->Yb + s, ldn, h->YS + s * h->ldts, h->ldts, h->tlo, st), "split Y");
      SBR_CK(split_tf32_rm(kk, kk, h->WtX, nb, h->GS, h->ldts, h->tlo, st), "split W^T X");
      GemmTcLaunch gz{};
      gz.A0 = gz.A1 = (const __half*)h->YS;
      gz.B0 = gz.B1 = (const __half*)h->GS;
      gz.K = kk;
      gz.lo_off = h->tlo;
      gz.a_rows = M;
      gz.ld_a = h->ldts;
      gz.b_rows = kk;
      gz.ld_b = h->ldts;
      gz.arow0 = s;
      gz.brow0 = 0;
      gz.Mrows = Mt;
      gz.Ncols = kk;
      gz.X = h->Xb + s;
      gz.ldx = ldn;
      gz.Zs = h->ZS + s * h->ldts;
      gz.ldz = h->ldts;
      gz.num_sms = h->nsm;
      SBR_CK(launch_zform_tf32(gz, st), "zform_tf32");
      GemmTcLaunch gs{};
      gs.A0 = (const __half*)h->YS;
      gs.A1 = (const __half*)h->ZS;
      gs.B0 = (const __half*)h->ZS;
      gs.B1 = (const __half*)h->YS;
      gs.K = kk;
      gs.lo_off = h->tlo;
      gs.a_rows = gs.b_rows = M;
      gs.ld_a = gs.ld_b = h->ldts;
      gs.arow0 = gs.brow0 = s;
      gs.Mrows = gs.Ncols = Mt;
      gs.C = A + (r0 + s) + (dist ? 0 : (r0 + s) * lda);   // distributed: local columns via the ownership map
      gs.ldc = lda;
      gs.num_sms = h->nsm;
      if (dist) {   // this rank's columns of the trailing region only
        gs.own_P = P;
        gs.own_rank = rank;
        gs.own_org = r0 + s;
        gs.nbo = nb;
      }
      SBR_CK(launch_syr2k_tf32(gs, st), "syr2k_tf32");
      h->launches += 4;
    } else if (Mt > 0) {
      Scope sc(h, SBR_K_SYR2K, 4.0 * Mt * Mt + 4.0 * Mt * kk * 3, 2.0 * Mt * Mt * kk + 2.0 * Mt * kk * kk);
      SBR_CK(gemm_nn(Mt, kk, kk, -0.5f, h->Yb + s, ldn, h->WtX, nb, false, 1.f, h->Xb + s, ldn, h->Zb + s, ldn, st),
             "Z");
      SBR_CK(syr2k_lower(Mt, kk, h->Yb + s, ldn, h->Zb + s, ldn, A + (r0 + s) + (r0 + s) * lda, lda, st), "syr2k");
      h->launches += 2;
    }
  }
  }
band_out:
  if (!dist) {
    Scope sc(h, SBR_K_OTHER, 8.0 * (b + 1) * n, 0);
    SBR_CK(extract_band(n, b, A, lda, AB, ldab, kexp, flag, st), "extract_band");
    h->launches += 1;
  } else {   // each rank its own columns of the band, summed over the ranks; rank 0 returns it
    Scope sc(h, SBR_K_OTHER, 8.0 * (b + 1) * n, 0);
    SBR_CK(cudaMemsetAsync(h->ABd, 0, sizeof(float) * (b + 1) * n, st), "zero band");
    SBR_CK(extract_band(n, b, A, lda, h->ABd, b + 1, n <= b + 1 ? nullptr : kexp, flag, st, ncols_loc, cm),
           "extract_band");
    SBR_CM(h->comm->all_reduce_sum_f32(h->ABd, (size_t)(b + 1) * n, st), "all-reduce band");
    if (lead && AB)
      SBR_CK(cudaMemcpy2DAsync(AB, ldab * sizeof(float), h->ABd, (b + 1) * sizeof(float), (b + 1) * sizeof(float), n,
                               cudaMemcpyDeviceToDevice, st),
             "band out");
    h->launches += 1;
  }
  return latch_status(h, st);   // errors found on the device are reported by sbr_sync / the next call
}

}  // namespace

extern "C" {

int sbr_create(sbr_handle_t* out, int device, void* stream) {
  if (!out) return -1;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess) {
    cudaGetLastError();
    return SBR_ERR_CUDA;
  }
  if (device < 0 || device >= ndev) return -2;
  SBR_CK(cudaSetDevice(device), "cudaSetDevice");
  sbr_ctx* h = new sbr_ctx();
  h->device = device;
  h->stream = (cudaStream_t)stream;
  cudaDeviceGetAttribute(&h->nsm, cudaDevAttrMultiProcessorCount, device);
  const char* pm = getenv("SBR_PANEL");   // "tsqr": the paper's TSQR panel only (ablation)
  if (pm && strcmp(pm, "tsqr") == 0) h->panel_mode = 1;
  const char* tt = getenv("SBR_TF32_TC");  // "0": 3xTF32 mode on the SIMT fp32 kernels (ablation)
  if (tt && strcmp(tt, "0") == 0) h->tf32_tc = false;
  const char* fz = getenv("SBR_FUSED");    // "1": the fused FP16 chain kernel, "0": the per-kernel chain
  if (fz) h->fused = strcmp(fz, "1") == 0;
  *out = h;
  return SBR_OK;
}

int sbr_form_q(sbr_handle_t h, int64_t n, int b, int nb, const float* A, int64_t lda, const float* W, int64_t ldw,
               float* Q, int64_t ldq) {
  if (!h) return -1;
  if (n < 1) return -2;
  if (b < 1 || b > 64) return -3;
  if (nb < b || nb % b != 0 || nb > 4096) return -4;
  if (!A) return -5;
  if (lda < n) return -6;
  if (!W) return -7;
  if (ldw < n) return -8;
  if (!Q) return -9;
  if (ldq < n) return -10;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  cudaStream_t st = h->stream;
  SBR_CK(set_identity(n, Q, ldq, st), "Q = I");
  h->launches++;
  const int64_t ncols = n - b;
  if (ncols <= 0) return SBR_OK;
  // backward accumulation Q = H_1 (H_2 (... I)): block J (last first) updates Q[r0:, r0:] -=
  // W_J (Y_J^T Q[r0:, r0:]) -- two 3xTF32 tcgen05 products per block over [hi | lo] splits
  const int64_t M0 = n - b;
  const int64_t loM = (M0 + 31) / 32 * 32, ldM = 2 * loM;
  const int64_t lok = (nb + 31) / 32 * 32, ldk = 2 * lok;
  // split operands in handle-owned memory (a per-call cudaMallocAsync of these GB-sized buffers
  // costs more than the products when the pool returns the pages in between)
  const size_t nQS = align_up(sizeof(float) * M0 * ldM), nYS = align_up(sizeof(float) * nb * ldM),
               nWS = align_up(sizeof(float) * M0 * ldk);
  const size_t need = nQS + nYS + 2 * nWS;
  if (h->fq_bytes < need) {
    SBR_CK(cudaStreamSynchronize(st), "sync");   // a previous call may still use the old buffer
    if (h->fq) cudaFree(h->fq);
    h->fq = nullptr;
    h->fq_bytes = 0;
    if (cudaMalloc(&h->fq, need) != cudaSuccess) {
      cudaGetLastError();
      return SBR_ERR_NOMEM;
    }
    h->fq_bytes = need;
  }
  float* QS = (float*)h->fq;
  float* YS = (float*)((char*)h->fq + nQS);
  float* WS = (float*)((char*)h->fq + nQS + nYS);
  float* TS = (float*)((char*)h->fq + nQS + nYS + nWS);
  const int64_t nblk = (ncols + nb - 1) / nb;
  cudaError_t e = cudaSuccess;
  for (int64_t J = nblk - 1; J >= 0 && e == cudaSuccess; --J) {
    const int64_t c0 = J * nb, r0 = c0 + b, M = n - r0;
    const int k = (int)std::min<int64_t>(nb, ncols - c0);
    float* Qs = Q + r0 + r0 * ldq;
    Scope sc(h, SBR_K_OTHER, 4.0 * M * M * 4 + 8.0 * M * k * 4, 3 * 4.0 * M * M * k);
    if ((e = split_tf32_cm(M, k, A + r0 + c0 * lda, lda, true, YS, ldM, loM, st)) != cudaSuccess) break;
    if ((e = split_tf32_rm(M, k, W + r0 + c0 * ldw, ldw, WS, ldk, lok, st)) != cudaSuccess) break;
    if ((e = split_tf32_cm(M, (int)M, Qs, ldq, false, QS, ldM, loM, st)) != cudaSuccess) break;
    GemmTcLaunch g1{};   // T^T = Q_sub^T Y_J  (M x k), written split row-major
    g1.A0 = g1.A1 = (const __half*)QS;
    g1.B0 = g1.B1 = (const __half*)YS;
    g1.K = M;
    g1.lo_off = loM;
    g1.a_rows = M;
    g1.ld_a = ldM;
    g1.b_rows = k;
    g1.ld_b = ldM;
    g1.Mrows = M;
    g1.Ncols = k;
    g1.Zs = TS;
    g1.ldz = ldk;
    g1.zlo_off = lok;
    g1.num_sms = h->nsm;
    if ((e = launch_gemm_split_tf32(g1, st)) != cudaSuccess) break;
    GemmTcLaunch g2{};   // Q_sub -= W_J T
    g2.A0 = g2.A1 = (const __half*)WS;
    g2.B0 = g2.B1 = (const __half*)TS;
    g2.K = k;
    g2.lo_off = lok;
    g2.a_rows = M;
    g2.ld_a = ldk;
    g2.b_rows = M;
    g2.ld_b = ldk;
    g2.Mrows = M;
    g2.Ncols = M;
    g2.C = Qs;
    g2.ldc = ldq;
    g2.num_sms = h->nsm;
    if ((e = launch_gemm_sub_tf32(g2, st)) != cudaSuccess) break;
    h->launches += 5;
  }
  SBR_CK(e, "form_q");
  return SBR_OK;
}

}  // extern "C" (reopened below)

namespace {

// 3xTF32 split workspace of the back-transformation calls (handle-owned, grown on demand)
float* fq_grow(sbr_ctx* h, size_t need, int* rc) {
  *rc = SBR_OK;
  if (h->fq_bytes < need) {
    if (cudaStreamSynchronize(h->stream) != cudaSuccess) {   // a previous call may still use the old buffer
      *rc = SBR_ERR_CUDA;
      return nullptr;
    }
    if (h->fq) cudaFree(h->fq);
    h->fq = nullptr;
    h->fq_bytes = 0;
    if (cudaMalloc(&h->fq, need) != cudaSuccess) {
      cudaGetLastError();
      *rc = SBR_ERR_NOMEM;
      return nullptr;
    }
    h->fq_bytes = need;
  }
  return (float*)h->fq;
}

// T^T = Bc^T Yc (rb x ka, split row-major into TS) and C -= Wr T^T^T -- the two 3xTF32 tcgen05
// products of one WY application C <- C - W (Y^T C) (sbr_form_q's pattern):
//   C  : M x kc column-major (the rows the reflectors touch),  Y, W: M x ka column-major
cudaError_t wy_apply_tf32(sbr_ctx* h, int64_t M, int64_t kc, int64_t ka, const float* Y, int64_t ldy, bool unit_y,
                          const float* W, int64_t ldw, float* C, int64_t ldc, float* CS, float* YS, float* WS,
                          float* TS, int64_t ldM, int64_t loM, int64_t ldk, int64_t lok, cudaStream_t st) {
  cudaError_t e;
  if ((e = split_tf32_cm(M, (int)ka, Y, ldy, unit_y, YS, ldM, loM, st)) != cudaSuccess) return e;
  if ((e = split_tf32_rm(M, (int)ka, W, ldw, WS, ldk, lok, st)) != cudaSuccess) return e;
  if ((e = split_tf32_cm(M, (int)kc, C, ldc, false, CS, ldM, loM, st)) != cudaSuccess) return e;
  GemmTcLaunch g1{};   // T^T = C^T Y  (kc x ka), written split row-major
  g1.A0 = g1.A1 = (const __half*)CS;
  g1.B0 = g1.B1 = (const __half*)YS;
  g1.K = M;
  g1.lo_off = loM;
  g1.a_rows = kc;
  g1.ld_a = ldM;
  g1.b_rows = ka;
  g1.ld_b = ldM;
  g1.Mrows = kc;
  g1.Ncols = ka;
  g1.Zs = TS;
  g1.ldz = ldk;
  g1.zlo_off = lok;
  g1.num_sms = h->nsm;
  if ((e = launch_gemm_split_tf32(g1, st)) != cudaSuccess) return e;
  GemmTcLaunch g2{};   // C -= W T
  g2.A0 = g2.A1 = (const __half*)WS;
  g2.B0 = g2.B1 = (const __half*)TS;
  g2.K = ka;
  g2.lo_off = lok;
  g2.a_rows = M;
  g2.ld_a = ldk;
  g2.b_rows = kc;
  g2.ld_b = ldk;
  g2.Mrows = M;
  g2.Ncols = kc;
  g2.C = C;
  g2.ldc = ldc;
  g2.num_sms = h->nsm;
  return launch_gemm_sub_tf32(g2, st);
}

}  // namespace

extern "C" {

int sbr_apply_q(sbr_handle_t h, int64_t n, int b, int nb, const float* A, int64_t lda, const float* W, int64_t ldw,
                float* X, int64_t ldx, int64_t kx) {
  if (!h) return -1;
  if (n < 1) return -2;
  if (b < 1 || b > 64) return -3;
  if (nb < b || nb % b != 0 || nb > 4096) return -4;
  if (!A) return -5;
  if (lda < n) return -6;
  if (!W) return -7;
  if (ldw < n) return -8;
  if (!X) return -9;
  if (ldx < n) return -10;
  if (kx < 0) return -11;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  cudaStream_t st = h->stream;
  const int64_t ncols = n - b;
  if (ncols <= 0 || kx == 0) return SBR_OK;
  // X <- Q X = Q_0 (Q_1 (... (Q_last X))): block J (last first): X[r0:] -= W_J (Y_J^T X[r0:])
  const int64_t M0 = n - b;
  const int64_t loM = (M0 + 31) / 32 * 32, ldM = 2 * loM;
  const int64_t lok = (nb + 31) / 32 * 32, ldk = 2 * lok;
  const size_t nXS = align_up(sizeof(float) * kx * ldM), nYS = align_up(sizeof(float) * nb * ldM),
               nWS = align_up(sizeof(float) * M0 * ldk), nTS = align_up(sizeof(float) * kx * ldk);
  int rc = SBR_OK;
  float* base = fq_grow(h, nXS + nYS + nWS + nTS, &rc);
  if (rc != SBR_OK) return rc;
  float* XS = base;
  float* YS = (float*)((char*)base + nXS);
  float* WS = (float*)((char*)base + nXS + nYS);
  float* TS = (float*)((char*)base + nXS + nYS + nWS);
  const int64_t nblk = (ncols + nb - 1) / nb;
  for (int64_t J = nblk - 1; J >= 0; --J) {
    const int64_t c0 = J * nb, r0 = c0 + b, M = n - r0;
    const int k = (int)std::min<int64_t>(nb, ncols - c0);
    Scope sc(h, SBR_K_OTHER, 4.0 * M * kx * 4 + 8.0 * M * k * 4, 3 * 4.0 * M * kx * k);
    SBR_CK(wy_apply_tf32(h, M, kx, k, A + r0 + c0 * lda, lda, true, W + r0 + c0 * ldw, ldw, X + r0, ldx, XS, YS, WS,
                         TS, ldM, loM, ldk, lok, st),
           "apply_q");
    h->launches += 5;
  }
  return SBR_OK;
}

}  // extern "C"

namespace {

// Alg. 2: W of the column range [ca, ce) (whole nb-blocks) formed recursively --
// left half, right half, then W_R <- W_R - W_L (Y_L^T W_R), which turns the per-block factors
// into ONE W with Q = I - W Y^T over those columns.
int form_w_rec(sbr_ctx* h, int64_t n, int b, int nb, const float* A, int64_t lda, float* Wo, int64_t ldwo,
               int64_t ca, int64_t ce, float* CS, float* YS, float* WS, float* TS, int64_t ldM, int64_t loM,
               int64_t ldk, int64_t lok) {
  const int64_t nblk = (ce - ca + nb - 1) / nb;
  if (nblk <= 1) return SBR_OK;
  const int64_t cm = ca + (nblk / 2) * nb;
  int rc = form_w_rec(h, n, b, nb, A, lda, Wo, ldwo, ca, cm, CS, YS, WS, TS, ldM, loM, ldk, lok);
  if (rc == SBR_OK) rc = form_w_rec(h, n, b, nb, A, lda, Wo, ldwo, cm, ce, CS, YS, WS, TS, ldM, loM, ldk, lok);
  if (rc != SBR_OK) return rc;
  // merge: rows the left reflectors touch, r >= ca + b; W_R is zero above cm + b, so T = Y_L^T W_R
  // only needs rows >= cm + b, where Y_L is its stored tail (the unit rows lie above)
  const int64_t kL = cm - ca, kR = ce - cm, rL = ca + b, rR = cm + b;
  const int64_t ML = n - rL, MR = n - rR;
  cudaStream_t st = h->stream;
  Scope sc(h, SBR_K_OTHER, 4.0 * (ML * (kL + kR) + MR * (kL + kR)) * 4, 3 * 2.0 * (MR + ML) * kL * kR);
  cudaError_t e;
  if ((e = split_tf32_cm(MR, (int)kL, A + rR + ca * lda, lda, false, YS, ldM, loM, st)) != cudaSuccess) return SBR_ERR_CUDA;
  if ((e = split_tf32_cm(MR, (int)kR, Wo + rR + cm * ldwo, ldwo, false, CS, ldM, loM, st)) != cudaSuccess)
    return SBR_ERR_CUDA;
  if ((e = split_tf32_rm(ML, (int)kL, Wo + rL + ca * ldwo, ldwo, WS, ldk, lok, st)) != cudaSuccess) return SBR_ERR_CUDA;
  GemmTcLaunch g1{};   // T^T = W_R^T Y_L  (kR x kL)
  g1.A0 = g1.A1 = (const __half*)CS;
  g1.B0 = g1.B1 = (const __half*)YS;
  g1.K = MR;
  g1.lo_off = loM;
  g1.a_rows = kR;
  g1.ld_a = ldM;
  g1.b_rows = kL;
  g1.ld_b = ldM;
  g1.Mrows = kR;
  g1.Ncols = kL;
  g1.Zs = TS;
  g1.ldz = ldk;
  g1.zlo_off = lok;
  g1.num_sms = h->nsm;
  if ((e = launch_gemm_split_tf32(g1, st)) != cudaSuccess) return SBR_ERR_CUDA;
  GemmTcLaunch g2{};   // W_R[rL:] -= W_L T
  g2.A0 = g2.A1 = (const __half*)WS;
  g2.B0 = g2.B1 = (const __half*)TS;
  g2.K = kL;
  g2.lo_off = lok;
  g2.a_rows = ML;
  g2.ld_a = ldk;
  g2.b_rows = kR;
  g2.ld_b = ldk;
  g2.Mrows = ML;
  g2.Ncols = kR;
  g2.C = Wo + rL + cm * ldwo;
  g2.ldc = ldwo;
  g2.num_sms = h->nsm;
  if ((e = launch_gemm_sub_tf32(g2, st)) != cudaSuccess) return SBR_ERR_CUDA;
  h->launches += 5;
  return SBR_OK;
}

}  // namespace

extern "C" {

int sbr_form_w(sbr_handle_t h, int64_t n, int b, int nb, const float* A, int64_t lda, const float* W, int64_t ldw,
               float* Wo, int64_t ldwo) {
  if (!h) return -1;
  if (n < 1) return -2;
  if (b < 1 || b > 64) return -3;
  if (nb < b || nb % b != 0 || nb > 4096) return -4;
  if (!A) return -5;
  if (lda < n) return -6;
  if (!W) return -7;
  if (ldw < n) return -8;
  if (!Wo) return -9;
  if (ldwo < n) return -10;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  cudaStream_t st = h->stream;
  const int64_t ncols = n - b;
  if (ncols <= 0) return SBR_OK;
  // start: the per-block W_J with zeros above each block's rows (Wo[:, c] = W[:, c] for r >= r0(J))
  SBR_CK(copy_block_w(n, b, nb, W, ldw, Wo, ldwo, st), "W blocks");
  h->launches += 1;
  const int64_t M0 = n - b;
  const int64_t loM = (M0 + 31) / 32 * 32, ldM = 2 * loM;
  const int64_t kmax = (ncols + 1) / 2 + nb, lok = (kmax + 31) / 32 * 32, ldk = 2 * lok;
  const size_t nCS = align_up(sizeof(float) * kmax * ldM), nYS = align_up(sizeof(float) * kmax * ldM),
               nWS = align_up(sizeof(float) * M0 * ldk), nTS = align_up(sizeof(float) * kmax * ldk);
  int rc = SBR_OK;
  float* base = fq_grow(h, nCS + nYS + nWS + nTS, &rc);
  if (rc != SBR_OK) return rc;
  float* CS = base;
  float* YS = (float*)((char*)base + nCS);
  float* WS = (float*)((char*)base + nCS + nYS);
  float* TS = (float*)((char*)base + nCS + nYS + nWS);
  rc = form_w_rec(h, n, b, nb, A, lda, Wo, ldwo, 0, ncols, CS, YS, WS, TS, ldM, loM, ldk, lok);
  if (rc == SBR_ERR_CUDA) set_err("form_w", cudaGetLastError());
  return rc;
}

// ---------------------------------------------------------------- stage two
static char* s2_grow(sbr_ctx* h, size_t need, int* rc) {
  *rc = SBR_OK;
  if (h->s2_bytes < need) {
    if (cudaStreamSynchronize(h->stream) != cudaSuccess) {
      *rc = SBR_ERR_CUDA;
      return nullptr;
    }
    if (h->s2) cudaFree(h->s2);
    h->s2 = nullptr;
    h->s2_bytes = 0;
    if (cudaMalloc(&h->s2, need) != cudaSuccess) {
      cudaGetLastError();
      *rc = SBR_ERR_NOMEM;
      return nullptr;
    }
    h->s2_bytes = need;
  }
  return (char*)h->s2;
}

static int stage2_run(sbr_ctx* h, int64_t n, int b, const float* AB, int64_t ldab, double* d, double* e, double* lam,
                      char* ws) {
  cudaStream_t st = h->stream;
  if (AB) {
    // bulge chase: per step ~ 3 b x b fp64 blocks read + written
    const int64_t steps = n > 2 && b > 1 ? (n - 2) * ((n + b - 1) / b) / 2 : 0;
    Scope sc(h, SBR_K_STAGE2, 48.0 * b * b * (double)steps, 8.0 * b * b * (double)steps);
    SBR_CK(band_to_tridiag(n, b, AB, ldab, ws, d, e, st), "band_to_tridiag");
    h->launches += (n > 2 && b > 1) ? 3 : 2;
  }
  if (lam) {
    Scope sc(h, SBR_K_STAGE2, 16.0 * n, 4.0 * 53.0 * (double)n * n);
    SBR_CK(tridiag_eigenvalues(n, d, e, ws, lam, st), "tridiag_eigenvalues");
    h->launches += 2;
  }
  return SBR_OK;
}

static size_t s2_align(size_t x) { return (x + 255) & ~size_t(255); }

int sbr_band_to_tridiag(sbr_handle_t h, int64_t n, int b, const float* AB, int64_t ldab, double* d, double* e) {
  if (!h) return -1;
  if (n < 0) return -2;
  if (b < 1 || b > 64) return -3;
  if (!AB && n > 0) return -4;
  if (ldab < b + 1) return -5;
  if (!d && n > 0) return -6;
  if (!e && n > 1) return -7;
  if (n == 0) return SBR_OK;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  int rc = SBR_OK;
  char* ws = s2_grow(h, stage2_ws_bytes(n, b), &rc);
  if (rc != SBR_OK) return rc;
  return stage2_run(h, n, b, AB, ldab, d, e, nullptr, ws);
}

int sbr_tridiag_eigenvalues(sbr_handle_t h, int64_t n, const double* d, const double* e, double* lam) {
  if (!h) return -1;
  if (n < 0) return -2;
  if (!d && n > 0) return -3;
  if (!e && n > 1) return -4;
  if (!lam && n > 0) return -5;
  if (n == 0) return SBR_OK;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  int rc = SBR_OK;
  char* ws = s2_grow(h, tridiag_eig_ws_bytes(n), &rc);
  if (rc != SBR_OK) return rc;
  return stage2_run(h, n, 1, nullptr, 0, const_cast<double*>(d), const_cast<double*>(e), lam, ws);
}

int sbr_band_eigenvalues(sbr_handle_t h, int64_t n, int b, const float* AB, int64_t ldab, double* lam) {
  if (!h) return -1;
  if (n < 0) return -2;
  if (b < 1 || b > 64) return -3;
  if (!AB && n > 0) return -4;
  if (ldab < b + 1) return -5;
  if (!lam && n > 0) return -6;
  if (n == 0) return SBR_OK;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  const size_t sde = s2_align(sizeof(double) * 2 * n);
  const size_t sw = std::max(stage2_ws_bytes(n, b), tridiag_eig_ws_bytes(n));
  int rc = SBR_OK;
  char* base = s2_grow(h, sde + sw, &rc);
  if (rc != SBR_OK) return rc;
  double* d = (double*)base;
  double* e = d + n;
  char* ws = base + sde;
  if ((rc = stage2_run(h, n, b, AB, ldab, d, e, nullptr, ws)) != SBR_OK) return rc;
  return stage2_run(h, n, b, nullptr, 0, d, e, lam, ws);
}

int sbr_eigenvalues(sbr_handle_t h, int mode, int64_t n, int b, int nb, float* A, int64_t lda, double* lam) {
  if (!h) return -1;
  if (mode != SBR_FP16_FP32ACC && mode != SBR_3XTF32 && mode != SBR_BF16_FP32ACC) return -2;
  if (n < 1) return -3;
  if (b < 1 || b > 64) return -4;
  if (!lam) return -8;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  const size_t sab = s2_align(sizeof(float) * (size_t)(b + 1) * n);
  const size_t sde = s2_align(sizeof(double) * 2 * n);
  const size_t sw = std::max(stage2_ws_bytes(n, b), tridiag_eig_ws_bytes(n));
  int rc = SBR_OK;
  char* base = s2_grow(h, sab + sde + sw, &rc);
  if (rc != SBR_OK) return rc;
  float* AB = (float*)base;
  double* d = (double*)(base + sab);
  double* e = d + n;
  char* ws = base + sab + sde;
  rc = sbr_reduce(h, mode, n, b, nb, A, lda, AB, b + 1, nullptr, 0);
  if (rc != SBR_OK) return rc;   // argument positions 1-7 coincide with sbr_reduce's
  if ((rc = stage2_run(h, n, b, AB, b + 1, d, e, nullptr, ws)) != SBR_OK) return rc;
  return stage2_run(h, n, b, nullptr, 0, d, e, lam, ws);
}

int sbr_set_stream(sbr_handle_t h, void* stream) {
  if (!h) return -1;
  h->stream = (cudaStream_t)stream;
  return SBR_OK;
}

int sbr_destroy(sbr_handle_t h) {
  if (!h) return -1;
  cudaSetDevice(h->device);
  cudaStreamSynchronize(h->stream);
  drain_stats(h);
  delete h->comm;
  for (auto e : h->ev_pool) cudaEventDestroy(e);
  if (h->ws) cudaFree(h->ws);
  if (h->e2e) cudaFree(h->e2e);
  if (h->fq) cudaFree(h->fq);
  if (h->s2) cudaFree(h->s2);
  if (h->ptrace) cudaFree(h->ptrace);
  if (h->pinned) cudaFreeHost(h->pinned);
  for (auto e : h->slot_ev)
    if (e) cudaEventDestroy(e);
  delete h;
  return SBR_OK;
}

int sbr_workspace_query(sbr_handle_t h, int64_t n, int b, int nb, int mode, size_t* bytes) {
  if (!bytes) return -6;
  if (n < 1) return -2;
  if (b < 1 || b > 64) return -3;
  if (nb < b || nb % b != 0 || nb > 4096) return -4;
  if (mode != SBR_FP16_FP32ACC && mode != SBR_3XTF32 && mode != SBR_BF16_FP32ACC) return -5;
  if (n <= b + 1) {
    *bytes = 0;
    return SBR_OK;
  }
  (void)h;
  return ensure_ws(nullptr, n, b, nb, mode, bytes);
}

int sbr_reduce(sbr_handle_t h, int mode, int64_t n, int b, int nb, float* A, int64_t lda, float* AB, int64_t ldab,
               float* W, int64_t ldw) {
  int rc = validate(h, mode, n, b, nb, A, lda, AB, ldab, W, ldw);
  if (rc != SBR_OK) return rc;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  return reduce_device(h, mode, n, b, nb, A, lda, AB, ldab, W, ldw);
}

int sbr_reduce_host(sbr_handle_t h, int mode, int64_t n, int b, int nb, float* A, int64_t lda, float* AB,
                    int64_t ldab, float* W, int64_t ldw, int outputs) {
  int rc = validate(h, mode, n, b, nb, A, lda, AB, ldab, W, ldw);
  if (rc != SBR_OK) return rc;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  const size_t sa = align_up((size_t)n * n * sizeof(float));
  const size_t sab = align_up((size_t)(b + 1) * n * sizeof(float));
  const size_t sw = W ? align_up((size_t)n * std::max<int64_t>(1, n - b) * sizeof(float)) : 0;
  const size_t need = sa + sab + sw;
  if (h->e2e_bytes < need) {
    if (h->e2e) cudaFree(h->e2e);
    h->e2e = nullptr;
    h->e2e_bytes = 0;
    if (cudaMalloc(&h->e2e, need) != cudaSuccess) {
      cudaGetLastError();
      return SBR_ERR_NOMEM;
    }
    h->e2e_bytes = need;
  }
  float* dA = (float*)h->e2e;
  float* dAB = (float*)((char*)h->e2e + sa);
  float* dW = W ? (float*)((char*)h->e2e + sa + sab) : nullptr;
  cudaStream_t st = h->stream;
  SBR_CK(cudaMemcpy2DAsync(dA, n * sizeof(float), A, lda * sizeof(float), n * sizeof(float), n,
                           cudaMemcpyHostToDevice, st),
         "H2D A");
  rc = reduce_device(h, mode, n, b, nb, dA, n, dAB, b + 1, dW, n);
  if (rc != SBR_OK) return rc;
  SBR_CK(cudaMemcpy2DAsync(AB, ldab * sizeof(float), dAB, (b + 1) * sizeof(float), (b + 1) * sizeof(float), n,
                           cudaMemcpyDeviceToHost, st),
         "D2H AB");
  if (outputs & SBR_OUT_Y) {
    SBR_CK(cudaMemcpy2DAsync(A, lda * sizeof(float), dA, n * sizeof(float), n * sizeof(float), n,
                             cudaMemcpyDeviceToHost, st),
           "D2H A");
  }
  if (W && (outputs & SBR_OUT_W) && n > b) {
    SBR_CK(cudaMemcpy2DAsync(W, ldw * sizeof(float), dW, n * sizeof(float), n * sizeof(float), n - b,
                             cudaMemcpyDeviceToHost, st),
           "D2H W");
  }
  SBR_CK(cudaStreamSynchronize(st), "sync");
  return poll_latched(h, true);   // the call returns after the results are on the host: report now
}

int sbr_get_unique_id(void* id) {
  if (!id) return -1;
  if (const char* e = nccl::load()) {
    std::lock_guard<std::mutex> lk(g_err_mu);
    g_last_err = e;
    return SBR_ERR_NCCL;
  }
  nccl::UniqueId u;
  SBR_NC(nccl::get_unique_id(&u), "ncclGetUniqueId");
  memcpy(id, &u, sizeof(u));
  return SBR_OK;
}

static int create_dist_common(sbr_handle_t* out, int device, void* stream, int rank, int nranks,
                              const std::function<sbr::Comm*(std::string*)>& make) {
  int rc = sbr_create(out, device, stream);
  if (rc != SBR_OK) return rc;
  sbr_ctx* h = *out;
  h->rank = rank;
  h->nranks = nranks;
  std::string msg;
  h->comm = make(&msg);
  if (!h->comm) {
    {
      std::lock_guard<std::mutex> lk(g_err_mu);
      g_last_err = msg;
    }
    sbr_destroy(h);
    *out = nullptr;
    return SBR_ERR_NCCL;
  }
  return SBR_OK;
}

int sbr_create_dist(sbr_handle_t* out, int device, void* stream, const void* unique_id, int rank, int nranks) {
  if (!out) return -1;
  if (!unique_id) return -4;
  if (nranks < 1) return -6;
  if (rank < 0 || rank >= nranks) return -5;
  return create_dist_common(out, device, stream, rank, nranks, [&](std::string* msg) {
    return sbr::make_nccl_comm(unique_id, rank, nranks, msg);
  });
}

int sbr_create_dist_local(sbr_handle_t* out, int device, void* stream, int group, int rank, int nranks) {
  if (!out) return -1;
  if (nranks < 1 || nranks > 16) return -6;
  if (rank < 0 || rank >= nranks) return -5;
  SBR_CK(cudaSetDevice(device), "cudaSetDevice");
  return create_dist_common(out, device, stream, rank, nranks, [&](std::string* msg) {
    return sbr::make_local_comm(group, rank, nranks, msg);
  });
}

int64_t sbr_local_cols(int64_t n, int nb, int rank, int nranks) {
  if (n < 0 || nb < 1 || nranks < 1 || rank < 0 || rank >= nranks) return -1;
  return local_cols(n, nb, nranks, rank);
}

int sbr_reduce_dist(sbr_handle_t h, int mode, int64_t n, int b, int nb, float* A, int64_t lda, float* AB,
                    int64_t ldab, float* W, int64_t ldw) {
  if (!h) return -1;
  const bool lead = h->rank == 0;
  // outputs: the band on rank 0 (other ranks may pass AB = NULL); W_local on every rank (or NULL)
  int rc = validate(h, mode, n, b, nb, A, lda, lead ? AB : A, ldab < b + 1 && !lead ? b + 1 : ldab, W, ldw);
  if (rc != SBR_OK) return rc;
  if (h->nranks > 1) {
    if (!h->comm) return SBR_ERR_NCCL;
    // the tensor-core FP16 path with column blocks that align with the pass's tile groups and the
    // SYR2K's tiles (configs 4/5: nb = 1024 / 2048)
    // FP16: the pass's 128-row tile groups (pass_dist_align); 3xTF32: 128-column tiles, b % 4 == 0 and
    // a 16-byte aligned A; both: the SYR2K's 256-column tiles
    const bool ok16 = (mode == SBR_FP16_FP32ACC || mode == SBR_BF16_FP32ACC) && b % 8 == 0 && nb % pass_dist_align(b) == 0 && nb % 256 == 0;
    const bool ok32 = mode == SBR_3XTF32 && h->tf32_tc && b % 4 == 0 && nb % 256 == 0 && lda % 4 == 0 &&
                      ((uintptr_t)A & 15) == 0;
    if (!ok16 && !ok32) {
      std::lock_guard<std::mutex> lk(g_err_mu);
      g_last_err = "sbr_reduce_dist with nranks > 1: FP16 mode with b % 8 == 0 and nb a multiple of " +
                   std::to_string(pass_dist_align(b)) + ", or 3xTF32 with b % 4 == 0 and nb a multiple of 256";
      return SBR_ERR_UNSUPPORTED;
    }
  }
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  return reduce_device(h, mode, n, b, nb, A, lda, AB, ldab, W, ldw);
}

int sbr_rank(sbr_handle_t h) { return h ? h->rank : -1; }
int sbr_nranks(sbr_handle_t h) { return h ? h->nranks : -1; }

int sbr_sync(sbr_handle_t h) {
  if (!h) return -1;
  SBR_CK(cudaStreamSynchronize(h->stream), "sync");
  return poll_latched(h, true);
}

const char* sbr_status_string(int status) {
  static thread_local std::string s;
  switch (status) {
    case SBR_OK: return "ok";
    case SBR_ERR_NONFINITE: return "input contains Inf or NaN";
    case SBR_ERR_CUDA: {
      std::lock_guard<std::mutex> lk(g_err_mu);
      s = "CUDA error: " + g_last_err;
      return s.c_str();
    }
    case SBR_ERR_NCCL: return "NCCL error";
    case SBR_ERR_NOMEM: return "device out of memory";
    case SBR_ERR_UNSUPPORTED: return "unsupported argument combination";
    default:
      if (status < 0) {
        s = "invalid argument " + std::to_string(-status);
        return s.c_str();
      }
      return "unknown status";
  }
}

int sbr_generate_symmetric(sbr_handle_t h, uint64_t seed, int64_t n, float* A, int64_t lda) {
  if (!h) return -1;
  if (n < 0) return -3;
  if (!A) return -4;
  if (lda < std::max<int64_t>(1, n)) return -5;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  SBR_CK(gen_symmetric(seed, n, A, lda, h->stream), "gen_symmetric");
  h->launches += (n + 65534) / 65535;
  return SBR_OK;
}

int sbr_set_kernel_timing(sbr_handle_t h, int enable) {
  if (!h) return -1;
  h->timing = enable != 0;
  return SBR_OK;
}

int sbr_reset_kernel_stats(sbr_handle_t h) {
  if (!h) return -1;
  drain_stats(h);
  for (auto& s : h->stats) s = Stat();
  return SBR_OK;
}

int sbr_kernel_stats(sbr_handle_t h, int kid, int64_t* launches, double* ms, double* bytes, double* flops) {
  if (!h) return -1;
  if (kid < 0 || kid >= SBR_K_COUNT) return -2;
  drain_stats(h);
  const Stat& s = h->stats[kid];
  if (launches) *launches = s.launches;
  if (ms) *ms = s.ms;
  if (bytes) *bytes = s.bytes;
  if (flops) *flops = s.flops;
  return SBR_OK;
}

int64_t sbr_launch_count(sbr_handle_t h) { return h ? h->launches : -1; }

const char* sbr_version(void) { return "libsbr 0.1 sm_100a"; }

}  // extern "C"

// ====================================================================== test hooks
#include "../../include/sbr_testing.h"

namespace {

__global__ void f32cm_to_f16rm_kernel(int64_t rows, int cols, const float* src, int64_t lds, __half* dst,
                                      int64_t ldd) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < rows * cols;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = e / cols;
    const int c = (int)(e % cols);
    dst[r * ldd + c] = cvt16(src[r + c * lds]);
  }
}

__global__ void f16_to_f32_kernel(int64_t rows, int cols, const __half* src, int64_t lds, bool rowmajor, float* dst,
                                  int64_t ldd) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < rows * cols;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = e % rows;
    const int c = (int)(e / rows);
    dst[r + c * ldd] = from16(rowmajor ? src[r * lds + c] : src[r + c * lds]);
  }
}

struct DevBuf {
  void* p = nullptr;
  explicit DevBuf(size_t bytes) {
    if (cudaMalloc(&p, bytes) != cudaSuccess) p = nullptr;
  }
  ~DevBuf() {
    if (p) cudaFree(p);
  }
};

}  // namespace

extern "C" {

int sbr_test_pass_fp16_part(sbr_handle_t h, int64_t M, int b, int rank, int nranks, const float* OA, int64_t ldoa,
                            const float* W, int64_t ldw, float* X, int64_t ldx);

int sbr_test_pass_fp16(sbr_handle_t h, int64_t M, int b, const float* OA, int64_t ldoa, const float* W, int64_t ldw,
                       float* X, int64_t ldx) {
  return sbr_test_pass_fp16_part(h, M, b, 0, 1, OA, ldoa, W, ldw, X, ldx);
}

int sbr_test_pass_fp16_part(sbr_handle_t h, int64_t M, int b, int rank, int nranks, const float* OA, int64_t ldoa,
                            const float* W, int64_t ldw, float* X, int64_t ldx) {
  if (!h) return -1;
  if (nranks < 1 || rank < 0 || rank >= nranks) return -4;
  if (M < 1) return -2;
  if (b < 1 || b > 64) return -3;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  cudaStream_t st = h->stream;
  const int64_t ldwh = (M + 7) / 8 * 8;
  const int64_t ldsh = (M + 7) / 8 * 8;
  DevBuf sh(sizeof(__half) * ldsh * M), wh(sizeof(__half) * ldwh * 64);
  if (!sh.p || !wh.p) return SBR_ERR_NOMEM;
  SBR_CK(shadow_init(M, const_cast<float*>(OA), ldoa, (__half*)sh.p, ldsh, nullptr, st), "shadow");   // k = 0: read only
  SBR_CK(to_half_cm(M, b, pass_bn(b), W, ldw, (__half*)wh.p, ldwh, st), "W->fp16");
  SBR_CK(zero_matrix(M, b, X, ldx, st), "zero X");
  PassLaunch pl{};
  pl.shadow = (__half*)sh.p;
  pl.n = M;
  pl.ld_shadow = ldsh;
  pl.Wh = (__half*)wh.p;
  pl.M = M;
  pl.ld_wh = ldwh;
  pl.r0 = 0;
  pl.b = b;
  pl.X = X;
  pl.ldx = ldx;
  pl.num_sms = h->nsm;
  pl.seg_rows = 8;
  pl.rank = rank;
  pl.nranks = nranks;
  SBR_CK(launch_pass_tc(pl, st), "pass_tc");
  SBR_CK(cudaStreamSynchronize(st), "sync");
  return SBR_OK;
}

int sbr_test_syr2k_fp16(sbr_handle_t h, int64_t M, int K, const float* Y, int64_t ldy, const float* Z, int64_t ldz,
                        float* C, int64_t ldc, float* S, int64_t lds) {
  if (!h) return -1;
  if (M < 1) return -2;
  if (K < 1) return -3;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  cudaStream_t st = h->stream;
  const int64_t kp = (K + 7) / 8 * 8;
  const int64_t ldsh = (M + 7) / 8 * 8;
  DevBuf yh(sizeof(__half) * M * kp), zh(sizeof(__half) * M * kp), sh(sizeof(__half) * ldsh * M);
  if (!yh.p || !zh.p || !sh.p) return SBR_ERR_NOMEM;
  SBR_CK(cudaMemsetAsync(sh.p, 0, sizeof(__half) * ldsh * M, st), "memset");
  f32cm_to_f16rm_kernel<<<256, 256, 0, st>>>(M, K, Y, ldy, (__half*)yh.p, kp);
  f32cm_to_f16rm_kernel<<<256, 256, 0, st>>>(M, K, Z, ldz, (__half*)zh.p, kp);
  GemmTcLaunch gs{};
  gs.A0 = (__half*)yh.p;
  gs.A1 = (__half*)zh.p;
  gs.B0 = (__half*)zh.p;
  gs.B1 = (__half*)yh.p;
  gs.K = K;
  gs.a_rows = gs.b_rows = M;
  gs.ld_a = gs.ld_b = kp;
  gs.arow0 = gs.brow0 = 0;
  gs.Mrows = gs.Ncols = M;
  gs.C = C;
  gs.ldc = ldc;
  gs.shadow = (__half*)sh.p;
  gs.ld_shadow = ldsh;
  gs.num_sms = h->nsm;
  SBR_CK(launch_syr2k_tc(gs, st), "syr2k_tc");
  if (S) f16_to_f32_kernel<<<256, 256, 0, st>>>(M, (int)M, (__half*)sh.p, ldsh, false, S, lds);
  SBR_CK(cudaStreamSynchronize(st), "sync");
  return SBR_OK;
}

int sbr_test_zform_fp16(sbr_handle_t h, int64_t M, int K, const float* Y, int64_t ldy, const float* G, int64_t ldg,
                        const float* X, int64_t ldx, float* Z, int64_t ldz) {
  if (!h) return -1;
  if (M < 1) return -2;
  if (K < 1) return -3;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  cudaStream_t st = h->stream;
  const int64_t kp = (K + 7) / 8 * 8;
  DevBuf yh(sizeof(__half) * M * kp), gh(sizeof(__half) * K * kp), zh(sizeof(__half) * M * kp);
  if (!yh.p || !gh.p || !zh.p) return SBR_ERR_NOMEM;
  f32cm_to_f16rm_kernel<<<256, 256, 0, st>>>(M, K, Y, ldy, (__half*)yh.p, kp);
  f32cm_to_f16rm_kernel<<<256, 256, 0, st>>>(K, K, G, ldg, (__half*)gh.p, kp);
  GemmTcLaunch gz{};
  gz.A0 = gz.A1 = (__half*)yh.p;
  gz.B0 = gz.B1 = (__half*)gh.p;
  gz.K = K;
  gz.a_rows = M;
  gz.ld_a = kp;
  gz.b_rows = K;
  gz.ld_b = kp;
  gz.Mrows = M;
  gz.Ncols = K;
  gz.X = X;
  gz.ldx = ldx;
  gz.Zh = (__half*)zh.p;
  gz.ldz = kp;
  gz.num_sms = h->nsm;
  SBR_CK(launch_zform_tc(gz, st), "zform_tc");
  f16_to_f32_kernel<<<256, 256, 0, st>>>(M, K, (__half*)zh.p, kp, true, Z, ldz);
  SBR_CK(cudaStreamSynchronize(st), "sync");
  return SBR_OK;
}

int sbr_test_pass_tf32(sbr_handle_t h, int64_t M, int b, const float* OA, int64_t ldoa, const float* S,
                       int64_t lds, int64_t sw, const float* W, int64_t ldw, float* X, int64_t ldx) {
  if (!h) return -1;
  if (M < 1) return -2;
  if (b < 1 || b > 64) return -3;
  if (ldoa < M || ldoa % 4 != 0) return -5;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  cudaStream_t st = h->stream;
  const int64_t ldws = (M + 3) / 4 * 4;
  DevBuf ws(sizeof(float) * ldws * 64);
  if (!ws.p) return SBR_ERR_NOMEM;
  SBR_CK(zero_matrix(M, b, X, ldx, st), "zero X");
  for (int c = 0; c < b; c += 32) {
    const int bh = std::min(32, b - c);
    SBR_CK(split_tf32_w(M, bh, 32, W + c * ldw, ldw, (float*)ws.p, ldws, st), "split W");
    PassTf32Launch pl{};
    pl.A = OA;
    pl.n = M;
    pl.lda = ldoa;
    pl.r0 = 0;
    pl.S = S;
    pl.lds = lds;
    pl.sw = S ? sw : 0;
    pl.WS = (float*)ws.p;
    pl.ldws = ldws;
    pl.M = M;
    pl.b = bh;
    pl.X = X + c * ldx;
    pl.ldx = ldx;
    pl.num_sms = h->nsm;
    SBR_CK(launch_pass_tf32(pl, st), "pass_tf32");
  }
  SBR_CK(cudaStreamSynchronize(st), "sync");
  return SBR_OK;
}

int sbr_test_syr2k_tf32(sbr_handle_t h, int64_t M, int K, const float* Y, int64_t ldy, const float* Z, int64_t ldz,
                        float* C, int64_t ldc) {
  if (!h) return -1;
  if (M < 1) return -2;
  if (K < 1) return -3;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  cudaStream_t st = h->stream;
  const int64_t lo = (K + 31) / 32 * 32, ld = 2 * lo;
  DevBuf ys(sizeof(float) * M * ld), zs(sizeof(float) * M * ld);
  if (!ys.p || !zs.p) return SBR_ERR_NOMEM;
  SBR_CK(split_tf32_rm(M, K, Y, ldy, (float*)ys.p, ld, lo, st), "split Y");
  SBR_CK(split_tf32_rm(M, K, Z, ldz, (float*)zs.p, ld, lo, st), "split Z");
  GemmTcLaunch gs{};
  gs.A0 = (const __half*)ys.p;
  gs.A1 = (const __half*)zs.p;
  gs.B0 = (const __half*)zs.p;
  gs.B1 = (const __half*)ys.p;
  gs.K = K;
  gs.lo_off = lo;
  gs.a_rows = gs.b_rows = M;
  gs.ld_a = gs.ld_b = ld;
  gs.Mrows = gs.Ncols = M;
  gs.C = C;
  gs.ldc = ldc;
  gs.num_sms = h->nsm;
  SBR_CK(launch_syr2k_tf32(gs, st), "syr2k_tf32");
  SBR_CK(cudaStreamSynchronize(st), "sync");
  return SBR_OK;
}

int sbr_test_zform_tf32(sbr_handle_t h, int64_t M, int K, const float* Y, int64_t ldy, const float* G, int64_t ldg,
                        const float* X, int64_t ldx, float* Z, int64_t ldz) {
  if (!h) return -1;
  if (M < 1) return -2;
  if (K < 1) return -3;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  cudaStream_t st = h->stream;
  const int64_t lo = (K + 31) / 32 * 32, ld = 2 * lo;
  DevBuf ys(sizeof(float) * M * ld), gs_(sizeof(float) * K * ld), zs(sizeof(float) * M * ld);
  if (!ys.p || !gs_.p || !zs.p) return SBR_ERR_NOMEM;
  SBR_CK(split_tf32_rm(M, K, Y, ldy, (float*)ys.p, ld, lo, st), "split Y");
  SBR_CK(split_tf32_rm(K, K, G, ldg, (float*)gs_.p, ld, lo, st), "split G");
  GemmTcLaunch gz{};
  gz.A0 = gz.A1 = (const __half*)ys.p;
  gz.B0 = gz.B1 = (const __half*)gs_.p;
  gz.K = K;
  gz.lo_off = lo;
  gz.a_rows = M;
  gz.ld_a = ld;
  gz.b_rows = K;
  gz.ld_b = ld;
  gz.Mrows = M;
  gz.Ncols = K;
  gz.X = X;
  gz.ldx = ldx;
  gz.Zs = (float*)zs.p;
  gz.ldz = ld;
  gz.num_sms = h->nsm;
  SBR_CK(launch_zform_tf32(gz, st), "zform_tf32");
  // Z = hi + lo back to column-major fp32
  SBR_CK(splitsum_rm_to_cm(M, K, (const float*)zs.p, ld, lo, Z, ldz, st), "Z unsplit");
  SBR_CK(cudaStreamSynchronize(st), "sync");
  return SBR_OK;
}

}  // extern "C"

extern "C" int sbr_test_panel(sbr_handle_t h, int64_t m, int b, float* P, int64_t ldp, float* Y, float* W,
                              int64_t ldyw, int64_t* trace_host) {
  if (!h) return -1;
  if (m < 1) return -2;
  if (b < 1 || b > 64) return -3;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  int rc = ensure_ws(h, m + b, b, b, 0, nullptr);
  if (rc != SBR_OK) return rc;
  cudaStream_t st = h->stream;
  DevBuf tr(trace_host ? sizeof(int64_t) * 16 : 0);
  if (trace_host) {
    if (!tr.p) return SBR_ERR_NOMEM;
    SBR_CK(cudaMemsetAsync(tr.p, 0, sizeof(int64_t) * 16, st), "memset");
  }
  PanelArgs pa{};
  pa.P = P;
  pa.ldp = ldp;
  pa.m = (int)m;
  pa.b = b;
  pa.Y = Y;
  pa.ldy = ldyw;
  pa.W = W;
  pa.ldw = ldyw;
  pa.row0 = 0;
  pa.M = m;
  pa.ws_v = h->pv;
  pa.ws_tau = h->ptau;
  pa.ws_r = h->pr;
  pa.ws_q = h->pq;
  pa.ws_misc = h->pmisc;
  pa.trace = trace_host ? (int64_t*)tr.p : nullptr;
  bool chol = false;
  if (h->panel_mode == 0 && m > 512) {
    const cudaError_t ce = launch_panel_chol(pa, h->chol_ws, h->chol_launches, st);
    if (ce == cudaSuccess) {
      h->chol_launches++;
      chol = true;
    } else if (ce != cudaErrorNotSupported) {
      SBR_CK(ce, "panel_chol");
    }
  }
  if (!chol) {
    const cudaError_t te = launch_panel(pa, h->panel_ctas, st);
    SBR_CK(te, "panel");
    if (pa.over_capacity) return SBR_ERR_UNSUPPORTED;
  }
  if (trace_host) {
    SBR_CK(cudaMemcpyAsync(trace_host, tr.p, sizeof(int64_t) * 16, cudaMemcpyDeviceToHost, st), "trace D2H");
    SBR_CK(cudaStreamSynchronize(st), "sync");
  }
  return SBR_OK;
}

// Per-panel phase trace of the reduction: arm (cap > 0: the next cap CholeskyQR panels of
// sbr_reduce record their 16 globaltimer stamps), then read (host != NULL: copies the stamps
// of the recorded panels, returns their count in *count).  Diagnostic only.
extern "C" int sbr_test_panel_trace(sbr_handle_t h, int cap, int64_t* host, int* count) {
  if (!h) return -1;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  if (cap > 0) {
    if (h->ptrace) cudaFree(h->ptrace);
    h->ptrace = nullptr;
    SBR_CK(cudaMalloc(&h->ptrace, sizeof(int64_t) * 32 * (size_t)cap), "trace alloc");
    SBR_CK(cudaMemsetAsync(h->ptrace, 0, sizeof(int64_t) * 32 * (size_t)cap, h->stream), "trace memset");
    h->ptrace_cap = cap;
    h->ptrace_used = 0;
  }
  if (host) {
    if (!count) return -4;
    SBR_CK(cudaStreamSynchronize(h->stream), "sync");
    *count = h->ptrace_used;
    if (h->ptrace_used > 0)
      SBR_CK(cudaMemcpy(host, h->ptrace, sizeof(int64_t) * 32 * (size_t)h->ptrace_used, cudaMemcpyDeviceToHost),
             "trace D2H");
  }
  return SBR_OK;
}

// Declined CholeskyQR panels (TSQR fallback taken) since the last call with reset != 0.
extern "C" int sbr_test_panel_declines(sbr_handle_t h, int reset, int64_t* count) {
  if (!h) return -1;
  if (!count) return -3;
  *count = 0;
  if (!h->chol_ws) return SBR_OK;
  SBR_CK(cudaSetDevice(h->device), "cudaSetDevice");
  unsigned v = 0;
  SBR_CK(cudaMemcpyAsync(&v, panel_chol_declines(h->chol_ws), sizeof(unsigned), cudaMemcpyDeviceToHost, h->stream),
         "declines D2H");
  SBR_CK(cudaStreamSynchronize(h->stream), "sync");
  *count = v;
  if (reset) SBR_CK(cudaMemsetAsync(panel_chol_declines(h->chol_ws), 0, sizeof(unsigned), h->stream), "reset");
  return SBR_OK;
}

namespace sbr { void set_knob(int k, int v); }
extern "C" int sbr_test_set_knob(int k, int value) {
  if (k < 0 || k >= sbr::KNOB_COUNT) return -1;
  sbr::set_knob(k, value);
  return SBR_OK;
}

// host-only: the pass's tile share of `rank` (test hook for the multi-GPU partition)
extern "C" int sbr_test_pass_partition(int64_t M, int b, int rank, int nranks, int64_t* t0, int64_t* t1,
                                       int64_t* total) {
  if (M < 1) return -1;
  if (b < 1 || b > 64) return -2;
  if (nranks < 1 || rank < 0 || rank >= nranks) return -3;
  if (!t0 || !t1 || !total) return -5;
  pass_partition(M, b, rank, nranks, t0, t1, total);
  return SBR_OK;
}

// host-only: the pass tiles `rank` of `nranks` walks for block origin c0 in sbr_reduce_dist
extern "C" int64_t sbr_test_pass_owned_tiles(int64_t n, int b, int nb, int64_t c0, int rank, int nranks, int* IJ,
                                             int64_t cap) {
  if (n < 1 || b < 1 || b > 64 || nb < b || nranks < 1 || rank < 0 || rank >= nranks || c0 < 0 || c0 + b >= n) return -1;
  return pass_owned_tiles(n - c0 - b, b, c0, b, nb, nranks, rank, IJ, cap);
}

// host-only: (I, J) tile coordinates of tiles [t0, t1) in the pass's order, IJ[2k], IJ[2k+1]
extern "C" int sbr_test_pass_tiles(int64_t M, int b, int64_t t0, int64_t t1, int* IJ) {
  if (M < 1) return -1;
  if (b < 1 || b > 64) return -2;
  if (t0 < 0 || t1 < t0) return -3;
  if (!IJ && t1 > t0) return -5;
  pass_tiles(M, b, t0, t1, IJ);
  return SBR_OK;
}

namespace sbr {
SBR_OP16_SETTER(api)
cudaError_t set_op16_all(int bf16, cudaStream_t st) {
  for (auto f : {set_op16_chain, set_op16_gemm, set_op16_misc, set_op16_panel, set_op16_chol, set_op16_skinny,
                 set_op16_pass, set_op16_api}) {
    const cudaError_t e = f(bf16, st);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}
}  // namespace sbr
