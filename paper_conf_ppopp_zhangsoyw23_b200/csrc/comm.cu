// comm.cu -- NCCL and in-process ("local") implementations of comm.h.
#include <condition_variable>
#include <map>
#include <memory>
#include <mutex>
#include <vector>

#include "comm.h"
#include "nccl_rt.h"

namespace sbr {

// ------------------------------------------------------------------------------ NCCL
namespace {
constexpr int kNcclFloat64 = 8;

class NcclComm : public Comm {
 public:
  NcclComm(nccl::Comm c, int rank, int n) : c_(c), rank_(rank), n_(n) {}
  ~NcclComm() override {
    if (c_) nccl::comm_destroy(c_);
  }
  int broadcast(void* buf, size_t bytes, int root, cudaStream_t st) override {
    return check(nccl::broadcast(buf, bytes, nccl::kUint8, root, c_, st), "ncclBroadcast");
  }
  int all_reduce_sum_f32(float* buf, size_t count, cudaStream_t st) override {
    return check(nccl::all_reduce_sum_f32(buf, count, c_, st), "ncclAllReduce");
  }
  int all_reduce_sum_f64(double* buf, size_t count, cudaStream_t st) override {
    return check(nccl::all_reduce_sum(buf, count, kNcclFloat64, c_, st), "ncclAllReduce");
  }
  int rank() const override { return rank_; }
  int size() const override { return n_; }
  const char* kind() const override { return "nccl"; }

 private:
  int check(int r, const char* what) {
    if (r != 0) err_ = std::string(what) + ": " + nccl::error_string(r);
    return r;
  }
  nccl::Comm c_;
  int rank_, n_;
};
}  // namespace

Comm* make_nccl_comm(const void* unique_id, int rank, int nranks, std::string* msg) {
  if (const char* e = nccl::load()) {
    *msg = e;
    return nullptr;
  }
  nccl::UniqueId u;
  memcpy(&u, unique_id, sizeof(u));
  nccl::Comm c = nullptr;
  const int r = nccl::comm_init_rank(&c, nranks, u, rank);
  if (r != 0) {
    *msg = std::string("ncclCommInitRank: ") + nccl::error_string(r);
    return nullptr;
  }
  return new NcclComm(c, rank, nranks);
}

// ------------------------------------------------------------------------------ local
namespace {

constexpr int kMaxLocal = 16;

template <typename T>
struct Ptrs {
  const T* p[kMaxLocal];
};

template <typename T>
__global__ void sum_ranks_kernel(Ptrs<T> src, int n, size_t count, T* dst) {
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (size_t)gridDim.x * blockDim.x) {
    T s = 0;
    for (int r = 0; r < n; ++r) s += src.p[r][i];   // same order on every rank: identical sums
    dst[i] = s;
  }
}

struct Slot {
  void* buf = nullptr;
  int device = 0;
  cudaEvent_t ready = nullptr, done = nullptr;
  void* tmp = nullptr;
  size_t tmp_bytes = 0;
};

struct Group {
  int n = 0;
  std::mutex mu;
  std::condition_variable cv;
  int count = 0;
  long generation = 0;
  Slot slots[kMaxLocal];
  int members = 0;
  void barrier() {
    std::unique_lock<std::mutex> lk(mu);
    const long gen = generation;
    if (++count == n) {
      count = 0;
      ++generation;
      cv.notify_all();
    } else {
      cv.wait(lk, [&] { return generation != gen; });
    }
  }
};

std::mutex g_groups_mu;
std::map<int, std::shared_ptr<Group>> g_groups;

class LocalComm : public Comm {
 public:
  LocalComm(std::shared_ptr<Group> g, int key, int rank) : g_(std::move(g)), key_(key), rank_(rank) {
    Slot& s = g_->slots[rank_];
    cudaGetDevice(&s.device);
    cudaEventCreateWithFlags(&s.ready, cudaEventDisableTiming);
    cudaEventCreateWithFlags(&s.done, cudaEventDisableTiming);
  }
  ~LocalComm() override {
    Slot& s = g_->slots[rank_];
    if (s.ready) cudaEventDestroy(s.ready);
    if (s.done) cudaEventDestroy(s.done);
    if (s.tmp) cudaFree(s.tmp);
    s = Slot();
    std::lock_guard<std::mutex> lk(g_groups_mu);
    if (--g_->members == 0) g_groups.erase(key_);
  }
  int broadcast(void* buf, size_t bytes, int root, cudaStream_t st) override {
    Slot& me = g_->slots[rank_];
    me.buf = buf;
    if (int r = ck(cudaEventRecord(me.ready, st))) return r;
    g_->barrier();
    int rc = 0;
    if (rank_ != root) {
      Slot& rs = g_->slots[root];
      rc = ck(cudaStreamWaitEvent(st, rs.ready, 0));
      if (!rc) rc = ck(cudaMemcpyAsync(buf, rs.buf, bytes, cudaMemcpyDefault, st));
      if (!rc) rc = ck(cudaEventRecord(me.done, st));
    }
    g_->barrier();
    if (rank_ == root && !rc)
      for (int q = 0; q < g_->n && !rc; ++q)
        if (q != root) rc = ck(cudaStreamWaitEvent(st, g_->slots[q].done, 0));   // buf stays until copied
    g_->barrier();
    return rc;
  }
  int all_reduce_sum_f32(float* buf, size_t count, cudaStream_t st) override { return all_reduce(buf, count, st); }
  int all_reduce_sum_f64(double* buf, size_t count, cudaStream_t st) override { return all_reduce(buf, count, st); }
  int rank() const override { return rank_; }
  int size() const override { return g_->n; }
  const char* kind() const override { return "local"; }

 private:
  template <typename T>
  int all_reduce(T* buf, size_t count, cudaStream_t st) {
    Slot& me = g_->slots[rank_];
    const size_t bytes = count * sizeof(T);
    if (me.tmp_bytes < bytes) {
      if (me.tmp) cudaFree(me.tmp);
      me.tmp = nullptr;
      me.tmp_bytes = 0;
      if (int r = ck(cudaMalloc(&me.tmp, bytes))) return r;
      me.tmp_bytes = bytes;
    }
    me.buf = buf;
    int rc = ck(cudaEventRecord(me.ready, st));
    g_->barrier();
    Ptrs<T> src{};
    for (int q = 0; q < g_->n; ++q) {
      src.p[q] = static_cast<const T*>(g_->slots[q].buf);
      if (!rc) rc = ck(cudaStreamWaitEvent(st, g_->slots[q].ready, 0));
    }
    if (!rc && count) {
      const int blocks = (int)std::min<size_t>((count + 255) / 256, 1184);
      sum_ranks_kernel<T><<<blocks, 256, 0, st>>>(src, g_->n, count, static_cast<T*>(me.tmp));
      rc = ck(cudaGetLastError());
    }
    if (!rc) rc = ck(cudaEventRecord(me.done, st));
    g_->barrier();
    for (int q = 0; q < g_->n && !rc; ++q) rc = ck(cudaStreamWaitEvent(st, g_->slots[q].done, 0));
    if (!rc && count) rc = ck(cudaMemcpyAsync(buf, me.tmp, bytes, cudaMemcpyDeviceToDevice, st));
    g_->barrier();
    return rc;
  }
  int ck(cudaError_t e) {
    if (e == cudaSuccess) return 0;
    err_ = std::string("local comm: ") + cudaGetErrorString(e);
    return (int)e;
  }
  std::shared_ptr<Group> g_;
  int key_, rank_;
};

}  // namespace

Comm* make_local_comm(int key, int rank, int nranks, std::string* msg) {
  if (nranks < 1 || nranks > kMaxLocal) {
    *msg = "local communicator: 1 <= nranks <= 16";
    return nullptr;
  }
  std::shared_ptr<Group> g;
  {
    std::lock_guard<std::mutex> lk(g_groups_mu);
    auto it = g_groups.find(key);
    if (it == g_groups.end()) {
      g = std::make_shared<Group>();
      g->n = nranks;
      g_groups[key] = g;
    } else {
      g = it->second;
      if (g->n != nranks) {
        *msg = "local communicator: nranks differs from the group's";
        return nullptr;
      }
    }
    ++g->members;
  }
  return new LocalComm(g, key, rank);
}

}  // namespace sbr
