// nccl_rt.cu -- minimal runtime binding to NCCL (dlopen): the multi-GPU path of libsbr
// needs only unique-id creation, communicator init/destroy, all-reduce and
// broadcast.  Loading at run time keeps libsbr linkable and loadable on hosts without NCCL
// (the single-GPU path never touches it) and reuses the NCCL already loaded by the process
// (torch's wheel) instead of pulling in a second copy.
#include <dlfcn.h>

#include <mutex>

#include "nccl_rt.h"

namespace sbr {
namespace nccl {

namespace {
struct Api {
  bool loaded = false;
  std::string err;
  int (*getUniqueId)(UniqueId*) = nullptr;
  int (*commInitRank)(Comm*, int, UniqueId, int) = nullptr;
  int (*commDestroy)(Comm) = nullptr;
  int (*allReduce)(const void*, void*, size_t, int, int, Comm, cudaStream_t) = nullptr;
  int (*broadcast)(const void*, void*, size_t, int, int, Comm, cudaStream_t) = nullptr;
  const char* (*getErrorString)(int) = nullptr;
};
Api g_api;
std::mutex g_mu;

template <typename F>
bool sym(void* h, const char* name, F& out) {
  out = reinterpret_cast<F>(dlsym(h, name));
  return out != nullptr;
}
}  // namespace

const char* load(void) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (g_api.loaded) return nullptr;
  void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);   // the copy already in the process, if any
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) {
    g_api.err = std::string("cannot load libnccl.so.2: ") + dlerror();
    return g_api.err.c_str();
  }
  bool ok = sym(h, "ncclGetUniqueId", g_api.getUniqueId) && sym(h, "ncclCommInitRank", g_api.commInitRank) &&
            sym(h, "ncclCommDestroy", g_api.commDestroy) && sym(h, "ncclAllReduce", g_api.allReduce) &&
            sym(h, "ncclBroadcast", g_api.broadcast) && sym(h, "ncclGetErrorString", g_api.getErrorString);
  if (!ok) {
    g_api.err = "libnccl.so.2 lacks a required symbol";
    return g_api.err.c_str();
  }
  g_api.loaded = true;
  return nullptr;
}

const char* error_string(int r) { return g_api.getErrorString ? g_api.getErrorString(r) : "NCCL not loaded"; }
int get_unique_id(UniqueId* id) { return g_api.getUniqueId(id); }
int comm_init_rank(Comm* c, int nranks, const UniqueId& id, int rank) { return g_api.commInitRank(c, nranks, id, rank); }
int comm_destroy(Comm c) { return g_api.commDestroy(c); }
int all_reduce_sum_f32(float* buf, size_t count, Comm c, cudaStream_t st) {
  return g_api.allReduce(buf, buf, count, kFloat32, kSum, c, st);
}
int all_reduce_sum(void* buf, size_t count, int dtype, Comm c, cudaStream_t st) {
  return g_api.allReduce(buf, buf, count, dtype, kSum, c, st);
}
int broadcast(void* buf, size_t count, int dtype, int root, Comm c, cudaStream_t st) {
  return g_api.broadcast(buf, buf, count, dtype, root, c, st);
}

}  // namespace nccl
}  // namespace sbr
