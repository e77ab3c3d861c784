// nccl_rt.h -- the few NCCL entry points libsbr uses, resolved with dlopen (nccl_rt.cu).
// Types and enum values follow nccl.h (NCCL 2.x C ABI).
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>

#include <string>

namespace sbr {
namespace nccl {

struct UniqueId {
  char internal[128];
};
typedef struct ncclComm* Comm;

constexpr int kFloat16 = 6;   // ncclFloat16
constexpr int kFloat32 = 7;   // ncclFloat32
constexpr int kUint8 = 1;     // ncclUint8
constexpr int kSum = 0;       // ncclSum

const char* load(void);       // nullptr on success, else a message
const char* error_string(int r);
int get_unique_id(UniqueId* id);
int comm_init_rank(Comm* c, int nranks, const UniqueId& id, int rank);
int comm_destroy(Comm c);
int all_reduce_sum_f32(float* buf, size_t count, Comm c, cudaStream_t st);   // in place
int all_reduce_sum(void* buf, size_t count, int dtype, Comm c, cudaStream_t st);   // in place
int broadcast(void* buf, size_t count, int dtype, int root, Comm c, cudaStream_t st);   // in place

}  // namespace nccl
}  // namespace sbr
