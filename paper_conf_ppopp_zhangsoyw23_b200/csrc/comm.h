// comm.h -- the collectives of the multi-GPU reduction (sbr_reduce_dist).
//
// Two implementations behind one interface, both stream-ordered on the caller's stream:
//   * NCCL (one process per GPU, communicator from a unique id; NVLink / NVSwitch), and
//   * "local": P ranks that are handles in ONE process (one host thread each, any devices
//     including the same one), exchanging through device memory with host-side barriers.
//     This is how the sharded reduction is exercised on a single B200 (tests), and it runs the
//     very same kernels and call sequence as NCCL ranks.
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>

#include <string>

namespace sbr {

class Comm {
 public:
  virtual ~Comm() {}
  // in place; 0 = ok, otherwise an error (message in err())
  virtual int broadcast(void* buf, size_t bytes, int root, cudaStream_t st) = 0;
  virtual int all_reduce_sum_f32(float* buf, size_t count, cudaStream_t st) = 0;
  virtual int all_reduce_sum_f64(double* buf, size_t count, cudaStream_t st) = 0;
  virtual int rank() const = 0;
  virtual int size() const = 0;
  virtual const char* kind() const = 0;
  const std::string& err() const { return err_; }

 protected:
  std::string err_;
};

// NCCL communicator (rank / nranks from a 128-byte unique id); nullptr + *msg on failure
Comm* make_nccl_comm(const void* unique_id, int rank, int nranks, std::string* msg);
// in-process group `key` of nranks handles (every rank must create its Comm with the same key)
Comm* make_local_comm(int key, int rank, int nranks, std::string* msg);

}  // namespace sbr
