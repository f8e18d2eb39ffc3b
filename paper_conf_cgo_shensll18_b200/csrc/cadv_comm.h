// cadv_comm.h — collectives used by multi-rank contexts (comm.cpp).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>

namespace cadv {

// All calls are collective (every rank, same order) and stream-ordered on
// `s`; they return 0 on success, else 1 with `err` set.  Device buffers.
class Comm {
 public:
  Comm(int r, int n) : rank(r), nranks(n) {}
  virtual ~Comm() {}
  virtual int allreduce_sum_u64(uint64_t* d, size_t n, cudaStream_t s) = 0;  // in place
  virtual int allreduce_max_u32(uint32_t* d, size_t n, cudaStream_t s) = 0;  // in place
  // recv = nranks * bytes, rank p's contribution at p * bytes
  virtual int allgather(const void* send, void* recv, size_t bytes, cudaStream_t s) = 0;
  // bytes [soff[p], soff[p] + scnt[p]) of send go to rank p, which receives
  // them at its roff[me]; rcnt[p] = what p sends here (host arrays of nranks)
  virtual int alltoallv(const void* send, const uint64_t* soff, const uint64_t* scnt, void* recv,
                        const uint64_t* roff, const uint64_t* rcnt, cudaStream_t s) = 0;
  // Peer memory: every rank passes the base of one of its device allocations
  // (slot = which of the caller's buffers); peers[p] = rank p's allocation
  // mapped into this process (CUDA IPC over NVLink for NCCL contexts, plain
  // pointers for in-process loopback ranks), so kernels can store into it.
  // Mappings are cached per (slot, peer) and reopened when a peer reallocates.
  virtual int map_peers(int slot, void* local, void** peers, cudaStream_t s) = 0;
  // All ranks reach this point with their queued work complete.
  virtual int barrier(cudaStream_t s) = 0;
  const int rank, nranks;
  std::string err;
};

struct LoopbackGroup;
LoopbackGroup* loopback_group_new(int nranks);
void loopback_group_delete(LoopbackGroup* g);
int loopback_group_size(const LoopbackGroup* g);
Comm* make_loopback_comm(LoopbackGroup* g, int rank);
Comm* make_nccl_comm(const void* id128, int rank, int nranks, std::string* err);
int nccl_unique_id(void* out128, std::string* err);

}  // namespace cadv
