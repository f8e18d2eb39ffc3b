// cadv_comm.h — collectives used by multi-rank contexts (comm.cpp).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

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

// CUDA IPC shares whole driver allocations: cudaIpcGetMemHandle(p) names the
// allocation that CONTAINS p (small cudaMallocs may share one), and
// cudaIpcOpenMemHandle maps it once per process, returning its base.  So a
// peer publishes (handle, p - base) and the importer opens every handle once.
struct IpcRef {
  cudaIpcMemHandle_t h;
  uint64_t offset;  // of the published pointer inside the allocation
};
int ipc_export(void* p, IpcRef* out, std::string* err);
class IpcCache {
 public:
  ~IpcCache();
  // the peer pointer for r (the allocation mapped on first use); null on error
  void* open(const IpcRef& r, std::string* err);

 private:
  struct Entry {
    cudaIpcMemHandle_t h;
    void* base;
  };
  std::vector<Entry> open_;
};

// Host-side exchange of small blobs between the ranks (handles, offsets,
// barriers) for the peer backend: a TCP star through rank 0 (one process per
// rank) or the in-process loopback group (thread ranks).
class Bootstrap {
 public:
  Bootstrap(int r, int n) : rank(r), nranks(n) {}
  virtual ~Bootstrap() {}
  // every rank contributes `bytes`; out = nranks * bytes in rank order; 0 = ok
  virtual int allgather(const void* in, void* out, size_t bytes) = 0;
  int barrier() {
    char c = 0;
    std::vector<char> v((size_t)nranks);
    return allgather(&c, v.data(), 1);
  }
  const int rank, nranks;
};
Bootstrap* make_tcp_bootstrap(const char* addr, int rank, int nranks, int timeout_s, std::string* err);

// The library's own collectives over peer device memory (comm_peer.cu): data
// is staged in device buffers and read by the peers' kernels through CUDA IPC
// mappings (or plain pointers for same-process ranks); the bootstrap carries
// only handles, offsets and barriers.
class PeerComm : public Comm {
 public:
  PeerComm(Bootstrap* b, bool owns, bool same_process);
  ~PeerComm() override;
  int allreduce_sum_u64(uint64_t* d, size_t n, cudaStream_t s) override;
  int allreduce_max_u32(uint32_t* d, size_t n, cudaStream_t s) override;
  int allgather(const void* send, void* recv, size_t bytes, cudaStream_t s) override;
  int alltoallv(const void* send, const uint64_t* soff, const uint64_t* scnt, void* recv, const uint64_t* roff,
                const uint64_t* rcnt, cudaStream_t s) override;
  int map_peers(int slot, void* local, void** peers, cudaStream_t s) override;
  int barrier(cudaStream_t s) override;

 private:
  template <typename T, bool SUM>
  int reduce(T* d, size_t n, cudaStream_t s);
  int stage_in(const void* d, size_t bytes, cudaStream_t s);
  int exchange(int slot, void* local, const void* extra, size_t extra_bytes, void** peers,
               std::vector<uint8_t>* all_extra);
  int grow(void** buf, size_t* cap, size_t bytes);
  int finish(int e);
  int cu(cudaError_t e);
  int boot(int e);
  Bootstrap* boot_;
  bool owns_, same_process_;
  void* stage_ = nullptr;
  size_t stage_cap_ = 0;
  void* tmp_ = nullptr;
  std::vector<void*> graveyard_;
  IpcCache ipc_;
};
Comm* make_peer_comm(const char* addr, int rank, int nranks, std::string* err);

struct LoopbackGroup;
LoopbackGroup* loopback_group_new(int nranks);
void loopback_group_delete(LoopbackGroup* g);
int loopback_group_size(const LoopbackGroup* g);
Comm* make_loopback_comm(LoopbackGroup* g, int rank);
Comm* make_nccl_comm(const void* id128, int rank, int nranks, std::string* err);
int nccl_unique_id(void* out128, std::string* err);

}  // namespace cadv
