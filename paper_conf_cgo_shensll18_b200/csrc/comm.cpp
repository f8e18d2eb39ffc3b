// comm.cpp — the collectives of a multi-rank context.
//
// Two backends behind one small interface:
//   NCCL      one process per GPU (the product path).  libnccl is opened with
//             dlopen at cadv_create time, preferring the copy the process has
//             already loaded (torch's), so libcadv has no link-time NCCL
//             dependency and there is one NCCL per process.
//   loopback  N ranks = N threads of one process (tests on a single GPU):
//             the peer backend's device kernels (comm_peer.cu) over the
//             ranks' buffers, with the group's host barrier as bootstrap.
//             Same call sequence as NCCL, so the analysis code that drives
//             the collectives is the one the NCCL path runs.
// (A third backend, peer over TCP bootstrap + CUDA IPC, is in comm_peer.cu.)
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>
#include <string.h>

#include <condition_variable>
#include <mutex>
#include <string>
#include <vector>

#include "cadv_comm.h"

namespace cadv {

// ------------------------------------------------------------------ NCCL
namespace {

struct NcclApi {
  void* lib = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

std::mutex g_nccl_mu;
NcclApi g_nccl;

bool load_nccl(std::string* err) {
  std::lock_guard<std::mutex> lk(g_nccl_mu);
  if (g_nccl.lib) return true;
  void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);  // the process's NCCL (e.g. torch's)
  if (!h) {
    const char* p = getenv("CADV_NCCL_LIB");
    h = dlopen(p ? p : "libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  }
  if (!h) {
    *err = std::string("cannot load libnccl.so.2: ") + dlerror();
    return false;
  }
  NcclApi a;
  a.lib = h;
#define SYM(f, name)                                                  \
  *(void**)&a.f = dlsym(h, name);                                     \
  if (!a.f) {                                                         \
    *err = std::string("libnccl lacks ") + name;                      \
    return false;                                                     \
  }
  SYM(GetUniqueId, "ncclGetUniqueId");
  SYM(CommInitRank, "ncclCommInitRank");
  SYM(CommDestroy, "ncclCommDestroy");
  SYM(AllReduce, "ncclAllReduce");
  SYM(AllGather, "ncclAllGather");
  SYM(Send, "ncclSend");
  SYM(Recv, "ncclRecv");
  SYM(GroupStart, "ncclGroupStart");
  SYM(GroupEnd, "ncclGroupEnd");
  SYM(GetErrorString, "ncclGetErrorString");
#undef SYM
  g_nccl = a;
  return true;
}

class NcclComm : public Comm {
 public:
  NcclComm(int rank, int nranks, ncclComm_t c) : Comm(rank, nranks), comm_(c) {}
  ~NcclComm() override {
    if (dev_) cudaFree(dev_);
    if (comm_) g_nccl.CommDestroy(comm_);
  }
  int allreduce_sum_u64(uint64_t* d, size_t n, cudaStream_t s) override {
    return ck(g_nccl.AllReduce(d, d, n, ncclUint64, ncclSum, comm_, s));
  }
  int allreduce_max_u32(uint32_t* d, size_t n, cudaStream_t s) override {
    return ck(g_nccl.AllReduce(d, d, n, ncclUint32, ncclMax, comm_, s));
  }
  int allgather(const void* send, void* recv, size_t bytes, cudaStream_t s) override {
    return ck(g_nccl.AllGather(send, recv, bytes, ncclUint8, comm_, s));
  }
  int alltoallv(const void* send, const uint64_t* soff, const uint64_t* scnt, void* recv, const uint64_t* roff,
                const uint64_t* rcnt, cudaStream_t s) override {
    int e = ck(g_nccl.GroupStart());
    if (e) return e;
    for (int p = 0; p < nranks; ++p) {
      if (scnt[p]) e |= ck(g_nccl.Send((const uint8_t*)send + soff[p], scnt[p], ncclUint8, p, comm_, s));
      if (rcnt[p]) e |= ck(g_nccl.Recv((uint8_t*)recv + roff[p], rcnt[p], ncclUint8, p, comm_, s));
    }
    e |= ck(g_nccl.GroupEnd());
    return e;
  }
  int map_peers(int slot, void* local, void** peers, cudaStream_t s) override {
    (void)slot;
    IpcRef h;
    if (ipc_export(local, &h, &err)) return 1;
    if (!dev_) {
      if (cu(cudaMalloc(&dev_, (size_t)(nranks + 1) * sizeof h))) return 1;
    }
    uint8_t* d = (uint8_t*)dev_;
    if (cu(cudaMemcpyAsync(d, &h, sizeof h, cudaMemcpyHostToDevice, s))) return 1;
    if (ck(g_nccl.AllGather(d, d + sizeof h, sizeof h, ncclUint8, comm_, s))) return 1;
    std::vector<IpcRef> all(nranks);
    if (cu(cudaMemcpyAsync(all.data(), d + sizeof h, nranks * sizeof h, cudaMemcpyDeviceToHost, s))) return 1;
    if (cu(cudaStreamSynchronize(s))) return 1;
    for (int p = 0; p < nranks; ++p) {
      if (p == rank) { peers[p] = local; continue; }
      if (!(peers[p] = ipc_.open(all[p], &err))) return 1;
    }
    return 0;
  }
  int barrier(cudaStream_t s) override {
    if (!dev_ && cu(cudaMalloc(&dev_, (size_t)(nranks + 1) * sizeof(IpcRef)))) return 1;
    if (ck(g_nccl.AllReduce(dev_, dev_, 1, ncclUint32, ncclMax, comm_, s))) return 1;
    return cu(cudaStreamSynchronize(s));
  }

 private:
  IpcCache ipc_;
  void* dev_ = nullptr;
  int cu(cudaError_t e) {
    if (e == cudaSuccess) return 0;
    err = std::string("CUDA IPC: ") + cudaGetErrorString(e);
    return 1;
  }
  int ck(ncclResult_t r) {
    if (r == ncclSuccess) return 0;
    err = std::string("NCCL: ") + g_nccl.GetErrorString(r);
    return 1;
  }
  ncclComm_t comm_;
};

}  // namespace

int nccl_unique_id(void* out128, std::string* err) {
  if (!load_nccl(err)) return 1;
  ncclUniqueId id;
  ncclResult_t r = g_nccl.GetUniqueId(&id);
  if (r != ncclSuccess) {
    *err = std::string("ncclGetUniqueId: ") + g_nccl.GetErrorString(r);
    return 1;
  }
  memcpy(out128, &id, sizeof id);
  return 0;
}

Comm* make_nccl_comm(const void* id128, int rank, int nranks, std::string* err) {
  if (!load_nccl(err)) return nullptr;
  ncclUniqueId id;
  memcpy(&id, id128, sizeof id);
  ncclComm_t c = nullptr;
  ncclResult_t r = g_nccl.CommInitRank(&c, nranks, id, rank);
  if (r != ncclSuccess) {
    *err = std::string("ncclCommInitRank: ") + g_nccl.GetErrorString(r);
    return nullptr;
  }
  return new NcclComm(rank, nranks, c);
}

// ------------------------------------------------------------------ loopback
struct LoopbackGroup {
  explicit LoopbackGroup(int n) : n(n), slot(n) {}
  int n;
  std::mutex mu;
  std::condition_variable cv;
  int arrived = 0;
  uint64_t generation = 0;
  std::vector<std::vector<uint8_t>> slot;  // per-rank host blob (bootstrap allgather)
  void barrier() {
    std::unique_lock<std::mutex> lk(mu);
    const uint64_t g = generation;
    if (++arrived == n) {
      arrived = 0;
      ++generation;
      cv.notify_all();
    } else {
      cv.wait(lk, [&] { return generation != g; });
    }
  }
};

LoopbackGroup* loopback_group_new(int nranks) { return nranks >= 1 ? new LoopbackGroup(nranks) : nullptr; }
void loopback_group_delete(LoopbackGroup* g) { delete g; }
int loopback_group_size(const LoopbackGroup* g) { return g->n; }

namespace {

// The loopback group as a bootstrap: thread ranks exchange host blobs
// through the group's slots under its barrier.  The data path is PeerComm's
// (device kernels reading the other ranks' staging buffers directly: one
// process, one address space), the same kernels the multi-process peer
// backend runs over CUDA IPC mappings.
class LoopbackBootstrap : public Bootstrap {
 public:
  LoopbackBootstrap(LoopbackGroup* g, int rank) : Bootstrap(rank, g->n), g_(g) {}
  int allgather(const void* in, void* out, size_t bytes) override {
    g_->slot[rank].assign((const uint8_t*)in, (const uint8_t*)in + bytes);
    g_->barrier();
    for (int p = 0; p < nranks; ++p) memcpy((uint8_t*)out + (size_t)p * bytes, g_->slot[p].data(), bytes);
    g_->barrier();  // nobody rewrites a slot before every rank has read it
    return 0;
  }

 private:
  LoopbackGroup* g_;
};

}  // namespace

Comm* make_loopback_comm(LoopbackGroup* g, int rank) {
  return new PeerComm(new LoopbackBootstrap(g, rank), true, true);
}

}  // namespace cadv
