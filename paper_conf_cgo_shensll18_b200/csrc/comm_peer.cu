// comm_peer.cu — the library's own collectives over peer device memory
// (DESIGN.md §9 "Peer backend").
//
// Data never goes through the host: every rank stages its contribution in a
// device buffer, the ranks exchange the buffers' CUDA IPC handles (a few
// hundred bytes, over a host bootstrap), and each rank's kernel READS the
// peers' staged data through the IPC mappings -- over NVLink / NVSwitch
// between B200s, through the local HBM when the ranks share a GPU (the
// 2-process tests).  One kernel per collective:
//   allreduce   out[i] = op over ranks of peer_p[i]          (k_peer_reduce)
//   allgather   out[p * bytes + j] = peer_p[j]              (k_peer_gather)
//   alltoallv   recv[roff[p] + j] = peer_p[soff_p[me] + j]  (k_peer_gather, per-rank offsets)
// The bootstrap (host) carries only handles, offsets and barriers:
//   TcpBootstrap   one process per rank, a star of TCP connections through
//                  rank 0 (127.0.0.1 on one node);
//   the in-process loopback group (comm.cpp) provides the same three host
//   primitives for thread ranks and shares these kernels and this class.
#include <arpa/inet.h>
#include <cuda_runtime.h>
#include <errno.h>
#include <netdb.h>
#include <netinet/in.h>
#include <netinet/tcp.h>
#include <poll.h>
#include <string.h>
#include <sys/socket.h>
#include <time.h>
#include <unistd.h>

#include <string>
#include <vector>

#include "cadv_comm.h"

namespace cadv {

constexpr int PEER_MAX = 64;

namespace {

struct PeerPtrs {
  const uint8_t* p[PEER_MAX];
  uint64_t off[PEER_MAX];  // byte offset into peer p's buffer
  uint64_t cnt[PEER_MAX];  // bytes taken from peer p
  uint64_t dst[PEER_MAX];  // byte offset of p's part in the output
};

// out[i] = op_p src_p[i] for n elements of T (op: sum or max)
template <typename T, bool SUM>
__global__ void __launch_bounds__(256) k_peer_reduce(const __grid_constant__ PeerPtrs P, int G, T* out, uint64_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    T a = ((const T*)P.p[0])[i];
    for (int r = 1; r < G; ++r) {
      const T b = ((const T*)P.p[r])[i];
      a = SUM ? a + b : (a > b ? a : b);
    }
    out[i] = a;
  }
}

// out[dst[p] + j] = src_p[off[p] + j], j < cnt[p]; blockIdx.y = p.  16-byte
// vectors when the three addresses allow it.
__global__ void __launch_bounds__(256) k_peer_gather(const __grid_constant__ PeerPtrs P, uint8_t* out) {
  const int r = blockIdx.y;
  const uint64_t n = P.cnt[r];
  const uint8_t* s = P.p[r] + P.off[r];
  uint8_t* d = out + P.dst[r];
  const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x, nt = (uint64_t)gridDim.x * blockDim.x;
  if ((((uintptr_t)s | (uintptr_t)d | n) & 15) == 0) {
    for (uint64_t i = tid; i < n / 16; i += nt) ((uint4*)d)[i] = ((const uint4*)s)[i];
  } else {
    for (uint64_t i = tid; i < n; i += nt) d[i] = s[i];
  }
}

unsigned grid_for(uint64_t n) {
  const uint64_t g = (n + 255) / 256;
  return (unsigned)(g < 1 ? 1 : (g > 1184 ? 1184 : g));
}

}  // namespace

// ------------------------------------------------------------------ CUDA IPC
namespace {
typedef int (*GetAddressRange_t)(unsigned long long*, size_t*, unsigned long long);  // cuMemGetAddressRange_v2
GetAddressRange_t address_range_fn() {
  static GetAddressRange_t f = [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &p, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      p = nullptr;
    return (GetAddressRange_t)p;
  }();
  return f;
}
}  // namespace

int ipc_export(void* p, IpcRef* out, std::string* err) {
  GetAddressRange_t f = address_range_fn();
  unsigned long long base = 0;
  size_t size = 0;
  if (!f || f(&base, &size, (unsigned long long)(uintptr_t)p) != 0) {
    *err = "CUDA IPC: cannot resolve the allocation base (cuMemGetAddressRange)";
    return 1;
  }
  cudaError_t e = cudaIpcGetMemHandle(&out->h, (void*)(uintptr_t)base);
  if (e != cudaSuccess) {
    cudaGetLastError();
    *err = std::string("CUDA IPC: ") + cudaGetErrorString(e);
    return 1;
  }
  out->offset = (uint64_t)(uintptr_t)p - base;
  return 0;
}

IpcCache::~IpcCache() {
  for (auto& e : open_)
    if (e.base) cudaIpcCloseMemHandle(e.base);
}

void* IpcCache::open(const IpcRef& r, std::string* err) {
  for (auto& e : open_)
    if (!memcmp(&e.h, &r.h, sizeof r.h)) return (uint8_t*)e.base + r.offset;
  void* base = nullptr;
  cudaError_t e = cudaIpcOpenMemHandle(&base, r.h, cudaIpcMemLazyEnablePeerAccess);
  if (e != cudaSuccess) {
    cudaGetLastError();
    *err = std::string("CUDA IPC open: ") + cudaGetErrorString(e);
    return nullptr;
  }
  open_.push_back(Entry{r.h, base});
  return (uint8_t*)base + r.offset;
}

// ------------------------------------------------------------------ TCP bootstrap
namespace {

int send_all(int fd, const void* b, size_t n) {
  const char* p = (const char*)b;
  while (n) {
    ssize_t k = ::send(fd, p, n, MSG_NOSIGNAL);
    if (k < 0 && errno == EINTR) continue;
    if (k <= 0) return 1;
    p += k;
    n -= (size_t)k;
  }
  return 0;
}

int recv_all(int fd, void* b, size_t n) {
  char* p = (char*)b;
  while (n) {
    ssize_t k = ::recv(fd, p, n, 0);
    if (k < 0 && errno == EINTR) continue;
    if (k <= 0) return 1;
    p += k;
    n -= (size_t)k;
  }
  return 0;
}

class TcpBootstrap : public Bootstrap {
 public:
  TcpBootstrap(int rank, int nranks) : Bootstrap(rank, nranks), fds_(nranks, -1) {}
  ~TcpBootstrap() override {
    for (int fd : fds_)
      if (fd >= 0) ::close(fd);
    if (listen_ >= 0) ::close(listen_);
  }
  // host:port of rank 0; every rank calls it (rank 0 accepts nranks - 1 peers)
  int connect_all(const char* addr, int timeout_s, std::string* err) {
    std::string a(addr ? addr : "");
    const size_t c = a.rfind(':');
    if (c == std::string::npos) { *err = "bootstrap address must be host:port"; return 1; }
    const std::string host = a.substr(0, c);
    const int port = atoi(a.c_str() + c + 1);
    sockaddr_in sa{};
    sa.sin_family = AF_INET;
    sa.sin_port = htons((uint16_t)port);
    if (inet_pton(AF_INET, host.c_str(), &sa.sin_addr) != 1) { *err = "bootstrap host must be an IPv4 address"; return 1; }
    const time_t t_end = time(nullptr) + timeout_s;
    if (rank == 0) {
      listen_ = ::socket(AF_INET, SOCK_STREAM, 0);
      int one = 1;
      setsockopt(listen_, SOL_SOCKET, SO_REUSEADDR, &one, sizeof one);
      if (::bind(listen_, (sockaddr*)&sa, sizeof sa) || ::listen(listen_, nranks)) {
        *err = std::string("bootstrap bind/listen: ") + strerror(errno);
        return 1;
      }
      for (int k = 1; k < nranks; ++k) {
        pollfd pf{listen_, POLLIN, 0};
        const int left = (int)(t_end - time(nullptr));
        if (left <= 0 || ::poll(&pf, 1, left * 1000) <= 0) { *err = "bootstrap: timed out waiting for ranks"; return 1; }
        int fd = ::accept(listen_, nullptr, nullptr);
        int32_t r = -1;
        if (fd < 0 || recv_all(fd, &r, 4) || r <= 0 || r >= nranks || fds_[r] >= 0) {
          *err = "bootstrap: bad peer hello";
          return 1;
        }
        setsockopt(fd, IPPROTO_TCP, TCP_NODELAY, &one, sizeof one);
        fds_[r] = fd;
      }
    } else {
      while (true) {
        int fd = ::socket(AF_INET, SOCK_STREAM, 0);
        if (::connect(fd, (sockaddr*)&sa, sizeof sa) == 0) {
          int one = 1;
          setsockopt(fd, IPPROTO_TCP, TCP_NODELAY, &one, sizeof one);
          const int32_t r = rank;
          if (send_all(fd, &r, 4)) { ::close(fd); *err = "bootstrap: hello failed"; return 1; }
          fds_[0] = fd;
          break;
        }
        ::close(fd);
        if (time(nullptr) >= t_end) { *err = "bootstrap: cannot reach rank 0"; return 1; }
        usleep(20000);
      }
    }
    return 0;
  }
  int allgather(const void* in, void* out, size_t bytes) override {
    uint8_t* o = (uint8_t*)out;
    if (rank == 0) {
      memcpy(o, in, bytes);
      for (int p = 1; p < nranks; ++p)
        if (recv_all(fds_[p], o + (size_t)p * bytes, bytes)) return 1;
      for (int p = 1; p < nranks; ++p)
        if (send_all(fds_[p], o, (size_t)nranks * bytes)) return 1;
      return 0;
    }
    if (send_all(fds_[0], in, bytes)) return 1;
    return recv_all(fds_[0], o, (size_t)nranks * bytes);
  }

 private:
  std::vector<int> fds_;
  int listen_ = -1;
};

}  // namespace

Bootstrap* make_tcp_bootstrap(const char* addr, int rank, int nranks, int timeout_s, std::string* err) {
  auto* b = new TcpBootstrap(rank, nranks);
  if (b->connect_all(addr, timeout_s, err)) {
    delete b;
    return nullptr;
  }
  return b;
}

// ------------------------------------------------------------------ PeerComm
PeerComm::PeerComm(Bootstrap* b, bool owns, bool same_process)
    : Comm(b->rank, b->nranks), boot_(b), owns_(owns), same_process_(same_process) {}

PeerComm::~PeerComm() {
  if (stage_) cudaFree(stage_);
  for (void* p : graveyard_) cudaFree(p);
  if (tmp_) cudaFree(tmp_);
  if (owns_) delete boot_;
}

int PeerComm::cu(cudaError_t e) {
  if (e == cudaSuccess) return 0;
  cudaGetLastError();
  err = std::string("peer comm: ") + cudaGetErrorString(e);
  return 1;
}

int PeerComm::boot(int e) {
  if (e) err = "peer comm: bootstrap exchange failed";
  return e;
}

int PeerComm::grow(void** buf, size_t* cap, size_t bytes) {
  if (*cap >= bytes) return 0;
  // an exported buffer is never freed while the communicator lives (see DevBuf::exported)
  if (*buf) graveyard_.push_back(*buf);
  *buf = nullptr;
  *cap = 0;
  const size_t want = 2 * bytes + 256;
  if (cu(cudaMalloc(buf, want))) return 1;
  *cap = want;
  return 0;
}

// Publishes `local` (base of a device allocation, or null) of this rank
// together with `extra` bytes of host data; fills peers[p] (mapped device
// pointers, local for p == rank) and all_extra (nranks * extra_bytes).
int PeerComm::exchange(int slot, void* local, const void* extra, size_t extra_bytes, void** peers,
                       std::vector<uint8_t>* all_extra) {
  struct Rec { IpcRef ref; uint64_t ptr; uint32_t has; };
  std::vector<uint8_t> mine(sizeof(Rec) + extra_bytes, 0), all((sizeof(Rec) + extra_bytes) * nranks);
  Rec r{};
  r.has = local != nullptr;
  r.ptr = (uint64_t)(uintptr_t)local;
  if (local && !same_process_ && ipc_export(local, &r.ref, &err)) return 1;
  memcpy(mine.data(), &r, sizeof r);
  if (extra_bytes) memcpy(mine.data() + sizeof r, extra, extra_bytes);
  if (boot(boot_->allgather(mine.data(), all.data(), mine.size()))) return 1;
  (void)slot;
  for (int p = 0; p < nranks; ++p) {
    Rec q;
    memcpy(&q, all.data() + (size_t)p * mine.size(), sizeof q);
    if (all_extra) {
      all_extra->resize((size_t)nranks * extra_bytes);
      memcpy(all_extra->data() + (size_t)p * extra_bytes, all.data() + (size_t)p * mine.size() + sizeof q, extra_bytes);
    }
    if (!peers) continue;
    if (p == rank || !q.has) { peers[p] = p == rank ? local : nullptr; continue; }
    if (same_process_) { peers[p] = (void*)(uintptr_t)q.ptr; continue; }
    if (!(peers[p] = ipc_.open(q.ref, &err))) return 1;
  }
  return 0;
}

int PeerComm::stage_in(const void* d, size_t bytes, cudaStream_t s) {
  if (grow(&stage_, &stage_cap_, bytes ? bytes : 16)) return 1;
  if (bytes && cu(cudaMemcpyAsync(stage_, d, bytes, cudaMemcpyDeviceToDevice, s))) return 1;
  return cu(cudaStreamSynchronize(s));  // staged before the peers read it
}

template <typename T, bool SUM>
int PeerComm::reduce(T* d, size_t n, cudaStream_t s) {
  const size_t bytes = n * sizeof(T);
  if (stage_in(d, bytes, s)) return finish(1);
  void* peers[PEER_MAX];
  if (exchange(0, stage_, nullptr, 0, peers, nullptr)) return finish(1);
  PeerPtrs P{};
  for (int p = 0; p < nranks; ++p) P.p[p] = (const uint8_t*)peers[p];
  if (n) {
    k_peer_reduce<T, SUM><<<grid_for(n), 256, 0, s>>>(P, nranks, d, n);
    if (cu(cudaGetLastError())) return finish(1);
  }
  return finish(cu(cudaStreamSynchronize(s)));
}

int PeerComm::allreduce_sum_u64(uint64_t* d, size_t n, cudaStream_t s) {
  if (nranks > PEER_MAX) { err = "peer comm: too many ranks"; return 1; }
  return reduce<uint64_t, true>(d, n, s);
}
int PeerComm::allreduce_max_u32(uint32_t* d, size_t n, cudaStream_t s) {
  if (nranks > PEER_MAX) { err = "peer comm: too many ranks"; return 1; }
  return reduce<uint32_t, false>(d, n, s);
}

int PeerComm::allgather(const void* send, void* recv, size_t bytes, cudaStream_t s) {
  if (stage_in(send, bytes, s)) return finish(1);
  void* peers[PEER_MAX];
  if (exchange(0, stage_, nullptr, 0, peers, nullptr)) return finish(1);
  PeerPtrs P{};
  for (int p = 0; p < nranks; ++p) {
    P.p[p] = (const uint8_t*)peers[p];
    P.off[p] = 0;
    P.cnt[p] = bytes;
    P.dst[p] = (uint64_t)p * bytes;
  }
  if (bytes) {
    k_peer_gather<<<dim3(grid_for(bytes / 16 + 1), nranks), 256, 0, s>>>(P, (uint8_t*)recv);
    if (cu(cudaGetLastError())) return finish(1);
  }
  return finish(cu(cudaStreamSynchronize(s)));
}

int PeerComm::alltoallv(const void* send, const uint64_t* soff, const uint64_t* scnt, void* recv, const uint64_t* roff,
                        const uint64_t* rcnt, cudaStream_t s) {
  uint64_t end = 0;
  for (int p = 0; p < nranks; ++p) end = soff[p] + scnt[p] > end ? soff[p] + scnt[p] : end;
  if (stage_in(send, end, s)) return finish(1);
  // every rank's (soff, scnt) rows travel with the handles
  std::vector<uint64_t> mine(2 * (size_t)nranks);
  for (int p = 0; p < nranks; ++p) { mine[p] = soff[p]; mine[nranks + p] = scnt[p]; }
  std::vector<uint8_t> rows;
  void* peers[PEER_MAX];
  if (exchange(0, stage_, mine.data(), mine.size() * 8, peers, &rows)) return finish(1);
  PeerPtrs P{};
  uint64_t mx = 0;
  for (int p = 0; p < nranks; ++p) {
    const uint64_t* row = (const uint64_t*)(rows.data() + (size_t)p * mine.size() * 8);
    if (row[nranks + rank] != rcnt[p]) { err = "peer comm alltoallv: send / receive counts disagree"; return finish(1); }
    P.p[p] = (const uint8_t*)peers[p];
    P.off[p] = row[rank];
    P.cnt[p] = rcnt[p];
    P.dst[p] = roff[p];
    mx = rcnt[p] > mx ? rcnt[p] : mx;
  }
  if (mx) {
    k_peer_gather<<<dim3(grid_for(mx / 16 + 1), nranks), 256, 0, s>>>(P, (uint8_t*)recv);
    if (cu(cudaGetLastError())) return finish(1);
  }
  return finish(cu(cudaStreamSynchronize(s)));
}

int PeerComm::map_peers(int slot, void* local, void** peers, cudaStream_t s) {
  if (cu(cudaStreamSynchronize(s))) return finish(1);
  return exchange(1 + slot, local, nullptr, 0, peers, nullptr);
}

int PeerComm::barrier(cudaStream_t s) {
  const int e = cu(cudaStreamSynchronize(s));
  return finish(e);
}

// second bootstrap barrier: nobody restages before every rank has read;
// a failed rank still takes part (no rank is left waiting)
int PeerComm::finish(int e) {
  const int b = boot_->barrier();
  if (b && !e) err = "peer comm: bootstrap barrier failed";
  return e | b;
}

Comm* make_peer_comm(const char* addr, int rank, int nranks, std::string* err) {
  if (nranks > PEER_MAX) {
    *err = "peer comm: at most 64 ranks";
    return nullptr;
  }
  Bootstrap* b = make_tcp_bootstrap(addr, rank, nranks, 120, err);
  if (!b) return nullptr;
  return new PeerComm(b, true, false);
}

}  // namespace cadv
