// cadv.cu — the C ABI of libcadv (include/cadv.h): context, trace
// registration, and the synchronous analysis entry points.
#include <cuda_runtime.h>
#include <cstdlib>
#include <stdio.h>
#include <string.h>

#include <string>

#include "cadv_impl.h"
#include "common.cuh"

namespace cadv {

cudaError_t ensure(cadv_ctx* c, BufId id, size_t bytes, void** out) {
  DevBuf& b = c->buf[id];
  if (bytes == 0) bytes = 16;
  if (b.bytes < bytes) {
    if (b.p) {
      cudaError_t e = cudaStreamSynchronize(c->stream);
      if (e != cudaSuccess) return e;
      if (b.exported) c->graveyard.push_back(b.p);
      else cudaFree(b.p);
      b.p = nullptr;
      b.bytes = 0;
    }
    size_t want = b.exported ? 2 * bytes : bytes + bytes / 8;  // headroom so slightly larger calls do not reallocate
    cudaError_t e = cudaMalloc(&b.p, want);
    if (e != cudaSuccess) {
      cudaGetLastError();
      e = cudaMalloc(&b.p, bytes);
      if (e != cudaSuccess) { b.p = nullptr; return e; }
      want = bytes;
    }
    b.bytes = want;
  }
  *out = b.p;
  return cudaSuccess;
}

cudaError_t ensure_host(cadv_ctx* c, size_t bytes, void** out) {
  if (c->host_pinned_bytes < bytes) {
    if (c->host_pinned) cudaFreeHost(c->host_pinned);
    c->host_pinned = nullptr;
    c->host_pinned_bytes = 0;
    cudaError_t e = cudaMallocHost(&c->host_pinned, bytes);
    if (e != cudaSuccess) return e;
    c->host_pinned_bytes = bytes;
  }
  *out = c->host_pinned;
  return cudaSuccess;
}

Scalars* scalars(cadv_ctx* c) { return (Scalars*)c->buf[B_SCALARS].p; }

void prof_begin(cadv_ctx* c, const char* src) {
  c->prof_skip = false;
  if (!c->profiling) return;
  if (c->profiling == 2 && strncmp(src, "k_scan<", 7) != 0) {
    c->prof_skip = true;
    return;
  }
  uint32_t k = c->nprof;
  while (c->prof_ev.size() < 2ull * (k + 1)) {
    cudaEvent_t e;
    if (cudaEventCreate(&e) != cudaSuccess) { c->profiling = 0; return; }
    c->prof_ev.push_back(e);
  }
  if (c->prof_src.size() <= k) c->prof_src.resize(k + 1);
  c->prof_src[k] = src;
  cudaEventRecord(c->prof_ev[2 * k], c->stream);
}

void prof_end(cadv_ctx* c) {
  if (!c->profiling || c->prof_skip || c->prof_ev.size() < 2ull * (c->nprof + 1)) return;
  cudaEventRecord(c->prof_ev[2 * c->nprof + 1], c->stream);
  c->nprof++;
}

// after the stream is synchronised: per-launch times and kernel names
static void prof_collect(cadv_ctx* c) {
  c->prof_ms.assign(c->nprof, 0.f);
  c->prof_name.assign(c->nprof, std::string());
  for (uint32_t k = 0; k < c->nprof; ++k) {
    cudaEventElapsedTime(&c->prof_ms[k], c->prof_ev[2 * k], c->prof_ev[2 * k + 1]);
    std::string src = c->prof_src[k] ? c->prof_src[k] : "";
    size_t a = src.find("<<<");
    std::string nm = src.substr(0, a);
    // the launched name: the identifier (with its template arguments) before "<<<"
    int depth = 0;
    size_t i = nm.size();
    while (i > 0) {
      const char ch = nm[i - 1];
      if (ch == '>') depth++;
      else if (ch == '<') depth--;
      else if (depth == 0 && (ch == ' ' || ch == '(' || ch == ',' || ch == ';')) break;
      --i;
    }
    nm = nm.substr(i);
    c->prof_name[k] = nm;
  }
}

// Every rank's per-call status words, max-reduced over the ranks before any
// exchange: bad record / group (err_code), site id >= nsites, CTA-id range,
// unsupported reuse line, workspace to grow (`again`, set by the host).
__global__ void k_agree_flags(const Scalars* s, const uint64_t* f1, const uint64_t* f2, uint32_t again, uint32_t* out) {
  if (threadIdx.x == 0) {
    out[0] = s->err_code;
    out[1] = ((f1 && *f1) || (f2 && *f2)) ? 1u : 0u;
    out[2] = (uint32_t)(s->max_cta > 0xffffffffull ? 0xffffffffull : s->max_cta);
    out[3] = s->unsup_index != ~0ull ? 1u : 0u;
    out[4] = again;
  }
}

}  // namespace cadv

using namespace cadv;

namespace {

cadv_status fail(cadv_ctx* c, cadv_status s, const std::string& msg) {
  if (c) c->err = msg;
  return s;
}

cadv_status cuda_fail(cadv_ctx* c, cudaError_t e, const char* where) {
  cudaGetLastError();
  std::string m = std::string(where) + ": " + cudaGetErrorString(e);
  return fail(c, e == cudaErrorMemoryAllocation ? CADV_ERR_OOM : CADV_ERR_CUDA, m);
}

#define CK(expr, where)                                     \
  do {                                                      \
    cudaError_t _e = (expr);                                \
    if (_e != cudaSuccess) return cuda_fail(c, _e, where);  \
  } while (0)

bool pow2(uint32_t x) { return x && !(x & (x - 1)); }
uint32_t ilog2(uint32_t x) {
  uint32_t l = 0;
  while ((1u << l) < x) ++l;
  return l;
}

// Starts an analysis: zero the per-call scalars, start the device timer.
cadv_status begin_call(cadv_ctx* c) {
  void* p;
  CK(ensure(c, B_SCALARS, sizeof(Scalars), &p), "workspace");
  CK(cudaMemsetAsync(p, 0, sizeof(Scalars), c->stream), "memset");
  CK(cudaMemsetAsync(&((Scalars*)p)->err_index, 0xff, sizeof(unsigned long long), c->stream), "memset");
  CK(cudaMemsetAsync(&((Scalars*)p)->unsup_index, 0xff, sizeof(unsigned long long), c->stream), "memset");
  c->launches = 0;
  c->nprof = 0;
  for (auto& v : c->counts) v = 0;
  CK(cudaEventRecord(c->ev0, c->stream), "event");
  return CADV_OK;
}

// Ends an analysis: stop the timer, copy `nout` bytes of device results plus
// the scalars to pinned host memory, synchronise, check the error scalars.
cadv_status end_call(cadv_ctx* c, const void* d_out, size_t nout, void** h_out) {
  CK(cudaEventRecord(c->ev1, c->stream), "event");
  void* h;
  CK(ensure_host(c, nout + sizeof(Scalars) + 64, &h), "pinned host");
  Scalars* hs = (Scalars*)h;
  CK(cudaMemcpyAsync(hs, scalars(c), sizeof(Scalars), cudaMemcpyDeviceToHost, c->stream), "D2H");
  uint8_t* hr = (uint8_t*)h + ((sizeof(Scalars) + 63) & ~size_t(63));
  if (nout) CK(cudaMemcpyAsync(hr, d_out, nout, cudaMemcpyDeviceToHost, c->stream), "D2H");
  CK(cudaStreamSynchronize(c->stream), "kernel execution");
  float ms = 0.f;
  CK(cudaEventElapsedTime(&ms, c->ev0, c->ev1), "event");
  c->elapsed_ms = ms;
  prof_collect(c);
  if (hs->err_code) {
    char b[200];
    snprintf(b, sizeof b, "%s at trace position %llu",
             hs->err_code == 1 ? "invalid record" :
             hs->err_code == 2 ? "warp-level group longer than 32 records or with a repeated lane" :
             hs->err_code == 4 ? "warp-level group whose records differ in kind or site" :
                                 "trace invariant violated",
             (unsigned long long)(hs->err_index == ~0ull ? 0 : hs->err_index + c->global_offset));
    return fail(c, CADV_ERR_BAD_TRACE, b);
  }
  if (hs->unsup_index != ~0ull) {
    char b[200];
    snprintf(b, sizeof b, "memory record at trace position %llu: its reuse-distance line (addr / line_bytes) is >= 2^58",
             (unsigned long long)(hs->unsup_index + c->global_offset));
    return fail(c, CADV_ERR_UNSUPPORTED, b);
  }
  *h_out = hr;
  return CADV_OK;
}

// Multi-rank load: the run keys
// (cta, tid / 32, winst, family) of every shard's first and last record, so
// that a shard boundary splitting a warp-level group is detected.
cadv_status load_trace_collective(cadv_ctx* c) {
  const int G = c->nranks;
  void* p;
  CK(ensure(c, B_COMM, 64 + (size_t)G * 64 + 64, &p), "workspace");
  uint32_t* d = (uint32_t*)p;
  uint32_t h[16] = {0};
  h[0] = c->t.warp_contiguous ? 0u : 1u;
  if (c->t.n) {
    const uint64_t at[2] = {0, c->t.n - 1};
    for (int k = 0; k < 2; ++k) {
      uint32_t cta, winst;
      uint16_t tid;
      uint8_t meta;
      CK(cudaMemcpy(&cta, c->t.cta + at[k], 4, cudaMemcpyDeviceToHost), "D2H");
      CK(cudaMemcpy(&winst, c->t.winst + at[k], 4, cudaMemcpyDeviceToHost), "D2H");
      CK(cudaMemcpy(&tid, c->t.tid + at[k], 2, cudaMemcpyDeviceToHost), "D2H");
      CK(cudaMemcpy(&meta, c->t.meta + at[k], 1, cudaMemcpyDeviceToHost), "D2H");
      h[1 + 4 * k] = 1;
      h[2 + 4 * k] = cta;
      h[3 + 4 * k] = ((uint32_t)tid >> 5) | (((meta & 3u) == 2u) ? 0x10000u : 0u);
      h[4 + 4 * k] = winst;
    }
  }
  CK(cudaMemcpyAsync(d, h, 64, cudaMemcpyHostToDevice, c->stream), "H2D");
  if (c->comm->allgather(d, d + 16, 64, c->stream)) return fail(c, CADV_ERR_NCCL, c->comm->err);
  std::vector<uint32_t> all((size_t)G * 16);
  CK(cudaMemcpyAsync(all.data(), d + 16, (size_t)G * 64, cudaMemcpyDeviceToHost, c->stream), "D2H");
  CK(cudaStreamSynchronize(c->stream), "collective");
  c->split_group = false;
  c->noncontig_any = false;
  const uint32_t* prev_last = nullptr;
  for (int r = 0; r < G; ++r) {
    const uint32_t* e = all.data() + (size_t)r * 16;
    if (e[0]) c->noncontig_any = true;
    if (!e[1]) continue;  // empty shard
    if (prev_last && prev_last[0] && prev_last[1] == e[2] && prev_last[2] == e[3] && prev_last[3] == e[4])
      c->split_group = true;
    prev_last = e + 5;
  }
  return CADV_OK;
}

}  // namespace

extern "C" {

CADV_API const char* cadv_version(void) { return "cadv 0.1 (sm_100a)"; }

}  // extern "C"

namespace {

cadv_status create_ctx(cadv_ctx** out, int device, void* cuda_stream, const void* nccl_unique_id,
                       LoopbackGroup* group, int rank, int nranks, const char* peer_addr = nullptr) {
  if (!out) return CADV_ERR_INVALID_ARG;
  *out = nullptr;
  if (nranks < 1 || rank < 0 || rank >= nranks) return CADV_ERR_INVALID_ARG;
  if (nranks > 1 && !nccl_unique_id && !group && !peer_addr) return CADV_ERR_INVALID_ARG;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
    cudaGetLastError();
    return CADV_ERR_CUDA;
  }
  cudaDeviceProp prop;
  if (cudaGetDeviceProperties(&prop, device) != cudaSuccess) return CADV_ERR_CUDA;
  if (prop.major != 10) return CADV_ERR_CUDA;  // built for sm_100a only
  if (cudaSetDevice(device) != cudaSuccess) return CADV_ERR_CUDA;
  cadv_ctx* c = new cadv_ctx();
  c->device = device;
  c->stream = (cudaStream_t)cuda_stream;
  c->rank = rank;
  c->nranks = nranks;
  c->num_sms = prop.multiProcessorCount;
  if (const char* e = getenv("CADV_SCAN_CTAS")) c->scan_ctas = atoi(e);
  if (const char* e = getenv("CADV_SCAN_SPLIT")) c->scan_split = atoi(e);
  if (cudaEventCreate(&c->ev0) != cudaSuccess || cudaEventCreate(&c->ev1) != cudaSuccess ||
      cudaMallocHost(&c->hstage, 512) != cudaSuccess) {
    if (c->hstage) cudaFreeHost(c->hstage);
    delete c;
    return CADV_ERR_CUDA;
  }
  if (group) {
    c->comm = make_loopback_comm(group, rank);
  } else if (peer_addr) {
    std::string err;
    c->comm = make_peer_comm(peer_addr, rank, nranks, &err);
    if (!c->comm) {
      fprintf(stderr, "cadv_create_peer: %s\n", err.c_str());
      cudaEventDestroy(c->ev0);
      cudaEventDestroy(c->ev1);
      cudaFreeHost(c->hstage);
      delete c;
      return CADV_ERR_NCCL;
    }
  } else if (nccl_unique_id) {
    std::string err;
    c->comm = make_nccl_comm(nccl_unique_id, rank, nranks, &err);
    if (!c->comm) {
      fprintf(stderr, "cadv_create: %s\n", err.c_str());
      cudaEventDestroy(c->ev0);
      cudaEventDestroy(c->ev1);
      cudaFreeHost(c->hstage);
      delete c;
      return CADV_ERR_NCCL;
    }
  }
  *out = c;
  return CADV_OK;
}

}  // namespace

extern "C" {

CADV_API cadv_status cadv_create(cadv_ctx** out, int device, void* cuda_stream, const void* nccl_unique_id, int rank,
                                 int nranks) {
  return create_ctx(out, device, cuda_stream, nccl_unique_id, nullptr, rank, nranks);
}

CADV_API cadv_status cadv_nccl_unique_id(void* out128) {
  if (!out128) return CADV_ERR_INVALID_ARG;
  std::string err;
  if (nccl_unique_id(out128, &err)) {
    fprintf(stderr, "cadv_nccl_unique_id: %s\n", err.c_str());
    return CADV_ERR_NCCL;
  }
  return CADV_OK;
}

CADV_API cadv_status cadv_create_peer(cadv_ctx** out, int device, void* cuda_stream, const char* bootstrap_addr,
                                     int rank, int nranks) {
  if (!bootstrap_addr) return CADV_ERR_INVALID_ARG;
  return create_ctx(out, device, cuda_stream, nullptr, nullptr, rank, nranks, bootstrap_addr);
}

CADV_API int cadv_bootstrap_selftest(const char* bootstrap_addr, int rank, int nranks, const void* in, void* out,
                                     uint64_t bytes) {
  if (!bootstrap_addr || nranks < 1 || rank < 0 || rank >= nranks || (bytes && (!in || !out))) return 1;
  std::string err;
  Bootstrap* b = make_tcp_bootstrap(bootstrap_addr, rank, nranks, 60, &err);
  if (!b) {
    fprintf(stderr, "cadv_bootstrap_selftest: %s\n", err.c_str());
    return 2;
  }
  int e = b->allgather(in, out, bytes);
  e |= b->barrier();
  delete b;
  return e ? 3 : 0;
}

CADV_API void* cadv_loopback_group_create(int nranks) { return nranks >= 1 ? loopback_group_new(nranks) : nullptr; }

CADV_API cadv_status cadv_loopback_group_destroy(void* group) {
  if (!group) return CADV_ERR_INVALID_ARG;
  loopback_group_delete((LoopbackGroup*)group);
  return CADV_OK;
}

CADV_API cadv_status cadv_create_loopback(cadv_ctx** out, int device, void* cuda_stream, void* group, int rank) {
  if (!group) return CADV_ERR_INVALID_ARG;
  int n = loopback_group_size((LoopbackGroup*)group);
  return create_ctx(out, device, cuda_stream, nullptr, (LoopbackGroup*)group, rank, n);
}

CADV_API cadv_status cadv_destroy(cadv_ctx* c) {
  if (!c) return CADV_ERR_INVALID_ARG;
  cudaSetDevice(c->device);
  cudaStreamSynchronize(c->stream);
  delete c->comm;  // (closes its peer mappings before the buffers go)
  c->comm = nullptr;
  for (auto& b : c->buf)
    if (b.p) cudaFree(b.p);
  for (void* p : c->graveyard) cudaFree(p);
  if (c->host_pinned) cudaFreeHost(c->host_pinned);
  if (c->hstage) cudaFreeHost(c->hstage);
  if (c->ev0) cudaEventDestroy(c->ev0);
  if (c->ev1) cudaEventDestroy(c->ev1);
  for (auto e : c->prof_ev) cudaEventDestroy(e);
  if (c->tc_buf) cudaFree(c->tc_buf);
  delete c;
  return CADV_OK;
}

CADV_API const char* cadv_last_error(const cadv_ctx* c) { return c ? c->err.c_str() : "null context"; }
CADV_API float cadv_last_elapsed_ms(const cadv_ctx* c) { return c ? c->elapsed_ms : 0.f; }
CADV_API uint32_t cadv_last_launches(const cadv_ctx* c) { return c ? c->launches : 0; }

CADV_API uint64_t cadv_last_count(const cadv_ctx* c, int which) {
  return (c && which >= 0 && which < 4) ? c->counts[which] : 0;
}

CADV_API cadv_status cadv_set_profiling(cadv_ctx* c, int enable) {
  if (!c) return CADV_ERR_INVALID_ARG;
  if (enable < 0 || enable > 2) return CADV_ERR_INVALID_ARG;
  c->profiling = enable;
  return CADV_OK;
}

CADV_API uint32_t cadv_last_kernel_times(const cadv_ctx* c, const char** names, float* ms, uint32_t max) {
  if (!c) return 0;
  uint32_t k = (uint32_t)c->prof_ms.size();
  for (uint32_t i = 0; i < k && i < max; ++i) {
    if (names) names[i] = c->prof_name[i].c_str();
    if (ms) ms[i] = c->prof_ms[i];
  }
  return k;
}

CADV_API cadv_status cadv_load_trace(cadv_ctx* c, const cadv_trace_desc* d, uint64_t global_offset) {
  if (!c || !d) return CADV_ERR_INVALID_ARG;
  c->err.clear();
  c->loaded = false;
  if (d->n >= 0xffffffffull) return fail(c, CADV_ERR_UNSUPPORTED, "a shard must hold fewer than 2^32 - 1 records");
  if (d->n && (!d->addr || !d->cta || !d->tid || !d->site || !d->winst || !d->meta))
    return fail(c, CADV_ERR_INVALID_ARG, "NULL trace column");
  if (((uintptr_t)d->addr & 7) || ((uintptr_t)d->cta & 3) || ((uintptr_t)d->tid & 1) || ((uintptr_t)d->site & 3) ||
      ((uintptr_t)d->winst & 3))
    return fail(c, CADV_ERR_INVALID_ARG, "trace columns must be naturally aligned");
  CK(cudaSetDevice(c->device), "cudaSetDevice");
  cadv_status s = CADV_OK;
  const bool copy = !d->on_device && d->n;
  // device columns are only registered (no device work, no synchronisation)
  if (copy && (s = begin_call(c)) != CADV_OK) return s;
  c->t = *d;
  c->t.on_device = 1;
  c->global_offset = global_offset;
  if (copy) {
    const void* src[6] = {d->addr, d->cta, d->tid, d->site, d->winst, d->meta};
    size_t es[6] = {8, 4, 2, 4, 4, 1};
    void* dst[6];
    for (int k = 0; k < 6; ++k) {
      CK(ensure(c, (BufId)(B_HOST_COPY0 + k), es[k] * d->n, &dst[k]), "trace copy");
      CK(cudaMemcpyAsync(dst[k], src[k], es[k] * d->n, cudaMemcpyHostToDevice, c->stream), "H2D");
    }
    c->t.addr = (const uint64_t*)dst[0];
    c->t.cta = (const uint32_t*)dst[1];
    c->t.tid = (const uint16_t*)dst[2];
    c->t.site = (const uint32_t*)dst[3];
    c->t.winst = (const uint32_t*)dst[4];
    c->t.meta = (const uint8_t*)dst[5];
  }
  if (copy) {
    void* h;
    s = end_call(c, nullptr, 0, &h);
    if (s != CADV_OK) return s;
  } else {
    c->launches = 0;
    c->nprof = 0;
    c->prof_ms.clear();
    c->prof_name.clear();
    c->elapsed_ms = 0.f;
  }
  c->max_cta = 0;  // R0's CTA-id range comes out of each analysis' streaming pass
  if (c->comm) {
    s = load_trace_collective(c);
    if (s != CADV_OK) return s;
  }
  c->loaded = true;
  return CADV_OK;
}

}  // extern "C"

namespace {

struct Req {
  bool rd = false, md = false, bd = false;
  uint32_t rd_lbs = 7, md_lbs = 7, md_ws = 5, bd_ws = 5;
  int scope = CADV_SCOPE_CTA, log2bins = 0;
  uint32_t nbins = 66, nsites = 0;
  bool md_sites = false, bd_sites = false;
  // data-centric attribution (cadv_data_centric): nobj > 0 object line extents
  // on the device; the RD / MD histograms get one row per object + 1
  uint32_t nobj = 0;
  const uint64_t* obj_lo = nullptr;
  const uint64_t* obj_hi = nullptr;
};

cadv_status check_args(cadv_ctx* c, uint32_t line_bytes, uint32_t warp_size, bool check_line, bool check_warp) {
  if (check_line && (!pow2(line_bytes) || line_bytes > 4096))
    return fail(c, CADV_ERR_INVALID_ARG, "line_bytes must be 2^k <= 4096");
  if (check_warp && (!pow2(warp_size) || warp_size > 32))
    return fail(c, CADV_ERR_INVALID_ARG, "warp_size must be 2^k <= 32");
  return CADV_OK;
}

// Runs the requested analyses with ONE streaming pass over the trace (k_scan)
// followed by the reuse tail (regroup, tiles, cross-tile) and the deferred
// branch-divergence resolution.  Device output layout in B_OUT2:
//   [rd hist nbins][rd stats 4][md hist 2(W+1)][md sites 2 nsites][md flag]
//   [bd totals 3][bd flag][bd sites 3 nsites]
constexpr cadv_status RETRY = (cadv_status)100;  // internal: workspace grown, run the call again

// (re)allocates the T_c table with `cap` entries; keep = entries to preserve
cudaError_t tc_resize(cadv_ctx* c, uint32_t cap, uint32_t keep) {
  uint32_t* nb = nullptr;
  cudaError_t e = cudaMalloc(&nb, 4ull * cap);
  if (e != cudaSuccess) return e;
  if ((e = cudaMemsetAsync(nb, 0, 4ull * cap, c->stream))) return e;
  if (keep && c->tc_buf &&
      (e = cudaMemcpyAsync(nb, c->tc_buf, 4ull * keep, cudaMemcpyDeviceToDevice, c->stream)))
    return e;
  if ((e = cudaStreamSynchronize(c->stream))) return e;
  if (c->tc_buf) cudaFree(c->tc_buf);
  c->tc_buf = nb;
  c->tc_cap = cap;
  return cudaSuccess;
}

cadv_status run_once(cadv_ctx* c, const Req& q, uint64_t* rd_hist, cadv_reuse_stats* rd_stats, uint64_t* md_hist,
                     cadv_site_mem* md_sites, uint64_t* bd_tot, cadv_site_branch* bd_sites);

cadv_status run_analyses(cadv_ctx* c, const Req& q, uint64_t* rd_hist, cadv_reuse_stats* rd_stats, uint64_t* md_hist,
                         cadv_site_mem* md_sites, uint64_t* bd_tot, cadv_site_branch* bd_sites) {
  if (!c->loaded) return fail(c, CADV_ERR_NO_TRACE, "no trace loaded");
  const bool noncontig = c->comm ? c->noncontig_any : !c->t.warp_contiguous;
  if (q.rd && (q.md || q.bd) && noncontig && (c->t.n || c->comm)) {
    // A non-warp-contiguous trace is reordered by (cta, warp) for the
    // divergence analyses (regroup_by_warp); reuse distance needs trace order
    // (reading R2), so it gets its own pass over the original columns.
    // Outputs are staged and written only when both passes succeed.
    Req a = q, b = q;
    a.md = a.bd = a.md_sites = a.bd_sites = false;
    b.rd = false;
    const size_t rows = (size_t)q.nobj + 1;
    std::vector<uint64_t> h(rows * q.nbins);
    cadv_reuse_stats st{};
    cadv_status s = run_analyses(c, a, h.data(), rd_stats ? &st : nullptr, nullptr, nullptr, nullptr, nullptr);
    if (s != CADV_OK) return s;
    const float ms = c->elapsed_ms;
    const uint32_t launches = c->launches;
    s = run_analyses(c, b, nullptr, nullptr, md_hist, md_sites, bd_tot, bd_sites);
    if (s != CADV_OK) return s;
    c->elapsed_ms += ms;
    c->launches += launches;
    memcpy(rd_hist, h.data(), h.size() * 8);
    if (rd_stats) *rd_stats = st;
    return CADV_OK;
  }
  if (q.bd) {
    // one T_c generation per call (identical on every rank: calls run in lockstep)
    if (++c->tc_gen >= (1u << 21)) {
      c->tc_gen = 1;
      if (c->tc_buf) CK(cudaMemsetAsync(c->tc_buf, 0, 4ull * c->tc_cap, c->stream), "memset");
    }
  }
  for (int attempt = 0;; ++attempt) {
    cadv_status s = run_once(c, q, rd_hist, rd_stats, md_hist, md_sites, bd_tot, bd_sites);
    if (s != RETRY) return s;
    if (attempt > 4) return fail(c, CADV_ERR_OOM, "workspace did not converge");
  }
}

cadv_status run_once(cadv_ctx* c, const Req& q, uint64_t* rd_hist, cadv_reuse_stats* rd_stats, uint64_t* md_hist,
                     cadv_site_mem* md_sites, uint64_t* bd_tot, cadv_site_branch* bd_sites) {
  const bool multi = c->comm != nullptr;  // also a 1-rank NCCL / loopback context (plumbing tests)
  // (noncontig_any and split_group are all-gathered at load: every rank decides alike)
  if (multi && (q.md || q.bd) && !c->noncontig_any && c->split_group)
    return fail(c, CADV_ERR_BAD_TRACE, "a shard boundary splits a warp-level group (cta, warp, winst)");
  CK(cudaSetDevice(c->device), "cudaSetDevice");
  cadv_status s = begin_call(c);
  if (s != CADV_OK) return s;
  const uint32_t mdW = 1u << q.md_ws;
  const size_t rows = (size_t)q.nobj + 1;
  const size_t o_rdh = 0, o_rds = o_rdh + (q.rd ? rows * q.nbins : 0), o_mdh = o_rds + (q.rd ? 4 : 0);
  const size_t o_mds = o_mdh + (q.md ? rows * 2 * (mdW + 1) : 0);
  const size_t o_mdf = o_mds + (q.md && q.md_sites ? 2ull * q.nsites : 0);
  const size_t o_bdt = o_mdf + (q.md ? 1 : 0);
  const size_t o_bdf = o_bdt + 3;
  const size_t o_bds = o_bdf + 1;
  const size_t total = o_bds + (q.bd && q.bd_sites ? 3ull * q.nsites : 0);
  void* dv;
  CK(ensure(c, B_OUT2, total * 8 + 64, &dv), "workspace");
  CK(cudaMemsetAsync(dv, 0, total * 8 + 64, c->stream), "memset");
  uint64_t* d = (uint64_t*)dv;
  cadv_trace_desc t = c->t;
  if ((q.md || q.bd) && multi && c->noncontig_any) {
    // every (cta, warp32) stream to one rank, in trace order (collective)
    cudaError_t e = exchange_by_warp(c, &t);
    if (e != cudaSuccess) {
      if (!c->comm->err.empty()) return fail(c, CADV_ERR_NCCL, c->comm->err);
      if (e == cudaErrorNotSupported) return fail(c, CADV_ERR_UNSUPPORTED, "a rank would receive >= 2^32 records");
      return cuda_fail(c, e, "exchange by warp");
    }
  } else if ((q.md || q.bd) && !t.warp_contiguous && t.n) {
    CK(regroup_by_warp(c, &t), "regroup by warp");
  }
  // the scan's 1-D TMA copies need 16-byte aligned column bases
  if (t.n && (((uintptr_t)t.addr | (uintptr_t)t.cta | (uintptr_t)t.tid | (uintptr_t)t.site | (uintptr_t)t.winst |
               (uintptr_t)t.meta) & 15)) {
    const void* src[6] = {t.addr, t.cta, t.tid, t.site, t.winst, t.meta};
    const size_t es[6] = {8, 4, 2, 4, 4, 1};
    void* dst[6];
    for (int k = 0; k < 6; ++k) {
      if (!((uintptr_t)src[k] & 15)) { dst[k] = (void*)src[k]; continue; }
      CK(ensure(c, (BufId)(B_ALIGN0 + k), es[k] * t.n + 16, &dst[k]), "workspace");
      CK(cudaMemcpyAsync(dst[k], src[k], es[k] * t.n, cudaMemcpyDeviceToDevice, c->stream), "align copy");
    }
    t.addr = (const uint64_t*)dst[0]; t.cta = (const uint32_t*)dst[1]; t.tid = (const uint16_t*)dst[2];
    t.site = (const uint32_t*)dst[3]; t.winst = (const uint32_t*)dst[4]; t.meta = (const uint8_t*)dst[5];
  }
  ScanParams P;
  P.t = t;
  int flags = 0;
  RdState rs;
  if (q.rd && (t.n || multi)) {
    CK(rd_begin(c, q.scope, &rs), "reuse workspace");
    flags |= F_RD;
    P.lbs_rd = q.rd_lbs;
    P.cta_scope = q.scope == CADV_SCOPE_CTA;
    P.kout = rs.cta_scope ? rs.k1 : nullptr;
    P.vout = rs.v1;
    P.kcap = rs.chunk_cap;
    P.blkcnt = rs.blkcnt;
    P.hist0 = d + o_rdh;
  }
  if (q.md) {
    flags |= F_MD;
    P.lbs_md = q.md_lbs;
    P.ws_md = q.md_ws;
    P.md_hist = d + o_mdh;
    P.md_sites = q.md_sites ? d + o_mds : nullptr;
  }
  void* defer = nullptr;
  if (q.bd && (t.n || multi)) {
    flags |= F_BD;
    if (!c->tc_buf) CK(tc_resize(c, 1u << 16, 0), "workspace");
    if (!c->defer_cap) c->defer_cap = t.n / 8 + 4096;
    CK(ensure(c, B_DEFER, 16ull * c->defer_cap, &defer), "workspace");
    P.ws_bd = q.bd_ws;
    P.tc = c->tc_buf;
    P.tc_cap = c->tc_cap;
    P.tc_gen = c->tc_gen;
    P.defer_cap = c->defer_cap;
    P.bd_tot = d + o_bdt;
    P.bd_sites = q.bd_sites ? d + o_bds : nullptr;
    P.defer = defer;
    P.ndefer = &scalars(c)->ndefer;
  }
  P.nsites = (q.md_sites || q.bd_sites) ? q.nsites : 0;
  if (q.nobj) {
    flags |= F_OBJ;
    P.obj_lo = q.obj_lo;
    P.obj_hi = q.obj_hi;
    P.nobj = q.nobj;
    P.rd_nbins = q.nbins;
  }
  // one flag word for both site checks
  P.site_flag = d + (q.md ? o_mdf : o_bdf);
  if (flags && t.n) CK(launch_scan(c, flags, P), "scan launch");
  // R0 results of the pass: CTA-id range, T_c / deferred-group capacity; the
  // reuse compaction is queued behind them, so one synchronisation covers both
  bool again = false;  // workspace grown: run the call again
  {
    Scalars* hsp = (Scalars*)((uint8_t*)c->hstage + 64);
    CK(cudaMemcpyAsync(hsp, scalars(c), sizeof(Scalars), cudaMemcpyDeviceToHost, c->stream), "D2H");
    if (q.rd && (t.n || multi)) CK(rd_compact(c, rs), "reuse compaction");
    CK(cudaStreamSynchronize(c->stream), "scan");
    const Scalars hs = *hsp;
    c->max_cta = (uint32_t)hs.max_cta;
    // one rank: a bad / unsupported record ends the call here (its report
    // comes from end_call); several ranks first agree (below)
    if (!multi && (hs.err_code || hs.unsup_index != ~0ull)) {
      void* h0;
      s = end_call(c, nullptr, 0, &h0);
      return s != CADV_OK ? s : fail(c, CADV_ERR_BAD_TRACE, "invalid trace");
    }
    if (q.bd && t.n) {
      if (!multi && hs.max_cta >= (1u << 28)) return fail(c, CADV_ERR_UNSUPPORTED, "CTA ids must be < 2^28");
      if (hs.tc_overflow) {
        uint64_t cap = (uint64_t)c->tc_cap * 2;
        if (cap < hs.max_cta + 1) cap = hs.max_cta + 1;
        CK(tc_resize(c, (uint32_t)cap, 0), "workspace");
        again = true;
      }
      if (hs.ndefer > c->defer_cap) {
        c->defer_cap = hs.ndefer + hs.ndefer / 4 + 4096;
        again = true;
      }
    }
    if (q.rd && hs.kept_max > rs.chunk_cap) {  // a warp's kept records overflowed its region
      c->kcap_min = hs.kept_max + hs.kept_max / 8;
      again = true;
    }
    if (again && !hs.err_code && !multi) return RETRY;
  }
  if (multi) {
    // every rank learns whether any rank found a bad record / site id before
    // the exchanges (a failing rank must not leave the others in a collective)
    void* fb;
    CK(ensure(c, B_COMM, 64, &fb), "workspace");
    uint32_t* df = (uint32_t*)fb;
    CADV_LAUNCH(c, k_agree_flags<<<1, 32, 0, c->stream>>>(scalars(c), q.md ? d + o_mdf : nullptr,
                                                          q.bd ? d + o_bdf : nullptr, again ? 1u : 0u, df));
    if (c->comm->allreduce_max_u32(df, 5, c->stream)) return fail(c, CADV_ERR_NCCL, c->comm->err);
    uint32_t hf[5];
    CK(cudaMemcpyAsync(hf, df, 20, cudaMemcpyDeviceToHost, c->stream), "D2H");
    CK(cudaStreamSynchronize(c->stream), "scan");
    c->max_cta = hf[2];  // global CTA-id range
    if (hf[0] || hf[1] || hf[3]) {
      void* h0;
      s = end_call(c, nullptr, 0, &h0);  // reports this rank's own bad record, if it has one
      if (s != CADV_OK) return s;
      if (hf[0]) return fail(c, CADV_ERR_BAD_TRACE, "invalid record or warp-level group on another rank");
      if (hf[3]) return fail(c, CADV_ERR_UNSUPPORTED, "a reuse-distance line >= 2^58 on another rank");
      return fail(c, CADV_ERR_INVALID_ARG, "a record's site id is >= nsites (on some rank)");
    }
    if (q.bd && c->max_cta >= (1u << 28)) return fail(c, CADV_ERR_UNSUPPORTED, "CTA ids must be < 2^28");
    if (hf[4]) return RETRY;  // some rank grew its workspace: every rank runs the call again
  }
  if (q.rd && (t.n || multi)) {
    const ObjTab ot{q.obj_lo, q.obj_hi, q.nobj};
    cudaError_t e = rd_finish(c, rs, q.log2bins, q.nbins, d + o_rdh, d + o_rds, &ot);
    if (e != cudaSuccess) {
      if (multi && !c->comm->err.empty()) return fail(c, CADV_ERR_NCCL, c->comm->err);
      return cuda_fail(c, e, "reuse");
    }
  }
  if (q.bd && (t.n || multi)) {
    if (multi) {
      if (c->max_cta >= (1u << 28)) return fail(c, CADV_ERR_UNSUPPORTED, "CTA ids must be < 2^28");
      if (c->tc_cap < c->max_cta + 1) CK(tc_resize(c, c->max_cta + 1, c->tc_cap), "workspace");
      if (c->comm->allreduce_max_u32(c->tc_buf, c->max_cta + 1, c->stream))
        return fail(c, CADV_ERR_NCCL, c->comm->err);
    }
    // the deferred-group count stays on the device (the scan's read-back
    // already checked it against the capacity)
    CK(launch_bd_resolve(c, defer, P.ndefer, c->defer_cap, c->tc_buf, c->tc_gen, q.bd_ws, d + o_bdt,
                         q.bd_sites ? d + o_bds : nullptr, q.bd_sites ? q.nsites : 0),
       "bd resolve");
  }
  if (multi && c->comm->allreduce_sum_u64(d, total, c->stream)) return fail(c, CADV_ERR_NCCL, c->comm->err);
  void* h;
  s = end_call(c, d, total * 8, &h);
  if (s != CADV_OK) return s;
  const uint64_t* hr = (const uint64_t*)h;
  if ((q.md && hr[o_mdf]) || (q.bd && hr[o_bdf]))
    return fail(c, CADV_ERR_INVALID_ARG, "a record's site id is >= nsites");
  if (q.rd) {
    memcpy(rd_hist, hr + o_rdh, rows * q.nbins * 8);
    if (rd_stats) {  // (single row: not a data-centric call)
      uint64_t acc = 0;
      for (uint32_t b = 0; b < q.nbins; ++b) acc += hr[o_rdh + b];
      rd_stats->accesses = acc;
      rd_stats->inf = hr[o_rdh + q.nbins - 1];
      rd_stats->overflow = hr[o_rdh + q.nbins - 2];
      rd_stats->streaming = hr[o_rds];
      rd_stats->finite_sum = hr[o_rds + 1];
    }
  }
  if (q.md) {
    memcpy(md_hist, hr + o_mdh, rows * 2 * (mdW + 1) * 8);
    if (q.md_sites) memcpy(md_sites, hr + o_mds, 2ull * q.nsites * 8);
  }
  if (q.bd) {
    memcpy(bd_tot, hr + o_bdt, 3 * 8);
    if (q.bd_sites) memcpy(bd_sites, hr + o_bds, 3ull * q.nsites * 8);
  }
  return CADV_OK;
}

}  // namespace

extern "C" {

CADV_API cadv_status cadv_mem_divergence(cadv_ctx* c, uint32_t line_bytes, uint32_t warp_size, uint64_t* hist,
                                         cadv_site_mem* per_site, uint32_t nsites) {
  if (!c) return CADV_ERR_INVALID_ARG;
  c->err.clear();
  cadv_status s = check_args(c, line_bytes, warp_size, true, true);
  if (s != CADV_OK) return s;
  if (!hist) return fail(c, CADV_ERR_INVALID_ARG, "hist is NULL");
  if (per_site && nsites == 0) return fail(c, CADV_ERR_INVALID_ARG, "nsites must be > 0 with per_site");
  Req q;
  q.md = true;
  q.md_lbs = ilog2(line_bytes);
  q.md_ws = ilog2(warp_size);
  q.md_sites = per_site != nullptr;
  q.nsites = per_site ? nsites : 0;
  return run_analyses(c, q, nullptr, nullptr, hist, per_site, nullptr, nullptr);
}

CADV_API cadv_status cadv_branch_divergence(cadv_ctx* c, uint32_t warp_size, cadv_site_branch* per_site,
                                            uint32_t nsites, uint64_t totals[3]) {
  if (!c) return CADV_ERR_INVALID_ARG;
  c->err.clear();
  cadv_status s = check_args(c, 1, warp_size, false, true);
  if (s != CADV_OK) return s;
  if (!totals) return fail(c, CADV_ERR_INVALID_ARG, "totals is NULL");
  if (per_site && nsites == 0) return fail(c, CADV_ERR_INVALID_ARG, "nsites must be > 0 with per_site");
  Req q;
  q.bd = true;
  q.bd_ws = ilog2(warp_size);
  q.bd_sites = per_site != nullptr;
  q.nsites = per_site ? nsites : 0;
  return run_analyses(c, q, nullptr, nullptr, nullptr, nullptr, totals, per_site);
}

CADV_API cadv_status cadv_reuse_histogram(cadv_ctx* c, uint32_t line_bytes, int scope, int binning, uint64_t* hist,
                                          uint32_t nbins, cadv_reuse_stats* stats) {
  if (!c) return CADV_ERR_INVALID_ARG;
  c->err.clear();
  cadv_status s = check_args(c, line_bytes, 32, true, false);
  if (s != CADV_OK) return s;
  if (scope != CADV_SCOPE_CTA && scope != CADV_SCOPE_KERNEL) return fail(c, CADV_ERR_INVALID_ARG, "bad scope");
  if (binning != CADV_BINS_LINEAR && binning != CADV_BINS_LOG2) return fail(c, CADV_ERR_INVALID_ARG, "bad binning");
  if (nbins < 3 || !hist) return fail(c, CADV_ERR_INVALID_ARG, "nbins must be >= 3 and hist non-NULL");
  Req q;
  q.rd = true;
  q.rd_lbs = ilog2(line_bytes);
  q.scope = scope;
  q.log2bins = binning == CADV_BINS_LOG2;
  q.nbins = nbins;
  return run_analyses(c, q, hist, stats, nullptr, nullptr, nullptr, nullptr);
}

CADV_API cadv_status cadv_analyze(cadv_ctx* c, const cadv_analysis* a, uint64_t* rd_hist, cadv_reuse_stats* rd_stats,
                                  uint64_t* md_hist, cadv_site_mem* md_sites, uint64_t* bd_totals,
                                  cadv_site_branch* bd_sites) {
  if (!c || !a) return CADV_ERR_INVALID_ARG;
  c->err.clear();
  Req q;
  q.rd = rd_hist != nullptr;
  q.md = md_hist != nullptr;
  q.bd = bd_totals != nullptr;
  if (!q.rd && !q.md && !q.bd) return fail(c, CADV_ERR_INVALID_ARG, "no analysis requested");
  cadv_status s = check_args(c, q.rd ? a->rd_line_bytes : 1, 32, q.rd, false);
  if (s == CADV_OK) s = check_args(c, q.md ? a->md_line_bytes : 1, q.md ? a->md_warp_size : 32, q.md, q.md);
  if (s == CADV_OK) s = check_args(c, 1, q.bd ? a->bd_warp_size : 32, false, q.bd);
  if (s != CADV_OK) return s;
  if (q.rd) {
    if (a->rd_scope != CADV_SCOPE_CTA && a->rd_scope != CADV_SCOPE_KERNEL) return fail(c, CADV_ERR_INVALID_ARG, "bad scope");
    if (a->rd_binning != CADV_BINS_LINEAR && a->rd_binning != CADV_BINS_LOG2)
      return fail(c, CADV_ERR_INVALID_ARG, "bad binning");
    if (a->rd_nbins < 3) return fail(c, CADV_ERR_INVALID_ARG, "nbins must be >= 3");
    q.rd_lbs = ilog2(a->rd_line_bytes);
    q.scope = a->rd_scope;
    q.log2bins = a->rd_binning == CADV_BINS_LOG2;
    q.nbins = a->rd_nbins;
  }
  if ((md_sites || bd_sites) && a->nsites == 0) return fail(c, CADV_ERR_INVALID_ARG, "nsites must be > 0 with per_site");
  if (q.md) {
    q.md_lbs = ilog2(a->md_line_bytes);
    q.md_ws = ilog2(a->md_warp_size);
    q.md_sites = md_sites != nullptr;
  }
  if (q.bd) {
    q.bd_ws = ilog2(a->bd_warp_size);
    q.bd_sites = bd_sites != nullptr;
  }
  q.nsites = a->nsites;
  return run_analyses(c, q, rd_hist, rd_stats, md_hist, md_sites, bd_totals, bd_sites);
}

CADV_API cadv_status cadv_data_centric(cadv_ctx* c, const cadv_object* objs, uint32_t nobj, uint32_t line_bytes,
                                       int scope, int binning, uint32_t nbins, uint32_t warp_size, uint64_t* rd_hist,
                                       uint64_t* md_hist) {
  if (!c) return CADV_ERR_INVALID_ARG;
  c->err.clear();
  if (!rd_hist && !md_hist) return fail(c, CADV_ERR_INVALID_ARG, "no analysis requested");
  cadv_status s = check_args(c, line_bytes, md_hist ? warp_size : 32, true, md_hist != nullptr);
  if (s != CADV_OK) return s;
  if (nobj && !objs) return fail(c, CADV_ERR_INVALID_ARG, "objs is NULL");
  if (nobj > (1u << 24)) return fail(c, CADV_ERR_INVALID_ARG, "more than 2^24 objects");
  Req q;
  if (rd_hist) {
    if (scope != CADV_SCOPE_CTA && scope != CADV_SCOPE_KERNEL) return fail(c, CADV_ERR_INVALID_ARG, "bad scope");
    if (binning != CADV_BINS_LINEAR && binning != CADV_BINS_LOG2) return fail(c, CADV_ERR_INVALID_ARG, "bad binning");
    if (nbins < 3) return fail(c, CADV_ERR_INVALID_ARG, "nbins must be >= 3");
    q.rd = true;
    q.rd_lbs = ilog2(line_bytes);
    q.scope = scope;
    q.log2bins = binning == CADV_BINS_LOG2;
    q.nbins = nbins;
  }
  if (md_hist) {
    q.md = true;
    q.md_lbs = ilog2(line_bytes);
    q.md_ws = ilog2(warp_size);
  }
  // line extents: [base / L, ceil((base + bytes) / L)), ascending and disjoint
  const uint32_t lbs = ilog2(line_bytes);
  std::vector<uint64_t> ext(2ull * nobj);
  for (uint32_t k = 0; k < nobj; ++k) {
    const uint64_t b = objs[k].base, nb = objs[k].bytes;
    if (nb == 0 || b + nb < b) return fail(c, CADV_ERR_INVALID_ARG, "object " + std::to_string(k) + ": empty or wraps");
    ext[k] = b >> lbs;
    ext[nobj + k] = ((b + nb - 1) >> lbs) + 1;
    if (k && ext[nobj + k - 1] > ext[k])
      return fail(c, CADV_ERR_INVALID_ARG,
                  "objects " + std::to_string(k - 1) + " and " + std::to_string(k) + " are not ascending / share a line");
  }
  if (nobj) {
    void* dv;
    CK(cudaSetDevice(c->device), "cudaSetDevice");
    CK(ensure(c, B_OBJ, ext.size() * 8, &dv), "workspace");
    CK(cudaMemcpyAsync(dv, ext.data(), ext.size() * 8, cudaMemcpyHostToDevice, c->stream), "H2D");
    CK(cudaStreamSynchronize(c->stream), "H2D");
    q.nobj = nobj;
    q.obj_lo = (const uint64_t*)dv;
    q.obj_hi = (const uint64_t*)dv + nobj;
  }
  return run_analyses(c, q, rd_hist, nullptr, md_hist, nullptr, nullptr, nullptr);
}

}  // extern "C"
