// cadv.cu — the C ABI of libcadv (include/cadv.h): context, trace
// registration + ingest pass R0, and the synchronous analysis entry points.
#include <cuda_runtime.h>
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
      cudaFree(b.p);
      b.p = nullptr;
      b.bytes = 0;
    }
    size_t want = bytes + bytes / 8;  // headroom so slightly larger calls do not reallocate
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
  if (!c->profiling) return;
  uint32_t k = c->nprof;
  while (c->prof_ev.size() < 2ull * (k + 1)) {
    cudaEvent_t e;
    if (cudaEventCreate(&e) != cudaSuccess) { c->profiling = false; return; }
    c->prof_ev.push_back(e);
  }
  if (c->prof_src.size() <= k) c->prof_src.resize(k + 1);
  c->prof_src[k] = src;
  cudaEventRecord(c->prof_ev[2 * k], c->stream);
}

void prof_end(cadv_ctx* c) {
  if (!c->profiling || c->prof_ev.size() < 2ull * (c->nprof + 1)) return;
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
    size_t sp = nm.find_last_of(" (,");
    if (sp != std::string::npos) nm = nm.substr(sp + 1);
    c->prof_name[k] = nm;
  }
}

// ------------------------------------------------------------------ R0 ingest
// One streaming pass over (cta, meta): max CTA id and record count per kind.
__global__ void __launch_bounds__(256) k_ingest(const uint32_t* __restrict__ cta, const uint8_t* __restrict__ meta,
                                                uint64_t n, Scalars* s) {
  uint32_t mx = 0;
  uint32_t cnt[4] = {0, 0, 0, 0};
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    mx = max(mx, __ldg(cta + i));
    cnt[__ldg(meta + i) & 3u]++;
  }
  mx = __reduce_max_sync(FULL, mx);
#pragma unroll
  for (int k = 0; k < 4; ++k) cnt[k] = __reduce_add_sync(FULL, cnt[k]);
  if (lane_id() == 0) {
    atomicMax(&s->max_cta, (unsigned long long)mx);
#pragma unroll
    for (int k = 0; k < 4; ++k)
      if (cnt[k]) atomicAdd(&s->n_kind[k], (unsigned long long)cnt[k]);
  }
}

cudaError_t launch_ingest(cadv_ctx* c) {
  uint64_t n = c->t.n;
  if (n == 0) return cudaSuccess;
  uint64_t want = (n + 255) / 256;
  int grid = (int)(want < (uint64_t)c->num_sms * 8 ? want : (uint64_t)c->num_sms * 8);
  CADV_LAUNCH(c, k_ingest<<<grid, 256, 0, c->stream>>>(c->t.cta, c->t.meta, n, scalars(c)));
  return cudaGetLastError();
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
                                 "trace invariant violated",
             (unsigned long long)(hs->err_index == ~0ull ? 0 : hs->err_index + c->global_offset));
    return fail(c, CADV_ERR_BAD_TRACE, b);
  }
  *h_out = hr;
  return CADV_OK;
}

}  // namespace

extern "C" {

CADV_API const char* cadv_version(void) { return "cadv 0.1 (sm_100a)"; }

CADV_API cadv_status cadv_create(cadv_ctx** out, int device, void* cuda_stream, const void* nccl_unique_id, int rank,
                                 int nranks) {
  if (!out) return CADV_ERR_INVALID_ARG;
  *out = nullptr;
  if (nranks < 1 || rank < 0 || rank >= nranks) return CADV_ERR_INVALID_ARG;
  if (nranks > 1 && !nccl_unique_id) return CADV_ERR_INVALID_ARG;
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
  if (cudaEventCreate(&c->ev0) != cudaSuccess || cudaEventCreate(&c->ev1) != cudaSuccess) {
    delete c;
    return CADV_ERR_CUDA;
  }
  if (nranks > 1) {
    c->err = "multi-rank contexts are not available in this build";
    delete c;
    return CADV_ERR_UNSUPPORTED;
  }
  *out = c;
  return CADV_OK;
}

CADV_API cadv_status cadv_destroy(cadv_ctx* c) {
  if (!c) return CADV_ERR_INVALID_ARG;
  cudaSetDevice(c->device);
  cudaStreamSynchronize(c->stream);
  for (auto& b : c->buf)
    if (b.p) cudaFree(b.p);
  if (c->host_pinned) cudaFreeHost(c->host_pinned);
  if (c->ev0) cudaEventDestroy(c->ev0);
  if (c->ev1) cudaEventDestroy(c->ev1);
  for (auto e : c->prof_ev) cudaEventDestroy(e);
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
  c->profiling = enable != 0;
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
  cadv_status s = begin_call(c);
  if (s != CADV_OK) return s;
  c->t = *d;
  c->t.on_device = 1;
  c->global_offset = global_offset;
  if (!d->on_device && d->n) {
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
  CK(launch_ingest(c), "ingest launch");
  void* h;
  s = end_call(c, nullptr, 0, &h);
  if (s != CADV_OK) return s;
  Scalars* hs = (Scalars*)c->host_pinned;
  c->max_cta = (uint32_t)hs->max_cta;
  for (int k = 0; k < 4; ++k) c->n_kind[k] = hs->n_kind[k];
  c->loaded = true;
  return CADV_OK;
}

CADV_API cadv_status cadv_mem_divergence(cadv_ctx* c, uint32_t line_bytes, uint32_t warp_size, uint64_t* hist,
                                         cadv_site_mem* per_site, uint32_t nsites) {
  if (!c) return CADV_ERR_INVALID_ARG;
  c->err.clear();
  if (!c->loaded) return fail(c, CADV_ERR_NO_TRACE, "no trace loaded");
  if (!pow2(line_bytes) || line_bytes > 4096) return fail(c, CADV_ERR_INVALID_ARG, "line_bytes must be 2^k <= 4096");
  if (!pow2(warp_size) || warp_size > 32) return fail(c, CADV_ERR_INVALID_ARG, "warp_size must be 2^k <= 32");
  if (!hist) return fail(c, CADV_ERR_INVALID_ARG, "hist is NULL");
  if (per_site && nsites == 0) return fail(c, CADV_ERR_INVALID_ARG, "nsites must be > 0 with per_site");
  CK(cudaSetDevice(c->device), "cudaSetDevice");
  cadv_status s = begin_call(c);
  if (s != CADV_OK) return s;
  size_t hbytes = 2ull * (warp_size + 1) * 8, sbytes = per_site ? 2ull * nsites * 8 : 0;
  void* d_out;
  CK(ensure(c, B_HIST, hbytes + sbytes + 8, &d_out), "workspace");
  CK(cudaMemsetAsync(d_out, 0, hbytes + sbytes + 8, c->stream), "memset");
  cadv_trace_desc t = c->t;
  if (!t.warp_contiguous && t.n) CK(regroup_by_warp(c, &t), "regroup by warp");
  CK(launch_mem_div(c, t, ilog2(line_bytes), ilog2(warp_size), (uint64_t*)d_out,
                    per_site ? (uint64_t*)d_out + 2 * (warp_size + 1) : nullptr, per_site ? nsites : 0),
     "mem_div launch");
  void* h;
  s = end_call(c, d_out, hbytes + sbytes + 8, &h);
  if (s != CADV_OK) return s;
  const uint64_t* hr = (const uint64_t*)h;
  if (per_site && hr[2 * (warp_size + 1) + 2 * nsites])
    return fail(c, CADV_ERR_INVALID_ARG, "a memory record's site id is >= nsites");
  memcpy(hist, hr, hbytes);
  if (per_site) memcpy(per_site, hr + 2 * (warp_size + 1), sbytes);
  return CADV_OK;
}

CADV_API cadv_status cadv_branch_divergence(cadv_ctx* c, uint32_t warp_size, cadv_site_branch* per_site,
                                            uint32_t nsites, uint64_t totals[3]) {
  if (!c) return CADV_ERR_INVALID_ARG;
  c->err.clear();
  if (!c->loaded) return fail(c, CADV_ERR_NO_TRACE, "no trace loaded");
  if (!pow2(warp_size) || warp_size > 32) return fail(c, CADV_ERR_INVALID_ARG, "warp_size must be 2^k <= 32");
  if (!totals) return fail(c, CADV_ERR_INVALID_ARG, "totals is NULL");
  if (per_site && nsites == 0) return fail(c, CADV_ERR_INVALID_ARG, "nsites must be > 0 with per_site");
  if (c->t.n && c->max_cta >= (1u << 28)) return fail(c, CADV_ERR_UNSUPPORTED, "CTA ids must be < 2^28");
  CK(cudaSetDevice(c->device), "cudaSetDevice");
  cadv_status s = begin_call(c);
  if (s != CADV_OK) return s;
  size_t tbytes = 4 * 8, sbytes = per_site ? 3ull * nsites * 8 : 0;
  void* d_out;
  CK(ensure(c, B_HIST, tbytes + sbytes, &d_out), "workspace");
  CK(cudaMemsetAsync(d_out, 0, tbytes + sbytes, c->stream), "memset");
  uint32_t ncta = c->t.n ? c->max_cta + 1 : 1;
  void* d_tc;
  CK(ensure(c, B_TC, 4ull * ncta, &d_tc), "workspace");
  CK(cudaMemsetAsync(d_tc, 0, 4ull * ncta, c->stream), "memset");
  cadv_trace_desc t = c->t;
  if (t.n) {
    CK(launch_cta_maxtid(c, t, (uint32_t*)d_tc, ncta), "maxtid launch");
    if (!t.warp_contiguous) CK(regroup_by_warp(c, &t), "regroup by warp");
    CK(launch_branch_div(c, t, ilog2(warp_size), (const uint32_t*)d_tc,
                         per_site ? (uint64_t*)d_out + 4 : nullptr, per_site ? nsites : 0, (uint64_t*)d_out),
       "branch_div launch");
  }
  void* h;
  s = end_call(c, d_out, tbytes + sbytes, &h);
  if (s != CADV_OK) return s;
  const uint64_t* hr = (const uint64_t*)h;
  if (per_site && hr[3]) return fail(c, CADV_ERR_INVALID_ARG, "a basic-block record's site id is >= nsites");
  memcpy(totals, hr, 3 * 8);
  if (per_site) memcpy(per_site, hr + 4, sbytes);
  return CADV_OK;
}

CADV_API cadv_status cadv_reuse_histogram(cadv_ctx* c, uint32_t line_bytes, int scope, int binning, uint64_t* hist,
                                          uint32_t nbins, cadv_reuse_stats* stats) {
  if (!c) return CADV_ERR_INVALID_ARG;
  c->err.clear();
  if (!c->loaded) return fail(c, CADV_ERR_NO_TRACE, "no trace loaded");
  if (!pow2(line_bytes) || line_bytes > 4096) return fail(c, CADV_ERR_INVALID_ARG, "line_bytes must be 2^k <= 4096");
  if (scope != CADV_SCOPE_CTA && scope != CADV_SCOPE_KERNEL) return fail(c, CADV_ERR_INVALID_ARG, "bad scope");
  if (binning != CADV_BINS_LINEAR && binning != CADV_BINS_LOG2) return fail(c, CADV_ERR_INVALID_ARG, "bad binning");
  if (nbins < 3 || !hist) return fail(c, CADV_ERR_INVALID_ARG, "nbins must be >= 3 and hist non-NULL");
  CK(cudaSetDevice(c->device), "cudaSetDevice");
  cadv_status s = begin_call(c);
  if (s != CADV_OK) return s;
  size_t hbytes = (size_t)nbins * 8;
  void* d_out;
  CK(ensure(c, B_HIST, hbytes + 64, &d_out), "workspace");
  CK(cudaMemsetAsync(d_out, 0, hbytes + 64, c->stream), "memset");
  uint64_t* d_stats = (uint64_t*)((uint8_t*)d_out + hbytes);
  if (c->t.n) CK(run_reuse(c, ilog2(line_bytes), scope, binning == CADV_BINS_LOG2, nbins, (uint64_t*)d_out, d_stats),
                 "reuse");
  void* h;
  s = end_call(c, d_out, hbytes + 32, &h);
  if (s != CADV_OK) return s;
  const uint64_t* hr = (const uint64_t*)h;
  memcpy(hist, hr, hbytes);
  if (stats) {
    uint64_t acc = 0;
    for (uint32_t b = 0; b < nbins; ++b) acc += hr[b];
    stats->accesses = acc;
    stats->inf = hr[nbins - 1];
    stats->overflow = hr[nbins - 2];
    stats->streaming = hr[nbins + 0];
  }
  return CADV_OK;
}

}  // extern "C"
