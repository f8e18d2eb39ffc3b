// sort.cu — device-wide primitives: exclusive scans and a stable LSD radix
// sort of (key, value) pairs, plus the (cta, warp) regroup for traces that
// are not warp-contiguous.
//
// Radix sort: per pass of <= 8 bits, (1) every 4096-element tile counts its
// digits in shared memory (warp-aggregated with __match_any_sync), (2) the
// digit-major [digit][tile] count matrix is exclusive-scanned, (3) every
// tile ranks its elements stably — warp by warp, 32 elements at a time, with
// __match_any_sync giving the rank among equal digits in the same round and
// per-warp digit counters in shared memory giving the rank across rounds —
// and scatters them.  Stability is what the CTA regroup of the reuse path
// needs (within-CTA order is the access order).
#include <cuda_runtime.h>

#include "cadv_impl.h"
#include "common.cuh"

namespace cadv {
namespace {

constexpr int SCAN_NT = 512;
constexpr int SCAN_CH = 4096;  // elements per scan block (8 per thread)

template <typename T>
__device__ __forceinline__ T warp_incl_scan(T x) {
  const uint32_t lane = lane_id();
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T y = __shfl_up_sync(FULL, x, o);
    if (lane >= (uint32_t)o) x += y;
  }
  return x;
}

// Block-wide exclusive scan of one T per thread; returns prefix, *tot = sum.
template <typename T, int NT>
__device__ __forceinline__ T block_scan_t(T v, T* ws, T* tot) {
  const uint32_t lane = lane_id(), warp = threadIdx.x >> 5;
  T x = warp_incl_scan(v);
  if (lane == 31) ws[warp] = x;
  __syncthreads();
  if (warp == 0) {
    T s = lane < NT / 32 ? ws[lane] : T(0);
    s = warp_incl_scan(s);
    if (lane < NT / 32) ws[lane] = s;
  }
  __syncthreads();
  T base = warp ? ws[warp - 1] : T(0);
  *tot = ws[NT / 32 - 1];
  __syncthreads();
  return base + x - v;
}

template <typename T>
__global__ void __launch_bounds__(SCAN_NT) k_scan_reduce(const T* __restrict__ in, uint64_t n, T* __restrict__ part) {
  __shared__ T ws[SCAN_NT / 32];
  uint64_t base = (uint64_t)blockIdx.x * SCAN_CH;
  T s = 0;
  for (int k = 0; k < SCAN_CH / SCAN_NT; ++k) {
    uint64_t i = base + (uint64_t)k * SCAN_NT + threadIdx.x;
    if (i < n) s += in[i];
  }
  T tot;
  block_scan_t<T, SCAN_NT>(s, ws, &tot);
  if (threadIdx.x == 0) part[blockIdx.x] = tot;
}

// Exclusive scan of one chunk per block, offset by part[block] (if given).
template <typename T>
__global__ void __launch_bounds__(SCAN_NT) k_scan_chunk(const T* in, T* out, uint64_t n, const T* __restrict__ part,
                                                        T* d_total) {
  __shared__ T ws[SCAN_NT / 32];
  constexpr int IPT = SCAN_CH / SCAN_NT;
  uint64_t base = (uint64_t)blockIdx.x * SCAN_CH + (uint64_t)threadIdx.x * IPT;
  T v[IPT];
  T s = 0;
#pragma unroll
  for (int k = 0; k < IPT; ++k) {
    uint64_t i = base + k;
    v[k] = i < n ? in[i] : T(0);
    s += v[k];
  }
  T tot;
  T run = block_scan_t<T, SCAN_NT>(s, ws, &tot) + (part ? part[blockIdx.x] : T(0));
#pragma unroll
  for (int k = 0; k < IPT; ++k) {
    uint64_t i = base + k;
    if (i < n) out[i] = run;
    run += v[k];
  }
  if (d_total && blockIdx.x == gridDim.x - 1 && threadIdx.x == SCAN_NT - 1) *d_total = run;
}

// Exclusive scan of up to SCAN_SMALL elements in ONE launch (one block of
// 1024 threads, each a contiguous run): the scans of the reuse path's
// region counts, pair counts and radix digit matrices are this size, and a
// single launch beats reduce + scan-of-partials + chunk (three dependent
// launches, each a few microseconds of latency).  In place is allowed.
constexpr int SCAN_SMALL_NT = 1024;
constexpr uint64_t SCAN_SMALL = 128 * 1024;
template <typename T>
__global__ void __launch_bounds__(SCAN_SMALL_NT) k_scan_small(const T* in, T* out, uint64_t n, T* d_total) {
  __shared__ T ws[SCAN_SMALL_NT / 32];
  const uint64_t per = (n + SCAN_SMALL_NT - 1) / SCAN_SMALL_NT;
  const uint64_t lo = threadIdx.x * per, hi = lo + per < n ? lo + per : n;
  T s = 0;
  for (uint64_t i = lo; i < hi; ++i) s += in[i];
  T tot;
  T run = block_scan_t<T, SCAN_SMALL_NT>(s, ws, &tot);
  for (uint64_t i = lo; i < hi; ++i) {
    const T v = in[i];
    out[i] = run;
    run += v;
  }
  if (d_total && threadIdx.x == 0) *d_total = tot;
}

template <typename T>
cudaError_t scan_impl(cadv_ctx* c, const T* in, T* out, uint64_t n, T* d_total, int depth) {
  if (n == 0) return cudaSuccess;
  uint64_t nb = (n + SCAN_CH - 1) / SCAN_CH;
  if (nb > 1 && n <= SCAN_SMALL && depth == 0) {
    CADV_LAUNCH(c, k_scan_small<T><<<1, SCAN_SMALL_NT, 0, c->stream>>>(in, out, n, d_total));
    return cudaGetLastError();
  }
  if (nb == 1) {
    CADV_LAUNCH(c, k_scan_chunk<T><<<1, SCAN_NT, 0, c->stream>>>(in, out, n, nullptr, d_total));
    return cudaGetLastError();
  }
  // partial sums live in the scan scratch buffer, one level after another
  void* tmp;
  uint64_t need = 0, m = nb;
  for (int d = 0; m > 1; ++d) { need += m + 1; m = (m + SCAN_CH - 1) / SCAN_CH; }
  cudaError_t e = ensure(c, B_SCAN_TMP, (need + 64) * sizeof(T) * 2, &tmp);
  if (e != cudaSuccess) return e;
  // offset by depth so that recursion levels do not overlap
  T* part = (T*)tmp;
  uint64_t off = 0;
  m = (n + SCAN_CH - 1) / SCAN_CH;
  for (int d = 0; d < depth; ++d) { off += m + 1; m = (m + SCAN_CH - 1) / SCAN_CH; }
  part += off + 1;
  CADV_LAUNCH(c, k_scan_reduce<T><<<(unsigned)nb, SCAN_NT, 0, c->stream>>>(in, n, part));
  e = scan_impl<T>(c, part, part, nb, nullptr, depth + 1);
  if (e != cudaSuccess) return e;
  CADV_LAUNCH(c, k_scan_chunk<T><<<(unsigned)nb, SCAN_NT, 0, c->stream>>>(in, out, n, part, d_total));
  return cudaGetLastError();
}

// ------------------------------------------------------------------ radix sort
constexpr int RS_NT = 256;
constexpr int RS_IPT = 16;
constexpr int RS_TILE = RS_NT * RS_IPT;  // 4096
constexpr int RS_WARPS = RS_NT / 32;
constexpr int RS_PER_WARP = RS_TILE / RS_WARPS;  // 512 = 16 rounds of 32
constexpr int RS_MAXB = 9;                        // digit bits per pass (<= 512 buckets)

template <typename K>
__device__ __forceinline__ uint32_t digit(K k, int shift, uint32_t mask) {
  return (uint32_t)(k >> shift) & mask;
}

template <typename K>
__global__ void __launch_bounds__(RS_NT) k_rs_upsweep(const K* __restrict__ keys, uint64_t n, int shift, int bits,
                                                      uint32_t* __restrict__ counts, uint64_t ntiles) {
  __shared__ uint32_t h[1 << RS_MAXB];
  const uint32_t radix = 1u << bits, mask = radix - 1;
  for (uint32_t k = threadIdx.x; k < radix; k += RS_NT) h[k] = 0;
  __syncthreads();
  const uint32_t lane = lane_id(), warp = threadIdx.x >> 5;
  uint64_t base = (uint64_t)blockIdx.x * RS_TILE + (uint64_t)warp * RS_PER_WARP;
#pragma unroll 4
  for (int r = 0; r < RS_PER_WARP / 32; ++r) {
    uint64_t i = base + (uint64_t)r * 32 + lane;
    uint32_t d = i < n ? digit(keys[i], shift, mask) : 0xffffffffu;
    uint32_t m = __match_any_sync(FULL, d);
    if (d != 0xffffffffu && (uint32_t)(__ffs(m) - 1) == lane) atomicAdd(&h[d], (uint32_t)__popc(m));
  }
  __syncthreads();
  for (uint32_t k = threadIdx.x; k < radix; k += RS_NT) counts[(uint64_t)k * ntiles + blockIdx.x] = h[k];
}

template <typename K, typename V>
__global__ void __launch_bounds__(RS_NT) k_rs_scatter(const K* __restrict__ kin, const V* __restrict__ vin,
                                                      K* __restrict__ kout, V* __restrict__ vout, uint64_t n,
                                                      int shift, int bits, const uint32_t* __restrict__ offs,
                                                      uint64_t ntiles) {
  __shared__ uint32_t wc[RS_WARPS][1 << RS_MAXB];
  const uint32_t radix = 1u << bits, mask = radix - 1;
  const uint32_t lane = lane_id(), warp = threadIdx.x >> 5;
  for (uint32_t k = lane; k < radix; k += 32) wc[warp][k] = 0;
  __syncwarp();
  uint64_t base = (uint64_t)blockIdx.x * RS_TILE + (uint64_t)warp * RS_PER_WARP;
  K kr[RS_IPT];
  V vr[RS_IPT];
  uint32_t rk[RS_IPT];
#pragma unroll
  for (int r = 0; r < RS_IPT; ++r) {
    uint64_t i = base + (uint64_t)r * 32 + lane;
    bool ok = i < n;
    if (ok) { kr[r] = kin[i]; vr[r] = vin[i]; }
    uint32_t d = ok ? digit(kr[r], shift, mask) : 0xffffffffu;
    uint32_t m = __match_any_sync(FULL, d);
    uint32_t before = __popc(m & lanemask_lt());
    uint32_t prev = ok ? wc[warp][d] : 0;
    rk[r] = prev + before;
    __syncwarp();
    if (ok && (uint32_t)(__ffs(m) - 1) == lane) wc[warp][d] = prev + __popc(m);
    __syncwarp();
  }
  __syncthreads();
  // per digit: exclusive prefix over warps, plus the tile's global digit offset
  for (uint32_t d = threadIdx.x; d < radix; d += RS_NT) {
    uint32_t run = offs[(uint64_t)d * ntiles + blockIdx.x];
#pragma unroll
    for (int w = 0; w < RS_WARPS; ++w) {
      uint32_t t = wc[w][d];
      wc[w][d] = run;
      run += t;
    }
  }
  __syncthreads();
#pragma unroll
  for (int r = 0; r < RS_IPT; ++r) {
    uint64_t i = base + (uint64_t)r * 32 + lane;
    if (i < n) {
      uint32_t d = digit(kr[r], shift, mask);
      uint32_t dst = wc[warp][d] + rk[r];
      kout[dst] = kr[r];
      vout[dst] = vr[r];
    }
  }
}

// ------------------------------------------------------------------ (cta, warp) regroup
__global__ void k_warp_keys(const uint32_t* __restrict__ cta, const uint16_t* __restrict__ tid, uint64_t n,
                            uint64_t* __restrict__ key, uint32_t* __restrict__ idx) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    key[i] = ((uint64_t)__ldg(cta + i) << 5) | ((__ldg(tid + i) >> 5) & 31u);
    idx[i] = (uint32_t)i;
  }
}

__global__ void k_gather_all(cadv_trace_desc t, const uint32_t* __restrict__ idx, uint64_t* addr, uint32_t* cta,
                             uint16_t* tid, uint32_t* site, uint32_t* winst, uint8_t* meta) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < t.n; i += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t j = idx[i];
    addr[i] = t.addr[j];
    cta[i] = t.cta[j];
    tid[i] = t.tid[j];
    site[i] = t.site[j];
    winst[i] = t.winst[j];
    meta[i] = t.meta[j];
  }
}

}  // namespace

cudaError_t exclusive_scan_u32(cadv_ctx* c, const uint32_t* in, uint32_t* out, uint64_t n, uint32_t* d_total) {
  return scan_impl<uint32_t>(c, in, out, n, d_total, 0);
}
cudaError_t exclusive_scan_u64(cadv_ctx* c, const uint64_t* in, uint64_t* out, uint64_t n) {
  return scan_impl<unsigned long long>(c, (const unsigned long long*)in, (unsigned long long*)out, n, nullptr, 0);
}

template <typename K, typename V>
cudaError_t radix_sort_pairs(cadv_ctx* c, K* k0, V* v0, K* k1, V* v1, uint64_t n, int bit_lo, int bit_hi,
                             int* result_in) {
  *result_in = 0;
  if (n <= 1 || bit_hi <= bit_lo) return cudaSuccess;
  uint64_t ntiles = (n + RS_TILE - 1) / RS_TILE;
  void* hist;
  cudaError_t e = ensure(c, B_SORT_HIST, (1ull << RS_MAXB) * ntiles * 4 + 64, &hist);
  if (e != cudaSuccess) return e;
  int passes = (bit_hi - bit_lo + RS_MAXB - 1) / RS_MAXB;
  int per = (bit_hi - bit_lo + passes - 1) / passes;
  K* ki = k0; V* vi = v0; K* ko = k1; V* vo = v1;
  for (int shift = bit_lo; shift < bit_hi; shift += per) {
    int bits = per < bit_hi - shift ? per : bit_hi - shift;
    uint32_t* cnt = (uint32_t*)hist;
    CADV_LAUNCH(c, k_rs_upsweep<K><<<(unsigned)ntiles, RS_NT, 0, c->stream>>>(ki, n, shift, bits, cnt, ntiles));
    e = exclusive_scan_u32(c, cnt, cnt, (uint64_t)(1u << bits) * ntiles, nullptr);
    if (e != cudaSuccess) return e;
    CADV_LAUNCH(c, k_rs_scatter<K, V><<<(unsigned)ntiles, RS_NT, 0, c->stream>>>(ki, vi, ko, vo, n, shift, bits, cnt,
                                                                                ntiles));
    std::swap(ki, ko);
    std::swap(vi, vo);
    *result_in ^= 1;
  }
  return cudaGetLastError();
}

template cudaError_t radix_sort_pairs<uint32_t, uint64_t>(cadv_ctx*, uint32_t*, uint64_t*, uint32_t*, uint64_t*,
                                                          uint64_t, int, int, int*);
template cudaError_t radix_sort_pairs<uint64_t, uint32_t>(cadv_ctx*, uint64_t*, uint32_t*, uint64_t*, uint32_t*,
                                                          uint64_t, int, int, int*);
template cudaError_t radix_sort_pairs<uint32_t, uint32_t>(cadv_ctx*, uint32_t*, uint32_t*, uint32_t*, uint32_t*,
                                                          uint64_t, int, int, int*);

namespace {

__global__ void k_bucket_count64(const uint64_t* __restrict__ key, uint64_t n, int shift, unsigned long long* cnt) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t b = (uint32_t)(__ldg(key + i) >> shift);  // sorted keys: one atomic per run of a bucket in the warp
    const uint32_t peers = __match_any_sync(__activemask(), b);
    if (lane_id() == (uint32_t)(__ffs(peers) - 1)) atomicAdd(&cnt[b], (unsigned long long)__popc(peers));
  }
}

// out[r] = first position whose bucket >= bnd[r] (keys sorted)
__global__ void k_lower_bounds64(const uint64_t* __restrict__ key, uint64_t n, int shift, const uint64_t* bnd, int m,
                                 uint64_t* out) {
  const int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= m) return;
  uint64_t lo = 0, hi = n;
  while (lo < hi) {
    const uint64_t md = (lo + hi) >> 1;
    if ((key[md] >> shift) < bnd[r]) lo = md + 1;
    else hi = md;
  }
  out[r] = lo;
}

__global__ void k_max_key(const uint64_t* __restrict__ key, uint64_t n, uint32_t* out) {
  if (threadIdx.x == 0) *out = n ? (uint32_t)(key[n - 1] >> 5) : 0u;  // sorted: the last key is the largest
}

int bits_of(uint64_t v) {
  int b = 0;
  while (b < 64 && (v >> b)) ++b;
  return b;
}

// Stable sort of t's records by (cta << 5 | tid / 32): sorted keys in *keys,
// the permuted columns in `cols` (B_GATHER layout of regroup_by_warp).
cudaError_t sort_by_warp(cadv_ctx* c, const cadv_trace_desc& t, BufId kb0, BufId kb1, BufId vb0, BufId vb1, BufId gb,
                         const uint64_t** keys, cadv_trace_desc* out) {
  const uint64_t n = t.n;
  void *k0, *k1, *v0, *v1, *g;
  cudaError_t e;
  if ((e = ensure(c, kb0, n * 8, &k0)) || (e = ensure(c, kb1, n * 8, &k1)) || (e = ensure(c, vb0, n * 4, &v0)) ||
      (e = ensure(c, vb1, n * 4, &v1)) || (e = ensure(c, gb, n * 24 + 128, &g)))
    return e;
  const int grid = c->num_sms * 8;
  *out = t;
  if (n) {
    CADV_LAUNCH(c, k_warp_keys<<<grid, 256, 0, c->stream>>>(t.cta, t.tid, n, (uint64_t*)k0, (uint32_t*)v0));
    int res;
    if ((e = radix_sort_pairs<uint64_t, uint32_t>(c, (uint64_t*)k0, (uint32_t*)v0, (uint64_t*)k1, (uint32_t*)v1, n, 0,
                                                  37, &res)))
      return e;
    *keys = res ? (const uint64_t*)k1 : (const uint64_t*)k0;
    const uint32_t* idx = res ? (const uint32_t*)v1 : (const uint32_t*)v0;
    uint8_t* p = (uint8_t*)g;
    auto al = [&](uint64_t off) { return (off + 15) & ~uint64_t(15); };
    const uint64_t oa = 0, oc = al(n * 8), os = al(oc + n * 4), ow = al(os + n * 4), ot = al(ow + n * 4),
                   om = al(ot + n * 2);
    out->addr = (uint64_t*)(p + oa);
    out->cta = (uint32_t*)(p + oc);
    out->site = (uint32_t*)(p + os);
    out->winst = (uint32_t*)(p + ow);
    out->tid = (uint16_t*)(p + ot);
    out->meta = (uint8_t*)(p + om);
    CADV_LAUNCH(c, k_gather_all<<<grid, 256, 0, c->stream>>>(t, idx, (uint64_t*)out->addr, (uint32_t*)out->cta,
                                                             (uint16_t*)out->tid, (uint32_t*)out->site,
                                                             (uint32_t*)out->winst, (uint8_t*)out->meta));
  } else {
    *keys = (const uint64_t*)k0;
  }
  out->warp_contiguous = 1;
  return cudaGetLastError();
}

}  // namespace

// Multi-rank divergence on non-warp-contiguous shards: every
// (cta, warp32) record stream moves to ONE rank, so that each warp-level
// group is whole there.  Each rank sorts its shard stably by the stream key,
// the key space is cut into equal shares of the global record count (bucket
// histogram all-reduced), every rank sends its slice for rank r to r
// (alltoallv of the seven columns incl. the key), and r stably re-sorts what
// it received: slices arrive in rank order = trace order, so every stream
// keeps its trace order.  Collective; *out = this rank's streams.
cudaError_t exchange_by_warp(cadv_ctx* c, cadv_trace_desc* out) {
  cudaError_t e;
  Comm* cm = c->comm;
  const int G = c->nranks, me = c->rank;
  const uint64_t* keys = nullptr;
  cadv_trace_desc loc;
  if ((e = sort_by_warp(c, c->t, B_SORT_K0, B_SORT_K1, B_SORT_V0, B_SORT_V1, B_GATHER, &keys, &loc))) return e;
  const uint64_t n = c->t.n;
  void* cb;
  if ((e = ensure(c, B_COMM, (size_t)(2 * G + 4) * 8 + (size_t)G * G * 8 + 64, &cb))) return e;
  uint64_t* d_send = (uint64_t*)cb;
  uint64_t* d_mat = d_send + G + 2;
  // global key range -> bucket width (<= 2^20 buckets)
  uint32_t* dm = (uint32_t*)d_mat;
  CADV_LAUNCH(c, k_max_key<<<1, 32, 0, c->stream>>>(keys, n, dm));
  if (cm->allreduce_max_u32(dm, 1, c->stream)) return cudaErrorUnknown;
  uint32_t gmax = 0;
  if ((e = cudaMemcpyAsync(&gmax, dm, 4, cudaMemcpyDeviceToHost, c->stream)) || (e = cudaStreamSynchronize(c->stream)))
    return e;
  const int kbits = bits_of(((uint64_t)gmax << 5) | 31u);
  const int shift = kbits > 20 ? kbits - 20 : 0;
  const uint64_t nb = ((((uint64_t)gmax << 5) | 31u) >> shift) + 1;
  void* cntb;
  if ((e = ensure(c, B_XCH_CNT, (nb + 2 * G + 4) * 8 + 64, &cntb))) return e;
  unsigned long long* cnt = (unsigned long long*)cntb;
  uint64_t* d_bnd = (uint64_t*)(cnt + nb);
  if ((e = cudaMemsetAsync(cnt, 0, nb * 8, c->stream))) return e;
  if (n) CADV_LAUNCH(c, k_bucket_count64<<<c->num_sms * 4, 256, 0, c->stream>>>(keys, n, shift, cnt));
  if (cm->allreduce_sum_u64((uint64_t*)cnt, nb, c->stream)) return cudaErrorUnknown;
  std::vector<uint64_t> h(nb);
  if ((e = cudaMemcpyAsync(h.data(), cnt, nb * 8, cudaMemcpyDeviceToHost, c->stream)) ||
      (e = cudaStreamSynchronize(c->stream)))
    return e;
  uint64_t total = 0;
  for (uint64_t b = 0; b < nb; ++b) total += h[b];
  std::vector<uint64_t> bnd(G + 1, nb), pos(G + 1, 0);
  bnd[0] = 0;
  {
    uint64_t acc = 0, b = 0;
    for (int r = 1; r < G; ++r) {
      const uint64_t target = (uint64_t)((unsigned __int128)total * r / G);
      while (b < nb && acc + h[b] <= target) acc += h[b++];
      bnd[r] = b;
    }
  }
  pos[G] = n;
  if (n && G > 1) {
    if ((e = cudaMemcpyAsync(d_bnd, bnd.data() + 1, (G - 1) * 8, cudaMemcpyHostToDevice, c->stream))) return e;
    CADV_LAUNCH(c, k_lower_bounds64<<<1, 64, 0, c->stream>>>(keys, n, shift, d_bnd, G - 1, d_bnd + G));
    if ((e = cudaMemcpyAsync(pos.data() + 1, d_bnd + G, (G - 1) * 8, cudaMemcpyDeviceToHost, c->stream)) ||
        (e = cudaStreamSynchronize(c->stream)))
      return e;
  }
  std::vector<uint64_t> scnt(G), soff(G), rcnt(G), roff(G), mat((size_t)G * G);
  for (int r = 0; r < G; ++r) { soff[r] = pos[r]; scnt[r] = pos[r + 1] - pos[r]; }
  if ((e = cudaMemcpyAsync(d_send, scnt.data(), G * 8, cudaMemcpyHostToDevice, c->stream))) return e;
  if (cm->allgather(d_send, d_mat, G * 8, c->stream)) return cudaErrorUnknown;
  if ((e = cudaMemcpyAsync(mat.data(), d_mat, (size_t)G * G * 8, cudaMemcpyDeviceToHost, c->stream)) ||
      (e = cudaStreamSynchronize(c->stream)))
    return e;
  uint64_t Kn = 0;
  for (int p = 0; p < G; ++p) { rcnt[p] = mat[(size_t)p * G + me]; roff[p] = Kn; Kn += rcnt[p]; }
  for (int r = 0; r < G; ++r) {  // u32 positions per shard (decided alike on every rank)
    uint64_t kr = 0;
    for (int p = 0; p < G; ++p) kr += mat[(size_t)p * G + r];
    if (kr >= 0xffffffffull) return cudaErrorNotSupported;
  }
  // receive buffers: the key and the six columns, 16-byte aligned slices
  auto al = [](uint64_t x) { return (x + 15) & ~uint64_t(15); };
  const size_t es[7] = {8, 8, 4, 2, 4, 4, 1};
  size_t off[8];
  off[0] = 0;
  for (int k = 0; k < 7; ++k) off[k + 1] = al(off[k] + es[k] * Kn);
  void* rb;
  if ((e = ensure(c, B_WX_RECV, off[7] + 64, &rb))) return e;
  uint8_t* R = (uint8_t*)rb;
  const void* src[7] = {keys, loc.addr, loc.cta, loc.tid, loc.site, loc.winst, loc.meta};
  for (int k = 0; k < 7; ++k) {
    std::vector<uint64_t> so(G), sc(G), ro(G), rc(G);
    for (int p = 0; p < G; ++p) {
      so[p] = soff[p] * es[k]; sc[p] = scnt[p] * es[k]; ro[p] = roff[p] * es[k]; rc[p] = rcnt[p] * es[k];
    }
    if (cm->alltoallv(src[k], so.data(), sc.data(), R + off[k], ro.data(), rc.data(), c->stream))
      return cudaErrorUnknown;
  }
  cadv_trace_desc recv = c->t;
  recv.n = Kn;
  recv.addr = (const uint64_t*)(R + off[1]);
  recv.cta = (const uint32_t*)(R + off[2]);
  recv.tid = (const uint16_t*)(R + off[3]);
  recv.site = (const uint32_t*)(R + off[4]);
  recv.winst = (const uint32_t*)(R + off[5]);
  recv.meta = (const uint8_t*)(R + off[6]);
  // stable re-sort of the received slices (rank order = trace order)
  const uint64_t* k2;
  if ((e = sort_by_warp(c, recv, B_WX_K0, B_WX_K1, B_WX_V0, B_WX_V1, B_WX_COLS, &k2, out))) return e;
  out->n = Kn;
  return cudaSuccess;
}

cudaError_t regroup_by_warp(cadv_ctx* c, cadv_trace_desc* out) {
  const cadv_trace_desc& t = c->t;
  uint64_t n = t.n;
  void *k0, *k1, *v0, *v1, *g;
  cudaError_t e;
  if ((e = ensure(c, B_SORT_K0, n * 8, &k0)) || (e = ensure(c, B_SORT_K1, n * 8, &k1)) ||
      (e = ensure(c, B_SORT_V0, n * 4, &v0)) || (e = ensure(c, B_SORT_V1, n * 4, &v1)) ||
      (e = ensure(c, B_GATHER, n * 24 + 64, &g)))
    return e;
  int grid = c->num_sms * 8;
  CADV_LAUNCH(c, k_warp_keys<<<grid, 256, 0, c->stream>>>(t.cta, t.tid, n, (uint64_t*)k0, (uint32_t*)v0));
  const int bits = 37;  // (cta << 5 | warp): the CTA-id range is not known before the scan
  int res;
  e = radix_sort_pairs<uint64_t, uint32_t>(c, (uint64_t*)k0, (uint32_t*)v0, (uint64_t*)k1, (uint32_t*)v1, n, 0, bits,
                                           &res);
  if (e != cudaSuccess) return e;
  const uint32_t* idx = res ? (const uint32_t*)v1 : (const uint32_t*)v0;
  uint8_t* p = (uint8_t*)g;
  uint64_t* a = (uint64_t*)p;
  uint32_t* ct = (uint32_t*)(p + n * 8);
  uint32_t* st = (uint32_t*)(p + n * 12);
  uint32_t* wi = (uint32_t*)(p + n * 16);
  uint16_t* td = (uint16_t*)(p + n * 20);
  uint8_t* mt = (uint8_t*)(p + n * 22);
  CADV_LAUNCH(c, k_gather_all<<<grid, 256, 0, c->stream>>>(t, idx, a, ct, td, st, wi, mt));
  *out = t;
  out->addr = a;
  out->cta = ct;
  out->tid = td;
  out->site = st;
  out->winst = wi;
  out->meta = mt;
  out->warp_contiguous = 1;
  return cudaGetLastError();
}

}  // namespace cadv
