// regroup.cu — R1 regroup by CTA (CTA scope, one rank) without a global sort
// of the kept records.
//
// The scan leaves the kept records in per-warp regions, each in trace order
// (region w = records [w * chunk, w * chunk + cnt[w]) of the gapped buffer).
// CTA-major order with trace order inside a CTA (DESIGN.md reading
// R2) puts record i of CTA c of region w at
//     base(c) + sum_{w' < w} n(c, w') + rank of i among c's records in w,
// n(c, w) the number of c's kept records in region w.  A region only sees
// the CTAs resident while it was traced (a few hundred), so:
//   1. k_rg_count   one warp per region: a shared-memory table CTA -> n(c, w)
//                   (open addressing, RG_SLOTS slots); emits the region's
//                   (c, n) pairs into its slice of the pair buffer; a region
//                   with more than RG_MAX distinct CTAs sets the overflow flag
//                   and the host takes the squeeze + radix-sort path instead;
//   2. pairs packed in region order, stably radix-sorted by CTA (a few
//      hundred thousand pairs instead of the tens of millions of records),
//      exclusive scan of n in that order = the output offset of every (c, w);
//   3. k_rg_scatter one warp per region: rebuilds the table CTA -> offset,
//                   walks its records in order, rank = offset + earlier peers
//                   (__match_any_sync) and writes key and value once.
// Data movement: keys read twice, values once, both written once: 28 B per
// kept record instead of 80 B for squeeze + two radix passes.
#include <cuda_runtime.h>

#include "cadv_impl.h"
#include "common.cuh"

namespace cadv {
namespace {

constexpr uint32_t RG_SLOTS = 1024;  // table slots per region (power of two)
constexpr uint32_t RG_EMPTY = 0xffffffffu;

__device__ __forceinline__ uint32_t rg_hash(uint32_t c) { return (c * 0x9E3779B1u) >> (32 - 10); }

// Slot of CTA c in the region table (inserted if absent); RG_EMPTY if full.
__device__ __forceinline__ uint32_t rg_slot(uint32_t* tk, uint32_t c) {
  uint32_t h = rg_hash(c);
  for (uint32_t probe = 0; probe < RG_SLOTS; ++probe) {
    const uint32_t k = tk[h];
    if (k == c) return h;
    if (k == RG_EMPTY) {
      const uint32_t old = atomicCAS(&tk[h], RG_EMPTY, c);
      if (old == RG_EMPTY || old == c) return h;
    }
    h = (h + 1) & (RG_SLOTS - 1);
  }
  return RG_EMPTY;
}

// 1. per-region CTA counts -> pairs (cta, n) at pk/pn + w * RG_MAX, np[w];
//    the kept CTA-id range (radix bits) and the overflow flag in sc.  Counts
//    do not depend on order: RG_NT threads per region, warp-aggregated
//    shared-memory atomics.
constexpr int RG_NT = 256;
__global__ void __launch_bounds__(RG_NT) k_rg_count(const uint32_t* __restrict__ key, const uint64_t* __restrict__ cnt,
                                                    uint64_t chunk, uint32_t* __restrict__ pk,
                                                    uint32_t* __restrict__ pn, uint32_t* __restrict__ np,
                                                    Scalars* sc) {
  __shared__ uint32_t tk[RG_SLOTS], tn[RG_SLOTS];
  __shared__ uint32_t s_full, s_base;
  const uint32_t lane = lane_id(), tx = threadIdx.x, w = blockIdx.x;
  for (uint32_t k = tx; k < RG_SLOTS; k += RG_NT) { tk[k] = RG_EMPTY; tn[k] = 0; }
  if (tx == 0) { s_full = 0; s_base = 0; }
  __syncthreads();
  const uint64_t m = cnt[w];
  const uint32_t* kr = key + (uint64_t)w * chunk;
  uint32_t mx = 0, full = 0;
  constexpr int RB = 4;  // rounds whose loads are issued together
  for (uint64_t r0 = 0; r0 < m; r0 += RG_NT * RB) {  // (uniform trip count: every lane reaches the match)
    uint32_t cb[RB];
#pragma unroll
    for (int b = 0; b < RB; ++b) {
      const uint64_t r = r0 + (uint64_t)b * RG_NT + tx;
      cb[b] = r < m ? __ldg(kr + r) : RG_EMPTY;
    }
#pragma unroll
    for (int b = 0; b < RB; ++b) {
      const bool ok = r0 + (uint64_t)b * RG_NT + tx < m;
      const uint32_t c = cb[b];
      if (ok && c == RG_EMPTY) full = 1;  // (the table's empty marker: such a trace takes the radix path)
      const uint32_t peers = __match_any_sync(FULL, c);
      if (ok && c != RG_EMPTY && (uint32_t)(__ffs(peers) - 1) == lane) {  // one lane per CTA of the warp's 32 records
        const uint32_t s = rg_slot(tk, c);
        if (s != RG_EMPTY) atomicAdd(&tn[s], (uint32_t)__popc(peers));
        else full = 1;
        mx = max(mx, c);
      }
    }
  }
  if (full) s_full = 1;
  __syncthreads();
  // compact the table into the region's pair slice (order within a region is free)
  const uint32_t k = tx;
  for (uint32_t k0 = 0; k0 < RG_SLOTS; k0 += RG_NT) {
    const uint32_t kk = k0 + k, c = tk[kk];
    const bool used = c != RG_EMPTY;
    const uint32_t b = __ballot_sync(FULL, used);
    uint32_t wb = 0;
    if (lane == 0 && b) wb = atomicAdd(&s_base, (uint32_t)__popc(b));
    wb = __shfl_sync(FULL, wb, 0);
    if (used) {
      const uint32_t j = wb + __popc(b & lanemask_lt());
      if (j < RG_MAX) {
        pk[(uint64_t)w * RG_MAX + j] = c;
        pn[(uint64_t)w * RG_MAX + j] = tn[kk];
      }
    }
  }
  mx = __reduce_max_sync(FULL, mx);
  if (lane == 0 && mx) atomicMax(&sc->max_cta, (unsigned long long)mx);
  __syncthreads();
  if (tx == 0) {
    const uint32_t base = s_base;
    np[w] = base < RG_MAX ? base : RG_MAX;
    if (s_full || base > RG_MAX) sc->rg_overflow = 1;
  }
}

// 2a. pack the pair slices in region order: (cta, w << 10 | j), n
__global__ void k_rg_pack(const uint32_t* __restrict__ pk, const uint32_t* __restrict__ pn,
                          const uint32_t* __restrict__ np, const uint32_t* __restrict__ poff,
                          uint32_t* __restrict__ ok_, uint32_t* __restrict__ ov, uint32_t* __restrict__ on) {
  const uint32_t w = blockIdx.x, n = np[w], o = poff[w];
  for (uint32_t j = threadIdx.x; j < n; j += blockDim.x) {
    ok_[o + j] = pk[(uint64_t)w * RG_MAX + j];
    ov[o + j] = (w << 10) | j;
    on[o + j] = pn[(uint64_t)w * RG_MAX + j];
  }
}

// 2b. counts in CTA-sorted order (gathered through the sorted pair ids)
__global__ void k_rg_gather_n(const uint32_t* __restrict__ sv, const uint32_t* __restrict__ pn, uint64_t P,
                              uint32_t* __restrict__ sn) {
  for (uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; s < P; s += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t v = sv[s];
    sn[s] = pn[(uint64_t)(v >> 10) * RG_MAX + (v & 1023u)];
  }
}

// 2c. offsets back into the region slices: po[w][j] = offset of (c, w)
__global__ void k_rg_offsets(const uint32_t* __restrict__ sv, const uint32_t* __restrict__ so, uint64_t P,
                             uint32_t* __restrict__ po) {
  for (uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; s < P; s += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t v = sv[s];
    po[(uint64_t)(v >> 10) * RG_MAX + (v & 1023u)] = so[s];
  }
}

// 3. scatter: RG_NT threads per region; warp q takes the q-th contiguous
//    slice of the region (whole 32-record rounds).  The warps first count
//    their slices' CTAs, a prefix over the warps turns the region offsets of
//    the CTAs into per-slice starts, then every warp writes its slice in
//    order (rank among a round's peers by __match_any_sync; the peer group's
//    leader probes the table once).  Keys are written only when a later
//    kernel reads them (no segment list, or a segment longer than
//    SEG_TILE_MAX kept records).  (A variant that staged each region in
//    shared memory and wrote every (CTA, region) run contiguously was
//    measured slower, 0.23 -> 0.40 ms on C4: half the resident CTAs and four
//    block barriers per window.)
constexpr int RG_W = RG_NT / 32;
__global__ void __launch_bounds__(RG_NT) k_rg_scatter(const uint32_t* __restrict__ key,
                                                      const uint64_t* __restrict__ val,
                                                      const uint64_t* __restrict__ cnt, uint64_t chunk,
                                                      const uint32_t* __restrict__ pk, const uint32_t* __restrict__ po,
                                                      const uint32_t* __restrict__ np, const unsigned int* seg_cm,
                                                      uint32_t* __restrict__ kout, uint64_t* __restrict__ vout) {
  __shared__ uint32_t tk[RG_SLOTS];
  __shared__ uint32_t st[RG_W][RG_SLOTS];  // per slice: CTA counts, then starts
  const uint32_t lane = lane_id(), tx = threadIdx.x, q = tx >> 5, w = blockIdx.x;
  const bool keys = seg_cm == nullptr || seg_cm[1] > SEG_TILE_MAX;  // (only the bounds-tiled path reads keys)
  for (uint32_t k = tx; k < RG_SLOTS; k += RG_NT) tk[k] = RG_EMPTY;
  for (uint32_t k = tx; k < RG_W * RG_SLOTS; k += RG_NT) (&st[0][0])[k] = 0;
  __syncthreads();
  const uint32_t n = np[w];
  for (uint32_t j = tx; j < n; j += RG_NT) rg_slot(tk, pk[(uint64_t)w * RG_MAX + j]);
  __syncthreads();
  const uint64_t m = cnt[w];
  const uint32_t* kr = key + (uint64_t)w * chunk;
  const uint64_t* vr = val + (uint64_t)w * chunk;
  const uint64_t rounds = (m + 31) / 32, per = (rounds + RG_W - 1) / RG_W;
  const uint64_t lo = min(m, q * per * 32), hi = min(m, (q + 1) * per * 32);
  // (a) count the slice's CTAs (loads of 4 rounds issued together)
  for (uint64_t r0 = lo; r0 < hi; r0 += 128) {
    uint32_t cb[4];
#pragma unroll
    for (int b = 0; b < 4; ++b) cb[b] = r0 + 32 * b + lane < hi ? __ldg(kr + r0 + 32 * b + lane) : RG_EMPTY;
#pragma unroll
    for (int b = 0; b < 4; ++b) {
      const bool ok = r0 + 32 * b + lane < hi;
      const uint32_t peers = __match_any_sync(FULL, cb[b]);
      if (ok && (uint32_t)(__ffs(peers) - 1) == lane) st[q][rg_slot(tk, cb[b])] += __popc(peers);
      __syncwarp();
    }
  }
  __syncthreads();
  // (b) slice starts = the CTA's region offset + its records in earlier slices
  for (uint32_t j = tx; j < n; j += RG_NT) {
    const uint32_t s = rg_slot(tk, pk[(uint64_t)w * RG_MAX + j]);
    uint32_t run = po[(uint64_t)w * RG_MAX + j];
#pragma unroll
    for (int x = 0; x < RG_W; ++x) {
      const uint32_t t = st[x][s];
      st[x][s] = run;
      run += t;
    }
  }
  __syncthreads();
  // (c) write the slice in order
  uint32_t* const to = st[q];
  constexpr int RG_B = 4;  // rounds whose loads are issued together
  for (uint64_t r0 = lo; r0 < hi; r0 += 32 * RG_B) {
    uint32_t cb[RG_B];
    uint64_t vb[RG_B];
#pragma unroll
    for (int b = 0; b < RG_B; ++b) {
      const uint64_t r = r0 + 32 * b + lane;
      cb[b] = r < hi ? __ldg(kr + r) : RG_EMPTY;
      vb[b] = r < hi ? __ldg(vr + r) : 0ull;
    }
#pragma unroll
    for (int b = 0; b < RG_B; ++b) {
      const bool ok = r0 + 32 * b + lane < hi;
      const uint32_t c = cb[b];
      const uint32_t peers = __match_any_sync(FULL, c);
      const uint32_t lead = __ffs(peers) - 1;
      uint32_t s = 0;
      if (ok && lead == lane) s = rg_slot(tk, c);  // present: every CTA of the region is in the table
      s = __shfl_sync(FULL, s, lead);
      uint32_t dst = 0;
      if (ok) {
        dst = to[s] + __popc(peers & lanemask_lt());
        if (keys) kout[dst] = c;
        vout[dst] = vb[b];
      }
      __syncwarp();
      if (ok && (peers >> lane) == 1u) to[s] = dst + 1;  // the CTA's last record of the round
      __syncwarp();
    }
  }
}

// 4. the CTA segments of the output: for every CTA's first sorted pair,
//    (start, length) appended to seg (<= SEG_WARP_MAX kept records, or every
//    segment when seg_long is null) or to seg_long (unordered: segments are
//    independent); cm[0] = |seg|, cm[1] = longest, cm[3] = |seg_long|
//    (warp-aggregated counters)
__global__ void k_rg_segments(const uint32_t* __restrict__ sk, const uint32_t* __restrict__ sn,
                              const uint32_t* __restrict__ so, uint64_t P, uint2* __restrict__ seg,
                              uint2* __restrict__ seg_long, unsigned int* __restrict__ cm) {
  const uint32_t lane = lane_id();
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  uint32_t mx = 0;
  for (uint64_t base = ((blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5) * 32; base < P; base += nw * 32) {
    const uint64_t s = base + lane;
    uint32_t len = 0;
    if (s < P && (s == 0 || sk[s - 1] != sk[s])) {
      // the CTA's pairs are [s, x): galloping then binary search for x (a CTA
      // spread over many regions has a long run), length from the offsets
      const uint32_t c = sk[s];
      uint64_t lo = s, step = 1;  // sk[lo] == c
      while (lo + step < P && sk[lo + step] == c) { lo += step; step <<= 1; }
      uint64_t hi = lo + step < P ? lo + step : P;  // sk[hi] != c or hi == P
      while (hi - lo > 1) {
        const uint64_t md = (lo + hi) >> 1;
        if (sk[md] == c) lo = md;
        else hi = md;
      }
      len = so[lo] + sn[lo] - so[s];
    }
    mx = max(mx, len);
    const bool lg = len > SEG_WARP_MAX && seg_long != nullptr;
    const uint32_t bs = __ballot_sync(FULL, len && !lg), bl = __ballot_sync(FULL, lg);
    uint32_t os = 0, ol = 0;
    if (lane == 0) {
      if (bs) os = atomicAdd(&cm[0], (unsigned)__popc(bs));
      if (bl) ol = atomicAdd(&cm[3], (unsigned)__popc(bl));
    }
    os = __shfl_sync(FULL, os, 0);
    ol = __shfl_sync(FULL, ol, 0);
    if (len && !lg) seg[os + __popc(bs & lanemask_lt())] = make_uint2(so[s], len);
    if (lg) seg_long[ol + __popc(bl & lanemask_lt())] = make_uint2(so[s], len);
  }
  mx = __reduce_max_sync(FULL, mx);
  if (lane == 0 && mx) atomicMax(&cm[1], mx);
}

}  // namespace

// Phase 1 (queued before the scan's synchronisation): per-region CTA counts.
cudaError_t rg_count(cadv_ctx* c, const uint32_t* key, const uint64_t* cnt, uint64_t nregions, uint64_t chunk,
                     RgState* st) {
  void *pk, *pn, *np;
  cudaError_t e;
  if ((e = ensure(c, B_RG_PK, nregions * RG_MAX * 4 + 64, &pk)) ||
      (e = ensure(c, B_RG_PN, nregions * RG_MAX * 4 + 64, &pn)) ||
      (e = ensure(c, B_RG_NP, (nregions + 2) * 4 * 2 + 64, &np)))
    return e;
  st->pk = (uint32_t*)pk;
  st->pn = (uint32_t*)pn;
  st->np = (uint32_t*)np;
  st->poff = st->np + nregions + 2;
  st->nregions = nregions;
  if ((e = cudaMemsetAsync(st->np + nregions, 0, 8, c->stream))) return e;
  CADV_LAUNCH(c, k_rg_count<<<(unsigned)nregions, RG_NT, 0, c->stream>>>(key, cnt, chunk, st->pk, st->pn, st->np,
                                                                       scalars(c)));
  // region offsets of the packed pairs; the total arrives with the scan's read-back
  return exclusive_scan_u32(c, st->np, st->poff, nregions + 1, nullptr);
}

// Phases 2-3 (after the synchronisation; P = total pairs, no overflow).
cudaError_t rg_finish(cadv_ctx* c, const RgState& st, uint64_t P, int bits, const uint32_t* key,
                      const uint64_t* val, const uint64_t* cnt, uint64_t chunk, uint32_t* kout, uint64_t* vout,
                      uint2* seg, uint2* seg_long, unsigned int* seg_cm) {
  void *b;
  cudaError_t e;
  // packed pairs (ping-pong for the sort) + counts + offsets
  if ((e = ensure(c, B_RG_SORT, (P + 16) * 4 * 6 + 64, &b))) return e;
  uint32_t* k0 = (uint32_t*)b;
  uint32_t* k1 = k0 + (P + 16);
  uint32_t* v0 = k1 + (P + 16);
  uint32_t* v1 = v0 + (P + 16);
  uint32_t* n0 = v1 + (P + 16);
  uint32_t* n1 = n0 + (P + 16);
  CADV_LAUNCH(c, k_rg_pack<<<(unsigned)st.nregions, 128, 0, c->stream>>>(st.pk, st.pn, st.np, st.poff, k0, v0, n0));
  int res = 0;
  if ((e = radix_sort_pairs<uint32_t, uint32_t>(c, k0, v0, k1, v1, P, 0, bits, &res))) return e;
  const uint32_t* sv = res ? v1 : v0;
  const int grid = c->num_sms * 4;
  CADV_LAUNCH(c, k_rg_gather_n<<<grid, 256, 0, c->stream>>>(sv, st.pn, P, n1));
  if ((e = exclusive_scan_u32(c, n1, n0, P, nullptr))) return e;
  // the offsets overwrite the pair counts (pn is no longer needed)
  CADV_LAUNCH(c, k_rg_offsets<<<grid, 256, 0, c->stream>>>(sv, n0, P, st.pn));
  if (seg) {  // the CTA segments of the output (count and longest in seg_cm)
    if ((e = cudaMemsetAsync(seg_cm, 0, 16, c->stream))) return e;
    CADV_LAUNCH(c, k_rg_segments<<<grid, 256, 0, c->stream>>>(res ? k1 : k0, n1, n0, P, seg, seg_long, seg_cm));
  }
  // keys are written for the bounds-tiled path only (no segment list, a segment longer than
  // SEG_TILE_MAX, or CADV_RD_TILES)
  const unsigned int* keys_flag = (seg && getenv("CADV_RD_TILES") == nullptr) ? seg_cm : nullptr;
  CADV_LAUNCH(c, k_rg_scatter<<<(unsigned)st.nregions, RG_NT, 0, c->stream>>>(
                     key, val, cnt, chunk, st.pk, st.pn, st.np, keys_flag, kout, vout));
  return cudaGetLastError();
}

}  // namespace cadv
