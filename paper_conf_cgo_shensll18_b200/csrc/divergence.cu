// divergence.cu — memory divergence and branch divergence
// (Table 3) as single streaming passes over the trace.
//
// Both analyses work on warp-level groups: a "run" is a maximal contiguous
// sequence of records with the same (cta, tid/32, winst, family); with
// warp_contiguous traces each dynamic warp-level instruction is exactly one
// run of <= 32 records (include/cadv.h).  A group is a run restricted to one
// sub-warp (tid % 32) / W.
//
// Data movement (B200): persistent CTAs stream fixed tiles of TM records
// through a 2-stage shared-memory ring filled by 1-D TMA bulk copies
// (cp.async.bulk + mbarrier complete_tx), one copy per column.  A tile owns
// the groups that START inside it and is staged with a 1-record halo before
// and a 32-record halo after, so every owned group is complete in shared
// memory.  Each warp walks its 256-record sub-range in batches of 32
// records starting at a group start; all groups that are complete inside
// the batch are resolved at once with __match_any_sync:
//   MD: unique lines = lanes that are the lowest lane of their
//       (group, line) match set; degree = popc of those inside the group.
//   BD: active lanes = popc of the group's match set; live lanes from the
//       per-CTA thread count T_c (k_cta_maxtid, one warp-aggregated
//       atomicMax per CTA run).
// Histograms / per-site counters accumulate in shared memory and are flushed
// with one global atomic per non-zero counter per CTA.
#include <cuda_runtime.h>

#include "cadv_impl.h"
#include "common.cuh"

namespace cadv {
namespace {

constexpr int DV_TM = 2048;   // records owned per tile
constexpr int DV_NT = 256;    // threads per CTA (8 warps x 256 records)
constexpr int DV_S = 2;       // pipeline stages
constexpr int DV_HALO = 33;   // 1 before + 32 after
constexpr int DV_SMEM_SITES = 1024;

constexpr uint32_t DV_ROWS = DV_TM + DV_HALO;
constexpr uint32_t OFF_ADDR = 0;
constexpr uint32_t OFF_CTA = OFF_ADDR + stage_bytes<uint64_t>(DV_ROWS);
constexpr uint32_t OFF_TID = OFF_CTA + stage_bytes<uint32_t>(DV_ROWS);
constexpr uint32_t OFF_WINST = OFF_TID + stage_bytes<uint16_t>(DV_ROWS);
constexpr uint32_t OFF_META = OFF_WINST + stage_bytes<uint32_t>(DV_ROWS);
constexpr uint32_t STAGE_BYTES = ((OFF_META + stage_bytes<uint8_t>(DV_ROWS)) + 127) & ~127u;

struct TraceCols {
  const uint64_t* addr;
  const uint32_t* cta;
  const uint16_t* tid;
  const uint32_t* site;
  const uint32_t* winst;
  const uint8_t* meta;
  uint64_t n;
};

// View of one staged tile: record i (lo <= i < hi) of each column.
struct TileView {
  const uint8_t* st;
  uint64_t lo;
  uint32_t da, dc, dt, dw, dm;
  __device__ __forceinline__ uint64_t addr(uint64_t i) const {
    return *(const uint64_t*)(st + OFF_ADDR + da + (i - lo) * 8);
  }
  __device__ __forceinline__ uint32_t cta(uint64_t i) const {
    return *(const uint32_t*)(st + OFF_CTA + dc + (i - lo) * 4);
  }
  __device__ __forceinline__ uint32_t tid(uint64_t i) const {
    return *(const uint16_t*)(st + OFF_TID + dt + (i - lo) * 2);
  }
  __device__ __forceinline__ uint32_t winst(uint64_t i) const {
    return *(const uint32_t*)(st + OFF_WINST + dw + (i - lo) * 4);
  }
  __device__ __forceinline__ uint8_t meta(uint64_t i) const { return st[OFF_META + dm + (i - lo)]; }
};

__device__ __forceinline__ void tile_range(uint64_t tile, uint64_t n, uint64_t* lo, uint64_t* hi) {
  uint64_t t0 = tile * DV_TM;
  *lo = t0 ? t0 - 1 : 0;
  uint64_t h = t0 + DV_TM + 32;
  *hi = h < n ? h : n;
}

template <bool NEED_ADDR>
__device__ __forceinline__ void issue_tile(const TraceCols& t, uint64_t tile, uint8_t* st, uint64_t* bar) {
  uint64_t lo, hi;
  tile_range(tile, t.n, &lo, &hi);
  uint32_t d, bytes = 0;
  // total first (expect_tx must cover every copy of this phase)
  auto hull = [&](uintptr_t b, uintptr_t e) { return (uint32_t)(((e + 15) & ~(uintptr_t)15) - (b & ~(uintptr_t)15)); };
  if (NEED_ADDR) bytes += hull((uintptr_t)(t.addr + lo), (uintptr_t)(t.addr + hi));
  bytes += hull((uintptr_t)(t.cta + lo), (uintptr_t)(t.cta + hi));
  bytes += hull((uintptr_t)(t.tid + lo), (uintptr_t)(t.tid + hi));
  bytes += hull((uintptr_t)(t.winst + lo), (uintptr_t)(t.winst + hi));
  bytes += hull((uintptr_t)(t.meta + lo), (uintptr_t)(t.meta + hi));
  mbar_arrive_expect_tx(bar, bytes);
  if (NEED_ADDR) stage_column(t.addr, lo, hi, st + OFF_ADDR, bar, &d);
  stage_column(t.cta, lo, hi, st + OFF_CTA, bar, &d);
  stage_column(t.tid, lo, hi, st + OFF_TID, bar, &d);
  stage_column(t.winst, lo, hi, st + OFF_WINST, bar, &d);
  stage_column(t.meta, lo, hi, st + OFF_META, bar, &d);
}

__device__ __forceinline__ TileView make_view(const TraceCols& t, uint64_t tile, const uint8_t* st) {
  TileView v;
  uint64_t lo, hi;
  tile_range(tile, t.n, &lo, &hi);
  v.st = st;
  v.lo = lo;
  v.da = (uint32_t)((uintptr_t)(t.addr + lo) & 15);
  v.dc = (uint32_t)((uintptr_t)(t.cta + lo) & 15);
  v.dt = (uint32_t)((uintptr_t)(t.tid + lo) & 15);
  v.dw = (uint32_t)((uintptr_t)(t.winst + lo) & 15);
  v.dm = (uint32_t)((uintptr_t)(t.meta + lo) & 15);
  return v;
}

struct Rec {
  uint32_t cta, tid, winst;
  uint8_t meta;
};
__device__ __forceinline__ bool same_run(const Rec& a, const Rec& b) {
  return a.cta == b.cta && (a.tid >> 5) == (b.tid >> 5) && a.winst == b.winst && is_bb(a.meta) == is_bb(b.meta);
}
__device__ __forceinline__ Rec rec_at(const TileView& v, uint64_t i) {
  return Rec{v.cta(i), v.tid(i), v.winst(i), v.meta(i)};
}

__device__ __forceinline__ void report(Scalars* sc, uint64_t i, uint32_t code) {
  atomicMin(&sc->err_index, (unsigned long long)i);
  atomicMax(&sc->err_code, code);
}

// Walks the groups that start in [sub_lo, sub_hi) in batches of 32 records
// and calls op(lane-state) once per batch with every lane's membership.
// op(part, gs, rec, i): part = lane holds a record of a complete, owned
// group; gs = lane index (within the batch) of its run's first record.
template <class Op>
__device__ __forceinline__ void walk_runs(const TileView& v, uint64_t n, uint64_t sub_lo, uint64_t sub_hi,
                                          Scalars* sc, Op& op) {
  const uint32_t lane = lane_id();
  if (sub_lo >= sub_hi) return;
  // first run start inside the sub-range
  uint64_t g0;
  {
    uint64_t i = sub_lo + lane;
    bool st = false;
    if (i < sub_hi) st = (i == 0) || !same_run(rec_at(v, i), rec_at(v, i - 1));
    uint32_t b = __ballot_sync(FULL, st);
    if (!b) {
      if (sub_lo + 32 <= sub_hi && lane == 0) report(sc, sub_lo, 2);
      return;
    }
    g0 = sub_lo + __ffs(b) - 1;
  }
  while (g0 < sub_hi) {
    uint64_t i = g0 + lane;
    bool valid = i < n;
    Rec r{0, 0, 0, 0};
    if (valid) r = rec_at(v, i);
    // start flags (lane 0 is a run start by construction)
    Rec p;
    p.cta = __shfl_up_sync(FULL, r.cta, 1);
    p.tid = __shfl_up_sync(FULL, r.tid, 1);
    p.winst = __shfl_up_sync(FULL, r.winst, 1);
    p.meta = (uint8_t)__shfl_up_sync(FULL, (uint32_t)r.meta, 1);
    bool st = (lane == 0) || !valid || !same_run(r, p);
    uint32_t S = __ballot_sync(FULL, st);
    // does the record after the batch start a new run (or is the trace over)?
    bool e32;
    {
      uint64_t j = g0 + 32;
      e32 = j >= n;
      if (!e32) e32 = !same_run(rec_at(v, j), rec_at(v, j - 1));
    }
    uint32_t gs = 31u - __clz(S & lanemask_le());
    uint32_t after = (gs == 31) ? 0u : (S & ~((2u << gs) - 1u));
    bool complete = after ? true : e32;
    bool owned = (g0 + gs) < sub_hi;
    bool part = valid && owned && complete;
    op(part, gs, r, i);
    // advance to the first run start that was not resolved in this batch
    uint32_t bad = __ballot_sync(FULL, st && !(valid && owned && complete));
    if (bad & 1u) {
      // the batch's first run is incomplete: longer than 32 records
      if (valid && !complete && lane == 0) report(sc, g0, 2);
      break;
    }
    g0 += bad ? (uint32_t)(__ffs(bad) - 1) : 32u;
  }
}

struct MdOp {
  const TileView* v;
  uint32_t lbs, ws;
  uint32_t* s_hist;    // [2][33]
  uint32_t* s_sites;   // [DV_SMEM_SITES][2] or null
  uint64_t* g_sites;   // global [nsites][2] when nsites > DV_SMEM_SITES
  const uint32_t* site;
  uint32_t nsites;
  uint64_t* site_flag;
  Scalars* sc;
  __device__ __forceinline__ void operator()(bool part, uint32_t gs, const Rec& r, uint64_t i) {
    const uint32_t lane = lane_id();
    part = part && is_mem(r.meta);
    uint32_t tag = part ? ((gs << 5) | ((r.tid & 31u) >> ws)) : (1024u + lane);
    uint32_t mt = __match_any_sync(FULL, tag);
    uint64_t line = part ? (v->addr(i) >> lbs) : (~0ull - lane);
    uint32_t ml = __match_any_sync(FULL, line);
    uint32_t mm = mt & ml;
    bool first = part && (uint32_t)(__ffs(mm) - 1) == lane;
    uint32_t fl = __ballot_sync(FULL, first);
    uint32_t ln = __match_any_sync(FULL, part ? ((gs << 5) | (r.tid & 31u)) : (2048u + lane));
    if (part && __popc(ln) > 1) report(sc, i, 2);
    if (part && (uint32_t)(__ffs(mt) - 1) == lane) {
      uint32_t deg = __popc(fl & mt);
      atomicAdd(&s_hist[kind_of(r.meta) * 33 + deg], 1u);
      if (nsites) {
        uint32_t s = __ldg(site + i);
        if (s >= nsites) {
          *site_flag = 1;
        } else if (s_sites) {
          atomicAdd(&s_sites[2 * s], 1u);
          atomicAdd(&s_sites[2 * s + 1], deg);
        } else {
          atomicAdd((unsigned long long*)&g_sites[2 * s], 1ull);
          atomicAdd((unsigned long long*)&g_sites[2 * s + 1], (unsigned long long)deg);
        }
      }
    }
  }
};

struct BdOp {
  uint32_t ws;
  const uint32_t* tc;   // T_c per CTA id
  uint32_t* s_tot;      // [3]
  uint32_t* s_sites;    // [DV_SMEM_SITES][3] or null
  uint64_t* g_sites;
  const uint32_t* site;
  uint32_t nsites;
  uint64_t* site_flag;
  Scalars* sc;
  __device__ __forceinline__ void operator()(bool part, uint32_t gs, const Rec& r, uint64_t i) {
    const uint32_t lane = lane_id();
    part = part && is_bb(r.meta);
    uint32_t tag = part ? ((gs << 5) | ((r.tid & 31u) >> ws)) : (1024u + lane);
    uint32_t mt = __match_any_sync(FULL, tag);
    uint32_t ln = __match_any_sync(FULL, part ? ((gs << 5) | (r.tid & 31u)) : (2048u + lane));
    if (part && __popc(ln) > 1) report(sc, i, 2);
    if (part && (uint32_t)(__ffs(mt) - 1) == lane) {
      uint32_t active = __popc(mt);
      uint32_t W = 1u << ws;
      int64_t live = (int64_t)__ldg(tc + r.cta) - (int64_t)((r.tid >> ws) << ws);
      live = live < 0 ? 0 : (live > (int64_t)W ? (int64_t)W : live);
      uint32_t div = (int64_t)active < live ? 1u : 0u;
      atomicAdd(&s_tot[0], 1u);
      if (div) atomicAdd(&s_tot[1], 1u);
      atomicAdd(&s_tot[2], active);
      if (nsites) {
        uint32_t s = __ldg(site + i);
        if (s >= nsites) {
          *site_flag = 1;
        } else if (s_sites) {
          atomicAdd(&s_sites[3 * s], 1u);
          if (div) atomicAdd(&s_sites[3 * s + 1], 1u);
          atomicAdd(&s_sites[3 * s + 2], active);
        } else {
          atomicAdd((unsigned long long*)&g_sites[3 * s], 1ull);
          if (div) atomicAdd((unsigned long long*)&g_sites[3 * s + 1], 1ull);
          atomicAdd((unsigned long long*)&g_sites[3 * s + 2], (unsigned long long)active);
        }
      }
    }
  }
};

// MODE 0 = memory divergence, 1 = branch divergence.
template <int MODE>
__global__ void __launch_bounds__(DV_NT, 2)
    k_divergence(TraceCols t, uint32_t lbs, uint32_t ws, uint64_t* __restrict__ g_hist, uint64_t* __restrict__ g_sites,
                 uint32_t nsites, uint64_t* site_flag, const uint32_t* __restrict__ tc, Scalars* sc,
                 uint64_t ntiles) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ uint64_t full[DV_S];
  __shared__ uint32_t s_hist[2 * 33];
  constexpr int SW = MODE == 0 ? 2 : 3;
  uint32_t* s_sites = (uint32_t*)(smem + DV_S * STAGE_BYTES);
  const bool sites_in_smem = nsites && nsites <= DV_SMEM_SITES;
  const uint32_t tx = threadIdx.x, lane = lane_id(), warp = tx >> 5;
  for (uint32_t k = tx; k < 2 * 33; k += DV_NT) s_hist[k] = 0;
  if (sites_in_smem)
    for (uint32_t k = tx; k < SW * nsites; k += DV_NT) s_sites[k] = 0;
  if (tx == 0) {
    for (int s = 0; s < DV_S; ++s) mbar_init(&full[s], 1);
    fence_barrier_init();
  }
  __syncthreads();
  if (tx == 0) {
    for (int s = 0; s < DV_S; ++s) {
      uint64_t tile = blockIdx.x + (uint64_t)s * gridDim.x;
      if (tile < ntiles) issue_tile<MODE == 0>(t, tile, smem + s * STAGE_BYTES, &full[s]);
    }
  }
  MdOp md{nullptr, lbs, ws, s_hist, sites_in_smem ? s_sites : nullptr, g_sites, t.site, nsites, site_flag, sc};
  BdOp bd{ws, tc, s_hist, sites_in_smem ? s_sites : nullptr, g_sites, t.site, nsites, site_flag, sc};
  uint32_t j = 0;
  for (uint64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x, ++j) {
    const int s = j % DV_S;
    const uint8_t* st = smem + s * STAGE_BYTES;
    mbar_wait(&full[s], (j / DV_S) & 1u);
    TileView v = make_view(t, tile, st);
    uint64_t t0 = tile * DV_TM;
    uint64_t sub_lo = t0 + (uint64_t)warp * (DV_TM / (DV_NT / 32));
    uint64_t sub_hi = sub_lo + DV_TM / (DV_NT / 32);
    if (sub_hi > t.n) sub_hi = t.n;
    // per-record validity of the records this warp owns
    for (uint64_t i = sub_lo + lane; i < sub_hi; i += 32) {
      uint8_t m = v.meta(i);
      bool ok = meta_ok(m) && v.tid(i) < 1024u;
      if (MODE == 0 && ok) ok = addr_ok(v.addr(i), m);
      if (!ok) report(sc, i, 1);
    }
    if (MODE == 0) {
      md.v = &v;
      walk_runs(v, t.n, sub_lo, sub_hi, sc, md);
    } else {
      walk_runs(v, t.n, sub_lo, sub_hi, sc, bd);
    }
    __syncthreads();
    if (tx == 0) {
      uint64_t nt = tile + (uint64_t)DV_S * gridDim.x;
      if (nt < ntiles) {
        fence_proxy_async();
        issue_tile<MODE == 0>(t, nt, smem + s * STAGE_BYTES, &full[s]);
      }
    }
  }
  __syncthreads();
  if (MODE == 0) {
    for (uint32_t k = tx; k < 2 * 33; k += DV_NT) {
      uint32_t kind = k / 33, deg = k % 33;
      uint32_t W = 1u << ws;
      if (s_hist[k] && deg <= W) atomicAdd((unsigned long long*)&g_hist[kind * (W + 1) + deg], (unsigned long long)s_hist[k]);
    }
  } else {
    if (tx < 3 && s_hist[tx]) atomicAdd((unsigned long long*)&g_hist[tx], (unsigned long long)s_hist[tx]);
  }
  if (sites_in_smem)
    for (uint32_t k = tx; k < SW * nsites; k += DV_NT)
      if (s_sites[k]) atomicAdd((unsigned long long*)&g_sites[k], (unsigned long long)s_sites[k]);
}

// T_c = 1 + max tid over CTA c's basic-block records (one warp-aggregated
// atomicMax per run of equal CTA ids inside a warp's 32 records).
__global__ void __launch_bounds__(256) k_cta_maxtid(const uint32_t* __restrict__ cta, const uint16_t* __restrict__ tid,
                                                    const uint8_t* __restrict__ meta, uint64_t n,
                                                    uint32_t* __restrict__ tc, uint32_t ncta, Scalars* sc) {
  const uint32_t lane = lane_id();
  for (uint64_t base = (blockIdx.x * (uint64_t)blockDim.x + (threadIdx.x & ~31u)); base < n;
       base += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t i = base + lane;
    bool bb = false;
    uint32_t c = 0, v = 0;
    if (i < n) {
      uint8_t m = __ldg(meta + i);
      bb = is_bb(m) && meta_ok(m);
      c = __ldg(cta + i);
      v = (uint32_t)__ldg(tid + i) + 1u;
      if (bb && c >= ncta) bb = false;
    }
    uint32_t key = bb ? c : (0xf0000000u + lane);
    uint32_t mk = __match_any_sync(FULL, key);
    uint32_t mx = __reduce_max_sync(mk, bb ? v : 0u);
    if (bb && (uint32_t)(__ffs(mk) - 1) == lane) atomicMax(&tc[c], mx);
  }
}

int g_dv_blocks[2] = {0, 0};

template <int MODE>
cudaError_t launch_div(cadv_ctx* c, const cadv_trace_desc& d, uint32_t lbs, uint32_t ws, uint64_t* hist,
                       uint64_t* sites, uint32_t nsites, uint64_t* flag, const uint32_t* tc) {
  if (d.n == 0) return cudaSuccess;
  constexpr int SW = MODE == 0 ? 2 : 3;
  size_t smem = (size_t)DV_S * STAGE_BYTES + (size_t)SW * DV_SMEM_SITES * 4;
  auto kern = k_divergence<MODE>;
  if (!g_dv_blocks[MODE]) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    int nb = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, kern, DV_NT, smem);
    if (e != cudaSuccess) return e;
    g_dv_blocks[MODE] = nb > 0 ? nb : 1;
  }
  uint64_t ntiles = (d.n + DV_TM - 1) / DV_TM;
  uint64_t cap = (uint64_t)g_dv_blocks[MODE] * c->num_sms;
  int grid = (int)(ntiles < cap ? ntiles : cap);
  TraceCols t{d.addr, d.cta, d.tid, d.site, d.winst, d.meta, d.n};
  if (MODE == 0)
    CADV_LAUNCH(c, k_divergence<0><<<grid, DV_NT, smem, c->stream>>>(t, lbs, ws, hist, sites, nsites, flag, tc,
                                                                      scalars(c), ntiles));
  else
    CADV_LAUNCH(c, k_divergence<1><<<grid, DV_NT, smem, c->stream>>>(t, lbs, ws, hist, sites, nsites, flag, tc,
                                                                      scalars(c), ntiles));
  return cudaGetLastError();
}

}  // namespace

cudaError_t launch_mem_div(cadv_ctx* c, const cadv_trace_desc& t, uint32_t lb_shift, uint32_t w_shift,
                           uint64_t* d_hist, uint64_t* d_sites, uint32_t nsites) {
  // the site-overflow flag lives right after the per-site block (see cadv.cu)
  uint64_t* flag = d_hist + 2 * ((1u << w_shift) + 1) + 2ull * nsites;
  return launch_div<0>(c, t, lb_shift, w_shift, d_hist, d_sites, nsites, flag, nullptr);
}

cudaError_t launch_cta_maxtid(cadv_ctx* c, const cadv_trace_desc& t, uint32_t* d_tc, uint32_t ncta) {
  if (t.n == 0) return cudaSuccess;
  uint64_t want = (t.n + 255) / 256;
  int grid = (int)(want < (uint64_t)c->num_sms * 8 ? want : (uint64_t)c->num_sms * 8);
  CADV_LAUNCH(c, k_cta_maxtid<<<grid, 256, 0, c->stream>>>(t.cta, t.tid, t.meta, t.n, d_tc, ncta, scalars(c)));
  return cudaGetLastError();
}

cudaError_t launch_branch_div(cadv_ctx* c, const cadv_trace_desc& t, uint32_t w_shift, const uint32_t* d_tc,
                              uint64_t* d_sites, uint32_t nsites, uint64_t* d_totals) {
  uint64_t* flag = d_totals + 3;
  return launch_div<1>(c, t, 0, w_shift, d_totals, d_sites, nsites, flag, d_tc);
}

}  // namespace cadv
