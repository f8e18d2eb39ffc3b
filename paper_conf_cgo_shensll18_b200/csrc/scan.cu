// scan.cu — the fused streaming pass over the raw trace.
//
// One kernel, k_scan<F>, reads each needed trace column exactly once from
// HBM and computes, for the flags in F:
//   F_RD  R1: validation, line keys and run compression of raw-adjacent
//         records of the same (scope, line) (reuse.cu §"run compression"),
//         kept records written in trace order (decoupled look-back);
//   F_MD  M1-M3: unique lines per warp-level group, per kind, per site;
//   F_BD  B1-B3: active lanes per warp-level BB group; groups with every
//         lane of their (sub-)warp active are never divergent and are
//         counted at once, the others go to a short deferred list that
//         k_bd_resolve classifies once T_c (1 + max tid of the CTA's BB
//         records, reduced with fire-and-forget RED.MAX) is complete.
//
// Data movement: persistent CTAs (2 per SM x 16 warps) stream 1024-record
// tiles through a 3-stage shared-memory ring filled by 1-D TMA bulk copies
// (cp.async.bulk.shared::cluster.global + mbarrier complete_tx), one copy
// per column, with a 1-record halo before and 32 after.  Every warp owns 64
// records of a tile:
//   phase 1 (RD): two aligned 32-record windows; a record's predecessor comes
//     from __shfl_up_sync (lane 0: carried from the previous window), chains
//     of stores are cut every 16 (weight <= 16), and the one kept record
//     whose run reaches the window end is carried to the next window.
//   phase 2 (MD/BD): batches of 32 records starting at a group start; when
//     lanes ascend and lines are non-decreasing inside every group (the
//     common, coalesced case) group boundaries and "new line" flags come from
//     one __shfl_up_sync per field and a handful of ballots; otherwise the
//     batch falls back to __match_any_sync on (group, line).
#include <cuda_runtime.h>

#include "cadv_impl.h"
#include "common.cuh"

namespace cadv {
namespace {

constexpr int SC_TM = 1024;                 // records owned per tile
constexpr int SC_NT = 512;                  // 16 warps
constexpr int SC_WARPS = SC_NT / 32;
constexpr int SC_WR = SC_TM / SC_WARPS;     // 64 records per warp
constexpr int SC_S = 3;                     // pipeline stages
constexpr int SC_SITES = 1024;              // per-site counters kept in shared memory up to this many sites
constexpr uint32_t SC_ROWS = SC_TM + 33;    // + 1 before, + 32 after

constexpr uint32_t O_ADDR = 0;
constexpr uint32_t O_CTA = O_ADDR + stage_bytes<uint64_t>(SC_ROWS);
constexpr uint32_t O_TID = O_CTA + stage_bytes<uint32_t>(SC_ROWS);
constexpr uint32_t O_WINST = O_TID + stage_bytes<uint16_t>(SC_ROWS);
constexpr uint32_t O_SITE = O_WINST + stage_bytes<uint32_t>(SC_ROWS);
constexpr uint32_t O_META = O_SITE + stage_bytes<uint32_t>(SC_ROWS);
constexpr uint32_t O_STAGE = (O_META + stage_bytes<uint8_t>(SC_ROWS) + 127) & ~127u;

constexpr uint64_t LINE_MASK = (1ull << 58) - 1;
constexpr int VB_STORE = 58, VB_DUP = 59, VB_W = 60;
constexpr uint64_t LB_AGG = 1ull << 62, LB_PRE = 2ull << 62, LB_VAL = (1ull << 62) - 1;

struct ScanArgs {
  const uint64_t* addr;
  const uint32_t* cta;
  const uint16_t* tid;
  const uint32_t* site;
  const uint32_t* winst;
  const uint8_t* meta;
  uint64_t n, ntiles;
  // RD
  uint32_t lbs_rd;
  int cta_scope;
  uint32_t* kout;
  uint64_t* vout;
  uint64_t* status;
  uint64_t* hist0;
  // MD
  uint32_t lbs_md, ws_md;
  uint64_t* md_hist;   // [2][W+1]
  uint64_t* md_sites;  // [nsites][2] or null
  // BD
  uint32_t ws_bd;
  uint32_t* tc;        // T_c per CTA id (RED.MAX)
  uint64_t* bd_tot;    // [3] exec, divergent, threads
  uint64_t* bd_sites;  // [nsites][3] or null
  uint4* defer;        // deferred partial groups
  unsigned long long* ndefer;
  uint32_t nsites;
  uint64_t* site_flag;
  Scalars* sc;
};

__device__ __forceinline__ uint64_t ld_volatile(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.volatile.global.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}

__device__ __forceinline__ void report(Scalars* sc, uint64_t i, uint32_t code) {
  atomicMin(&sc->err_index, (unsigned long long)i);
  atomicMax(&sc->err_code, code);
}

__device__ __forceinline__ void red_max(uint32_t* p, uint32_t v) {
  asm volatile("red.relaxed.gpu.global.max.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

struct View {
  const uint8_t* st;
  uint64_t lo;
  uint32_t da, dc, dt, dw, ds, dm;
  __device__ __forceinline__ uint32_t li(uint64_t i) const { return (uint32_t)(i - lo); }
  __device__ __forceinline__ uint64_t addr(uint64_t i) const { return *(const uint64_t*)(st + O_ADDR + da + li(i) * 8); }
  __device__ __forceinline__ uint32_t cta(uint64_t i) const { return *(const uint32_t*)(st + O_CTA + dc + li(i) * 4); }
  __device__ __forceinline__ uint32_t tid(uint64_t i) const { return *(const uint16_t*)(st + O_TID + dt + li(i) * 2); }
  __device__ __forceinline__ uint32_t winst(uint64_t i) const {
    return *(const uint32_t*)(st + O_WINST + dw + li(i) * 4);
  }
  __device__ __forceinline__ uint32_t site(uint64_t i) const { return *(const uint32_t*)(st + O_SITE + ds + li(i) * 4); }
  __device__ __forceinline__ uint8_t meta(uint64_t i) const { return st[O_META + dm + li(i)]; }
};

__device__ __forceinline__ void tile_range(uint64_t tile, uint64_t n, uint64_t* lo, uint64_t* hi) {
  uint64_t t0 = tile * SC_TM;
  *lo = t0 ? t0 - 1 : 0;
  uint64_t h = t0 + SC_TM + 32;
  *hi = h < n ? h : n;
}

__device__ __forceinline__ uint32_t hull(const void* b, const void* e) {
  return (uint32_t)((((uintptr_t)e + 15) & ~(uintptr_t)15) - ((uintptr_t)b & ~(uintptr_t)15));
}

template <int F>
__device__ __forceinline__ void issue_tile(const ScanArgs& A, uint64_t tile, uint8_t* st, uint64_t* bar) {
  constexpr bool NA = (F & (F_RD | F_MD)) != 0, NG = (F & (F_MD | F_BD)) != 0;
  uint64_t lo, hi;
  tile_range(tile, A.n, &lo, &hi);
  uint32_t bytes = hull(A.cta + lo, A.cta + hi) + hull(A.meta + lo, A.meta + hi);
  if (NA) bytes += hull(A.addr + lo, A.addr + hi);
  if (NG) bytes += hull(A.tid + lo, A.tid + hi) + hull(A.winst + lo, A.winst + hi) + hull(A.site + lo, A.site + hi);
  mbar_arrive_expect_tx(bar, bytes);
  uint32_t d;
  if (NA) stage_column(A.addr, lo, hi, st + O_ADDR, bar, &d);
  stage_column(A.cta, lo, hi, st + O_CTA, bar, &d);
  if (NG) {
    stage_column(A.tid, lo, hi, st + O_TID, bar, &d);
    stage_column(A.winst, lo, hi, st + O_WINST, bar, &d);
    stage_column(A.site, lo, hi, st + O_SITE, bar, &d);
  }
  stage_column(A.meta, lo, hi, st + O_META, bar, &d);
}

__device__ __forceinline__ View make_view(const ScanArgs& A, uint64_t tile, const uint8_t* st) {
  View v;
  uint64_t lo, hi;
  tile_range(tile, A.n, &lo, &hi);
  v.st = st;
  v.lo = lo;
  v.da = (uint32_t)((uintptr_t)(A.addr + lo) & 15);
  v.dc = (uint32_t)((uintptr_t)(A.cta + lo) & 15);
  v.dt = (uint32_t)((uintptr_t)(A.tid + lo) & 15);
  v.dw = (uint32_t)((uintptr_t)(A.winst + lo) & 15);
  v.ds = (uint32_t)((uintptr_t)(A.site + lo) & 15);
  v.dm = (uint32_t)((uintptr_t)(A.meta + lo) & 15);
  return v;
}

struct Rec {
  uint32_t cta, tid, winst;
  uint32_t meta;
};
__device__ __forceinline__ bool same_run(const Rec& a, const Rec& b) {
  return a.cta == b.cta && ((a.tid ^ b.tid) >> 5) == 0 && a.winst == b.winst &&
         ((a.meta & 3u) == 2u) == ((b.meta & 3u) == 2u);
}
__device__ __forceinline__ Rec rec_at(const View& v, uint64_t i) { return Rec{v.cta(i), v.tid(i), v.winst(i), v.meta(i)}; }

// ------------------------------------------------------------------ phase 1: validation + run compression
struct RdWarp {
  uint32_t cnt;        // kept records in the warp buffer
  uint32_t ndup;       // dropped repeats (RD 0)
};

template <int F>
__device__ __forceinline__ RdWarp phase1(const ScanArgs& A, const View& v, uint64_t s0, uint64_t s1, uint64_t* wbv,
                                         uint32_t* wbk) {
  constexpr bool RD = (F & F_RD) != 0, NA = (F & (F_RD | F_MD)) != 0, NG = (F & (F_MD | F_BD)) != 0;
  const uint32_t lane = lane_id();
  RdWarp out{0, 0};
  // carried state of the record just before the window
  bool c_mem = false, c_st = false;
  uint64_t c_line = 0;
  uint32_t c_scope = 0;
  if (RD && s0 > 0) {
    uint8_t m = v.meta(s0 - 1);
    if (is_mem(m) && meta_ok(m)) {
      uint64_t a = v.addr(s0 - 1);
      if (addr_ok(a, m)) {
        c_mem = true;
        c_st = is_store(m);
        c_line = a >> A.lbs_rd;
        c_scope = A.cta_scope ? v.cta(s0 - 1) : 0u;
      }
    }
  }
  uint64_t cstart = 0;  // global index of the current store chain's first store
  bool pv = false, pst = false;
  uint64_t pline = 0;
  uint32_t pscope = 0, pw = 0;
  for (uint64_t base = s0; base < s1; base += 32) {
    const uint64_t i = base + lane;
    const uint32_t lim = (uint32_t)((s1 - base) < 32 ? (s1 - base) : 32);
    const bool valid = lane < lim;
    uint8_t m = 2;
    uint64_t a = 0;
    bool ok = true;
    if (valid) {
      m = v.meta(i);
      ok = meta_ok(m);
      if (NA && ok && is_mem(m)) {
        a = v.addr(i);
        ok = addr_ok(a, m);
      }
      if (NG && ok) ok = v.tid(i) < 1024u;
      if (!ok) report(A.sc, i, 1);
    }
    if (!RD) continue;
    const bool mem = valid && ok && is_mem(m);
    const bool st = mem && is_store(m);
    const uint64_t line = a >> A.lbs_rd;
    const uint32_t scope = (A.cta_scope && mem) ? v.cta(i) : 0u;
    // predecessor (lane 0: carried)
    bool q_mem = __shfl_up_sync(FULL, (int)mem, 1) != 0, q_st = __shfl_up_sync(FULL, (int)st, 1) != 0;
    uint64_t q_line = __shfl_up_sync(FULL, line, 1);
    uint32_t q_scope = __shfl_up_sync(FULL, scope, 1);
    if (lane == 0) { q_mem = c_mem; q_st = c_st; q_line = c_line; q_scope = c_scope; }
    const bool same = mem && q_mem && scope == q_scope && line == q_line;
    const bool dup = same && !st;
    const bool elig = same && st && q_st && i != s0;
    const uint32_t Mnon = __ballot_sync(FULL, st && !elig);
    const uint32_t below = Mnon & lanemask_le();
    const uint64_t cs = below ? base + (31u - __clz(below)) : cstart;
    const bool merged = elig && ((i - cs) & 15u) != 0;
    const bool keep = mem && !dup && !merged;
    const uint32_t Mmerged = __ballot_sync(FULL, merged);
    const uint32_t Mdup = __ballot_sync(FULL, dup);
    if (Mnon) cstart = base + (31u - __clz(Mnon));
    c_mem = __shfl_sync(FULL, (int)mem, lim - 1) != 0;
    c_st = __shfl_sync(FULL, (int)st, lim - 1) != 0;
    c_line = __shfl_sync(FULL, line, lim - 1);
    c_scope = __shfl_sync(FULL, scope, lim - 1);
    // the record carried from the previous window ends before this window's
    // first non-merged lane
    if (pv) {
      uint32_t e = __ffs(~Mmerged) - 1;
      uint32_t w = pw + (pst ? e : 0u);
      bool hd = e < lim && ((Mdup >> e) & 1u);
      if (lane == 0) {
        wbv[out.cnt] = pline | ((uint64_t)pst << VB_STORE) | ((uint64_t)hd << VB_DUP) | ((uint64_t)(w - 1) << VB_W);
        wbk[out.cnt] = pscope;
      }
      out.cnt++;
      pv = false;
    }
    // end of each kept record's run: next non-merged lane (stores) or the next lane (loads)
    const uint32_t after = ~Mmerged & ~lanemask_le();
    const uint32_t e_l = st ? (after ? (uint32_t)(__ffs(after) - 1) : 32u) : lane + 1;
    const bool fin = keep && e_l < lim;
    const bool pend = keep && e_l >= lim;
    const uint32_t Mfin = __ballot_sync(FULL, fin);
    if (fin) {
      uint32_t w = e_l - lane;
      bool hd = (Mdup >> e_l) & 1u;
      uint32_t pos = out.cnt + __popc(Mfin & lanemask_lt());
      wbv[pos] = line | ((uint64_t)st << VB_STORE) | ((uint64_t)hd << VB_DUP) | ((uint64_t)(w - 1) << VB_W);
      wbk[pos] = scope;
    }
    out.cnt += __popc(Mfin);
    const uint32_t Mp = __ballot_sync(FULL, pend);
    if (Mp) {
      const uint32_t p = __ffs(Mp) - 1;
      pv = true;
      pline = __shfl_sync(FULL, line, p);
      pscope = __shfl_sync(FULL, scope, p);
      pst = __shfl_sync(FULL, (int)st, p) != 0;
      pw = pst ? lim - p : 1u;
    }
    out.ndup += __popc(Mdup);
  }
  if (RD && pv) {
    // the record after the sub-range decides has_dup (it is never merged into us)
    bool hd = false;
    if (s1 < A.n) {
      uint8_t m = v.meta(s1);
      if (is_mem(m) && !is_store(m) && meta_ok(m) && c_mem) {
        uint64_t a = v.addr(s1);
        uint32_t sc = A.cta_scope ? v.cta(s1) : 0u;
        hd = addr_ok(a, m) && (a >> A.lbs_rd) == c_line && sc == c_scope;
      }
    }
    if (lane == 0) {
      wbv[out.cnt] = pline | ((uint64_t)pst << VB_STORE) | ((uint64_t)hd << VB_DUP) | ((uint64_t)(pw - 1) << VB_W);
      wbk[out.cnt] = pscope;
    }
    out.cnt++;
  }
  __syncwarp();
  return out;
}

// ------------------------------------------------------------------ phase 2: warp-level groups
struct GroupSmem {
  uint32_t* md_hist;   // [2][33]
  uint32_t* md_sites;  // [SC_SITES][2] or null
  uint32_t* bd_tot;    // [3]
  uint32_t* bd_sites;  // [SC_SITES][3] or null
};

template <int F>
__device__ __forceinline__ void phase2(const ScanArgs& A, const View& v, uint64_t s0, uint64_t s1, GroupSmem& G) {
  constexpr bool MD = (F & F_MD) != 0, BD = (F & F_BD) != 0;
  const uint32_t lane = lane_id();
  const uint64_t n = A.n;
  if (s0 >= s1) return;
  uint64_t g0;
  {
    uint64_t i = s0 + lane;
    bool st = false;
    if (i < s1) st = (i == 0) || !same_run(rec_at(v, i), rec_at(v, i - 1));
    uint32_t b = __ballot_sync(FULL, st);
    if (!b) {
      if (s0 + 32 <= s1 && lane == 0) report(A.sc, s0, 2);
      return;
    }
    g0 = s0 + __ffs(b) - 1;
  }
  const uint32_t ws_md = A.ws_md, ws_bd = A.ws_bd;
  while (g0 < s1) {
    const uint64_t i = g0 + lane;
    const bool valid = i < n;
    Rec r{0xffffffffu, 0, 0, 2};
    if (valid) r = rec_at(v, i);
    Rec p;
    p.cta = __shfl_up_sync(FULL, r.cta, 1);
    p.tid = __shfl_up_sync(FULL, r.tid, 1);
    p.winst = __shfl_up_sync(FULL, r.winst, 1);
    p.meta = __shfl_up_sync(FULL, r.meta, 1);
    const bool st = lane == 0 || !valid || !same_run(r, p);
    const uint32_t S = __ballot_sync(FULL, st);
    bool e32;
    {
      const uint64_t j = g0 + 32;
      e32 = j >= n;
      if (!e32) {
        Rec l31;
        l31.cta = __shfl_sync(FULL, r.cta, 31);
        l31.tid = __shfl_sync(FULL, r.tid, 31);
        l31.winst = __shfl_sync(FULL, r.winst, 31);
        l31.meta = __shfl_sync(FULL, r.meta, 31);
        e32 = !same_run(rec_at(v, j), l31);
      }
    }
    const uint32_t gs = 31u - __clz(S & lanemask_le());
    const uint32_t after = (gs == 31) ? 0u : (S & ~((2u << gs) - 1u));
    const bool complete = after ? true : e32;
    const bool owned = (g0 + gs) < s1;
    const bool part = valid && owned && complete;
    // lanes ascending inside runs? (then no lane repeats and sub-warps are contiguous)
    const uint32_t lt = r.tid & 31u;
    const bool asc_ok = st || lt > (p.tid & 31u);
    const bool asc = __all_sync(FULL, asc_ok || !part);
    const bool is_bb_rec = (r.meta & 3u) == 2u;
    if (MD) {
      const bool pm = part && !is_bb_rec;
      const uint64_t line = pm ? (v.addr(i) >> A.lbs_md) : 0ull;
      const uint64_t pl = __shfl_up_sync(FULL, line, 1);
      const uint32_t sub = lt >> ws_md, psub = (p.tid & 31u) >> ws_md;
      const bool gst = st || sub != psub;
      const bool mono_ok = gst || line >= pl;
      const bool fast = asc && __all_sync(FULL, mono_ok || !pm);
      uint32_t deg = 0, gmask = 0;
      bool leader;
      if (fast) {
        const uint32_t SG = __ballot_sync(FULL, gst);
        const uint32_t g = 31u - __clz(SG & lanemask_le());
        const uint32_t nx = (g == 31) ? 0u : (SG & ~((2u << g) - 1u));
        const uint32_t ge = nx ? (uint32_t)(__ffs(nx) - 1) : 32u;
        gmask = (ge == 32 ? FULL : ((1u << ge) - 1u)) & ~((1u << g) - 1u);
        const uint32_t NL = __ballot_sync(FULL, pm && (gst || line != pl));
        deg = __popc(NL & gmask);
        leader = pm && lane == g;
      } else {
        const uint32_t tag = pm ? ((gs << 5) | (lt >> ws_md)) : (1024u + lane);
        const uint32_t mt = __match_any_sync(FULL, tag);
        const uint32_t ml = __match_any_sync(FULL, pm ? line : (~0ull - lane));
        const bool first = pm && (uint32_t)(__ffs(mt & ml) - 1) == lane;
        const uint32_t fl = __ballot_sync(FULL, first);
        const uint32_t ln = __match_any_sync(FULL, pm ? ((gs << 5) | lt) : (2048u + lane));
        if (pm && __popc(ln) > 1) report(A.sc, i, 2);
        gmask = mt;
        deg = __popc(fl & mt);
        leader = pm && (uint32_t)(__ffs(mt) - 1) == lane;
      }
      if (leader) {
        atomicAdd(&G.md_hist[(r.meta & 3u) * 33 + deg], 1u);
        if (A.nsites) {
          uint32_t s = v.site(i);
          if (s >= A.nsites) *A.site_flag = 1;
          else if (G.md_sites) { atomicAdd(&G.md_sites[2 * s], 1u); atomicAdd(&G.md_sites[2 * s + 1], deg); }
          else {
            atomicAdd((unsigned long long*)&A.md_sites[2 * s], 1ull);
            atomicAdd((unsigned long long*)&A.md_sites[2 * s + 1], (unsigned long long)deg);
          }
        }
      }
    }
    if (BD) {
      const bool pb = part && is_bb_rec;
      const uint32_t W = 1u << ws_bd;
      const uint32_t sub = lt >> ws_bd, psub = (p.tid & 31u) >> ws_bd;
      const bool gst = st || sub != psub;
      uint32_t active = 0, gmask = 0;
      bool leader;
      if (asc) {
        const uint32_t SG = __ballot_sync(FULL, gst);
        const uint32_t g = 31u - __clz(SG & lanemask_le());
        const uint32_t nx = (g == 31) ? 0u : (SG & ~((2u << g) - 1u));
        const uint32_t ge = nx ? (uint32_t)(__ffs(nx) - 1) : 32u;
        gmask = (ge == 32 ? FULL : ((1u << ge) - 1u)) & ~((1u << g) - 1u);
        active = __popc(gmask);
        leader = pb && lane == g;
        // T_c candidate: the group's last lane holds its largest tid
        if (pb && lane == ge - 1) red_max(A.tc + r.cta, r.tid + 1u);
      } else {
        const uint32_t tag = pb ? ((gs << 5) | (lt >> ws_bd)) : (1024u + lane);
        const uint32_t mt = __match_any_sync(FULL, tag);
        const uint32_t ln = __match_any_sync(FULL, pb ? ((gs << 5) | lt) : (2048u + lane));
        if (pb && __popc(ln) > 1) report(A.sc, i, 2);
        gmask = mt;
        active = __popc(mt);
        leader = pb && (uint32_t)(__ffs(mt) - 1) == lane;
        if (pb) red_max(A.tc + r.cta, r.tid + 1u);
      }
      // groups with all W lanes of their (sub-)warp active can never be divergent
      const bool full = active == W;
      const bool deferred = leader && !full;
      if (leader) {
        atomicAdd(&G.bd_tot[0], 1u);
        atomicAdd(&G.bd_tot[2], active);
      }
      uint32_t s = 0;
      if (leader && A.nsites) {
        s = v.site(i);
        if (s >= A.nsites) { *A.site_flag = 1; }
        else if (G.bd_sites) { atomicAdd(&G.bd_sites[3 * s], 1u); atomicAdd(&G.bd_sites[3 * s + 2], active); }
        else {
          atomicAdd((unsigned long long*)&A.bd_sites[3 * s], 1ull);
          atomicAdd((unsigned long long*)&A.bd_sites[3 * s + 2], (unsigned long long)active);
        }
      }
      const uint32_t MD_ = __ballot_sync(FULL, deferred);
      if (MD_) {
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(A.ndefer, (unsigned long long)__popc(MD_));
        base = __shfl_sync(FULL, base, 0);
        if (deferred) {
          uint32_t k = __popc(MD_ & lanemask_lt());
          A.defer[base + k] = make_uint4(r.cta, r.tid >> ws_bd, active, (s < A.nsites && A.nsites) ? s : 0xffffffffu);
        }
      }
    }
    // advance to the first run start not resolved in this batch
    const uint32_t bad = __ballot_sync(FULL, st && !(valid && owned && complete));
    if (bad & 1u) {
      if (valid && !complete && lane == 0) report(A.sc, g0, 2);
      break;
    }
    g0 += bad ? (uint32_t)(__ffs(bad) - 1) : 32u;
  }
}

// ------------------------------------------------------------------ the fused kernel
template <int F>
__global__ void __launch_bounds__(SC_NT, 2) k_scan(ScanArgs A) {
  constexpr bool RD = (F & F_RD) != 0, MD = (F & F_MD) != 0, BD = (F & F_BD) != 0;
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ uint64_t full[SC_S];
  __shared__ uint32_t s_md_hist[2 * 33];
  __shared__ uint32_t s_bd_tot[3];
  __shared__ uint32_t s_wcnt[SC_WARPS];
  __shared__ uint64_t s_base;
  uint8_t* stages = smem;
  uint64_t* wbv_all = (uint64_t*)(smem + SC_S * O_STAGE);
  uint32_t* wbk_all = (uint32_t*)(wbv_all + SC_TM);
  uint32_t* sites = (uint32_t*)(wbk_all + SC_TM);
  const uint32_t tx = threadIdx.x, lane = lane_id(), warp = tx >> 5;
  const bool sites_smem = A.nsites && A.nsites <= SC_SITES;
  GroupSmem G{s_md_hist, (MD && sites_smem) ? sites : nullptr, s_bd_tot,
              (BD && sites_smem) ? sites + (MD ? 2 * SC_SITES : 0) : nullptr};
  for (uint32_t k = tx; k < 2 * 33; k += SC_NT) s_md_hist[k] = 0;
  if (tx < 3) s_bd_tot[tx] = 0;
  if (sites_smem)
    for (uint32_t k = tx; k < (uint32_t)((MD ? 2 : 0) + (BD ? 3 : 0)) * SC_SITES; k += SC_NT) sites[k] = 0;
  if (tx == 0) {
    for (int s = 0; s < SC_S; ++s) mbar_init(&full[s], 1);
    fence_barrier_init();
  }
  __syncthreads();
  if (tx == 0)
    for (int s = 0; s < SC_S; ++s) {
      uint64_t t = blockIdx.x + (uint64_t)s * gridDim.x;
      if (t < A.ntiles) issue_tile<F>(A, t, stages + s * O_STAGE, &full[s]);
    }
  uint32_t ndup = 0;
  uint32_t j = 0;
  for (uint64_t tile = blockIdx.x; tile < A.ntiles; tile += gridDim.x, ++j) {
    const int s = j % SC_S;
    const uint8_t* st = stages + s * O_STAGE;
    mbar_wait(&full[s], (j / SC_S) & 1u);
    const View v = make_view(A, tile, st);
    const uint64_t t0 = tile * SC_TM;
    uint64_t s0 = t0 + (uint64_t)warp * SC_WR, s1 = s0 + SC_WR;
    if (s1 > A.n) s1 = A.n;
    if (s0 > A.n) s0 = A.n;
    RdWarp rw = phase1<F>(A, v, s0, s1, wbv_all + warp * SC_WR, wbk_all + warp * SC_WR);
    ndup += rw.ndup;
    if (RD) {
      if (lane == 0) s_wcnt[warp] = rw.cnt;
      __syncthreads();
      if (warp == 0) {
        uint32_t c = lane < SC_WARPS ? s_wcnt[lane] : 0u;
        uint32_t x = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          uint32_t y = __shfl_up_sync(FULL, x, o);
          if (lane >= (uint32_t)o) x += y;
        }
        const uint32_t tot = __shfl_sync(FULL, x, 31);
        if (lane < SC_WARPS) s_wcnt[lane] = x - c;  // exclusive
        if (lane == 0) {
          // decoupled look-back for this tile's output offset
          uint64_t excl = 0;
          if (tile == 0) {
            atomicExch((unsigned long long*)&A.status[0], (unsigned long long)(LB_PRE | tot));
          } else {
            atomicExch((unsigned long long*)&A.status[tile], (unsigned long long)(LB_AGG | tot));
            int64_t k = (int64_t)tile - 1;
            while (k >= 0) {
              uint64_t sv = ld_volatile(A.status + k);
              if (sv & LB_PRE) { excl += sv & LB_VAL; break; }
              if (sv & LB_AGG) { excl += sv & LB_VAL; --k; }
            }
            __threadfence();
            atomicExch((unsigned long long*)&A.status[tile], (unsigned long long)(LB_PRE | (excl + tot)));
          }
          s_base = excl;
        }
      }
    }
    if (MD || BD) phase2<F>(A, v, s0, s1, G);
    if (RD) {
      __syncthreads();
      const uint64_t gb = s_base + s_wcnt[warp];
      const uint64_t* wbv = wbv_all + warp * SC_WR;
      const uint32_t* wbk = wbk_all + warp * SC_WR;
      for (uint32_t k = lane; k < rw.cnt; k += 32) {
        A.vout[gb + k] = wbv[k];
        if (A.kout) A.kout[gb + k] = wbk[k];
      }
    }
    __syncthreads();
    if (tx == 0) {
      uint64_t nt = tile + (uint64_t)SC_S * gridDim.x;
      if (nt < A.ntiles) {
        fence_proxy_async();
        issue_tile<F>(A, nt, stages + s * O_STAGE, &full[s]);
      }
    }
  }
  // ---- flush block-level counters
  if (RD && lane == 0 && ndup) atomicAdd((unsigned long long*)A.hist0, (unsigned long long)ndup);  // warp-uniform
  __syncthreads();
  if (MD) {
    const uint32_t W = 1u << A.ws_md;
    for (uint32_t k = tx; k < 2 * 33; k += SC_NT) {
      uint32_t kind = k / 33, deg = k % 33;
      if (s_md_hist[k] && deg <= W)
        atomicAdd((unsigned long long*)&A.md_hist[kind * (W + 1) + deg], (unsigned long long)s_md_hist[k]);
    }
    if (G.md_sites)
      for (uint32_t k = tx; k < 2 * A.nsites; k += SC_NT)
        if (G.md_sites[k]) atomicAdd((unsigned long long*)&A.md_sites[k], (unsigned long long)G.md_sites[k]);
  }
  if (BD) {
    if (tx < 3 && s_bd_tot[tx]) atomicAdd((unsigned long long*)&A.bd_tot[tx], (unsigned long long)s_bd_tot[tx]);
    if (G.bd_sites)
      for (uint32_t k = tx; k < 3 * A.nsites; k += SC_NT)
        if (G.bd_sites[k]) atomicAdd((unsigned long long*)&A.bd_sites[k], (unsigned long long)G.bd_sites[k]);
  }
}

// Deferred BD groups: divergent iff active < clamp(T_c - w*W, 0, W).
__global__ void __launch_bounds__(256) k_bd_resolve(const uint4* __restrict__ defer, uint64_t m,
                                                    const uint32_t* __restrict__ tc, uint32_t ws,
                                                    uint64_t* bd_tot, uint64_t* bd_sites, uint32_t nsites) {
  __shared__ uint32_t s_div[SC_SITES];
  const bool sm = nsites && nsites <= SC_SITES;
  if (sm)
    for (uint32_t k = threadIdx.x; k < nsites; k += blockDim.x) s_div[k] = 0;
  __syncthreads();
  uint32_t tot = 0;
  const uint32_t W = 1u << ws;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    uint4 d = defer[i];
    int64_t live = (int64_t)__ldg(tc + d.x) - (int64_t)d.y * W;
    live = live < 0 ? 0 : (live > (int64_t)W ? (int64_t)W : live);
    if ((int64_t)d.z < live) {
      tot++;
      if (d.w != 0xffffffffu) {
        if (sm) atomicAdd(&s_div[d.w], 1u);
        else atomicAdd((unsigned long long*)&bd_sites[3ull * d.w + 1], 1ull);
      }
    }
  }
  tot = __reduce_add_sync(FULL, tot);
  if (lane_id() == 0 && tot) atomicAdd((unsigned long long*)&bd_tot[1], (unsigned long long)tot);
  __syncthreads();
  if (sm)
    for (uint32_t k = threadIdx.x; k < nsites; k += blockDim.x)
      if (s_div[k]) atomicAdd((unsigned long long*)&bd_sites[3ull * k + 1], (unsigned long long)s_div[k]);
}

template <int F>
size_t scan_smem() {
  constexpr bool MD = (F & F_MD) != 0, BD = (F & F_BD) != 0;
  return (size_t)SC_S * O_STAGE + (size_t)SC_TM * 12 + (size_t)((MD ? 2 : 0) + (BD ? 3 : 0)) * SC_SITES * 4;
}

int g_scan_blocks[8] = {0, 0, 0, 0, 0, 0, 0, 0};

template <int F>
cudaError_t launch_scan_t(cadv_ctx* c, const ScanArgs& A) {
  size_t smem = scan_smem<F>();
  if (!g_scan_blocks[F]) {
    cudaError_t e = cudaFuncSetAttribute(k_scan<F>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    int nb = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_scan<F>, SC_NT, smem);
    if (e != cudaSuccess) return e;
    g_scan_blocks[F] = nb > 0 ? nb : 1;
  }
  uint64_t cap = (uint64_t)g_scan_blocks[F] * c->num_sms;
  int grid = (int)(A.ntiles < cap ? A.ntiles : cap);
  CADV_LAUNCH(c, k_scan<F><<<grid, SC_NT, smem, c->stream>>>(A));
  return cudaGetLastError();
}

}  // namespace

uint64_t scan_tiles(uint64_t n) { return (n + SC_TM - 1) / SC_TM; }

cudaError_t launch_scan(cadv_ctx* c, int flags, const ScanParams& P) {
  const cadv_trace_desc& t = P.t;
  if (t.n == 0) return cudaSuccess;
  ScanArgs A{};
  A.addr = t.addr; A.cta = t.cta; A.tid = t.tid; A.site = t.site; A.winst = t.winst; A.meta = t.meta;
  A.n = t.n;
  A.ntiles = scan_tiles(t.n);
  A.lbs_rd = P.lbs_rd; A.cta_scope = P.cta_scope; A.kout = P.kout; A.vout = P.vout; A.status = P.status;
  A.hist0 = P.hist0;
  A.lbs_md = P.lbs_md; A.ws_md = P.ws_md; A.md_hist = P.md_hist; A.md_sites = P.md_sites;
  A.ws_bd = P.ws_bd; A.tc = P.tc; A.bd_tot = P.bd_tot; A.bd_sites = P.bd_sites; A.defer = (uint4*)P.defer;
  A.ndefer = (unsigned long long*)P.ndefer;
  A.nsites = P.nsites; A.site_flag = P.site_flag; A.sc = scalars(c);
  switch (flags) {
    case 1: return launch_scan_t<1>(c, A);
    case 2: return launch_scan_t<2>(c, A);
    case 3: return launch_scan_t<3>(c, A);
    case 4: return launch_scan_t<4>(c, A);
    case 5: return launch_scan_t<5>(c, A);
    case 6: return launch_scan_t<6>(c, A);
    case 7: return launch_scan_t<7>(c, A);
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t launch_bd_resolve(cadv_ctx* c, const void* defer, uint64_t m, const uint32_t* tc, uint32_t ws,
                              uint64_t* bd_tot, uint64_t* bd_sites, uint32_t nsites) {
  if (m == 0) return cudaSuccess;
  uint64_t want = (m + 255) / 256;
  int grid = (int)(want < (uint64_t)c->num_sms * 4 ? want : (uint64_t)c->num_sms * 4);
  CADV_LAUNCH(c, k_bd_resolve<<<grid, 256, 0, c->stream>>>((const uint4*)defer, m, tc, ws, bd_tot, bd_sites, nsites));
  return cudaGetLastError();
}

}  // namespace cadv
