// scan.cu — the fused streaming pass over the raw trace (k_scan<F>).
//
// One kernel reads each needed trace column exactly once from HBM and
// computes, for the flags in F:
//   F_RD  R1: validation, line keys and run compression of raw-adjacent
//         records of the same (scope, line) (reuse.cu "run compression");
//         kept records are written in trace order into per-warp regions
//         that k_squeeze packs afterwards;
//   F_MD  M1-M3: unique lines per warp-level group, per kind and per site;
//   F_BD  B1-B3: active lanes per warp-level BB group; groups with all W
//         lanes of their (sub-)warp active can never be divergent and are
//         counted at once, the others go to a deferred list that
//         k_bd_resolve classifies once T_c (1 + max tid of the CTA's BB
//         records, reduced with fire-and-forget RED.MAX) is complete.
//
// Data movement (B200): one persistent CTA per SM, 20 independent warps.
// Every warp owns a contiguous chunk of the trace and streams it through a
// private ring of 3 x 128-record pieces in shared memory, filled by 1-D TMA
// bulk copies (cp.async.bulk + a per-warp mbarrier per piece).  There is no
// block-level barrier in the loop.  A warp walks its chunk in batches of 32
// records that start at a run start (run = records of one (cta, warp32,
// winst, family)); every run that is complete inside the batch is resolved
// at once:
//   fast path  (lanes ascend inside the run and, for MD, lines do not
//              decrease inside a sub-warp group): group boundaries and
//              "first use of a line" flags come from one __shfl_up_sync per
//              field plus ballots and popcounts;
//   otherwise  __match_any_sync on (group, line) and (group, lane).
// The batch then advances to the first run that is not complete.  Runs are
// owned by the chunk that contains their first record; reuse-distance run
// compression consumes exactly the chunk's records.
#include <cuda_runtime.h>

#include "cadv_impl.h"
#include "common.cuh"

namespace cadv {
namespace {

constexpr int KR = 128;                // records per piece
constexpr int KS = 3;                  // pieces in flight per warp
constexpr int RING = KR * KS;          // 384 ring slots: record j lives in stage (j / KR) % KS
constexpr int NWARP = 20;              // warps per CTA (one CTA per SM)
constexpr int NTHR = NWARP * 32;
constexpr int NSITE_SMEM = 1024;       // per-site counters kept in shared memory up to this many sites

__device__ __forceinline__ uint32_t ring_slot(uint32_t j) {  // chunk-relative record -> ring slot
  const uint32_t p = j >> 7;                                    // KR = 128
  return (p - (p / KS) * KS) * KR + (j & (KR - 1));
}

// per-warp ring (bytes); every column region is a multiple of 128 B
constexpr uint32_t R_ADDR = 0;
constexpr uint32_t R_CTA = R_ADDR + RING * 8;
constexpr uint32_t R_TID = R_CTA + RING * 4;
constexpr uint32_t R_WINST = R_TID + RING * 2;
constexpr uint32_t R_SITE = R_WINST + RING * 4;
constexpr uint32_t R_META = R_SITE + RING * 4;
constexpr uint32_t R_BYTES = R_META + RING;

constexpr uint64_t LINE_MASK = (1ull << 58) - 1;
constexpr int VB_STORE = 58, VB_DUP = 59, VB_W = 60;

struct ScanArgs {
  const uint64_t* addr;
  const uint32_t* cta;
  const uint16_t* tid;
  const uint32_t* site;
  const uint32_t* winst;
  const uint8_t* meta;
  uint64_t n;
  uint64_t chunk;        // records per warp chunk (multiple of KR)
  // RD
  uint32_t lbs_rd;
  int cta_scope;
  uint32_t* kout;        // gapped output: warp w writes from w * chunk
  uint64_t* vout;
  uint64_t* wcnt;        // kept records per warp
  uint64_t* hist0;
  // MD
  uint32_t lbs_md, ws_md;
  uint64_t* md_hist;     // [2][W+1]
  uint64_t* md_sites;    // [nsites][2] or null
  // BD
  uint32_t ws_bd;
  uint32_t* tc;          // T_c per CTA id (RED.MAX)
  uint64_t* bd_tot;      // [3] exec, divergent, threads
  uint64_t* bd_sites;    // [nsites][3] or null
  uint4* defer;          // deferred partial groups
  unsigned long long* ndefer;
  uint32_t nsites;
  uint64_t* site_flag;
  Scalars* sc;
};

__device__ __forceinline__ void report(Scalars* sc, uint64_t i, uint32_t code) {
  atomicMin(&sc->err_index, (unsigned long long)i);
  atomicMax(&sc->err_code, code);
}

__device__ __forceinline__ void red_max(uint32_t* p, uint32_t v) {
  asm volatile("red.relaxed.gpu.global.max.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// bits [a, e) of a lane mask, 0 <= a < e <= 32
__device__ __forceinline__ uint32_t bits_from(uint32_t a, uint32_t e) {
  const uint32_t hi = e >= 32 ? FULL : ((1u << e) - 1u);
  return hi & ~((1u << a) - 1u);
}

struct Counters {        // block-level shared-memory accumulators
  uint32_t* md_hist;     // [2][33]
  uint32_t* md_sites;    // [NSITE_SMEM][2] or null
  uint32_t* bd_tot;      // [3]
  uint32_t* bd_sites;    // [NSITE_SMEM][3] or null
};

// Per-site counter update: shared-memory counters when the site table fits,
// global counters otherwise; an out-of-range site raises the site flag.
__device__ __forceinline__ void site_add(const ScanArgs& A, uint32_t* smem_tab, uint64_t* gtab, uint32_t stride,
                                         uint32_t s, uint32_t v0, uint32_t v_last) {
  if (s >= A.nsites) { *A.site_flag = 1; return; }
  if (smem_tab) {
    atomicAdd(&smem_tab[stride * s], v0);
    atomicAdd(&smem_tab[stride * s + stride - 1], v_last);
  } else {
    atomicAdd((unsigned long long*)&gtab[stride * s], (unsigned long long)v0);
    atomicAdd((unsigned long long*)&gtab[stride * s + stride - 1], (unsigned long long)v_last);
  }
}

// Per-warp TMA issuer: global column pointers at the chunk start, ring
// shared-memory addresses, and the byte count of a full piece, computed once.
template <int F>
struct Issuer {
  static constexpr bool NA = (F & (F_RD | F_MD)) != 0, NG = (F & (F_MD | F_BD)) != 0;
  static constexpr uint32_t FULL_BYTES = KR * (4 + 1 + (NA ? 8 : 0) + (NG ? 2 + 4 + 4 : 0));
  const uint8_t *ga, *gc, *gt, *gw, *gs, *gm;  // column bytes at record c_lo
  uint32_t sa, sc, st, sw, ss, sm, sbar;       // shared addresses of stage 0 / barrier 0
  uint64_t c_lo, s_end;
  __device__ __forceinline__ void init(const ScanArgs& A, uint8_t* ring, uint64_t* bar, uint64_t lo, uint64_t end) {
    c_lo = lo;
    s_end = end;
    ga = (const uint8_t*)(A.addr + lo); gc = (const uint8_t*)(A.cta + lo); gt = (const uint8_t*)(A.tid + lo);
    gw = (const uint8_t*)(A.winst + lo); gs = (const uint8_t*)(A.site + lo); gm = (const uint8_t*)(A.meta + lo);
    const uint32_t r = smem_u32(ring);
    sa = r + R_ADDR; sc = r + R_CTA; st = r + R_TID; sw = r + R_WINST; ss = r + R_SITE; sm = r + R_META;
    sbar = smem_u32(bar);
  }
  __device__ __forceinline__ static void cp(uint32_t dst, const uint8_t* src, uint32_t bytes, uint32_t bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
                 "l"(src), "r"(bytes), "r"(bar)
                 : "memory");
  }
  // piece p -> stage p % KS
  __device__ __forceinline__ void issue(uint32_t p) const {
    const uint32_t stg = p % KS, bar = sbar + stg * 8;
    const uint64_t q0 = c_lo + (uint64_t)p * KR;
    const uint32_t off = p * KR;
    if (q0 + KR <= s_end) {
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(FULL_BYTES) : "memory");
      if (NA) cp(sa + stg * KR * 8, ga + (size_t)off * 8, KR * 8, bar);
      cp(sc + stg * KR * 4, gc + (size_t)off * 4, KR * 4, bar);
      if (NG) {
        cp(st + stg * KR * 2, gt + (size_t)off * 2, KR * 2, bar);
        cp(sw + stg * KR * 4, gw + (size_t)off * 4, KR * 4, bar);
        cp(ss + stg * KR * 4, gs + (size_t)off * 4, KR * 4, bar);
      }
      cp(sm + stg * KR, gm + off, KR, bar);
    } else {
      // the last (partial) piece: sizes rounded up to 16 bytes
      const uint32_t cnt = (uint32_t)(s_end - q0);
      auto r16 = [](uint32_t b) { return (b + 15u) & ~15u; };
      uint32_t bytes = r16(cnt * 4) + r16(cnt);
      if (NA) bytes += r16(cnt * 8);
      if (NG) bytes += r16(cnt * 2) + 2 * r16(cnt * 4);
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
      if (NA) cp(sa + stg * KR * 8, ga + (size_t)off * 8, r16(cnt * 8), bar);
      cp(sc + stg * KR * 4, gc + (size_t)off * 4, r16(cnt * 4), bar);
      if (NG) {
        cp(st + stg * KR * 2, gt + (size_t)off * 2, r16(cnt * 2), bar);
        cp(sw + stg * KR * 4, gw + (size_t)off * 4, r16(cnt * 4), bar);
        cp(ss + stg * KR * 4, gs + (size_t)off * 4, r16(cnt * 4), bar);
      }
      cp(sm + stg * KR, gm + off, r16(cnt), bar);
    }
  }
};

// run identity: (cta, warp32, winst, family)
__device__ __forceinline__ uint32_t run_hi(uint32_t tid, uint32_t meta) {
  return (tid >> 5) | (((meta & 3u) == 2u) ? 64u : 0u);
}

template <int F>
__global__ void __launch_bounds__(NTHR, 1) k_scan(ScanArgs A) {
  constexpr bool RD = (F & F_RD) != 0, MD = (F & F_MD) != 0, BD = (F & F_BD) != 0;
  constexpr bool NA = (F & (F_RD | F_MD)) != 0, NG = (F & (F_MD | F_BD)) != 0;
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ uint64_t bars[NWARP][KS];
  __shared__ uint32_t s_md_hist[2 * 33];
  __shared__ uint32_t s_bd_tot[3];
  const uint32_t tx = threadIdx.x, lane = lane_id(), warp = tx >> 5;
  uint32_t* sites = (uint32_t*)(smem + NWARP * R_BYTES);
  uint32_t* wh_all = sites + ((MD ? 2 : 0) + (BD ? 3 : 0)) * NSITE_SMEM;
  const bool sites_smem = A.nsites && A.nsites <= NSITE_SMEM;
  Counters C{s_md_hist, (MD && sites_smem) ? sites : nullptr, s_bd_tot,
             (BD && sites_smem) ? sites + (MD ? 2 * NSITE_SMEM : 0) : nullptr};
  for (uint32_t k = tx; k < 2 * 33; k += NTHR) s_md_hist[k] = 0;
  if (tx < 3) s_bd_tot[tx] = 0;
  if (sites_smem)
    for (uint32_t k = tx; k < (uint32_t)((MD ? 2 : 0) + (BD ? 3 : 0)) * NSITE_SMEM; k += NTHR) sites[k] = 0;
  __syncthreads();

  uint8_t* ring = smem + warp * R_BYTES;
  uint64_t* bar = bars[warp];
  const uint64_t gw = (uint64_t)blockIdx.x * NWARP + warp;
  const uint64_t c_lo = gw * A.chunk;
  const uint64_t c_hi = c_lo + A.chunk < A.n ? c_lo + A.chunk : A.n;
  uint32_t kept = 0, ndup = 0, bd_exec = 0, bd_threads = 0;
  uint32_t* whist = wh_all + warp * 68;  // warp-private MD histogram [2][33]
  for (uint32_t k = lane; k < 68; k += 32) whist[k] = 0;
  __syncwarp();
  if (c_lo < A.n) {
    const uint32_t clen = (uint32_t)(c_hi - c_lo);
    const uint64_t s_end = c_hi + 32 < A.n ? c_hi + 32 : A.n;     // lookahead for the last runs
    const uint32_t slen = (uint32_t)(s_end - c_lo);
    const uint32_t npieces = (slen + KR - 1) / KR;
    const uint64_t nrel64 = A.n - c_lo;
    const uint32_t nrel = nrel64 < 0xffffffffull ? (uint32_t)nrel64 : 0xffffffffu;
    if (lane == 0) {
      for (int s = 0; s < KS; ++s) mbar_init(&bar[s], 1);
      fence_barrier_init();
    }
    __syncwarp();
    uint32_t issued = 0, waited = 0;
    Issuer<F> io;
    io.init(A, ring, bar, c_lo, s_end);
    if (lane == 0)
      for (; issued < (uint32_t)KS && issued < npieces; ++issued) io.issue(issued);
    issued = __shfl_sync(FULL, issued, 0);
    const uint64_t* r_addr = (const uint64_t*)(ring + R_ADDR);
    const uint32_t* r_cta = (const uint32_t*)(ring + R_CTA);
    const uint16_t* r_tid = (const uint16_t*)(ring + R_TID);
    const uint32_t* r_winst = (const uint32_t*)(ring + R_WINST);
    const uint32_t* r_site = (const uint32_t*)(ring + R_SITE);
    const uint8_t* r_meta = ring + R_META;

    // previous record (the one before the batch), warp-uniform
    uint32_t p_cta = 0xffffffffu, p_tm = 3u << 16, p_winst = 0;  // meta 3: "no record"
    uint64_t p_addr = 0;
    if (c_lo > 0) {
      p_cta = __ldg(A.cta + c_lo - 1);
      uint32_t pm0 = __ldg(A.meta + c_lo - 1);
      if (NA) p_addr = __ldg(A.addr + c_lo - 1);
      // an invalid record never continues a run of compressible accesses
      if (!meta_ok((uint8_t)pm0) || (NA && is_mem((uint8_t)pm0) && !addr_ok(p_addr, (uint8_t)pm0))) pm0 = 3;
      p_tm = (pm0 << 16) | (NG ? (uint32_t)__ldg(A.tid + c_lo - 1) : 0u);
      if (NG) p_winst = __ldg(A.winst + c_lo - 1);
    }
    uint32_t p_rk = run_hi(p_tm & 0xffffu, p_tm >> 16);
    // RD carried state; r_* = the chunk's last record seen by the compression
    bool pv = false, pst = false, r_mem = false;
    uint64_t r_line = 0;
    uint32_t r_scope = 0;
    uint64_t pline = 0;
    uint32_t pscope = 0, pw = 0, cstart = 0;  // cstart: chunk-relative index of the current store chain start
    uint64_t* wbv = A.vout ? A.vout + gw * A.chunk : nullptr;
    uint32_t* wbk = A.kout ? A.kout + gw * A.chunk : nullptr;
    const uint32_t ws_md = A.ws_md, ws_bd = A.ws_bd;

    uint32_t g = 0;
    while (g < clen) {
      // ---- pieces needed for records [g, g + 33)
      const uint32_t need = (g + 33 < slen) ? g + 33 : slen;
      while (waited * KR < need) {
        mbar_wait(&bar[waited % KS], (waited / KS) & 1u);
        ++waited;
      }
      // ---- this batch's records (tm = tid | meta << 16)
      const uint32_t j = g + lane;
      const bool inb = j < slen;
      const uint32_t slot = ring_slot(j);
      uint32_t c = 0xfffffffeu, tm = 3u << 16, w = 0;
      uint64_t a = 0;
      if (inb) {
        c = r_cta[slot];
        tm = ((uint32_t)r_meta[slot] << 16) | (NG ? (uint32_t)r_tid[slot] : 0u);
        if (NG) w = r_winst[slot];
        if (NA) a = r_addr[slot];
      }
      // predecessor record
      uint32_t pc = __shfl_up_sync(FULL, c, 1), ptm = __shfl_up_sync(FULL, tm, 1), pwi = __shfl_up_sync(FULL, w, 1);
      const uint32_t rk = run_hi(tm & 0xffffu, tm >> 16);
      uint32_t prk = __shfl_up_sync(FULL, rk, 1);
      if (lane == 0) prk = p_rk;
      uint64_t pa = __shfl_up_sync(FULL, a, 1);
      if (lane == 0) { pc = p_cta; ptm = p_tm; pwi = p_winst; pa = p_addr; }
      uint32_t m = tm >> 16;
      const uint32_t t = tm & 0xffffu, pm = ptm >> 16, pt = ptm & 0xffffu;
      // ---- run structure (only needed for the divergence analyses)
      uint32_t adv;
      uint32_t S = 0, e32 = 1;
      bool rs = true;
      if (NG) {
        rs = !inb || c != pc || w != pwi || rk != prk;
        S = __ballot_sync(FULL, rs);
        // does the record after the batch start a new run?
        const uint32_t j32 = g + 32;
        const uint32_t c31 = __shfl_sync(FULL, c, 31), rk31 = __shfl_sync(FULL, rk, 31),
                       w31 = __shfl_sync(FULL, w, 31);
        if (j32 < nrel) {
          const uint32_t s32 = ring_slot(j32);
          const uint32_t c32 = r_cta[s32], tm32 = ((uint32_t)r_meta[s32] << 16) | r_tid[s32], w32 = r_winst[s32];
          e32 = (c32 != c31 || w32 != w31 || run_hi(tm32 & 0xffffu, tm32 >> 16) != rk31) ? 1u : 0u;
        }
      }
      const uint32_t S1 = S | 1u;                                   // lane 0 always opens a (pseudo) run
      const uint32_t gs = 31u - __clz(S1 & lanemask_le());          // first lane of this lane's run
      const bool complete = (S1 & ~lanemask_le() & ~((1u << gs) - 1u)) != 0 || e32;
      const bool real = (S >> gs) & 1u;                             // the run starts inside the batch
      const bool owned = real && (g + gs) < clen;
      if (NG) {
        const uint32_t inc = __ballot_sync(FULL, lane == gs && !complete);
        if (inc & 1u) {
          // the batch's first run is longer than 32 records
          if (lane == 0) report(A.sc, c_lo + g, 2);
          break;
        }
        adv = inc ? (uint32_t)(__ffs(inc) - 1) : 32u;
        if (g + adv > slen) adv = slen - g;
      } else {
        adv = (slen - g) < 32u ? (slen - g) : 32u;
      }
      // ---- per-record validity (each record of the chunk once)
      if (lane < adv && j < clen) {
        bool ok = meta_ok((uint8_t)m);
        if (NA && ok && is_mem((uint8_t)m)) ok = addr_ok(a, (uint8_t)m);
        if (NG && ok) ok = t < 1024u;
        if (!ok) {
          report(A.sc, c_lo + j, 1);
          m = 3;  // treat as "no record" below
        }
      }
      const bool part = inb && owned && complete;
      const uint32_t lt = t & 31u, plt = pt & 31u;
      const bool pmem = part && (m & 3u) < 2u;
      const bool pbb = part && (m & 3u) == 2u;
      // ---- M1-M3 memory divergence
      if (MD && __any_sync(FULL, pmem)) {
        const uint64_t line = a >> A.lbs_md, pl = pa >> A.lbs_md;
        const bool gst = rs || ((lt ^ plt) >> ws_md) != 0;
        const bool bad = pmem && !rs && (lt <= plt || (!gst && line < pl));
        uint32_t LEAD, deg;
        if (!__any_sync(FULL, bad)) {
          const uint32_t SG = __ballot_sync(FULL, gst);
          const uint32_t nxg = SG & ~lanemask_le();
          const uint32_t ge = nxg ? (uint32_t)(__ffs(nxg) - 1) : 32u;
          const uint32_t NL = __ballot_sync(FULL, pmem && (gst || line != pl));
          deg = __popc(NL & bits_from(lane, ge));
          LEAD = __ballot_sync(FULL, pmem && gst);
        } else {
          const uint32_t sub = lt >> ws_md;
          const uint32_t tag = pmem ? ((gs << 5) | sub) : (1024u + lane);
          const uint32_t mt = __match_any_sync(FULL, tag);
          const uint32_t ml = __match_any_sync(FULL, pmem ? line : (~0ull - lane));
          const uint32_t fl = __ballot_sync(FULL, pmem && (uint32_t)(__ffs(mt & ml) - 1) == lane);
          const uint32_t ln = __match_any_sync(FULL, pmem ? ((gs << 5) | lt) : (2048u + lane));
          if (pmem && __popc(ln) > 1) report(A.sc, c_lo + j, 2);
          deg = __popc(fl & mt);
          LEAD = __ballot_sync(FULL, pmem && (uint32_t)(__ffs(mt) - 1) == lane);
        }
        const uint32_t s = inb ? r_site[slot] : 0u;
        // leaders update the counters in parallel (shared-memory atomics)
        if ((LEAD >> lane) & 1u) {
          atomicAdd(&whist[(m & 3u) * 33 + deg], 1u);
          if (sites_smem) {
            if (s < A.nsites) { atomicAdd(&C.md_sites[2 * s], 1u); atomicAdd(&C.md_sites[2 * s + 1], deg); }
            else *A.site_flag = 1;
          } else if (A.nsites) {
            site_add(A, nullptr, A.md_sites, 2, s, 1, deg);
          }
        }
      }
      // ---- B1-B3 branch divergence
      if (BD && __any_sync(FULL, pbb)) {
        const uint32_t W = 1u << ws_bd;
        const bool gst = rs || ((lt ^ plt) >> ws_bd) != 0;
        const bool bad = pbb && !rs && lt <= plt;
        uint32_t LEAD, cnt;
        const uint32_t CN = __ballot_sync(FULL, pbb);
        if (!__any_sync(FULL, bad)) {
          const uint32_t SG = __ballot_sync(FULL, gst);
          const uint32_t nxg = SG & ~lanemask_le();
          const uint32_t ge = nxg ? (uint32_t)(__ffs(nxg) - 1) : 32u;
          cnt = __popc(CN & bits_from(lane, ge));
          LEAD = __ballot_sync(FULL, pbb && gst);
          // the group's last lane holds its largest tid
          if (pbb && ge == lane + 1u) red_max(A.tc + c, t + 1u);
        } else {
          const uint32_t sub = lt >> ws_bd;
          const uint32_t tag = pbb ? ((gs << 5) | sub) : (1024u + lane);
          const uint32_t mt = __match_any_sync(FULL, tag);
          const uint32_t ln = __match_any_sync(FULL, pbb ? ((gs << 5) | lt) : (2048u + lane));
          if (pbb && __popc(ln) > 1) report(A.sc, c_lo + j, 2);
          cnt = __popc(mt);
          LEAD = __ballot_sync(FULL, pbb && (uint32_t)(__ffs(mt) - 1) == lane);
          if (pbb) red_max(A.tc + c, t + 1u);
        }
        bd_exec += __popc(LEAD);
        bd_threads += __popc(CN);
        const uint32_t s = inb ? r_site[slot] : 0u;
        // leaders update the per-site counters (shared-memory atomics, different sites in parallel)
        const bool lead = (LEAD >> lane) & 1u;
        if (lead) {
          if (sites_smem) {
            if (s < A.nsites) { atomicAdd(&C.bd_sites[3 * s], 1u); atomicAdd(&C.bd_sites[3 * s + 2], cnt); }
            else *A.site_flag = 1;
          } else if (A.nsites) {
            site_add(A, nullptr, A.bd_sites, 3, s, 1, cnt);
          }
        }
        // groups with fewer than W lanes: divergence decided once T_c is known
        const bool dfr = lead && cnt < W;
        const uint32_t MDF = __ballot_sync(FULL, dfr);
        if (MDF) {
          unsigned long long base = 0;
          if (lane == 0) base = atomicAdd(A.ndefer, (unsigned long long)__popc(MDF));
          base = __shfl_sync(FULL, base, 0);
          if (dfr)
            A.defer[base + __popc(MDF & lanemask_lt())] =
                make_uint4(c, t >> ws_bd, cnt, (A.nsites && s < A.nsites) ? s : 0xffffffffu);
        }
      }
      // ---- R1 run compression over the consumed records of this chunk
      const uint32_t rlim = (clen - g) < adv ? (clen - g) : adv;
      const bool rd_any = RD && __any_sync(FULL, lane < rlim && (m & 3u) < 2u);
      if (RD && !rd_any) {
        // no memory record in this batch: close the carried record, forget the predecessor
        if (pv) {
          if (lane == 0) {
            wbv[kept] = pline | ((uint64_t)pst << VB_STORE) | ((uint64_t)(pw - 1) << VB_W);
            if (wbk) wbk[kept] = pscope;
          }
          kept++;
          pv = false;
        }
        if (rlim) r_mem = false;
      }
      if (RD && rd_any) {
        const uint32_t lim = rlim;  // records of this chunk in the batch
        const bool valid = lane < lim;
        const bool mem = valid && (m & 3u) < 2u;
        const bool st = mem && (m & 3u) == 1u;
        const uint64_t line = a >> A.lbs_rd;
        const uint32_t scope = A.cta_scope ? c : 0u;
        const bool q_mem = (pm & 3u) < 2u;
        const bool q_st = (pm & 3u) == 1u;
        const uint64_t q_line = pa >> A.lbs_rd;
        const uint32_t q_scope = A.cta_scope ? pc : 0u;
        const bool same = mem && q_mem && scope == q_scope && line == q_line;
        const bool dup = same && !st;
        const bool elig = same && st && q_st && !(g == 0 && lane == 0);
        const uint32_t Mnon = __ballot_sync(FULL, st && !elig);
        const uint32_t below = Mnon & lanemask_le();
        const uint32_t cs = below ? g + (31u - __clz(below)) : cstart;
        const bool merged = elig && ((g + lane - cs) & 15u) != 0;
        const bool keep = mem && !dup && !merged;
        const uint32_t Mmerged = __ballot_sync(FULL, merged);
        const uint32_t Mdup = __ballot_sync(FULL, dup);
        if (Mnon) cstart = g + (31u - __clz(Mnon));
        if (pv) {
          // the record carried from the previous batch ends before the first non-merged lane
          const uint32_t e = __ffs(~Mmerged) - 1;
          const uint32_t wgt = pw + (pst ? e : 0u);
          const bool hd = e < lim && ((Mdup >> e) & 1u);
          if (lane == 0) {
            wbv[kept] = pline | ((uint64_t)pst << VB_STORE) | ((uint64_t)hd << VB_DUP) | ((uint64_t)(wgt - 1) << VB_W);
            if (wbk) wbk[kept] = pscope;
          }
          kept++;
          pv = false;
        }
        const uint32_t after = ~Mmerged & ~lanemask_le();
        const uint32_t e_l = st ? (after ? (uint32_t)(__ffs(after) - 1) : 32u) : lane + 1;
        const bool fin = keep && e_l < lim;
        const uint32_t Mfin = __ballot_sync(FULL, fin);
        if (fin) {
          const uint32_t pos = kept + __popc(Mfin & lanemask_lt());
          const bool hd = (Mdup >> e_l) & 1u;
          wbv[pos] = line | ((uint64_t)st << VB_STORE) | ((uint64_t)hd << VB_DUP) | ((uint64_t)(e_l - lane - 1) << VB_W);
          if (wbk) wbk[pos] = scope;
        }
        kept += __popc(Mfin);
        const uint32_t Mp = __ballot_sync(FULL, keep && e_l >= lim);
        if (Mp) {
          const uint32_t pl_ = __ffs(Mp) - 1;
          pv = true;
          pline = __shfl_sync(FULL, line, pl_);
          pscope = __shfl_sync(FULL, scope, pl_);
          pst = __shfl_sync(FULL, (uint32_t)st, pl_) != 0;
          pw = pst ? lim - pl_ : 1u;
        }
        ndup += __popc(Mdup);
        if (lim) {
          r_mem = __shfl_sync(FULL, (uint32_t)mem, lim - 1) != 0;
          r_line = __shfl_sync(FULL, line, lim - 1);
          r_scope = __shfl_sync(FULL, scope, lim - 1);
        }
      }
      // ---- carry the last consumed record, advance, recycle fully consumed pieces
      const uint32_t last = adv - 1;
      p_cta = __shfl_sync(FULL, c, last);
      p_tm = __shfl_sync(FULL, (m << 16) | t, last);
      p_rk = __shfl_sync(FULL, rk, last);
      p_winst = __shfl_sync(FULL, w, last);
      p_addr = __shfl_sync(FULL, a, last);
      g += adv;
      while (issued < npieces && g >= (issued - KS + 1) * KR) {
        __syncwarp();
        if (lane == 0) {
          fence_proxy_async();
          io.issue(issued);
        }
        ++issued;
      }
    }
    // ---- drain the pieces still in flight (their barriers must complete before exit)
    while (waited < issued) {
      mbar_wait(&bar[waited % KS], (waited / KS) & 1u);
      ++waited;
    }
    if (RD && pv) {
      // the record after the chunk decides has_dup (it is never merged into us)
      bool hd = false;
      if (c_hi < A.n) {
        const uint8_t m2 = __ldg(A.meta + c_hi);
        if (is_mem(m2) && !is_store(m2) && meta_ok(m2) && r_mem) {
          const uint64_t a2 = __ldg(A.addr + c_hi);
          const uint32_t s2 = A.cta_scope ? __ldg(A.cta + c_hi) : 0u;
          hd = addr_ok(a2, m2) && (a2 >> A.lbs_rd) == r_line && s2 == r_scope;
        }
      }
      if (lane == 0) {
        wbv[kept] = pline | ((uint64_t)pst << VB_STORE) | ((uint64_t)hd << VB_DUP) | ((uint64_t)(pw - 1) << VB_W);
        if (wbk) wbk[kept] = pscope;
      }
      kept++;
    }
  }
  if (RD && lane == 0) {
    A.wcnt[gw] = kept;
    if (ndup) atomicAdd((unsigned long long*)A.hist0, (unsigned long long)ndup);
  }
  if (BD && lane == 0) {
    if (bd_exec) atomicAdd(&s_bd_tot[0], bd_exec);
    if (bd_threads) atomicAdd(&s_bd_tot[2], bd_threads);
  }
  if (MD) {
    __syncwarp();
    for (uint32_t k = lane; k < 66; k += 32)
      if (whist[k]) atomicAdd(&s_md_hist[k], whist[k]);
  }
  // ---- flush block-level counters
  __syncthreads();
  if (MD) {
    const uint32_t W = 1u << A.ws_md;
    for (uint32_t k = tx; k < 2 * 33; k += NTHR) {
      const uint32_t kind = k / 33, deg = k % 33;
      if (s_md_hist[k] && deg <= W)
        atomicAdd((unsigned long long*)&A.md_hist[kind * (W + 1) + deg], (unsigned long long)s_md_hist[k]);
    }
    if (C.md_sites)
      for (uint32_t k = tx; k < 2 * A.nsites; k += NTHR)
        if (C.md_sites[k]) atomicAdd((unsigned long long*)&A.md_sites[k], (unsigned long long)C.md_sites[k]);
  }
  if (BD) {
    if (tx < 3 && s_bd_tot[tx]) atomicAdd((unsigned long long*)&A.bd_tot[tx], (unsigned long long)s_bd_tot[tx]);
    if (C.bd_sites)
      for (uint32_t k = tx; k < 3 * A.nsites; k += NTHR)
        if (C.bd_sites[k]) atomicAdd((unsigned long long*)&A.bd_sites[k], (unsigned long long)C.bd_sites[k]);
  }
}

// Deferred BD groups: divergent iff active < clamp(T_c - w*W, 0, W).
__global__ void __launch_bounds__(256) k_bd_resolve(const uint4* __restrict__ defer, uint64_t m,
                                                    const uint32_t* __restrict__ tc, uint32_t ws,
                                                    uint64_t* bd_tot, uint64_t* bd_sites, uint32_t nsites) {
  __shared__ uint32_t s_div[NSITE_SMEM];
  const bool sm = nsites && nsites <= NSITE_SMEM;
  if (sm)
    for (uint32_t k = threadIdx.x; k < nsites; k += blockDim.x) s_div[k] = 0;
  __syncthreads();
  uint32_t tot = 0;
  const uint32_t W = 1u << ws;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint4 d = defer[i];
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

// Packs every warp's kept records from its gapped region to their final
// (exclusive-scan) offsets: one CTA per warp chunk.
__global__ void __launch_bounds__(256) k_squeeze(const uint32_t* __restrict__ kin, const uint64_t* __restrict__ vin,
                                                 uint32_t* __restrict__ kout, uint64_t* __restrict__ vout,
                                                 const uint64_t* __restrict__ cnt, const uint64_t* __restrict__ off,
                                                 uint64_t chunk) {
  const uint64_t b = blockIdx.x, m = cnt[b], o = off[b];
  const uint64_t src = b * chunk;
  for (uint64_t k = threadIdx.x; k < m; k += blockDim.x) {
    vout[o + k] = vin[src + k];
    if (kin) kout[o + k] = kin[src + k];
  }
}

template <int F>
size_t scan_smem() {
  constexpr bool MD = (F & F_MD) != 0, BD = (F & F_BD) != 0;
  return (size_t)NWARP * R_BYTES + (size_t)((MD ? 2 : 0) + (BD ? 3 : 0)) * NSITE_SMEM * 4 + (size_t)NWARP * 68 * 4;
}

int g_scan_ready[8] = {0, 0, 0, 0, 0, 0, 0, 0};
const char* const kScanName[8] = {"k_scan<0>", "k_scan<1>", "k_scan<2>", "k_scan<3>",
                                  "k_scan<4>", "k_scan<5>", "k_scan<6>", "k_scan<7>"};

template <int F>
cudaError_t launch_scan_t(cadv_ctx* c, const ScanArgs& A, uint64_t grid) {
  const size_t smem = scan_smem<F>();
  if (!g_scan_ready[F]) {
    cudaError_t e = cudaFuncSetAttribute(k_scan<F>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    g_scan_ready[F] = 1;
  }
  CADV_LAUNCH_N(c, kScanName[F], k_scan<F><<<(unsigned)grid, NTHR, smem, c->stream>>>(A));
  return cudaGetLastError();
}

}  // namespace

// One CTA per SM; every warp a contiguous chunk whose length is a multiple of KR.
void scan_geometry(cadv_ctx* c, uint64_t n, uint64_t* grid, uint64_t* nwarps, uint64_t* chunk) {
  uint64_t g = (uint64_t)c->num_sms;
  const uint64_t tw = g * NWARP;
  uint64_t ch = (n + tw - 1) / tw;
  ch = ((ch + KR - 1) / KR) * KR;
  if (ch == 0) ch = KR;
  *chunk = ch;
  const uint64_t need = (n + ch - 1) / ch;  // warps with records
  g = (need + NWARP - 1) / NWARP;
  if (g == 0) g = 1;
  *grid = g;
  *nwarps = g * NWARP;
}

cudaError_t launch_squeeze(cadv_ctx* c, const uint32_t* kin, const uint64_t* vin, uint32_t* kout, uint64_t* vout,
                           const uint64_t* cnt, const uint64_t* off, uint64_t nchunks, uint64_t chunk) {
  if (nchunks == 0) return cudaSuccess;
  CADV_LAUNCH(c, k_squeeze<<<(unsigned)nchunks, 256, 0, c->stream>>>(kin, vin, kout, vout, cnt, off, chunk));
  return cudaGetLastError();
}

cudaError_t launch_scan(cadv_ctx* c, int flags, const ScanParams& P) {
  const cadv_trace_desc& t = P.t;
  if (t.n == 0) return cudaSuccess;
  ScanArgs A{};
  A.addr = t.addr; A.cta = t.cta; A.tid = t.tid; A.site = t.site; A.winst = t.winst; A.meta = t.meta;
  A.n = t.n;
  uint64_t grid, nwarps;
  scan_geometry(c, t.n, &grid, &nwarps, &A.chunk);
  A.lbs_rd = P.lbs_rd; A.cta_scope = P.cta_scope; A.kout = P.kout; A.vout = P.vout; A.wcnt = P.blkcnt;
  A.hist0 = P.hist0;
  A.lbs_md = P.lbs_md; A.ws_md = P.ws_md; A.md_hist = P.md_hist; A.md_sites = P.md_sites;
  A.ws_bd = P.ws_bd; A.tc = P.tc; A.bd_tot = P.bd_tot; A.bd_sites = P.bd_sites; A.defer = (uint4*)P.defer;
  A.ndefer = P.ndefer;
  A.nsites = P.nsites; A.site_flag = P.site_flag; A.sc = scalars(c);
  switch (flags) {
    case 1: return launch_scan_t<1>(c, A, grid);
    case 2: return launch_scan_t<2>(c, A, grid);
    case 3: return launch_scan_t<3>(c, A, grid);
    case 4: return launch_scan_t<4>(c, A, grid);
    case 5: return launch_scan_t<5>(c, A, grid);
    case 6: return launch_scan_t<6>(c, A, grid);
    case 7: return launch_scan_t<7>(c, A, grid);
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t launch_bd_resolve(cadv_ctx* c, const void* defer, uint64_t m, const uint32_t* tc, uint32_t ws,
                              uint64_t* bd_tot, uint64_t* bd_sites, uint32_t nsites) {
  if (m == 0) return cudaSuccess;
  const uint64_t want = (m + 255) / 256;
  const int grid = (int)(want < (uint64_t)c->num_sms * 4 ? want : (uint64_t)c->num_sms * 4);
  CADV_LAUNCH(c, k_bd_resolve<<<grid, 256, 0, c->stream>>>((const uint4*)defer, m, tc, ws, bd_tot, bd_sites, nsites));
  return cudaGetLastError();
}

}  // namespace cadv
