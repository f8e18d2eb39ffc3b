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
// Data movement (B200): one persistent CTA per SM, 16 independent warps
// (128 registers).  Every warp owns a contiguous chunk of the trace and
// streams it through a private stage-major ring of 2 x 256-record pieces in
// shared memory, filled by 1-D TMA bulk copies (cp.async.bulk, one elected
// lane, one mbarrier per stage).  There is no block-level barrier in the
// loop.  A step = one piece: every lane takes 8 consecutive records, builds
// 8-bit masks from the comparisons with each record's predecessor (RD line /
// scope equality, run starts, MD line changes and decreases), and the warp
// combines lanes with ballots, shuffles and one segmented suffix scan:
//   R1   duplicate loads are counted and dropped, store chains merged; the
//        kept records are written to the warp's region of the kept buffer;
//   M/B  runs (records of one (cta, warp32, winst, family)) complete in the
//        step are queued in shared memory and finalized 32 at a time
//        (flush_runs); the run open at the step end is carried.  Runs whose
//        lines decrease (MD), analysis warp sizes below 32 and malformed
//        runs take an exact pairwise walk over global memory.
// Runs are owned by the chunk that contains their first record; reuse-
// distance run compression consumes exactly the chunk's records.
#include <cuda_runtime.h>

#include "cadv_impl.h"
#include "common.cuh"

namespace cadv {
namespace {

constexpr int LPR = 8;                 // consecutive records per lane in one warp step
constexpr int KR = 32 * LPR;           // records per piece = one warp step
constexpr int KS = 2;                  // ring stages per warp (piece p and piece p + 1 in flight)
constexpr int NWARP = 16;              // warps per CTA (one CTA per SM; 4 per SM sub-partition)
constexpr int NTHR = NWARP * 32;
constexpr int NSITE_SMEM = 512;        // per-site counters kept in shared memory up to this many sites
// per-warp queue of complete runs awaiting finalization: a round of enqueues
// (<= 32) starts with at most QCAP - 32 entries queued
template <int F>
constexpr int qcap() { return (F & F_OBJ) ? 40 : 64; }
constexpr int OBJ_SMEM = 64;           // F_OBJ: object rows (objects + 1) kept in shared memory up to this many

// per-warp ring, stage-major: stage s occupies [s * STG_BYTES, (s + 1) * STG_BYTES)
// and holds the KR records of one piece column by column (every column region
// a multiple of 128 B), so one stage base + constant offsets address a piece
constexpr uint32_t S_ADDR = 0;
constexpr uint32_t S_CTA = S_ADDR + KR * 8;
constexpr uint32_t S_TID = S_CTA + KR * 4;
constexpr uint32_t S_WINST = S_TID + KR * 2;
constexpr uint32_t S_SITE = S_WINST + KR * 4;
constexpr uint32_t S_META = S_SITE + KR * 4;
constexpr uint32_t STG_BYTES = S_META + KR;
constexpr uint32_t R_BYTES = KS * STG_BYTES;

// piece number g of the warp (counted over all its chunks) -> its ring stage
__device__ __forceinline__ uint32_t stage_of(uint32_t g) { return (g % KS) * STG_BYTES; }

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
  uint64_t chunk;        // records per chunk (multiple of KR); warps claim chunks dynamically
  uint64_t nchunks;
  uint64_t nbig;         // chunks [0, nbig) have `chunk` records, the rest chunk_s (the tail: less imbalance)
  uint64_t chunk_s;
  // RD
  uint32_t lbs_rd;
  int cta_scope;
  uint32_t* kout;        // gapped output: warp w writes from w * chunk
  uint64_t* vout;
  uint64_t* wcnt;        // kept records per warp
  uint64_t kcap;         // kept-record region capacity per warp (writes beyond it are dropped; the host reruns)
  uint64_t* hist0;
  // MD
  uint32_t lbs_md, ws_md;
  uint64_t* md_hist;     // [2][W+1]
  uint64_t* md_sites;    // [nsites][2] or null
  // BD
  uint32_t ws_bd;
  uint32_t* tc;          // T_c per CTA id (RED.MAX of gen << 11 | T_c)
  uint32_t tc_cap, tc_gen;
  uint64_t defer_cap;
  uint64_t* bd_tot;      // [3] exec, divergent, threads
  uint64_t* bd_sites;    // [nsites][3] or null
  uint4* defer;          // deferred partial groups
  unsigned long long* ndefer;
  uint32_t nsites;
  uint64_t* site_flag;
  Scalars* sc;
  // F_OBJ: line extents of the data objects; hist0 / md_hist hold one row per object + 1
  const uint64_t* obj_lo;
  const uint64_t* obj_hi;
  uint32_t nobj, rd_nbins;
  uint32_t one;          // = 1 (opaque to the compiler: see add_if)
};

__device__ __forceinline__ void report(Scalars* sc, uint64_t i, uint32_t code) {
  atomicMin(&sc->err_index, (unsigned long long)i);
  atomicMax(&sc->err_code, code);
}

__device__ __forceinline__ void red_max(uint32_t* p, uint32_t v) {
  asm volatile("red.relaxed.gpu.global.max.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// bit 0 of each byte of v -> bits 0..3
__device__ __forceinline__ uint32_t gather4(uint32_t v) { return ((v & 0x01010101u) * 0x10204080u) >> 28; }
// bit 0 of each of the 8 bytes (x: bytes 0-3, y: bytes 4-7) -> bits 0..7
__device__ __forceinline__ uint32_t gather8(uint32_t x, uint32_t y) { return gather4(x) | (gather4(y) << 4); }

// bits [a, e) of a lane mask, 0 <= a < e <= 32
__device__ __forceinline__ uint32_t bits_from(uint32_t a, uint32_t e) {
  const uint32_t hi = e >= 32 ? FULL : ((1u << e) - 1u);
  return hi & ~((1u << a) - 1u);
}

// T_c candidate of one BB group (RED.MAX, tagged with the call's generation);
// a CTA id beyond the table's capacity makes the host grow it and rerun.
__device__ __forceinline__ void tc_update(const ScanArgs& A, uint32_t cta, uint32_t maxtid) {
  if (cta < A.tc_cap) {
    red_max(A.tc + cta, (A.tc_gen << 11) | (maxtid + 1u));
  } else {
    A.sc->tc_overflow = 1;
    atomicMax(&A.sc->max_cta, (unsigned long long)cta);
  }
}

struct Counters {        // block-level shared-memory accumulators
  uint32_t* md_hist;     // [2][33]
  uint32_t* md_sites;    // [NSITE_SMEM][2] or null
  uint32_t* bd_tot;      // [3]
  uint32_t* bd_sites;    // [NSITE_SMEM][3] or null
  // F_OBJ with at most OBJ_SMEM rows (else null: global tables and atomics)
  const uint64_t* olo;   // [OBJ_SMEM] object line extents
  const uint64_t* ohi;
  uint32_t* mdo;         // [rows][2][33] MD histogram per object row
  uint32_t* dup;         // [rows] dropped duplicate loads (RD 0) per object row
  uint32_t* wh_all;      // per-warp MD histograms [NWARP][68], then the run queues
  bool sites_smem;       // per-site counters in shared memory (nsites <= NSITE_SMEM)
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

// Per-warp TMA issue of piece p (records [c_lo + p KR, ...) of the warp's
// stream) into ring stage p % KS: one 1-D bulk copy per column, completion
// counted on the stage's mbarrier.  Called by the whole (converged) warp with
// warp-uniform operands: one elected lane (elect.sync inside the asm, so
// ptxas needs no per-lane loop to move the operands to uniform registers)
// issues the expect-tx and every copy of a full piece from ONE asm block
// (one election, destinations = stage base + constant column offsets).
#define CADV_CP(DOFF, SRC, BYTES) \
  "@p cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0+" #DOFF "], [" SRC "], " #BYTES ", [%1];\n"
template <int F>
__device__ __forceinline__ void issue_full(const ScanArgs& A, uint32_t dst, uint32_t bar, uint32_t q0) {
  // (q0 < n < 2^32: 32-bit element offsets, so the addresses are IMAD.WIDEs on the FMA pipe)
  constexpr bool NA = (F & (F_RD | F_MD)) != 0, NG = (F & (F_MD | F_BD)) != 0;
  static_assert(KR == 256 && S_CTA == 2048 && S_TID == 3072 && S_WINST == 3584 && S_SITE == 4608 && S_META == 5632,
                "column offsets / byte counts below are for 256-record pieces");
  if (NA && NG) {
    asm volatile(
        "{\n.reg .pred p;\nelect.sync _|p, 0xffffffff;\n"
        "@p mbarrier.arrive.expect_tx.shared::cta.b64 _, [%1], 5888;\n"
        CADV_CP(0, "%2", 2048) CADV_CP(2048, "%3", 1024) CADV_CP(3072, "%4", 512) CADV_CP(3584, "%5", 1024)
        CADV_CP(4608, "%6", 1024) CADV_CP(5632, "%7", 256) "}" ::"r"(dst), "r"(bar),
        "l"(A.addr + q0),
        "l"(A.cta + q0), "l"(A.tid + q0), "l"(A.winst + q0), "l"(A.site + q0), "l"(A.meta + q0)
        : "memory");
  } else if (NA) {
    asm volatile(
        "{\n.reg .pred p;\nelect.sync _|p, 0xffffffff;\n"
        "@p mbarrier.arrive.expect_tx.shared::cta.b64 _, [%1], 3328;\n"
        CADV_CP(0, "%2", 2048) CADV_CP(2048, "%3", 1024) CADV_CP(5632, "%4", 256) "}" ::"r"(dst), "r"(bar),
        "l"(A.addr + q0), "l"(A.cta + q0), "l"(A.meta + q0)
        : "memory");
  } else {
    asm volatile(
        "{\n.reg .pred p;\nelect.sync _|p, 0xffffffff;\n"
        "@p mbarrier.arrive.expect_tx.shared::cta.b64 _, [%1], 3840;\n"
        CADV_CP(2048, "%2", 1024) CADV_CP(3072, "%3", 512) CADV_CP(3584, "%4", 1024) CADV_CP(4608, "%5", 1024)
        CADV_CP(5632, "%6", 256) "}" ::"r"(dst), "r"(bar), "l"(A.cta + q0), "l"(A.tid + q0), "l"(A.winst + q0),
        "l"(A.site + q0), "l"(A.meta + q0)
        : "memory");
  }
}
#undef CADV_CP
template <int F>
__device__ __forceinline__ void bulk_cp(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile(
      "{\n.reg .pred p;\nelect.sync _|p, 0xffffffff;\n"
      "@p cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n}" ::"r"(dst),
      "l"(src), "r"(bytes), "r"(bar)
      : "memory");
}
// the partial last piece of a stream: sizes rounded up to 16 bytes (sources stay in the padded columns)
template <int F>
__device__ __noinline__ void issue_partial(const ScanArgs& A, uint32_t dst, uint32_t bar, uint64_t q0, uint32_t cnt) {
  constexpr bool NA = (F & (F_RD | F_MD)) != 0, NG = (F & (F_MD | F_BD)) != 0;
  auto r16 = [](uint32_t b_) { return (b_ + 15u) & ~15u; };
  uint32_t bytes = r16(cnt * 4) + r16(cnt);
  if (NA) bytes += r16(cnt * 8);
  if (NG) bytes += r16(cnt * 2) + 2 * r16(cnt * 4);
  asm volatile(
      "{\n.reg .pred p;\nelect.sync _|p, 0xffffffff;\n@p mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n}" ::"r"(bar),
      "r"(bytes)
      : "memory");
  if (NA) bulk_cp<F>(dst + S_ADDR, A.addr + q0, r16(cnt * 8), bar);
  bulk_cp<F>(dst + S_CTA, A.cta + q0, r16(cnt * 4), bar);
  if (NG) {
    bulk_cp<F>(dst + S_TID, A.tid + q0, r16(cnt * 2), bar);
    bulk_cp<F>(dst + S_WINST, A.winst + q0, r16(cnt * 4), bar);
    bulk_cp<F>(dst + S_SITE, A.site + q0, r16(cnt * 4), bar);
  }
  bulk_cp<F>(dst + S_META, A.meta + q0, r16(cnt), bar);
}
template <int F>
__device__ __forceinline__ void issue_piece(const ScanArgs& A, uint32_t ring, uint32_t bar0, uint64_t c_lo,
                                            uint64_t s_end, uint32_t p, uint32_t g) {
  // piece p of the chunk = the warp's piece g (ring stage and mbarrier by g)
  const uint32_t stg = g % KS, bar = bar0 + stg * 8, dst = ring + stg * STG_BYTES;
  const uint32_t q0 = (uint32_t)c_lo + p * KR;  // < n < 2^32 (cadv_load_trace)
  if ((uint64_t)q0 + KR <= s_end) issue_full<F>(A, dst, bar, q0);
  else issue_partial<F>(A, dst, bar, q0, (uint32_t)(s_end - q0));
}

// shared-memory re-reads of ring values (asm: not folded into the registers
// that held them, which are dead by then)
__device__ __forceinline__ uint64_t lds_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.shared.u64 %0, [%1];" : "=l"(v) : "r"(smem_u32(p)));
  return v;
}
__device__ __forceinline__ uint32_t lds_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(smem_u32(p)));
  return v;
}

// row of a line among the data objects (F_OBJ): binary search of the extents,
// with explicit shared-memory loads when the table is in shared memory (a
// generic load would wait on the long scoreboard)
__device__ __forceinline__ uint32_t row_of(const ScanArgs& A, const Counters& C, uint64_t line) {
  if (!C.olo) return obj_row(A.obj_lo, A.obj_hi, A.nobj, line);
  uint32_t a = 0, b = A.nobj;  // a = number of extents starting at or before the line
  while (a < b) {
    const uint32_t m = (a + b) >> 1;
    if (lds_u64(C.olo + m) <= line) a = m + 1;
    else b = m;
  }
  return (a && line < lds_u64(C.ohi + a - 1)) ? a - 1 : A.nobj;
}

// Mask building off the integer ALU pipe (the scan's bottleneck): m += bit
// when the condition holds, as a predicated IMAD by an opaque 1 (FMA pipe)
// instead of SEL + IADD3 on the ALU pipe.
__device__ __forceinline__ void add_if_nz(uint32_t& m, uint32_t x, uint32_t one, uint32_t bit) {
  asm("{\n.reg .pred q;\nsetp.ne.u32 q, %1, 0;\n@q mad.lo.u32 %0, %2, %3, %0;\n}" : "+r"(m) : "r"(x), "r"(one), "r"(bit));
}
__device__ __forceinline__ void add_if_lt(uint32_t& m, uint64_t a, uint64_t b, uint32_t one, uint32_t bit) {
  asm("{\n.reg .pred q;\nsetp.lt.u64 q, %1, %2;\n@q mad.lo.u32 %0, %3, %4, %0;\n}" : "+r"(m) : "l"(a), "l"(b), "r"(one), "r"(bit));
}

// run identity: (cta, warp32, winst, family)
__device__ __forceinline__ uint32_t run_hi(uint32_t tid, uint32_t meta) {
  return (tid >> 5) | (((meta & 3u) == 2u) ? 64u : 0u);
}

// ------------------------------------------------------------------ group finishing
// row (F_OBJ): the object row of the group's first record
template <int F>
__device__ __forceinline__ void finish_md(const ScanArgs& A, const Counters& C, uint32_t* whist, bool sites_smem,
                                          uint32_t kind, uint32_t deg, uint32_t s, uint32_t row) {
  if (F & F_OBJ) {
    if (C.mdo) atomicAdd(&C.mdo[row * 66 + kind * 33 + deg], 1u);
    else atomicAdd((unsigned long long*)&A.md_hist[(row * 2 + kind) * ((1u << A.ws_md) + 1) + deg], 1ull);
  } else {
    atomicAdd(&whist[kind * 33 + deg], 1u);
  }
  if (sites_smem) {
    if (s < A.nsites) { atomicAdd(&C.md_sites[2 * s], 1u); atomicAdd(&C.md_sites[2 * s + 1], deg); }
    else *A.site_flag = 1;
  } else if (A.nsites) {
    site_add(A, nullptr, A.md_sites, 2, s, 1, deg);
  }
}

// BD per-site counters of one complete group (exec, threads)
__device__ __forceinline__ void bd_sites_add(const ScanArgs& A, const Counters& C, bool sites_smem, uint32_t s,
                                             uint32_t cnt) {
  if (sites_smem) {
    if (s < A.nsites) { atomicAdd(&C.bd_sites[3 * s], 1u); atomicAdd(&C.bd_sites[3 * s + 2], cnt); }
    else *A.site_flag = 1;
  } else if (A.nsites) {
    site_add(A, nullptr, A.bd_sites, 3, s, 1, cnt);
  }
}

// Warp-cooperative exact resolution of ONE run [g0, g0 + nrec), nrec <= 32,
// re-read from global memory (recently streamed: L2) one record per lane:
// the run's sub-warp groups (tid % 32 >> ws, analysis warp size 2^ws) with
// their distinct lines (MD: __match_any_sync on the line within the group,
// first lane of each line counted) or their lane sets (BD).  Used for runs
// whose lines are not non-decreasing (MD: the fast path counts line changes)
// and for analysis warp sizes below 32; the whole warp calls it with
// warp-uniform arguments.  The run's records share kind, CTA and site (the
// scan checks R19).  exec / thr / mxc: the caller's BD accumulators.
// The run's records come from global memory (SMEM = false: g0 = trace
// position; queued runs whose stage was recycled) or from the warp's ring
// stage (SMEM = true: ta / aa point at the run's first record there).
template <int F, bool SMEM>
__device__ __forceinline__ void walk_warp(const ScanArgs& A, const Counters& C, uint32_t* whist, bool sites_smem,
                                          uint64_t g0, const uint16_t* ta, const uint64_t* aa, uint32_t nrec,
                                          uint32_t kind, uint32_t cta, uint32_t s, uint32_t& exec, uint32_t& thr,
                                          uint32_t& mxc) {
  const uint32_t lane = lane_id();
  const bool bb = kind == 2u;
  const uint32_t ws = bb ? A.ws_bd : A.ws_md;
  const bool v = lane < nrec;
  const uint32_t vm = nrec >= 32u ? FULL : ((1u << nrec) - 1u);
  const uint32_t t = v ? (SMEM ? (uint32_t)ta[lane] : (uint32_t)__ldg(A.tid + g0 + lane)) : 0u;
  const uint32_t lb = t & 31u;
  // lane set of the run; a repeated lane makes the popcount fall short
  const uint32_t M = __reduce_or_sync(FULL, v ? 1u << lb : 0u);
  if ((uint32_t)__popc(M) != nrec) {
    if (lane == 0) report(A.sc, g0, 2);
    return;
  }
  const uint32_t sub = v ? (lb >> ws) : 32u;                 // the record's sub-warp group
  const uint32_t ps = __match_any_sync(FULL, sub) & vm;     // lanes of the same group
  const bool lead = v && (ps & lanemask_lt()) == 0u;        // the group's first record
  const uint32_t c = __popc(ps);
  if (bb) {
    const uint32_t W = 1u << ws;
    const uint32_t gm = M & ((W == 32u ? FULL : ((1u << W) - 1u)) << ((lb >> ws) << ws));  // the group's lanes
    if (lead) {
      exec += 1;
      thr += c;
      mxc = max(mxc, cta);
      tc_update(A, cta, (t & ~31u) | (31u - __clz(gm)));
      bd_sites_add(A, C, sites_smem, s, c);
    }
    // groups with fewer than W lanes wait for T_c (warp-aggregated append)
    const bool need = lead && c < W;
    const uint32_t dm = __ballot_sync(FULL, need);
    if (dm) {
      const uint32_t leader = __ffs(dm) - 1;
      unsigned long long b = 0;
      if (lane == leader) b = atomicAdd(A.ndefer, (unsigned long long)__popc(dm));
      b = __shfl_sync(FULL, b, leader);
      const unsigned long long slot = b + __popc(dm & lanemask_lt());
      if (need && slot < A.defer_cap)
        A.defer[slot] = make_uint4(cta, t >> ws, c, (A.nsites && s < A.nsites) ? s : 0xffffffffu);
    }
  } else {
    const uint64_t line = v ? ((SMEM ? aa[lane] : __ldg(A.addr + g0 + lane)) >> A.lbs_md) : 0ull;
    const uint32_t pl = __match_any_sync(FULL, line) & ps;  // same group, same line
    const bool first = v && (pl & lanemask_lt()) == 0u;
    const uint32_t deg = __popc(__ballot_sync(FULL, first) & ps);
    if (lead) finish_md<F>(A, C, whist, sites_smem, kind, deg, s, (F & F_OBJ) ? row_of(A, C, line) : 0u);
  }
}

// run aggregates packed for the segmented scans: deg | cnt << 10 | viol << 20
constexpr uint32_t PK_CNT = 10, PK_VIOL = 20, PK_M = 1023;

// Finalizes the queued complete runs (one per lane, the warp converged).  A
// run is one warp32 instruction of one CTA: with W = 32 it is the group, and
// when its lines never decrease (viol = 0) deg = the number of line changes.
// Entries are self-contained (run start j, aggregate u, lane bits m, kind |
// tid, CTA and site of the first record, copied from the ring when queued),
// so flushes are batched across steps.
template <int F>
struct RunQueue {  // six columns of QCAP words from one base (one live register)
  uint32_t* b;
  static constexpr uint32_t C = qcap<F>();
  __device__ __forceinline__ uint32_t& j(uint32_t i) const { return b[i]; }
  __device__ __forceinline__ uint32_t& u(uint32_t i) const { return b[C + i]; }
  __device__ __forceinline__ uint32_t& m(uint32_t i) const { return b[2 * C + i]; }
  __device__ __forceinline__ uint32_t& kt(uint32_t i) const { return b[3 * C + i]; }
  __device__ __forceinline__ uint32_t& cta(uint32_t i) const { return b[4 * C + i]; }
  __device__ __forceinline__ uint32_t& site(uint32_t i) const { return b[5 * C + i]; }
  __device__ __forceinline__ uint32_t* carry() const { return b + 6 * C; }  // the carried run's first record
};

template <int F>
__device__ __noinline__ void flush_runs(const ScanArgs& A, const Counters* Cp, uint32_t qn, uint64_t c_lo,
                                        const uint8_t* stg, uint32_t sbase) {
  // (the block's counter table lives in shared memory: the streaming loop
  // keeps no register for it across the call)
  constexpr bool MD = (F & F_MD) != 0, BD = (F & F_BD) != 0;
  const Counters C = *Cp;
  const bool sites_smem = C.sites_smem;
  const uint32_t lane = lane_id(), warp = threadIdx.x >> 5;
  uint32_t* const whist = C.wh_all + warp * 68;
  const RunQueue<F> Q{C.wh_all + NWARP * 68 + warp * (RunQueue<F>::C * 6 + 4)};
  uint32_t exec = 0, thr = 0, mxc = 0;
  for (uint32_t q0 = 0; q0 < qn; q0 += 32) {
    const uint32_t q = q0 + lane;
    bool md = false, bd = false, slow = false;
    uint32_t j = 0, u = 0, m = 0, t = 0, kind = 0, cta = 0, s = 0, cnt = 0;
    if (q < qn) {
      j = Q.j(q);
      u = Q.u(q);
      m = Q.m(q);
      const uint32_t kt = Q.kt(q);
      kind = kt >> 16;
      t = kt & 0xffffu;
      cta = Q.cta(q);
      s = Q.site(q);
      const bool bb = kind == 2u;
      cnt = (u >> PK_CNT) & PK_M;
      if (bb ? BD : MD) {
        if (cnt > 32) report(A.sc, c_lo + j, 2);  // a lane must repeat
        else if (bb ? A.ws_bd != 5u : ((u >> PK_VIOL) || A.ws_md != 5u)) slow = true;  // (BB: no address test)
        else if ((uint32_t)__popc(m) != cnt) report(A.sc, c_lo + j, 2);
        else if (bb) bd = true;
        else md = true;
      }
    }
    // F_OBJ: the group's object from its first record's address (global; recently streamed, L2).
    // (Computing the row when the run is queued, from the ring, was measured slower:
    // k_scan<11> 3.95 -> 4.27 ms - the streaming loop carries the search.)
    if (MD && md)
      finish_md<F>(A, C, whist, sites_smem, kind, u & PK_M, s,
                   (F & F_OBJ) ? row_of(A, C, __ldg(A.addr + c_lo + j) >> A.lbs_md) : 0u);
    if (BD) {
      if (bd) {
        exec += 1;
        thr += cnt;
        mxc = max(mxc, cta);
        tc_update(A, cta, (t & ~31u) | (31u - __clz(m)));
        bd_sites_add(A, C, sites_smem, s, cnt);
      }
      // groups with fewer than 32 active lanes wait for T_c (warp-aggregated append)
      const bool need = bd && cnt < 32u;
      const uint32_t dm = __ballot_sync(FULL, need);
      if (dm) {
        const uint32_t leader = __ffs(dm) - 1;
        unsigned long long b = 0;
        if (lane == leader) b = atomicAdd(A.ndefer, (unsigned long long)__popc(dm));
        b = __shfl_sync(FULL, b, leader);
        const unsigned long long slot = b + __popc(dm & lanemask_lt());
        if (need && slot < A.defer_cap)
          A.defer[slot] = make_uint4(cta, t >> 5, cnt, (A.nsites && s < A.nsites) ? s : 0xffffffffu);
      }
    }
    // runs that need the exact walk: the whole warp takes them one by one,
    // from the ring when the run lies in the current step's stage (records
    // [sbase, sbase + KR) of the chunk: usually every queued run of an
    // irregular trace, whose queue fills each step), else from global memory
    for (uint32_t sm = __ballot_sync(FULL, slow); sm; sm &= sm - 1) {
      const uint32_t src = __ffs(sm) - 1;
      const uint32_t rj = __shfl_sync(FULL, j, src), rn = __shfl_sync(FULL, cnt, src);
      const uint32_t rk = __shfl_sync(FULL, kind, src), rc = __shfl_sync(FULL, cta, src);
      const uint32_t rs = __shfl_sync(FULL, s, src);
      if (rj >= sbase && rj + rn <= sbase + KR)
        walk_warp<F, true>(A, C, whist, sites_smem, 0, (const uint16_t*)(stg + S_TID) + (rj - sbase),
                           (const uint64_t*)(stg + S_ADDR) + (rj - sbase), rn, rk, rc, rs, exec, thr, mxc);
      else
        walk_warp<F, false>(A, C, whist, sites_smem, c_lo + rj, nullptr, nullptr, rn, rk, rc, rs, exec, thr, mxc);
    }
  }
  if (BD) {
    exec = __reduce_add_sync(FULL, exec);
    thr = __reduce_add_sync(FULL, thr);
    mxc = __reduce_max_sync(FULL, mxc);  // the CTA-id range of the BB groups (T_c table size)
    if (lane == 0 && exec) {
      atomicAdd(&C.bd_tot[0], exec);
      atomicAdd(&C.bd_tot[2], thr);
      atomicMax(&A.sc->max_cta, (unsigned long long)mxc);
    }
  }
}

// Segmented suffix scans: lane l gets the sum (OR) of lanes l .. h, h the
// first lane >= l whose head flag is set (h = 31 if none).  The head flag
// rides in bit 31 of the sum (v < 2^30: adding a lane's packed value to one
// without the flag copies that lane's flag); lane 31 always stops a segment,
// so no lane ever reads past it.
// The lane-bit masks of one valid run are disjoint, so they are ADDED
// (predicated IMADs by an opaque 1, off the ALU pipe); a repeated lane makes
// a carry, so popc(mask) < count still exposes it (flush_runs).
__device__ __forceinline__ void seg_scan2(uint32_t& v, uint32_t& m, uint32_t head, uint32_t one) {
  uint32_t x = v | ((head || lane_id() == 31u) ? 0x80000000u : 0u);
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t xo = __shfl_down_sync(FULL, x, d), mo = __shfl_down_sync(FULL, m, d);
    asm("{\n.reg .pred q;\nsetp.lt.s32 q, %2, 0;\n@!q mad.lo.u32 %0, %4, %3, %0;\n@!q mad.lo.u32 %1, %4, %5, %1;\n}"
        : "+r"(x), "+r"(m) : "r"(x), "r"(xo), "r"(one), "r"(mo));
  }
  v = x & 0x7fffffffu;
}

// r[k] for a lane-varying k < 8 (a 3-level select tree instead of local memory)
__device__ __forceinline__ uint32_t sel8(const uint32_t (&r)[8], uint32_t k) {
  const bool b0 = k & 1u, b1 = k & 2u, b2 = k & 4u;
  const uint32_t x01 = b0 ? r[1] : r[0], x23 = b0 ? r[3] : r[2];
  const uint32_t x45 = b0 ? r[5] : r[4], x67 = b0 ? r[7] : r[6];
  return b2 ? (b1 ? x67 : x45) : (b1 ? x23 : x01);
}

template <int F>
__global__ void __launch_bounds__(NTHR, 1) k_scan(const __grid_constant__ ScanArgs A) {
  constexpr bool RD = (F & F_RD) != 0, MD = (F & F_MD) != 0, BD = (F & F_BD) != 0;
  constexpr bool NA = (F & (F_RD | F_MD)) != 0, NG = (F & (F_MD | F_BD)) != 0;
  constexpr bool OBJ = (F & F_OBJ) != 0;
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ uint64_t bars[NWARP][KS];
  __shared__ uint32_t s_md_hist[2 * 33];
  __shared__ uint32_t s_bd_tot[3];
  const uint32_t tx = threadIdx.x, lane = lane_id(), warp = tx >> 5;
  uint32_t* sites = (uint32_t*)(smem + NWARP * R_BYTES);
  uint32_t* wh_all = sites + ((MD ? 2 : 0) + (BD ? 3 : 0)) * NSITE_SMEM;
  const bool sites_smem = A.nsites && A.nsites <= NSITE_SMEM;
  // F_OBJ tables after the run queues (scan_smem)
  uint8_t* objm = smem + NWARP * R_BYTES + ((MD ? 2 : 0) + (BD ? 3 : 0)) * NSITE_SMEM * 4 + NWARP * 68 * 4 +
                  NWARP * (qcap<F>() * 24 + 16);
  const bool obj_sm = OBJ && A.nobj < OBJ_SMEM;
  uint64_t* s_olo = (uint64_t*)objm;
  uint64_t* s_ohi = s_olo + OBJ_SMEM;
  uint32_t* s_dup = (uint32_t*)(s_ohi + OBJ_SMEM);
  uint32_t* s_mdo = s_dup + OBJ_SMEM;
  __shared__ Counters s_C;
  if (tx == 0)
    s_C = Counters{s_md_hist, (MD && sites_smem) ? sites : nullptr, s_bd_tot,
                   (BD && sites_smem) ? sites + (MD ? 2 * NSITE_SMEM : 0) : nullptr,
                   obj_sm ? s_olo : nullptr, obj_sm ? s_ohi : nullptr, (obj_sm && MD) ? s_mdo : nullptr,
                   obj_sm ? s_dup : nullptr, wh_all, sites_smem};
  const Counters& C = s_C;
  if (obj_sm) {
    for (uint32_t k = tx; k < A.nobj; k += NTHR) { s_olo[k] = A.obj_lo[k]; s_ohi[k] = A.obj_hi[k]; }
    for (uint32_t k = tx; k < OBJ_SMEM; k += NTHR) s_dup[k] = 0;
    if (MD)
      for (uint32_t k = tx; k < (A.nobj + 1) * 66; k += NTHR) s_mdo[k] = 0;
  }
  for (uint32_t k = tx; k < 2 * 33; k += NTHR) s_md_hist[k] = 0;
  if (tx < 3) s_bd_tot[tx] = 0;
  if (sites_smem)
    for (uint32_t k = tx; k < (uint32_t)((MD ? 2 : 0) + (BD ? 3 : 0)) * NSITE_SMEM; k += NTHR) sites[k] = 0;
  uint32_t* whist = wh_all + warp * 68;  // warp-private MD histogram [2][33]
  constexpr uint32_t QCAP = qcap<F>();
  const RunQueue<F> Q{wh_all + NWARP * 68 + warp * (QCAP * 6 + 4)};
  for (uint32_t k = lane; k < 68; k += 32) whist[k] = 0;
  __syncthreads();

  uint8_t* ring = smem + warp * R_BYTES;
  uint64_t* bar = bars[warp];
  uint32_t ndup = 0;
  // F_OBJ: duplicate loads counted per object row (run of one line per lane)
  uint64_t dc_line = ~0ull;
  uint32_t dc_row = 0, dc_cnt = 0;
  auto dc_flush = [&]() {
    if (dc_cnt) {
      if (C.dup) atomicAdd(&C.dup[dc_row], dc_cnt);
      else atomicAdd((unsigned long long*)&A.hist0[(uint64_t)dc_row * A.rd_nbins], (unsigned long long)dc_cnt);
      dc_cnt = 0;
    }
  };
  if (lane == 0) {
    for (int s = 0; s < KS; ++s) mbar_init(&bar[s], 1);
    fence_barrier_init();
  }
  __syncwarp();
  const uint32_t ring_s = smem_u32(ring), bar_s = smem_u32(bar);
  // Chunks are claimed dynamically (irregular traces have very uneven work
  // per record); each chunk is one reuse-distance region in trace order.
  // pg: pieces this warp issued before the current chunk (ring stage and
  // mbarrier phase run on across chunks).
  uint32_t pg = 0;
  for (uint64_t cid = __shfl_sync(FULL, lane == 0 ? atomicAdd(&A.sc->chunk_next, 1ull) : 0ull, 0); cid < A.nchunks;
       cid = __shfl_sync(FULL, lane == 0 ? atomicAdd(&A.sc->chunk_next, 1ull) : 0ull, 0)) {
    const uint64_t c_lo = cid < A.nbig ? cid * A.chunk : A.nbig * A.chunk + (cid - A.nbig) * A.chunk_s;
    const uint64_t c_len = cid < A.nbig ? A.chunk : A.chunk_s;
    const uint64_t c_hi = c_lo + c_len < A.n ? c_lo + c_len : A.n;
    uint32_t kept = 0;
    const uint32_t clen = (uint32_t)(c_hi - c_lo);
    // the chunk's last run may reach 32 records past its end; one more record
    // decides whether the last kept reuse record is followed by a duplicate
    const uint64_t s_end = c_hi + 32 < A.n ? c_hi + 32 : A.n;
    const uint32_t slen = (uint32_t)(s_end - c_lo);
    const uint32_t npieces = (slen + KR - 1) / KR;
    uint32_t issued = npieces < (uint32_t)KS ? npieces : (uint32_t)KS, waited = 0;
    fence_proxy_async();  // (the previous chunk's last reads of these stages precede the copies)
    for (uint32_t p = 0; p < issued; ++p) issue_piece<F>(A, ring_s, bar_s, c_lo, s_end, p, pg + p);
    // the record before the step (warp-uniform); meta 3 = "no record"
    // p_kb: kind bits of that record (bit 0 memory, 1 store, 2 BB; 0 = invalid / none)
    uint32_t p_cta = 0xffffffffu, p_t = 0, p_kb = 0, p_winst = 0, p_site = 0;
    uint64_t p_addr = 0;
    if (c_lo > 0) {
      p_cta = __ldg(A.cta + c_lo - 1);
      uint32_t pm0 = __ldg(A.meta + c_lo - 1);
      if (NA) p_addr = __ldg(A.addr + c_lo - 1);
      // an invalid record never continues a run of compressible accesses
      if (!meta_ok((uint8_t)pm0) || (NA && is_mem((uint8_t)pm0) && !addr_ok(p_addr, (uint8_t)pm0))) pm0 = 3;
      p_kb = (pm0 & 3u) < 2u ? (1u | ((pm0 & 1u) << 1)) : ((pm0 & 3u) == 2u ? 4u : 0u);
      if (NG) p_t = __ldg(A.tid + c_lo - 1);
      if (NG) p_winst = __ldg(A.winst + c_lo - 1);
      if (NG) p_site = __ldg(A.site + c_lo - 1);
    }
    // the run open at the step end (warp-uniform); owned iff it starts in the chunk
    bool cr_on = false, cr_own = false;
    uint32_t cr_v = 0, cr_mask = 0, cr_j = 0;
    uint32_t qn = 0;  // queued complete runs (warp-uniform)
    // RD: the last kept record when its compression run reaches the step end
    bool open_rd = false;
    uint64_t* wbv = A.vout ? A.vout + cid * A.kcap : nullptr;
    uint32_t* wbk = A.kout ? A.kout + cid * A.kcap : nullptr;

    for (uint32_t p = 0; p < npieces; ++p) {
      const uint32_t base = p * KR;
      if (base >= clen && !(NG && cr_on && cr_own) && !(RD && open_rd)) break;
      // piece p + 1 goes into the stage of piece p - 1 (consumed)
      if (p >= 1 && issued < npieces) {
        fence_proxy_async();
        issue_piece<F>(A, ring_s, bar_s, c_lo, s_end, issued, pg + issued);
        ++issued;
      }
      mbar_wait(&bar[(pg + p) % KS], ((pg + p) / KS) & 1u);
      waited = p + 1;
      // ---- this lane's LPR consecutive records (vector shared-memory loads)
      const uint32_t j0 = base + lane * LPR;
      // this step's stage in the ring; the lane's records start at slot lane * LPR
      const uint8_t* stg = ring + stage_of(pg + p);
      const uint32_t sl = lane * LPR;
      const uint64_t* r_addr = (const uint64_t*)(stg + S_ADDR);
      const uint32_t* r_cta = (const uint32_t*)(stg + S_CTA);
      const uint16_t* r_tid = (const uint16_t*)(stg + S_TID);
      const uint32_t* r_winst = (const uint32_t*)(stg + S_WINST);
      const uint32_t* r_site = (const uint32_t*)(stg + S_SITE);
      const uint8_t* r_meta = stg + S_META;
      uint32_t c[LPR], t[LPR], w[LPR], mmx, mmy, tor = 0;
      uint32_t sdm = 0;  // NG: site changes (a group's records share their site, reading R19)
      uint64_t a[LPR];
      {
        const uint4 c0 = *(const uint4*)(r_cta + sl), c1 = *(const uint4*)(r_cta + sl + 4);
        c[0] = c0.x; c[1] = c0.y; c[2] = c0.z; c[3] = c0.w; c[4] = c1.x; c[5] = c1.y; c[6] = c1.z; c[7] = c1.w;
        const uint2 mm = *(const uint2*)(r_meta + sl);
        mmx = mm.x;
        mmy = mm.y;
        if (NG) {
          const uint4 t4 = *(const uint4*)(r_tid + sl);
          tor = t4.x | t4.y | t4.z | t4.w;
          t[0] = t4.x & 0xffffu; t[1] = t4.x >> 16; t[2] = t4.y & 0xffffu; t[3] = t4.y >> 16;
          t[4] = t4.z & 0xffffu; t[5] = t4.z >> 16; t[6] = t4.w & 0xffffu; t[7] = t4.w >> 16;
          const uint4 w0 = *(const uint4*)(r_winst + sl), w1 = *(const uint4*)(r_winst + sl + 4);
          w[0] = w0.x; w[1] = w0.y; w[2] = w0.z; w[3] = w0.w; w[4] = w1.x; w[5] = w1.y; w[6] = w1.z; w[7] = w1.w;
          {  // site changes, compared at once (the site registers die here)
            const uint4 s0 = *(const uint4*)(r_site + sl), s1 = *(const uint4*)(r_site + sl + 4);
            uint32_t psi = __shfl_up_sync(FULL, s1.w, 1);
            if (lane == 0) psi = p_site;
            p_site = __shfl_sync(FULL, s1.w, 31);
            const uint32_t one = A.one;
            add_if_nz(sdm, s0.x ^ psi, one, 1u);
            add_if_nz(sdm, s0.y ^ s0.x, one, 2u);
            add_if_nz(sdm, s0.z ^ s0.y, one, 4u);
            add_if_nz(sdm, s0.w ^ s0.z, one, 8u);
            add_if_nz(sdm, s1.x ^ s0.w, one, 16u);
            add_if_nz(sdm, s1.y ^ s1.x, one, 32u);
            add_if_nz(sdm, s1.z ^ s1.y, one, 64u);
            add_if_nz(sdm, s1.w ^ s1.z, one, 128u);
          }
        } else {
#pragma unroll
          for (int k = 0; k < LPR; ++k) t[k] = w[k] = 0;
        }
        if (NA) {
#pragma unroll
          for (int q = 0; q < LPR / 2; ++q) {
            const uint4 v = *(const uint4*)(r_addr + sl + 2 * q);
            a[2 * q] = ((uint64_t)v.y << 32) | v.x;
            a[2 * q + 1] = ((uint64_t)v.w << 32) | v.z;
          }
        } else {
#pragma unroll
          for (int k = 0; k < LPR; ++k) a[k] = 0;
        }
      }
      // owned / in-stream records of the lane (all of them except near the chunk end)
      uint32_t ownm = 0xffu, inbm = 0xffu;
      if (base + KR > clen) {  // (warp-uniform: only the chunk's last steps)
        ownm = j0 >= clen ? 0u : (clen - j0 >= LPR ? 0xffu : (1u << (clen - j0)) - 1u);
        inbm = j0 >= slen ? 0u : (slen - j0 >= LPR ? 0xffu : (1u << (slen - j0)) - 1u);
      }
      // kind masks (bit k = record k) from the meta bytes
      const uint32_t glo = gather8(mmx, mmy), ghi = gather8(mmx >> 1, mmy >> 1);
      uint32_t okm = inbm;
      {
        // validation trigger: SWAR over the lane's records, 4 per meta word (byte
        // permutes gather the low address byte / the address's top byte of 4
        // records); a superset of the bad records (it may also fire on records
        // past the chunk) - the exact per-record check below decides
        uint32_t trig = 0;
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const uint32_t v = h ? mmy : mmx, v1 = v >> 1;
          const uint32_t K = (~v1 & 0x01010101u) * 0xffu;  // memory records (kind bit 1 clear)
          const uint32_t S = (v >> 2) & 0x07070707u;        // log2(bytes)
          // (1 << log2(bytes)) - 1 per memory record (bit 4 set iff more than 16 bytes)
          const uint32_t M = __byte_perm(0x07030100u, 0x7f3f1f0fu, __byte_perm(S | (S >> 4), 0u, 0x0020u)) & K;
          trig |= (v & 0xe0e0e0e0u) | (v & v1 & 0x01010101u);  // reserved bits, kind 3
          if (NA) {
            const int i = 4 * h;
            const uint32_t L = __byte_perm(__byte_perm((uint32_t)a[i], (uint32_t)a[i + 1], 0x0040u),
                                           __byte_perm((uint32_t)a[i + 2], (uint32_t)a[i + 3], 0x0040u), 0x5410u);
            const uint32_t H = __byte_perm(__byte_perm((uint32_t)(a[i] >> 32), (uint32_t)(a[i + 1] >> 32), 0x0073u),
                                           __byte_perm((uint32_t)(a[i + 2] >> 32), (uint32_t)(a[i + 3] >> 32), 0x0073u),
                                           0x5410u);
            // misaligned / > 16 B; RD: address >= 2^58 (a superset of line >= 2^58, the packing limit)
            trig |= ((L | 0x10101010u) & M) | (RD ? (H & K & 0xfcfcfcfcu) : 0u);
          } else {
            trig |= M & 0x10101010u;
          }
        }
        if (__any_sync(FULL, trig != 0 || (NG && (tor & 0xfc00fc00u)))) {
#pragma unroll
          for (int k = 0; k < LPR; ++k) {
            if (!((ownm >> k) & 1u)) continue;
            const uint8_t m = (uint8_t)(((k < 4 ? mmx : mmy) >> (8 * (k & 3))) & 0xffu);
            bool ok = meta_ok(m);
            if (NA && ok && is_mem(m)) ok = addr_ok(a[k], m);
            if (NG && ok) ok = t[k] < 1024u;
            if (!ok) {
              report(A.sc, c_lo + j0 + k, 1);
              okm &= ~(1u << k);
            } else if (RD && is_mem(m) && ((a[k] >> A.lbs_rd) >> 58)) {
              // a valid record whose line does not fit the kept-record packing
              atomicMin(&A.sc->unsup_index, (unsigned long long)(c_lo + j0 + k));
            }
          }
        }
      }
      const uint32_t memm = ~ghi & okm, stm = glo & ~ghi & okm, bbm = ~glo & ghi & okm;

      // predecessor of record 0: the previous lane's last record (lane 0: the carry)
      uint32_t pc = __shfl_up_sync(FULL, c[LPR - 1], 1);
      uint32_t pkb = __shfl_up_sync(FULL, ((memm >> 7) & 1u) | ((stm >> 6) & 2u) | ((bbm >> 5) & 4u), 1);
      uint32_t pt = NG ? __shfl_up_sync(FULL, t[LPR - 1], 1) : 0u, pwi = NG ? __shfl_up_sync(FULL, w[LPR - 1], 1) : 0u;
      uint64_t pa = NA ? __shfl_up_sync(FULL, a[LPR - 1], 1) : 0ull;
      if (lane == 0) { pc = p_cta; pkb = p_kb; pt = p_t; pwi = p_winst; pa = p_addr; }

      // ---- every comparison with the predecessor first, so that the record
      //      registers die here (kept-record writes below re-read the ring)
      // RD  eqm: same (scope, line) as the predecessor (32-bit halves, line bits only, lbs <= 12)
      // NG  rsm: run starts ((cta, winst, warp32) differ); nlm: MD line changes; vim: line decreases
      uint32_t eqm = 0, rsm = 0, nlm = 0, vim = 0;
      uint64_t tl5 = 0;  // NG: the records' lanes, 5 bits each
      {
        const uint32_t one = A.one;
        const uint32_t mlr = ~((1u << A.lbs_rd) - 1u), msc = A.cta_scope ? 0xffffffffu : 0u;
        const uint32_t mlm = ~((1u << A.lbs_md) - 1u);
#pragma unroll
        for (int k = 0; k < LPR; ++k) {
          const uint64_t qa = k == 0 ? pa : a[k - 1];
          const uint32_t qc = k == 0 ? pc : c[k - 1];
          const uint32_t dlo = (uint32_t)a[k] ^ (uint32_t)qa, dhi = (uint32_t)(a[k] >> 32) ^ (uint32_t)(qa >> 32);
          if (RD) add_if_nz(eqm, (dlo & mlr) | dhi | ((c[k] ^ qc) & msc), one, 1u << k);  // (inverted below)
          if (NG) {
            const uint32_t qw = k == 0 ? pwi : w[k - 1], qt = k == 0 ? pt : t[k - 1];
            add_if_nz(rsm, (c[k] ^ qc) | (w[k] ^ qw) | ((t[k] ^ qt) & ~31u), one, 1u << k);
            if (MD) {
              add_if_nz(nlm, (dlo & mlm) | dhi, one, 1u << k);
              add_if_lt(vim, a[k], qa, one, 1u << k);  // only where the line changes (masked below)
            }
            tl5 |= (uint64_t)(t[k] & 31u) << (5 * k);
          }
        }
        eqm = ~eqm & 0xffu;
      }
      // ---- carry the step's last record to the next step
      p_cta = __shfl_sync(FULL, c[LPR - 1], 31);
      p_kb = __shfl_sync(FULL, ((memm >> 7) & 1u) | ((stm >> 6) & 2u) | ((bbm >> 5) & 4u), 31);
      if (NG) p_t = __shfl_sync(FULL, t[LPR - 1], 31);
      if (NG) p_winst = __shfl_sync(FULL, w[LPR - 1], 31);
      if (NA) p_addr = __shfl_sync(FULL, a[LPR - 1], 31);

      // ================= R1: run compression of the chunk's records
      // dup  : a load repeating its predecessor's (scope, line): RD 0, never kept;
      // chain: consecutive stores to one (scope, line); every 16th one is kept
      //        with the weight of the chain piece it heads.  Chains are cut at
      //        step starts and at the chunk end (both only split a piece).
      if (RD) {
        const uint32_t pm = ((memm << 1) | (pkb & 1u)) & 0xffu, ps = ((stm << 1) | ((pkb >> 1) & 1u)) & 0xffu;
        const uint32_t dupm = eqm & memm & ~stm & pm;
        const uint32_t contm = eqm & stm & ps & (lane == 0 ? 0xfeu : 0xffu);
        // breaks: records that do not continue a store chain (the chunk end is one)
        const uint32_t brk = (~contm | ~ownm) & 0xffu;
        const uint32_t sb = lane * LPR;
        const uint32_t hb = __ballot_sync(FULL, brk != 0);
        const uint32_t lt = hb & lanemask_lt(), gt = hb & ~lanemask_le();
        const uint32_t fbk = brk ? (uint32_t)(__ffs(brk) - 1) : (uint32_t)LPR;
        const uint32_t lastb = brk ? sb + 31u - __clz(brk) : 0u;
        const uint32_t sv = __shfl_sync(FULL, lastb, lt ? 31u - __clz(lt) : 0u);
        const uint32_t nv = __shfl_sync(FULL, (sb + fbk) | (((dupm >> fbk) & 1u) << 16), gt ? (uint32_t)(__ffs(gt) - 1) : 0u);
        const uint32_t nb_l = gt ? (nv & 0xffffu) : (uint32_t)KR;  // first break after the lane
        const bool nd_l = gt && (nv >> 16);
        // chain records before the lane's first break continue a chain started at
        // sv: the one at chain position 16 m (if any) is kept
        const uint32_t k0 = ((lt ? sv : 0u) - sb) & 15u;
        uint32_t keepm = (memm & ~dupm & brk) | (k0 < fbk ? (1u << k0) : 0u);
        keepm &= ownm;
        if (open_rd && lane == 0 && (dupm & 1u) && kept - 1 < A.kcap) wbv[kept - 1] |= 1ull << VB_DUP;  // the previous step's open piece
        const uint32_t nk = __popc(keepm);
        uint32_t x = nk;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t y = __shfl_up_sync(FULL, x, o);
          if (lane >= (uint32_t)o) x = A.one * y + x;  // (IMAD: off the ALU pipe)
        }
        const uint32_t tot = __shfl_sync(FULL, x, 31);
        uint32_t pos = kept + x - nk;
        bool last_open = false;
        for (uint32_t km = keepm; km; km &= km - 1) {  // (~7 % of the records are kept)
          const uint32_t k = __ffs(km) - 1;
          const uint32_t after = brk & (0xffu << (k + 1)) & 0xffu;
          const uint32_t ab = after ? (uint32_t)(__ffs(after) - 1) : 0u;
          const uint32_t nb = after ? sb + ab : nb_l;   // the first break after record k
          const bool nd = after ? ((dupm >> ab) & 1u) != 0 : nd_l;
          uint32_t wgt = nb - (sb + k);
          bool hd = nd;
          if (wgt > 16u) { wgt = 16u; hd = false; }      // the chain goes on with another kept store
          else last_open = nb == (uint32_t)KR;           // decided by the next step's first record
          if (pos < A.kcap) {
            wbv[pos] = (lds_u64(r_addr + sl + k) >> A.lbs_rd) | ((uint64_t)((stm >> k) & 1u) << VB_STORE) |
                       ((uint64_t)hd << VB_DUP) | ((uint64_t)(wgt - 1u) << VB_W);
            if (wbk) wbk[pos] = A.cta_scope ? lds_u32(r_cta + sl + k) : 0u;
          }
          ++pos;
        }
        open_rd = __ballot_sync(FULL, last_open) != 0;
        kept += tot;
        if (OBJ) {
          // runs of consecutive duplicate loads: a duplicate repeats its
          // predecessor's line, so a run is one line (one lookup, one count)
          uint32_t dm = dupm & ownm;
          while (dm) {
            const uint32_t k = __ffs(dm) - 1, len = __ffs(~(dm >> k)) - 1;
            const uint64_t ln = lds_u64(r_addr + sl + k) >> A.lbs_rd;
            if (ln != dc_line) {
              dc_flush();
              dc_line = ln;
              dc_row = row_of(A, C, ln);
            }
            dc_cnt += len;
            dm &= ~(((1u << len) - 1u) << k);
          }
        } else {
          ndup += __popc(dupm & ownm);
        }
        __syncwarp();
      }

      // ================= M1-M3 / B1-B3: runs = warp-level groups
      if (NG) {
        vim &= nlm;
        rsm |= (bbm ^ ((bbm << 1) | ((pkb >> 2) & 1u))) & 0xffu;  // BB and memory records never share a run
        rsm |= ~inbm & 0xffu;  // every record past the stream is a run of its own (never finalized)
        nlm |= rsm;
        vim &= ~rsm;
        {
          // a record continuing a run must have its predecessor's kind and site
          // (both valid records): else the group mixes static instructions
          const uint32_t kcm = (stm ^ ((stm << 1) | ((pkb >> 1) & 1u))) & 0xffu;
          const uint32_t pvm = ((okm << 1) | (pkb ? 1u : 0u)) & 0xffu;
          const uint32_t gv = (sdm | kcm) & ~rsm & ownm & okm & pvm;
          if (__any_sync(FULL, gv != 0) && gv) report(A.sc, c_lo + j0 + __ffs(gv) - 1, 4);
        }
        // lane bits of each in-lane run piece (backward)
        uint32_t rm[LPR];
        uint32_t m = 0;
#pragma unroll
        for (int k = LPR - 1; k >= 0; --k) {
          m = A.one * (1u << (tl5 >> (5 * k) & 31u)) + m;  // disjoint lanes: + == | (IMAD, FMA pipe)
          rm[k] = m;
          if ((rsm >> k) & 1u) m = 0;
        }
        // the lane's prefix (records before its first run start)
        const uint32_t fr = rsm ? (uint32_t)(__ffs(rsm) - 1) : (uint32_t)LPR;
        const uint32_t pre = (1u << fr) - 1u;
        uint32_t u = __popc(nlm & pre) | (fr << PK_CNT) | (__popc(vim & pre) << PK_VIOL);
        const uint32_t head = rsm != 0;
        seg_scan2(u, m, head, A.one);
        const uint32_t S_next = __shfl_down_sync(FULL, u, 1), M_next = __shfl_down_sync(FULL, m, 1);
        const uint32_t heads = __ballot_sync(FULL, head);
        // ---- the run carried in from the previous step ends at the first head
        if (cr_on) {
          cr_v += __shfl_sync(FULL, u, 0);
          cr_mask |= __shfl_sync(FULL, m, 0);
          if (((cr_v >> PK_CNT) & PK_M) > 32) {  // a lane repeats: bad trace (stop counting)
            if (lane == 0 && cr_own) report(A.sc, c_lo + cr_j, 2);
            cr_own = false;
          }
          if (heads) {
            if (cr_own) {
              if (lane == 0) {
                Q.j(qn) = cr_j;
                Q.u(qn) = cr_v;
                Q.m(qn) = cr_mask;
                Q.kt(qn) = Q.carry()[0];
                Q.cta(qn) = Q.carry()[1];
                Q.site(qn) = Q.carry()[2];
              }
              ++qn;
            }
            cr_on = false;
          }
        }
        // ---- runs starting in this lane that end in this step are queued
        const bool above = (heads & ~lanemask_le()) != 0;
        const uint32_t lastk = rsm ? 31u - __clz(rsm) : 0u;
        const uint32_t starts = rsm & inbm;
        const bool tail_open = !above && ((starts >> lastk) & 1u);  // continues past the step end
        const uint32_t todo = starts & ownm & ~(tail_open ? 1u << lastk : 0u);
        // rounds over the lanes' run starts (one per lane per round; usually one round)
        for (uint32_t td = todo;;) {
          const uint32_t bm = __ballot_sync(FULL, td != 0);
          if (!bm) break;
          if (qn > QCAP - 32) {  // room for one more round
            __syncwarp();
            flush_runs<F>(A, &s_C, qn, c_lo, stg, base);
            qn = 0;
            __syncwarp();
          }
          if (td) {
            const uint32_t k = __ffs(td) - 1;
            td &= td - 1;
            const uint32_t nxt = rsm & (0xfeu << k) & 0xffu;
            const uint32_t seg = (nxt ? (nxt & (0u - nxt)) - 1u : 0xffu) & (0xffu << k);
            uint32_t u2 = __popc(nlm & seg) | (__popc(seg) << PK_CNT) | (__popc(vim & seg) << PK_VIOL);
            uint32_t m2 = sel8(rm, k);
            if (k == lastk) { u2 += S_next; m2 |= M_next; }  // closed by a later lane's head
            const uint32_t pos = qn + __popc(bm & lanemask_lt());
            Q.j(pos) = j0 + k;
            Q.u(pos) = u2;
            Q.m(pos) = m2;
            Q.kt(pos) = ((r_meta[sl + k] & 3u) << 16) | r_tid[sl + k];
            Q.cta(pos) = r_cta[sl + k];
            Q.site(pos) = A.nsites ? r_site[sl + k] : 0u;
          }
          qn += __popc(bm);
        }
        if (qn >= 32) {
          __syncwarp();
          flush_runs<F>(A, &s_C, qn, c_lo, stg, base);
          qn = 0;
        }
        // ---- the last head lane's open run becomes the carry
        if (heads) {
          const uint32_t hl = 31u - __clz(heads);
          uint32_t tu = 0, tmk = 0;
          if (tail_open) {
            const uint32_t msk = 0xffu << lastk;
            tu = __popc(nlm & msk) | ((LPR - lastk) << PK_CNT) | (__popc(vim & msk) << PK_VIOL);
            tmk = sel8(rm, lastk);
            if (lane < 31) { tu += S_next; tmk |= M_next; }
            // the carried run's first record (its stage is recycled before the run closes)
            const uint32_t sl0 = sl + lastk;
            Q.carry()[0] = ((r_meta[sl0] & 3u) << 16) | r_tid[sl0];
            Q.carry()[1] = r_cta[sl0];
            Q.carry()[2] = A.nsites ? r_site[sl0] : 0u;
          }
          cr_on = __shfl_sync(FULL, (uint32_t)tail_open, hl) != 0;
          cr_v = __shfl_sync(FULL, tu, hl);
          cr_mask = __shfl_sync(FULL, tmk, hl);
          cr_j = __shfl_sync(FULL, j0 + lastk, hl);
          cr_own = cr_j < clen;

        }
        __syncwarp();
      }
      __syncwarp();
    }
    // a run open at the end of the stream ends with the trace; then the rest of the queue
    if (NG && cr_on && cr_own) {
      if (lane == 0) {
        Q.j(qn) = cr_j;
        Q.u(qn) = cr_v;
        Q.m(qn) = cr_mask;
        Q.kt(qn) = Q.carry()[0];
        Q.cta(qn) = Q.carry()[1];
        Q.site(qn) = Q.carry()[2];
      }
      ++qn;
    }
    if (NG && qn) {
      __syncwarp();
      flush_runs<F>(A, &s_C, qn, c_lo, nullptr, 0xffffffffu);
    }
    // no bulk copy may still target the ring when the chunk (CTA) is done
    for (uint32_t q = waited; q < issued; ++q) mbar_wait(&bar[(pg + q) % KS], ((pg + q) / KS) & 1u);
    pg += issued;
    if (RD && lane == 0) {
      A.wcnt[cid] = kept;
      if (kept > A.kcap) atomicMax(&A.sc->kept_max, (unsigned long long)kept);
    }
    __syncwarp();
  }

  if (RD && !OBJ) {
    const uint32_t d = __reduce_add_sync(FULL, ndup);
    if (lane == 0 && d) atomicAdd((unsigned long long*)A.hist0, (unsigned long long)d);
  }
  if (RD && OBJ) dc_flush();
  if (MD && !OBJ) {
    __syncwarp();
    for (uint32_t k = lane; k < 66; k += 32)
      if (whist[k]) atomicAdd(&s_md_hist[k], whist[k]);
  }
  // ---- flush block-level counters
  __syncthreads();
  if (RD && obj_sm)
    for (uint32_t k = tx; k <= A.nobj; k += NTHR)
      if (s_dup[k]) atomicAdd((unsigned long long*)&A.hist0[(uint64_t)k * A.rd_nbins], (unsigned long long)s_dup[k]);
  if (MD && obj_sm) {
    const uint32_t W = 1u << A.ws_md;
    for (uint32_t k = tx; k < (A.nobj + 1) * 66; k += NTHR) {
      const uint32_t row = k / 66, kind = (k % 66) / 33, deg = k % 33;
      if (s_mdo[k] && deg <= W)
        atomicAdd((unsigned long long*)&A.md_hist[(row * 2 + kind) * (W + 1) + deg], (unsigned long long)s_mdo[k]);
    }
  }
  if (MD && !OBJ) {
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
// m: number of deferred groups, read on the device (no host round trip)
__global__ void __launch_bounds__(256) k_bd_resolve(const uint4* __restrict__ defer,
                                                    const unsigned long long* __restrict__ pm, uint64_t cap,
                                                    const uint32_t* __restrict__ tc, uint32_t gen, uint32_t ws,
                                                    uint64_t* bd_tot, uint64_t* bd_sites, uint32_t nsites) {
  const uint64_t m = *pm < cap ? *pm : cap;
  __shared__ uint32_t s_div[NSITE_SMEM];
  const bool sm = nsites && nsites <= NSITE_SMEM;
  if (sm)
    for (uint32_t k = threadIdx.x; k < nsites; k += blockDim.x) s_div[k] = 0;
  __syncthreads();
  uint32_t tot = 0;
  const uint32_t W = 1u << ws;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint4 d = defer[i];
    const uint32_t v = __ldg(tc + d.x);
    const uint32_t tcv = (v >> 11) == gen ? (v & 0x7ffu) : 0u;  // 1 + max tid of the CTA's BB records
    int64_t live = (int64_t)tcv - (int64_t)d.y * W;
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
// Also R0's CTA-id range of the kept records (the radix sort's key bits).
__global__ void __launch_bounds__(256) k_squeeze(const uint32_t* __restrict__ kin, const uint64_t* __restrict__ vin,
                                                 uint32_t* __restrict__ kout, uint64_t* __restrict__ vout,
                                                 const uint64_t* __restrict__ cnt, const uint64_t* __restrict__ off,
                                                 uint64_t chunk, Scalars* sc) {
  const uint64_t b = blockIdx.x, m = cnt[b], o = off[b];
  const uint64_t src = b * chunk;
  uint32_t mx = 0;
  // 4 elements per thread per round: all loads issued before the stores
  for (uint64_t k0 = threadIdx.x; k0 < m; k0 += 4ull * blockDim.x) {
    uint64_t v[4];
    uint32_t key[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const uint64_t k = k0 + (uint64_t)u * blockDim.x;
      if (k < m) {
        v[u] = vin[src + k];
        key[u] = kin ? kin[src + k] : 0u;
      }
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const uint64_t k = k0 + (uint64_t)u * blockDim.x;
      if (k < m) {
        vout[o + k] = v[u];
        if (kin) {
          kout[o + k] = key[u];
          mx = max(mx, key[u]);
        }
      }
    }
  }
  mx = __reduce_max_sync(FULL, mx);
  if (lane_id() == 0 && mx) atomicMax(&sc->max_cta, (unsigned long long)mx);
}

template <int F>
size_t scan_smem() {
  constexpr bool MD = (F & F_MD) != 0, BD = (F & F_BD) != 0, OBJ = (F & F_OBJ) != 0;
  return (size_t)NWARP * R_BYTES + (size_t)((MD ? 2 : 0) + (BD ? 3 : 0)) * NSITE_SMEM * 4 + (size_t)NWARP * 68 * 4 +
         (size_t)NWARP * (qcap<F>() * 24 + 16) + (OBJ ? (size_t)OBJ_SMEM * (16 + 4 + (MD ? 66 * 4 : 0)) : 0);
}

const char* const kScanName[16] = {"k_scan<0>", "k_scan<1>", "k_scan<2>", "k_scan<3>", "k_scan<4>", "k_scan<5>",
                                   "k_scan<6>", "k_scan<7>", "k_scan<8>", "k_scan<9>", "k_scan<10>", "k_scan<11>",
                                   "k_scan<12>", "k_scan<13>", "k_scan<14>", "k_scan<15>"};

template <int F>
cudaError_t launch_scan_t(cadv_ctx* c, const ScanArgs& A, uint64_t grid) {
  const size_t smem = scan_smem<F>();
  if (!(c->attr_set & (1u << F))) {
    cudaError_t e = cudaFuncSetAttribute(k_scan<F>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    c->attr_set |= 1u << F;
  }
  CADV_LAUNCH_N(c, kScanName[F], k_scan<F><<<(unsigned)grid, NTHR, smem, c->stream>>>(A));
  return cudaGetLastError();
}

}  // namespace

// One CTA per SM; the trace is cut into chunks of a multiple of KR records,
// 1-4 per warp (CADV_SCAN_SPLIT overrides), which the warps claim
// dynamically; *nchunks = number of chunks (= reuse-distance regions).  With
// more than one chunk per warp, the last half chunk per warp of the trace is
// cut into quarter chunks (n < 2^31): warps that claim late finish at nearly
// the same time even when the work per record is very uneven.
// Chunks [0, *nbig) have *chunk records, the others *chunk_s.
void scan_geometry(cadv_ctx* c, uint64_t n, uint64_t* grid, uint64_t* nchunks, uint64_t* chunk, uint64_t* nbig,
                   uint64_t* chunk_s) {
  uint64_t g = (uint64_t)c->num_sms;
  if (c->scan_ctas > 0 && (uint64_t)c->scan_ctas < g) g = (uint64_t)c->scan_ctas;
  // up to 4 chunks per warp, none shorter than 64 steps (16 K records):
  // each chunk start waits for its first bulk copy with nothing to overlap
  // (8 K-record chunks cost C2 0.38 -> 0.49 ms).  A trace below 2^28 records
  // that already has 4 full chunks per warp gets 6: with fewer records per
  // warp the cost variance between chunks is a larger share of the kernel
  // (C3 BFS 2.19 -> 2.03 ms), while on C4 the extra regions cost the regroup
  // more than they save.
  uint64_t split = n / (g * NWARP * 16384);
  split = split < 1 ? 1 : (split > 4 ? 4 : split);
  if (split == 4 && n < (1ull << 28)) split = 6;
  if (c->scan_split > 0) split = (uint64_t)c->scan_split;
  const uint64_t tw = g * NWARP * split;
  uint64_t ch = (n + tw - 1) / tw;
  ch = ((ch + KR - 1) / KR) * KR;
  if (ch == 0) ch = KR;
  uint64_t nb = (n + ch - 1) / ch, cs = ch, nc = nb;
  // (n < 2^31: the tail's extra regions cost kept-record workspace, which a
  // 4e9-record context cannot spare)
  if (split > 1 && n < (1ull << 31) && getenv("CADV_SCAN_NOTAIL") == nullptr) {
    cs = ((ch / 4 + KR - 1) / KR) * KR;
    uint64_t tq = 2;  // tail quarter chunks per warp
    if (const char* ev = getenv("CADV_SCAN_TAIL")) tq = (uint64_t)atoi(ev);
    const uint64_t tail = g * NWARP * (ch / 4) * tq;
    nb = n > tail ? (n - tail) / ch : 0;
    const uint64_t rest = n - nb * ch;
    nc = nb + (rest + cs - 1) / cs;
  }
  *chunk = ch;
  *nchunks = nc ? nc : 1;
  if (nbig) *nbig = nb;
  if (chunk_s) *chunk_s = cs;
  uint64_t gg = (*nchunks + NWARP - 1) / NWARP;
  if (gg > g) gg = g;
  *grid = gg ? gg : 1;
}

cudaError_t launch_squeeze(cadv_ctx* c, const uint32_t* kin, const uint64_t* vin, uint32_t* kout, uint64_t* vout,
                           const uint64_t* cnt, const uint64_t* off, uint64_t nchunks, uint64_t chunk) {
  if (nchunks == 0) return cudaSuccess;
  CADV_LAUNCH(c, k_squeeze<<<(unsigned)nchunks, 256, 0, c->stream>>>(kin, vin, kout, vout, cnt, off, chunk, scalars(c)));
  return cudaGetLastError();
}

cudaError_t launch_scan(cadv_ctx* c, int flags, const ScanParams& P) {
  const cadv_trace_desc& t = P.t;
  if (t.n == 0) return cudaSuccess;
  ScanArgs A{};
  A.addr = t.addr; A.cta = t.cta; A.tid = t.tid; A.site = t.site; A.winst = t.winst; A.meta = t.meta;
  A.n = t.n;
  uint64_t grid;
  scan_geometry(c, t.n, &grid, &A.nchunks, &A.chunk, &A.nbig, &A.chunk_s);
  A.lbs_rd = P.lbs_rd; A.cta_scope = P.cta_scope; A.kout = P.kout; A.vout = P.vout; A.wcnt = P.blkcnt;
  A.kcap = P.kcap;
  A.hist0 = P.hist0;
  A.lbs_md = P.lbs_md; A.ws_md = P.ws_md; A.md_hist = P.md_hist; A.md_sites = P.md_sites;
  A.ws_bd = P.ws_bd; A.tc = P.tc; A.tc_cap = P.tc_cap; A.tc_gen = P.tc_gen; A.defer_cap = P.defer_cap;
  A.bd_tot = P.bd_tot; A.bd_sites = P.bd_sites; A.defer = (uint4*)P.defer;
  A.ndefer = P.ndefer;
  A.nsites = P.nsites; A.site_flag = P.site_flag; A.sc = scalars(c);
  A.obj_lo = P.obj_lo; A.obj_hi = P.obj_hi; A.nobj = P.nobj; A.rd_nbins = P.rd_nbins;
  A.one = 1;
  switch (flags) {
    case 1: return launch_scan_t<1>(c, A, grid);
    case 2: return launch_scan_t<2>(c, A, grid);
    case 3: return launch_scan_t<3>(c, A, grid);
    case 4: return launch_scan_t<4>(c, A, grid);
    case 5: return launch_scan_t<5>(c, A, grid);
    case 6: return launch_scan_t<6>(c, A, grid);
    case 7: return launch_scan_t<7>(c, A, grid);
    // data-centric attribution (cadv_data_centric): reuse and / or memory divergence per object
    case F_OBJ | 1: return launch_scan_t<F_OBJ | 1>(c, A, grid);
    case F_OBJ | 2: return launch_scan_t<F_OBJ | 2>(c, A, grid);
    case F_OBJ | 3: return launch_scan_t<F_OBJ | 3>(c, A, grid);
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t launch_bd_resolve(cadv_ctx* c, const void* defer, const unsigned long long* m, uint64_t cap,
                              const uint32_t* tc, uint32_t tc_gen, uint32_t ws, uint64_t* bd_tot, uint64_t* bd_sites,
                              uint32_t nsites) {
  const uint64_t want = (cap + 255) / 256;
  const int grid = (int)(want < (uint64_t)c->num_sms * 4 ? (want ? want : 1) : (uint64_t)c->num_sms * 4);
  CADV_LAUNCH(c, k_bd_resolve<<<grid, 256, 0, c->stream>>>((const uint4*)defer, m, cap, tc, tc_gen, ws, bd_tot,
                                                           bd_sites, nsites));
  return cudaGetLastError();
}

}  // namespace cadv
