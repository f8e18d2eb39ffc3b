// cadv_impl.h — internal context and launcher declarations of libcadv.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "../../include/cadv.h"
#include "cadv_comm.h"

namespace cadv {

// Device workspace buffer that only grows (allocation happens on the first
// call that needs it; later calls of the same size allocate nothing).
struct DevBuf {
  void* p = nullptr;
  size_t bytes = 0;
  // exported to peer processes (CUDA IPC, map_peers): never freed while the
  // context lives (an importer may still map it, and a freed range that the
  // driver hands out again would collide with that mapping); grown 2x
  bool exported = false;
};

// Small per-call device scalars (zeroed at the start of every analysis).
struct Scalars {
  unsigned long long err_index;  // first offending record (ULLONG_MAX = none)
  unsigned int err_code;         // 1 = bad record, 2 = run longer than 32 / duplicate lane,
                                 // 3 = internal invariant, 4 = group mixes kinds / sites
  unsigned long long unsup_index;  // first memory record whose reuse line is >= 2^58 (ULLONG_MAX = none)
  unsigned long long kept_max;   // scan (RD): most kept records of one chunk (region capacity check)
  unsigned long long chunk_next; // scan: next chunk to claim
  unsigned int tile_counter;     // dynamic tile assignment
  unsigned long long count[8];   // generic counters (kept records, entries, ...)
  unsigned long long max_cta;    // scan: max CTA id of the trace (shard)
  unsigned long long n_kind[4];  // (unused)
  unsigned long long tc_overflow;  // scan: a CTA id >= the T_c capacity was seen
  unsigned long long ndefer;     // branch divergence: deferred partial groups
  unsigned long long rd_line_min, rd_line_max;  // reuse cross-tile phase: entry line range
  unsigned long long rg_overflow;  // regroup: a scan region holds more than RG_MAX distinct CTAs
};

enum BufId {
  B_SCALARS, B_HOST_COPY0, B_HOST_COPY1, B_HOST_COPY2, B_HOST_COPY3, B_HOST_COPY4, B_HOST_COPY5,
  B_HIST, B_SITES, B_TC,
  B_SORT_K0, B_SORT_K1, B_SORT_V0, B_SORT_V1, B_SORT_HIST, B_SCAN_TMP,
  B_GATHER,
  B_RD_KEY, B_RD_VAL, B_RD_TILESTAT, B_RD_TILEW, B_RD_TILEQ, B_RD_ENT, B_RD_ENT_KEY0, B_RD_ENT_KEY1,
  B_RD_ENT_IDX0, B_RD_ENT_IDX1, B_RD_XQ, B_RD_XQ2, B_RD_XTMP, B_DEFER, B_OUT2,
  B_ALIGN0, B_ALIGN1, B_ALIGN2, B_ALIGN3, B_ALIGN4, B_ALIGN5,
  B_XCH_K0, B_XCH_K1, B_XCH_V0, B_XCH_V1, B_XCH_CNT, B_COMM, B_OBJ, B_RD_ENT_ALL,
  B_RG_PK, B_RG_PN, B_RG_NP, B_RG_SORT, B_RG_SEG,
  B_WX_RECV, B_WX_K0, B_WX_K1, B_WX_V0, B_WX_V1, B_WX_COLS,
  B_XE_OWN, B_XE_SEND, B_XE_CNT, B_XE_ALLP, B_RD_XQR,
  B_COUNT
};

}  // namespace cadv

struct cadv_ctx {
  int device = 0;
  cudaStream_t stream = nullptr;
  int rank = 0, nranks = 1;
  cadv::Comm* comm = nullptr;            // collectives when nranks > 1 (NCCL or loopback)
  cadv::LoopbackGroup* loopback = nullptr;
  bool split_group = false;              // a shard boundary splits a warp-level group (load_trace)
  int num_sms = 148;
  int scan_ctas = 0;     // CADV_SCAN_CTAS (testing): cap on the scan grid, 0 = one CTA per SM
  int scan_split = 0;    // CADV_SCAN_SPLIT: chunks per scan warp (0 = default 4)
  // registered trace (device pointers)
  bool loaded = false;
  cadv_trace_desc t{};
  uint64_t global_offset = 0;
  // R0 results (from the streaming pass of the last analysis)
  uint32_t max_cta = 0;               // of the current trace (shard; global after a multi-rank scan)
  uint64_t n_kind[4] = {0, 0, 0, 0};  // (unused)
  // B2 T_c table, kept across calls: entry = generation << 11 | T_c, so a new
  // call needs no clearing; capacity and the deferred-group buffer grow on demand
  uint32_t* tc_buf = nullptr;
  uint32_t tc_cap = 0, tc_gen = 0;
  uint64_t defer_cap = 0;
  // bookkeeping
  std::string err;
  float elapsed_ms = 0.f;
  uint32_t launches = 0;
  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  cadv::DevBuf buf[cadv::B_COUNT];
  void* host_pinned = nullptr;
  size_t host_pinned_bytes = 0;
  // small pinned staging for the per-call scalars read back mid-call (one
  // stream synchronisation for the scan scalars, kept count and CTA range)
  void* hstage = nullptr;  // 512 B: [0] kept records, [1] kept CTA-id max, +64: Scalars
  // per-kernel profiling (cadv_set_profiling)
  int profiling = 0;                  // 1: every launch, 2: k_scan<F> launches only
  bool prof_skip = false;             // the current launch is not profiled (mode 2)
  std::vector<cudaEvent_t> prof_ev;   // 2 per launch
  std::vector<const char*> prof_src;  // stringified launch expression
  std::vector<std::string> prof_name;
  std::vector<float> prof_ms;
  uint32_t nprof = 0;
  uint64_t counts[4] = {0, 0, 0, 0};  // cadv_last_count
  // max-dynamic-shared-memory opt-ins done on this context's device (the
  // attribute is per device context, so it is tracked per cadv_ctx):
  // bits 0-15 k_scan<F>, bit 16 k_rd_seg, 17 k_rd_tile, 18 k_merge_count_block
  uint32_t attr_set = 0;
  std::vector<void*> graveyard;  // replaced exported buffers (freed at cadv_destroy)
  int seg_ctas = 0;           // k_rd_seg CTAs per SM for seg_ctas_smem bytes of shared memory
  size_t seg_ctas_smem = 0;
  bool noncontig_any = false;
  // kept-record region capacity of a scan warp = max(chunk / 4, kcap_min)
  // records; a region that overflows raises kcap_min to its kept count + 1/8
  // (for the context's lifetime) and the call runs again
  uint64_t kcap_min = 0; // multi-rank: some rank's shard is not warp-contiguous (load_trace)
};

namespace cadv {

// Returns a device buffer of at least `bytes` (grown if needed).
cudaError_t ensure(cadv_ctx* c, BufId id, size_t bytes, void** out);
// Pinned host staging area for results.
cudaError_t ensure_host(cadv_ctx* c, size_t bytes, void** out);
Scalars* scalars(cadv_ctx* c);

// ---- launchers (each returns cudaSuccess or the launch error; they add the
// number of kernels they launched to c->launches)
// Stable (cta, tid/32) ordering of a non-warp-contiguous trace: fills `out`
// with device copies of every column in that order.
cudaError_t regroup_by_warp(cadv_ctx* c, cadv_trace_desc* out);
// Multi-rank, non-warp-contiguous shards: every (cta, warp32) stream moved
// to one rank and sorted there (collective); *out = this rank's records.
cudaError_t exchange_by_warp(cadv_ctx* c, cadv_trace_desc* out);

// ---- the fused streaming pass (scan.cu)
// F_OBJ: data-centric attribution (cadv_data_centric): the RD bin-0 counts
// of dropped duplicate loads and the MD groups go to the row of their object.
enum { F_RD = 1, F_MD = 2, F_BD = 4, F_OBJ = 8 };
struct ScanParams {
  cadv_trace_desc t;
  // reuse distance: run compression output
  uint32_t lbs_rd = 0;
  int cta_scope = 1;
  uint32_t* kout = nullptr;    // gapped per-warp regions (scan_geometry) of kcap records
  uint64_t* vout = nullptr;
  uint64_t kcap = 0;
  uint64_t* blkcnt = nullptr;  // kept records per scan warp chunk
  uint64_t* hist0 = nullptr;
  // memory divergence
  uint32_t lbs_md = 0, ws_md = 5;
  uint64_t* md_hist = nullptr;
  uint64_t* md_sites = nullptr;
  // branch divergence
  uint32_t ws_bd = 5;
  uint32_t* tc = nullptr;
  uint32_t tc_cap = 0, tc_gen = 0;
  uint64_t defer_cap = 0;
  uint64_t* bd_tot = nullptr;
  uint64_t* bd_sites = nullptr;
  void* defer = nullptr;
  unsigned long long* ndefer = nullptr;
  uint32_t nsites = 0;
  uint64_t* site_flag = nullptr;
  // data objects (F_OBJ): line extents, rows of rd_nbins (RD) / 2 (W + 1) (MD) bins
  const uint64_t* obj_lo = nullptr;
  const uint64_t* obj_hi = nullptr;
  uint32_t nobj = 0;
  uint32_t rd_nbins = 0;
};
uint64_t scan_tiles(uint64_t n);
void scan_geometry(cadv_ctx* c, uint64_t n, uint64_t* grid, uint64_t* nchunks, uint64_t* chunk, uint64_t* nbig = nullptr,
                   uint64_t* chunk_s = nullptr);
cudaError_t launch_squeeze(cadv_ctx* c, const uint32_t* kin, const uint64_t* vin, uint32_t* kout, uint64_t* vout,
                           const uint64_t* cnt, const uint64_t* off, uint64_t nblocks, uint64_t chunk_cap);
cudaError_t launch_scan(cadv_ctx* c, int flags, const ScanParams& P);
cudaError_t launch_bd_resolve(cadv_ctx* c, const void* defer, const unsigned long long* m, uint64_t cap,
                              const uint32_t* tc, uint32_t tc_gen, uint32_t ws, uint64_t* bd_tot, uint64_t* bd_sites,
                              uint32_t nsites);

// ---- reuse distance around the scan (reuse.cu)
// R1 regroup by CTA through per-region CTA tables (regroup.cu; CTA scope on
// one rank): a region = one scan warp's kept records
constexpr uint32_t RG_MAX = 768;  // distinct CTAs per region (more: squeeze + radix sort)
// CTA segments (CTA scope, one rank): <= SEG_WARP_MAX kept records go to the
// segment kernel (one warp each), <= SEG_TILE_MAX to one tile each (k_rd_tile
// over a segment list, no cross-tile queries); any longer segment sends the
// whole call to the tiled CTA-major sequence (bounds, keys, cross-tile phase)
constexpr uint32_t SEG_WARP_MAX = 256, SEG_TILE_MAX = 4096;
struct RgState {
  uint32_t* pk = nullptr;    // [region][RG_MAX] CTA ids
  uint32_t* pn = nullptr;    // [region][RG_MAX] record counts, later output offsets
  uint32_t* np = nullptr;    // [region + 1] pairs per region
  uint32_t* poff = nullptr;  // [region + 1] exclusive scan of np (poff[nregions] = total)
  uint64_t nregions = 0;
};
cudaError_t rg_count(cadv_ctx* c, const uint32_t* key, const uint64_t* cnt, uint64_t nregions, uint64_t chunk,
                     RgState* st);
// seg (nullable, >= P entries): the output's CTA segments (start, length), unordered;
// seg_cm[0] = their number, seg_cm[1] = the longest (device)
cudaError_t rg_finish(cadv_ctx* c, const RgState& st, uint64_t P, int bits, const uint32_t* key,
                      const uint64_t* val, const uint64_t* cnt, uint64_t chunk, uint32_t* kout, uint64_t* vout,
                      uint2* seg, uint2* seg_long, unsigned int* seg_cm);

struct RdState {
  int cta_scope = 1;
  uint32_t* k0 = nullptr;   // final kept records (after the squeeze) / radix sort ping
  uint32_t* k1 = nullptr;   // scan output (gapped) / radix sort pong
  uint64_t* v0 = nullptr;
  uint64_t* v1 = nullptr;
  uint64_t* blkcnt = nullptr;  // [grid] kept per scan block, then [grid] offsets
  uint64_t grid = 0, chunk_cap = 0;
  bool rg = false;  // regroup through region tables (regroup.cu) instead of squeeze + radix sort
  RgState rgs;
};
// R1 compaction of the scan's per-warp regions (exclusive scan of the counts
// + squeeze), queued on the stream; the kept count and the kept CTA-id range
// arrive in c->hstage (words 0, 1) once the stream reaches them.
cudaError_t rd_compact(cadv_ctx* c, const RdState& st);
// workspace for the run-compression output of the scan
cudaError_t rd_begin(cadv_ctx* c, int scope, RdState* st);
// CTA regroup, tiles, cross-tile phase after the scan wrote the kept records
// obj (n = 0: off): d_hist holds (obj.n + 1) rows of nbins, one per object + unattributed
struct ObjTab;
cudaError_t rd_finish(cadv_ctx* c, const RdState& st, int log2bins, uint32_t nbins, uint64_t* d_hist,
                      uint64_t* d_stats, const ObjTab* obj = nullptr);

// ---- device-wide primitives (sort.cu)
// Stable LSD radix sort of (key, value) pairs on bits [bit_lo, bit_hi) of the
// key.  Ping-pongs between (k0,v0) and (k1,v1); returns 0 if the result is in
// (k0,v0), 1 if in (k1,v1).
template <typename K, typename V>
cudaError_t radix_sort_pairs(cadv_ctx* c, K* k0, V* v0, K* k1, V* v1, uint64_t n, int bit_lo, int bit_hi,
                             int* result_in);
// Exclusive scan of n u32 values in place (out may alias in); *d_total (nullable) = sum.
cudaError_t exclusive_scan_u32(cadv_ctx* c, const uint32_t* in, uint32_t* out, uint64_t n, uint32_t* d_total);
cudaError_t exclusive_scan_u64(cadv_ctx* c, const uint64_t* in, uint64_t* out, uint64_t n);

}  // namespace cadv

namespace cadv {
void prof_begin(cadv_ctx* c, const char* src);
void prof_end(cadv_ctx* c);
}  // namespace cadv

#define CADV_LAUNCH_N(c, name, ...)         \
  do {                                      \
    cadv::prof_begin((c), (name));          \
    __VA_ARGS__;                            \
    cadv::prof_end((c));                    \
    (c)->launches++;                        \
  } while (0)

#define CADV_LAUNCH(c, ...)                 \
  do {                                      \
    cadv::prof_begin((c), #__VA_ARGS__);    \
    __VA_ARGS__;                            \
    cadv::prof_end((c));                    \
    (c)->launches++;                        \
  } while (0)
