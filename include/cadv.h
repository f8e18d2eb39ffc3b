/*
 * cadv.h — C ABI of libcadv, the B200 (sm_100a) analysis library for
 * CUDAAdvisor-style memory / basic-block traces.
 *
 * Paper: Shen, Song, Li, Liu, "CUDAAdvisor: LLVM-Based Runtime Profiling for
 * Modern GPUs", CGO'18.  "P:Lnnn" = line nnn of /root/reference/PAPER.md.
 *
 * The library analyses a trace that is already resident in GPU memory (or is
 * copied there by cadv_load_trace) and returns small integer histograms:
 *   - cadv_reuse_histogram   reuse distance
 *   - cadv_mem_divergence    memory divergence
 *   - cadv_branch_divergence branch divergence (Table 3)
 * Every output is an integer and is bit-exact against the CPU oracle in
 * oracle/ (tests/).  All kernels are hand-written sm_100a CUDA; there is no
 * CPU fallback: without a usable device every call fails with CADV_ERR_CUDA.
 *
 * ---------------------------------------------------------------- trace
 * One record per instrumented lane event, structure of arrays (P:L235:
 * "Record() packs all the arguments along with CTA ID and thread ID into one
 * entry"; P:L345 the same for passBasicBlock()):
 *   addr[i]  u64  effective byte address of a load/store (ignored for BB)
 *   cta[i]   u32  linearised CTA id; unique per kernel instance in the trace
 *   tid[i]   u16  linearised thread id inside the CTA, < 1024
 *   site[i]  u32  static instruction id (load/store) or basic-block id
 *   winst[i] u32  dynamic warp-instruction number of the record's warp:
 *                 per (cta, tid/32) and per family (memory vs BB), shared by
 *                 the lanes of one warp-level instruction instance and
 *                 non-decreasing in trace order (reading R9)
 *   meta[i]  u8   bits 0-1 kind (0 load, 1 store, 2 basic block),
 *                 bits 2-4 log2(access bytes) (0..4 = 1..16 B), bits 5-7 zero
 * Trace order is the order in which the instrumentation appended records.
 * Pointers must be naturally aligned for their element type.
 *
 * Per-record validity (checked by every analysis over the columns it reads,
 * violation -> CADV_ERR_BAD_TRACE, first offending index in cadv_last_error):
 *   kind <= 2; meta bits 5-7 zero; memory records: log2 bytes <= 4,
 *   addr % bytes == 0, addr < 2^58; tid < 1024 (divergence analyses).
 * Group validity (divergence analyses): a group (cta, tid/W, winst, family)
 *   holds at most one record per lane.  With warp_contiguous = 1 the caller
 *   also promises that the records of one (cta, tid/32, winst, family) form
 *   one contiguous run of at most 32 records; longer runs -> BAD_TRACE.
 *
 * ---------------------------------------------------------------- conventions
 * Ownership: the context owns all device workspace.  Device trace pointers
 *   passed with on_device = 1 are borrowed and must stay valid until the next
 *   cadv_load_trace or cadv_destroy; host pointers (on_device = 0) are copied
 *   to the device inside cadv_load_trace.  Output arrays are caller-owned
 *   HOST memory and are written only when the call returns CADV_OK.
 * Streams: all work of a context runs on the CUDA stream given to
 *   cadv_create (NULL = legacy default stream).  Every analysis call is
 *   synchronous: it returns after the host outputs are filled.
 * Threads: calls on one context must not run concurrently.
 * Multi-GPU: one context per rank.  With nranks > 1 every rank calls every
 *   function with identical parameters on its own position-range shard of
 *   the trace and receives the identical global result (DESIGN.md
 *   "Multi-GPU").
 * Errors: functions return a cadv_status; details via cadv_last_error().
 * Environment (testing only): CADV_SCAN_CTAS=n, read by cadv_create, caps
 *   the streaming pass at n CTAs so that each warp's contiguous chunk spans
 *   many 256-record steps even for small traces; results do not change.
 */
#ifndef CADV_H
#define CADV_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define CADV_API __attribute__((visibility("default")))

typedef struct cadv_ctx cadv_ctx; /* opaque; one per GPU / rank */

typedef enum {
  CADV_OK = 0,
  CADV_ERR_INVALID_ARG = 1, /* bad parameter (line size, warp size, nbins, nsites, NULL) */
  CADV_ERR_BAD_TRACE = 2,   /* a record violates the trace format above */
  CADV_ERR_NO_TRACE = 3,    /* analysis called before cadv_load_trace */
  CADV_ERR_OOM = 4,         /* device workspace allocation failed */
  CADV_ERR_CUDA = 5,        /* CUDA runtime error / no usable sm_100 device */
  CADV_ERR_NCCL = 6,        /* multi-GPU communication failed */
  CADV_ERR_UNSUPPORTED = 7  /* a limit of this implementation (see message) */
} cadv_status;

enum { CADV_KIND_LOAD = 0, CADV_KIND_STORE = 1, CADV_KIND_BB = 2 };
enum { CADV_SCOPE_CTA = 0, CADV_SCOPE_KERNEL = 1 };
enum { CADV_BINS_LINEAR = 0, CADV_BINS_LOG2 = 1 };

typedef struct {
  const uint64_t *addr;
  const uint32_t *cta;
  const uint16_t *tid;
  const uint32_t *site;
  const uint32_t *winst;
  const uint8_t *meta;
  uint64_t n;          /* records in this shard; n < 2^32 */
  int on_device;       /* 1: device pointers (borrowed); 0: host pointers (copied) */
  int warp_contiguous; /* 1: every warp-level group is one contiguous run (see above) */
} cadv_trace_desc;

typedef struct {
  uint64_t accesses;  /* memory records analysed = sum of the histogram */
  uint64_t inf;       /* accesses with no reuse (∞ bin) */
  uint64_t streaming; /* accesses to elements "never reused by the same CTA" */
  uint64_t overflow;  /* finite distances beyond the last exact bin */
  uint64_t finite_sum; /* sum of all finite distances (exact, overflow included): the
                          average reuse distance of Eq. (1), is
                          finite_sum / (accesses - inf) */
} cadv_reuse_stats;

typedef struct { uint64_t groups, sum_deg; } cadv_site_mem;                 /* per memory site */
typedef struct { uint64_t exec, divergent, threads; } cadv_site_branch;     /* per BB site */

/* Creates a context on `device` (must be an sm_100 GPU).  `cuda_stream` is a
 * cudaStream_t (NULL = default stream).  nccl_unique_id: NULL for one GPU, or
 * the 128-byte ncclUniqueId shared by all ranks (rank in [0, nranks), one
 * process per GPU; cadv_create is then collective).  libnccl.so.2 is opened
 * at run time (the copy the process already loaded, else the default search
 * path or $CADV_NCCL_LIB); CADV_ERR_NCCL if that or ncclCommInitRank fails.
 * A non-NULL id with nranks = 1 builds a one-rank communicator that runs the
 * multi-rank code path (exchange included) against itself. */
CADV_API cadv_status cadv_create(cadv_ctx **out, int device, void *cuda_stream,
                                 const void *nccl_unique_id, int rank, int nranks);

/* Writes a fresh 128-byte ncclUniqueId to out128 (call on rank 0, broadcast
 * it to the other ranks, e.g. with torch.distributed, before cadv_create). */
CADV_API cadv_status cadv_nccl_unique_id(void *out128);

/* Multi-rank context over the library's OWN collectives (no NCCL): every
 * collective is one kernel that reads the peers' staged device buffers
 * through CUDA IPC mappings (NVLink / NVSwitch between GPUs; local HBM when
 * ranks share a GPU), with a host TCP bootstrap for the IPC handles,
 * offsets and barriers: bootstrap_addr = "a.b.c.d:port" of rank 0 (every
 * rank passes the same string; rank 0 listens there).  One process per rank;
 * collective like cadv_create.  CADV_ERR_NCCL if the bootstrap fails within
 * 120 s. */
CADV_API cadv_status cadv_create_peer(cadv_ctx **out, int device, void *cuda_stream, const char *bootstrap_addr,
                                      int rank, int nranks);

/* Host-only check of the peer backend's TCP bootstrap (no GPU needed):
 * allgathers `bytes` bytes from every rank into out[nranks * bytes] and
 * returns 0 on success. */
CADV_API int cadv_bootstrap_selftest(const char *bootstrap_addr, int rank, int nranks, const void *in, void *out,
                                     uint64_t bytes);

/* In-process multi-rank contexts for testing on one GPU: a group of nranks
 * ranks that exchange data through host staging instead of NCCL.  Each rank
 * is a thread of the calling process holding its own context (created with
 * cadv_create_loopback(.., group, rank)); every collective call blocks until
 * all ranks of the group made it.  The group must outlive its contexts. */
CADV_API void *cadv_loopback_group_create(int nranks);
CADV_API cadv_status cadv_loopback_group_destroy(void *group);
CADV_API cadv_status cadv_create_loopback(cadv_ctx **out, int device, void *cuda_stream, void *group, int rank);

/* Registers the trace (or this rank's shard of it).  global_offset = trace
 * position of this shard's first record (0 for one GPU).  Host columns are
 * copied to the device here; device columns are only registered.  R0 (record
 * validation, CTA-id range) runs inside each analysis' streaming pass; each
 * analysis validates the columns it reads.
 * Multi-rank: shards are consecutive position ranges in rank order (rank r's
 * records precede rank r+1's in the trace; empty shards allowed).  The call
 * is collective (global CTA-id range; shard-edge group keys).  Divergence
 * analyses then need warp_contiguous shards whose boundaries do not split a
 * warp-level group (else CADV_ERR_UNSUPPORTED / CADV_ERR_BAD_TRACE); reuse
 * distance accepts any position split. */
CADV_API cadv_status cadv_load_trace(cadv_ctx *ctx, const cadv_trace_desc *desc, uint64_t global_offset);

/* Reuse-distance histogram over the load/store records (number of
 * distinct elements accessed between two consecutive uses of the same
 * element; a store starts a new element A').
 *   line_bytes: power of two in [1, 4096]; 1 = memory-element model,
 *               >1 = cache-line model (element = addr / line_bytes)
 *   scope:      CADV_SCOPE_CTA (per CTA after regrouping) or
 *               CADV_SCOPE_KERNEL (whole trace as one sequence)
 *   binning:    LINEAR: hist[d] for d <= nbins-3, hist[nbins-2] = d >= nbins-2
 *               LOG2:   hist[0] = {0}, hist[k] = [2^(k-1), 2^k - 1] for
 *                       1 <= k <= nbins-3, hist[nbins-2] = d >= 2^(nbins-3)
 *               both:   hist[nbins-1] = ∞ (no previous use of the element)
 *   hist[nbins] (nbins >= 3), stats (nullable): host outputs. */
CADV_API cadv_status cadv_reuse_histogram(cadv_ctx *ctx, uint32_t line_bytes, int scope, int binning,
                                          uint64_t *hist, uint32_t nbins, cadv_reuse_stats *stats);

/* Memory divergence ("the number of unique cache lines touched by
 * each instruction"): one count per dynamic warp-level load/store, i.e. per
 * group (cta, tid / warp_size, winst) of memory records.
 *   line_bytes: power of two in [1, 4096]; warp_size: power of two <= 32
 *   hist[2 * (warp_size + 1)]: row 0 loads, row 1 stores, column = number of
 *       unique lines (1..warp_size; column 0 stays 0)
 *   per_site[nsites] (nullable): per memory site {groups, sum of degrees};
 *       nsites must exceed every memory record's site id. */
CADV_API cadv_status cadv_mem_divergence(cadv_ctx *ctx, uint32_t line_bytes, uint32_t warp_size, uint64_t *hist,
                                         cadv_site_mem *per_site, uint32_t nsites);

/* Branch divergence (how many times a block executes, how many
 * threads execute it, how often it makes the warp diverge; Table 3).  One
 * execution per group (cta, tid / warp_size, winst) of BB records;
 * active = distinct lanes in the group; live = clamp(T_c - w*warp_size, 0,
 * warp_size) with T_c = 1 + max tid over CTA c's BB records; the execution
 * is divergent iff active < live (reading R12).
 *   per_site[nsites] (nullable): per BB site {exec, divergent, threads}
 *   totals[3]: {exec, divergent, threads} summed over all sites.
 * Limit: CTA ids must be < 2^28 (else CADV_ERR_UNSUPPORTED). */
CADV_API cadv_status cadv_branch_divergence(cadv_ctx *ctx, uint32_t warp_size, cadv_site_branch *per_site,
                                            uint32_t nsites, uint64_t totals[3]);

/* Parameters of cadv_analyze (one fused pass for several analyses). */
typedef struct {
  uint32_t rd_line_bytes; int rd_scope; int rd_binning; uint32_t rd_nbins;  /* as cadv_reuse_histogram */
  uint32_t md_line_bytes; uint32_t md_warp_size;                            /* as cadv_mem_divergence */
  uint32_t bd_warp_size;                                                    /* as cadv_branch_divergence */
  uint32_t nsites;                                                          /* for md_sites / bd_sites */
} cadv_analysis;

/* Runs every analysis whose output pointer is non-NULL (rd_hist: reuse;
 * md_hist: memory divergence; bd_totals: branch divergence) with ONE
 * streaming pass over the trace (the passes above share it), and writes the
 * same outputs as the individual calls with the same parameters would.
 * rd_stats, md_sites, bd_sites are optional as in the individual calls. */
CADV_API cadv_status cadv_analyze(cadv_ctx *ctx, const cadv_analysis *a, uint64_t *rd_hist,
                                  cadv_reuse_stats *rd_stats, uint64_t *md_hist, cadv_site_mem *md_sites,
                                  uint64_t *bd_totals, cadv_site_branch *bd_sites);

/* One data object (an allocation): bytes [base, base + bytes). */
typedef struct { uint64_t base, bytes; } cadv_object;

/* Data-centric attribution (the profiler "associates the memory
 * accesses in GPU kernels with the data allocation ... utilizes this
 * effective address to associate the memory access with data object"):
 * the reuse-distance and memory-divergence histograms split per data object
 * (reading R18).
 *   objs[nobj]: ascending, non-empty byte ranges; at line granularity
 *       (line_bytes) a line belongs to the object whose range it
 *       intersects, and no line may intersect two objects (else
 *       CADV_ERR_INVALID_ARG).  Lines in no object form the extra row nobj
 *       ("unattributed").  nobj = 0 is allowed (one row).  The table is
 *       copied; objs is not retained.
 *   rd_hist[(nobj + 1) * nbins] (nullable): row k = the reuse distances
 *       (as cadv_reuse_histogram with line_bytes, scope, binning, nbins) of
 *       the accesses whose line belongs to object k.
 *   md_hist[(nobj + 1) * 2 * (warp_size + 1)] (nullable): row k = the
 *       memory-divergence histogram (as cadv_mem_divergence) of the groups
 *       whose FIRST record's line belongs to object k.
 * At least one of rd_hist / md_hist must be non-NULL.  One streaming pass
 * computes both; multi-rank contexts return the global rows on every rank. */
CADV_API cadv_status cadv_data_centric(cadv_ctx *ctx, const cadv_object *objs, uint32_t nobj, uint32_t line_bytes,
                                       int scope, int binning, uint32_t nbins, uint32_t warp_size,
                                       uint64_t *rd_hist, uint64_t *md_hist);

/* Releases the context and all its device workspace. */
CADV_API cadv_status cadv_destroy(cadv_ctx *ctx);

/* Human-readable detail of the last non-OK status on ctx ("" if none). */
CADV_API const char *cadv_last_error(const cadv_ctx *ctx);

/* Device time (CUDA events on the context's stream) of the last successful
 * cadv_load_trace / analysis call, in milliseconds (0 for a load of device
 * columns: they are only registered, no device work runs). */
CADV_API float cadv_last_elapsed_ms(const cadv_ctx *ctx);

/* Number of kernels the last call launched (for bench.py's gpu_launches). */
CADV_API uint32_t cadv_last_launches(const cadv_ctx *ctx);

/* Per-kernel timing of the calls that follow: CUDA events are recorded on
 * the context's stream around every kernel launch (enable = 1) or around the
 * launches of the fused streaming pass k_scan<F> only (enable = 2, what a
 * timed loop needs for the dominant kernel's roofline without the host cost
 * of 2 event records per launch).  0 (default) turns it off. */
CADV_API cadv_status cadv_set_profiling(cadv_ctx *ctx, int enable);

/* Kernel names and device times (ms) of the last call's launches, in launch
 * order, when profiling was enabled.  Returns the number of launches and
 * fills at most `max` entries; names stay valid until the next call. */
CADV_API uint32_t cadv_last_kernel_times(const cadv_ctx *ctx, const char **names, float *ms, uint32_t max);

/* Work counters of the last cadv_reuse_histogram call (for roofline
 * accounting): which = 0 kept records after run compression, 1 cross-tile
 * entries, 2 cross-tile queries, 3 tiles.  0 for unknown `which`. */
CADV_API uint64_t cadv_last_count(const cadv_ctx *ctx, int which);

/* Library version string. */
CADV_API const char *cadv_version(void);

#ifdef __cplusplus
}
#endif
#endif /* CADV_H */
