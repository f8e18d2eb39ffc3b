// reuse.cu — reuse-distance histograms on B200.
//
// Definition (PAPER.md L248 + DESIGN.md readings R1-R8): per scope (CTA, or
// the whole kernel), walk the memory records in trace order; the element of
// an access is its line (addr / line_bytes) renamed by write epoch (a store
// starts a new element A'); RD(i) = number of distinct elements accessed
// strictly between the previous use P(i) of i's element and i; ∞ if none.
//
// Identity used on the device:
//   RD(i) = |window (P(i), i)| - #{ j < i : P(j) > P(i) }
// (the second term counts the window's records whose element is used again
// inside the window).  The pipeline:
//   R1 k_scan<F_RD>  (scan.cu) one streaming pass over (addr, cta, meta):
//                    validation, line keys, and run compression of
//                    raw-adjacent records of the same (scope, line): a load
//                    repeating the previous record's element has RD 0 and is
//                    dropped (counted in bin 0); consecutive stores are merged
//                    into one record of weight w (w distinct one-shot
//                    elements).  Kept records are written in trace order.
//   R1b              stable radix sort of kept records by CTA id (CTA scope).
//   R2/R3 k_rd_tile  fixed-capacity tiles of the CTA-major kept sequence
//                    (boundaries snapped to segment starts): in shared memory,
//                    a stable merge sort by line gives the local previous
//                    occurrence P, a counting merge sort of the local queries
//                    by P gives #{j < i : P(j) > P(i)} (merge-path,
//                    inversion counting), and R4 bins every local RD.
//   R3 (cross-tile)  only for segments cut by a tile boundary: one entry per
//                    (tile piece, line) carries first/last occurrence data;
//                    entries are sorted by (segment, line, tile) and linked;
//                    cross-tile queries get RD from prefix sums plus a global
//                    inversion count on the compacted cross-tile set.
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <vector>

#include "cadv_impl.h"
#include "common.cuh"

namespace cadv {
namespace {

// kept-record value layout
constexpr uint64_t LINE_MASK = (1ull << 58) - 1;
constexpr int VB_STORE = 58, VB_DUP = 59, VB_W = 60;  // weight - 1 in bits 60..63

constexpr uint64_t LB_VAL = (1ull << 62) - 1;  // look-back status value bits (scan.cu)

// ------------------------------------------------------------------ tile bounds
constexpr int TL_CAP = 4096;   // tile capacity (kept records)
constexpr int TL_NOM = 3584;   // nominal tile length
constexpr int TL_SNAP = 512;   // boundary snapped to a segment start within this window

__global__ void k_tile_bounds(const uint32_t* __restrict__ key, uint64_t K, uint32_t* __restrict__ bounds,
                              uint64_t ntiles) {
  const uint32_t lane = lane_id();
  uint64_t w = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t k = w; k <= ntiles; k += nw) {
    uint64_t b;
    if (k == 0) b = 0;
    else if (k == ntiles) b = K;
    else {
      uint64_t x0 = k * TL_NOM;
      b = x0;
      if (key) {
        uint64_t end = x0 + TL_SNAP < K ? x0 + TL_SNAP : K;
        for (uint64_t base = x0; base < end; base += 32) {
          uint64_t x = base + lane;
          bool ss = x < end && __ldg(key + x) != __ldg(key + x - 1);
          uint32_t bm = __ballot_sync(FULL, ss);
          if (bm) { b = base + __ffs(bm) - 1; break; }
        }
      }
    }
    if (lane == 0) bounds[k] = (uint32_t)b;
  }
}

// The CTA segments of a CTA-major kept sequence (multi-rank CTA scope, after
// the exchange): every position where the key changes starts one; its end by
// galloping + binary search; appended as k_rg_segments does (short list
// <= SEG_WARP_MAX, long list, cm[0] / cm[3] counts, cm[1] longest).
__global__ void k_key_segments(const uint32_t* __restrict__ key, uint64_t K, uint2* __restrict__ seg,
                               uint2* __restrict__ seg_long, unsigned int* __restrict__ cm) {
  const uint32_t lane = lane_id();
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  uint32_t mx = 0;
  for (uint64_t base = ((blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5) * 32; base < K; base += nw * 32) {
    const uint64_t s = base + lane;
    uint32_t len = 0;
    if (s < K && (s == 0 || key[s - 1] != key[s])) {
      const uint32_t c = key[s];
      uint64_t lo = s, step = 1;
      while (lo + step < K && key[lo + step] == c) { lo += step; step <<= 1; }
      uint64_t hi = lo + step < K ? lo + step : K;
      while (hi - lo > 1) {
        const uint64_t md = (lo + hi) >> 1;
        if (key[md] == c) lo = md;
        else hi = md;
      }
      len = (uint32_t)(lo + 1 - s);
    }
    mx = max(mx, len);
    const bool lg = len > SEG_WARP_MAX;
    const uint32_t bs = __ballot_sync(FULL, len && !lg), bl = __ballot_sync(FULL, lg);
    uint32_t os = 0, ol = 0;
    if (lane == 0) {
      if (bs) os = atomicAdd(&cm[0], (unsigned)__popc(bs));
      if (bl) ol = atomicAdd(&cm[3], (unsigned)__popc(bl));
    }
    os = __shfl_sync(FULL, os, 0);
    ol = __shfl_sync(FULL, ol, 0);
    if (len && !lg) seg[os + __popc(bs & lanemask_lt())] = make_uint2((uint32_t)s, len);
    if (lg) seg_long[ol + __popc(bl & lanemask_lt())] = make_uint2((uint32_t)s, len);
  }
  mx = __reduce_max_sync(FULL, mx);
  if (lane == 0 && mx) atomicMax(&cm[1], mx);
}

// ------------------------------------------------------------------ block merge sort (shared memory)
// Stable merge sort of N = NT*IPT items held in (ka, pa); result ends in the
// buffer returned (0 = a, 1 = b).  COUNT: for every item from the right run
// of a merge, cnt[idx(key)] += number of left-run items still unmerged =
// number of earlier items with a larger key (inversion count per item;
// keys are distinct when COUNT is used).
template <int NT, int IPT, typename K, typename P, bool COUNT>
__device__ int block_merge_sort(K* ka, P* pa, K* kb, P* pb, uint16_t* cnt, K pad_key) {
  constexpr int N = NT * IPT;
  const uint32_t t = threadIdx.x;
  // thread-local sort of IPT consecutive items (insertion sort, stable)
  {
    K k[IPT];
    P p[IPT];
#pragma unroll
    for (int j = 0; j < IPT; ++j) { k[j] = ka[t * IPT + j]; p[j] = pa[t * IPT + j]; }
    if (COUNT) {
#pragma unroll
      for (int j = 0; j < IPT; ++j) {
        uint32_t c = 0;
#pragma unroll
        for (int q = 0; q < j; ++q) c += k[q] > k[j] ? 1u : 0u;
        if (c && k[j] != pad_key) cnt[(uint32_t)(k[j] & 0xfffu)] += (uint16_t)c;
      }
    }
#pragma unroll
    for (int j = 1; j < IPT; ++j) {
      K kk = k[j];
      P pp = p[j];
      int q = j - 1;
      while (q >= 0 && k[q] > kk) { k[q + 1] = k[q]; p[q + 1] = p[q]; --q; }
      k[q + 1] = kk;
      p[q + 1] = pp;
    }
#pragma unroll
    for (int j = 0; j < IPT; ++j) { ka[t * IPT + j] = k[j]; pa[t * IPT + j] = p[j]; }
  }
  __syncthreads();
  K* ks = ka; P* ps = pa; K* kd = kb; P* pd = pb;
  int res = 0;
  for (int w = IPT; w < N; w <<= 1) {
    const uint32_t o = t * IPT;
    const uint32_t s0 = (o / (2 * w)) * (2 * w);
    const K* Ak = ks + s0;
    const K* Bk = ks + s0 + w;
    const P* Ap = ps + s0;
    const P* Bp = ps + s0 + w;
    const uint32_t d = o - s0;
    uint32_t lo = d > (uint32_t)w ? d - w : 0, hi = d < (uint32_t)w ? d : (uint32_t)w;
    while (lo < hi) {
      uint32_t mid = (lo + hi) >> 1;
      if (!(Bk[d - 1 - mid] < Ak[mid])) lo = mid + 1;
      else hi = mid;
    }
    uint32_t a = lo, b = d - lo;
#pragma unroll
    for (int j = 0; j < IPT; ++j) {
      bool takeA = a < (uint32_t)w && (b >= (uint32_t)w || !(Bk[b] < Ak[a]));
      if (takeA) {
        kd[o + j] = Ak[a];
        pd[o + j] = Ap[a];
        ++a;
      } else {
        K kk = Bk[b];
        kd[o + j] = kk;
        pd[o + j] = Bp[b];
        if (COUNT && kk != pad_key && a < (uint32_t)w) cnt[(uint32_t)(kk & 0xfffu)] += (uint16_t)(w - a);
        ++b;
      }
    }
    __syncthreads();
    K* tk = ks; ks = kd; kd = tk;
    P* tp = ps; ps = pd; pd = tp;
    res ^= 1;
  }
  return res;
}

// Bank-conflict-free placement of sort keys: thread t owns logical items
// 8t..8t+7; XOR-swizzling the low 3 index bits with bits of the 8-group index
// spreads a warp's same-j accesses over all banks (u32: bits 5..7, u64: bits
// 4..6, matching 32 resp. 16 lanes per shared-memory wavefront).
template <typename K>
__device__ __forceinline__ uint32_t swz(uint32_t i) {
  return sizeof(K) == 8 ? (i ^ ((i >> 4) & 7u)) : (i ^ ((i >> 5) & 7u));
}

// Compare-exchange for the base-case sorting network.
template <typename K>
__device__ __forceinline__ void cas(K& a, K& b) {
  K lo = a < b ? a : b, hi = a < b ? b : a;
  a = lo;
  b = hi;
}

// Merge sort of N = NT*8 DISTINCT keys in shared memory (no payload): base
// case = Batcher's 19-comparator network on 8 registers per thread, then
// log2(NT) merge-path levels.  COUNT: cnt[key & 0xfff] += number of earlier
// (left) keys greater than the key, i.e. the per-element inversion count.
template <int NT, typename K, bool COUNT>
__device__ int block_sort_keys(K* ka, K* kb, uint16_t* cnt, K pad_key, uint32_t N = NT * 8) {
  // N: power of two <= NT * 8; keys [0, N) are sorted (callers pad with pad_key)
  constexpr int IPT = 8;
  const uint32_t t = threadIdx.x;
  const bool act = t * IPT < N;
  if (act) {
    K k[IPT];
#pragma unroll
    for (int j = 0; j < IPT; ++j) k[j] = ka[swz<K>(t * IPT + j)];
    if (COUNT) {
#pragma unroll
      for (int j = 1; j < IPT; ++j) {
        uint32_t c = 0;
#pragma unroll
        for (int q = 0; q < j; ++q) c += k[q] > k[j] ? 1u : 0u;
        if (c && k[j] != pad_key) cnt[(uint32_t)(k[j] & 0xfffu)] += (uint16_t)c;
      }
    }
    cas(k[0], k[1]); cas(k[2], k[3]); cas(k[4], k[5]); cas(k[6], k[7]);
    cas(k[0], k[2]); cas(k[1], k[3]); cas(k[4], k[6]); cas(k[5], k[7]);
    cas(k[1], k[2]); cas(k[5], k[6]);
    cas(k[0], k[4]); cas(k[1], k[5]); cas(k[2], k[6]); cas(k[3], k[7]);
    cas(k[2], k[4]); cas(k[3], k[5]);
    cas(k[1], k[2]); cas(k[3], k[4]); cas(k[5], k[6]);
#pragma unroll
    for (int j = 0; j < IPT; ++j) ka[swz<K>(t * IPT + j)] = k[j];
  }
  // levels whose merges stay inside one warp's 32 * IPT items sync the warp only
  __syncwarp();
  K* ks = ka;
  K* kd = kb;
  int res = 0;
  for (uint32_t w = IPT; w < N; w <<= 1) {
    const uint32_t o = t * IPT;
    if (act) {
    const uint32_t s0 = (o / (2 * w)) * (2 * w);
    const uint32_t d = o - s0;
    auto A_ = [&](uint32_t i) { return ks[swz<K>(s0 + i)]; };
    auto B_ = [&](uint32_t i) { return ks[swz<K>(s0 + w + i)]; };
    uint32_t lo = d > w ? d - w : 0, hi = d < w ? d : w;
    while (lo < hi) {
      const uint32_t mid = (lo + hi) >> 1;
      if (A_(mid) < B_(d - 1 - mid)) lo = mid + 1;
      else hi = mid;
    }
    uint32_t a = lo, b = d - lo;
    K va = a < w ? A_(a) : pad_key, vb = b < w ? B_(b) : pad_key;
#pragma unroll
    for (int j = 0; j < IPT; ++j) {
      const bool takeA = a < w && (b >= w || va < vb);
      if (takeA) {
        kd[swz<K>(o + j)] = va;
        ++a;
        va = a < w ? A_(a) : pad_key;
      } else {
        kd[swz<K>(o + j)] = vb;
        if (COUNT && vb != pad_key && a < w) cnt[(uint32_t)(vb & 0xfffu)] += (uint16_t)(w - a);
        ++b;
        vb = b < w ? B_(b) : pad_key;
      }
    }
    }
    if (4 * w <= 32 * IPT) __syncwarp();
    else __syncthreads();
    K* tk = ks;
    ks = kd;
    kd = tk;
    res ^= 1;
  }
  if (N <= 16u * IPT) __syncthreads();  // the last level synced one warp only: callers read everything
  return res;
}

// ------------------------------------------------------------------ R2-R4 tile kernel
constexpr int TL_NT = 512;            // 8 keys per thread -> TL_CAP
constexpr int TL_LSEG = 16;           // segments per segment-list tile
constexpr int TL_SMEM_BINS = 1024;

// Shared memory of one tile (<= 113 KB so that two CTAs fit on an SM).
// key[2] holds the packed (line - min line) << 12 | position sort keys;
// after P is known, key[r] is reused for the query keys (2 x u32 arrays) and
// key[r^1] for the weighted prefix (u32) and the inversion counts (u16).
struct TileSmem {
  uint64_t key[2][TL_CAP];
  uint8_t sdw[TL_CAP];        // store | has_dup << 1 | weight << 2
  uint8_t ffl[TL_CAP];        // first_in_piece | last_in_piece << 1
  uint8_t fnx[TL_CAP];        // the record's element is used again later in the tile
  uint16_t sgs[TL_CAP];       // local start of the record's segment
  uint16_t pl[TL_CAP];        // local previous use + 1 (0 = none)
  uint16_t qx[TL_CAP];        // number of local queries before the record
  uint16_t es[TL_CAP];        // entry slot + 1 (0 = none); earlier: per-thread scan temp
  uint32_t hist[TL_SMEM_BINS];
  uint32_t ws[TL_NT / 32 + 1];
  uint32_t misc[8];
  unsigned long long lmin, lmax;
  // segment-list tiles: the tile's segments (global start, local start), <= TL_LSEG
  uint32_t lsb[TL_LSEG];
  uint32_t lsp[TL_LSEG + 1];
  uint32_t nls;
};
// the warp path of k_rd_tile keeps 256 u32 per warp in pl + qx
static_assert(offsetof(TileSmem, qx) == offsetof(TileSmem, pl) + sizeof(uint16_t) * TL_CAP, "pl, qx adjacent");
static_assert(sizeof(uint16_t) * TL_CAP * 2 >= 16 * 256 * 4 && TL_CAP >= 16 * 16 * 4, "warp path scratch");
// WIDE tiles (line range >= 2^52, practically never) keep lines and positions
// in separate arrays.
struct TileSmemWide {
  TileSmem base;
  uint16_t ps[2][TL_CAP];
};

// Where a rank's tiles sit in the global kept sequence (kernel scope over
// ranks; zeros / K for one GPU and for CTA scope): entry positions, tile ids
// and the continuation of the one segment across shard edges are global.
struct TilePos {
  uint64_t pos_base;   // global kept position of this rank's first kept record
  uint32_t tile_base;  // global index of this rank's first tile
  uint64_t k_glob;     // kept records of all ranks
};

struct EntryCols {
  uint32_t* seg;
  uint64_t* line;
  uint32_t* tile;
  uint32_t* f;      // global kept position of the piece's first use of the line
  uint32_t* fa;     // local queries of the piece before f
  uint32_t* fw;     // tile-local weighted position of f
  uint8_t* ff;      // bit0 load, bit1 no dup, bit2 local next, bit3 head piece, bit4 f == l
  uint32_t* l;      // global kept position of the piece's last use of the line
  uint32_t* lw;     // tile-local weighted position of l
  uint32_t* ld;     // local queries of the piece whose previous use lies after l
  uint8_t* lf;      // bit0 store, bit1 no dup, bits 2.. weight of l
};

// One CTA per tile [bounds[t], bounds[t+1]) of the CTA-major kept sequence.
// A "piece" is the part of one segment (CTA, or the whole trace for kernel
// scope) inside the tile; pieces cut by the tile's start (head) or end
// (tail) are "partial" and emit one entry per distinct line for the
// cross-tile phase.
// MODE (by the tile's line range R = max - min line):
//   0  R < 2^20: packed u32 sort keys (line - min) << 12 | position (every
//      tile of the paper-shaped workloads at 128 B lines);
//   1  R < 2^52: packed u64 keys;  2: lines and positions in separate arrays.
// The MODE 0 launch covers all tiles and lists the others (sc->count[4] /
// tile_list + ntiles, sc->count[3] / wide_list) for the MODE 1 / 2 launches.
// ------------------------------------------------------------------ R2-R4 segment kernel
// CTA scope on one rank with every CTA segment <= 256 kept records (every
// segment of the paper-shaped workloads at 128 B lines): the regroup knows
// the segments, so no tiles are needed.  Persistent warps take whole
// segments from a global counter and resolve each exactly like the tile
// kernel's warp path (rounds of 32 records: previous use from
// __match_any_sync or a per-warp line -> last-position hash table, weighted
// prefix, reused-position bitmap + bit-sliced compare), but with 64-bit line
// keys (no tile line range) and no block barrier until the final flush.
constexpr int SG_NT = 256, SG_W = SG_NT / 32;
// 384 hash slots per warp (load factor <= 2/3 at 256 distinct lines) keep the
// CTA under 40 KB of shared memory: 5 CTAs (40 warps) per SM.  The histogram
// is last so that the launch allocates only the bins it uses.
constexpr uint32_t SG_HS = 384;
struct SegSmem {
  unsigned long long hk[SG_W][SG_HS];  // line -> (slot) ; ~0 = empty
  uint16_t hp[SG_W][SG_HS];            // slot -> last position
  uint32_t wpi[SG_W][256];           // inclusive weighted prefix by position
  uint32_t rw[SG_W][16];             // reused-position bitmap [8] + word prefix counts [8]
  uint32_t hist[TL_SMEM_BINS];
};

// dynamic shared memory of k_rd_seg: the histogram only when it fits, then
// the object extents of a data-centric call with <= SG_OBJ_SMEM objects
constexpr uint32_t SG_OBJ_SMEM = 64;
// histogram words: one private copy per warp when they fit (no shared-memory
// atomics between warps on the hot bins), else one per CTA, else none (global)
__host__ __device__ constexpr uint64_t seg_hist_words(uint64_t hbins) {
  return hbins * SG_W <= TL_SMEM_BINS ? hbins * SG_W : (hbins <= TL_SMEM_BINS ? hbins : 0);
}
__host__ __device__ constexpr size_t seg_obj_offset(uint64_t hbins) {
  return (offsetof(SegSmem, hist) + 4 * seg_hist_words(hbins) + 15) & ~(size_t)15;
}
__host__ __device__ constexpr size_t seg_smem_bytes(uint64_t hbins, uint32_t nobj) {
  return nobj && nobj <= SG_OBJ_SMEM ? seg_obj_offset(hbins) + 16 * SG_OBJ_SMEM
                                     : offsetof(SegSmem, hist) + 4 * seg_hist_words(hbins);
}

// Shared-memory accesses by 32-bit shared-window address (computed once per
// warp): no generic-to-shared conversion (S2UR SR_CgaCtaId + ULEA) inside the
// round loop.
__device__ __forceinline__ uint64_t sh_ld64(uint32_t a) {
  uint64_t v;
  asm volatile("ld.shared.u64 %0, [%1];" : "=l"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t sh_ld32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t sh_ld16(uint32_t a) {
  uint16_t v;
  asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sh_st32(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void sh_st16(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u16 [%0], %1;" ::"r"(a), "h"((uint16_t)v) : "memory");
}
__device__ __forceinline__ void sh_add32(uint32_t a, uint32_t v) {
  asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void sh_or32(uint32_t a, uint32_t v) {
  asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ uint64_t sh_cas64(uint32_t a, uint64_t cmp, uint64_t v) {
  uint64_t o;
  asm volatile("atom.shared.cas.b64 %0, [%1], %2, %3;" : "=l"(o) : "r"(a), "l"(cmp), "l"(v) : "memory");
  return o;
}

// Inclusive warp scan step: x += the value o lanes below (when that lane
// exists), with the shuffle's in-range predicate guarding the add (no SEL).
__device__ __forceinline__ uint32_t scan_up_add(uint32_t x, uint32_t o) {
  asm("{\n\t.reg .pred p;\n\t.reg .b32 y;\n\t"
      "shfl.sync.up.b32 y|p, %0, %1, 0, 0xffffffff;\n\t"
      "@p add.u32 %0, %0, y;\n\t}"
      : "+r"(x)
      : "r"(o));
  return x;
}

// OBJ: data-centric rows (O.n > 0); the reuse-only instance carries none of it.
template <bool OBJ>
__global__ void __launch_bounds__(SG_NT, 5) k_rd_seg(const uint64_t* __restrict__ val, const uint2* __restrict__ seg,
                                                     const unsigned int* __restrict__ seg_cm, unsigned int* next,
                                                     int log2bins, uint32_t nbins, uint64_t* __restrict__ g_hist,
                                                     uint64_t* __restrict__ g_stream, ObjTab O) {
  extern __shared__ __align__(16) uint8_t sg_smem[];
  SegSmem& S = *reinterpret_cast<SegSmem*>(sg_smem);
  if (seg_cm[1] > SEG_TILE_MAX) return;  // the call takes the bounds-tiled path (queued before the host knew)
  const uint32_t tx = threadIdx.x, warp = tx >> 5, lane = lane_id();
  const uint32_t nobj = OBJ ? O.n : 0u;
  const uint32_t hbins = (nobj + 1) * nbins;
  const uint32_t hwords = (uint32_t)seg_hist_words(hbins);
  const bool smem_hist = hwords != 0, whist = hwords > hbins;
  for (uint32_t k = tx; k < hwords; k += SG_NT) S.hist[k] = 0;
  if (OBJ && nobj <= SG_OBJ_SMEM) {  // data-centric rows: the object extents in shared memory (seg_smem_bytes)
    uint64_t* so = reinterpret_cast<uint64_t*>(sg_smem + seg_obj_offset(hbins));
    for (uint32_t k = tx; k < nobj; k += SG_NT) { so[k] = O.lo[k]; so[SG_OBJ_SMEM + k] = O.hi[k]; }
    O.lo = so;
    O.hi = so + SG_OBJ_SMEM;
  }
  __syncthreads();
  const uint32_t nseg = seg_cm[0];
  const uint32_t HK = smem_u32(S.hk[warp]);   // u64 [SG_HS]
  const uint32_t HP = smem_u32(S.hp[warp]);   // u16 [SG_HS]
  const uint32_t WPI = smem_u32(S.wpi[warp]); // u32 [256]
  const uint32_t RW = smem_u32(S.rw[warp]);   // u32 [8] bitmap words, then [8] word prefix counts
  const uint32_t CW8 = RW + 32;
  const uint32_t H = smem_u32(S.hist) + (whist ? 4 * warp * hbins : 0u);
  uint32_t stream = 0, ninf = 0;  // ninf: the infinity bin (reuse-only instance) counted in a register
  unsigned long long rdsum = 0;
  // The next segment is claimed (and its descriptor and first round loaded)
  // while the current one is resolved; round r + 1's records are loaded at
  // the top of round r.  Segments are independent, so the claim order does
  // not matter.
  uint32_t sg = __shfl_sync(FULL, lane == 0 ? atomicAdd(next, 1u) : 0u, 0);
  uint2 sd = sg < nseg ? seg[sg] : make_uint2(0u, 0u);
  uint64_t vnext = lane < sd.y ? __ldg(val + sd.x + lane) : 0ull;
  while (sg < nseg) {
    const uint64_t* const vs = val + sd.x + lane;
    const uint32_t n = sd.y;  // <= SEG_WARP_MAX (k_rg_segments lists longer ones apart)
    const uint32_t sg_n = __shfl_sync(FULL, lane == 0 ? atomicAdd(next, 1u) : 0u, 0);
    const uint2 sd_n = sg_n < nseg ? seg[sg_n] : make_uint2(0u, 0u);
    for (uint32_t k = lane; k < SG_HS; k += 32)
      asm volatile("st.shared.u64 [%0], %1;" ::"r"(HK + 8 * k), "l"(~0ull) : "memory");
    if (lane < 16) sh_st32(RW + 4 * lane, 0u);
    __syncwarp();
    uint32_t wb = 0, rtot = 0;          // running weight, reused positions (warp-uniform)
    uint32_t qbits = 0, hbits = 0;      // this lane's positions 32 r + lane: query / has-dup flags
    for (uint32_t r = 0; 32 * r < n; ++r) {
      const uint32_t i = 32 * r + lane;
      const bool valid = i < n;
      const uint64_t v = vnext;
      vnext = (i + 32 < n) ? __ldg(vs + 32 * (r + 1)) : 0ull;
      const unsigned long long line = valid ? (v & LINE_MASK) : ~0ull;
      const bool st = (v >> VB_STORE) & 1u, hd = (v >> VB_DUP) & 1u;
      const uint32_t w = valid ? (uint32_t)(v >> VB_W) + 1u : 0u;
      // previous use of the line: an earlier lane of this round, else the table
      // lines that share their high half (every lane, the usual case): a 32-bit
      // match, much cheaper than the 64-bit one (k_rd_seg 0.49 -> 0.37 ms on C4)
      const uint32_t lhi = (uint32_t)(line >> 32);
      const uint32_t peers = __all_sync(FULL, lhi == __shfl_sync(FULL, lhi, 0))
                                 ? __match_any_sync(FULL, (uint32_t)line) : __match_any_sync(FULL, line);
      // weighted prefix (inclusive) by position (independent of the match: overlaps its latency)
      uint32_t xw = w;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) xw = scan_up_add(xw, o);
      const uint32_t lower = peers & lanemask_lt();
      int32_t pp = -1;
      uint32_t hs = 0;  // the group's first lane: the line's slot (bit 16: present) or the first empty slot
      if (valid) {
        if (lower) {
          pp = (int32_t)(32 * r + 31 - __clz(lower));
        } else {
          uint32_t h = __umulhi((uint32_t)((line * 0x9E3779B97F4A7C15ull) >> 32), SG_HS);
          while (true) {
            const unsigned long long k = sh_ld64(HK + 8 * h);
            if (k == line) { pp = (int32_t)sh_ld16(HP + 2 * h); hs = h | 0x10000u; break; }
            if (k == ~0ull) { hs = h; break; }
            h = h + 1 == SG_HS ? 0u : h + 1;
          }
        }
      }
      hs = __shfl_sync(FULL, hs, __ffs(peers) - 1);
      const bool q = valid && !st && pp >= 0;  // a local query: RD = window - reused in window
      const int32_t P = q ? pp : -1;
      __syncwarp();
      if (valid && (peers >> lane) == 1u) {  // the line's last lane in this round records it
        uint32_t h = hs & 0xffffu;
        if (!(hs >> 16)) {
          // new line: claim a slot from the first empty one the probe saw (lanes
          // of other new lines insert concurrently, so with CAS)
          while (true) {
            const unsigned long long k = sh_cas64(HK + 8 * h, ~0ull, line);
            if (k == ~0ull || k == line) break;
            h = h + 1 == SG_HS ? 0u : h + 1;
          }
        }
        sh_st16(HP + 2 * h, i);
      }
      if (valid) sh_st32(WPI + 4 * i, wb + xw);
      // reused positions inside the window (P, i): earlier rounds (bitmap R) ...
      uint32_t cnt = 0;
      if (q && (uint32_t)P < 32 * r) {
        const uint32_t pw = (uint32_t)P >> 5, pb = (uint32_t)P & 31u;
        cnt = rtot - (sh_ld32(CW8 + 4 * pw) + __popc(sh_ld32(RW + 4 * pw) & (0xffffffffu >> (31u - pb))));
      }
      // ... and this round: lanes s < lane with P(s) > P (bit-sliced compare)
      // (MSB first over the bits positions of this round can have: P < 32 (r + 1))
      const uint32_t qm = __ballot_sync(FULL, q);
      const uint32_t pv = q ? (uint32_t)P : 0u;
      uint32_t gt = 0, eq = FULL;
  // one ballot and three predicated logic ops per bit: with my bit 0 the lanes
  // still equal above that have it set are greater; eq keeps the lanes whose
  // bit equals mine
#define SG_CMP_BIT(kb)                                                       \
  asm("{\n\t.reg .pred p;\n\t.reg .b32 b, t;\n\t"                          \
      "and.b32 t, %2, %3;\n\tsetp.ne.u32 p, t, 0;\n\t"                        \
      "vote.sync.ballot.b32 b, p, 0xffffffff;\n\t"                            \
      "@!p lop3.b32 %1, %1, %0, b, 0xF8;\n\t"                                 \
      "@p and.b32 %0, %0, b;\n\t@!p lop3.b32 %0, %0, b, 0, 0x30;\n\t}"          \
      : "+r"(eq), "+r"(gt)                                                   \
      : "r"(pv), "n"(1u << (kb)));
      switch (r) {
        default: SG_CMP_BIT(7);  // fall through
        case 2: case 3: SG_CMP_BIT(6);  // fall through
        case 1: SG_CMP_BIT(5);  // fall through
        case 0: SG_CMP_BIT(4); SG_CMP_BIT(3); SG_CMP_BIT(2); SG_CMP_BIT(1); SG_CMP_BIT(0);
      }
#undef SG_CMP_BIT
      cnt += __popc(gt & qm & lanemask_lt());
      __syncwarp();
      // R4
      if (valid) {
        if (q) {
          const uint32_t rd = (wb + xw - w) - sh_ld32(WPI + 4 * (uint32_t)P) - cnt;
          uint32_t bin = rd_bin(rd, log2bins, nbins);
          rdsum += rd;
          if (OBJ) bin += obj_row(O, line) * nbins;
          if (smem_hist) sh_add32(H + 4 * bin, 1u);
          else atomicAdd((unsigned long long*)&g_hist[bin], 1ull);
        } else {
          const uint32_t cntb = st ? w : 1u;
          if (!OBJ) {
            ninf += cntb;
          } else {
            const uint32_t bin = nbins - 1 + obj_row(O, line) * nbins;
            if (smem_hist) sh_add32(H + 4 * bin, cntb);
            else atomicAdd((unsigned long long*)&g_hist[bin], (unsigned long long)cntb);
          }
        }
        if (st) stream += w - 1;  // all but the last of merged stores are one-shot elements
      }
      qbits |= (uint32_t)q << r;
      hbits |= (uint32_t)hd << r;
      // R += { P(s) } of this round's queries; word prefix counts
      if (q) sh_or32(RW + 4 * ((uint32_t)P >> 5), 1u << (P & 31));
      __syncwarp();
      const uint32_t nr = lane < 8 ? sh_ld32(RW + 4 * lane) : 0u;
      uint32_t pc = __popc(nr), xc = pc;
#pragma unroll
      for (int o = 1; o < 8; o <<= 1) xc = scan_up_add(xc, o);
      if (lane < 8) sh_st32(CW8 + 4 * lane, xc - pc);
      rtot += __popc(qm);  // every position is reused at most once: the round's P are new bits
      wb += __shfl_sync(FULL, xw, 31);
      __syncwarp();
    }
    // streaming: positions whose element is never used again (not reused, no dup);
    // bit r of this lane's masks = position 32 r + lane
    {
      uint32_t reused = 0;
#pragma unroll
      for (int k = 0; k < 8; ++k) reused |= ((sh_ld32(RW + 4 * k) >> lane) & 1u) << k;
      const uint32_t nr = n > lane ? (n - lane + 31) / 32 : 0u;  // this lane's positions
      stream += __popc(((1u << nr) - 1u) & ~(qbits | hbits | reused));
    }
    __syncwarp();
    sg = sg_n;
    sd = sd_n;
    vnext = lane < sd.y ? __ldg(val + sd.x + lane) : 0ull;
  }
  stream = __reduce_add_sync(FULL, stream);
  if (lane == 0 && stream) atomicAdd((unsigned long long*)g_stream, (unsigned long long)stream);
#pragma unroll
  for (int o = 16; o; o >>= 1) rdsum += __shfl_xor_sync(FULL, rdsum, o);
  if (lane == 0 && rdsum) atomicAdd((unsigned long long*)g_stream + 1, rdsum);
  if (!OBJ) {
    ninf = __reduce_add_sync(FULL, ninf);
    if (lane == 0 && ninf) {
      if (smem_hist) sh_add32(H + 4 * (nbins - 1), ninf);
      else atomicAdd((unsigned long long*)&g_hist[nbins - 1], (unsigned long long)ninf);
    }
  }
  __syncthreads();
  if (smem_hist)
    for (uint32_t k = tx; k < hbins; k += SG_NT) {
      uint32_t v = S.hist[k];
      if (whist)
        for (int x = 1; x < SG_W; ++x) v += S.hist[x * hbins + k];
      if (v) atomicAdd((unsigned long long*)&g_hist[k], (unsigned long long)v);
    }
}

template <int MODE>
__global__ void __launch_bounds__(TL_NT, MODE == 2 ? 1 : 2)
    k_rd_tile(const uint32_t* __restrict__ key, const uint64_t* __restrict__ val, uint64_t K,
              const uint32_t* __restrict__ bounds, uint32_t ntiles, int log2bins, uint32_t nbins,
              uint64_t* __restrict__ g_hist, uint64_t* __restrict__ g_stream, uint32_t* __restrict__ tile_w,
              uint32_t* __restrict__ tile_q, EntryCols E, Scalars* sc, uint32_t* wide_list, ObjTab O,
              TilePos TP, const uint2* __restrict__ tl, const uint32_t* __restrict__ tofs) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  TileSmem& S = *reinterpret_cast<TileSmem*>(smem_raw);
  const uint32_t tx = threadIdx.x;
  constexpr bool WIDE = MODE == 2;
  const uint32_t tile = MODE == 0 ? blockIdx.x : MODE == 1 ? wide_list[ntiles + 2 + blockIdx.x] : wide_list[blockIdx.x];
  // tl (segment list, CTA scope on one rank): the tile is whole segments
  // tl[tofs[tile] .. tofs[tile + 1]) (one segment when tofs is null), placed
  // one after the other; gpos maps a tile position to its kept record
  uint64_t b = 0, e = 0;
  if (!tl) {
    b = bounds[tile];
    e = bounds[tile + 1];
  } else {
    if (tx == 0) {
      const uint32_t j0 = tofs ? tofs[tile] : tile, j1 = tofs ? tofs[tile + 1] : tile + 1;
      uint32_t acc = 0;
      for (uint32_t j = j0; j < j1; ++j) {
        const uint2 d = tl[j];
        S.lsb[j - j0] = d.x;
        S.lsp[j - j0] = acc;
        acc += d.y;
      }
      S.lsp[j1 - j0] = acc;
      S.nls = j1 - j0;
    }
    __syncthreads();
    e = S.lsp[S.nls];
  }
  const uint32_t m = (uint32_t)(e - b);
  auto lseg = [&](uint32_t x) {  // the list segment holding tile position x
    uint32_t lo = 0, hi = S.nls - 1;
    while (lo < hi) {
      const uint32_t md = (lo + hi + 1) >> 1;
      if (S.lsp[md] <= x) lo = md;
      else hi = md - 1;
    }
    return lo;
  };
  auto gpos = [&](uint32_t x) -> uint64_t {
    if (!tl) return b + x;
    const uint32_t j = lseg(x);
    return (uint64_t)S.lsb[j] + (x - S.lsp[j]);
  };
  // data-centric attribution: one row of nbins per object + 1 (O.n = 0: one row)
  const uint32_t hbins = (O.n + 1) * nbins;
  const bool smem_hist = hbins <= TL_SMEM_BINS;
  // ---- line range of the tile (packed keys need < 2^52)
  if (tx == 0) {
    S.lmin = ~0ull;
    S.lmax = 0;
    S.misc[2] = m;
    S.misc[3] = S.misc[4] = S.misc[5] = S.misc[6] = 0;  // warp path: longest segment, weight / query totals, queue
  }
  __syncthreads();
  {
    uint64_t mn = ~0ull, mx = 0;
    for (uint32_t x = tx; x < m; x += TL_NT) {
      uint64_t l = __ldg(val + gpos(x)) & LINE_MASK;
      mn = l < mn ? l : mn;
      mx = l > mx ? l : mx;
    }
    for (int o = 16; o; o >>= 1) {
      uint64_t a2 = __shfl_xor_sync(FULL, mn, o), z2 = __shfl_xor_sync(FULL, mx, o);
      mn = a2 < mn ? a2 : mn;
      mx = z2 > mx ? z2 : mx;
    }
    if (lane_id() == 0 && m) {
      atomicMin(&S.lmin, (unsigned long long)mn);
      atomicMax(&S.lmax, (unsigned long long)mx);
    }
  }
  __syncthreads();
  const uint64_t lmin = m ? S.lmin : 0;
  if (MODE == 0 && m && ((S.lmax - lmin) >> 20)) {
    // handled by the MODE 1 / MODE 2 instances
    if (tx == 0) {
      if ((S.lmax - lmin) >> 52) {
        const unsigned long long k = atomicAdd((unsigned long long*)&sc->count[3], 1ull);
        wide_list[k] = tile;
      } else {
        const unsigned long long k = atomicAdd((unsigned long long*)&sc->count[4], 1ull);
        wide_list[ntiles + 2 + k] = tile;
      }
    }
    return;
  }
  if (smem_hist)
    for (uint32_t k = tx; k < hbins; k += TL_NT) S.hist[k] = 0;
  uint32_t* const K32a = reinterpret_cast<uint32_t*>(S.key[0]);
  uint32_t* const K32b = reinterpret_cast<uint32_t*>(S.key[1]);
  // ---- segment starts (blocked: thread owns 8 consecutive positions)
  constexpr int IPT = TL_CAP / TL_NT;
  uint32_t ssm = 0, ss_local = 0;
#pragma unroll
  for (int j = 0; j < IPT; ++j) {
    uint32_t x = tx * IPT + j;
    uint64_t gx = b + x;
    bool sflag = x < m && (tl ? S.lsp[lseg(x)] == x : (TP.pos_base + gx == 0 || (key && __ldg(key + gx) != __ldg(key + gx - 1))));
    if (sflag) { ssm |= 1u << j; ss_local = x; }
  }
  uint32_t* tmax = reinterpret_cast<uint32_t*>(S.es);
  tmax[tx] = block_inclusive_max<TL_NT>(ss_local, S.ws);
  __syncthreads();
  {
    uint32_t cur = tx ? tmax[tx - 1] : 0u;
#pragma unroll
    for (int j = 0; j < IPT; ++j) {
      uint32_t x = tx * IPT + j;
      if ((ssm >> j) & 1u) {
        cur = x;
        if (x > 0) atomicMin(&S.misc[2], x);  // start of the tile's second segment
      }
      S.sgs[x] = (uint16_t)cur;
    }
  }
  // (kernel scope over ranks: the one segment continues across the shards' kept records)
  const bool head_cont = !tl && m > 0 && TP.pos_base + b > 0 && (!key || __ldg(key + b) == __ldg(key + b - 1));
  const bool tail_cont = !tl && m > 0 && TP.pos_base + e < TP.k_glob && (!key || __ldg(key + e) == __ldg(key + e - 1));
  __syncthreads();
  for (uint32_t x = tx; x < TL_CAP; x += TL_NT) S.es[x] = 0;
  // ---- warp path (MODE 0): the tile holds whole segments of <= 256 kept
  //      records each (every CTA of the paper-shaped workloads at 128 B
  //      lines): warp w resolves segments w, w + 16, ... alone with the same
  //      two sorts as below over <= 256 keys (<= 5 merge levels instead of 9,
  //      warp syncs only).  Segments cut by a tile boundary, longer segments
  //      and the wider key modes take the block path.
  if (MODE == 0 && !tl && !head_cont && !tail_cont && m) {
    uint32_t ml = 0;
#pragma unroll
    for (int j = 0; j < IPT; ++j) {
      const uint32_t x = tx * IPT + j;
      if (x < m) ml = max(ml, x - S.sgs[x] + 1u);
    }
    ml = __reduce_max_sync(FULL, ml);
    if (lane_id() == 0) atomicMax(&S.misc[3], ml);
    __syncthreads();
    if (S.misc[3] <= 256u) {
      uint32_t nseg;
      uint32_t so = block_exclusive_scan<TL_NT>(__popc(ssm), S.ws, &nseg);
#pragma unroll
      for (int j = 0; j < IPT; ++j)
        if ((ssm >> j) & 1u) S.es[so++] = (uint16_t)(tx * IPT + j);
      __syncthreads();
      uint32_t stream = 0, wt = 0, qt = 0;
      unsigned long long rdsum = 0;
      const uint32_t warp = tx >> 5, lane = lane_id();
      // warp-private scratch (arrays the block path would use): a line -> last
      // position hash table of 512 slots (key[0] / key[1]), the inclusive
      // weighted prefix by segment position (pl + qx), the "reused" position
      // bitmap R and its word prefix counts (ffl)
      uint32_t* const HK = reinterpret_cast<uint32_t*>(S.key) + warp * 1024;
      uint32_t* const HP = HK + 512;
      uint32_t* const WPI = reinterpret_cast<uint32_t*>(S.pl) + warp * 256;
      uint32_t* const RW = reinterpret_cast<uint32_t*>(S.ffl) + warp * 16;  // [8] bitmap words
      uint32_t* const CW8 = RW + 8;                                          // [8] set bits before each word
      // segments longest first would be ideal; a shared counter hands them out in order
      for (uint32_t sg = __shfl_sync(FULL, lane == 0 ? atomicAdd(&S.misc[6], 1u) : 0u, 0); sg < nseg;
           sg = __shfl_sync(FULL, lane == 0 ? atomicAdd(&S.misc[6], 1u) : 0u, 0)) {
        const uint32_t s0 = S.es[sg], n = (sg + 1 < nseg ? S.es[sg + 1] : m) - s0;
        for (uint32_t k = lane; k < 512; k += 32) HK[k] = 0xffffffffu;
        if (lane < 8) { RW[lane] = 0; CW8[lane] = 0; }
        __syncwarp();
        uint32_t wb = 0, qn = 0, rtot = 0;   // running weight, queries, reused positions (warp-uniform)
        uint32_t qbits = 0, hbits = 0;       // this lane's positions 32 r + lane: query / has-dup flags
        for (uint32_t r = 0; 32 * r < n; ++r) {
          const uint32_t i = 32 * r + lane;
          const bool valid = i < n;
          const uint64_t v = valid ? __ldg(val + b + s0 + i) : 0ull;
          const uint64_t lfull = v & LINE_MASK;
          const uint32_t line = valid ? (uint32_t)(lfull - lmin) : 0xffffffffu;  // MODE 0: < 2^20
          const bool st = (v >> VB_STORE) & 1u, hd = (v >> VB_DUP) & 1u;
          const uint32_t w = valid ? (uint32_t)(v >> VB_W) + 1u : 0u;
          // previous use of the line: an earlier lane of this round, else the table
          const uint32_t peers = __match_any_sync(FULL, line);
          const uint32_t lower = peers & lanemask_lt();
          int32_t pp = -1;
          if (valid) {
            if (lower) {
              pp = (int32_t)(32 * r + 31 - __clz(lower));
            } else {
              uint32_t h = (line * 0x9E3779B1u) >> 23;
              while (true) {
                const uint32_t k = HK[h];
                if (k == line) { pp = (int32_t)HP[h]; break; }
                if (k == 0xffffffffu) break;
                h = (h + 1) & 511u;
              }
            }
          }
          const bool q = valid && !st && pp >= 0;  // a local query: RD = window - reused in window
          const int32_t P = q ? pp : -1;
          __syncwarp();
          if (valid && (peers >> lane) == 1u) {  // the line's last lane in this round records it
            uint32_t h = (line * 0x9E3779B1u) >> 23;
            while (true) {  // lanes of other lines insert concurrently: claim slots with CAS
              const uint32_t k = atomicCAS(&HK[h], 0xffffffffu, line);
              if (k == 0xffffffffu || k == line) break;
              h = (h + 1) & 511u;
            }
            HP[h] = i;
          }
          // weighted prefix (inclusive) by position
          uint32_t xw = w;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(FULL, xw, o);
            if (lane >= (uint32_t)o) xw += y;
          }
          if (valid) WPI[i] = wb + xw;
          // reused positions inside the window (P, i): earlier rounds (bitmap R) ...
          uint32_t cnt = 0;
          if (q && (uint32_t)P < 32 * r) {
            const uint32_t pw = (uint32_t)P >> 5, pb = (uint32_t)P & 31u;
            cnt = rtot - (CW8[pw] + __popc(RW[pw] & (0xffffffffu >> (31u - pb))));
          }
          // ... and this round: lanes s < lane with P(s) > P (bit-sliced compare)
          const uint32_t qm = __ballot_sync(FULL, q);
          const uint32_t pv = q ? (uint32_t)P : 0u;
          uint32_t gt = 0, eq = FULL;
#pragma unroll
          for (int kb = 7; kb >= 0; --kb) {
            const uint32_t bk = __ballot_sync(FULL, (pv >> kb) & 1u);
            if ((pv >> kb) & 1u) eq &= bk;
            else { gt |= eq & bk; eq &= ~bk; }
          }
          cnt += __popc(gt & qm & lanemask_lt());
          __syncwarp();
          // R4
          if (valid) {
            uint32_t bin, cntb = 1;
            if (q) {
              const uint32_t rd = (wb + xw - w) - WPI[P] - cnt;
              bin = rd_bin(rd, log2bins, nbins);
              rdsum += rd;
            } else {
              bin = nbins - 1;
              if (st) cntb = w;
            }
            if (O.n) bin += obj_row(O, lfull) * nbins;
            if (smem_hist) atomicAdd(&S.hist[bin], cntb);
            else atomicAdd((unsigned long long*)&g_hist[bin], (unsigned long long)cntb);
            if (st) stream += w - 1;  // all but the last of merged stores are one-shot elements
          }
          qbits |= (uint32_t)q << r;
          hbits |= (uint32_t)hd << r;
          // R += { P(s) } of this round's queries (shared-memory atomics; every
          // lane finished reading R above); word prefix counts
          if (q) atomicOr(&RW[(uint32_t)P >> 5], 1u << (P & 31));
          __syncwarp();
          const uint32_t nr = lane < 8 ? RW[lane] : 0u;
          uint32_t pc = __popc(nr), xc = pc;
#pragma unroll
          for (int o = 1; o < 8; o <<= 1) {
            const uint32_t y = __shfl_up_sync(FULL, xc, o);
            if (lane >= (uint32_t)o) xc += y;
          }
          if (lane < 8) CW8[lane] = xc - pc;
          rtot = __shfl_sync(FULL, xc, 7);
          wb += __shfl_sync(FULL, xw, 31);
          qn += __popc(qm);
          __syncwarp();
        }
        // streaming: positions whose element is never used again (not reused, no dup)
        for (uint32_t r = 0; 32 * r < n; ++r) {
          const uint32_t i = 32 * r + lane;
          if (i < n && !((qbits >> r) & 1u) && !((hbits >> r) & 1u) && !((RW[i >> 5] >> (i & 31u)) & 1u)) stream += 1;
        }
        wt += wb;
        qt += qn;
        __syncwarp();
      }
      if (lane == 0) {
        atomicAdd(&S.misc[4], wt);
        atomicAdd(&S.misc[5], qt);
      }
      stream = __reduce_add_sync(FULL, stream);
      if (lane == 0 && stream) atomicAdd((unsigned long long*)g_stream, (unsigned long long)stream);
#pragma unroll
      for (int o = 16; o; o >>= 1) rdsum += __shfl_xor_sync(FULL, rdsum, o);
      if (lane == 0 && rdsum) atomicAdd((unsigned long long*)g_stream + 1, rdsum);
      __syncthreads();
      if (tx == 0) {
        tile_w[TP.tile_base + tile] = S.misc[4];
        tile_q[TP.tile_base + tile] = S.misc[5];
      }
      if (smem_hist)
        for (uint32_t k = tx; k < hbins; k += TL_NT)
          if (S.hist[k]) atomicAdd((unsigned long long*)&g_hist[k], (unsigned long long)S.hist[k]);
      return;
    }
  }
  // ---- block path: load (striped)
  uint16_t* PSW = WIDE ? reinterpret_cast<TileSmemWide*>(smem_raw)->ps[0] : nullptr;
  for (uint32_t x = tx; x < TL_CAP; x += TL_NT) {
    if (x < m) {
      uint64_t v = __ldg(val + gpos(x));
      uint64_t l = v & LINE_MASK;
      if (MODE == 0) K32a[swz<uint32_t>(x)] = (uint32_t)(((l - lmin) << 12) | x);
      else S.key[0][WIDE ? x : swz<uint64_t>(x)] = WIDE ? l : (((l - lmin) << 12) | x);
      uint32_t w = (uint32_t)(v >> VB_W) + 1u;
      S.sdw[x] = (uint8_t)(((v >> VB_STORE) & 1u) | (((v >> VB_DUP) & 1u) << 1) | (w << 2));
    } else {
      if (MODE == 0) K32a[swz<uint32_t>(x)] = 0xffffffffu;
      else S.key[0][WIDE ? x : swz<uint64_t>(x)] = ~0ull;
      S.sdw[x] = 0;
    }
    if (WIDE) PSW[x] = (uint16_t)x;
    S.fnx[x] = 0;
  }
  __syncthreads();
  const uint32_t lastseg = m ? S.sgs[m - 1] : 0u;
  const uint32_t second = S.misc[2];
  auto partial = [&](uint32_t x) {
    uint32_t sg = S.sgs[x];
    return (sg == 0 && head_cont) || (sg == lastseg && tail_cont);
  };
  // ---- sort by (line, position): runs of equal lines in position order
  int r;
  if (WIDE) {
    TileSmemWide& SW = *reinterpret_cast<TileSmemWide*>(smem_raw);
    r = block_merge_sort<TL_NT, IPT, uint64_t, uint16_t, false>(S.key[0], SW.ps[0], S.key[1], SW.ps[1], nullptr,
                                                                ~0ull);
  } else {
    // only the first N1 keys (m records + pads, a power of two) take part: a
    // short tile (one segment of the segment list) sorts fewer levels
    uint32_t N1 = 256;
    while (N1 < m) N1 <<= 1;
    if (MODE == 1) r = block_sort_keys<TL_NT, uint64_t, false>(S.key[0], S.key[1], nullptr, ~0ull, N1);
    else r = block_sort_keys<TL_NT, uint32_t, false>(K32a, K32b, nullptr, 0xffffffffu, N1);
  }
  const uint64_t* KS = S.key[r];
  const uint32_t* KS32 = r ? K32b : K32a;
  const uint16_t* PW = WIDE ? reinterpret_cast<TileSmemWide*>(smem_raw)->ps[r] : nullptr;
  auto POS = [&](uint32_t s_) -> uint32_t {
    return WIDE ? PW[s_] : MODE == 0 ? (KS32[swz<uint32_t>(s_)] & 0xfffu) : (uint32_t)(KS[swz<uint64_t>(s_)] & 0xfffu);
  };
  auto LN = [&](uint32_t s_) -> uint64_t {
    return WIDE ? KS[s_] : MODE == 0 ? (uint64_t)(KS32[swz<uint32_t>(s_)] >> 12) : (KS[swz<uint64_t>(s_)] >> 12);
  };
  // ---- previous local use; first / last use of the line in its piece
  uint32_t isent = 0, nent = 0;
#pragma unroll
  for (int j = 0; j < IPT; ++j) {
    const uint32_t s_ = tx * IPT + j;
    if (s_ >= m) continue;
    const uint32_t x = POS(s_);
    const uint64_t l = LN(s_);
    const uint32_t sg = S.sgs[x];
    const bool prev_same = s_ > 0 && LN(s_ - 1) == l && S.sgs[POS(s_ - 1)] == sg;
    const bool next_same = s_ + 1 < m && LN(s_ + 1) == l && S.sgs[POS(s_ + 1)] == sg;
    const bool st = S.sdw[x] & 1u;
    uint32_t p = 0;
    if (prev_same && !st) {
      p = POS(s_ - 1) + 1u;
      S.fnx[p - 1] = 1;
    }
    S.pl[x] = (uint16_t)p;
    S.ffl[x] = (uint8_t)((prev_same ? 0u : 1u) | (next_same ? 0u : 2u));
    if (!prev_same && partial(x)) {
      isent |= 1u << j;
      nent++;
    }
  }
  // ---- entry slots, one per (partial piece, line), allocated in sorted order
  uint32_t etot;
  const uint32_t eoff = block_exclusive_scan<TL_NT>(nent, S.ws, &etot);
  if (tx == 0)
    S.misc[1] = etot ? (uint32_t)atomicAdd((unsigned long long*)&sc->count[1], (unsigned long long)etot) : 0u;
  __syncthreads();
  const uint32_t ebase = S.misc[1];
  if (isent) {
    uint32_t run = eoff;
#pragma unroll
    for (int j = 0; j < IPT; ++j) {
      if (!((isent >> j) & 1u)) continue;
      const uint32_t s_ = tx * IPT + j;
      const uint32_t x = POS(s_);
      const uint32_t slot = ebase + run;
      E.seg[slot] = key ? __ldg(key + b + x) : 0u;
      E.line[slot] = WIDE ? LN(s_) : LN(s_) + lmin;
      E.tile[slot] = TP.tile_base + tile;
      S.es[x] = (uint16_t)(run + 1);
      run++;
    }
  }
  __syncthreads();
  if (etot) {
    // the last use of a run (if different from the first) shares the run's slot
#pragma unroll
    for (int j = 0; j < IPT; ++j) {
      const uint32_t s_ = tx * IPT + j;
      if (s_ >= m) continue;
      const uint32_t x = POS(s_);
      const uint32_t f = S.ffl[x];
      if ((f & 2u) && !(f & 1u) && partial(x)) {
        uint32_t q = s_;
        while (!(S.ffl[POS(q)] & 1u)) --q;
        S.es[x] = S.es[POS(q)];
      }
    }
    __syncthreads();
  }
  // ---- position-order prefix counts: local queries and weights
  uint32_t* QK = reinterpret_cast<uint32_t*>(S.key[r]);          // 2 x TL_CAP u32 (the sorted keys are dead now)
  uint32_t* QK2 = QK + TL_CAP;
  uint32_t* WP = reinterpret_cast<uint32_t*>(S.key[r ^ 1]);      // TL_CAP u32
  uint16_t* CNT = reinterpret_cast<uint16_t*>(WP + TL_CAP);       // TL_CAP u16
  uint32_t nq = 0, wsum = 0;
#pragma unroll
  for (int j = 0; j < IPT; ++j) {
    const uint32_t x = tx * IPT + j;
    if (x < m) {
      nq += S.pl[x] ? 1u : 0u;
      wsum += S.sdw[x] >> 2;
    }
  }
  uint32_t Q, WT;
  uint32_t qoff = block_exclusive_scan<TL_NT>(nq, S.ws, &Q);
  uint32_t woff = block_exclusive_scan<TL_NT>(wsum, S.ws, &WT);
#pragma unroll
  for (int j = 0; j < IPT; ++j) {
    const uint32_t x = tx * IPT + j;
    S.qx[x] = (uint16_t)qoff;
    WP[x] = woff;
    if (x < m) {
      if (S.pl[x]) {
        QK[swz<uint32_t>(qoff)] = ((uint32_t)(S.pl[x] - 1u) << 12) | x;
        qoff++;
      }
      woff += S.sdw[x] >> 2;
    }
  }
  uint32_t NQ = 64;
  while (NQ < Q) NQ <<= 1;
  for (uint32_t k = Q + tx; k < NQ; k += TL_NT) QK[swz<uint32_t>(k)] = 0xffffffffu;
  for (uint32_t x = tx; x < TL_CAP; x += TL_NT) CNT[x] = 0;
  __syncthreads();
  // ---- counting sort of the queries by previous use:
  //      CNT[x] = #{ local queries y < x : P(y) > P(x) }
  const int r2 = block_sort_keys<TL_NT, uint32_t, true>(QK, QK2, CNT, 0xffffffffu, NQ);
  const uint32_t* QS = r2 ? QK2 : QK;
  // ---- R4: bin the local accesses
  uint32_t stream = 0;
  unsigned long long rdsum = 0;  // finite distances (Eq. (1)'s average reuse distance)
#pragma unroll
  for (int j = 0; j < IPT; ++j) {
    const uint32_t x = tx * IPT + j;
    if (x >= m) continue;
    const uint32_t sdw = S.sdw[x];
    const bool st = sdw & 1u, hd = (sdw >> 1) & 1u;
    const uint32_t w = sdw >> 2;
    uint32_t bin = 0xffffffffu, cntb = 1;
    const bool head_first = S.sgs[x] == 0 && head_cont && (S.ffl[x] & 1u);
    if (S.pl[x]) {
      const uint32_t p = S.pl[x] - 1u;
      const uint32_t rd = (WP[x] - WP[p] - (uint32_t)(S.sdw[p] >> 2)) - CNT[x];
      bin = rd_bin(rd, log2bins, nbins);
      rdsum += rd;
    } else if (st) {
      bin = nbins - 1;
      cntb = w;
    } else if (!head_first) {
      bin = nbins - 1;
    }
    if (bin != 0xffffffffu) {
      if (O.n) bin += obj_row(O, __ldg(val + gpos(x)) & LINE_MASK) * nbins;
      if (smem_hist) atomicAdd(&S.hist[bin], cntb);
      else atomicAdd((unsigned long long*)&g_hist[bin], (unsigned long long)cntb);
    }
    if (st) stream += w - 1;  // all but the last of merged stores are one-shot elements
    const bool deferred = partial(x) && S.ffl[x] != 0;
    if (!deferred && !S.pl[x] && !hd && !S.fnx[x]) stream += 1;
  }
  // ---- entry payloads of partial pieces
  if (etot) {
    for (uint32_t x = tx; x < m; x += TL_NT) {
      if (!S.es[x]) continue;
      const uint32_t slot = ebase + S.es[x] - 1;
      const uint32_t f = S.ffl[x];
      const uint32_t sdw = S.sdw[x];
      if (f & 1u) {
        const bool head_piece = S.sgs[x] == 0 && head_cont;
        E.f[slot] = (uint32_t)(TP.pos_base + b + x);
        E.fa[slot] = (uint32_t)S.qx[x] - (uint32_t)S.qx[S.sgs[x]];
        E.fw[slot] = WP[x];
        E.ff[slot] = (uint8_t)(((sdw & 1u) ? 0u : 1u) | (((sdw >> 1) & 1u) ? 0u : 2u) | (S.fnx[x] ? 4u : 0u) |
                               (head_piece ? 8u : 0u) | ((f & 2u) ? 16u : 0u));
      }
      if (f & 2u) {
        const uint32_t pend = (S.sgs[x] == lastseg && tail_cont) ? m : second;
        // queries of the piece whose previous use lies in (x, pend)
        const uint32_t lo_key = (x + 1) << 12, hi_key = pend << 12;
        uint32_t a0 = 0, a1 = Q;
        while (a0 < a1) { uint32_t md = (a0 + a1) >> 1; if (QS[swz<uint32_t>(md)] < lo_key) a0 = md + 1; else a1 = md; }
        uint32_t c0 = a0, c1 = Q;
        while (c0 < c1) { uint32_t md = (c0 + c1) >> 1; if (QS[swz<uint32_t>(md)] < hi_key) c0 = md + 1; else c1 = md; }
        E.l[slot] = (uint32_t)(TP.pos_base + b + x);
        E.lw[slot] = WP[x];
        E.ld[slot] = c0 - a0;
        E.lf[slot] = (uint8_t)((sdw & 1u) | (((sdw >> 1) & 1u) ? 0u : 2u) | ((sdw >> 2) << 2));
      }
    }
  }
  // ---- flush
  stream = __reduce_add_sync(FULL, stream);
  if (lane_id() == 0 && stream) atomicAdd((unsigned long long*)g_stream, (unsigned long long)stream);
#pragma unroll
  for (int o = 16; o; o >>= 1) rdsum += __shfl_xor_sync(FULL, rdsum, o);
  if (lane_id() == 0 && rdsum) atomicAdd((unsigned long long*)g_stream + 1, rdsum);
  if (tx == 0) {
    tile_w[TP.tile_base + tile] = WT;
    tile_q[TP.tile_base + tile] = Q;
  }
  __syncthreads();
  if (smem_hist)
    for (uint32_t k = tx; k < hbins; k += TL_NT)
      if (S.hist[k]) atomicAdd((unsigned long long*)&g_hist[k], (unsigned long long)S.hist[k]);
}

// ------------------------------------------------------------------ cross-tile phase
__global__ void k_ent_line_range(const uint64_t* __restrict__ line, uint64_t E, unsigned long long* mn,
                                 unsigned long long* mx) {
  uint64_t a = ~0ull, z = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < E; i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t v = line[i];
    a = v < a ? v : a;
    z = v > z ? v : z;
  }
  for (int o = 16; o; o >>= 1) {
    uint64_t a2 = __shfl_xor_sync(FULL, a, o), z2 = __shfl_xor_sync(FULL, z, o);
    a = a2 < a ? a2 : a;
    z = z2 > z ? z2 : z;
  }
  if (lane_id() == 0) { atomicMin(mn, (unsigned long long)a); atomicMax(mx, (unsigned long long)z); }
}

// composite sort key (seg, line - minl, tile) when it fits in 64 bits; else
// one field at a time (field 0 = tile, 1 = line, 2 = seg) through idx.
__global__ void k_ent_key(const uint32_t* __restrict__ seg, const uint64_t* __restrict__ line,
                          const uint32_t* __restrict__ tile, uint64_t E, uint64_t minl, int lb, int tb, int field,
                          const uint32_t* __restrict__ idx_in, uint64_t* __restrict__ key, uint32_t* __restrict__ idx) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < E; i += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t j = idx_in ? idx_in[i] : (uint32_t)i;
    uint64_t k;
    if (field < 0) k = ((uint64_t)seg[j] << (lb + tb)) | ((line[j] - minl) << tb) | tile[j];
    else if (field == 0) k = tile[j];
    else if (field == 1) k = line[j] - minl;
    else k = seg[j];
    key[i] = k;
    idx[i] = j;
  }
}

struct CrossOut {
  uint32_t* xpos;   // query global kept position
  uint32_t* xq;     // its previous use (global kept position)
  int64_t* part;    // RD before subtracting the cross-tile dominance count
  uint64_t* xline;  // its line (data-centric rows)
};

__global__ void k_link(const uint32_t* __restrict__ order, uint64_t E, EntryCols En,
                       const unsigned long long* __restrict__ tile_wb, const unsigned long long* __restrict__ tile_qb,
                       uint32_t nbins, uint64_t* g_hist, uint64_t* g_stream, CrossOut X, Scalars* sc, ObjTab O) {
  uint32_t stream = 0;
  for (uint64_t k = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < E; k += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t e = order[k];
    int64_t pv = -1, nx = -1;
    if (k > 0) {
      uint32_t p = order[k - 1];
      if (En.seg[p] == En.seg[e] && En.line[p] == En.line[e]) pv = p;
    }
    if (k + 1 < E) {
      uint32_t q = order[k + 1];
      if (En.seg[q] == En.seg[e] && En.line[q] == En.line[e]) nx = q;
    }
    uint8_t ff = En.ff[e], lf = En.lf[e];
    bool f_load = ff & 1u, f_nodup = ff & 2u, f_next = ff & 4u, head = ff & 8u, f_is_l = ff & 16u;
    bool next_load = nx >= 0 && (En.ff[nx] & 1u);
    // RD of the piece's first use (deferred by the tile kernel when the piece is a head piece)
    bool linked = false;
    if (head && f_load) {
      if (pv >= 0) {
        linked = true;
        uint32_t p = (uint32_t)pv;
        uint64_t gwf = tile_wb[En.tile[e]] + En.fw[e];
        uint64_t gwl = tile_wb[En.tile[p]] + En.lw[p];
        uint32_t wl = En.lf[p] >> 2;
        uint64_t B = tile_qb[En.tile[e]] - tile_qb[En.tile[p] + 1];
        int64_t part = (int64_t)(gwf - gwl - wl) - (int64_t)En.fa[e] - (int64_t)B - (int64_t)En.ld[p];
        unsigned long long slot = atomicAdd((unsigned long long*)&sc->count[2], 1ull);
        X.xpos[slot] = En.f[e];
        X.xq[slot] = En.l[p];
        X.part[slot] = part;
        X.xline[slot] = En.line[e];
      } else {
        const uint32_t row = O.n ? obj_row(O, En.line[e]) : 0u;
        atomicAdd((unsigned long long*)&g_hist[(uint64_t)row * nbins + nbins - 1], 1ull);
      }
    }
    // streaming of the deferred first / last uses
    bool f_pnone = !f_load || !linked;
    bool f_next_any = f_is_l ? next_load : f_next;
    if (f_pnone && f_nodup && !f_next_any) stream++;
    if (!f_is_l) {
      bool l_store = lf & 1u, l_nodup = lf & 2u;
      if (l_store && l_nodup && !next_load) stream++;
    }
  }
  stream = __reduce_add_sync(FULL, stream);
  if (lane_id() == 0 && stream) atomicAdd((unsigned long long*)g_stream, (unsigned long long)stream);
}

// one level of a device-wide merge sort with inversion counting: runs of
// width w are merged pairwise; items of the right run add the number of
// larger items in the left run to cnt[id] (keys are distinct).  Merge path:
// each thread finds where its MP_IT consecutive output positions start in the
// two runs with one binary search along its diagonal, then merges them
// sequentially - a right-run item leaves lenA - a larger left items behind.
constexpr int MP_IT = 8;
__global__ void __launch_bounds__(256) k_merge_count(const uint32_t* __restrict__ kin, const uint32_t* __restrict__ iin,
                                                     uint32_t* __restrict__ kout, uint32_t* __restrict__ iout,
                                                     uint64_t M, uint64_t w, uint32_t* __restrict__ cnt) {
  const uint64_t nthr = (M + MP_IT - 1) / MP_IT;
  for (uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; t < nthr; t += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t d0 = t * MP_IT;
    const uint64_t s = (d0 / (2 * w)) * (2 * w);
    const uint64_t d = d0 - s;
    const uint64_t lenA = M - s < w ? M - s : w;
    const uint64_t lenB = M - s > w ? (M - s - w < w ? M - s - w : w) : 0;
    const uint32_t* A = kin + s;
    const uint32_t* B = kin + s + lenA;
    // a = number of left-run items among the pair's first d outputs
    uint64_t lo = d > lenB ? d - lenB : 0, hi = d < lenA ? d : lenA;
    while (lo < hi) {
      const uint64_t mid = (lo + hi) >> 1;
      if (__ldg(A + mid) <= __ldg(B + (d - 1 - mid))) lo = mid + 1;
      else hi = mid;
    }
    uint64_t ia = lo, ib = d - lo;
    uint32_t ka = ia < lenA ? __ldg(A + ia) : 0u, kb = ib < lenB ? __ldg(B + ib) : 0u;
#pragma unroll
    for (int k = 0; k < MP_IT; ++k) {
      const uint64_t o = d + k;
      if (o >= lenA + lenB) break;
      if (ia < lenA && (ib >= lenB || ka <= kb)) {
        kout[s + o] = ka;
        iout[s + o] = __ldg(iin + s + ia);
        ++ia;
        if (ia < lenA) ka = __ldg(A + ia);
      } else {
        const uint32_t id = __ldg(iin + s + lenA + ib);
        kout[s + o] = kb;
        iout[s + o] = id;
        if (lenA - ia) cnt[id] += (uint32_t)(lenA - ia);
        ++ib;
        if (ib < lenB) kb = __ldg(B + ib);
      }
    }
  }
}

// The same level with shared-memory staging: block b produces the pair's
// outputs [MPB_T b', MPB_T (b' + 1)) - the two input stretches that feed them
// (found by one merge-path search per block boundary) are loaded coalesced
// into shared memory, each thread merges MP_IT outputs from there.
constexpr int MPB_NT = 256, MPB_T = MPB_NT * MP_IT;  // 2048 outputs per block
__device__ __forceinline__ uint64_t merge_split(const uint32_t* A, uint64_t lenA, const uint32_t* B, uint64_t lenB,
                                                uint64_t d) {
  uint64_t lo = d > lenB ? d - lenB : 0, hi = d < lenA ? d : lenA;
  while (lo < hi) {
    const uint64_t mid = (lo + hi) >> 1;
    if (A[mid] <= B[d - 1 - mid]) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}
__global__ void __launch_bounds__(MPB_NT) k_merge_count_tiled(const uint32_t* __restrict__ kin,
                                                              const uint32_t* __restrict__ iin,
                                                              uint32_t* __restrict__ kout, uint32_t* __restrict__ iout,
                                                              uint64_t M, uint64_t w, uint32_t* __restrict__ cnt) {
  __shared__ uint32_t sk[MPB_T], si[MPB_T];
  __shared__ uint64_t s_a[2];
  const uint64_t o0 = (uint64_t)blockIdx.x * MPB_T;  // blocks never straddle a pair: 2 w is a multiple of MPB_T
  const uint64_t s = (o0 / (2 * w)) * (2 * w);
  const uint64_t lenA = M - s < w ? M - s : w;
  const uint64_t lenB = M - s > w ? (M - s - w < w ? M - s - w : w) : 0;
  const uint64_t d0 = o0 - s;
  const uint64_t dn = d0 + MPB_T < lenA + lenB ? d0 + MPB_T : lenA + lenB;
  const uint32_t* A = kin + s;
  const uint32_t* B = kin + s + lenA;
  if (threadIdx.x < 2) s_a[threadIdx.x] = merge_split(A, lenA, B, lenB, threadIdx.x ? dn : d0);
  __syncthreads();
  const uint64_t a0 = s_a[0], a1 = s_a[1], b0 = d0 - a0, b1 = dn - a1;
  const uint32_t na = (uint32_t)(a1 - a0), nt = (uint32_t)(dn - d0);
  for (uint32_t x = threadIdx.x; x < nt; x += MPB_NT) {
    if (x < na) { sk[x] = A[a0 + x]; si[x] = iin[s + a0 + x]; }
    else { sk[x] = B[b0 + x - na]; si[x] = iin[s + lenA + b0 + x - na]; }
  }
  __syncthreads();
  // local merge of sk[0, na) and sk[na, nt): this thread's outputs [d, d + MP_IT)
  const uint32_t nb = nt - na, d = threadIdx.x * MP_IT;
  if (d >= nt) return;
  uint32_t lo = d > nb ? d - nb : 0, hi = d < na ? d : na;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (sk[mid] <= sk[na + d - 1 - mid]) lo = mid + 1;
    else hi = mid;
  }
  uint32_t ia = lo, ib = d - lo;
#pragma unroll
  for (int k = 0; k < MP_IT; ++k) {
    const uint32_t o = d + k;
    if (o >= nt) break;
    if (ia < na && (ib >= nb || sk[ia] <= sk[na + ib])) {
      kout[o0 + o] = sk[ia];
      iout[o0 + o] = si[ia];
      ++ia;
    } else {
      const uint32_t id = si[na + ib];
      kout[o0 + o] = sk[na + ib];
      iout[o0 + o] = id;
      const uint64_t left = lenA - (a0 + ia);  // left-run items still unmerged: all larger
      if (left) cnt[id] += (uint32_t)left;
      ++ib;
    }
  }
}

// The first 12 levels of that merge sort in shared memory: block b sorts the
// 4096 items [4096 b, 4096 b + 4096) by key (keys are distinct previous-use
// positions), adding to cnt[id] the number of earlier items in the block
// with a larger key.  Global k_merge_count levels continue from w = 4096.
constexpr int MC_BLOCK = 4096;
struct MergeBlockSmem {
  uint64_t ka[MC_BLOCK], kb[MC_BLOCK];
  uint16_t c[MC_BLOCK];
};
__global__ void __launch_bounds__(512) k_merge_count_block(const uint32_t* __restrict__ kin,
                                                           const uint32_t* __restrict__ iin,
                                                           uint32_t* __restrict__ kout, uint32_t* __restrict__ iout,
                                                           uint64_t M, uint32_t* __restrict__ cnt) {
  extern __shared__ __align__(16) uint8_t mc_raw[];
  MergeBlockSmem& S = *reinterpret_cast<MergeBlockSmem*>(mc_raw);
  const uint64_t base = (uint64_t)blockIdx.x * MC_BLOCK;
  const uint32_t n = (uint32_t)(M - base < MC_BLOCK ? M - base : MC_BLOCK);
  for (uint32_t i = threadIdx.x; i < MC_BLOCK; i += blockDim.x) {
    S.ka[swz<uint64_t>(i)] = i < n ? ((uint64_t)kin[base + i] << 12) | i : ~0ull;
    S.c[i] = 0;
  }
  __syncthreads();
  const int res = block_sort_keys<512, uint64_t, true>(S.ka, S.kb, S.c, ~0ull, MC_BLOCK);
  const uint64_t* src = res ? S.kb : S.ka;
  for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) {
    const uint64_t v = src[swz<uint64_t>(i)];
    kout[base + i] = (uint32_t)(v >> 12);
    iout[base + i] = iin[base + (v & 0xfffu)];
    if (S.c[i]) cnt[iin[base + i]] += S.c[i];
  }
}

__global__ void k_iota_gather(const uint32_t* __restrict__ order, const uint32_t* __restrict__ xq, uint64_t M,
                              uint32_t* __restrict__ k, uint32_t* __restrict__ id, uint32_t* __restrict__ cnt) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < M; i += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t j = order[i];
    k[i] = xq[j];
    id[i] = j;
    cnt[j] = 0;
  }
}

constexpr uint32_t XF_SMEM_BINS = 4096;
// O.n > 0 (data-centric attribution): the query's row comes from its line
__global__ void __launch_bounds__(256) k_cross_final(const int64_t* __restrict__ part,
                                                     const uint32_t* __restrict__ cnt, uint64_t M, int log2bins,
                                                     uint32_t nbins, uint64_t* g_hist, uint64_t* g_stats,
                                                     Scalars* sc, ObjTab O, const uint64_t* __restrict__ xline) {
  unsigned long long rdsum = 0;
  __shared__ uint32_t h[XF_SMEM_BINS];
  const uint32_t hbins = (O.n + 1) * nbins;
  const bool sm = hbins <= XF_SMEM_BINS;
  if (sm)
    for (uint32_t k = threadIdx.x; k < hbins; k += blockDim.x) h[k] = 0;
  __syncthreads();
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < M; i += (uint64_t)gridDim.x * blockDim.x) {
    int64_t rd = part[i] - (int64_t)cnt[i];
    if (rd < 0) {
      atomicMax(&sc->err_code, 3u);
      rd = 0;
    }
    uint32_t b = rd_bin((uint64_t)rd, log2bins, nbins);
    if (O.n) b += obj_row(O, __ldg(xline + i)) * nbins;
    rdsum += (unsigned long long)rd;
    if (sm) {
      // warp-aggregated: one shared-memory atomic per distinct bin in the warp
      const uint32_t peers = __match_any_sync(__activemask(), b);
      if (lane_id() == (uint32_t)(__ffs(peers) - 1)) atomicAdd(&h[b], (uint32_t)__popc(peers));
    } else {
      atomicAdd((unsigned long long*)&g_hist[b], 1ull);
    }
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) rdsum += __shfl_xor_sync(FULL, rdsum, o);
  if (lane_id() == 0 && rdsum) atomicAdd((unsigned long long*)g_stats + 1, rdsum);
  __syncthreads();
  if (sm)
    for (uint32_t k = threadIdx.x; k < hbins; k += blockDim.x)
      if (h[k]) atomicAdd((unsigned long long*)&g_hist[k], (unsigned long long)h[k]);
}

__global__ void k_widen(const uint32_t* a, unsigned long long* o, uint64_t nvalid, uint64_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    o[i] = i < nvalid ? a[i] : 0ull;
}

__global__ void k_iota(uint32_t* p, uint64_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    p[i] = (uint32_t)i;
}

// ---- multi-rank exchange helpers
__global__ void k_bucket_count(const uint32_t* __restrict__ key, uint64_t K, int shift, unsigned long long* cnt) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < K; i += (uint64_t)gridDim.x * blockDim.x) {
    // keys are sorted: one atomic per run of equal buckets inside a warp
    const uint32_t b = __ldg(key + i) >> shift;
    const uint32_t peers = __match_any_sync(__activemask(), b);
    if ((lane_id()) == (uint32_t)(__ffs(peers) - 1)) atomicAdd(&cnt[b], (unsigned long long)__popc(peers));
  }
}

// out[r] = first position whose bucket >= bnd[r], r < m (keys sorted)
__global__ void k_lower_bounds(const uint32_t* __restrict__ key, uint64_t K, int shift, const uint64_t* bnd, int m,
                               uint64_t* out) {
  const int r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= m) return;
  uint64_t lo = 0, hi = K;
  while (lo < hi) {
    const uint64_t md = (lo + hi) >> 1;
    if ((uint64_t)(key[md] >> shift) < bnd[r]) lo = md + 1;
    else hi = md;
  }
  out[r] = lo;
}

// Exchange over peer memory: every rank stores its slice for rank r straight
// into r's receive buffers (CUDA IPC mappings over NVLink / NVSwitch, or the
// in-process loopback ranks' buffers), one launch for all destinations.
constexpr int MAX_RANKS = 64;
struct PushArgs {
  const uint32_t* key;
  const uint64_t* val;
  uint32_t* pk[MAX_RANKS];
  uint64_t* pv[MAX_RANKS];
  uint64_t soff[MAX_RANKS], scnt[MAX_RANKS], doff[MAX_RANKS];
};
__global__ void __launch_bounds__(256) k_push(const __grid_constant__ PushArgs P) {
  const int r = blockIdx.y;
  const uint64_t n = P.scnt[r];
  const uint32_t* ks = P.key ? P.key + P.soff[r] : nullptr;
  const uint64_t* vs = P.val + P.soff[r];
  uint32_t* kd = P.key ? P.pk[r] + P.doff[r] : nullptr;
  uint64_t* vd = P.pv[r] + P.doff[r];
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    if (ks) kd[i] = __ldg(ks + i);
    vd[i] = __ldg(vs + i);
  }
}

int bits_for(uint64_t maxv) {
  int b = 0;
  while (b < 64 && (maxv >> b)) ++b;
  return b;
}


}  // namespace

cudaError_t rd_begin(cadv_ctx* c, int scope, RdState* st) {
  cudaError_t e;
  const uint64_t n = c->t.n;
  const uint64_t nmem = n;  // memory records <= records (R0 counts now come out of the scan)
  st->cta_scope = scope == CADV_SCOPE_CTA;
  uint64_t grid, nw, chunk;
  scan_geometry(c, n, &grid, &nw, &chunk);
  st->grid = nw;  // one kept-record region per scan chunk (scan_geometry: nchunks)
  // region capacity: max(chunk / 4, kcap_min) records (run compression keeps
  // ~7 % of the paper-shaped traces; a region that overflows raises kcap_min
  // and the call runs again, see run_once), so C5's 4e9 records need 24 B per
  // kept slot, not per record
  uint64_t kcap = chunk / 4 > c->kcap_min ? chunk / 4 : c->kcap_min;
  kcap = ((kcap + 255) / 256) * 256;
  if (kcap > chunk) kcap = chunk;
  st->chunk_cap = kcap;
  // the scan writes kept records into per-warp regions of (k1, v1) (stride
  // kcap); the regroup / squeeze packs them into (k0, v0); the CTA radix sort
  // then ping-pongs between the two pairs.
  const uint64_t gap = nw * kcap + 16, cap = (nmem > gap ? gap : nmem) + 16;
  void *k0 = nullptr, *k1 = nullptr, *v0, *v1, *bc;
  if ((e = ensure(c, B_RD_VAL, (gap > cap ? gap : cap) * 8, &v0)) || (e = ensure(c, B_SORT_V1, gap * 8, &v1))) return e;
  if (st->cta_scope && ((e = ensure(c, B_RD_KEY, (gap > cap ? gap : cap) * 4, &k0)) ||
                        (e = ensure(c, B_SORT_K1, gap * 4, &k1))))
    return e;
  if ((e = ensure(c, B_RD_TILESTAT, (2 * nw + 8) * 8, &bc))) return e;
  if ((e = cudaMemsetAsync(bc, 0, (2 * nw + 8) * 8, c->stream))) return e;
  st->k0 = (uint32_t*)k0;
  st->k1 = (uint32_t*)k1;
  st->v0 = (uint64_t*)v0;
  st->v1 = (uint64_t*)v1;
  st->blkcnt = (uint64_t*)bc;
  st->rg = st->cta_scope && c->comm == nullptr && getenv("CADV_REGROUP_RADIX") == nullptr;
  return cudaSuccess;
}

// Multi-rank contexts: every rank's kept records (CTA-major after the local
// sort) are redistributed so that each scope lives on one rank: CTA ranges
// balanced by kept-record counts (CTA scope), or everything to rank 0
// (kernel scope: one scope).  A scope's records arrive from the ranks in rank
// order = trace order, and a stable sort by scope restores the global
// CTA-major order exactly.  Collective: every rank calls it.
cudaError_t rd_exchange(cadv_ctx* c, int cta_scope, const uint32_t** key, const uint64_t** val, uint64_t* K) {
  cudaError_t e;
  const int G = c->nranks, me = c->rank;
  Comm* cm = c->comm;
  std::vector<uint64_t> scnt(G, 0), soff(G, 0), rcnt(G, 0), roff(G, 0);
  void* cb;
  if ((e = ensure(c, B_COMM, (size_t)(G + 2) * 8 + (size_t)G * G * 8 + 64, &cb))) return e;
  uint64_t* d_send = (uint64_t*)cb;
  uint64_t* d_mat = d_send + G + 2;
  const uint64_t Kl = *K;
  {
    // every rank's CTA-id range of its kept records -> the global range
    uint32_t* dm = (uint32_t*)d_mat;
    if ((e = cudaMemcpyAsync(dm, &c->max_cta, 4, cudaMemcpyHostToDevice, c->stream))) return e;
    if (cm->allreduce_max_u32(dm, 1, c->stream)) return cudaErrorUnknown;
    uint32_t gm = 0;
    if ((e = cudaMemcpyAsync(&gm, dm, 4, cudaMemcpyDeviceToHost, c->stream))) return e;
    if ((e = cudaStreamSynchronize(c->stream))) return e;
    c->max_cta = gm;
  }
  if (!cta_scope) {
    scnt[0] = Kl;
  } else {
    const int cbits = bits_for(c->max_cta);
    const int shift = cbits > 20 ? cbits - 20 : 0;
    const uint64_t nb = ((uint64_t)c->max_cta >> shift) + 1;
    void* cntb;
    if ((e = ensure(c, B_XCH_CNT, (nb + 2 * G + 4) * 8 + 64, &cntb))) return e;
    unsigned long long* cnt = (unsigned long long*)cntb;
    uint64_t* d_bnd = (uint64_t*)(cnt + nb);
    if ((e = cudaMemsetAsync(cnt, 0, nb * 8, c->stream))) return e;
    if (Kl) CADV_LAUNCH(c, k_bucket_count<<<c->num_sms * 4, 256, 0, c->stream>>>(*key, Kl, shift, cnt));
    if (cm->allreduce_sum_u64((uint64_t*)cnt, nb, c->stream)) return cudaErrorUnknown;
    std::vector<uint64_t> h(nb);
    if ((e = cudaMemcpyAsync(h.data(), cnt, nb * 8, cudaMemcpyDeviceToHost, c->stream))) return e;
    if ((e = cudaStreamSynchronize(c->stream))) return e;
    // rank r owns buckets [bnd[r], bnd[r+1]): equal shares of the global kept count
    uint64_t total = 0;
    for (uint64_t b = 0; b < nb; ++b) total += h[b];
    std::vector<uint64_t> bnd(G + 1, nb);
    bnd[0] = 0;
    uint64_t acc = 0, b = 0;
    for (int r = 1; r < G; ++r) {
      const uint64_t target = (uint64_t)((unsigned __int128)total * r / G);
      while (b < nb && acc + h[b] <= target) acc += h[b++];
      bnd[r] = b;
    }
    std::vector<uint64_t> pos(G + 1, 0);
    pos[G] = Kl;
    if (Kl && G > 1) {
      if ((e = cudaMemcpyAsync(d_bnd, bnd.data() + 1, (G - 1) * 8, cudaMemcpyHostToDevice, c->stream))) return e;
      CADV_LAUNCH(c, k_lower_bounds<<<1, 32, 0, c->stream>>>(*key, Kl, shift, d_bnd, G - 1, d_bnd + G));
      if ((e = cudaMemcpyAsync(pos.data() + 1, d_bnd + G, (G - 1) * 8, cudaMemcpyDeviceToHost, c->stream))) return e;
      if ((e = cudaStreamSynchronize(c->stream))) return e;
    } else {
      for (int r = 1; r < G; ++r) pos[r] = 0;
    }
    for (int r = 0; r < G; ++r) {
      soff[r] = pos[r];
      scnt[r] = pos[r + 1] - pos[r];
    }
  }
  // the G x G count matrix: row p = what rank p sends to each rank
  std::vector<uint64_t> mat((size_t)G * G);
  if ((e = cudaMemcpyAsync(d_send, scnt.data(), G * 8, cudaMemcpyHostToDevice, c->stream))) return e;
  if (cm->allgather(d_send, d_mat, G * 8, c->stream)) return cudaErrorUnknown;
  if ((e = cudaMemcpyAsync(mat.data(), d_mat, (size_t)G * G * 8, cudaMemcpyDeviceToHost, c->stream))) return e;
  if ((e = cudaStreamSynchronize(c->stream))) return e;
  uint64_t Kn = 0;
  for (int p = 0; p < G; ++p) {
    rcnt[p] = mat[(size_t)p * G + me];
    roff[p] = Kn;
    Kn += rcnt[p];
  }
  // kept positions are u32: decided from the all-gathered matrix, so every
  // rank takes the same branch (no rank may leave the others in a collective)
  for (int r = 0; r < G; ++r) {
    uint64_t kr = 0;
    for (int p = 0; p < G; ++p) kr += mat[(size_t)p * G + r];
    if (kr >= 0xffffffffull) return cudaErrorNotSupported;
  }
  void *rk0, *rk1 = nullptr, *rv0, *rv1;
  c->buf[B_XCH_V0].exported = c->buf[B_XCH_K0].exported = true;  // mapped by the peers (k_push)
  if ((e = ensure(c, B_XCH_V0, Kn * 8 + 16, &rv0)) || (e = ensure(c, B_XCH_V1, Kn * 8 + 16, &rv1))) return e;
  if (cta_scope &&
      ((e = ensure(c, B_XCH_K0, Kn * 4 + 16, &rk0)) || (e = ensure(c, B_XCH_K1, Kn * 4 + 16, &rk1))))
    return e;
  auto scaled = [&](const std::vector<uint64_t>& v, uint64_t f) {
    std::vector<uint64_t> o(v);
    for (auto& x : o) x *= f;
    return o;
  };
  const bool via_nccl = getenv("CADV_EXCHANGE") && !strcmp(getenv("CADV_EXCHANGE"), "nccl");
  if (via_nccl || G > MAX_RANKS) {
    // baseline: NCCL grouped send / receive
    if (cta_scope && cm->alltoallv(*key, scaled(soff, 4).data(), scaled(scnt, 4).data(), rk0,
                                   scaled(roff, 4).data(), scaled(rcnt, 4).data(), c->stream))
      return cudaErrorUnknown;
    if (cm->alltoallv(*val, scaled(soff, 8).data(), scaled(scnt, 8).data(), rv0, scaled(roff, 8).data(),
                      scaled(rcnt, 8).data(), c->stream))
      return cudaErrorUnknown;
  } else {
    // peer memory: map the receive buffers of every rank, store the slices directly
    PushArgs P{};
    void* pk[MAX_RANKS];
    void* pv[MAX_RANKS];
    if (cta_scope && cm->map_peers(0, rk0, pk, c->stream)) return cudaErrorUnknown;
    if (cm->map_peers(1, rv0, pv, c->stream)) return cudaErrorUnknown;
    P.key = cta_scope ? *key : nullptr;
    P.val = *val;
    uint64_t maxc = 0;
    for (int r = 0; r < G; ++r) {
      P.pk[r] = cta_scope ? (uint32_t*)pk[r] : nullptr;
      P.pv[r] = (uint64_t*)pv[r];
      P.soff[r] = soff[r];
      P.scnt[r] = scnt[r];
      uint64_t d = 0;  // where my slice starts in rank r's buffer: what ranks < me send to r
      for (int p = 0; p < me; ++p) d += mat[(size_t)p * G + r];
      P.doff[r] = d;
      maxc = scnt[r] > maxc ? scnt[r] : maxc;
    }
    if (maxc) {
      const uint64_t want = (maxc + 255) / 256;
      const dim3 grid((unsigned)(want < (uint64_t)c->num_sms * 4 ? want : (uint64_t)c->num_sms * 4), G);
      CADV_LAUNCH(c, k_push<<<grid, 256, 0, c->stream>>>(P));
      if ((e = cudaGetLastError())) return e;
    }
    if (cm->barrier(c->stream)) return cudaErrorUnknown;  // every slice has landed
  }
  *K = Kn;
  *val = (const uint64_t*)rv0;
  *key = nullptr;
  if (cta_scope && Kn) {
    int res, bits = bits_for(c->max_cta);
    if (bits == 0) bits = 1;
    if ((e = radix_sort_pairs<uint32_t, uint64_t>(c, (uint32_t*)rk0, (uint64_t*)rv0, (uint32_t*)rk1, (uint64_t*)rv1,
                                                  Kn, 0, bits, &res)))
      return e;
    *key = res ? (const uint32_t*)rk1 : (const uint32_t*)rk0;
    *val = res ? (const uint64_t*)rv1 : (const uint64_t*)rv0;
  }
  return cudaSuccess;
}

// ---- kernel scope over ranks, distributed cross-tile phase
namespace {

__device__ __forceinline__ uint32_t line_owner(uint64_t line, int G) {
  uint64_t z = line + 0x9E3779B97F4A7C15ull;  // splitmix64 finaliser: lines spread evenly over the ranks
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  z ^= z >> 31;
  return (uint32_t)(((z >> 32) * (uint64_t)G) >> 32);
}

__global__ void k_ent_owner(const uint64_t* __restrict__ line, uint64_t n, int G, uint32_t* own, uint32_t* idx,
                            unsigned long long* cnt) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t o = line_owner(__ldg(line + i), G);
    own[i] = o;
    idx[i] = (uint32_t)i;
    atomicAdd(&cnt[o], 1ull);
  }
}

// entry columns permuted: dst[k] = src[perm[k]]
__global__ void k_ent_permute(const uint32_t* __restrict__ perm, uint64_t n, EntryCols S, EntryCols D) {
  for (uint64_t k = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < n; k += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t i = perm[k];
    D.line[k] = S.line[i]; D.seg[k] = S.seg[i]; D.tile[k] = S.tile[i];
    D.f[k] = S.f[i]; D.fa[k] = S.fa[i]; D.fw[k] = S.fw[i]; D.ff[k] = S.ff[i];
    D.l[k] = S.l[i]; D.lw[k] = S.lw[i]; D.ld[k] = S.ld[i]; D.lf[k] = S.lf[i];
  }
}

// cross queries permuted into position order (send layout): dst[k] = src[perm[k]]
__global__ void k_xq_permute(const uint32_t* __restrict__ perm, uint64_t n, CrossOut S, CrossOut D) {
  for (uint64_t k = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < n; k += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t i = perm[k];
    D.xpos[k] = S.xpos[i]; D.xq[k] = S.xq[i]; D.part[k] = S.part[i]; D.xline[k] = S.xline[i];
  }
}

// cnt[j] += number of the queries of ranks before this one whose previous
// use lies after query j's (their positions all precede j's): per earlier
// rank r, M_r minus the upper bound of xq[j] in r's sorted previous uses
__global__ void k_count_greater(const uint32_t* __restrict__ xq, uint64_t M, const uint32_t* __restrict__ allp,
                                const uint64_t* __restrict__ off, int me, uint32_t* cnt) {
  for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j < M; j += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t x = xq[j];
    uint32_t add = 0;
    for (int r = 0; r < me; ++r) {
      uint64_t lo = off[r], hi = off[r + 1];
      const uint64_t b = hi;
      while (lo < hi) {
        const uint64_t md = (lo + hi) >> 1;
        if (allp[md] <= x) lo = md + 1;
        else hi = md;
      }
      add += (uint32_t)(b - lo);
    }
    cnt[j] += add;
  }
}

EntryCols carve_entries(void* base, uint64_t n) {
  EntryCols E;
  uint8_t* p = (uint8_t*)base;
  auto take = [&](size_t bytes) { uint8_t* q = p; p += (bytes + 15) & ~size_t(15); return q; };
  E.line = (uint64_t*)take(n * 8);
  E.seg = (uint32_t*)take(n * 4);
  E.tile = (uint32_t*)take(n * 4);
  E.f = (uint32_t*)take(n * 4);
  E.fa = (uint32_t*)take(n * 4);
  E.fw = (uint32_t*)take(n * 4);
  E.l = (uint32_t*)take(n * 4);
  E.lw = (uint32_t*)take(n * 4);
  E.ld = (uint32_t*)take(n * 4);
  E.ff = (uint8_t*)take(n);
  E.lf = (uint8_t*)take(n);
  return E;
}
constexpr size_t ENT_BYTES = 4 + 8 + 4 + 4 + 4 + 4 + 1 + 4 + 4 + 4 + 1;

CrossOut carve_queries(void* base, uint64_t n) {
  CrossOut X;
  X.xpos = (uint32_t*)base;
  X.xq = X.xpos + n;
  X.part = (int64_t*)(((uintptr_t)(X.xq + n) + 15) & ~(uintptr_t)15);
  X.xline = (uint64_t*)(X.part + n);
  return X;
}

// send counts (per destination rank, in the sender's order) -> the G x G
// matrix all-gathered; fills soff / scnt / roff / rcnt (in elements) and
// returns the number of elements this rank receives
int counts_matrix(cadv_ctx* c, const std::vector<uint64_t>& scnt, std::vector<uint64_t>* soff,
                  std::vector<uint64_t>* roff, std::vector<uint64_t>* rcnt, uint64_t* total, cudaError_t* e) {
  const int G = c->nranks, me = c->rank;
  void* cb;
  if ((*e = ensure(c, B_COMM, (size_t)(G + 2) * 8 + (size_t)G * G * 8 + 64, &cb))) return 1;
  uint64_t* d_send = (uint64_t*)cb;
  uint64_t* d_mat = d_send + G + 2;
  std::vector<uint64_t> mat((size_t)G * G);
  if ((*e = cudaMemcpyAsync(d_send, scnt.data(), G * 8, cudaMemcpyHostToDevice, c->stream))) return 1;
  if (c->comm->allgather(d_send, d_mat, G * 8, c->stream)) { *e = cudaErrorUnknown; return 1; }
  if ((*e = cudaMemcpyAsync(mat.data(), d_mat, (size_t)G * G * 8, cudaMemcpyDeviceToHost, c->stream)) ||
      (*e = cudaStreamSynchronize(c->stream)))
    return 1;
  soff->assign(G, 0);
  roff->assign(G, 0);
  rcnt->assign(G, 0);
  uint64_t a = 0, b = 0;
  for (int p = 0; p < G; ++p) {
    (*soff)[p] = a;
    a += scnt[p];
    (*rcnt)[p] = mat[(size_t)p * G + me];
    (*roff)[p] = b;
    b += (*rcnt)[p];
  }
  *total = b;
  return 0;
}

int a2av_col(cadv_ctx* c, const void* src, void* dst, size_t es, const std::vector<uint64_t>& soff,
             const std::vector<uint64_t>& scnt, const std::vector<uint64_t>& roff, const std::vector<uint64_t>& rcnt) {
  const int G = c->nranks;
  std::vector<uint64_t> so(G), sc(G), ro(G), rc(G);
  for (int p = 0; p < G; ++p) { so[p] = soff[p] * es; sc[p] = scnt[p] * es; ro[p] = roff[p] * es; rc[p] = rcnt[p] * es; }
  return c->comm->alltoallv(src, so.data(), sc.data(), dst, ro.data(), rc.data(), c->stream);
}

}  // namespace

// Every rank's cross-tile entries to the owner of their line (line hash):
// all entries of one line meet on one rank, which links them (k_link) and
// emits the cross-tile queries locally.  Collective; *En / *nent become the
// entries this rank owns.
cudaError_t exchange_entries_by_line(cadv_ctx* c, EntryCols* En, unsigned long long* nent) {
  cudaError_t e;
  const int G = c->nranks;
  const uint64_t n = *nent;
  void *ob, *sb, *cb2;
  if ((e = ensure(c, B_XE_OWN, n * 16 + 64, &ob)) || (e = ensure(c, B_XE_SEND, n * ENT_BYTES + 16 * 16, &sb)) ||
      (e = ensure(c, B_XE_CNT, (size_t)G * 8 + 64, &cb2)))
    return e;
  uint32_t* own0 = (uint32_t*)ob;
  uint32_t* idx0 = own0 + n;
  uint32_t* own1 = idx0 + n;
  uint32_t* idx1 = own1 + n;
  unsigned long long* dcnt = (unsigned long long*)cb2;
  if ((e = cudaMemsetAsync(dcnt, 0, (size_t)G * 8, c->stream))) return e;
  EntryCols S = carve_entries(sb, n);
  if (n) {
    CADV_LAUNCH(c, k_ent_owner<<<c->num_sms * 4, 256, 0, c->stream>>>(En->line, n, G, own0, idx0, dcnt));
    int res, bits = bits_for((uint64_t)(G - 1));
    if (bits == 0) bits = 1;
    if ((e = radix_sort_pairs<uint32_t, uint32_t>(c, own0, idx0, own1, idx1, n, 0, bits, &res))) return e;
    CADV_LAUNCH(c, k_ent_permute<<<c->num_sms * 4, 256, 0, c->stream>>>(res ? idx1 : idx0, n, *En, S));
  }
  std::vector<uint64_t> scnt(G), soff, roff, rcnt;
  if ((e = cudaMemcpyAsync(scnt.data(), dcnt, (size_t)G * 8, cudaMemcpyDeviceToHost, c->stream)) ||
      (e = cudaStreamSynchronize(c->stream)))
    return e;
  uint64_t N = 0;
  if (counts_matrix(c, scnt, &soff, &roff, &rcnt, &N, &e)) return e ? e : cudaErrorUnknown;
  void* rb;
  if ((e = ensure(c, B_RD_ENT_ALL, N * ENT_BYTES + 16 * 16, &rb))) return e;
  EntryCols R = carve_entries(rb, N);
  if (a2av_col(c, S.line, R.line, 8, soff, scnt, roff, rcnt) || a2av_col(c, S.seg, R.seg, 4, soff, scnt, roff, rcnt) ||
      a2av_col(c, S.tile, R.tile, 4, soff, scnt, roff, rcnt) || a2av_col(c, S.f, R.f, 4, soff, scnt, roff, rcnt) ||
      a2av_col(c, S.fa, R.fa, 4, soff, scnt, roff, rcnt) || a2av_col(c, S.fw, R.fw, 4, soff, scnt, roff, rcnt) ||
      a2av_col(c, S.l, R.l, 4, soff, scnt, roff, rcnt) || a2av_col(c, S.lw, R.lw, 4, soff, scnt, roff, rcnt) ||
      a2av_col(c, S.ld, R.ld, 4, soff, scnt, roff, rcnt) || a2av_col(c, S.ff, R.ff, 1, soff, scnt, roff, rcnt) ||
      a2av_col(c, S.lf, R.lf, 1, soff, scnt, roff, rcnt))
    return cudaErrorUnknown;
  *En = R;
  *nent = N;
  return cudaSuccess;
}

// The cross-tile queries to the rank holding their position ([base[r],
// base[r+1]) of the global kept sequence).  Collective; *X / *M become this
// rank's queries (capacity in B_RD_XQR).
cudaError_t exchange_queries_by_pos(cadv_ctx* c, CrossOut* X, unsigned long long* M, const std::vector<uint64_t>& base) {
  cudaError_t e;
  const int G = c->nranks;
  const uint64_t m = *M;
  void *kb, *sb, *db;
  if ((e = ensure(c, B_XE_OWN, m * 16 + 64, &kb)) || (e = ensure(c, B_XE_SEND, m * 24 + 256, &sb)) ||
      (e = ensure(c, B_XE_CNT, (size_t)(2 * G + 4) * 8 + 64, &db)))
    return e;
  uint32_t* k0 = (uint32_t*)kb;
  uint32_t* i0 = k0 + m;
  uint32_t* k1 = i0 + m;
  uint32_t* i1 = k1 + m;
  CrossOut S = carve_queries(sb, m);
  std::vector<uint64_t> pos(G + 1, 0);
  pos[G] = m;
  if (m) {
    if ((e = cudaMemcpyAsync(k0, X->xpos, m * 4, cudaMemcpyDeviceToDevice, c->stream))) return e;
    CADV_LAUNCH(c, k_iota<<<c->num_sms * 4, 256, 0, c->stream>>>(i0, m));
    int res;
    if ((e = radix_sort_pairs<uint32_t, uint32_t>(c, k0, i0, k1, i1, m, 0, 32, &res))) return e;
    const uint32_t* sk = res ? k1 : k0;
    CADV_LAUNCH(c, k_xq_permute<<<c->num_sms * 4, 256, 0, c->stream>>>(res ? i1 : i0, m, *X, S));
    if (G > 1) {
      uint64_t* d_bnd = (uint64_t*)db;
      if ((e = cudaMemcpyAsync(d_bnd, base.data() + 1, (G - 1) * 8, cudaMemcpyHostToDevice, c->stream))) return e;
      CADV_LAUNCH(c, k_lower_bounds<<<1, 64, 0, c->stream>>>(sk, m, 0, d_bnd, G - 1, d_bnd + G));
      if ((e = cudaMemcpyAsync(pos.data() + 1, d_bnd + G, (G - 1) * 8, cudaMemcpyDeviceToHost, c->stream)) ||
          (e = cudaStreamSynchronize(c->stream)))
        return e;
    }
  }
  std::vector<uint64_t> scnt(G), soff, roff, rcnt;
  for (int r = 0; r < G; ++r) scnt[r] = pos[r + 1] - pos[r];
  uint64_t N = 0;
  if (counts_matrix(c, scnt, &soff, &roff, &rcnt, &N, &e)) return e ? e : cudaErrorUnknown;
  void* rb;
  if ((e = ensure(c, B_RD_XQR, N * 24 + 256, &rb))) return e;
  CrossOut R = carve_queries(rb, N);
  R.part = (int64_t*)(((uintptr_t)(R.xq + N) + 15) & ~(uintptr_t)15);
  if (a2av_col(c, S.xpos, R.xpos, 4, soff, scnt, roff, rcnt) || a2av_col(c, S.xq, R.xq, 4, soff, scnt, roff, rcnt) ||
      a2av_col(c, S.part, R.part, 8, soff, scnt, roff, rcnt) ||
      a2av_col(c, S.xline, R.xline, 8, soff, scnt, roff, rcnt))
    return cudaErrorUnknown;
  *X = R;
  *M = N;
  return cudaSuccess;
}

// cnt[j] += the queries of earlier ranks (smaller positions) with a larger
// previous use than query j's: every rank's previous uses, sorted, are
// all-gathered and each query counts the larger ones by binary search.
// Collective (sorted = this rank's M previous uses in ascending order).
cudaError_t add_earlier_ranks(cadv_ctx* c, const uint32_t* sorted, uint64_t M, const uint32_t* xq, uint32_t* cnt) {
  cudaError_t e;
  const int G = c->nranks, me = c->rank;
  std::vector<uint64_t> scnt(G, M), soff(G, 0), roff, rcnt, dummy;
  uint64_t N = 0;
  if (counts_matrix(c, scnt, &dummy, &roff, &rcnt, &N, &e)) return e ? e : cudaErrorUnknown;
  void *ab, *ob;
  if ((e = ensure(c, B_XE_ALLP, N * 4 + 64, &ab)) || (e = ensure(c, B_XE_CNT, (size_t)(G + 2) * 8 + 64, &ob))) return e;
  if (a2av_col(c, sorted, ab, 4, soff, scnt, roff, rcnt)) return cudaErrorUnknown;
  std::vector<uint64_t> off(G + 1, 0);
  for (int p = 0; p < G; ++p) off[p + 1] = off[p] + rcnt[p];
  if ((e = cudaMemcpyAsync(ob, off.data(), (G + 1) * 8, cudaMemcpyHostToDevice, c->stream))) return e;
  if (M && me > 0)
    CADV_LAUNCH(c, k_count_greater<<<c->num_sms * 4, 256, 0, c->stream>>>(xq, M, (const uint32_t*)ab,
                                                                             (const uint64_t*)ob, me, cnt));
  return cudaGetLastError();
}

cudaError_t rd_compact(cadv_ctx* c, const RdState& S) {
  cudaError_t e;
  uint64_t* h = (uint64_t*)c->hstage;
  h[0] = h[1] = 0;
  if (!S.grid) return cudaSuccess;
  // pack the per-block regions: offsets = exclusive scan of the block counts
  uint64_t* off = S.blkcnt + S.grid + 4;
  if ((e = exclusive_scan_u64(c, S.blkcnt, off, S.grid + 1))) return e;
  if ((e = cudaMemcpyAsync(&h[0], off + S.grid, 8, cudaMemcpyDeviceToHost, c->stream))) return e;
  if (S.rg) {
    // regroup tables (regroup.cu): pair total, overflow flag and CTA-id range
    // arrive with the same read-back; the squeeze only runs on overflow
    RgState& G = const_cast<RdState&>(S).rgs;
    if ((e = rg_count(c, S.k1, S.blkcnt, S.grid, S.chunk_cap, &G))) return e;
    h[2] = h[3] = 0;
    if ((e = cudaMemcpyAsync(&h[2], G.poff + S.grid, 4, cudaMemcpyDeviceToHost, c->stream))) return e;
    if ((e = cudaMemcpyAsync(&h[3], &scalars(c)->rg_overflow, 8, cudaMemcpyDeviceToHost, c->stream))) return e;
    return cudaMemcpyAsync(&h[1], &scalars(c)->max_cta, 8, cudaMemcpyDeviceToHost, c->stream);
  }
  if ((e = launch_squeeze(c, (const uint32_t*)S.k1, (const uint64_t*)S.v1, (uint32_t*)S.k0, (uint64_t*)S.v0, S.blkcnt,
                          off, S.grid, S.chunk_cap)))
    return e;
  return cudaMemcpyAsync(&h[1], &scalars(c)->max_cta, 8, cudaMemcpyDeviceToHost, c->stream);
}

// The listed segments (257 .. SEG_TILE_MAX kept records each, CTA scope, one
// rank) packed next-fit, in list order, into tiles of <= TL_CAP kept records
// and <= TL_LSEG segments (the host reads the lengths back: a few hundred KB
// at most); k_rd_tile's block path resolves each tile without entries (no
// segment is cut); tiles whose line range is too wide for packed keys go to
// the MODE 1 / 2 instances as in the bounds-tiled path.
cudaError_t rd_segment_tiles(cadv_ctx* c, const uint64_t* val, const uint2* tl, uint32_t ntl, int log2bins,
                             uint32_t nbins, uint64_t* d_hist, uint64_t* d_stats, const ObjTab& O) {
  cudaError_t e;
  Scalars* sc = scalars(c);
  std::vector<uint2> hs(ntl);
  if ((e = cudaMemcpyAsync(hs.data(), tl, (size_t)ntl * sizeof(uint2), cudaMemcpyDeviceToHost, c->stream)) ||
      (e = cudaStreamSynchronize(c->stream)))
    return e;
  std::vector<uint32_t> tofs;
  tofs.reserve(ntl / 2 + 2);
  uint32_t acc = TL_CAP + 1, nin = 0;
  for (uint32_t j = 0; j < ntl; ++j) {
    if (acc + hs[j].y > (uint32_t)TL_CAP || nin == (uint32_t)TL_LSEG) {
      tofs.push_back(j);
      acc = 0;
      nin = 0;
    }
    acc += hs[j].y;
    ++nin;
  }
  tofs.push_back(ntl);
  const uint32_t nt = (uint32_t)tofs.size() - 1;
  void *lst, *tw, *tq;
  if ((e = ensure(c, B_RD_XTMP, (3 * (uint64_t)nt + 8 + (uint64_t)nt + 2) * 4 + 64, &lst)) ||
      (e = ensure(c, B_RD_TILEW, ((uint64_t)nt + 2) * 8 * 2, &tw)) ||
      (e = ensure(c, B_RD_TILEQ, ((uint64_t)nt + 2) * 8 * 2, &tq)))
    return e;
  uint32_t* wide_list = (uint32_t*)lst + 2;
  uint32_t* d_tofs = (uint32_t*)lst + 3 * (uint64_t)nt + 8;
  if ((e = cudaMemcpyAsync(d_tofs, tofs.data(), tofs.size() * 4, cudaMemcpyHostToDevice, c->stream))) return e;
  if (!(c->attr_set & (1u << 17))) {
    if ((e = cudaFuncSetAttribute(k_rd_tile<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(TileSmem))) ||
        (e = cudaFuncSetAttribute(k_rd_tile<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(TileSmem))) ||
        (e = cudaFuncSetAttribute(k_rd_tile<2>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  (int)sizeof(TileSmemWide))))
      return e;
    c->attr_set |= 1u << 17;
  }
  const EntryCols En{};
  const TilePos TP{0, 0, 0};
  CADV_LAUNCH(c, k_rd_tile<0><<<nt, TL_NT, sizeof(TileSmem), c->stream>>>(
                     nullptr, val, 0, nullptr, nt, log2bins, nbins, d_hist, d_stats, (uint32_t*)tw, (uint32_t*)tq, En,
                     sc, wide_list, O, TP, tl, d_tofs));
  static_assert(64 + sizeof(Scalars) + 64 + 16 <= 512, "pinned staging (cadv_create: 512 bytes)");
  unsigned long long* cnt = (unsigned long long*)((uint8_t*)c->hstage + 64 + sizeof(Scalars) + 64);
  if ((e = cudaMemcpyAsync(cnt, &sc->count[3], 16, cudaMemcpyDeviceToHost, c->stream)) ||
      (e = cudaStreamSynchronize(c->stream)))
    return e;
  if (cnt[1])
    CADV_LAUNCH(c, k_rd_tile<1><<<(unsigned)cnt[1], TL_NT, sizeof(TileSmem), c->stream>>>(
                       nullptr, val, 0, nullptr, nt, log2bins, nbins, d_hist, d_stats, (uint32_t*)tw, (uint32_t*)tq,
                       En, sc, wide_list, O, TP, tl, d_tofs));
  if (cnt[0])
    CADV_LAUNCH(c, k_rd_tile<2><<<(unsigned)cnt[0], TL_NT, sizeof(TileSmemWide), c->stream>>>(
                       nullptr, val, 0, nullptr, nt, log2bins, nbins, d_hist, d_stats, (uint32_t*)tw, (uint32_t*)tq,
                       En, sc, wide_list, O, TP, tl, d_tofs));
  return cudaGetLastError();
}

// Every CTA segment <= SEG_TILE_MAX kept records (CTA scope): no
// cross-segment term exists, so every segment is resolved alone - short ones
// by a warp of the segment kernel, long ones by the tile kernel over the
// packed segment list.  The segment kernel is queued before the host reads
// the segment counts (persistent grid: it reads them on the device and does
// nothing when a segment is longer than SEG_TILE_MAX), so the read-back
// overlaps it.  *done = false: a longer segment (or CADV_RD_TILES) - the
// caller takes the bounds-tiled path.  nseg_max: an upper bound of the
// number of segments (grid size).
cudaError_t rd_segments(cadv_ctx* c, const uint64_t* val, const uint2* seg, const uint2* seg_long,
                        unsigned int* seg_cm, uint64_t nseg_max, int log2bins, uint32_t nbins, uint64_t* d_hist,
                        uint64_t* d_stats, const ObjTab& O, bool* done) {
  cudaError_t e;
  *done = false;
  if (getenv("CADV_RD_TILES") != nullptr) return cudaSuccess;
  const auto kseg = O.n ? k_rd_seg<true> : k_rd_seg<false>;
  if (!(c->attr_set & (1u << 16))) {
    for (const auto kf : {k_rd_seg<true>, k_rd_seg<false>})
      if ((e = cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    (int)(sizeof(SegSmem) + 16 * SG_OBJ_SMEM + 16))))
        return e;
    c->attr_set |= 1u << 16;
  }
  const uint64_t hbins = (uint64_t)(O.n + 1) * nbins;
  const size_t smem = seg_smem_bytes(hbins, O.n);
  if (c->seg_ctas_smem != smem) {
    if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&c->seg_ctas, kseg, SG_NT, smem))) return e;
    if (c->seg_ctas < 1) c->seg_ctas = 1;
    c->seg_ctas_smem = smem;
  }
  const unsigned grid = (unsigned)std::min<uint64_t>((uint64_t)c->num_sms * c->seg_ctas, (nseg_max + SG_W - 1) / SG_W);
  if (grid)
    CADV_LAUNCH_N(c, "k_rd_seg", kseg<<<grid, SG_NT, smem, c->stream>>>(val, seg, seg_cm, seg_cm + 2, log2bins, nbins,
                                                                        d_hist, d_stats, O));
  unsigned int* hcm = (unsigned int*)((uint8_t*)c->hstage + 40);
  if ((e = cudaMemcpyAsync(hcm, seg_cm, 16, cudaMemcpyDeviceToHost, c->stream))) return e;
  if ((e = cudaStreamSynchronize(c->stream))) return e;
  if (hcm[1] > SEG_TILE_MAX) return cudaSuccess;
  const uint32_t nlong = hcm[3];
  if (nlong && (e = rd_segment_tiles(c, val, seg_long, nlong, log2bins, nbins, d_hist, d_stats, O))) return e;
  c->counts[1] = 0;
  c->counts[3] = nlong;
  *done = true;
  return cudaGetLastError();
}

cudaError_t rd_finish(cadv_ctx* c, const RdState& S, int log2bins, uint32_t nbins, uint64_t* d_hist,
                      uint64_t* d_stats, const ObjTab* obj) {
  cudaError_t e;
  const ObjTab O = obj ? *obj : ObjTab{nullptr, nullptr, 0u};
  const int cta_scope = S.cta_scope;
  const int grid_ls = c->num_sms * 4;
  Scalars* sc = scalars(c);
  uint64_t K = 0;
  const uint32_t* key = nullptr;
  const uint64_t* val = nullptr;
  if (S.grid) {
    // rd_compact ran and the caller synchronised the stream
    void *k0 = S.k0, *k1 = S.k1, *v0 = S.v0, *v1 = S.v1;
    K = ((const uint64_t*)c->hstage)[0];
    const unsigned long long mxc = ((const unsigned long long*)c->hstage)[1];  // CTA-id range (scan / squeeze)
    if (mxc > c->max_cta) c->max_cta = (uint32_t)mxc;
    c->counts[0] = K;
    // ---- R1b regroup by CTA (stable)
    val = (const uint64_t*)v0;
    if (S.rg && K) {
      const uint64_t* hs = (const uint64_t*)c->hstage;
      int bits = bits_for(c->max_cta);
      if (bits == 0) bits = 1;
      if (hs[3] == 0) {  // every region's CTAs fit its table
        const uint64_t P = hs[2];
        void* sb;
        if ((e = ensure(c, B_RG_SEG, (P + 16) * 16 + 64, &sb))) return e;
        uint2* seg = (uint2*)sb;                  // segments of <= SEG_WARP_MAX kept records
        uint2* seg_long = seg + (P + 16);         // longer ones
        unsigned int* seg_cm = (unsigned int*)(seg_long + (P + 16));  // |seg|, longest, next, |seg_long|
        if ((e = rg_finish(c, S.rgs, P, bits, (const uint32_t*)k1, (const uint64_t*)v1, S.blkcnt, S.chunk_cap,
                           (uint32_t*)k0, (uint64_t*)v0, seg, seg_long, seg_cm)))
          return e;
        key = (const uint32_t*)k0;
        val = (const uint64_t*)v0;
        bool done = false;
        if ((e = rd_segments(c, val, seg, seg_long, seg_cm, P, log2bins, nbins, d_hist, d_stats, O, &done))) return e;
        if (done) return cudaSuccess;
      } else {  // overflow: pack, then the radix sort
        if ((e = launch_squeeze(c, (const uint32_t*)k1, (const uint64_t*)v1, (uint32_t*)k0, (uint64_t*)v0, S.blkcnt,
                                S.blkcnt + S.grid + 4, S.grid, S.chunk_cap)))
          return e;
        int res;
        if ((e = radix_sort_pairs<uint32_t, uint64_t>(c, (uint32_t*)k0, (uint64_t*)v0, (uint32_t*)k1, (uint64_t*)v1,
                                                      K, 0, bits, &res)))
          return e;
        key = res ? (const uint32_t*)k1 : (const uint32_t*)k0;
        val = res ? (const uint64_t*)v1 : (const uint64_t*)v0;
      }
    } else if (cta_scope && K) {
      int res;
      int bits = bits_for(c->max_cta);
      if (bits == 0) bits = 1;
      if ((e = radix_sort_pairs<uint32_t, uint64_t>(c, (uint32_t*)k0, (uint64_t*)v0, (uint32_t*)k1, (uint64_t*)v1, K,
                                                    0, bits, &res)))
        return e;
      key = res ? (const uint32_t*)k1 : (const uint32_t*)k0;
      val = res ? (const uint64_t*)v1 : (const uint64_t*)v0;
    }
  }
  // Kernel scope over ranks ("spread"): the kept records stay on their rank
  // and are tiled there as consecutive parts of the global kept sequence;
  // only the cross-tile entries (first / last use of each line per tile
  // piece) and the per-tile weight / query counts travel, to rank 0, which
  // runs the cross-tile phase over all of them.  CTA scope
  // redistributes the kept records by CTA range instead (rd_exchange).
  const bool spread = c->comm != nullptr && !cta_scope;
  if (c->comm && !spread && (e = rd_exchange(c, cta_scope, &key, &val, &K))) return e;
  if (c->comm && cta_scope && K) {
    // the rank's CTA range, CTA-major: the same segment path as one rank
    void* sb;
    if ((e = ensure(c, B_RG_SEG, (K + 16) * 16 + 64, &sb))) return e;
    uint2* seg = (uint2*)sb;
    uint2* seg_long = seg + (K + 16);
    unsigned int* seg_cm = (unsigned int*)(seg_long + (K + 16));
    if ((e = cudaMemsetAsync(seg_cm, 0, 16, c->stream))) return e;
    CADV_LAUNCH(c, k_key_segments<<<grid_ls, 256, 0, c->stream>>>(key, K, seg, seg_long, seg_cm));
    bool done = false;
    if ((e = rd_segments(c, val, seg, seg_long, seg_cm, K, log2bins, nbins, d_hist, d_stats, O, &done))) return e;
    if (done) return cudaSuccess;
  }
  const uint64_t ntiles_loc = (K + TL_NOM - 1) / TL_NOM;
  uint64_t ntiles = ntiles_loc;  // tiles of all ranks (global tile ids)
  TilePos TP{0, 0, K};
  std::vector<uint64_t> kk;       // spread: (K, ntiles) of every rank
  if (spread) {
    const int G = c->nranks;
    void* cb;
    if ((e = ensure(c, B_COMM, (size_t)(2 + 2 * G) * 8 + 64, &cb))) return e;
    uint64_t* d = (uint64_t*)cb;
    const uint64_t mine[2] = {K, ntiles_loc};
    if ((e = cudaMemcpyAsync(d, mine, 16, cudaMemcpyHostToDevice, c->stream))) return e;
    if (c->comm->allgather(d, d + 2, 16, c->stream)) return cudaErrorUnknown;
    kk.resize(2 * G);
    if ((e = cudaMemcpyAsync(kk.data(), d + 2, 16 * G, cudaMemcpyDeviceToHost, c->stream))) return e;
    if ((e = cudaStreamSynchronize(c->stream))) return e;
    uint64_t kg = 0, tg = 0;
    for (int r = 0; r < G; ++r) {
      if (r == c->rank) { TP.pos_base = kg; TP.tile_base = (uint32_t)tg; }
      kg += kk[2 * r];
      tg += kk[2 * r + 1];
    }
    if (kg >= 0xffffffffull) return cudaErrorNotSupported;  // global kept positions are u32
    TP.k_glob = kg;
    ntiles = tg;
    if (kg == 0) return cudaSuccess;  // every rank sees it
  } else if (K == 0) {
    return cudaSuccess;
  }
  // ---- tiles
  c->counts[3] = ntiles_loc;
  void *bnd, *tw, *tq;
  if ((e = ensure(c, B_RD_XTMP, (3 * ntiles_loc + 8) * 4 + 64, &bnd))) return e;  // bounds + MODE 2 / MODE 1 lists
  if ((e = ensure(c, B_RD_TILEW, (ntiles + 2) * 8 * 2, &tw))) return e;
  if ((e = ensure(c, B_RD_TILEQ, (ntiles + 2) * 8 * 2, &tq))) return e;
  if (spread && ((e = cudaMemsetAsync(tw, 0, (ntiles + 2) * 4, c->stream)) ||
                 (e = cudaMemsetAsync(tq, 0, (ntiles + 2) * 4, c->stream))))
    return e;
  if (ntiles_loc)
    CADV_LAUNCH(c, k_tile_bounds<<<(unsigned)((ntiles_loc + 1 + 7) / 8), 256, 0, c->stream>>>(key, K, (uint32_t*)bnd,
                                                                                             ntiles_loc));
  // entries: at most one per kept record
  void* ent;
  size_t ent_bytes = K * (4 + 8 + 4 + 4 + 4 + 4 + 1 + 4 + 4 + 4 + 1) + 16 * 16;
  if ((e = ensure(c, B_RD_ENT, ent_bytes, &ent))) return e;
  EntryCols En;
  {
    uint8_t* p = (uint8_t*)ent;
    auto take = [&](size_t bytes) { uint8_t* q = p; p += (bytes + 15) & ~size_t(15); return q; };
    En.line = (uint64_t*)take(K * 8);
    En.seg = (uint32_t*)take(K * 4);
    En.tile = (uint32_t*)take(K * 4);
    En.f = (uint32_t*)take(K * 4);
    En.fa = (uint32_t*)take(K * 4);
    En.fw = (uint32_t*)take(K * 4);
    En.l = (uint32_t*)take(K * 4);
    En.lw = (uint32_t*)take(K * 4);
    En.ld = (uint32_t*)take(K * 4);
    En.ff = (uint8_t*)take(K);
    En.lf = (uint8_t*)take(K);
  }
  if (!(c->attr_set & (1u << 17))) {
    if ((e = cudaFuncSetAttribute(k_rd_tile<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(TileSmem))) ||
        (e = cudaFuncSetAttribute(k_rd_tile<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(TileSmem))) ||
        (e = cudaFuncSetAttribute(k_rd_tile<2>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  (int)sizeof(TileSmemWide))))
      return e;
    c->attr_set |= 1u << 17;
  }
  uint32_t* tile_w = (uint32_t*)tw;
  uint32_t* tile_q = (uint32_t*)tq;
  uint32_t* wide_list = (uint32_t*)bnd + (ntiles_loc + 2);
  if (ntiles_loc) {
    CADV_LAUNCH(c, k_rd_tile<0><<<(unsigned)ntiles_loc, TL_NT, sizeof(TileSmem), c->stream>>>(
                       key, val, K, (const uint32_t*)bnd, (uint32_t)ntiles_loc, log2bins, nbins, d_hist, d_stats,
                       tile_w, tile_q, En, sc, wide_list, O, TP, nullptr, nullptr));
    if ((e = cudaGetLastError())) return e;
  }
  unsigned long long cnt14[4];  // count[1..4]: entries, cross queries, MODE 2 tiles, MODE 1 tiles
  if ((e = cudaMemcpyAsync(cnt14, &sc->count[1], 32, cudaMemcpyDeviceToHost, c->stream))) return e;
  if ((e = cudaStreamSynchronize(c->stream))) return e;
  if (cnt14[3]) {
    CADV_LAUNCH(c, k_rd_tile<1><<<(unsigned)cnt14[3], TL_NT, sizeof(TileSmem), c->stream>>>(
                       key, val, K, (const uint32_t*)bnd, (uint32_t)ntiles_loc, log2bins, nbins, d_hist, d_stats,
                       tile_w, tile_q, En, sc, wide_list, O, TP, nullptr, nullptr));
    if ((e = cudaGetLastError())) return e;
  }
  if (cnt14[2]) {
    CADV_LAUNCH(c, k_rd_tile<2><<<(unsigned)cnt14[2], TL_NT, sizeof(TileSmemWide), c->stream>>>(
                       key, val, K, (const uint32_t*)bnd, (uint32_t)ntiles_loc, log2bins, nbins, d_hist, d_stats,
                       tile_w, tile_q, En, sc, wide_list, O, TP, nullptr, nullptr));
    if ((e = cudaGetLastError())) return e;
  }
  unsigned long long nent = cnt14[0];
  if (cnt14[2] || cnt14[3]) {  // the wider-key tiles add entries too
    if ((e = cudaMemcpyAsync(&nent, &sc->count[1], 8, cudaMemcpyDeviceToHost, c->stream))) return e;
    if ((e = cudaStreamSynchronize(c->stream))) return e;
  }
  c->counts[1] = nent;
  // tile weight / local-query counts (u64); spread: summed over ranks (each rank filled its own tiles)
  void* wide;
  if ((e = ensure(c, B_RD_XQ2, (ntiles + 2) * 16 + 64, &wide))) return e;
  unsigned long long* w64 = (unsigned long long*)wide;
  unsigned long long* q64 = w64 + (ntiles + 2);
  if (spread) {
    CADV_LAUNCH(c, k_widen<<<64, 256, 0, c->stream>>>(tile_w, w64, ntiles, ntiles + 1));
    CADV_LAUNCH(c, k_widen<<<64, 256, 0, c->stream>>>(tile_q, q64, ntiles, ntiles + 1));
    if (c->comm->allreduce_sum_u64((uint64_t*)w64, 2 * (ntiles + 2), c->stream)) return cudaErrorUnknown;
    // each rank links the entries of the lines it owns (line hash)
    if ((e = exchange_entries_by_line(c, &En, &nent))) return e;
  } else if (nent) {
    CADV_LAUNCH(c, k_widen<<<64, 256, 0, c->stream>>>(tile_w, w64, ntiles, ntiles + 1));
    CADV_LAUNCH(c, k_widen<<<64, 256, 0, c->stream>>>(tile_q, q64, ntiles, ntiles + 1));
  }
  if (nent == 0 && !spread) return cudaSuccess;
  // ---- cross-tile phase
  // tile prefix sums of weights and local query counts
  unsigned long long* twb = (unsigned long long*)((uint8_t*)tw + (ntiles + 2) * 8);
  unsigned long long* tqb = (unsigned long long*)((uint8_t*)tq + (ntiles + 2) * 8);
  if ((e = exclusive_scan_u64(c, (const uint64_t*)w64, (uint64_t*)twb, ntiles + 1))) return e;
  if ((e = exclusive_scan_u64(c, (const uint64_t*)q64, (uint64_t*)tqb, ntiles + 1))) return e;
  // sort entries by (seg, line, tile)
  void *ek0, *ek1, *ei0, *ei1;
  if ((e = ensure(c, B_RD_ENT_KEY0, nent * 8, &ek0)) || (e = ensure(c, B_RD_ENT_KEY1, nent * 8, &ek1)) ||
      (e = ensure(c, B_RD_ENT_IDX0, nent * 4, &ei0)) || (e = ensure(c, B_RD_ENT_IDX1, nent * 4, &ei1)))
    return e;
  unsigned long long* mm = &sc->rd_line_min;  // rd_line_min, rd_line_max are adjacent
  if ((e = cudaMemsetAsync(mm, 0xff, 8, c->stream)) || (e = cudaMemsetAsync(mm + 1, 0, 8, c->stream))) return e;
  CADV_LAUNCH(c, k_ent_line_range<<<grid_ls, 256, 0, c->stream>>>(En.line, nent, mm, mm + 1));
  unsigned long long hmm[2];
  if ((e = cudaMemcpyAsync(hmm, mm, 16, cudaMemcpyDeviceToHost, c->stream))) return e;
  if ((e = cudaStreamSynchronize(c->stream))) return e;
  uint64_t minl = hmm[0];
  int lb = bits_for(hmm[1] - hmm[0]);
  int tb = bits_for(ntiles);
  int sb = cta_scope ? bits_for(c->max_cta) : 0;
  const uint32_t* order = nullptr;
  if (nent == 0) {
    // (spread: this rank owns no line; it still takes part in the exchanges below)
  } else if (sb + lb + tb <= 64) {
    CADV_LAUNCH(c, k_ent_key<<<grid_ls, 256, 0, c->stream>>>(En.seg, En.line, En.tile, nent, minl, lb, tb, -1, nullptr,
                                                             (uint64_t*)ek0, (uint32_t*)ei0));
    int res;
    if ((e = radix_sort_pairs<uint64_t, uint32_t>(c, (uint64_t*)ek0, (uint32_t*)ei0, (uint64_t*)ek1, (uint32_t*)ei1,
                                                  nent, 0, sb + lb + tb, &res)))
      return e;
    order = res ? (const uint32_t*)ei1 : (const uint32_t*)ei0;
  } else {
    // one field at a time, least significant first (stable passes)
    const uint32_t* idx = nullptr;
    uint32_t* ib[2] = {(uint32_t*)ei0, (uint32_t*)ei1};
    int cur = 0;
    int fb[3] = {tb, lb, sb};
    for (int field = 0; field < 3; ++field) {
      if (fb[field] == 0) continue;
      uint32_t* dst = ib[cur];
      uint32_t* alt = ib[cur ^ 1];
      CADV_LAUNCH(c, k_ent_key<<<grid_ls, 256, 0, c->stream>>>(En.seg, En.line, En.tile, nent, minl, lb, tb, field,
                                                               idx, (uint64_t*)ek1, alt));
      // keys in ek1, idx in alt -> sort into (ek0, dst) or back
      int res;
      if ((e = radix_sort_pairs<uint64_t, uint32_t>(c, (uint64_t*)ek1, alt, (uint64_t*)ek0, dst, nent, 0, fb[field],
                                                    &res)))
        return e;
      idx = res ? dst : alt;
      cur = (idx == ib[0]) ? 1 : 0;
    }
    order = idx ? idx : (const uint32_t*)ei0;
  }
  // link
  void *xq, *xq2;
  if ((e = ensure(c, B_RD_XQ, nent * (4 + 4 + 8 + 8) + 64, &xq))) return e;
  CrossOut X;
  X.xpos = (uint32_t*)xq;
  X.xq = X.xpos + nent;
  X.part = (int64_t*)(((uintptr_t)(X.xq + nent) + 15) & ~(uintptr_t)15);
  X.xline = (uint64_t*)(X.part + nent);
  if (nent)
    CADV_LAUNCH(c, k_link<<<grid_ls, 256, 0, c->stream>>>(order, nent, En, twb, tqb, nbins, d_hist, d_stats, X, sc, O));
  unsigned long long M = 0;
  if ((e = cudaMemcpyAsync(&M, &sc->count[2], 8, cudaMemcpyDeviceToHost, c->stream))) return e;
  if ((e = cudaStreamSynchronize(c->stream))) return e;
  if (!nent) M = 0;
  if (spread) {
    // the queries to the ranks holding their positions (collective)
    std::vector<uint64_t> base(c->nranks + 1, 0);
    for (int r = 0; r < c->nranks; ++r) base[r + 1] = base[r] + kk[2 * r];
    if ((e = exchange_queries_by_pos(c, &X, &M, base))) return e;
  }
  c->counts[2] = M;
  if (M == 0 && !spread) return cudaSuccess;
  if ((e = ensure(c, B_RD_ENT_IDX0, M * 4 + 64, &ei0)) || (e = ensure(c, B_RD_ENT_IDX1, M * 4 + 64, &ei1))) return e;
  // sort cross queries by position, then count inversions of their previous uses
  if ((e = ensure(c, B_RD_ENT_KEY1, M * 8 + nent * 8, &ek1))) return e;
  if ((e = ensure(c, B_SORT_K0, M * 4 * 2 + 64, &xq2))) return e;
  uint32_t* pk0 = (uint32_t*)xq2;
  uint32_t* pk1 = pk0 + M;
  uint32_t* pi0 = (uint32_t*)ei0;
  uint32_t* pi1 = (uint32_t*)ei1;
  int res = 0;
  if (M) {
    if ((e = cudaMemcpyAsync(pk0, X.xpos, M * 4, cudaMemcpyDeviceToDevice, c->stream))) return e;
    CADV_LAUNCH(c, k_iota<<<grid_ls, 256, 0, c->stream>>>(pi0, M));
    // (positions < the global kept count: only its bits, 3 passes instead of 4 below 2^27)
    if ((e = radix_sort_pairs<uint32_t, uint32_t>(c, pk0, pi0, pk1, pi1, M, 0, bits_for(TP.k_glob), &res))) return e;
  }
  const uint32_t* ord = res ? pi1 : pi0;
  // keys = previous use in position order; ids = cross-query index
  uint32_t* ka = (uint32_t*)ek0;
  uint32_t* kb = ka + M;
  uint32_t* ia = (uint32_t*)ek1;
  uint32_t* ib = ia + M;
  void* cntb;
  if ((e = ensure(c, B_GATHER, M * 4 + 64, &cntb))) return e;
  uint32_t* cnt = (uint32_t*)cntb;
  if ((e = ensure(c, B_RD_ENT_KEY0, M * 8 + 64, &ek0))) return e;
  ka = (uint32_t*)ek0;
  kb = ka + M;
  if (M) {
    CADV_LAUNCH(c, k_iota_gather<<<grid_ls, 256, 0, c->stream>>>(ord, X.xq, M, ka, ia, cnt));
    if (!(c->attr_set & (1u << 18))) {
      if ((e = cudaFuncSetAttribute(k_merge_count_block, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    (int)sizeof(MergeBlockSmem))))
        return e;
      c->attr_set |= 1u << 18;
    }
    CADV_LAUNCH(c, k_merge_count_block<<<(unsigned)((M + MC_BLOCK - 1) / MC_BLOCK), 512, sizeof(MergeBlockSmem),
                                         c->stream>>>(ka, ia, kb, ib, M, cnt));
    std::swap(ka, kb);
    std::swap(ia, ib);
    for (uint64_t w = MC_BLOCK; w < M; w <<= 1) {
      if (getenv("CADV_MERGE_UNTILED"))
        CADV_LAUNCH(c, k_merge_count<<<grid_ls, 256, 0, c->stream>>>(ka, ia, kb, ib, M, w, cnt));
      else
        CADV_LAUNCH(c, k_merge_count_tiled<<<(unsigned)((M + MPB_T - 1) / MPB_T), MPB_NT, 0, c->stream>>>(
                           ka, ia, kb, ib, M, w, cnt));
      std::swap(ka, kb);
      std::swap(ia, ib);
    }
  }
  // ka: this rank's previous uses in ascending order; with ranks, the queries
  // of the earlier ranks (all at smaller positions) add their larger ones
  if (spread && (e = add_earlier_ranks(c, ka, M, X.xq, cnt))) return e;
  if (M)
    CADV_LAUNCH(c, k_cross_final<<<grid_ls, 256, 0, c->stream>>>(X.part, cnt, M, log2bins, nbins, d_hist, d_stats, sc,
                                                                        O, X.xline));
  return cudaGetLastError();
}

}  // namespace cadv
