// common.cuh — shared device helpers of libcadv (sm_100a only).
//
// Nothing here is shared with oracle/ (the CPU reference); the two sides are
// independent implementations of the same definitions.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/cadv.h"

#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ < 1000)
#error "libcadv is written for sm_100a (B200) only"
#endif

namespace cadv {

constexpr uint32_t FULL = 0xffffffffu;

// ------------------------------------------------------------------ records
// meta byte: bits 0-1 kind, bits 2-4 log2(bytes), bits 5-7 reserved (zero)
__device__ __forceinline__ uint32_t kind_of(uint8_t m) { return m & 3u; }
__device__ __forceinline__ bool is_mem(uint8_t m) { return (m & 3u) < 2u; }
__device__ __forceinline__ bool is_store(uint8_t m) { return (m & 3u) == 1u; }
__device__ __forceinline__ bool is_bb(uint8_t m) { return (m & 3u) == 2u; }

// Per-record validity over the columns the caller reads (include/cadv.h).
__device__ __forceinline__ bool meta_ok(uint8_t m) {
  return (m & 3u) != 3u && (m >> 5) == 0 && (((m & 3u) == 2u) || ((m >> 2) & 7u) <= 4u);
}
// (any 64-bit address is valid; the reuse path's own limit on line
// numbers, < 2^58, is CADV_ERR_UNSUPPORTED, not a bad record)
__device__ __forceinline__ bool addr_ok(uint64_t a, uint8_t m) {
  if ((m & 3u) == 2u) return true;
  uint64_t bytes = 1ull << ((m >> 2) & 7u);
  return (a & (bytes - 1)) == 0;
}

// ------------------------------------------------------------------ data objects
// Data-centric attribution (cadv_data_centric): n line-granular
// object extents [lo[k], hi[k]) in ascending, disjoint order (the host builds
// them from the byte ranges).  Row of a line = the extent holding it, or n
// (unattributed).  Binary search; lo / hi may live in global or shared memory.
struct ObjTab {
  const uint64_t* lo;
  const uint64_t* hi;
  uint32_t n;
};
__device__ __forceinline__ uint32_t obj_row(const uint64_t* lo, const uint64_t* hi, uint32_t n, uint64_t line) {
  uint32_t a = 0, b = n;  // a = number of extents starting at or before the line
  while (a < b) {
    const uint32_t m = (a + b) >> 1;
    if (lo[m] <= line) a = m + 1;
    else b = m;
  }
  return (a && line < hi[a - 1]) ? a - 1 : n;
}
__device__ __forceinline__ uint32_t obj_row(const ObjTab& O, uint64_t line) { return obj_row(O.lo, O.hi, O.n, line); }

// ------------------------------------------------------------------ lane helpers
__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31u; }
__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t r;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t lanemask_le() {
  uint32_t r;
  asm("mov.u32 %0, %%lanemask_le;" : "=r"(r));
  return r;
}

// ------------------------------------------------------------------ block scan
// Exclusive scan of one u32 per thread over a block of NT threads.  `ws` must
// hold NT/32 + 1 words.  Returns the exclusive prefix; *total = block sum.
template <int NT>
__device__ __forceinline__ uint32_t block_exclusive_scan(uint32_t v, uint32_t* ws, uint32_t* total) {
  const uint32_t lane = lane_id(), warp = threadIdx.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(FULL, x, o);
    if (lane >= (uint32_t)o) x += y;
  }
  if (lane == 31) ws[warp] = x;
  __syncthreads();
  if (warp == 0) {
    uint32_t s = lane < NT / 32 ? ws[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(FULL, s, o);
      if (lane >= (uint32_t)o) s += y;
    }
    if (lane < NT / 32) ws[lane] = s;  // inclusive warp prefix
    if (lane == NT / 32 - 1) ws[NT / 32] = s;
  }
  __syncthreads();
  uint32_t base = warp ? ws[warp - 1] : 0;
  *total = ws[NT / 32];
  __syncthreads();
  return base + x - v;
}

// Inclusive max-scan of one u32 per thread over the block (same workspace rule).
template <int NT>
__device__ __forceinline__ uint32_t block_inclusive_max(uint32_t v, uint32_t* ws) {
  const uint32_t lane = lane_id(), warp = threadIdx.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(FULL, x, o);
    if (lane >= (uint32_t)o) x = max(x, y);
  }
  if (lane == 31) ws[warp] = x;
  __syncthreads();
  if (warp == 0) {
    uint32_t s = lane < NT / 32 ? ws[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(FULL, s, o);
      if (lane >= (uint32_t)o) s = max(s, y);
    }
    if (lane < NT / 32) ws[lane] = s;
  }
  __syncthreads();
  uint32_t r = warp ? max(ws[warp - 1], x) : x;
  __syncthreads();
  return r;
}

// ------------------------------------------------------------------ TMA 1-D bulk copies
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_barrier_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
// Bulk global->shared copy (cp.async.bulk, SASS UBLKCP), completion counted
// on `bar` in bytes.  dst/src 16-byte aligned, bytes a multiple of 16.
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(phase)
      : "memory");
}

// One column of a tile staged in shared memory by a 1-D bulk copy.  The
// copied byte range is the 16-byte-aligned hull of the records [lo, hi);
// the extra bytes lie in the same 16-byte chunks as valid records, so they
// are always mapped.  Element i lives at smem + delta + (i - lo) * size.
struct ColStage {
  uint32_t delta;  // byte offset of record lo inside the staged buffer
};

template <typename T>
__device__ __forceinline__ uint32_t stage_column(const T* base, uint64_t lo, uint64_t hi, void* dst, uint64_t* bar,
                                                 uint32_t* delta) {
  uintptr_t b = (uintptr_t)(base + lo), e = (uintptr_t)(base + hi);
  uintptr_t a0 = b & ~(uintptr_t)15, a1 = (e + 15) & ~(uintptr_t)15;
  *delta = (uint32_t)(b - a0);
  uint32_t bytes = (uint32_t)(a1 - a0);
  if (bytes) tma_load_1d(dst, (const void*)a0, bytes, bar);
  return bytes;
}
// bytes a column of `cnt` records of type T can occupy once staged
template <typename T>
__host__ __device__ constexpr uint32_t stage_bytes(uint32_t cnt) {
  return ((cnt * (uint32_t)sizeof(T) + 31u) & ~15u);
}

// ------------------------------------------------------------------ reuse-distance binning
// LINEAR: d <= nbins-3 exact, else nbins-2.  LOG2: 0 -> 0, d in
// [2^(k-1), 2^k-1] -> k while k <= nbins-3, else nbins-2.  (∞ = nbins-1.)
__device__ __forceinline__ uint32_t rd_bin(uint64_t d, int log2bins, uint32_t nbins) {
  if (!log2bins) return d <= (uint64_t)(nbins - 3) ? (uint32_t)d : nbins - 2;
  if (d == 0) return 0;
  uint32_t k = 64u - (uint32_t)__clzll((long long)d);
  return k <= nbins - 3 ? k : nbins - 2;
}

}  // namespace cadv
