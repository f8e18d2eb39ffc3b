/* cadv_record.cuh — device-side trace producer for hand-instrumented sm_100a
 * kernels (the step before the analysed hot path).
 *
 * the instrumentation records, per dynamic memory access,
 * the address, access width, the executing CTA and thread, "appended to a
 * trace buffer by atomic operations"; P:L396-398 blames those per-access
 * atomics for most of the 10-120x profiling overhead.  Here one elected lane
 * per warp-level instruction reserves the slots of all active lanes with ONE
 * atomicAdd, so the records of a warp instruction are contiguous and in lane
 * order (warp_contiguous traces, include/cadv.h), and the same lane numbers
 * the instruction with the per-(CTA, warp, family) counter `winst` that the
 * analyses group by (reading R9).
 *
 * Usage inside a kernel (the buffer lives in device memory; see
 * paper_conf_cgo_shensll18_b200/producer/__init__.py for a host-side allocator):
 *     cadv_record_bb(T, SITE_LOOP);                 // a basic block entered
 *     cadv_record_load(T, &a[i], sizeof a[i], SITE_LD_A);  float x = a[i];
 *     cadv_record_store(T, &c[i], sizeof c[i], SITE_ST_C); c[i] = x;
 * Call sites must be reached by the lanes that execute the access (the active
 * mask of the call is the warp instruction's lane set); place __syncwarp()
 * where the program reconverges if the analysis should see one group there.
 * Records past `capacity` are dropped (count still advances: check it).
 */
#ifndef CADV_RECORD_CUH
#define CADV_RECORD_CUH

#include <stdint.h>

typedef struct {
  uint64_t *addr;                 /* byte address (0 for BB records)              */
  uint32_t *cta;                  /* cta_base + linear blockIdx                   */
  uint16_t *tid;                  /* linear threadIdx (< 1024)                    */
  uint32_t *site;                 /* static site id                               */
  uint32_t *winst;                /* per (cta, warp32, family) instruction number */
  uint8_t *meta;                  /* kind | log2(bytes) << 2                      */
  unsigned long long *count;      /* records appended so far (device, zeroed)     */
  unsigned long long capacity;    /* length of the columns                        */
  uint32_t *winst_ctr;            /* [2 * warps of the launch], zeroed per launch */
  uint32_t cta_base;              /* makes CTA ids unique across launches         */
} cadv_dev_trace;

#ifdef __CUDACC__

__device__ __forceinline__ uint32_t cadv_linear_cta_() {
  return blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
}
__device__ __forceinline__ uint32_t cadv_linear_tid_() {
  return threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
}

/* family 0 = memory (load / store), 1 = basic block (separate winst numbering) */
__device__ __forceinline__ void cadv_emit_(const cadv_dev_trace &T, uint64_t a, uint8_t meta, uint32_t site,
                                           uint32_t family) {
  const uint32_t mask = __activemask();
  const uint32_t t = cadv_linear_tid_(), lane = t & 31u;
  const uint32_t leader = (uint32_t)__ffs(mask) - 1u;
  const uint32_t rank = __popc(mask & ((1u << lane) - 1u));
  unsigned long long base = 0;
  uint32_t w = 0;
  if (lane == leader) {
    base = atomicAdd(T.count, (unsigned long long)__popc(mask));
    const uint32_t wpc = (blockDim.x * blockDim.y * blockDim.z + 31u) >> 5;
    w = atomicAdd(&T.winst_ctr[2u * (cadv_linear_cta_() * wpc + (t >> 5)) + family], 1u);
  }
  base = __shfl_sync(mask, base, leader);
  w = __shfl_sync(mask, w, leader);
  const unsigned long long i = base + rank;
  if (i < T.capacity) {
    T.addr[i] = a;
    T.cta[i] = T.cta_base + cadv_linear_cta_();
    T.tid[i] = (uint16_t)t;
    T.site[i] = site;
    T.winst[i] = w;
    T.meta[i] = meta;
  }
}

__device__ __forceinline__ uint8_t cadv_meta_(uint32_t kind, uint32_t bytes) {
  uint32_t lg = 0;
  while ((1u << lg) < bytes) ++lg;
  return (uint8_t)(kind | (lg << 2));
}

__device__ __forceinline__ void cadv_record_load(const cadv_dev_trace &T, const void *p, uint32_t bytes,
                                                 uint32_t site) {
  cadv_emit_(T, (uint64_t)(uintptr_t)p, cadv_meta_(0u, bytes), site, 0u);
}
__device__ __forceinline__ void cadv_record_store(const cadv_dev_trace &T, const void *p, uint32_t bytes,
                                                  uint32_t site) {
  cadv_emit_(T, (uint64_t)(uintptr_t)p, cadv_meta_(1u, bytes), site, 0u);
}
__device__ __forceinline__ void cadv_record_bb(const cadv_dev_trace &T, uint32_t site) {
  cadv_emit_(T, 0ull, (uint8_t)2u, site, 1u);
}

#endif /* __CUDACC__ */
#endif /* CADV_RECORD_CUH */
