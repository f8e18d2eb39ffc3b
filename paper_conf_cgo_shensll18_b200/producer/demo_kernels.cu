// demo_kernels.cu — hand-instrumented sm_100a kernels that produce REAL
// traces on the B200 through include/cadv_record.cuh:
// the vecAdd of config 1 and the naive / shared-memory-tiled SGEMM of
// config 2, each compiled twice (TR = 0: plain, TR = 1: instrumented) so the
// instrumentation overhead can be measured against the paper's 10-120x
// (P:L396-398).  Sites and control flow follow tracegen's recipes (DESIGN.md
// §5), so the closed forms pinned for the generated C1 / C2 traces hold for
// the device-produced ones.  libcadv_demo.so; C ABI below.
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/cadv_record.cuh"

namespace {

enum { V_ENTRY, V_HDR, V_BODY, V_EXIT, V_LDA, V_LDB, V_STC };

template <bool TR>
__global__ void k_vecadd(const float* __restrict__ a, const float* __restrict__ b, float* __restrict__ c, int n,
                         cadv_dev_trace T) {
  const int t = blockIdx.x * blockDim.x + threadIdx.x;
  if (TR) cadv_record_bb(T, V_ENTRY);
  for (int i = t;; i += gridDim.x * blockDim.x) {  // grid-stride (config 1: one CTA)
    if (TR) cadv_record_bb(T, V_HDR);
    if (i >= n) break;
    if (TR) {
      cadv_record_bb(T, V_BODY);
      cadv_record_load(T, a + i, 4, V_LDA);
    }
    const float x = a[i];
    if (TR) cadv_record_load(T, b + i, 4, V_LDB);
    const float y = b[i];
    if (TR) cadv_record_store(T, c + i, 4, V_STC);
    c[i] = x + y;
  }
  if (TR) {
    __syncwarp();  // the warp reconverges at the exit block
    cadv_record_bb(T, V_EXIT);
  }
}

constexpr int TS = 16;

// sites: naive 0..6, tiled 7..13 (tracegen "sgemm": ld A, ld B, st C, entry, header, body, exit)
template <bool TR>
__global__ void k_sgemm_naive(const float* __restrict__ A, const float* __restrict__ B, float* __restrict__ C, int n,
                              int bb, cadv_dev_trace T) {
  const int row = blockIdx.y * TS + threadIdx.y, col = blockIdx.x * TS + threadIdx.x;
  if (TR && bb) cadv_record_bb(T, 3);
  float acc = 0.f;
  for (int k = 0; k < n; ++k) {
    if (TR) {
      if (bb) { cadv_record_bb(T, 4); cadv_record_bb(T, 5); }
      cadv_record_load(T, A + (size_t)row * n + k, 4, 0);
      cadv_record_load(T, B + (size_t)k * n + col, 4, 1);
    }
    acc += A[(size_t)row * n + k] * B[(size_t)k * n + col];
  }
  if (TR) {
    if (bb) cadv_record_bb(T, 4);
    cadv_record_store(T, C + (size_t)row * n + col, 4, 2);
  }
  C[(size_t)row * n + col] = acc;
  if (TR && bb) cadv_record_bb(T, 6);
}

template <bool TR>
__global__ void k_sgemm_tiled(const float* __restrict__ A, const float* __restrict__ B, float* __restrict__ C, int n,
                              int bb, cadv_dev_trace T) {
  __shared__ float As[TS][TS], Bs[TS][TS];
  const int tx = threadIdx.x, ty = threadIdx.y;
  const int row = blockIdx.y * TS + ty, col = blockIdx.x * TS + tx;
  if (TR && bb) cadv_record_bb(T, 10);
  float acc = 0.f;
  for (int t = 0; t < n / TS; ++t) {
    if (TR) {
      if (bb) { cadv_record_bb(T, 11); cadv_record_bb(T, 12); }
      cadv_record_load(T, A + (size_t)row * n + t * TS + tx, 4, 7);
      cadv_record_load(T, B + (size_t)(t * TS + ty) * n + col, 4, 8);
    }
    As[ty][tx] = A[(size_t)row * n + t * TS + tx];
    Bs[ty][tx] = B[(size_t)(t * TS + ty) * n + col];
    __syncthreads();
#pragma unroll
    for (int k = 0; k < TS; ++k) acc += As[ty][k] * Bs[k][tx];
    __syncthreads();
  }
  if (TR) {
    if (bb) cadv_record_bb(T, 11);
    cadv_record_store(T, C + (size_t)row * n + col, 4, 9);
  }
  C[(size_t)row * n + col] = acc;
  if (TR && bb) cadv_record_bb(T, 13);
}

__global__ void k_fill(float* p, size_t n, float s) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    p[i] = s * (float)(i % 97);
}

struct Bufs {
  float *a = nullptr, *b = nullptr, *c = nullptr;
  ~Bufs() {
    cudaFree(a);
    cudaFree(b);
    cudaFree(c);
  }
  cudaError_t alloc(size_t na, size_t nb, size_t nc) {
    cudaError_t e;
    if ((e = cudaMalloc(&a, na * 4)) || (e = cudaMalloc(&b, nb * 4)) || (e = cudaMalloc(&c, nc * 4))) return e;
    k_fill<<<256, 256>>>(a, na, 0.5f);
    k_fill<<<256, 256>>>(b, nb, 0.25f);
    return cudaGetLastError();
  }
};

// times `launch()` over `reps` launches with CUDA events (after one warm-up)
template <class F>
cudaError_t timed(F launch, int reps, float* ms) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaError_t e;
  launch();
  if ((e = cudaDeviceSynchronize())) return e;
  cudaEventRecord(e0);
  for (int r = 0; r < reps; ++r) launch();
  cudaEventRecord(e1);
  if ((e = cudaEventSynchronize(e1))) return e;
  float t = 0.f;
  cudaEventElapsedTime(&t, e0, e1);
  if (ms) *ms = t / reps;
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  return cudaGetLastError();
}

}  // namespace

extern "C" {

// vecAdd over n fp32 with a grid-stride loop (config 1: 1 CTA x 64 threads).  T == NULL: the plain kernel,
// timed over `reps` launches.  Else the instrumented kernel writes its trace
// from position 0 (*T->count and the winst counters are reset before every
// launch); after `reps` timed launches the buffer holds the last launch's
// trace.  Returns a cudaError_t.
__attribute__((visibility("default"))) int cadv_demo_vecadd(int n, int ctas, int threads, const cadv_dev_trace* T,
                                                            int reps, float* ms) {
  Bufs B;
  cudaError_t e = B.alloc(n, n, n);
  if (e) return e;
  const size_t warps = (size_t)ctas * ((threads + 31) / 32);
  if (!T) return timed([&] { k_vecadd<false><<<ctas, threads>>>(B.a, B.b, B.c, n, cadv_dev_trace{}); }, reps, ms);
  const cadv_dev_trace T1 = *T;
  return timed([&] {
    cudaMemsetAsync(T1.count, 0, 8);
    cudaMemsetAsync(T1.winst_ctr, 0, 8 * warps);
    k_vecadd<true><<<ctas, threads>>>(B.a, B.b, B.c, n, T1);
  }, reps < 1 ? 1 : reps, ms);
}

// Config-2 SGEMM n^3 with 16 x 16 CTAs: variant 0 naive, 1 tiled; bb = 1 adds
// the basic-block records.  CTA ids start at cta_base.  The trace is appended
// at the current *T->count (call naive then tiled for the C2 trace); timed
// launches rewrite the same positions, so the buffer ends with one launch.
__attribute__((visibility("default"))) int cadv_demo_sgemm(int n, int variant, int bb, const cadv_dev_trace* T,
                                                           uint32_t cta_base, int reps, float* ms) {
  if (n % TS) return (int)cudaErrorInvalidValue;
  Bufs B;
  cudaError_t e = B.alloc((size_t)n * n, (size_t)n * n, (size_t)n * n);
  if (e) return e;
  const dim3 grid(n / TS, n / TS), block(TS, TS);
  const size_t warps = (size_t)grid.x * grid.y * (TS * TS / 32);
  if (!T) {
    return timed([&] {
      if (variant) k_sgemm_tiled<false><<<grid, block>>>(B.a, B.b, B.c, n, bb, cadv_dev_trace{});
      else k_sgemm_naive<false><<<grid, block>>>(B.a, B.b, B.c, n, bb, cadv_dev_trace{});
    }, reps, ms);
  }
  cadv_dev_trace T1 = *T;
  T1.cta_base = cta_base;
  unsigned long long start = 0;
  if ((e = cudaMemcpy(&start, T1.count, 8, cudaMemcpyDeviceToHost))) return e;
  return timed([&] {
    cudaMemcpyAsync(T1.count, &start, 8, cudaMemcpyHostToDevice);
    cudaMemsetAsync(T1.winst_ctr, 0, 8 * warps);
    if (variant) k_sgemm_tiled<true><<<grid, block>>>(B.a, B.b, B.c, n, bb, T1);
    else k_sgemm_naive<true><<<grid, block>>>(B.a, B.b, B.c, n, bb, T1);
  }, reps < 1 ? 1 : reps, ms);
}

}  // extern "C"
