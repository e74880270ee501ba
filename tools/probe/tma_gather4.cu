// tma_gather4.cu -- throughput of Blackwell TMA tile::gather4 (cp.async.bulk.tensor.2d ... tile::gather4):
// four random rows of a 2D fp32 tensor per request into shared memory, completion on an mbarrier.
// Rows of W floats from a table of T rows (T = products-shaped 2,449,029); W = 4 (the K = 1 SDDMM's 4-byte
// values fetched as 16-byte rows) and W = 48 (the K = 47 gathers).  Every thread of a warp issues its own
// requests into its own ring of slots (one mbarrier per slot); rows / s and GB/s over the whole grid,
// best over CTAs per SM.  A request that never completes is reported (bounded spin), not waited for.
#include <cstdio>
#include <cstdint>
#include <cuda.h>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t mix(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
  return x;
}
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int W, int SLOTS>
__global__ void __launch_bounds__(32) g4(const __grid_constant__ CUtensorMap tm, uint32_t T, int iters, int* bad,
                                         float* sink) {
  constexpr int SS = (4 * W + 31) / 32 * 32;  // slot stride in floats: 128-byte aligned TMA destinations
  __shared__ __align__(128) float buf[32 * SLOTS * SS];
  __shared__ __align__(8) uint64_t mb[32 * SLOTS];
  const int lane = threadIdx.x;
  for (int s = 0; s < SLOTS; ++s)
    asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_u32(&mb[lane * SLOTS + s])));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const uint32_t bytes = 4 * W * 4;
  uint32_t h = (blockIdx.x * 32 + lane) * 7919u + 1u;
  for (int i = 0; i < iters; ++i) {
    const int s = i % SLOTS;
    const uint32_t bar = smem_u32(&mb[lane * SLOTS + s]);
    if (i >= SLOTS) {  // wait for this slot's previous request (phase (i / SLOTS - 1) & 1)
      const uint32_t ph = (uint32_t)((i / SLOTS - 1) & 1);
      uint32_t ok = 0;
      long long t0 = clock64();
      while (!ok) {
        asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                     : "=r"(ok) : "r"(bar), "r"(ph) : "memory");
        if (!ok && clock64() - t0 > 2000000000ll) { atomicExch(bad, 1); return; }
      }
    }
    asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
    int32_t r[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) { h = mix(h + 0x9e3779b9u); r[q] = (int32_t)(h % T); }
    const uint32_t dst = smem_u32(&buf[(lane * SLOTS + s) * SS]);
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
        ::"r"(dst), "l"(&tm), "r"(0), "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(bar)
        : "memory");
  }
  for (int s = 0; s < SLOTS; ++s) {
    const int last = iters - 1 - ((iters - 1 - s + SLOTS) % SLOTS);  // last request that used slot s
    if (last < 0) continue;
    const uint32_t ph = (uint32_t)((last / SLOTS) & 1);
    uint32_t ok = 0;
    long long t0 = clock64();
    while (!ok) {
      asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                   : "=r"(ok) : "r"(smem_u32(&mb[lane * SLOTS + s])), "r"(ph) : "memory");
      if (!ok && clock64() - t0 > 2000000000ll) { atomicExch(bad, 2); return; }
    }
  }
  if (buf[lane] == 12345.f) *sink = buf[lane];
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                             const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

template <int W, int SLOTS>
static void run(EncodeFn enc, float* t, uint32_t T, int* bad, float* sink, int sms) {
  CUtensorMap tm;
  cuuint64_t dims[2] = {(cuuint64_t)W, (cuuint64_t)T};
  cuuint64_t strides[1] = {(cuuint64_t)W * 4};
  cuuint32_t box[2] = {(cuuint32_t)W, 1};
  cuuint32_t es[2] = {1, 1};
  CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, t, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) { printf("{\"W\": %d, \"encode_error\": %d}\n", W, (int)r); return; }
  const int iters = 4096;
  for (int cps : {4, 8, 16}) {
    cudaMemset(bad, 0, 4);
    g4<W, SLOTS><<<sms * cps, 32>>>(tm, T, 64, bad, sink);
    cudaError_t e = cudaDeviceSynchronize();
    int hb = 0;
    cudaMemcpy(&hb, bad, 4, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess || hb) { printf("{\"W\": %d, \"ctas_per_sm\": %d, \"error\": \"%s\", \"bad\": %d}\n", W, cps, cudaGetErrorString(e), hb); return; }
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    cudaEventRecord(a);
    g4<W, SLOTS><<<sms * cps, 32>>>(tm, T, iters, bad, sink);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    cudaMemcpy(&hb, bad, 4, cudaMemcpyDeviceToHost);
    const double rows = (double)sms * cps * 32 * iters * 4;
    printf("{\"W\": %d, \"slots_per_thread\": %d, \"ctas_per_sm\": %d, \"rows_per_s_G\": %.1f, \"GBps\": %.1f, \"bad\": %d}\n",
           W, SLOTS, cps, rows / (ms * 1e-3) / 1e9, rows * W * 4 / (ms * 1e-3) / 1e9, hb);
  }
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
  if (!fn) { printf("no cuTensorMapEncodeTiled\n"); return 1; }
  const uint32_t T = 2449029;
  float* t; int* bad; float* sink;
  cudaMalloc(&t, (size_t)T * 48 * 4);
  cudaMemset(t, 0, (size_t)T * 48 * 4);
  cudaMalloc(&bad, 4); cudaMalloc(&sink, 4);
  run<4, 8>((EncodeFn)fn, t, T, bad, sink, sms);
  run<48, 1>((EncodeFn)fn, t, T, bad, sink, sms);
  return 0;
}
