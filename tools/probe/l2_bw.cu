// l2_bw.cu -- measured L2 read bandwidth of this B200 (the roof of gathers served by L2).
// A persistent grid (all SMs, 8 x 256 threads each) reads a buffer that fits in L2 (48 MB)
// with 16-byte loads, many passes; bytes read / time.  Also the HBM read bandwidth with a
// 4 GB buffer for reference.  Prints one JSON line.
#include <cstdio>
#include <cuda_runtime.h>

__global__ void rd(const float4* __restrict__ p, size_t n, int passes, float* sink) {
  float4 acc = make_float4(0, 0, 0, 0);
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  for (int r = 0; r < passes; ++r)
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += stride) {
      float4 v = __ldcg(p + i);
      acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
  if (acc.x + acc.y + acc.z + acc.w == 12345.f) *sink = acc.x;
}

static double bw(size_t bytes, int passes, int reps) {
  float4* p; float* sink;
  cudaMalloc(&p, bytes); cudaMalloc(&sink, 4);
  cudaMemset(p, 0, bytes);
  int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const size_t n = bytes / 16;
  rd<<<sms * 8, 256>>>(p, n, 1, sink);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  double best = 0;
  for (int r = 0; r < reps; ++r) {
    cudaEventRecord(a);
    rd<<<sms * 8, 256>>>(p, n, passes, sink);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    const double gbs = (double)bytes * passes / (ms * 1e-3) / 1e9;
    if (gbs > best) best = gbs;
  }
  cudaFree(p); cudaFree(sink);
  return best;
}

int main() {
  const double l2 = bw(48ull << 20, 50, 5);
  const double hbm = bw(4ull << 30, 1, 5);
  printf("{\"l2_read_gbs\": %.1f, \"hbm_read_gbs\": %.1f, \"how\": \"tools/probe/l2_bw.cu: persistent grid "
         "(SMs x 8 x 256 threads), ld.global.cg 16-byte reads; L2: 48 MB buffer x 50 passes; HBM: 4 GB x 1; "
         "best of 5\"}\n", l2, hbm);
  return 0;
}
