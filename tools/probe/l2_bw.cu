// l2_bw.cu -- measured L2 read bandwidth of this B200 (the roof of gathers served by L2).
// A persistent grid (all SMs, B x 256 threads each) reads a buffer that fits in L2 (48 MB)
// with 16-byte ld.global.cg loads (L1 bypassed), UNR independent loads in flight per thread,
// many passes; bytes read / time, best over (blocks per SM, unroll).  Also the HBM read
// bandwidth with a 4 GB buffer for reference.  Prints one JSON line.
#include <cstdio>
#include <cuda_runtime.h>

template <int UNR>
__global__ void rd(const float4* __restrict__ p, size_t n, int passes, float* sink) {
  float4 acc = make_float4(0, 0, 0, 0);
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  const size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  for (int r = 0; r < passes; ++r) {
    size_t i = tid;
    for (; i + (UNR - 1) * stride < n; i += UNR * stride) {
      float4 v[UNR];
#pragma unroll
      for (int u = 0; u < UNR; ++u) v[u] = __ldcg(p + i + u * stride);
#pragma unroll
      for (int u = 0; u < UNR; ++u) { acc.x += v[u].x; acc.y += v[u].y; acc.z += v[u].z; acc.w += v[u].w; }
    }
    for (; i < n; i += stride) {
      float4 v = __ldcg(p + i);
      acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
  }
  if (acc.x + acc.y + acc.z + acc.w == 12345.f) *sink = acc.x;
}

template <int UNR>
static double bw1(const float4* p, size_t bytes, int passes, int reps, int bps, float* sink) {
  int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const size_t n = bytes / 16;
  rd<UNR><<<sms * bps, 256>>>(p, n, 1, sink);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  double best = 0;
  for (int r = 0; r < reps; ++r) {
    cudaEventRecord(a);
    rd<UNR><<<sms * bps, 256>>>(p, n, passes, sink);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    const double gbs = (double)bytes * passes / (ms * 1e-3) / 1e9;
    if (gbs > best) best = gbs;
  }
  return best;
}

static double bw(size_t bytes, int passes, int reps, char* cfg) {
  float4* p; float* sink;
  cudaMalloc(&p, bytes); cudaMalloc(&sink, 4);
  cudaMemset(p, 0, bytes);
  double best = 0;
  for (int bps : {4, 8}) {
    const double r[3] = {bw1<1>(p, bytes, passes, reps, bps, sink), bw1<4>(p, bytes, passes, reps, bps, sink),
                         bw1<8>(p, bytes, passes, reps, bps, sink)};
    const int u[3] = {1, 4, 8};
    for (int k = 0; k < 3; ++k)
      if (r[k] > best) { best = r[k]; sprintf(cfg, "%d blocks/SM x 256, %d loads in flight", bps, u[k]); }
  }
  cudaFree(p); cudaFree(sink);
  return best;
}

int main() {
  char c1[96], c2[96];
  const double l2 = bw(48ull << 20, 50, 5, c1);
  const double hbm = bw(4ull << 30, 1, 5, c2);
  printf("{\"l2_read_gbs\": %.1f, \"l2_cfg\": \"%s\", \"hbm_read_gbs\": %.1f, \"hbm_cfg\": \"%s\", \"how\": "
         "\"tools/probe/l2_bw.cu: persistent grid, ld.global.cg 16-byte reads, best over blocks/SM in {4,8} and "
         "loads in flight per thread in {1,4,8}; L2: 48 MB buffer x 50 passes; HBM: 4 GB x 1; best of 5\"}\n",
         l2, c1, hbm, c2);
  return 0;
}
