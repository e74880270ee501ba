// gather_rate.cu -- measured rate of random 4-byte gathers on this B200: the roof of the K = 1
// SDDMM (one V[col] gather per stored entry).  A random 32-lane gather touches 32
// different 128-byte lines, and the L1tex pipeline processes them one wavefront at a time
// (B300_MICROARCH.md "L1tex wavefront queue": ~2 cycles per wavefront within one LDG), so the rate
// is bounded per SM, not by L2 or HBM bytes.  Table sizes of the workload graphs' V vectors (N
// floats, L2-resident); indices either computed in registers (a hash: the pure gather rate) or
// streamed coalesced from a 512 MB int32 array (the SDDMM's col_idx stream); ld.global.nc (L1
// allocating) and ld.global.cg (L2 only).  Best over (blocks per SM, gathers in flight per thread).
// Prints one JSON line.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t mix(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
  return x;
}

template <int UNR, bool STREAM, bool CG>
__global__ void g(const float* __restrict__ t, uint32_t T, const int32_t* __restrict__ idx, size_t n,
                  float* sink) {
  float acc = 0.f;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i + (UNR - 1) * stride < n; i += UNR * stride) {
    int32_t c[UNR];
#pragma unroll
    for (int u = 0; u < UNR; ++u) c[u] = STREAM ? __ldcs(idx + i + u * stride) : (int32_t)(mix((uint32_t)(i + u * stride)) % T);
    float v[UNR];
#pragma unroll
    for (int u = 0; u < UNR; ++u) v[u] = CG ? __ldcg(t + c[u]) : __ldg(t + c[u]);
#pragma unroll
    for (int u = 0; u < UNR; ++u) acc += v[u];
  }
  if (acc == 12345.f) *sink = acc;
}

__global__ void fill_idx(int32_t* idx, size_t n, uint32_t T) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    idx[i] = (int32_t)(mix((uint32_t)i * 2654435761u + 7u) % T);
}

template <int UNR, bool STREAM, bool CG>
static double rate(const float* t, uint32_t T, const int32_t* idx, size_t n, int bps, float* sink) {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  g<UNR, STREAM, CG><<<sms * bps, 256>>>(t, T, idx, n, sink);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  double best = 0;
  for (int r = 0; r < 5; ++r) {
    cudaEventRecord(a);
    g<UNR, STREAM, CG><<<sms * bps, 256>>>(t, T, idx, n, sink);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    const double r1 = (double)n / (ms * 1e-3);
    if (r1 > best) best = r1;
  }
  return best;
}

template <bool STREAM, bool CG>
static double best_rate(const float* t, uint32_t T, const int32_t* idx, size_t n, float* sink, char* cfg) {
  double best = 0;
  for (int bps : {4, 8}) {
    double r;
    r = rate<4, STREAM, CG>(t, T, idx, n, bps, sink); if (r > best) { best = r; sprintf(cfg, "%d blocks/SM, 4 in flight", bps); }
    r = rate<8, STREAM, CG>(t, T, idx, n, bps, sink); if (r > best) { best = r; sprintf(cfg, "%d blocks/SM, 8 in flight", bps); }
    r = rate<16, STREAM, CG>(t, T, idx, n, bps, sink); if (r > best) { best = r; sprintf(cfg, "%d blocks/SM, 16 in flight", bps); }
  }
  return best;
}

// random ROW gathers: a group of LPG lanes reads one random row of W float4 (row = K floats, K = 4W)
// from a table of T rows that exceeds L2 (the products-shaped operands of the K = 47 / 100 gathers);
// row ids from a hash, bytes = rows x K x 4 / time: the DRAM roof of gathers with no reuse
template <int LPG, int W, int UNR>
__global__ void rows_k(const float4* __restrict__ t, uint32_t T, size_t nrows, float* sink) {
  const int lane = threadIdx.x & 31, grp = lane / LPG, lig = lane % LPG;
  const size_t gw = (blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5;
  const size_t nw = ((size_t)gridDim.x * blockDim.x) >> 5;
  constexpr int G = 32 / LPG, NJ = (W + LPG - 1) / LPG;
  float acc = 0.f;
  for (size_t r0 = gw * G * UNR; r0 < nrows; r0 += nw * G * UNR) {
    float4 v[UNR][NJ];
#pragma unroll
    for (int u = 0; u < UNR; ++u) {
      const uint32_t row = mix((uint32_t)(r0 + u * G + grp) * 2654435761u + 1u) % T;
#pragma unroll
      for (int j = 0; j < NJ; ++j) {
        const int c = lig + j * LPG;
        v[u][j] = c < W ? __ldg(t + (size_t)row * W + c) : make_float4(0, 0, 0, 0);
      }
    }
#pragma unroll
    for (int u = 0; u < UNR; ++u)
#pragma unroll
      for (int j = 0; j < NJ; ++j) acc += v[u][j].x + v[u][j].y + v[u][j].z + v[u][j].w;
  }
  if (acc == 12345.f) *sink = acc;
}

template <int LPG, int W, int UNR>
static double row_gbs(const float4* t, uint32_t T, size_t nrows, int bps, float* sink) {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  rows_k<LPG, W, UNR><<<sms * bps, 256>>>(t, T, nrows, sink);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  double best = 0;
  for (int r = 0; r < 5; ++r) {
    cudaEventRecord(a);
    rows_k<LPG, W, UNR><<<sms * bps, 256>>>(t, T, nrows, sink);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    const double g = (double)nrows * W * 16 / (ms * 1e-3) / 1e9;
    if (g > best) best = g;
  }
  return best;
}

template <int LPG, int W>
static double row_best(const float4* t, uint32_t T, size_t nrows, float* sink, char* cfg) {
  double best = 0;
  for (int bps : {4, 8}) {
    double r;
    r = row_gbs<LPG, W, 2>(t, T, nrows, bps, sink); if (r > best) { best = r; sprintf(cfg, "%d blocks/SM, %d lanes/row, 2 rows in flight per group", bps, LPG); }
    r = row_gbs<LPG, W, 4>(t, T, nrows, bps, sink); if (r > best) { best = r; sprintf(cfg, "%d blocks/SM, %d lanes/row, 4 rows in flight per group", bps, LPG); }
    r = row_gbs<LPG, W, 8>(t, T, nrows, bps, sink); if (r > best) { best = r; sprintf(cfg, "%d blocks/SM, %d lanes/row, 8 rows in flight per group", bps, LPG); }
  }
  return best;
}

static void row_probes() {
  const uint32_t T = 2449029;  // products-shaped rows
  float4* t;
  float* sink;
  cudaMalloc(&t, (size_t)T * 25 * 16);
  cudaMalloc(&sink, 4);
  cudaMemset(t, 0, (size_t)T * 25 * 16);
  const size_t nrows = 64ull << 20;
  char c1[128], c2[128], c3[128];
  const double g48 = row_best<4, 12>(t, T, nrows, sink, c1);
  const double g48b = row_best<8, 12>(t, T, nrows, sink, c3);
  const double g100 = row_best<16, 25>(t, T, nrows, sink, c2);
  printf(", \"row_gathers\": {\"how\": \"64 Mi random rows (hash ids) of K floats from a table of 2,449,029 rows (products-shaped, > L2), a lane group per row with 16-byte loads; GB/s = rows x K x 4 / t, best of 5 over 4/8 blocks/SM x 256 threads and 2/4/8 rows in flight per group\", "
         "\"K48_gbs\": %.1f, \"K48_cfg\": \"%s\", \"K48_8lanes_gbs\": %.1f, \"K48_8lanes_cfg\": \"%s\", \"K100_gbs\": %.1f, \"K100_cfg\": \"%s\"}",
         g48, c1, g48b, c3, g100, c2);
  cudaFree(t);
  cudaFree(sink);
}

int main() {
  const size_t n = 128ull << 20;
  const uint32_t Ts[3] = {169343, 232965, 2449029};
  float* t; int32_t* idx; float* sink;
  cudaMalloc(&t, (size_t)Ts[2] * 4);
  cudaMalloc(&idx, n * 4);
  cudaMalloc(&sink, 4);
  cudaMemset(t, 0, (size_t)Ts[2] * 4);
  int sms = 0, clk = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("{\"how\": \"tools/probe/gather_rate.cu: random 4-byte gathers from an L2-resident table of N floats, 128 Mi gathers per launch, best of 5 over 4/8 blocks/SM x 256 threads and 4/8/16 gathers in flight\", \"sms\": %d, \"rows\": [", sms);
  for (int k = 0; k < 3; ++k) {
    fill_idx<<<sms * 8, 256>>>(idx, n, Ts[k]);
    cudaDeviceSynchronize();
    char c1[64], c2[64], c3[64];
    const double pure_nc = best_rate<false, false>(t, Ts[k], idx, n, sink, c1);
    const double str_nc = best_rate<true, false>(t, Ts[k], idx, n, sink, c2);
    const double str_cg = best_rate<true, true>(t, Ts[k], idx, n, sink, c3);
    printf("%s{\"N\": %u, \"pure_nc_Gps\": %.1f, \"pure_cfg\": \"%s\", \"stream_nc_Gps\": %.1f, \"stream_nc_cfg\": \"%s\", "
           "\"stream_cg_Gps\": %.1f, \"stream_cg_cfg\": \"%s\", \"pure_per_sm_clk_at_max\": %.3f}",
           k ? ", " : "", Ts[k], pure_nc / 1e9, c1, str_nc / 1e9, c2, str_cg / 1e9, c3, pure_nc / (sms * (double)clk * 1e3));
  }
  printf("], \"sm_clock_max_mhz\": %.0f", clk / 1e3);
  cudaFree(t);
  cudaFree(idx);
  row_probes();
  printf("}\n");
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) { fprintf(stderr, "%s\n", cudaGetErrorString(e)); return 1; }
  return 0;
}
