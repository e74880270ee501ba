// elementwise.cu -- small HBM-bound helpers around the layers: ReLU backward
// mask, padded row copies, softmax cross-entropy (training loss) and SGD.
#include <algorithm>
#include <cmath>

#include "internal.h"

namespace granii {

static unsigned blocks_for(int64_t n) { return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), 148 * 16)); }

// Row-wise helpers: lane groups of L = 2^lg lanes own a row (L = the smallest power of two >= the
// row's vector count, at most 32), so no per-element 64-bit division; 16-byte accesses when every
// row start is 16-byte aligned (V = 4). Loads of one thread stay independent across the unrolled
// column loop, which keeps enough bytes in flight per SM for HBM.
template <int V> struct Vec;
template <> struct Vec<4> {
  using T = float4;
  __device__ static T ld(const float* p) { return *reinterpret_cast<const float4*>(p); }
  __device__ static void st(float* p, T v) { *reinterpret_cast<float4*>(p) = v; }
  __device__ static float& at(T& v, int i) { return i == 0 ? v.x : i == 1 ? v.y : i == 2 ? v.z : v.w; }
};
template <> struct Vec<1> {
  using T = float;
  __device__ static T ld(const float* p) { return *p; }
  __device__ static void st(float* p, T v) { *p = v; }
  __device__ static float& at(T& v, int) { return v; }
};

// dst = (out == NULL || out > 0) ? g * rs[r] : 0  -- ReLU' mask (optional, ReLU'(0) = 0) fused with an
// optional row scale (the inner D^-1/2 of the DYN_UPD backward, so its SpMM needs no column scale);
// out == rs == NULL is a padded row copy (g * 1.f is exact)
template <int V>
__global__ void __launch_bounds__(256) k_scale_mask(int64_t rows, int K, int Kv, int lg, const float* __restrict__ out,
                                                    int64_t ldo, const float* __restrict__ g, int64_t ldg,
                                                    const float* __restrict__ rs, float* __restrict__ dst,
                                                    int64_t ldd) {
  using VT = Vec<V>;
  const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int lig = threadIdx.x & ((1 << lg) - 1);
  const int64_t ngrp = ((int64_t)gridDim.x * blockDim.x) >> lg;
  for (int64_t r = tid >> lg; r < rows; r += ngrp) {
    const float s = rs ? rs[r] : 1.f;
#pragma unroll 2
    for (int k = lig; k < Kv; k += 1 << lg) {
      if (V > 1 && k * V + V > K) {  // ragged tail of a row whose start is aligned: element by element
        for (int c = k * V; c < K; ++c) {
          const float x = g[r * ldg + c] * s;
          dst[r * ldd + c] = (!out || out[r * ldo + c] > 0.f) ? x : 0.f;
        }
        continue;
      }
      typename VT::T v = VT::ld(g + r * ldg + (int64_t)k * V);
      typename VT::T o;
      if (out) o = VT::ld(out + r * ldo + (int64_t)k * V);
#pragma unroll
      for (int i = 0; i < V; ++i) {
        const float x = VT::at(v, i) * s;
        VT::at(v, i) = (!out || VT::at(o, i) > 0.f) ? x : 0.f;
      }
      VT::st(dst + r * ldd + (int64_t)k * V, v);
    }
  }
}

static inline bool al16(const void* p) { return ((uintptr_t)p & 15u) == 0; }

static void rowwise_shape(int64_t rows, int64_t K, bool v4, int* Kv, int* lg, unsigned* blocks) {
  *Kv = (int)(v4 ? (K + 3) / 4 : K);
  int l = 0;
  while (l < 5 && (1 << l) < *Kv) ++l;
  *lg = l;
  *blocks = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(rows << l, 256), 148 * 16));
}

static granii_status scale_mask_impl(int64_t rows, int64_t K, const float* out, int64_t ldo, const float* g,
                                     int64_t ldg, const float* rs, float* dst, int64_t ldd, cudaStream_t st) {
  const bool v4 = ldg % 4 == 0 && ldd % 4 == 0 && al16(g) && al16(dst) &&
                  (!out || (ldo % 4 == 0 && al16(out)));
  int Kv, lg;
  unsigned blocks;
  rowwise_shape(rows, K, v4, &Kv, &lg, &blocks);
  if (v4) k_scale_mask<4><<<blocks, 256, 0, st>>>(rows, (int)K, Kv, lg, out, ldo, g, ldg, rs, dst, ldd);
  else k_scale_mask<1><<<blocks, 256, 0, st>>>(rows, (int)K, Kv, lg, out, ldo, g, ldg, rs, dst, ldd);
  GR_CHECK_LAUNCH();
  return GRANII_OK;
}

granii_status launch_scale_mask(int64_t rows, int64_t K, const float* out, int64_t ldo, const float* g, int64_t ldg,
                                const float* rs, float* dst, int64_t ldd, cudaStream_t st) {
  if (rows * K == 0) return GRANII_OK;
  ProfScope ps("elementwise", st, (out ? 12.0 : 8.0) * rows * K, 0.0, 1);
  return scale_mask_impl(rows, K, out, ldo, g, ldg, rs, dst, ldd, st);
}

// one warp per row
__global__ void k_softmax_xent(int64_t rows, int64_t C, const float* __restrict__ Z, int64_t ldz,
                               const int32_t* __restrict__ y, float inv_n, float* __restrict__ dZ, int64_t lddz,
                               float* __restrict__ loss) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r = warp; r < rows; r += nw) {
    const float* z = Z + r * ldz;
    float m = -INFINITY;
    for (int64_t c = lane; c < C; c += 32) m = fmaxf(m, z[c]);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
    float s = 0.f;
    for (int64_t c = lane; c < C; c += 32) s += expf(z[c] - m);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    const int32_t t = y[r];
    for (int64_t c = lane; c < C; c += 32) {
      const float p = expf(z[c] - m) / s;
      dZ[r * lddz + c] = (p - (c == t ? 1.f : 0.f)) * inv_n;
    }
    if (loss && lane == 0) loss[r] = logf(s) + m - z[t];
  }
}

__global__ void k_sgd(int64_t n, float lr, const float* __restrict__ g, float* __restrict__ p) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    p[i] -= lr * g[i];
}

granii_status launch_relu_mask(int64_t rows, int64_t K, const float* out, int64_t ldo, const float* g, int64_t ldg,
                               float* dst, int64_t ldd, cudaStream_t st) {
  if (rows * K == 0) return GRANII_OK;
  ProfScope ps("elementwise", st, 12.0 * rows * K, 0.0, 1);
  return scale_mask_impl(rows, K, out, ldo, g, ldg, nullptr, dst, ldd, st);
}

granii_status launch_copy_rows(int64_t rows, int64_t K, const float* src, int64_t lds, float* dst, int64_t ldd,
                               cudaStream_t st) {
  if (rows * K == 0) return GRANII_OK;
  ProfScope ps("elementwise", st, 8.0 * rows * K, 0.0, 1);
  return scale_mask_impl(rows, K, nullptr, 0, src, lds, nullptr, dst, ldd, st);
}

struct RankPtrs {
  const float* p[16];
};
__global__ void k_rank_sum(int n, RankPtrs src, size_t count, float* __restrict__ out) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < count; i += (size_t)gridDim.x * blockDim.x) {
    float s = src.p[0][i];
    for (int q = 1; q < n; ++q) s += src.p[q][i];
    out[i] = s;
  }
}

granii_status launch_rank_sum(int n, const float* const* src, size_t count, float* out, cudaStream_t st) {
  if (n < 1 || n > 16) return fail(GRANII_ERR_UNSUPPORTED, "loopback group larger than 16 ranks");
  if (count == 0) return GRANII_OK;
  RankPtrs rp{};
  for (int q = 0; q < n; ++q) rp.p[q] = src[q];
  ProfScope ps("elementwise", st, 4.0 * (n + 1) * count, 0.0, 1);
  k_rank_sum<<<blocks_for((int64_t)count), 256, 0, st>>>(n, rp, count, out);
  GR_CHECK_LAUNCH();
  return GRANII_OK;
}

// test support (granii_debug_spin): hold a stream busy for `us` microseconds of wall time
__global__ void k_spin(int64_t ns) {
  uint64_t t0, t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  do {
    __nanosleep(1000);
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  } while ((int64_t)(t - t0) < ns);
}

granii_status launch_spin(int64_t us, cudaStream_t st) {
  ProfScope ps("elementwise", st, 0.0, 0.0, 1);
  k_spin<<<1, 1, 0, st>>>(us * 1000);
  GR_CHECK_LAUNCH();
  return GRANII_OK;
}

// C <= LPG * NV (the classifier widths: 41, 47): an LPG-lane group per row holds its logits in
// registers -- one coalesced load, max and sum by fixed xor butterflies, one store -- so every load
// of the 32 / LPG rows of a warp is in flight at once (the warp-per-row loop above re-reads the row
// three times with a dependent round trip each)
template <int LPG, int NV>
__global__ void __launch_bounds__(256) k_softmax_xent_reg(int64_t rows, int64_t C, const float* __restrict__ Z,
                                                          int64_t ldz, const int32_t* __restrict__ y, float inv_n,
                                                          float* __restrict__ dZ, int64_t lddz,
                                                          float* __restrict__ loss) {
  constexpr int G = 32 / LPG;
  const int lane = threadIdx.x & 31, lg = lane % LPG;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r0 = warp * G; r0 < rows; r0 += nw * G) {
    const int64_t r = r0 + lane / LPG;
    const bool live = r < rows;
    const float* z = Z + (live ? r : 0) * ldz;
    float v[NV];
    float m = -INFINITY;
#pragma unroll
    for (int q = 0; q < NV; ++q) {
      const int64_t c = lg + q * LPG;
      v[q] = (live && c < C) ? __ldg(z + c) : -INFINITY;
      m = fmaxf(m, v[q]);
    }
#pragma unroll
    for (int o = LPG / 2; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
    float s = 0.f;
#pragma unroll
    for (int q = 0; q < NV; ++q) {
      v[q] = live ? expf(v[q] - m) : 0.f;
      s += v[q];
    }
#pragma unroll
    for (int o = LPG / 2; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (!live) continue;
    const int32_t t = y[r];
#pragma unroll
    for (int q = 0; q < NV; ++q) {
      const int64_t c = lg + q * LPG;
      if (c < C) dZ[r * lddz + c] = (v[q] / s - (c == t ? 1.f : 0.f)) * inv_n;
    }
    if (loss && lg == 0) loss[r] = logf(s) + m - z[t];
  }
}

granii_status launch_softmax_xent(int64_t rows, int64_t C, const float* Z, int64_t ldz, const int32_t* y,
                                  int64_t n_total, float* dZ, int64_t lddz, float* loss, cudaStream_t st) {
  if (rows == 0) return GRANII_OK;
  ProfScope ps("elementwise", st, 8.0 * rows * C + 8.0 * rows, 0.0, 1);
  const unsigned b = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(rows, 8), 148 * 16));
  if (C <= 64) {
    const unsigned b2 = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(rows, 16), 148 * 16));
    k_softmax_xent_reg<16, 4><<<b2, 256, 0, st>>>(rows, C, Z, ldz, y, 1.f / (float)n_total, dZ, lddz, loss);
  } else {
    k_softmax_xent<<<b, 256, 0, st>>>(rows, C, Z, ldz, y, 1.f / (float)n_total, dZ, lddz, loss);
  }
  GR_CHECK_LAUNCH();
  return GRANII_OK;
}

granii_status launch_sgd(int64_t n, float lr, const float* g, float* p, cudaStream_t st) {
  if (n == 0) return GRANII_OK;
  ProfScope ps("elementwise", st, 12.0 * n, 2.0 * n, 1);
  k_sgd<<<blocks_for(n), 256, 0, st>>>(n, lr, g, p);
  GR_CHECK_LAUNCH();
  return GRANII_OK;
}

}  // namespace granii

namespace granii {

// GIN PRE composition (R23): vals_e = 1 + eps where col(e) is the row's own diagonal, 1 elsewhere.
// Column ids live in the gather layout when partitioned: the diagonal of local row r is diag0 + r.
__global__ void k_gin_vals(int64_t R, const int64_t* __restrict__ row_ptr, const int32_t* __restrict__ col_idx,
                           int64_t diag0, float one_eps, float* __restrict__ vals) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; r < R; r += nw)
    for (int64_t e = row_ptr[r] + lane; e < row_ptr[r + 1]; e += 32)
      vals[e] = (int64_t)col_idx[e] == diag0 + r ? one_eps : 1.f;
}

granii_status launch_gin_vals(const granii_graph_s* g, float eps, float* vals, cudaStream_t st) {
  if (g->n_rows == 0) return GRANII_OK;
  ProfScope ps("sddmm", st, 8.0 * (double)g->local_nnz + 8.0 * (double)g->n_rows, 0.0, 1);
  const int64_t diag0 = g->world > 1 ? (int64_t)g->rank * g->max_rows : 0;
  k_gin_vals<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(g->n_rows, 8), 148 * 32)), 256, 0, st>>>(
      g->n_rows, g->row_ptr, g->col_idx, diag0, 1.f + eps, vals);
  GR_CHECK_LAUNCH();
  return GRANII_OK;
}

}  // namespace granii
