// sddmm.cu -- g-SDDMM on Ã's pattern ("a standard matrix
// multiplication guided by a sparse mask", L92 edge-based aggregation) and the
// GAT attention of Eq. 4 (L127-L131; reading R8: single-head GAT [25]).
//
//   DOT : e = scale * <U_r, V_c>        K = 1 with U = V = dinv gives Ñ (Eq. 3)
//   ADD : e = scale * (U_r + V_c)       K = 1 with U = el, V = er (additive attention)
//   | LEAKYRELU : e = max(e, 0.2 e)
//   | ROW_SOFTMAX : alpha_e = exp(e - m_r) / sum_r exp(e - m_r)
//
// B200 design: HBM-bound streaming over col_idx (4 B/entry)
// plus an L2-resident gather of V (dinv/er: N floats) and a 4 B/entry write.
// Group-per-row with LPG lanes striding the row keeps col_idx reads and e/alpha
// writes coalesced; LPG follows the average degree.  For K > 1 a warp owns a
// row: U_r lives in registers, LPG-lane groups each take an entry, gather V_c
// with 16-byte loads and reduce with shuffles.  Softmax is fused: a row that
// fits one step of 4 x LPG entries is scored, reduced (max, sum) and normalised
// in registers, alpha written once; longer rows write their scores with an
// online (max, sum) per lane and normalise them in a coalesced second sweep.
// The 4-byte V gather (one L1 wavefront per entry) happens once per entry.
// No atomics.
#include <algorithm>
#include <cmath>

#include "cache.cuh"
#include "internal.h"

namespace granii {

struct SddmmArgs {
  int64_t n_rows;
  const int64_t* __restrict__ row_ptr;
  const int32_t* __restrict__ col_idx;
  const float* __restrict__ U;
  int64_t ldu;
  const float* __restrict__ V;
  int64_t ldv;
  int64_t K;
  float scale;
  float* __restrict__ out;
  const int32_t* __restrict__ order;       // light rows (degree-descending), n_rows of them
  const longlong2* __restrict__ ord_rp;    // their entry ranges, same order
  int64_t n_seg;                           // heavy-row segments: warp-wide items
  const int64_t* __restrict__ seg_lo;
  const int64_t* __restrict__ seg_hi;
  const int32_t* __restrict__ seg_row;
  int l2hint;                              // cache.cuh: V kept in L2, col_idx / out streamed
  int64_t cap;                             // softmax: scores staged per warp in shared memory (floats)
};

template <bool ADD, bool LRELU>
__device__ __forceinline__ float score1(float u, float v, float scale) {
  float e = ADD ? scale * (u + v) : scale * (u * v);
  if (LRELU) e = e > 0.f ? e : 0.2f * e;
  return e;
}

// warp-uniform (max, sum) butterfly of per-lane online softmax states
__device__ __forceinline__ void ms_merge(float& m, float& s, float m2, float s2) {
  const float mn = fmaxf(m, m2);
  const float a1 = (m == -INFINITY) ? 0.f : s * __expf(m - mn);
  const float a2 = (m2 == -INFINITY) ? 0.f : s2 * __expf(m2 - mn);
  m = mn;
  s = a1 + a2;
}

// Fused row softmax of one row by a whole warp (rows longer than one group step).  Up to a.cap
// entries the scores are staged in this warp's slice of shared memory: one sweep of coalesced
// column loads and UW independent V gathers per lane, the row max, exp in place with the row sum,
// then alpha written once -- every lane touches only its own slots (k = lane + 32 j), so no
// barrier.  Longer rows (cap < n <= seg_len) write their scores with an online (max, sum) per lane
// and normalise them in a second, coalesced sweep.
template <bool ADD, bool LRELU>
__device__ __forceinline__ void sddmm1_softmax_warp(const SddmmArgs& a, int64_t t, int lane, float* buf,
                                                    const L2Pol& pol) {
  constexpr int UW = 8;
  const int64_t row = a.order[t];
  const longlong2 rr = a.ord_rp[t];
  const int64_t rs = rr.x, n = rr.y - rr.x;
  const float u = __ldg(a.U + row * a.ldu);
  const bool staged = n <= a.cap;
  float m = -INFINITY, s = 0.f;
  for (int64_t k0 = 0; k0 < n; k0 += 32 * UW) {
    int32_t c[UW];
    float v[UW];
#pragma unroll
    for (int q = 0; q < UW; ++q) {
      const int64_t k = k0 + 32 * q + lane;
      c[q] = ldg_stream(a.col_idx + rs + (k < n ? k : n - 1), pol.stream);
    }
#pragma unroll
    for (int q = 0; q < UW; ++q) v[q] = ldg_pol(a.V + (int64_t)c[q] * a.ldv, pol.keep);
    float mn = m;
#pragma unroll
    for (int q = 0; q < UW; ++q) {
      const int64_t k = k0 + 32 * q + lane;
      v[q] = score1<ADD, LRELU>(u, v[q], a.scale);
      if (k < n) {
        if (staged) buf[k] = v[q];
        else st_pol(a.out + rs + k, v[q], pol.stream);
        mn = fmaxf(mn, v[q]);
      } else {
        v[q] = -INFINITY;
      }
    }
    if (!staged && mn > -INFINITY) {  // online sum (streamed rows only)
      s = (m == -INFINITY ? 0.f : s * __expf(m - mn));
#pragma unroll
      for (int q = 0; q < UW; ++q) s += __expf(v[q] - mn);
    }
    m = mn;
  }
  if (staged) {
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, off));
    for (int64_t k = lane; k < n; k += 32) {
      const float x = __expf(buf[k] - m);
      buf[k] = x;
      s += x;
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
    const float inv = 1.f / s;
    for (int64_t k = lane; k < n; k += 32) st_pol(a.out + rs + k, buf[k] * inv, pol.stream);
    __syncwarp();  // the next row reuses the slice
  } else {
#pragma unroll
    for (int off = 16; off > 0; off >>= 1)
      ms_merge(m, s, __shfl_xor_sync(0xffffffffu, m, off), __shfl_xor_sync(0xffffffffu, s, off));
    const float inv = 1.f / s;
    for (int64_t k = lane; k < n; k += 32) st_pol(a.out + rs + k, __expf(a.out[rs + k] - m) * inv, pol.stream);
  }
}

// K == 1: group of LPG lanes per row
template <int LPG, bool ADD, bool LRELU, bool SOFTMAX>
__global__ void __launch_bounds__(256) k_sddmm1(SddmmArgs a) {
  extern __shared__ float sm_buf[];  // softmax: a.cap floats per warp
  constexpr int G = 32 / LPG;
  const int lane = threadIdx.x & 31, grp = lane / LPG, lig = lane % LPG;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const L2Pol pol = make_l2pol(a.l2hint);
  // heavy-row segments: all 32 lanes stride the segment (scores only; the softmax of
  // heavy rows is the segmented 3-phase pass launched afterwards)
  for (int64_t t = warp; t < a.n_seg; t += nwarps) {
    const int64_t row = a.seg_row[t], hi = a.seg_hi[t];
    const float u = __ldg(a.U + row * a.ldu);
    int64_t e = a.seg_lo[t] + lane;
    for (; e + 96 < hi; e += 128) {
      int32_t c[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) c[q] = ldg_stream(a.col_idx + e + 32 * q, pol.stream);
#pragma unroll
      for (int q = 0; q < 4; ++q)
        st_pol(a.out + e + 32 * q, score1<ADD, LRELU>(u, ldg_pol(a.V + (int64_t)c[q] * a.ldv, pol.keep), a.scale),
               pol.stream);
    }
    for (; e < hi; e += 32) {
      const int32_t c = ldg_stream(a.col_idx + e, pol.stream);
      st_pol(a.out + e, score1<ADD, LRELU>(u, ldg_pol(a.V + (int64_t)c * a.ldv, pol.keep), a.scale), pol.stream);
    }
  }
  constexpr int U4 = 4;
  for (int64_t t0 = warp * G; t0 < a.n_rows; t0 += nwarps * G) {
    if constexpr (SOFTMAX) {
      // the unit's first row is its longest (degree-descending schedule): if it exceeds one group
      // step, the warp takes the unit's rows one at a time (warp-uniform branch)
      const longlong2 r0 = a.ord_rp[t0];
      if (r0.y - r0.x > U4 * LPG) {
        float* buf = sm_buf + (threadIdx.x >> 5) * a.cap;
        for (int q = 0; q < G && t0 + q < a.n_rows; ++q) sddmm1_softmax_warp<ADD, LRELU>(a, t0 + q, lane, buf, pol);
        continue;
      }
    }
    const int64_t t = t0 + grp;
    const bool live = t < a.n_rows;
    const int64_t row = live ? a.order[t] : 0;
    const longlong2 rr = live ? a.ord_rp[t] : make_longlong2(0, 0);  // independent of order[t]
    const int64_t rs = rr.x, re = rr.y;
    const float u = live ? __ldg(a.U + row * a.ldu) : 0.f;
    if constexpr (!SOFTMAX) {
      // scores only: 4 independent col -> V gathers in flight per lane
      int64_t e = rs + lig;
      for (; e + (U4 - 1) * LPG < re; e += U4 * LPG) {
        int32_t c[U4];
#pragma unroll
        for (int q = 0; q < U4; ++q) c[q] = ldg_stream(a.col_idx + e + q * LPG, pol.stream);
#pragma unroll
        for (int q = 0; q < U4; ++q)
          st_pol(a.out + e + q * LPG, score1<ADD, LRELU>(u, ldg_pol(a.V + (int64_t)c[q] * a.ldv, pol.keep), a.scale),
                 pol.stream);
      }
      for (; e < re; e += LPG) {
        const int32_t c = ldg_stream(a.col_idx + e, pol.stream);
        st_pol(a.out + e, score1<ADD, LRELU>(u, ldg_pol(a.V + (int64_t)c * a.ldv, pol.keep), a.scale), pol.stream);
      }
      continue;
    }
    // Fused row softmax.  Steps of U4 x LPG entries issue every load at once (lanes past the
    // row's end re-read its last entry, branch-free, and are masked out).  A row of one step keeps
    // its scores in registers: max and sum by fixed xor butterflies, alpha written once.  Longer
    // rows stream: the scores are written with an online (max, sum) per lane, then re-read
    // (coalesced) and normalised -- the 4-byte V gathers, one L1 wavefront each, happen once.
    const bool one = re > rs && re - rs <= U4 * LPG;  // uniform within the group (empty rows stream: no loads)
    float x[U4];
    float m = -INFINITY, s = 0.f;
    if (one) {
      int32_t c[U4];
#pragma unroll
      for (int q = 0; q < U4; ++q) {
        const int64_t e = rs + q * LPG + lig;
        c[q] = ldg_stream(a.col_idx + (e < re ? e : re - 1), pol.stream);
      }
#pragma unroll
      for (int q = 0; q < U4; ++q) x[q] = ldg_pol(a.V + (int64_t)c[q] * a.ldv, pol.keep);
#pragma unroll
      for (int q = 0; q < U4; ++q) {
        x[q] = rs + q * LPG + lig < re ? score1<ADD, LRELU>(u, x[q], a.scale) : -INFINITY;
        m = fmaxf(m, x[q]);
      }
    } else {
      for (int64_t e0 = rs; e0 < re; e0 += U4 * LPG) {
        int32_t c[U4];
        float y[U4];
#pragma unroll
        for (int q = 0; q < U4; ++q) {
          const int64_t e = e0 + q * LPG + lig;
          c[q] = ldg_stream(a.col_idx + (e < re ? e : re - 1), pol.stream);
        }
#pragma unroll
        for (int q = 0; q < U4; ++q) y[q] = ldg_pol(a.V + (int64_t)c[q] * a.ldv, pol.keep);
        float mn = m;
#pragma unroll
        for (int q = 0; q < U4; ++q) {
          const int64_t e = e0 + q * LPG + lig;
          y[q] = score1<ADD, LRELU>(u, y[q], a.scale);
          if (e < re) {
            st_pol(a.out + (e), y[q], pol.stream);
            mn = fmaxf(mn, y[q]);
          } else {
            y[q] = -INFINITY;
          }
        }
        if (mn > -INFINITY) {
          s = (m == -INFINITY ? 0.f : s * __expf(m - mn));
#pragma unroll
          for (int q = 0; q < U4; ++q) s += __expf(y[q] - mn);
          m = mn;
        }
      }
    }
    // row max over the group (fixed xor butterfly), then each lane's sum rescaled to it
    float mr = m;
#pragma unroll
    for (int off = LPG / 2; off > 0; off >>= 1) mr = fmaxf(mr, __shfl_xor_sync(0xffffffffu, mr, off));
    if (one) {
#pragma unroll
      for (int q = 0; q < U4; ++q) {
        x[q] = __expf(x[q] - mr);  // exp(-inf) = 0 for the masked lanes
        s += x[q];
      }
    } else {
      s = m == -INFINITY ? 0.f : s * __expf(m - mr);
    }
#pragma unroll
    for (int off = LPG / 2; off > 0; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
    const float inv = 1.f / s;
    if (one) {
#pragma unroll
      for (int q = 0; q < U4; ++q) {
        const int64_t e = rs + q * LPG + lig;
        if (e < re) st_pol(a.out + (e), x[q] * inv, pol.stream);
      }
    } else {
      for (int64_t e2 = rs + lig; e2 < re; e2 += LPG) st_pol(a.out + (e2), __expf(a.out[e2] - mr) * inv, pol.stream);
    }
  }
}

static int lpg_for_softmax(float avg);
static int lpg_for_degree(float avg);
static bool sddmm_tile_enabled(const granii_graph_s* g);

// ---------------------------------------------------------------- K = 1 over entry tiles
// The degree-ordered kernel above keeps one dependent chain per lane group (order -> entry range
// -> col -> V -> exp -> store) and so few bytes in flight per SM that products-shaped inputs reach
// ~1.8 TB/s.  Here a CTA owns a tile of tile_e consecutive entries of Ã in CSR order: (A) every
// thread loads 16 column ids with four 16-byte streaming loads and issues its 16 V gathers at once
// (4096 independent gathers per CTA), parking V_c in shared memory; (B) the tile's rows (row_ptr
// slice in shared memory) are scored, max-reduced, exponentiated and normalised in shared memory
// by lane groups (rows of >= TILE_BIG in-tile entries by the whole CTA); (C) the tile is written
// back with full-line 16-byte stores.  A row cut by a tile boundary keeps its scores and leaves its
// in-tile (max, sum) in st_first / st_last; k_sddmm1_xstats combines a crossing row's partials in
// tile order and k_sddmm1_xnorm normalises its entries (alpha = exp(e - m) / s, the same formula).
constexpr int TILE_E = (int)granii_graph_s::tile_e;
constexpr int TILE_T = 256;
constexpr int TILE_RCH = 512;   // rows per row_ptr chunk in shared memory
constexpr int TILE_BIG = 512;   // in-tile row length processed by the whole CTA

struct TileArgs {
  int64_t n_rows, nnz, n_tiles;
  const int64_t* __restrict__ row_ptr;
  const int32_t* __restrict__ col_idx;
  const int32_t* __restrict__ tile_row;
  const float* __restrict__ U;
  int64_t ldu;
  const float* __restrict__ V;
  int64_t ldv;
  float scale;
  float* __restrict__ out;
  float2* st_first;   // softmax: in-tile (max, sum) of the tile's first row (if it began earlier)
  float2* st_last;    // ... and of its last row (if it continues into the next tile)
  float2* fin_first;  // crossing rows' final (max, 1/sum), per tile it enters / begins in
  float2* fin_last;
  int l2hint;
};

template <int LPG, bool ADD, bool LRELU, bool SOFTMAX>
__global__ void __launch_bounds__(TILE_T) k_sddmm1_tile(TileArgs a) {
  __shared__ __align__(16) float sv[TILE_E];
  __shared__ int32_t srp[TILE_RCH + 1];
  __shared__ float sred[2][TILE_T / 32];
  __shared__ int32_t sbig[TILE_E / TILE_BIG + 1];
  __shared__ int s_nbig;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const L2Pol pol = make_l2pol(a.l2hint);
  const int64_t t = blockIdx.x;
  const int64_t e0 = t * TILE_E, e1 = min(e0 + (int64_t)TILE_E, a.nnz);
  const int ne = (int)(e1 - e0);
  // (A) column ids (coalesced 16-byte streaming loads), then 16 independent V gathers per thread
  {
    int32_t c[16];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int j = warp * 512 + q * 128 + lane * 4;
      if (j + 3 < ne) {
        const int4 v = ldg_stream(reinterpret_cast<const int4*>(a.col_idx + e0 + j), pol.stream);
        c[4 * q] = v.x; c[4 * q + 1] = v.y; c[4 * q + 2] = v.z; c[4 * q + 3] = v.w;
      } else {
#pragma unroll
        for (int r = 0; r < 4; ++r) c[4 * q + r] = j + r < ne ? ldg_stream(a.col_idx + e0 + j + r, pol.stream) : 0;
      }
    }
    float v[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) v[i] = ldg_pol(a.V + (int64_t)c[i] * a.ldv, pol.keep);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int j = warp * 512 + q * 128 + lane * 4;
      if (j + 3 < ne) {
        *reinterpret_cast<float4*>(sv + j) = make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
      } else {
#pragma unroll
        for (int r = 0; r < 4; ++r)
          if (j + r < ne) sv[j + r] = v[4 * q + r];
      }
    }
  }
  // (B) rows of the tile
  const int64_t r0 = a.tile_row[t];
  const int64_t rend = (t + 1 < a.n_tiles) ? (int64_t)a.tile_row[t + 1] + 1 : a.n_rows;
  const bool first_cut = SOFTMAX && a.row_ptr[r0] < e0;  // r0 began in an earlier tile
  const int64_t rlast = rend - 1;                          // holds entry e1 when it continues
  const bool last_cut = SOFTMAX && t + 1 < a.n_tiles && a.row_ptr[rlast] < e1;
  constexpr int G = 32 / LPG;
  const int grp = lane / LPG, lig = lane % LPG;
  for (int64_t c0 = r0; c0 < rend; c0 += TILE_RCH) {
    const int nr = (int)min((int64_t)TILE_RCH, rend - c0);
    __syncthreads();  // sv complete (first chunk) / srp and sbig free (later chunks)
    if (tid == 0) s_nbig = 0;
    for (int k = tid; k <= nr; k += TILE_T) {
      const int64_t p = a.row_ptr[c0 + k];
      srp[k] = (int32_t)(min(max(p, e0), e1) - e0);
    }
    __syncthreads();
    for (int k0 = warp * G; k0 < nr; k0 += (TILE_T / 32) * G) {  // warp-uniform trip count
      const int k = k0 + grp;
      const bool live = k < nr;
      int lo = live ? srp[k] : 0, hi = live ? srp[k + 1] : 0;
      if (hi - lo >= TILE_BIG) {  // deferred to the whole CTA
        if (lig == 0) sbig[atomicAdd(&s_nbig, 1)] = k;
        hi = lo;
      }
      const int64_t row = c0 + k;
      const float u = hi > lo ? __ldg(a.U + row * a.ldu) : 0.f;
      if constexpr (!SOFTMAX) {
        for (int j = lo + lig; j < hi; j += LPG) sv[j] = score1<ADD, LRELU>(u, sv[j], a.scale);
      } else {
        // a row of <= RS x LPG entries that no tile boundary cuts stays in registers (one read and
        // one write of shared memory per entry); longer and cut rows sweep shared memory three times
        constexpr int RS = 4;
        const bool fc = first_cut && row == r0, lc = last_cut && row == rlast;
        const bool reg = hi - lo <= RS * LPG && !(fc || lc);
        float x[RS];
        float m = -INFINITY;
        if (reg) {
#pragma unroll
          for (int q = 0; q < RS; ++q) {
            const int j = lo + q * LPG + lig;
            x[q] = j < hi ? score1<ADD, LRELU>(u, sv[j], a.scale) : -INFINITY;
            m = fmaxf(m, x[q]);
          }
        } else {
          for (int j = lo + lig; j < hi; j += LPG) {
            const float e = score1<ADD, LRELU>(u, sv[j], a.scale);
            sv[j] = e;
            m = fmaxf(m, e);
          }
        }
#pragma unroll
        for (int off = LPG / 2; off > 0; off >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, off));
        float s = 0.f;
        if (reg) {
#pragma unroll
          for (int q = 0; q < RS; ++q) {
            x[q] = __expf(x[q] - m);  // exp(-inf) = 0 past the row's end
            s += x[q];
          }
        } else {
          for (int j = lo + lig; j < hi; j += LPG) {
            const float e = __expf(sv[j] - m);
            if (!(fc || lc)) sv[j] = e;  // a cut row keeps its scores
            s += e;
          }
        }
#pragma unroll
        for (int off = LPG / 2; off > 0; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
        if (fc || lc) {
          if (lig == 0 && hi > lo) {
            if (fc) a.st_first[t] = make_float2(m, s);
            if (lc) a.st_last[t] = make_float2(m, s);
          }
        } else if (hi > lo) {
          const float inv = 1.f / s;
          if (reg) {
#pragma unroll
            for (int q = 0; q < RS; ++q) {
              const int j = lo + q * LPG + lig;
              if (j < hi) sv[j] = x[q] * inv;
            }
          } else {
            for (int j = lo + lig; j < hi; j += LPG) sv[j] *= inv;
          }
        }
      }
    }
    __syncthreads();
    const int nbig = s_nbig;
    for (int b = 0; b < nbig; ++b) {  // CTA-uniform
      const int k = sbig[b], lo = srp[k], hi = srp[k + 1];
      const int64_t row = c0 + k;
      const float u = __ldg(a.U + row * a.ldu);
      if constexpr (!SOFTMAX) {
        for (int j = lo + tid; j < hi; j += TILE_T) sv[j] = score1<ADD, LRELU>(u, sv[j], a.scale);
      } else {
        float m = -INFINITY;
        for (int j = lo + tid; j < hi; j += TILE_T) {
          const float x = score1<ADD, LRELU>(u, sv[j], a.scale);
          sv[j] = x;
          m = fmaxf(m, x);
        }
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, off));
        if (lane == 0) sred[0][warp] = m;
        __syncthreads();
        m = sred[0][0];
#pragma unroll
        for (int w = 1; w < TILE_T / 32; ++w) m = fmaxf(m, sred[0][w]);
        const bool cut = (first_cut && row == r0) || (last_cut && row == rlast);
        float s = 0.f;
        for (int j = lo + tid; j < hi; j += TILE_T) {
          const float x = __expf(sv[j] - m);
          if (!cut) sv[j] = x;
          s += x;
        }
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
        if (lane == 0) sred[1][warp] = s;
        __syncthreads();
        s = 0.f;
#pragma unroll
        for (int w = 0; w < TILE_T / 32; ++w) s += sred[1][w];
        if (cut) {
          if (tid == 0) {
            if (first_cut && row == r0) a.st_first[t] = make_float2(m, s);
            if (last_cut && row == rlast) a.st_last[t] = make_float2(m, s);
          }
        } else {
          const float inv = 1.f / s;
          for (int j = lo + tid; j < hi; j += TILE_T) sv[j] *= inv;
        }
        __syncthreads();  // sred reused by the next big row
      }
    }
  }
  __syncthreads();
  // (C) write the tile back
  if ((reinterpret_cast<uintptr_t>(a.out) & 15) == 0) {
    for (int j = tid * 4; j < ne; j += TILE_T * 4) {
      if (j + 3 < ne) st_pol(reinterpret_cast<float4*>(a.out + e0 + j), *reinterpret_cast<const float4*>(sv + j), pol.stream);
      else
        for (int r = j; r < ne; ++r) st_pol(a.out + e0 + r, sv[r], pol.stream);
    }
  } else {
    for (int j = tid; j < ne; j += TILE_T) st_pol(a.out + e0 + j, sv[j], pol.stream);
  }
}

// crossing rows: the tile a cut row begins in combines the row's in-tile partials in tile order
// (fixed lane assignment + butterfly) and hands (max, 1/sum) to every tile it touches
__global__ void k_sddmm1_xstats(TileArgs a) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t t = warp; t + 1 < a.n_tiles; t += nwarps) {
    const int64_t e0 = t * TILE_E, e1 = e0 + TILE_E;
    const int64_t rl = a.tile_row[t + 1];
    const int64_t p = a.row_ptr[rl];
    if (p >= e1 || p < e0) continue;  // no row continues past e1, or it began in an earlier tile
    const int64_t tb = (a.row_ptr[rl + 1] - 1) / TILE_E;
    float m = -INFINITY, s = 0.f;
    for (int64_t q = t + lane; q <= tb; q += 32) {
      const float2 f = q == t ? a.st_last[t] : a.st_first[q];
      ms_merge(m, s, f.x, f.y);
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1)
      ms_merge(m, s, __shfl_xor_sync(0xffffffffu, m, off), __shfl_xor_sync(0xffffffffu, s, off));
    const float2 fin = make_float2(m, 1.f / s);
    for (int64_t q = t + lane; q <= tb; q += 32) {
      if (q == t) a.fin_last[t] = fin;
      else a.fin_first[q] = fin;
    }
  }
}

__device__ __forceinline__ void xnorm_range(float* __restrict__ out, int64_t lo, int64_t hi, float2 f, int lane) {
  int64_t j = lo + lane;
  for (; j + 96 < hi; j += 128) {
    float x[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) x[q] = out[j + 32 * q];
#pragma unroll
    for (int q = 0; q < 4; ++q) out[j + 32 * q] = __expf(x[q] - f.x) * f.y;
  }
  for (; j < hi; j += 32) out[j] = __expf(out[j] - f.x) * f.y;
}

__global__ void k_sddmm1_xnorm(TileArgs a) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t t = warp; t < a.n_tiles; t += nwarps) {
    const int64_t e0 = t * TILE_E, e1 = min(e0 + (int64_t)TILE_E, a.nnz);
    const int64_t r0 = a.tile_row[t];
    if (a.row_ptr[r0] < e0) xnorm_range(a.out, e0, min(a.row_ptr[r0 + 1], e1), a.fin_first[t], lane);
    if (t + 1 < a.n_tiles) {
      const int64_t p = a.row_ptr[a.tile_row[t + 1]];
      if (p < e1 && p >= e0) xnorm_range(a.out, p, e1, a.fin_last[t], lane);
    }
  }
}

// Entry tiles where they measured faster (B200, tools/sddmm_tile_ab.py, profiles/r02/sddmm_tile/): large
// graphs of moderate degree -- products-shaped (130 M entries, avg 53): normalisation 0.815 -> 0.614 ms,
// scores + softmax 1.076 -> 0.994 ms.  The degree-ordered kernel keeps dense-degree graphs (Reddit, avg
// 508: a warp streams one row's sorted columns; 0.472 vs 0.554 ms) and small ones (arxiv: 315 tiles
// fill two CTAs per SM; 0.015 vs 0.019 ms).  GRANII_SDDMM_TILE=0/1 forces either (A/B runs, tests).
static bool sddmm_tile_enabled(const granii_graph_s* g) {
  const char* e = getenv("GRANII_SDDMM_TILE");
  if (e) return atoi(e) != 0;
  return g->avg_deg() < 128.f && g->local_nnz >= (16ll << 20);
}

template <int LPG, bool ADD, bool LR, bool SM>
static void go_tile(const TileArgs& a, cudaStream_t st) {
  k_sddmm1_tile<LPG, ADD, LR, SM><<<(unsigned)a.n_tiles, TILE_T, 0, st>>>(a);
}

template <bool ADD, bool LR, bool SM>
static void go_tile_lpg(int lpg, const TileArgs& a, cudaStream_t st) {
  switch (lpg) {
    case 32: go_tile<32, ADD, LR, SM>(a, st); break;
    case 16: go_tile<16, ADD, LR, SM>(a, st); break;
    case 8: go_tile<8, ADD, LR, SM>(a, st); break;
    default: go_tile<4, ADD, LR, SM>(a, st); break;
  }
}

static granii_status launch_sddmm1_tile(const granii_graph_s* g, bool add, bool lr, bool sm, const float* U,
                                        int64_t ldu, const float* V, int64_t ldv, float scale, float* out, int sms,
                                        cudaStream_t st) {
  if (g->n_tiles == 0) return GRANII_OK;  // no stored entries
  TileArgs a{g->n_rows, g->local_nnz, g->n_tiles, g->row_ptr, g->col_idx, g->tile_row, U, ldu, V, ldv, scale, out,
             nullptr, nullptr, nullptr, nullptr, l2hint_enabled()};
  if (sm) {
    GR_CUDA(cudaMallocAsync((void**)&a.st_first, 4 * std::max<int64_t>(g->n_tiles, 1) * sizeof(float2), st));
    a.st_last = a.st_first + g->n_tiles;
    a.fin_first = a.st_last + g->n_tiles;
    a.fin_last = a.fin_first + g->n_tiles;
  }
  int lpg = sm ? lpg_for_softmax(g->avg_deg()) : lpg_for_degree(g->avg_deg());
  if (getenv("GRANII_SDDMM_TILE_LPG")) lpg = atoi(getenv("GRANII_SDDMM_TILE_LPG"));  // sweeps
  if (add) {
    if (lr) { if (sm) go_tile_lpg<true, true, true>(lpg, a, st); else go_tile_lpg<true, true, false>(lpg, a, st); }
    else { if (sm) go_tile_lpg<true, false, true>(lpg, a, st); else go_tile_lpg<true, false, false>(lpg, a, st); }
  } else {
    if (lr) { if (sm) go_tile_lpg<false, true, true>(lpg, a, st); else go_tile_lpg<false, true, false>(lpg, a, st); }
    else { if (sm) go_tile_lpg<false, false, true>(lpg, a, st); else go_tile_lpg<false, false, false>(lpg, a, st); }
  }
  GR_CHECK_LAUNCH();
  if (sm) {
    const unsigned b = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(g->n_tiles, 8), (int64_t)sms * 8));
    k_sddmm1_xstats<<<b, 256, 0, st>>>(a);
    k_sddmm1_xnorm<<<b, 256, 0, st>>>(a);
    GR_CHECK_LAUNCH();
    GR_CUDA(cudaFreeAsync(a.st_first, st));
  }
  return GRANII_OK;
}

// K > 1 dot: warp per row, LPG lanes per entry, VEC-wide loads, NJ chunks per lane.
template <int VEC, int LPG, int NJ>
__global__ void __launch_bounds__(256) k_sddmm_dot(SddmmArgs a) {
  constexpr int G = 32 / LPG;
  const int lane = threadIdx.x & 31, grp = lane / LPG, lig = lane % LPG;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t t = warp; t < a.n_seg + a.n_rows; t += nwarps) {  // heavy segments first, then light rows
    const bool seg = t < a.n_seg;
    const int64_t row = seg ? a.seg_row[t] : a.order[t - a.n_seg];
    const int64_t rs = seg ? a.seg_lo[t] : a.row_ptr[row], re = seg ? a.seg_hi[t] : a.row_ptr[row + 1];
    float u[NJ][VEC];
#pragma unroll
    for (int j = 0; j < NJ; ++j)
#pragma unroll
      for (int v = 0; v < VEC; ++v) {
        const int64_t k = (int64_t)(lig + j * LPG) * VEC + v;
        u[j][v] = k < a.K ? __ldg(a.U + row * a.ldu + k) : 0.f;
      }
    for (int64_t e0 = rs; e0 < re; e0 += G) {
      const int64_t e = e0 + grp;
      const bool p = e < re;
      const int32_t c = p ? __ldg(a.col_idx + e) : 0;
      float acc = 0.f;
#pragma unroll
      for (int j = 0; j < NJ; ++j) {
        const int64_t k = (int64_t)(lig + j * LPG) * VEC;
        if (p && k < a.K) {
          const float* vp = a.V + (int64_t)c * a.ldv + k;
          if constexpr (VEC == 4) {
            const float4 t4 = __ldg(reinterpret_cast<const float4*>(vp));
            acc = fmaf(u[j][0], t4.x, acc);
            acc = fmaf(u[j][1], t4.y, acc);
            acc = fmaf(u[j][2], t4.z, acc);
            acc = fmaf(u[j][3], t4.w, acc);
          } else {
            acc = fmaf(u[j][0], __ldg(vp), acc);
          }
        }
      }
#pragma unroll
      for (int off = LPG / 2; off > 0; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
      if (p && lig == 0) a.out[e] = a.scale * acc;
    }
  }
}

// row softmax in place over CSR values (used after the K > 1 dot SDDMM)
template <int LPG>
__global__ void __launch_bounds__(256) k_row_softmax(int64_t n_rows, const int32_t* __restrict__ order,
                                                     const int64_t* __restrict__ row_ptr, float* __restrict__ x) {
  constexpr int G = 32 / LPG;
  const int lane = threadIdx.x & 31, grp = lane / LPG, lig = lane % LPG;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t t0 = warp * G; t0 < n_rows; t0 += nwarps * G) {
    const bool live = t0 + grp < n_rows;
    const int64_t row = live ? order[t0 + grp] : 0;
    const int64_t rs = live ? row_ptr[row] : 0, re = live ? row_ptr[row + 1] : 0;
    float m = -INFINITY, s = 0.f;
    for (int64_t e = rs + lig; e < re; e += LPG) {
      const float v = x[e];
      if (v > m) { s = s * expf(m - v) + 1.f; m = v; } else { s += expf(v - m); }
    }
#pragma unroll
    for (int off = LPG / 2; off > 0; off >>= 1) {
      const float m2 = __shfl_xor_sync(0xffffffffu, m, off), s2 = __shfl_xor_sync(0xffffffffu, s, off);
      const float mn = fmaxf(m, m2);
      const float a1 = (m == -INFINITY) ? 0.f : s * expf(m - mn);
      const float a2 = (m2 == -INFINITY) ? 0.f : s2 * expf(m2 - mn);
      m = mn;
      s = a1 + a2;
    }
    const float inv = 1.f / s;
    for (int64_t e = rs + lig; e < re; e += LPG) x[e] = expf(x[e] - m) * inv;
  }
}

// ---------------------------------------------------------------- segmented softmax of heavy rows
__device__ __forceinline__ void ms_combine(float& m, float& s, float m2, float s2) {
  const float mn = fmaxf(m, m2);
  const float a1 = (m == -INFINITY) ? 0.f : s * expf(m - mn);
  const float a2 = (m2 == -INFINITY) ? 0.f : s2 * expf(m2 - mn);
  m = mn;
  s = a1 + a2;
}

// phase 1: (max, sum exp) of each segment's scores (warp per segment, fixed lane order)
__global__ void k_seg_stats(int64_t n_seg, const int64_t* __restrict__ lo, const int64_t* __restrict__ hi,
                            const float* __restrict__ x, float2* __restrict__ ms) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t t = warp; t < n_seg; t += nwarps) {
    float m = -INFINITY, s = 0.f;
    for (int64_t e = lo[t] + lane; e < hi[t]; e += 32) ms_combine(m, s, x[e], 1.f);
#pragma unroll
    for (int off = 16; off > 0; off >>= 1)
      ms_combine(m, s, __shfl_xor_sync(0xffffffffu, m, off), __shfl_xor_sync(0xffffffffu, s, off));
    if (lane == 0) ms[t] = make_float2(m, s);
  }
}

// phase 2: combine the segments of each heavy row in order
__global__ void k_heavy_stats(int64_t n_heavy, const int32_t* __restrict__ seg_ptr, const float2* __restrict__ ms,
                              float2* __restrict__ hms) {
  for (int64_t h = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; h < n_heavy; h += (int64_t)gridDim.x * blockDim.x) {
    float m = -INFINITY, s = 0.f;
    for (int32_t q = seg_ptr[h]; q < seg_ptr[h + 1]; ++q) ms_combine(m, s, ms[q].x, ms[q].y);
    hms[h] = make_float2(m, 1.f / s);
  }
}

// phase 3: alpha = exp(e - m_row) / sum_row
__global__ void k_seg_norm(int64_t n_seg, const int64_t* __restrict__ lo, const int64_t* __restrict__ hi,
                           const int32_t* __restrict__ seg_heavy, const float2* __restrict__ hms, float* __restrict__ x) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t t = warp; t < n_seg; t += nwarps) {
    const float2 r = hms[seg_heavy[t]];
    for (int64_t e = lo[t] + lane; e < hi[t]; e += 32) x[e] = expf(x[e] - r.x) * r.y;
  }
}

static granii_status heavy_softmax(const granii_graph_s* g, float* out, int sms, cudaStream_t st) {
  if (g->n_seg == 0) return GRANII_OK;
  float2 *ms = nullptr, *hms = nullptr;
  GR_CUDA(cudaMallocAsync((void**)&ms, g->n_seg * sizeof(float2), st));
  GR_CUDA(cudaMallocAsync((void**)&hms, g->n_heavy * sizeof(float2), st));
  const unsigned bw = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(g->n_seg, 8), (int64_t)sms * 8));
  k_seg_stats<<<bw, 256, 0, st>>>(g->n_seg, g->seg_lo, g->seg_hi, out, ms);
  k_heavy_stats<<<(unsigned)ceil_div(g->n_heavy, 256), 256, 0, st>>>(g->n_heavy, g->seg_ptr, ms, hms);
  k_seg_norm<<<bw, 256, 0, st>>>(g->n_seg, g->seg_lo, g->seg_hi, g->seg_heavy, hms, out);
  GR_CHECK_LAUNCH();
  GR_CUDA(cudaFreeAsync(ms, st));
  GR_CUDA(cudaFreeAsync(hms, st));
  return GRANII_OK;
}

// fused row softmax: one step of 4 x LPG entries (held in registers) covers a row of average degree
static int lpg_for_softmax(float avg) {
  if (avg >= 96.f) return 32;
  if (avg >= 24.f) return 16;  // products-shaped (avg 53): 1.45 -> 1.15 ms vs the streaming-only kernel
  if (avg >= 4.f) return 8;    // arxiv-shaped (avg 7.6): 8 lanes beat 4 (more rows per step in flight)
  return 4;
}

static int lpg_for_degree(float avg) {
  if (avg >= 24.f) return 32;
  if (avg >= 12.f) return 16;
  if (avg >= 6.f) return 8;
  return 4;
}

template <int LPG, bool ADD, bool LR, bool SM>
static void go1(const SddmmArgs& a, int blocks, int sms, cudaStream_t st) {
  // three full waves of resident CTAs: the degree-ordered rows are irregular, and CTAs that start
  // as others finish balance the tail (B200 products-shaped, scores + softmax per layer: 8 CTAs / SM
  // where 6 fit 1.21 ms, persistent 1.07, 2 waves 1.01, 3 waves 0.99; GRANII_SDDMM_WAVES overrides)
  const int wv = getenv("GRANII_SDDMM_WAVES") ? atoi(getenv("GRANII_SDDMM_WAVES")) : 3;
  const size_t smem = SM ? (size_t)a.cap * 8 * sizeof(float) : 0;
  const int64_t cap = (int64_t)sms * std::max(wv, 1) * resident_ctas((const void*)k_sddmm1<LPG, ADD, LR, SM>, 256, smem);
  const int64_t b = std::max<int64_t>(1, std::min<int64_t>(cap, (int64_t)blocks * std::max(wv, 1)));
  k_sddmm1<LPG, ADD, LR, SM><<<(unsigned)b, 256, smem, st>>>(a);
}

template <bool ADD, bool LR, bool SM>
static void go1_lpg(int lpg, const SddmmArgs& a, int blocks, int sms, cudaStream_t st) {
  switch (lpg) {
    case 32: go1<32, ADD, LR, SM>(a, blocks, sms, st); break;
    case 16: go1<16, ADD, LR, SM>(a, blocks, sms, st); break;
    case 8: go1<8, ADD, LR, SM>(a, blocks, sms, st); break;
    default: go1<4, ADD, LR, SM>(a, blocks, sms, st); break;
  }
}

granii_status launch_sddmm(const granii_graph_s* g, uint32_t op, const float* U, int64_t ldu, const float* V,
                           int64_t ldv, int64_t K, float scale, float* out, cudaStream_t st) {
  if (g->n_rows == 0) return GRANII_OK;
  DevInfo di;
  GR_TRY(dev_info(&di));
  const uint32_t base = op & 0xF;
  const bool lr = op & GRANII_SDDMM_LEAKYRELU, sm = op & GRANII_SDDMM_ROW_SOFTMAX;
  const int64_t n_light = g->n_rows - g->n_heavy;
  SddmmArgs a{n_light, g->row_ptr, g->col_idx, U, ldu, V, ldv, K, scale, out, g->order + g->n_heavy,
              g->ord_rp + g->n_heavy, g->n_seg, g->seg_lo, g->seg_hi, g->seg_row, l2hint_enabled(), 0};
  // fused softmax: rows longer than one group step are scored into shared memory (4 KB per warp,
  // 32 KB per CTA), GRANII_SDDMM_CAP overrides (0: every long row streams through global memory)
  a.cap = getenv("GRANII_SDDMM_CAP") ? atoi(getenv("GRANII_SDDMM_CAP")) : 1024;
  // algorithmic bytes: per entry col id + V row (4K) + out; per row row_ptr + U row
  const double nnz = (double)g->local_nnz, R = (double)g->n_rows;
  const double gathered = (double)g->n_cols * 4.0 * (double)K;  // V, read once in the compulsory count
  // "sddmm" (K = 1: one 4-byte V gather per entry, bound by the gather rate, bench.py) / "sddmm_dot"
  ProfScope ps(K == 1 ? "sddmm" : "sddmm_dot", st, nnz * (8.0 + 4.0 * K) + R * (8.0 + 4.0 * K), 2.0 * nnz * K, (K > 1 && sm) ? 2 : 1,
               nnz * 8.0 + R * (8.0 + 4.0 * K) + gathered, gathered <= 0.6 * (double)di.l2_bytes);
  if (K == 1 && sddmm_tile_enabled(g)) {
    ps.add_launches(sm ? 2 : 0);
    return launch_sddmm1_tile(g, base == GRANII_SDDMM_ADD, lr, sm, U, ldu, V, ldv, scale, out, di.sms, st);
  }
  if (K == 1) {
    const int lpg = sm ? lpg_for_softmax(g->avg_deg()) : lpg_for_degree(g->avg_deg());
    const int64_t units = ceil_div(n_light, 32 / lpg) + g->n_seg;
    const int blocks = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(units, 8), (int64_t)di.sms * 8));
    const bool add = base == GRANII_SDDMM_ADD;
    // dispatch the 8 (add, lrelu, softmax) variants
    if (add) {
      if (lr) { if (sm) go1_lpg<true, true, true>(lpg, a, blocks, di.sms, st); else go1_lpg<true, true, false>(lpg, a, blocks, di.sms, st); }
      else { if (sm) go1_lpg<true, false, true>(lpg, a, blocks, di.sms, st); else go1_lpg<true, false, false>(lpg, a, blocks, di.sms, st); }
    } else {
      if (lr) { if (sm) go1_lpg<false, true, true>(lpg, a, blocks, di.sms, st); else go1_lpg<false, true, false>(lpg, a, blocks, di.sms, st); }
      else { if (sm) go1_lpg<false, false, true>(lpg, a, blocks, di.sms, st); else go1_lpg<false, false, false>(lpg, a, blocks, di.sms, st); }
    }
    GR_CHECK_LAUNCH();
    if (sm) GR_TRY(heavy_softmax(g, out, di.sms, st));
    return GRANII_OK;
  }
  if (base != GRANII_SDDMM_DOT) return fail(GRANII_ERR_INVALID_ARG, "SDDMM ADD requires K == 1");
  if (lr) return fail(GRANII_ERR_UNSUPPORTED, "LEAKYRELU with K > 1 is not supported");
  const bool vec4 = (ldu % 4 == 0) && (ldv % 4 == 0) && ((uintptr_t)V % 16 == 0);
  const int blocks = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n_light + g->n_seg, 8), (int64_t)di.sms * 8));
#define GO(VEC, LPG, NJ) \
  k_sddmm_dot<VEC, LPG, NJ><<<(unsigned)persistent_grid(k_sddmm_dot<VEC, LPG, NJ>, 256, di.sms, blocks), 256, 0, st>>>(a)
  if (vec4) {
    if (K <= 16) GO(4, 4, 1);
    else if (K <= 32) GO(4, 8, 1);
    else if (K <= 64) GO(4, 16, 1);
    else if (K <= 128) GO(4, 32, 1);
    else if (K <= 256) GO(4, 32, 2);
    else if (K <= 512) GO(4, 32, 4);
    else if (K <= 1024) GO(4, 32, 8);
    else return fail(GRANII_ERR_UNSUPPORTED, "SDDMM DOT with K > 1024");
  } else {
    if (K <= 32) GO(1, 32, 1);
    else if (K <= 64) GO(1, 32, 2);
    else if (K <= 128) GO(1, 32, 4);
    else if (K <= 256) GO(1, 32, 8);
    else if (K <= 512) GO(1, 32, 16);
    else return fail(GRANII_ERR_UNSUPPORTED, "unaligned SDDMM DOT with K > 512");
  }
#undef GO
  GR_CHECK_LAUNCH();
  if (sm) {
    const int lpg = lpg_for_degree(g->avg_deg());
    const int64_t units = ceil_div(n_light, 32 / lpg);
    const int b2 = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(units, 8), (int64_t)di.sms * 8));
    switch (lpg) {
      case 32: k_row_softmax<32><<<(unsigned)persistent_grid(k_row_softmax<32>, 256, di.sms, b2), 256, 0, st>>>(n_light, a.order, g->row_ptr, out); break;
      case 16: k_row_softmax<16><<<(unsigned)persistent_grid(k_row_softmax<16>, 256, di.sms, b2), 256, 0, st>>>(n_light, a.order, g->row_ptr, out); break;
      case 8: k_row_softmax<8><<<(unsigned)persistent_grid(k_row_softmax<8>, 256, di.sms, b2), 256, 0, st>>>(n_light, a.order, g->row_ptr, out); break;
      default: k_row_softmax<4><<<(unsigned)persistent_grid(k_row_softmax<4>, 256, di.sms, b2), 256, 0, st>>>(n_light, a.order, g->row_ptr, out); break;
    }
    GR_CHECK_LAUNCH();
    GR_TRY(heavy_softmax(g, out, di.sms, st));
  }
  return GRANII_OK;
}

}  // namespace granii
