// spmm.cu -- g-SpMM (+, x) on CSR (unweighted form L117):
//   Y_i = rs_i * sum_{e in row i} w_e * cs_{c(e)} * X[c(e), k0:k0+kw]   (+ ReLU)
//
// B200 design: the op is a gather -- per stored entry it reads
// one K-row of X (4K bytes) -- so it is bound by the L2->SM gather bandwidth
// when X fits in L2 and by HBM when it does not.  Two schedules:
//   * warp-per-row (dense-degree graphs): the warp loads 32 column ids (+w)
//     coalesced, then G = 32/LPG lane groups each take one neighbour at a time
//     and gather its row slice with 16-byte loads (VEC = 4), U neighbours per
//     group in flight; groups are reduced with shuffles at the end.
//   * group-per-row (sparse graphs, avg degree < 16): an LPG-lane group owns a
//     row, 32/LPG rows per warp.
// Rows are visited in the degree-descending schedule computed at graph
// creation (round-robin over warps = LPT balance for power-law graphs).
// Row/column scales fuse the two row-broadcasts of Eq. 2 (L115) into the
// gather and the epilogue.  No atomics: each output row is written once by
// one warp/group, reduction order fixed => bitwise reproducible.
#include <algorithm>

#include "cache.cuh"
#include "internal.h"

namespace granii {

template <int VEC>
struct VecT;
template <>
struct VecT<4> {
  using T = float4;
};
template <>
struct VecT<1> {
  using T = float;
};

template <int VEC>
__device__ __forceinline__ void ldv(const float* p, float (&v)[VEC]) {
  if constexpr (VEC == 4) {
    float4 t = __ldg(reinterpret_cast<const float4*>(p));
    v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
  } else {
    v[0] = __ldg(p);
  }
}
// the gathered operand: L2 policy `pol` (keep: evict_last)
template <int VEC>
__device__ __forceinline__ void ldv(const float* p, float (&v)[VEC], uint64_t pol) {
  if constexpr (VEC == 4) {
    float4 t = ldg_pol(reinterpret_cast<const float4*>(p), pol);
    v[0] = t.x; v[1] = t.y; v[2] = t.z; v[3] = t.w;
  } else {
    v[0] = ldg_pol(p, pol);
  }
}
template <int VEC>
__device__ __forceinline__ void stv(float* p, const float (&v)[VEC], uint64_t pol) {
  if constexpr (VEC == 4) {
    st_pol(reinterpret_cast<float4*>(p), make_float4(v[0], v[1], v[2], v[3]), pol);
  } else {
    st_pol(p, v[0], pol);
  }
}
template <int VEC>
__device__ __forceinline__ void stv(float* p, const float (&v)[VEC]) {
  if constexpr (VEC == 4) {
    *reinterpret_cast<float4*>(p) = make_float4(v[0], v[1], v[2], v[3]);
  } else {
    p[0] = v[0];
  }
}

struct SpmmArgs {
  int64_t n_rows;                          // light rows (scheduled through `order`)
  const int64_t* __restrict__ row_ptr;
  const int32_t* __restrict__ col_idx;
  const float* __restrict__ vals;
  const float* __restrict__ X;
  int64_t ldx;
  int64_t k0, kw;        // column slice [k0, k0+kw)
  float* __restrict__ Y;
  int64_t ldy;
  const float* __restrict__ rs;
  const float* __restrict__ cs;
  int relu;
  const int32_t* __restrict__ order;       // light rows, degree-descending
  const longlong2* __restrict__ ord_rp;    // their entry ranges, same order
  int64_t n_lwide;                         // group-per-row kernel: order[0 .. n_lwide) get a warp each
  // heavy rows (degree > GRANII_SEG) are cut into segments: warp-wide work items whose
  // unscaled partial sums go to `partial` [n_seg][ldp] and are combined in fixed order
  int64_t n_seg;
  const int64_t* __restrict__ seg_lo;
  const int64_t* __restrict__ seg_hi;
  float* __restrict__ partial;
  int64_t ldp;
  // optional dense addend fused in the epilogue: Y_i = act(rs_i * sum + beta * B_i)
  // (GIN's ε self term, TAGCN's Horner step); B holds the owned rows
  const float* __restrict__ B;
  int64_t ldb;
  float beta;
  // block-phased mode (owner_off != nullptr; layer.cu gathered_spmm, N1): only the entries whose
  // column lies in the owner blocks [p0, p1) of the gather buffer, block `skip` excluded (-1: none).
  // `first`: start from zero, else from the raw partial already in Y (light rows) / partial
  // (segments); `last`: apply the epilogue.
  const int32_t* __restrict__ owner_off;   // [n_rows][G1]
  const int32_t* __restrict__ ord_off;     // owner_off of the light rows in schedule order [n_rows][G1]
  const int32_t* __restrict__ seg_row;     // row of each heavy segment
  int G1, p0, p1, skip, first, last;
  // fused additive attention (GAT, Eq. 4-6; ATT kernels): the weights are computed on the fly,
  // w_e = exp(LeakyReLU(el_i + er_c) - m_i) / s_i with an online row max m_i and sum s_i; er
  // travels in `cs` (prefetched a chunk ahead like a column scale), heavy segments leave their
  // (m, s) in seg_ms for the softmax-aware combine
  const float* __restrict__ el;
  float2* __restrict__ seg_ms;
  int l2hint;                              // L2 eviction priorities on (cache.cuh; GRANII_L2HINT)
};

// online-softmax state of one row (or segment), warp-uniform m, per-lane partial s
struct AttState {
  float el, m, s;
};

// part r (0, or 1 after a skipped block) of the entries of `row` within [l0, h0) whose column lies
// in the phase's owner blocks
// (o: the row's owner offsets, base: its first entry)
__device__ __forceinline__ void phase_part(const SpmmArgs& a, const int32_t* o, int64_t base, int r, int64_t l0,
                                           int64_t h0, int64_t& lo, int64_t& hi) {
  const int b0 = r == 0 ? a.p0 : a.skip + 1;
  const int b1 = (r == 0 && a.skip >= 0) ? a.skip : a.p1;
  lo = max(l0, base + (int64_t)o[b0]);
  hi = min(h0, base + (int64_t)o[b1]);
}

// continue a phased accumulation from the raw partial stored by the previous phase
template <int LPG, int NJ, int VEC>
__device__ __forceinline__ void load_partial(const float* y, const bool (&colok)[NJ], float (&acc)[NJ][VEC]) {
#pragma unroll
  for (int j = 0; j < NJ; ++j)
    if (colok[j]) ldv<VEC>(y + j * LPG * VEC, acc[j]);
}

// One chunk of 32 entries of a row, one per lane: column id and weight.  Lanes
// past the range's end reuse its last column with w = 0, so every later step is
// branch-free (the padded gathers hit L1 and add exact zeros).
template <bool W>
__device__ __forceinline__ void load_chunk(const SpmmArgs& a, int64_t e, int64_t re, int lane, int32_t& c, float& w,
                                           const L2Pol& pol) {
  const bool valid = e + lane < re;
  const int64_t ee = valid ? e + lane : re - 1;
  c = ldg_stream(a.col_idx + ee, pol.stream);
  w = valid ? (W ? ldg_stream(a.vals + ee, pol.stream) : 1.f) : 0.f;
}

// The whole warp accumulates entries [rs0, re): G = 32/LPG lane groups each take a
// neighbour, U neighbours per group in flight; acc holds this lane's group partial.
template <int VEC, int LPG, int NJ, bool W, bool CS, int U, bool ATT = false>
__device__ __forceinline__ void warp_range(const SpmmArgs& a, int64_t rs0, int64_t re, int lane, int grp,
                                           const char* const (&xbj)[NJ], uint32_t row_bytes, float (&acc)[NJ][VEC],
                                           const L2Pol& pol, AttState* at = nullptr) {
  constexpr int G = 32 / LPG;
  if (rs0 >= re) return;
  // distance-2 prefetch: (c0, w0, cs0) = next chunk, (c1, w1) = the chunk after; the
  // dependent col-scale gather cs[c] of a chunk is issued one chunk before its use
  int32_t c0, c1 = 0;
  float w0, w1 = 0.f, cs0 = 1.f;
  load_chunk<W>(a, rs0, re, lane, c0, w0, pol);
  if (CS) cs0 = ldg_pol(a.cs + c0, pol.keep);
  if (rs0 + 32 < re) load_chunk<W>(a, rs0 + 32, re, lane, c1, w1, pol);
  for (int64_t base = rs0; base < re; base += 32) {
    const int32_t c = c0;
    float w = CS ? w0 * cs0 : w0;
    if constexpr (ATT) {
      // scores of this chunk (cs0 = er of the lane's column; padding lanes have w0 = 0), chunk max
      // over the warp, rescale of the running state when it grows, then the chunk's weights
      const float z = at->el + cs0;
      const float ev = w0 != 0.f ? (z > 0.f ? z : 0.2f * z) : -INFINITY;
      float cm = ev;
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) cm = fmaxf(cm, __shfl_xor_sync(0xffffffffu, cm, off));
      if (cm > at->m) {  // warp-uniform
        const float f = __expf(at->m - cm);  // 0 on the first chunk (m = -inf)
#pragma unroll
        for (int j = 0; j < NJ; ++j)
#pragma unroll
          for (int v = 0; v < VEC; ++v) acc[j][v] *= f;
        at->s *= f;
        at->m = cm;
      }
      w = w0 != 0.f ? __expf(ev - at->m) : 0.f;
      at->s += w;
    }
    if (base + 32 < re) {
      c0 = c1;
      w0 = w1;
      if (CS) cs0 = ldg_pol(a.cs + c0, pol.keep);                               // c1 landed a chunk ago
      if (base + 64 < re) load_chunk<W>(a, base + 64, re, lane, c1, w1, pol);  // two chunks ahead
    }
    const int cnt = (int)((re - base) < 32 ? (re - base) : 32);
    const int steps = (cnt + G * U - 1) / (G * U);  // warp-uniform
    for (int s = 0; s < steps; ++s) {
      uint32_t cu[U];
      float wu[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int i = s * G * U + u * G + grp;  // <= 31
        cu[u] = (uint32_t)__shfl_sync(0xffffffffu, c, i);
        wu[u] = __shfl_sync(0xffffffffu, w, i);
      }
      float x[U][NJ][VEC];
#pragma unroll
      for (int u = 0; u < U; ++u) {
#pragma unroll
        for (int j = 0; j < NJ; ++j)
          ldv<VEC>(reinterpret_cast<const float*>(xbj[j] + (uint64_t)cu[u] * row_bytes), x[u][j], pol.keep);
      }
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int j = 0; j < NJ; ++j)
#pragma unroll
          for (int v = 0; v < VEC; ++v) acc[j][v] = fmaf(wu[u], x[u][j][v], acc[j][v]);
    }
  }
}

// per-lane column offsets of a slice: lanes past it re-read its last in-bounds
// vector (ldx >= k0 + kw rounded to VEC), so gathers are unconditional; never stored
template <int VEC, int LPG, int NJ>
__device__ __forceinline__ void slice_setup(const SpmmArgs& a, int lig, bool (&colok)[NJ], const char* (&xbj)[NJ]) {
  const int last = (int)((a.kw - 1) / VEC);
  const char* __restrict__ xb = reinterpret_cast<const char*>(a.X + a.k0);
#pragma unroll
  for (int j = 0; j < NJ; ++j) {
    const int v = lig + j * LPG;
    colok[j] = v <= last;
    xbj[j] = xb + (uint32_t)((v <= last ? v : last) * VEC * 4);  // one 64-bit base per vector
  }
}

template <int NJ, int VEC>
__device__ __forceinline__ void zero(float (&acc)[NJ][VEC]) {
#pragma unroll
  for (int j = 0; j < NJ; ++j)
#pragma unroll
    for (int v = 0; v < VEC; ++v) acc[j][v] = 0.f;
}

// sum the G lane groups (fixed butterfly order)
template <int LPG, int NJ, int VEC>
__device__ __forceinline__ void reduce_groups(float (&acc)[NJ][VEC]) {
#pragma unroll
  for (int off = LPG; off < 32; off <<= 1)
#pragma unroll
    for (int j = 0; j < NJ; ++j)
#pragma unroll
      for (int v = 0; v < VEC; ++v) acc[j][v] += __shfl_xor_sync(0xffffffffu, acc[j][v], off);
}

template <int LPG, int NJ, int VEC>
__device__ __forceinline__ void store_row(float* y, const bool (&colok)[NJ], const float (&acc)[NJ][VEC], float s,
                                          int relu, const float* b = nullptr, float beta = 0.f,
                                          const L2Pol* pol = nullptr) {
#pragma unroll
  for (int j = 0; j < NJ; ++j) {
    if (!colok[j]) continue;
    float o[VEC];
    float bv[VEC];
    if (b) ldv<VEC>(b + j * LPG * VEC, bv);
#pragma unroll
    for (int v = 0; v < VEC; ++v) {
      o[v] = acc[j][v] * s;
      if (b) o[v] = fmaf(beta, bv[v], o[v]);
      if (relu) o[v] = fmaxf(o[v], 0.f);
    }
    if (pol) stv<VEC>(y + j * LPG * VEC, o, pol->stream);  // the output row: written once
    else stv<VEC>(y + j * LPG * VEC, o);
  }
}

// heavy-row segments first (largest work first), as warp-wide items
template <int VEC, int LPG, int NJ, bool W, bool CS, bool PH, int U, bool ATT = false>
__device__ __forceinline__ void do_segment(const SpmmArgs& a, int64_t t, int lane, int grp, int lig,
                                           const bool (&colok)[NJ], const char* const (&xbj)[NJ],
                                           uint32_t row_bytes, const L2Pol& pol) {
  float acc[NJ][VEC];
  zero(acc);
  float* part = a.partial + t * a.ldp + (int64_t)lig * VEC;
  if constexpr (ATT) {
    AttState at{__ldg(a.el + a.seg_row[t]), -INFINITY, 0.f};
    warp_range<VEC, LPG, NJ, false, true, U, true>(a, a.seg_lo[t], a.seg_hi[t], lane, grp, xbj, row_bytes, acc, pol,
                                                   &at);
    reduce_groups<LPG>(acc);
    float st = at.s;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) st += __shfl_xor_sync(0xffffffffu, st, off);
    if (grp == 0) store_row<LPG>(part, colok, acc, 1.f, 0);
    if (lane == 0) a.seg_ms[t] = make_float2(at.m, st);
    return;
  }
  if constexpr (PH) {
    if (!a.first && grp == 0) load_partial<LPG>(part, colok, acc);
    for (int r = 0; r < (a.skip >= 0 ? 2 : 1); ++r) {  // the range(s) are computed when needed
      int64_t lo, hi;
      const int64_t sr = a.seg_row[t];
      phase_part(a, a.owner_off + sr * a.G1, a.row_ptr[sr], r, a.seg_lo[t], a.seg_hi[t], lo, hi);
      warp_range<VEC, LPG, NJ, W, CS, U>(a, lo, hi, lane, grp, xbj, row_bytes, acc, pol);
    }
  } else {
    warp_range<VEC, LPG, NJ, W, CS, U>(a, a.seg_lo[t], a.seg_hi[t], lane, grp, xbj, row_bytes, acc, pol);
  }
  reduce_groups<LPG>(acc);
  if (grp == 0) store_row<LPG>(part, colok, acc, 1.f, 0);
}

// one row, the whole warp: G lane groups share its entries
template <int VEC, int LPG, int NJ, bool W, bool CS, bool PH, int U, bool ATT = false>
__device__ __forceinline__ void warp_row(const SpmmArgs& a, int64_t t, int lane, int grp, int lig,
                                         const bool (&colok)[NJ], const char* const (&xbj)[NJ], uint32_t row_bytes,
                                         const L2Pol& pol) {
    // t: position in the light-row schedule; the row and its entry range are independent loads
    const int64_t row = a.order[t];
    const longlong2 rr = a.ord_rp[t];
    float acc[NJ][VEC];
    zero(acc);
    float* y = a.Y + row * a.ldy + a.k0 + (int64_t)lig * VEC;
    if constexpr (ATT) {
      AttState at{__ldg(a.el + row), -INFINITY, 0.f};
      warp_range<VEC, LPG, NJ, false, true, U, true>(a, rr.x, rr.y, lane, grp, xbj, row_bytes, acc, pol, &at);
      reduce_groups<LPG>(acc);
      float st = at.s;
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) st += __shfl_xor_sync(0xffffffffu, st, off);
      const float inv = st > 0.f ? 1.f / st : 0.f;
      if (grp == 0) store_row<LPG>(y, colok, acc, (a.rs ? __ldg(a.rs + row) : 1.f) * inv, a.relu, nullptr, 0.f, &pol);
      return;
    }
    if constexpr (PH) {
      if (!a.first && grp == 0) load_partial<LPG>(y, colok, acc);
      for (int r = 0; r < (a.skip >= 0 ? 2 : 1); ++r) {
        int64_t lo, hi;
        phase_part(a, a.ord_off + t * a.G1, rr.x, r, 0, INT64_MAX, lo, hi);
        warp_range<VEC, LPG, NJ, W, CS, U>(a, lo, hi, lane, grp, xbj, row_bytes, acc, pol);
      }
    } else {
      warp_range<VEC, LPG, NJ, W, CS, U>(a, rr.x, rr.y, lane, grp, xbj, row_bytes, acc, pol);
    }
    reduce_groups<LPG>(acc);
    if (grp == 0) {
      if (PH && !a.last) store_row<LPG>(y, colok, acc, 1.f, 0);
      else
        store_row<LPG>(y, colok, acc, a.rs ? __ldg(a.rs + row) : 1.f, a.relu,
                       a.B ? a.B + row * a.ldb + a.k0 + (int64_t)lig * VEC : nullptr, a.beta, &pol);
    }
}

// ------------------------------------------------------------------ warp-per-row
// defaults (tools/spmm_sweep.py on B200, Reddit- and products-shaped graphs): 16-byte gathers of
// <= 2 vectors per lane keep 2 neighbours per group in flight at 4 blocks/SM (64 registers);
// wider rows keep the register budget of 3 blocks/SM
template <int VEC, int NJ>
constexpr int spmm_minb() { return VEC == 4 && NJ <= 2 ? 4 : 3; }
template <int VEC, int LPG, int NJ>
constexpr int spmm_unroll() { return VEC == 4 && NJ <= 2 ? 2 : (LPG >= 8 ? 4 : 32 / (32 / LPG)); }

template <int VEC, int LPG, int NJ, bool W, bool CS, bool PH, int UU = 0, int MINB = 0, bool ATT = false>
__global__ void __launch_bounds__(256, MINB > 0 ? MINB : spmm_minb<VEC, NJ>()) k_spmm_warp(SpmmArgs a) {
  constexpr int G = 32 / LPG;
  constexpr int U = UU > 0 ? UU : spmm_unroll<VEC, LPG, NJ>();  // neighbours per group per step
  static_assert(32 % (G * U) == 0, "G*U must divide 32");
  const int lane = threadIdx.x & 31, grp = lane / LPG, lig = lane % LPG;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  bool colok[NJ];
  const char* xbj[NJ];
  slice_setup<VEC, LPG>(a, lig, colok, xbj);
  const uint32_t row_bytes = (uint32_t)(a.ldx * 4);
  const L2Pol pol = make_l2pol(a.l2hint);
  for (int64_t t = warp; t < a.n_seg + a.n_rows; t += nwarps) {
    if (t < a.n_seg) {
      do_segment<VEC, LPG, NJ, W, CS, PH, U, ATT>(a, t, lane, grp, lig, colok, xbj, row_bytes, pol);
      continue;
    }
    warp_row<VEC, LPG, NJ, W, CS, PH, U, ATT>(a, t - a.n_seg, lane, grp, lig, colok, xbj, row_bytes, pol);
  }
}

// ------------------------------------------------------------------ group-per-row
template <int VEC, int LPG, int NJ, bool W, bool CS, bool PH>
__global__ void __launch_bounds__(256, 3) k_spmm_group(SpmmArgs a) {
  constexpr int G = 32 / LPG;
  constexpr int U = 4;
  constexpr int UW = 32 / G >= 4 ? 4 : 32 / G;
  const int lane = threadIdx.x & 31, grp = lane / LPG, lig = lane % LPG;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  bool colok[NJ];
  const char* xbj[NJ];
  slice_setup<VEC, LPG>(a, lig, colok, xbj);
  const uint32_t row_bytes = (uint32_t)(a.ldx * 4);
  const L2Pol pol = make_l2pol(a.l2hint);
  // heavy segments, then the wide light rows (degree > wide_deg): whole warps, largest first
  for (int64_t t = warp; t < a.n_seg + a.n_lwide; t += nwarps) {
    if (t < a.n_seg) do_segment<VEC, LPG, NJ, W, CS, PH, UW>(a, t, lane, grp, lig, colok, xbj, row_bytes, pol);
    else warp_row<VEC, LPG, NJ, W, CS, PH, UW>(a, t - a.n_seg, lane, grp, lig, colok, xbj, row_bytes, pol);
  }
  // the other light rows: one LPG-lane group per row
  for (int64_t t0 = a.n_lwide + warp * G; t0 < a.n_rows; t0 += nwarps * G) {
    const int64_t t = t0 + grp;
    if (t >= a.n_rows) continue;
    const int64_t row = a.order[t];
    const longlong2 rr = a.ord_rp[t];
    float acc[NJ][VEC];
    zero(acc);
    float* y = a.Y + row * a.ldy + a.k0 + (int64_t)lig * VEC;
    if (PH && !a.first) load_partial<LPG>(y, colok, acc);
    for (int part = 0; part < (PH && a.skip >= 0 ? 2 : 1); ++part) {
      int64_t rs0, re;
      if constexpr (PH) {
        phase_part(a, a.ord_off + t * a.G1, rr.x, part, 0, INT64_MAX, rs0, re);
      } else {
        rs0 = rr.x;
        re = rr.y;
      }
    for (int64_t e = rs0; e < re; e += U) {
      uint32_t cu[U];
      float wu[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {  // entries past the row end: last entry, weight 0
        const bool ok = e + u < re;
        const int64_t ee = ok ? e + u : re - 1;
        cu[u] = (uint32_t)ldg_stream(a.col_idx + ee, pol.stream);
        wu[u] = ok ? (W ? ldg_stream(a.vals + ee, pol.stream) : 1.f) : 0.f;
        if (CS) wu[u] *= ldg_pol(a.cs + cu[u], pol.keep);
      }
      float x[U][NJ][VEC];
#pragma unroll
      for (int u = 0; u < U; ++u) {
#pragma unroll
        for (int j = 0; j < NJ; ++j)
          ldv<VEC>(reinterpret_cast<const float*>(xbj[j] + (uint64_t)cu[u] * row_bytes), x[u][j], pol.keep);
      }
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int j = 0; j < NJ; ++j)
#pragma unroll
          for (int v = 0; v < VEC; ++v) acc[j][v] = fmaf(wu[u], x[u][j][v], acc[j][v]);
    }
    }
    if (PH && !a.last) store_row<LPG>(y, colok, acc, 1.f, 0);
    else
      store_row<LPG>(y, colok, acc, a.rs ? __ldg(a.rs + row) : 1.f, a.relu,
                     a.B ? a.B + row * a.ldb + a.k0 + (int64_t)lig * VEC : nullptr, a.beta, &pol);
  }
}

// heavy rows: Y_r = rs_r * sum_{segments of r, in order} partial (+ ReLU)
__global__ void k_spmm_combine(int64_t n_heavy, const int32_t* __restrict__ heavy_rows,
                               const int32_t* __restrict__ seg_ptr, const float* __restrict__ partial, int64_t ldp,
                               int64_t k0, int64_t kw, float* __restrict__ Y, int64_t ldy,
                               const float* __restrict__ rs, int relu, const float* __restrict__ B, int64_t ldb,
                               float beta) {
  const int64_t total = n_heavy * kw;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t h = i / kw, k = i % kw;
    float s = 0.f;
    for (int32_t q = seg_ptr[h]; q < seg_ptr[h + 1]; ++q) s += partial[(int64_t)q * ldp + k];
    const int64_t row = heavy_rows[h];
    s *= rs ? rs[row] : 1.f;
    if (B) s = fmaf(beta, B[row * ldb + k0 + k], s);
    if (relu) s = fmaxf(s, 0.f);
    Y[row * ldy + k0 + k] = s;
  }
}

// heavy rows of the fused attention: Y_r = rs_r * sum_q partial_q exp(m_q - M) / sum_q s_q exp(m_q - M),
// M = max_q m_q, segments in fixed order
__global__ void k_spmm_combine_att(int64_t n_heavy, const int32_t* __restrict__ heavy_rows,
                                   const int32_t* __restrict__ seg_ptr, const float* __restrict__ partial,
                                   int64_t ldp, const float2* __restrict__ seg_ms, int64_t k0, int64_t kw,
                                   float* __restrict__ Y, int64_t ldy, const float* __restrict__ rs, int relu) {
  const int64_t total = n_heavy * kw;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t h = i / kw, k = i % kw;
    float M = -INFINITY;
    for (int32_t q = seg_ptr[h]; q < seg_ptr[h + 1]; ++q) M = fmaxf(M, seg_ms[q].x);
    float v = 0.f, S = 0.f;
    for (int32_t q = seg_ptr[h]; q < seg_ptr[h + 1]; ++q) {
      const float f = seg_ms[q].x == -INFINITY ? 0.f : __expf(seg_ms[q].x - M);
      v = fmaf(partial[(int64_t)q * ldp + k], f, v);
      S = fmaf(seg_ms[q].y, f, S);
    }
    const int64_t row = heavy_rows[h];
    float o = v * (S > 0.f ? 1.f / S : 0.f) * (rs ? rs[row] : 1.f);
    if (relu) o = fmaxf(o, 0.f);
    Y[row * ldy + k0 + k] = o;
  }
}

// ------------------------------------------------------------------ dispatch
template <int VEC, int LPG, int NJ, bool PH>
static granii_status launch_cfg(const SpmmArgs& a, bool warp_mode, bool w, bool cs, int sms, cudaStream_t st) {
  const int threads = 256;
  int64_t units = (warp_mode ? a.n_rows : a.n_lwide + ceil_div(a.n_rows - a.n_lwide, 32 / LPG)) + a.n_seg;
  // enough warps for 8 resident blocks/SM, capped by the work available
  int64_t blocks = std::min<int64_t>(ceil_div(units, threads / 32), (int64_t)sms * 8);
  blocks = std::max<int64_t>(blocks, 1);
#define GR_L(K) K<<<(unsigned)blocks, threads, 0, st>>>(a)
  if constexpr (VEC == 4 && !PH) {
    if (a.el) {  // fused attention: warp-per-row only (the caller checks spmm_att_supported)
      GR_L((k_spmm_warp<VEC, LPG, NJ, false, true, false, 0, 0, true>));
      GR_CHECK_LAUNCH();
      return GRANII_OK;
    }
  }
  // tuning hook (GRANII_SPMM_TUNE="U,MINB"): alternative unroll / occupancy for the
  // warp-per-row kernels of the dominant shapes (tools/spmm_sweep.py)
  if constexpr (!PH && VEC == 4 && NJ == 2 && (LPG == 8 || LPG == 16 || LPG == 32)) {
    const char* tune = getenv("GRANII_SPMM_TUNE");
    if (warp_mode && tune) {
      int u = 0, mb = 0;
      sscanf(tune, "%d,%d", &u, &mb);
      const int64_t bl = std::max<int64_t>(1, std::min<int64_t>(ceil_div(units, threads / 32), (int64_t)sms * 16));
#define GR_T2(W_, C_, U_, M_) k_spmm_warp<VEC, LPG, NJ, W_, C_, false, U_, M_><<<(unsigned)bl, threads, 0, st>>>(a)
#define GR_T(U_, M_)                  \
  do {                                \
    if (w && cs) GR_T2(true, true, U_, M_);   \
    else if (w) GR_T2(true, false, U_, M_);   \
    else if (cs) GR_T2(false, true, U_, M_);  \
    else GR_T2(false, false, U_, M_);         \
  } while (0)
      if (u == 4 && mb == 4) GR_T(4, 4);
      else if (u == 4 && mb == 3) GR_T(4, 3);
      else GR_T(2, 3);
#undef GR_T
#undef GR_T2
      GR_CHECK_LAUNCH();
      return GRANII_OK;
    }
  }
  if (warp_mode) {
    if (w && cs) GR_L((k_spmm_warp<VEC, LPG, NJ, true, true, PH>));
    else if (w) GR_L((k_spmm_warp<VEC, LPG, NJ, true, false, PH>));
    else if (cs) GR_L((k_spmm_warp<VEC, LPG, NJ, false, true, PH>));
    else GR_L((k_spmm_warp<VEC, LPG, NJ, false, false, PH>));
  } else {
    if (w && cs) GR_L((k_spmm_group<VEC, LPG, NJ, true, true, PH>));
    else if (w) GR_L((k_spmm_group<VEC, LPG, NJ, true, false, PH>));
    else if (cs) GR_L((k_spmm_group<VEC, LPG, NJ, false, true, PH>));
    else GR_L((k_spmm_group<VEC, LPG, NJ, false, false, PH>));
  }
#undef GR_L
  GR_CHECK_LAUNCH();
  return GRANII_OK;
}

// Pick (VEC, LPG, NJ) for a slice of width kw.  VEC=4 needs 16-byte aligned rows.
template <bool PH>
static granii_status launch_slice(const SpmmArgs& a, bool vec4, bool warp_mode, bool w, bool cs, int sms,
                                  cudaStream_t st) {
  const int64_t kw = a.kw;
  if (vec4) {
    if (kw <= 16) return launch_cfg<4, 4, 1, PH>(a, warp_mode, w, cs, sms, st);
    if (kw <= 32) return launch_cfg<4, 8, 1, PH>(a, warp_mode, w, cs, sms, st);
    if (kw <= 64) {
      if (warp_mode) return launch_cfg<4, 8, 2, PH>(a, warp_mode, w, cs, sms, st);  // 4 groups x 2 float4
      return launch_cfg<4, 16, 1, PH>(a, warp_mode, w, cs, sms, st);
    }
    if (kw <= 128) {
      if (warp_mode) return launch_cfg<4, 16, 2, PH>(a, warp_mode, w, cs, sms, st);
      return launch_cfg<4, 32, 1, PH>(a, warp_mode, w, cs, sms, st);
    }
    if (kw <= 256) return launch_cfg<4, 32, 2, PH>(a, warp_mode, w, cs, sms, st);
    if (kw <= 512) return launch_cfg<4, 32, 4, PH>(a, warp_mode, w, cs, sms, st);
    return launch_cfg<4, 32, 8, PH>(a, warp_mode, w, cs, sms, st);
  }
  if (kw <= 32) return launch_cfg<1, 32, 1, PH>(a, warp_mode, w, cs, sms, st);
  if (kw <= 64) return launch_cfg<1, 32, 2, PH>(a, warp_mode, w, cs, sms, st);
  if (kw <= 128) return launch_cfg<1, 32, 4, PH>(a, warp_mode, w, cs, sms, st);
  return launch_cfg<1, 32, 8, PH>(a, warp_mode, w, cs, sms, st);
}

// cols: rows of X the launch gathers from (the whole column space, or one owner block of a
// phased aggregation, whose footprint is 1/G of it)
// K slices of a vec4 SpMM over `cols` gathered rows (the automatic rule of spmm_slice_width)
int64_t spmm_slices(double avg_deg, double cols, int64_t K, int64_t l2_bytes) {
  int64_t kw = std::min<int64_t>(K, 1024);
  const double per_col = cols * 4.0;
  if (avg_deg >= 32.0 && per_col * (double)K > 0.6 * (double)l2_bytes) {
    const int64_t fit = (int64_t)(0.55 * (double)l2_bytes / per_col) / 64 * 64;
    if (fit >= 64) kw = std::min(kw, round_up(ceil_div(K, ceil_div(K, fit)), 64));
  }
  return ceil_div(K, std::max<int64_t>(kw, 1));
}

// Dynamic normalisation (Eq. 2): the pre-scale D̃^-½ of the aggregated operand is fused into the
// SpMM gather (one dependent 4-byte gather -- a whole L2 sector -- per entry and K slice) unless
// a separate row-broadcast pass (read + write N x K floats once) moves fewer bytes: dense graphs
// whose SpMM is K-sliced (Reddit 602 -> 1024: 10 slices x 118 M entries x 32 B vs 1.1 GB)
bool dyn_prescale(double nnz, double rows, double avg_deg, double cols, int64_t K, int64_t l2_bytes) {
  return nnz * 32.0 * (double)spmm_slices(avg_deg, cols, K, l2_bytes) > rows * (double)K * 8.0;
}

int64_t spmm_slice_width(const granii_graph_s* g, int64_t K, bool vec4, int64_t l2_bytes, int64_t cols) {
  // Keep the gathered column slice of X resident in L2: split
  // K into slices whose X footprint is <= ~45% of L2 when the graph is dense
  // enough for re-use (avg degree >= 32) and X itself does not fit.
  const int64_t maxw = vec4 ? 1024 : 256;
  int64_t kw = std::min<int64_t>(K, maxw);
  if (const char* env = getenv("GRANII_SPMM_SLICE")) {
    int64_t v = atoll(env);
    if (v > 0) return std::min<int64_t>(std::max<int64_t>(v, 1), maxw);
  }
  const double per_col = (double)cols * 4.0;
  if (g->avg_deg() >= 32.f && per_col * (double)K > 0.6 * (double)l2_bytes) {
    const int64_t unit = vec4 ? 64 : 32;
    const int64_t fit = (int64_t)(0.55 * (double)l2_bytes / per_col) / unit * unit;  // columns resident in L2
    if (fit >= unit) {  // otherwise a slice cannot stay resident: do not re-read col_idx for nothing
      const int64_t nsl = ceil_div(K, fit);
      kw = std::min(kw, round_up(ceil_div(K, nsl), unit));
    }
  }
  return kw;
}

granii_status launch_spmm(const granii_graph_s* g, const float* vals, const float* X, int64_t ldx, int64_t K,
                          float* Y, int64_t ldy, const float* rs, const float* cs, bool relu, cudaStream_t st) {
  return launch_spmm_ex(g, vals, X, ldx, K, Y, ldy, rs, cs, relu, nullptr, 0, 0.f, st);
}

static granii_status spmm_impl(const granii_graph_s* g, const float* vals, const float* X, int64_t ldx, int64_t K,
                               float* Y, int64_t ldy, const float* rs, const float* cs, bool relu, const float* B,
                               int64_t ldb, float beta, const SpmmPhase* ph, cudaStream_t st,
                               const float* att_el = nullptr) {
  if (g->n_rows == 0 || K == 0) return GRANII_OK;
  DevInfo di;
  GR_TRY(dev_info(&di));
  const bool vec4 = (ldx % 4 == 0) && (ldy % 4 == 0) && ((uintptr_t)X % 16 == 0) && ((uintptr_t)Y % 16 == 0) &&
                    (!B || ((ldb % 4 == 0) && ((uintptr_t)B % 16 == 0)));
  // a phase sees (p1 - p0 - [skip]) / G of every row on average
  const float share = ph ? float(ph->p1 - ph->p0 - (ph->skip >= 0 ? 1 : 0)) / float(g->world) : 1.f;
  const bool warp_mode = g->avg_deg() * share >= 16.f;
  SpmmArgs a{g->n_rows - g->n_heavy, g->row_ptr, g->col_idx, vals, X, ldx, 0, 0, Y, ldy, rs, cs, relu ? 1 : 0,
             g->order + g->n_heavy, g->ord_rp + g->n_heavy, std::max<int64_t>(0, g->n_wide - g->n_heavy), g->n_seg,
             g->seg_lo, g->seg_hi,
             nullptr, 0, B, ldb, beta};
  a.l2hint = l2hint_enabled();
  // phases slice like the whole aggregation: the 64-wide slices also keep the L1 hit rate
  const int64_t kw = spmm_slice_width(g, K, vec4, di.l2_bytes, g->n_cols);
  float* partial = nullptr;  // heavy-segment partials: this slice's columns start at partial + pk0
  bool own_partial = false;
  float2* seg_ms = nullptr;  // fused attention: (max, sum) of every heavy segment
  if (att_el) {
    if (ph || !warp_mode || !vec4 || vals || B)
      return fail(GRANII_ERR_UNSUPPORTED, "fused attention SpMM: warp-per-row, aligned, unphased only");
    a.el = att_el;
    a.seg_row = g->seg_row;  // el of a heavy segment's row
    if (g->n_seg > 0) GR_CUDA(cudaMallocAsync((void**)&seg_ms, (size_t)g->n_seg * sizeof(float2), st));
    a.seg_ms = seg_ms;
  }
  if (ph) {
    a.owner_off = g->owner_off;
    a.ord_off = g->ord_off + g->n_heavy * (g->world + 1);
    a.seg_row = g->seg_row;
    a.G1 = g->world + 1;
    a.p0 = ph->p0;
    a.p1 = ph->p1;
    a.skip = ph->skip;
    a.first = ph->first;
    a.last = ph->last;
    a.ldp = round_up(K, 4);  // kept across the phases for every slice
    partial = ph->partial;
  } else if (g->n_seg > 0) {  // stream-ordered scratch for the heavy-row partials (pool-backed, no sync)
    a.ldp = round_up(kw, 4);
    GR_CUDA(cudaMallocAsync((void**)&partial, (size_t)g->n_seg * a.ldp * sizeof(float), st));
    own_partial = true;
  }
  const bool combine = g->n_seg > 0 && (!ph || ph->last);
  // algorithmic bytes: per entry col id (+w, +cs) + one K-row of X;
  // per row row_ptr + the K-row of Y (+rs)
  const double nnz = (double)g->local_nnz, R = (double)g->n_rows;
  const double bytes = nnz * (4.0 + (vals ? 4.0 : 0.0) + (cs ? 4.0 : 0.0) + 4.0 * K) +
                       R * (8.0 + 4.0 * K + (rs ? 4.0 : 0.0) + (B ? 4.0 * K : 0.0) + (att_el ? 4.0 : 0.0));
  // compulsory bytes: the same streams, with X read once (its rows, not its gathers)
  const double compulsory = bytes - nnz * 4.0 * K + (double)g->n_cols * 4.0 * K;
  // the gathered slice stays in L2 (spmm_slice_width keeps it <= ~55 % of L2)
  const bool l2_res = (double)g->n_cols * 4.0 * (double)kw <= 0.6 * (double)di.l2_bytes;
  // a phased aggregation books its algorithmic bytes once (in its last phase)
  const bool book = !ph || ph->last;
  ProfScope ps("spmm", st, book ? bytes : 0.0, book ? 2.0 * nnz * K : 0.0, (int)ceil_div(K, kw),
               book ? compulsory : 0.0, l2_res);
  for (int64_t k0 = 0; k0 < K; k0 += kw) {
    a.k0 = k0;
    a.kw = std::min(kw, K - k0);
    a.partial = partial ? partial + (ph ? k0 : 0) : nullptr;
    // slices of a vec4 launch must stay 16-byte aligned
    const bool v4 = vec4 && (k0 % 4 == 0);
    if (ph) GR_TRY(launch_slice<true>(a, v4, warp_mode, vals != nullptr, cs != nullptr, di.sms, st));
    else GR_TRY(launch_slice<false>(a, v4, warp_mode, vals != nullptr, cs != nullptr, di.sms, st));
    if (combine && att_el) {
      const int64_t tot = g->n_heavy * a.kw;
      k_spmm_combine_att<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(tot, 256), 4096)), 256, 0, st>>>(
          g->n_heavy, g->order, g->seg_ptr, a.partial, a.ldp, seg_ms, a.k0, a.kw, Y, ldy, rs, relu ? 1 : 0);
      GR_CHECK_LAUNCH();
      ps.add_launches(1);
    } else if (combine) {
      const int64_t tot = g->n_heavy * a.kw;
      k_spmm_combine<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(tot, 256), 4096)), 256, 0, st>>>(
          g->n_heavy, g->order, g->seg_ptr, a.partial, a.ldp, a.k0, a.kw, Y, ldy, rs, relu ? 1 : 0, B, ldb, beta);
      GR_CHECK_LAUNCH();
      ps.add_launches(1);
    }
  }
  if (own_partial) GR_CUDA(cudaFreeAsync(partial, st));
  if (seg_ms) GR_CUDA(cudaFreeAsync(seg_ms, st));
  return GRANII_OK;
}

granii_status launch_spmm_ex(const granii_graph_s* g, const float* vals, const float* X, int64_t ldx, int64_t K,
                             float* Y, int64_t ldy, const float* rs, const float* cs, bool relu, const float* B,
                             int64_t ldb, float beta, cudaStream_t st) {
  return spmm_impl(g, vals, X, ldx, K, Y, ldy, rs, cs, relu, B, ldb, beta, nullptr, st);
}

bool spmm_att_supported(const granii_graph_s* g) { return g->avg_deg() >= 16.f; }

int l2hint_enabled() {
  const char* e = getenv("GRANII_L2HINT");
  return e && e[0] == '0' ? 0 : 1;
}

granii_status launch_spmm_att(const granii_graph_s* g, const float* el, const float* er, const float* X, int64_t ldx,
                              int64_t K, float* Y, int64_t ldy, const float* rs, bool relu, cudaStream_t st) {
  return spmm_impl(g, nullptr, X, ldx, K, Y, ldy, rs, er, relu, nullptr, 0, 0.f, nullptr, st, el);
}

granii_status launch_spmm_phase(const granii_graph_s* g, const float* vals, const float* X, int64_t ldx, int64_t K,
                                float* Y, int64_t ldy, const float* rs, const float* cs, bool relu, const float* B,
                                int64_t ldb, float beta, const SpmmPhase& ph, cudaStream_t st) {
  if (!g->owner_off) return fail(GRANII_ERR_INVALID_ARG, "phased SpMM needs a partitioned graph");
  return spmm_impl(g, vals, X, ldx, K, Y, ldy, rs, cs, relu, B, ldb, beta, &ph, st);
}

}  // namespace granii
