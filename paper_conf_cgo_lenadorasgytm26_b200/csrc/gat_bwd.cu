// gat_bwd.cu -- GAT backward (training, reading R22).
//
// The paper trains GAT (Table III "T", L324) but gives no backward; this is the
// chain rule of Eq. 4-6.  With z_ij = el_i + er_j, α = row softmax of
// LeakyReLU(z), dY = dout ⊙ σ'(Y) and (dX, Z) = (dY, Θ) for REUSE or
// (dT = dY Wᵀ, H) for RECOMP (each composition reverses its own forward):
//   dα_ij = <dX_i, Z_j>                          (K-wide SDDMM)
//   c_i   = Σ_j α_ij dα_ij = <dY_i, Y_i>         (row-local: Σ_j α_ij Z_j W.. = Y_i)
//   dz_ij = α_ij (dα_ij - c_i) · (z_ij > 0 ? 1 : 0.2)
//   del_i = Σ_j dz_ij        der_j = Σ_i dz_ij
//   out_j = Σ_i α_ij dX_i + del_j u + der_j v    (REUSE: dΘ with u,v = a_l,a_r;
//                                                 RECOMP: dH with u,v = W a_l, W a_r)
// B200 design: two warp-per-row passes in the degree-descending schedule,
// both gathers of K-wide rows (the SpMM's access pattern):
//   pass A (rows i): one sweep of K-wide gathers of Z_j for dα with an online
//     softmax (running max, Σ exp, Σ exp·(dα - c)·LeakyReLU'); writes del_i and the
//     row record {el_i, m_i, 1/s_i, c_i} into the tail of dX's row i (columns
//     [rec, rec+4), rec = K rounded to 4), so pass B's K-wide gather of dX_i
//     brings the record along (and the all-gather of dX carries it to other GPUs).
//   pass B (rows j, symmetric Ã: row j lists every i with j in N(i)): gathers
//     dX_i with its record, recomputes α_ij from it (α is never stored),
//     dots dX_i with the register-resident Z_j, accumulates the transposed
//     SpMM and der_j, and applies the rank-2 epilogue.
// Lane groups of LPG lanes own one edge at a time (LPG = K/4 up to 32), NJ
// float4 per lane cover K.  No atomics: every output is written once, in a
// fixed reduction order (bitwise reproducible).
#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>

#include "cache.cuh"
#include "internal.h"

namespace granii {

__device__ __forceinline__ float gb_warp_sum(float v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// this lane's NJ float4 slices of a K-wide row; columns >= K read as 0
// (p is 16-byte aligned with a row stride that is a multiple of 4 floats)
// (K <= 2048: the masks are 32-bit compares -- as int64 they cost a carry chain per element inside
// the gather loop, ~40 % of pass A's instructions at K = 47)
template <int LPG, int NJ>
__device__ __forceinline__ void gb_load_row(const float* __restrict__ p, int lg, int64_t K64, float (&v)[NJ][4]) {
  const int K = (int)K64;
#pragma unroll
  for (int j = 0; j < NJ; ++j) {
    const int col = 4 * (lg + j * LPG);
    if (col < K) {
      const float4 t = __ldg(reinterpret_cast<const float4*>(p + col));
      const int nv = K - col;  // valid elements of this vector (>= 4: all)
      v[j][0] = t.x;
      v[j][1] = nv > 1 ? t.y : 0.f;
      v[j][2] = nv > 2 ? t.z : 0.f;
      v[j][3] = nv > 3 ? t.w : 0.f;
    } else {
      v[j][0] = v[j][1] = v[j][2] = v[j][3] = 0.f;
    }
  }
}

// row r of a row-major operand: row ids are non-negative int32 and strides < 2^32 floats, so one
// 32 x 32 -> 64-bit multiply (IMAD.WIDE.U32) gives the exact offset
__device__ __forceinline__ const float* gb_row(const float* base, int32_t r, int64_t ld) {
  return base + (uint64_t)(uint32_t)r * (uint32_t)ld;
}

// K % 4 == 0: the gathered K-wide row without per-element masks -- lanes past the row re-read
// its last vector (finite data that only ever meets the zeros of the masked register-resident row,
// or feeds columns that are never stored)
template <int LPG, int NJ>
__device__ __forceinline__ void gb_load_row_cl(const float* __restrict__ p, int lg, int64_t K64, float (&v)[NJ][4]) {
  const int K = (int)K64;
#pragma unroll
  for (int j = 0; j < NJ; ++j) {
    const int col = 4 * (lg + j * LPG);
    const float4 t = __ldg(reinterpret_cast<const float4*>(p + (col < K ? col : K - 4)));
    v[j][0] = t.x;
    v[j][1] = t.y;
    v[j][2] = t.z;
    v[j][3] = t.w;
  }
}

template <int LPG, int NJ, bool CL>
__device__ __forceinline__ void gb_gather_row(const float* __restrict__ p, int lg, int64_t K, float (&v)[NJ][4]) {
  if constexpr (CL) gb_load_row_cl<LPG, NJ>(p, lg, K, v);
  else gb_load_row<LPG, NJ>(p, lg, K, v);
}

// this lane's share of <x, y>; never reduced per entry: every use is linear in the dot, so
// the lane shares are accumulated and reduced once per row
template <int NJ>
__device__ __forceinline__ float gb_pdot(const float (&x)[NJ][4], const float (&y)[NJ][4]) {
  float d = 0.f;
#pragma unroll
  for (int j = 0; j < NJ; ++j)
#pragma unroll
    for (int k = 0; k < 4; ++k) d = fmaf(x[j][k], y[j][k], d);
  return d;
}

// this lane's share of <x, z - p>: the difference is taken element by element before the dot, so
// dα_ij - c_i = <dX_i, Z_j - P_i> (P_i = Y_i or T_i, c_i = <dX_i, P_i>) keeps its accuracy when Z_j ≈ P_i
// -- the near-one-hot rows, where dα_ij and c_i agree to many digits and their fp32 difference would
// be rounding noise (measured: da_l of the products-shaped training step 3.2e-4 -> see DESIGN R22)
template <int NJ>
__device__ __forceinline__ float gb_pdot_diff(const float (&x)[NJ][4], const float (&z)[NJ][4],
                                              const float (&p)[NJ][4]) {
  float d = 0.f;
#pragma unroll
  for (int j = 0; j < NJ; ++j)
#pragma unroll
    for (int k = 0; k < 4; ++k) d = fmaf(x[j][k], z[j][k] - p[j][k], d);
  return d;
}

__device__ __forceinline__ float gb_lrelu(float z) { return z > 0.f ? z : 0.2f * z; }

// dY = dout ⊙ σ'(out) and c_r = <dY_r, out_r> (= <dY_r, Y_r>: where ReLU clips, dY = 0). Lane groups of
// L = 2^lg lanes own a row (L = the smallest power of two >= the row's vector count, at most 32), with
// 16-byte accesses when every row start is aligned (V = 4); the row loop is warp-uniform so the group's
// shuffle reduction never diverges.
template <int V>
__global__ void __launch_bounds__(256) k_gat_prep(int64_t R, int K, int Kv, int lg, const float* __restrict__ out,
                                                  int64_t ldo, const float* __restrict__ g, int64_t ldg, int relu,
                                                  float* __restrict__ dY, int64_t ldd, float* __restrict__ c) {
  const int L = 1 << lg, lane = threadIdx.x & 31, lig = lane & (L - 1);
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int rpw = 32 >> lg;  // rows per warp
  for (int64_t rb = warp * rpw; rb < R; rb += nw * rpw) {
    const int64_t r = rb + (lane >> lg);
    float s = 0.f;
    if (r < R) {
#pragma unroll 2
      for (int k = lig; k < Kv; k += L) {
        float o[V], d[V];
        if (V > 1 && k * V + V > K) {  // ragged tail of a row whose start is aligned: element by element
          for (int c = k * V; c < K; ++c) {
            const float oc = out[r * ldo + c];
            const float dc = (!relu || oc > 0.f) ? g[r * ldg + c] : 0.f;
            dY[r * ldd + c] = dc;
            s = fmaf(dc, oc, s);
          }
          continue;
        }
        if constexpr (V == 4) {
          const float4 o4 = *reinterpret_cast<const float4*>(out + r * ldo + (int64_t)k * 4);
          const float4 g4 = *reinterpret_cast<const float4*>(g + r * ldg + (int64_t)k * 4);
          o[0] = o4.x, o[1] = o4.y, o[2] = o4.z, o[3] = o4.w;
          d[0] = g4.x, d[1] = g4.y, d[2] = g4.z, d[3] = g4.w;
        } else {
          o[0] = out[r * ldo + k];
          d[0] = g[r * ldg + k];
        }
#pragma unroll
        for (int i = 0; i < V; ++i) {
          if (relu && !(o[i] > 0.f)) d[i] = 0.f;  // ReLU'(0) = 0
          s = fmaf(d[i], o[i], s);
        }
        if constexpr (V == 4) *reinterpret_cast<float4*>(dY + r * ldd + (int64_t)k * 4) = make_float4(d[0], d[1], d[2], d[3]);
        else dY[r * ldd + k] = d[0];
      }
    }
    for (int off = L >> 1; off; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
    if (r < R && lig == 0) c[r] = s;
  }
}

// Entries are consumed in chunks of 32: lane l loads the chunk's l-th column id and its
// per-column scalars with one coalesced load (the next chunk is prefetched while this one is
// processed), then lane groups take entries from the chunk by shuffles, U per group in flight,
// so only the K-wide row gathers sit on the critical path.
// Every entry contributes w·s'·<dX_i, Z_j - P_i> = w·s'·(dα_ij - c_i) to D (gb_pdot_diff), so
// del = D / S with no D - c·Cw cancellation at the end (Cw is left 0).  WT (the der-only path,
// a.tout): each entry's dα_ij - c_i is also reduced over its lane group and written in Ã's order.
template <int LPG, int NJ, int U, bool CL = false, bool WT = false>
__device__ __forceinline__ void gat_a_warp_row(const GatBwdArgs& a, int32_t r, int lane, int64_t seg = -1) {
  constexpr int G = 32 / LPG;
  static_assert(G * U <= 32, "one step must fit in a chunk");
  const int lg = lane % LPG, grp = lane / LPG;
  // a whole row, or (seg >= 0) one hub segment of it, whose online-softmax state goes to seg_a
  const int64_t b = seg >= 0 ? a.seg_lo[seg] : a.row_ptr[r], t = seg >= 0 ? a.seg_hi[seg] : a.row_ptr[r + 1];
  const float eli = a.el[r];
  const float ci = a.c[r];
  float xv[NJ][4], pv[NJ][4];
  gb_load_row<LPG, NJ>(a.dX + (int64_t)r * a.ldx, lg, a.K, xv);
  gb_load_row<LPG, NJ>(a.P + (int64_t)r * a.ldpp, lg, a.K, pv);
  // One sweep with an online softmax whose scalar work is done once per entry, by the lane that
  // loaded the entry's column (chunk of 32): its er (gathered a chunk ahead), score, slope s'; the
  // chunk's max over the warp (one rescale per chunk when it grows, warp-uniform m), then
  // w = exp(e - m).  The owner lane keeps S = Σ w and Cw = Σ w·s'; the lane groups that gather the
  // K-wide rows get w·s' by shuffle and keep D = Σ w·s'·(their share of dα).  Everything is
  // reduced once per row: del = (Σ D - c·Σ Cw) / Σ S.
  float m = -INFINITY, S = 0.f, Cw = 0.f, D = 0.f;
  int32_t c0 = 0, c1 = 0;
  float e0 = 0.f;
  if (b < t) {
    c0 = __ldg(a.col_idx + (b + lane < t ? b + lane : t - 1));
    e0 = __ldg(a.er + c0);
    if (b + 32 < t) c1 = __ldg(a.col_idx + (b + 32 + lane < t ? b + 32 + lane : t - 1));
  }
  for (int64_t base = b; base < t; base += 32) {
    const int32_t cc = c0;
    const float erc = e0;
    if (base + 32 < t) {  // distance-2 prefetch of the columns, distance 1 of their er
      c0 = c1;
      e0 = __ldg(a.er + c0);
      if (base + 64 < t) c1 = __ldg(a.col_idx + (base + 64 + lane < t ? base + 64 + lane : t - 1));
    }
    const int cnt = (int)(t - base < 32 ? t - base : 32);
    const float z = eli + erc;
    const float ev = lane < cnt ? gb_lrelu(z) : -INFINITY;
    float cm = ev;
#pragma unroll
    for (int o = 16; o; o >>= 1) cm = fmaxf(cm, __shfl_xor_sync(0xffffffffu, cm, o));
    if (cm > m) {  // warp-uniform
      const float f = __expf(m - cm);  // 0 on the first chunk (m = -inf)
      S *= f;
      Cw *= f;
      D *= f;
      m = cm;
    }
    const float w = lane < cnt ? __expf(ev - m) : 0.f;
    const float ws = w * (z > 0.f ? 1.f : 0.2f);
    S += w;
    Cw += ws;
    const int steps = (cnt + G * U - 1) / (G * U);  // warp-uniform
    for (int q = 0; q < steps; ++q) {
      int32_t j[U];
      float wu[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        j[u] = __shfl_sync(0xffffffffu, cc, q * G * U + u * G + grp);
        wu[u] = __shfl_sync(0xffffffffu, ws, q * G * U + u * G + grp);  // 0 past the chunk's end
      }
      float zv[U][NJ][4];
#pragma unroll
      for (int u = 0; u < U; ++u) gb_gather_row<LPG, NJ, CL>(gb_row(a.Z, j[u], a.ldz), lg, a.K, zv[u]);
      if constexpr (WT) {
#pragma unroll
        for (int u = 0; u < U; ++u) {
          float pd = gb_pdot_diff<NJ>(xv, zv[u], pv);
          D = fmaf(wu[u], pd, D);
#pragma unroll
          for (int o = LPG / 2; o; o >>= 1) pd += __shfl_xor_sync(0xffffffffu, pd, o);
          const int slot = q * G * U + u * G + grp;
          if (lg == 0 && slot < cnt) a.tout[base + slot] = pd;
        }
      } else {
#pragma unroll
        for (int u = 0; u < U; ++u) D = fmaf(wu[u], gb_pdot_diff<NJ>(xv, zv[u], pv), D);
      }
    }
  }
  Cw = 0.f;  // D already holds Σ w s' (dα - c): del = D / S
  S = gb_warp_sum(S);
  Cw = gb_warp_sum(Cw);
  D = gb_warp_sum(D);
  if (seg >= 0) {
    if (lane == 0) a.seg_a[seg] = make_float4(m, S, Cw, D);
    return;
  }
  const float inv_s = S > 0.f ? 1.f / S : 0.f;
  if (lane == 0) {
    a.del[r] = (D - ci * Cw) * inv_s;
    *reinterpret_cast<float4*>(a.dXw + (int64_t)r * a.ldx + a.rec) = make_float4(eli, m, inv_s, ci);
    if (WT) a.recs[r] = make_float4(eli, m, inv_s, ci);
  }
}

template <int LPG, int NJ, int U, bool CL = false>
__device__ __forceinline__ void gat_b_warp_row(const GatBwdArgs& a, int32_t r, int lane, int64_t seg = -1) {
  constexpr int G = 32 / LPG;
  static_assert(G * U <= 32, "one step must fit in a chunk");
  const int lg = lane % LPG, grp = lane / LPG;
  // a whole row, or (seg >= 0) one hub segment of it, whose partial sums go to seg_b / seg_der
  const int64_t b = seg >= 0 ? a.seg_lo[seg] : a.row_ptr[r], t = seg >= 0 ? a.seg_hi[seg] : a.row_ptr[r + 1];
  const float erj = a.er[r];
  float zr[NJ][4], acc[NJ][4];
  gb_load_row<LPG, NJ>(a.Z + (int64_t)r * a.ldz, lg, a.K, zr);
#pragma unroll
  for (int j = 0; j < NJ; ++j)
#pragma unroll
    for (int k = 0; k < 4; ++k) acc[j][k] = 0.f;
  // der = Σ_lanes Σ α s' (lane share of dα) - Σ α s' c_i, reduced once per row.  The per-entry
  // scalars are computed once, by the lane that loaded the entry's column: its record (gathered a
  // chunk ahead), α and α·s'; the lane groups that gather the K-wide rows get them by shuffle, and
  // the owner lane accumulates the α·s'·c_i correction itself.
  float dpart = 0.f, dcorr = 0.f;
  int32_t c0 = 0, c1 = 0;
  float4 r0 = make_float4(0.f, 0.f, 0.f, 0.f);
  if (b < t) {
    c0 = __ldg(a.col_idx + (b + lane < t ? b + lane : t - 1));
    r0 = __ldg(reinterpret_cast<const float4*>(gb_row(a.dX, c0, a.ldx) + a.rec));
    if (b + 32 < t) c1 = __ldg(a.col_idx + (b + 32 + lane < t ? b + 32 + lane : t - 1));
  }
  for (int64_t base = b; base < t; base += 32) {
    const int32_t cc = c0;
    const float4 rc = r0;
    if (base + 32 < t) {  // distance-2 prefetch of the columns, distance 1 of their records
      c0 = c1;
      r0 = __ldg(reinterpret_cast<const float4*>(gb_row(a.dX, c0, a.ldx) + a.rec));
      if (base + 64 < t) c1 = __ldg(a.col_idx + (base + 64 + lane < t ? base + 64 + lane : t - 1));
    }
    const int cnt = (int)(t - base < 32 ? t - base : 32);
    const float z = rc.x + erj;
    const float al = lane < cnt ? __expf(gb_lrelu(z) - rc.y) * rc.z : 0.f;
    const float as = al * (z > 0.f ? 1.f : 0.2f);
    dcorr = fmaf(as, rc.w, dcorr);
    const int steps = (cnt + G * U - 1) / (G * U);  // warp-uniform
    for (int q = 0; q < steps; ++q) {
      int32_t i[U];
      float au[U], su[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int src = q * G * U + u * G + grp;
        i[u] = __shfl_sync(0xffffffffu, cc, src);
        au[u] = __shfl_sync(0xffffffffu, al, src);  // 0 past the chunk's end
        su[u] = __shfl_sync(0xffffffffu, as, src);
      }
      float xv[U][NJ][4];
#pragma unroll
      for (int u = 0; u < U; ++u) gb_gather_row<LPG, NJ, CL>(gb_row(a.dX, i[u], a.ldx), lg, a.K, xv[u]);
#pragma unroll
      for (int u = 0; u < U; ++u) {
        dpart = fmaf(su[u], gb_pdot<NJ>(xv[u], zr), dpart);
#pragma unroll
        for (int j = 0; j < NJ; ++j)
#pragma unroll
          for (int k = 0; k < 4; ++k) acc[j][k] = fmaf(au[u], xv[u][j][k], acc[j][k]);
      }
    }
  }
#pragma unroll
  for (int o = LPG; o < 32; o <<= 1)
#pragma unroll
    for (int j = 0; j < NJ; ++j)
#pragma unroll
      for (int k = 0; k < 4; ++k) acc[j][k] += __shfl_xor_sync(0xffffffffu, acc[j][k], o);
  const float der = gb_warp_sum(dpart) - gb_warp_sum(dcorr);
  if (seg >= 0) {
    if (grp == 0) {
      float* o = a.seg_b + seg * a.ldp;
#pragma unroll
      for (int j = 0; j < NJ; ++j) {
        const int64_t col = 4 * (int64_t)(lg + j * LPG);
        if (col < a.K) *reinterpret_cast<float4*>(o + col) = make_float4(acc[j][0], acc[j][1], acc[j][2], acc[j][3]);
      }
    }
    if (lane == 0) a.seg_der[seg] = der;
    return;
  }
  const float delj = a.del_in[r];
  if (grp == 0) {
    float* o = a.out + (int64_t)r * a.ldo;
#pragma unroll
    for (int j = 0; j < NJ; ++j) {
      const int64_t col = 4 * (int64_t)(lg + j * LPG);
      if (col >= a.K) continue;
      float v[4];
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const int64_t cc = col + k < a.K ? col + k : col;  // clamped read; the value is not stored
        v[k] = acc[j][k] + delj * __ldg(a.u + cc) + der * __ldg(a.v + cc);
      }
      if (a.vec_store && col + 3 < a.K) {
        *reinterpret_cast<float4*>(o + col) = make_float4(v[0], v[1], v[2], v[3]);
      } else {
#pragma unroll
        for (int k = 0; k < 4; ++k)
          if (col + k < a.K) o[col + k] = v[k];
      }
    }
  }
  if (lane == 0) a.der[r] = der;
}

// ---------------------------------------------------------------- sparse graphs: group per row
// avg degree < 16 (the SpMM's group-per-row regime): an LPG-lane group owns a row, 32/LPG rows
// per warp, U entries per group in flight; no shuffles inside the (divergent) entry loops, the
// lane shares are reduced within the group at the end.
template <int LPG, int NJ, int U, bool WT = false>
__device__ __forceinline__ void gat_a_group_row(const GatBwdArgs& a, int64_t t0, int lane) {
  const int lg = lane % LPG;
  // the group's lanes run the same (divergent across groups) entry loop: WT's per-entry reduction
  // shuffles within the group only
  const unsigned gmask = LPG == 32 ? 0xffffffffu : (((1u << LPG) - 1u) << (lane & ~(LPG - 1)));
  const bool live = t0 < a.n_rows;
  const int32_t r = live ? a.order[t0] : 0;
  const int64_t b = live ? a.row_ptr[r] : 0, t = live ? a.row_ptr[r + 1] : 0;
  const float eli = live ? a.el[r] : 0.f, ci = live ? a.c[r] : 0.f;
  float xv[NJ][4], pv[NJ][4];
  gb_load_row<LPG, NJ>(a.dX + (int64_t)r * a.ldx, lg, live ? a.K : 0, xv);
  gb_load_row<LPG, NJ>(a.P + (int64_t)r * a.ldpp, lg, live ? a.K : 0, pv);
  float m = -INFINITY, S = 0.f, Cw = 0.f, D = 0.f;
  for (int64_t e = b; e < t; e += U) {
    int32_t j[U];
    float erj[U];
    float zv[U][NJ][4];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      j[u] = __ldg(a.col_idx + (e + u < t ? e + u : t - 1));
      erj[u] = __ldg(a.er + j[u]);
      gb_load_row<LPG, NJ>(gb_row(a.Z, j[u], a.ldz), lg, a.K, zv[u]);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (e + u < t) {
        float pd = gb_pdot_diff<NJ>(xv, zv[u], pv);  // this lane's share of dα - c_i
        if constexpr (WT) {
          float pf = pd;
#pragma unroll
          for (int o = LPG / 2; o; o >>= 1) pf += __shfl_xor_sync(gmask, pf, o);
          if (lg == 0) a.tout[e + u] = pf;
        }
        const float z = eli + erj[u];
        const float ev = gb_lrelu(z);
        const float sl = z > 0.f ? 1.f : 0.2f;
        if (ev > m) {
          const float sc = __expf(m - ev);
          S = fmaf(S, sc, 1.f);
          Cw = fmaf(Cw, sc, sl);
          D = fmaf(D, sc, sl * pd);
          m = ev;
        } else {
          const float w = __expf(ev - m);
          S += w;
          Cw = fmaf(w, sl, Cw);
          D = fmaf(w * sl, pd, D);
        }
      }
    }
  }
#pragma unroll
  for (int o = LPG / 2; o; o >>= 1) D += __shfl_xor_sync(0xffffffffu, D, o);
  Cw = 0.f;  // D already holds Σ w s' (dα - c): del = D / S
  const float inv_s = S > 0.f ? 1.f / S : 0.f;
  if (live && lg == 0) {
    a.del[r] = (D - ci * Cw) * inv_s;
    *reinterpret_cast<float4*>(a.dXw + (int64_t)r * a.ldx + a.rec) = make_float4(eli, m, inv_s, ci);
    if (WT) a.recs[r] = make_float4(eli, m, inv_s, ci);
  }
}

template <int LPG, int NJ, int U>
__device__ __forceinline__ void gat_b_group_row(const GatBwdArgs& a, int64_t t0, int lane) {
  const int lg = lane % LPG;
  const bool live = t0 < a.n_rows;
  const int32_t r = live ? a.order[t0] : 0;
  const int64_t b = live ? a.row_ptr[r] : 0, t = live ? a.row_ptr[r + 1] : 0;
  const float erj = live ? a.er[r] : 0.f;
  float zr[NJ][4], acc[NJ][4];
  gb_load_row<LPG, NJ>(a.Z + (int64_t)r * a.ldz, lg, live ? a.K : 0, zr);
#pragma unroll
  for (int j = 0; j < NJ; ++j)
#pragma unroll
    for (int k = 0; k < 4; ++k) acc[j][k] = 0.f;
  float dpart = 0.f, dcorr = 0.f;
  for (int64_t e = b; e < t; e += U) {
    int32_t i[U];
    float4 st[U];
    float xv[U][NJ][4];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      i[u] = __ldg(a.col_idx + (e + u < t ? e + u : t - 1));
      st[u] = __ldg(reinterpret_cast<const float4*>(gb_row(a.dX, i[u], a.ldx) + a.rec));
      gb_load_row<LPG, NJ>(gb_row(a.dX, i[u], a.ldx), lg, a.K, xv[u]);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const float z = st[u].x + erj;
      const float alpha = (e + u < t) ? __expf(gb_lrelu(z) - st[u].y) * st[u].z : 0.f;
      const float as = alpha * (z > 0.f ? 1.f : 0.2f);
      dpart = fmaf(as, gb_pdot<NJ>(xv[u], zr), dpart);
      if (lg == 0) dcorr = fmaf(as, st[u].w, dcorr);
#pragma unroll
      for (int j = 0; j < NJ; ++j)
#pragma unroll
        for (int k = 0; k < 4; ++k) acc[j][k] = fmaf(alpha, xv[u][j][k], acc[j][k]);
    }
  }
#pragma unroll
  for (int o = LPG / 2; o; o >>= 1) {
    dpart += __shfl_xor_sync(0xffffffffu, dpart, o);
    dcorr += __shfl_xor_sync(0xffffffffu, dcorr, o);
  }
  if (!live) return;
  const float der = dpart - dcorr;
  const float delj = a.del_in[r];
  float* o = a.out + (int64_t)r * a.ldo;
#pragma unroll
  for (int j = 0; j < NJ; ++j) {
    const int64_t col = 4 * (int64_t)(lg + j * LPG);
    if (col >= a.K) continue;
    float v[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int64_t cc = col + k < a.K ? col + k : col;
      v[k] = acc[j][k] + delj * __ldg(a.u + cc) + der * __ldg(a.v + cc);
    }
    if (a.vec_store && col + 3 < a.K) {
      *reinterpret_cast<float4*>(o + col) = make_float4(v[0], v[1], v[2], v[3]);
    } else {
#pragma unroll
      for (int k = 0; k < 4; ++k)
        if (col + k < a.K) o[col + k] = v[k];
    }
  }
  if (lg == 0) a.der[r] = der;
}

// One launch covers both schedules: warps [0, n_wide) take the wide rows order[0 .. n_wide)
// (all rows of a dense graph), the remaining warps take G rows each, one per lane group.
template <int LPG, int NJ, int U, int MINB = 0, bool CL = false, bool WT = false>
__global__ void __launch_bounds__(256, MINB > 0 ? MINB : (NJ <= 2 ? 4 : (NJ <= 4 ? 3 : (NJ <= 8 ? 2 : 1))))
    k_gat_bwd_a(GatBwdArgs a) {
  constexpr int G = 32 / LPG;
  const int lane = threadIdx.x & 31;
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  // hub segments first (warp-wide items, largest rows first), then the wide rows (a warp each),
  // then lane groups; one call site per schedule keeps the unrolled body inlined once
  const int64_t wr = w - a.n_seg;
  if (wr >= a.n_wide) {
    gat_a_group_row<LPG, NJ, U, WT>(a, a.n_wide + (wr - a.n_wide) * G + lane / LPG, lane);
    return;
  }
  const bool sg = w < a.n_seg;
  gat_a_warp_row<LPG, NJ, U, CL, WT>(a, sg ? a.seg_row[w] : a.order[wr], lane, sg ? w : -1);
}

template <int LPG, int NJ, int U, int MINB = 0, bool CL = false>
__global__ void __launch_bounds__(256, MINB > 0 ? MINB : (NJ <= 2 ? 3 : (NJ <= 8 ? 2 : 1))) k_gat_bwd_b(GatBwdArgs a) {
  constexpr int G = 32 / LPG;
  const int lane = threadIdx.x & 31;
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  // hub segments first (warp-wide items, largest rows first), then the wide rows (a warp each),
  // then lane groups; one call site per schedule keeps the unrolled body inlined once
  const int64_t wr = w - a.n_seg;
  if (wr >= a.n_wide) {
    gat_b_group_row<LPG, NJ, U>(a, a.n_wide + (wr - a.n_wide) * G + lane / LPG, lane);
    return;
  }
  const bool sg = w < a.n_seg;
  gat_b_warp_row<LPG, NJ, U, CL>(a, sg ? a.seg_row[w] : a.order[wr], lane, sg ? w : -1);
}

// hub rows: merge the segments' online-softmax states in fixed order -> del and the row record
__global__ void k_gat_a_combine(GatBwdArgs a) {
  for (int64_t h = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; h < a.n_heavy; h += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = a.heavy_rows[h];
    float m = -INFINITY, S = 0.f, Cw = 0.f, D = 0.f;
    for (int32_t q = a.seg_ptr[h]; q < a.seg_ptr[h + 1]; ++q) {
      const float4 v = a.seg_a[q];
      const float mn = fmaxf(m, v.x);
      const float f1 = m == -INFINITY ? 0.f : __expf(m - mn), f2 = v.x == -INFINITY ? 0.f : __expf(v.x - mn);
      S = S * f1 + v.y * f2;
      Cw = Cw * f1 + v.z * f2;
      D = D * f1 + v.w * f2;
      m = mn;
    }
    const float ci = a.c[r], inv_s = S > 0.f ? 1.f / S : 0.f;
    a.del[r] = (D - ci * Cw) * inv_s;
    *reinterpret_cast<float4*>(a.dXw + (int64_t)r * a.ldx + a.rec) = make_float4(a.el[r], m, inv_s, ci);
    if (a.recs) a.recs[r] = make_float4(a.el[r], m, inv_s, ci);
  }
}

// hub rows: out_r = sum of the segments' partial rows (fixed order) + del_r u + der_r v
__global__ void k_gat_b_combine(GatBwdArgs a) {
  const int64_t total = a.n_heavy * a.K;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t h = i / a.K, k = i % a.K;
    const int32_t r = a.heavy_rows[h];
    float acc = 0.f, der = 0.f;
    for (int32_t q = a.seg_ptr[h]; q < a.seg_ptr[h + 1]; ++q) {
      acc += a.seg_b[(int64_t)q * a.ldp + k];
      der += a.seg_der[q];
    }
    a.out[(int64_t)r * a.ldo + k] = acc + a.del_in[r] * a.u[k] + der * a.v[k];
    if (k == 0) a.der[r] = der;
  }
}

// ---------------------------------------------------------------- der only (RECOMP input layer)
// der_j = Σ_{i: j ∈ N(i)} dz_ij, dz_ij = α_ij (dα_ij - c_i) s'_ij -- the column sums of dz, which an
// input layer needs instead of pass B's K-wide transposed SpMM (that only feeds dH).  Two passes of
// 4-byte accesses instead of K-wide gathers:
//   k_gat_dz  (rows i of Ã, natural order): dz_ij from pass A's per-entry dα - c_i (tv, Ã order), row
//             i's record {el_i, m_i, 1/s_i, c_i} and a gathered er_j (L2-resident vector), written to
//             the graph's column-blocked layout (g->tblk: region b = the entries whose column lies in
//             block b, rows ascending -- natural order writes each region front to back);
//   k_gat_der (rows j of Ãᵀ, natural order = block by block): der_j = Σ tvb[tperm[e']] over Ãᵀ's row
//             j -- 4-byte gathers, but only within the current block's region (~ L2 / 3), so each
//             32-byte sector comes from DRAM about once.
// Hub rows (degree > seg_len, when the graph has segments) are warp-wide segments taken first (dz:
// independent per entry; der: partial sums merged per row in fixed order).  Every sum in a fixed order
// (bitwise reproducible), no atomics.
struct GatDzArgs {
  int64_t n_rows;              // every row i (hubs skipped when segmented)
  const int64_t* row_ptr;
  int64_t seg_len;
  int64_t n_seg;
  const int64_t* seg_lo;
  const int64_t* seg_hi;
  const int32_t* seg_row;
  const int32_t* col;
  const float* er;
  const float4* recs;
  const float* tv;             // dα - c_i, Ã order
  const int32_t* tblk;
  float* tvb;                  // dz, column-blocked
  int l2hint;
};

template <int U>
__device__ __forceinline__ void gat_dz_run(const GatDzArgs& a, int32_t i, int64_t e, int64_t re, int step,
                                           const L2Pol& pol) {
  const float4 rc = __ldg(a.recs + i);  // {el_i, m_i, 1/s_i, c_i}
  for (; e < re; e += (int64_t)U * step) {
    int32_t j[U], q[U];
    float d[U], erj[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t ee = e + (int64_t)u * step < re ? e + (int64_t)u * step : re - 1;
      j[u] = ldg_stream(a.col + ee, pol.stream);
      d[u] = ldg_stream(a.tv + ee, pol.stream);
      q[u] = ldg_stream(a.tblk + ee, pol.stream);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) erj[u] = ldg_pol(a.er + j[u], pol.keep);
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (e + (int64_t)u * step < re) {
        const float z = rc.x + erj[u];
        const float al = __expf(gb_lrelu(z) - rc.y) * rc.z;
        st_pol(a.tvb + q[u], al * (z > 0.f ? 1.f : 0.2f) * d[u], pol.stream);
      }
    }
  }
}

template <int LPG, int U>
__global__ void __launch_bounds__(256) k_gat_dz(GatDzArgs a) {
  constexpr int G = 32 / LPG;
  const int lane = threadIdx.x & 31, grp = lane / LPG, lig = lane % LPG;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const L2Pol pol = make_l2pol(a.l2hint);
  for (int64_t t = warp; t < a.n_seg; t += nwarps)
    gat_dz_run<U>(a, a.seg_row[t], a.seg_lo[t] + lane, a.seg_hi[t], 32, pol);
  for (int64_t i0 = warp * G; i0 < a.n_rows; i0 += nwarps * G) {
    const int64_t i = i0 + grp;
    if (i >= a.n_rows) continue;
    const int64_t rs = a.row_ptr[i], re = a.row_ptr[i + 1];
    if (a.n_seg > 0 && re - rs > a.seg_len) continue;  // a hub: its segments were taken above
    gat_dz_run<U>(a, (int32_t)i, rs + lig, re, LPG, pol);
  }
}

struct GatDerArgs {
  int64_t n_rows;              // every row j of Ãᵀ, natural order (hubs skipped when segmented)
  const int64_t* row_ptr;
  int64_t seg_len;
  const int32_t* tperm;
  const float* tvb;            // dz, column-blocked
  float* der;
  int64_t n_seg;
  const int64_t* seg_lo;
  const int64_t* seg_hi;
  float* seg_der;
  int l2hint;
};

template <int U>
__device__ __forceinline__ float gat_dz_sum(const GatDerArgs& a, int64_t e, int64_t re, int step, const L2Pol& pol) {
  float acc = 0.f;
  for (; e < re; e += (int64_t)U * step) {
    int32_t p[U];
    float v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t ee = e + (int64_t)u * step < re ? e + (int64_t)u * step : re - 1;
      p[u] = ldg_stream(a.tperm + ee, pol.stream);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = ldg_pol(a.tvb + p[u], pol.keep);
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (e + (int64_t)u * step < re) acc += v[u];
  }
  return acc;
}

template <int LPG, int U>
__global__ void __launch_bounds__(256) k_gat_der(GatDerArgs a) {
  constexpr int G = 32 / LPG;
  const int lane = threadIdx.x & 31, grp = lane / LPG, lig = lane % LPG;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const L2Pol pol = make_l2pol(a.l2hint);
  for (int64_t t = warp; t < a.n_seg; t += nwarps) {
    const float acc = gb_warp_sum(gat_dz_sum<U>(a, a.seg_lo[t] + lane, a.seg_hi[t], 32, pol));
    if (lane == 0) a.seg_der[t] = acc;
  }
  for (int64_t j0 = warp * G; j0 < a.n_rows; j0 += nwarps * G) {
    const int64_t j = j0 + grp;
    int64_t rs = 0, re = 0;
    bool hub = false;
    if (j < a.n_rows) {
      rs = a.row_ptr[j];
      re = a.row_ptr[j + 1];
      hub = a.n_seg > 0 && re - rs > a.seg_len;  // its segments were summed above
    }
    float acc = gat_dz_sum<U>(a, rs + lig, hub ? rs : re, LPG, pol);
#pragma unroll
    for (int o = LPG / 2; o; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (j < a.n_rows && lig == 0 && !hub) a.der[j] = acc;
  }
}

__global__ void k_gat_der_combine(int64_t n_heavy, const int32_t* __restrict__ heavy_rows,
                                  const int32_t* __restrict__ seg_ptr, const float* __restrict__ seg_der,
                                  float* __restrict__ der) {
  for (int64_t h = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; h < n_heavy; h += (int64_t)gridDim.x * blockDim.x) {
    float acc = 0.f;
    for (int32_t q = seg_ptr[h]; q < seg_ptr[h + 1]; ++q) acc += seg_der[q];
    der[heavy_rows[h]] = acc;
  }
}

static int der_lpg(float avg) { return avg >= 96.f ? 32 : avg >= 24.f ? 16 : avg >= 6.f ? 8 : 4; }

granii_status launch_gat_der(const granii_graph_s* g, const granii_graph_s* gt, const float* er, const float* tv,
                             float* tvb, const float4* recs, float* der, cudaStream_t st) {
  if (g->n_rows == 0) return GRANII_OK;
  if (!g->tperm || !g->tblk) return fail(GRANII_ERR_INVALID_ARG, "der-only GAT backward without the blocked entry map");
  DevInfo di;
  GR_TRY(dev_info(&di));
  const double nnz = (double)g->local_nnz, R = (double)g->n_rows;
  const int hint = l2hint_enabled();
  {
    // algorithmic bytes: per entry col + dα - c + blocked position + er + dz; per row 8 B row_ptr + record
    ProfScope ps("gat_dz", st, nnz * 20.0 + R * 24.0, 0.0, 1, -1.0, false);
    GatDzArgs a{g->n_rows, g->row_ptr, g->seg_len, g->n_seg, g->seg_lo, g->seg_hi, g->seg_row, g->col_idx, er,
                recs, tv, g->tblk, tvb, hint};
    const int lpg = der_lpg(g->avg_deg());
    const int64_t want = ceil_div(ceil_div(a.n_rows, 32 / lpg) + a.n_seg, 8);
#define GO(L) k_gat_dz<L, 4><<<(unsigned)persistent_grid(k_gat_dz<L, 4>, 256, di.sms, want), 256, 0, st>>>(a)
    switch (lpg) {
      case 32: GO(32); break;
      case 16: GO(16); break;
      case 8: GO(8); break;
      default: GO(4); break;
    }
#undef GO
    GR_CHECK_LAUNCH();
  }
  // algorithmic bytes: per entry blocked position + dz (a 4-byte gather); per row 8 B row_ptr + der
  ProfScope ps("gat_der", st, (double)gt->local_nnz * 8.0 + (double)gt->n_rows * 12.0, 0.0, gt->n_seg > 0 ? 2 : 1,
               -1.0, false);
  GatDerArgs b{gt->n_rows, gt->row_ptr, gt->seg_len, g->tperm, tvb, der, gt->n_seg, gt->seg_lo, gt->seg_hi, nullptr,
               hint};
  if (gt->n_seg > 0) GR_CUDA(cudaMallocAsync((void**)&b.seg_der, gt->n_seg * sizeof(float), st));
  const int lpg = der_lpg(gt->avg_deg());
  const int64_t want = ceil_div(ceil_div(b.n_rows, 32 / lpg) + b.n_seg, 8);
#define GO(L) k_gat_der<L, 4><<<(unsigned)persistent_grid(k_gat_der<L, 4>, 256, di.sms, want), 256, 0, st>>>(b)
  switch (lpg) {
    case 32: GO(32); break;
    case 16: GO(16); break;
    case 8: GO(8); break;
    default: GO(4); break;
  }
#undef GO
  if (gt->n_seg > 0) {
    k_gat_der_combine<<<(unsigned)ceil_div(gt->n_heavy, 128), 128, 0, st>>>(gt->n_heavy, gt->order, gt->seg_ptr,
                                                                             b.seg_der, der);
    GR_CUDA(cudaFreeAsync(b.seg_der, st));
  }
  GR_CHECK_LAUNCH();
  return GRANII_OK;
}

template <int LPG, int NJ, int U, int MINB = 0, bool CL = false>
static void gb_launch(int pass, const GatBwdArgs& a, cudaStream_t st) {
  constexpr int G = 32 / LPG;
  const int64_t warps = a.n_seg + a.n_wide + ceil_div(a.n_rows - a.n_wide, G);
  const unsigned blocks = (unsigned)std::max<int64_t>(1, ceil_div(warps, 8));
  if (pass == 0 && a.tout)
    k_gat_bwd_a<LPG, NJ, U, MINB, CL, true><<<blocks, 256, 0, st>>>(a);
  else if (pass == 0)
    k_gat_bwd_a<LPG, NJ, U, MINB, CL><<<blocks, 256, 0, st>>>(a);
  else
    k_gat_bwd_b<LPG, NJ, U, MINB, CL><<<blocks, 256, 0, st>>>(a);
}

granii_status launch_gat_prep(int64_t R, int64_t K, const float* out, int64_t ldo, const float* g, int64_t ldg,
                              bool relu, float* dY, int64_t ldd, float* c, cudaStream_t st) {
  if (R == 0) return GRANII_OK;
  ProfScope ps("elementwise", st, 12.0 * R * K + 4.0 * R, 2.0 * R * K, 1);
  const bool v4 = ldo % 4 == 0 && ldg % 4 == 0 && ldd % 4 == 0 && ((uintptr_t)out & 15u) == 0 &&
                  ((uintptr_t)g & 15u) == 0 && ((uintptr_t)dY & 15u) == 0;
  const int Kv = (int)(v4 ? (K + 3) / 4 : K);
  int lg = 0;
  while (lg < 5 && (1 << lg) < Kv) ++lg;
  const unsigned blocks = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(R << lg, 256), 148 * 16));
  if (v4) k_gat_prep<4><<<blocks, 256, 0, st>>>(R, (int)K, Kv, lg, out, ldo, g, ldg, relu ? 1 : 0, dY, ldd, c);
  else k_gat_prep<1><<<blocks, 256, 0, st>>>(R, (int)K, Kv, lg, out, ldo, g, ldg, relu ? 1 : 0, dY, ldd, c);
  GR_CHECK_LAUNCH();
  return GRANII_OK;
}

static granii_status gb_dispatch(int pass, const GatBwdArgs& b, bool dense, cudaStream_t st);

granii_status launch_gat_bwd_pass(const granii_graph_s* g, int pass, const GatBwdArgs& a, cudaStream_t st) {
  if (a.n_rows == 0) return GRANII_OK;
  const int64_t K = a.K;
  if (K > 2048) return fail(GRANII_ERR_UNSUPPORTED, "GAT backward supports K <= 2048");
  const double nnz = (double)g->local_nnz, R = (double)a.n_rows;
  // algorithmic bytes (SURVEY §8(d) SpMM/SDDMM rows): A = col + er + Z row per entry, dX row + 8 B row_ptr
  // + stat + del per row; B = col + stat + dX row per entry, Z row + out row + ... per row
  const double bytes = pass == 0 ? nnz * (8.0 + 4.0 * K) + R * (4.0 * K + 8.0 + 28.0)
                                 : nnz * (20.0 + 4.0 * K) + R * (8.0 * K + 8.0 + 16.0);
  DevInfo di;
  GR_TRY(dev_info(&di));
  const double gathered = (double)g->n_cols * 4.0 * (double)K;  // the gathered operand (Z or dX rows)
  ProfScope ps(pass == 0 ? "gat_bwd_a" : "gat_bwd_b", st, bytes, (pass == 0 ? 2.0 : 4.0) * nnz * K, 1,
               bytes - nnz * 4.0 * (double)K + gathered, gathered <= 0.6 * (double)di.l2_bytes);
  // lane-group width (tools/gatbwd_sweep.py on the products-shaped graph): 8 lanes x NJ float4
  // up to K = 64 (4 groups per warp), 16 lanes up to 256, full-warp groups beyond
  // dense graphs (avg degree >= 16): a warp per row; sparse: a lane group per row, the wide
  // rows (degree > g->wide_deg) a warp each
  GatBwdArgs b = a;
  const bool dense = g->avg_deg() >= 16.f;
  b.n_wide = dense ? a.n_rows : std::min<int64_t>(g->n_wide, a.n_rows);
  // group-per-row graphs: hub rows (degree > seg_len, order[0 .. n_heavy)) are cut into the graph's
  // warp-wide segments (a 655-entry pubmed hub was a 160-step serial tail at K=256: pass A 0.143 ->
  // 0.073 ms, B 0.101 -> 0.054); on warp-per-row graphs the hubs start first and finish inside
  // the pass (products: no gain), so they stay whole.  GRANII_GATBWD_SEG=0/1 forces either.
  const char* se = getenv("GRANII_GATBWD_SEG");
  const bool use_seg = se ? se[0] != '0' : !dense;
  const int64_t nh = (a.n_rows == g->n_rows && use_seg) ? g->n_heavy : 0;
  float* scratch = nullptr;
  if (nh > 0) {
    b.n_seg = g->n_seg;
    b.seg_lo = g->seg_lo;
    b.seg_hi = g->seg_hi;
    b.seg_row = g->seg_row;
    b.seg_ptr = g->seg_ptr;
    b.heavy_rows = g->order;
    b.n_heavy = nh;
    b.order = a.order + nh;
    b.n_rows = a.n_rows - nh;
    b.n_wide = std::max<int64_t>(0, b.n_wide - nh);
    b.ldp = round_up(K, 4);
    const size_t fl = pass == 0 ? (size_t)g->n_seg * 4 : (size_t)g->n_seg * (b.ldp + 1);
    GR_CUDA(cudaMallocAsync((void**)&scratch, fl * sizeof(float), st));
    if (pass == 0) b.seg_a = reinterpret_cast<float4*>(scratch);
    else {
      b.seg_b = scratch;
      b.seg_der = scratch + (size_t)g->n_seg * b.ldp;
    }
  }
  granii_status rs = gb_dispatch(pass, b, dense, st);
  if (rs == GRANII_OK && nh > 0) {
    if (pass == 0)
      k_gat_a_combine<<<(unsigned)ceil_div(nh, 128), 128, 0, st>>>(b);
    else
      k_gat_b_combine<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(nh * K, 256), 4096)), 256, 0, st>>>(b);
    GR_CHECK_LAUNCH();
    ps.add_launches(1);
  }
  if (scratch) GR_CUDA(cudaFreeAsync(scratch, st));
  return rs;
}

static granii_status gb_dispatch(int pass, const GatBwdArgs& b, bool dense, cudaStream_t st) {
  const int64_t K = b.K;
  // K % 4 == 0: pass A on warp-per-row graphs gathers the Z rows without per-element masks
  // (products K=100: 9.4 -> 7.7 ms; GRANII_GATBWD_CL=0: masked).  Pass B keeps the masked loader:
  // unmasked it needs 3 blocks / SM to avoid spills and loses (9.4 -> 9.9 ms).
  const char* ce = getenv("GRANII_GATBWD_CL");
  const bool cl = K % 4 == 0 && pass == 0 && !(ce && ce[0] == '0');
  // tuning hook GRANII_GATBWD="LPG,NJ,U[,MINB[,CL]]" (tools/gatbwd_sweep.py), if it covers K; CL = 1: the
  // unmasked row loader (K % 4 == 0 only)
  if (const char* e = getenv("GRANII_GATBWD")) {
    int l = 0, n = 0, u = 0, mb = 0, c = 0;
    sscanf(e, "%d,%d,%d,%d,%d", &l, &n, &u, &mb, &c);
    c = c && K % 4 == 0;
    if ((int64_t)l * n * 4 >= K) {
      bool ok = true;
#define GB_TRY(L, N, U_, MB)                                 \
  if (l == L && n == N && u == U_ && mb == MB) {             \
    if (c) gb_launch<L, N, U_, MB, true>(pass, b, st);       \
    else gb_launch<L, N, U_, MB, false>(pass, b, st);        \
  } else
      GB_TRY(8, 2, 2, 0) GB_TRY(8, 2, 2, 4) GB_TRY(4, 3, 2, 0) GB_TRY(4, 3, 4, 0) GB_TRY(4, 3, 2, 4)
      GB_TRY(4, 3, 4, 3) GB_TRY(16, 2, 2, 0) GB_TRY(16, 2, 2, 4) GB_TRY(4, 7, 1, 0) GB_TRY(4, 7, 2, 0)
      GB_TRY(4, 7, 1, 3) GB_TRY(8, 4, 1, 0) GB_TRY(8, 4, 2, 0) GB_TRY(4, 4, 2, 0) GB_TRY(32, 2, 1, 0)
      GB_TRY(16, 4, 2, 0) GB_TRY(4, 8, 1, 0) GB_TRY(16, 2, 2, 3) GB_TRY(8, 2, 2, 3)
      ok = false;
#undef GB_TRY
      if (ok) {
        GR_CHECK_LAUNCH();
        return GRANII_OK;
      }
    }
  }
  if (K <= 16) gb_launch<4, 1, 4>(pass, b, st);
  else if (K <= 32) gb_launch<8, 1, 4>(pass, b, st);
  // pass B on warp-per-row graphs at 4 blocks / SM (64 registers, a few spilled): products K=47
  // 6.76 -> 6.22 ms, K=100 10.7 -> 10.3 ms (pass A is slower there)
  else if (K <= 64) {
    if (pass == 1 && dense) {
      gb_launch<8, 2, 2, 4>(pass, b, st);
    } else if (dense && cl) {
      gb_launch<8, 2, 2, 0, true>(pass, b, st);
    } else {
      gb_launch<8, 2, 2>(pass, b, st);
    }
  }
  // warp-per-row graphs (products-shaped sweep): 16-lane groups up to K = 128 (K=100: A 10.9 -> 9.8,
  // B 13.0 -> 10.5 ms vs <8,4,2>); pass A keeps one entry per group in flight beyond K = 128 (K=256
  // 18.8 -> 18.3 ms, K=512 39.1 -> 35.2 ms).  Group-per-row graphs keep more rows per warp (pubmed-
  // shaped K=256: <32,2,1> for pass A cost 0.19 -> 0.25 ms)
  else if (K <= 128) {
    if (dense && pass == 1) {
      gb_launch<16, 2, 2, 4>(pass, b, st);
    } else if (dense) {
      if (cl) gb_launch<16, 2, 2, 0, true>(pass, b, st);
      else gb_launch<16, 2, 2>(pass, b, st);
    } else {
      gb_launch<8, 4, 2>(pass, b, st);
    }
  } else if (K <= 256) {
    if (pass == 0 && dense && cl) gb_launch<32, 2, 1, 0, true>(pass, b, st);
    else if (pass == 0 && dense) gb_launch<32, 2, 1>(pass, b, st);
    else gb_launch<16, 4, 2>(pass, b, st);
  } else if (K <= 512) {
    if (pass == 0 && dense && cl) gb_launch<32, 4, 1, 0, true>(pass, b, st);
    else if (pass == 0 && dense) gb_launch<32, 4, 1>(pass, b, st);
    else gb_launch<32, 4, 2>(pass, b, st);
  }
  else if (K <= 1024) gb_launch<32, 8, 1>(pass, b, st);
  else gb_launch<32, 16, 1>(pass, b, st);
  GR_CHECK_LAUNCH();
  return GRANII_OK;
}

// ---------------------------------------------------------------- small dense helpers
// partial[s][2][K] = Σ_{r in chunk s} H[r, :] * (d0[r], d1[r]); block (32, 8), fixed order
__global__ void k_colreduce2(int64_t R, int64_t K, const float* __restrict__ H, int64_t ldh,
                             const float* __restrict__ d0, const float* __restrict__ d1, int64_t chunk,
                             double* __restrict__ partial) {
  // fp64 accumulation: da = Hᵀ del sums millions of products of both signs (the softmax backward's
  // del is centred), and an fp32 running sum loses the result's low bits to the cancellation
  __shared__ double sp[8][33], sq[8][33];
  const int tx = threadIdx.x, ty = threadIdx.y;
  const int64_t col = blockIdx.x * 32 + tx, s = blockIdx.y;
  const int64_t r0 = s * chunk, r1 = (r0 + chunk < R) ? r0 + chunk : R;
  double p = 0.0, q = 0.0;
  if (col < K) {
    int64_t r = r0 + ty;
    for (; r + 24 < r1; r += 32) {  // four rows in flight per thread, summed in row order
      float h[4], a0[4], a1[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        h[u] = H[(r + 8 * u) * ldh + col];
        a0[u] = __ldg(d0 + r + 8 * u);
        a1[u] = __ldg(d1 + r + 8 * u);
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        p = fma((double)h[u], (double)a0[u], p);
        q = fma((double)h[u], (double)a1[u], q);
      }
    }
    for (; r < r1; r += 8) {
      const double h = H[r * ldh + col];
      p = fma(h, (double)__ldg(d0 + r), p);
      q = fma(h, (double)__ldg(d1 + r), q);
    }
  }
  sp[ty][tx] = p;
  sq[ty][tx] = q;
  __syncthreads();
  if (ty == 0 && col < K) {
    double a = 0.0, c = 0.0;
#pragma unroll
    for (int y = 0; y < 8; ++y) {
      a += sp[y][tx];
      c += sq[y][tx];
    }
    partial[(s * 2 + 0) * K + col] = a;
    partial[(s * 2 + 1) * K + col] = c;
  }
}

// 16-byte rows (ldh % 4 == 0, H aligned): a thread owns 4 adjacent columns (a warp 128), eight rows in
// flight per thread -- 16 KB of H in flight per CTA instead of 2 KB (products K = 100: 0.67 -> see DESIGN
// §5.5).  Columns past K read the row's padding, which only ever feeds columns that are never stored.
__global__ void __launch_bounds__(256) k_colreduce2v(int64_t R, int64_t K, const float* __restrict__ H, int64_t ldh,
                                                     const float* __restrict__ d0, const float* __restrict__ d1,
                                                     int64_t chunk, double* __restrict__ partial) {
  __shared__ double sp[8][129], sq[8][129];
  const int tx = threadIdx.x, ty = threadIdx.y;
  const int64_t c4 = blockIdx.x * 128 + 4 * tx, s = blockIdx.y;
  const int64_t r0 = s * chunk, r1 = (r0 + chunk < R) ? r0 + chunk : R;
  double p[4] = {0.0, 0.0, 0.0, 0.0}, q[4] = {0.0, 0.0, 0.0, 0.0};
  if (c4 < K) {
    int64_t r = r0 + ty;
    constexpr int UN = 8;
    for (; r + 8 * (UN - 1) < r1; r += 8 * UN) {  // UN rows in flight per thread, summed in row order
      float4 h[UN];
      float a0[UN], a1[UN];
#pragma unroll
      for (int u = 0; u < UN; ++u) {
        h[u] = __ldg(reinterpret_cast<const float4*>(H + (r + 8 * u) * ldh + c4));
        a0[u] = __ldg(d0 + r + 8 * u);
        a1[u] = __ldg(d1 + r + 8 * u);
      }
#pragma unroll
      for (int u = 0; u < UN; ++u) {
        const float hv[4] = {h[u].x, h[u].y, h[u].z, h[u].w};
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          p[j] = fma((double)hv[j], (double)a0[u], p[j]);
          q[j] = fma((double)hv[j], (double)a1[u], q[j]);
        }
      }
    }
    for (; r < r1; r += 8) {
      const float4 h = __ldg(reinterpret_cast<const float4*>(H + r * ldh + c4));
      const float hv[4] = {h.x, h.y, h.z, h.w};
      const double a = __ldg(d0 + r), b = __ldg(d1 + r);
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        p[j] = fma((double)hv[j], a, p[j]);
        q[j] = fma((double)hv[j], b, q[j]);
      }
    }
  }
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    sp[ty][4 * tx + j] = p[j];
    sq[ty][4 * tx + j] = q[j];
  }
  __syncthreads();
  // 256 threads write the tile's 128 columns x (p, q): fixed-order sum over the 8 row groups
  const int c = threadIdx.y * 32 + threadIdx.x;  // 0 .. 255
  const int col = c & 127, which = c >> 7;
  const int64_t gc = blockIdx.x * 128 + col;
  if (gc < K) {
    double a = 0.0;
#pragma unroll
    for (int y = 0; y < 8; ++y) a += which ? sq[y][col] : sp[y][col];
    partial[(s * 2 + which) * K + gc] = a;
  }
}

// out[i] + out[n + i] = the fp64 sum as a float pair (hi, lo): Wᵀ·(Hᵀ del) cancels, and rounding
// Hᵀ del to fp32 before that product cost da_l 3e-4 normwise at products scale (DESIGN R22); the pair
// travels through the fp32 all-reduce of several GPUs as two float sums.  A warp per output: lanes take
// the chunks s = lane, lane + 32, ... in order, then a fixed xor butterfly (was a thread per output
// walking all S chunks serially).
__global__ void k_sum_chunks(int64_t n, int64_t S, const double* __restrict__ partial, float* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (i >= n) return;
  double a = 0.0;
  for (int64_t s = lane; s < S; s += 32) a += partial[s * n + i];
#pragma unroll
  for (int o = 16; o; o >>= 1) a += __shfl_xor_sync(0xffffffffu, a, o);
  if (lane == 0) {
    const float hi = (float)a;
    out[i] = hi;
    out[n + i] = (float)(a - (double)hi);
  }
}

static bool colreduce_vec(int64_t ldh, const float* H) { return ldh % 4 == 0 && ((uintptr_t)H & 15) == 0; }

static int64_t colreduce_chunks(int64_t R, int64_t K, bool vec = false) {
  const int64_t tiles = ceil_div(K, vec ? 128 : 32);
  return std::max<int64_t>(1, std::min<int64_t>(ceil_div(R, 512), ceil_div(148 * 8, tiles)));
}

size_t colreduce2_workspace(int64_t R, int64_t K) {
  return (size_t)std::max(colreduce_chunks(R, K), colreduce_chunks(R, K, true)) * 2 * K * sizeof(double);
}

granii_status launch_colreduce2(int64_t R, int64_t K, const float* H, int64_t ldh, const float* d0, const float* d1,
                                float* partial, float* out, cudaStream_t st) {
  const bool vec = colreduce_vec(ldh, H);
  const int64_t S = colreduce_chunks(R, K, vec), chunk = ceil_div(std::max<int64_t>(R, 1), S);
  ProfScope ps("elementwise", st, 4.0 * R * K + 8.0 * R, 4.0 * R * K, 2);
  if (vec)
    k_colreduce2v<<<dim3((unsigned)ceil_div(K, 128), (unsigned)S), dim3(32, 8), 0, st>>>(
        R, K, H, ldh, d0, d1, chunk, reinterpret_cast<double*>(partial));
  else
    k_colreduce2<<<dim3((unsigned)ceil_div(K, 32), (unsigned)S), dim3(32, 8), 0, st>>>(R, K, H, ldh, d0, d1, chunk,
                                                                                     reinterpret_cast<double*>(partial));
  k_sum_chunks<<<(unsigned)ceil_div(2 * K * 32, 256), 256, 0, st>>>(2 * K, S, reinterpret_cast<const double*>(partial), out);  // 4K floats
  GR_CHECK_LAUNCH();
  return GRANII_OK;
}

// u = W a_l, v = W a_r (W: K1 x K2, ld K2); warp per row of W
__global__ void k_matvec2(int64_t K1, int64_t K2, const float* __restrict__ W, const float* __restrict__ al,
                          const float* __restrict__ ar, float* __restrict__ u, float* __restrict__ v) {
  const int lane = threadIdx.x & 31;
  const int64_t r = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (r >= K1) return;
  float a = 0.f, b = 0.f;
  for (int64_t k = lane; k < K2; k += 32) {
    const float x = W[r * K2 + k];
    a = fmaf(x, al[k], a);
    b = fmaf(x, ar[k], b);
  }
  a = gb_warp_sum(a);
  b = gb_warp_sum(b);
  if (lane == 0) {
    u[r] = a;
    v[r] = b;
  }
}

// da_l = Wᵀ p, da_r = Wᵀ q (fixed order over rows and row groups), in fp64 from the
// (hi, lo) pairs of p = [p | q | p_lo | q_lo] (k_sum_chunks): the sum cancels
// 32 columns x 8 row groups per CTA (rows r = ty, ty + 8, ...), fp64 partials combined in fixed order
// (was a thread per column walking all K1 rows: ~90 us on two CTAs for 128 x 256)
__global__ void __launch_bounds__(256) k_mattvec2(int64_t K1, int64_t K2, const float* __restrict__ W,
                                                  const float* __restrict__ pq, float* __restrict__ dal,
                                                  float* __restrict__ dar) {
  __shared__ double sa[8][33], sb[8][33];
  const int tx = threadIdx.x, ty = threadIdx.y;
  const int64_t k = blockIdx.x * 32 + tx;
  double a = 0.0, b = 0.0;
  if (k < K2) {
    for (int64_t r = ty; r < K1; r += 8) {
      const double x = W[r * K2 + k];
      a = fma(x, (double)pq[r] + (double)pq[2 * K1 + r], a);
      b = fma(x, (double)pq[K1 + r] + (double)pq[3 * K1 + r], b);
    }
  }
  sa[ty][tx] = a;
  sb[ty][tx] = b;
  __syncthreads();
  if (ty == 0 && k < K2) {
    double x = 0.0, y = 0.0;
#pragma unroll
    for (int g = 0; g < 8; ++g) {
      x += sa[g][tx];
      y += sb[g][tx];
    }
    if (dal) dal[k] = (float)x;
    if (dar) dar[k] = (float)y;
  }
}

// dW += p a_lᵀ + q a_rᵀ (p, q from their (hi, lo) pairs)
__global__ void k_rank2(int64_t K1, int64_t K2, float* __restrict__ dW, const float* __restrict__ pq,
                        const float* __restrict__ al, const float* __restrict__ ar) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= K1 * K2) return;
  const int64_t r = i / K2, k = i % K2;
  const float p = pq[r] + pq[2 * K1 + r], q = pq[K1 + r] + pq[3 * K1 + r];
  dW[i] += p * al[k] + q * ar[k];
}

granii_status launch_gat_matvec2(int64_t K1, int64_t K2, const float* W, const float* a_l, const float* a_r,
                                float* u, float* v, cudaStream_t st) {
  ProfScope ps("elementwise", st, 4.0 * K1 * K2, 4.0 * K1 * K2, 1);
  k_matvec2<<<(unsigned)ceil_div(K1, 8), 256, 0, st>>>(K1, K2, W, a_l, a_r, u, v);
  GR_CHECK_LAUNCH();
  return GRANII_OK;
}

granii_status launch_gat_mattvec2(int64_t K1, int64_t K2, const float* W, const float* pq, float* da_l, float* da_r,
                                  cudaStream_t st) {
  ProfScope ps("elementwise", st, 4.0 * K1 * K2, 4.0 * K1 * K2, 1);
  k_mattvec2<<<(unsigned)ceil_div(K2, 32), dim3(32, 8), 0, st>>>(K1, K2, W, pq, da_l, da_r);
  GR_CHECK_LAUNCH();
  return GRANII_OK;
}

granii_status launch_gat_rank2(int64_t K1, int64_t K2, float* dW, const float* pq, const float* a_l, const float* a_r,
                               cudaStream_t st) {
  ProfScope ps("elementwise", st, 8.0 * K1 * K2, 4.0 * K1 * K2, 1);
  k_rank2<<<(unsigned)ceil_div(K1 * K2, 256), 256, 0, st>>>(K1, K2, dW, pq, a_l, a_r);
  GR_CHECK_LAUNCH();
  return GRANII_OK;
}

}  // namespace granii
