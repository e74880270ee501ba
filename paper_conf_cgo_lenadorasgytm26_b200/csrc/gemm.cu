// gemm.cu -- the update GEMM (Θ = H W of Eq. 4)
// on 5th-generation tensor cores, fp32-accurate.
//
// C[M x N] = A[M x K] · B[K x N] (+ fused epilogue: row scale = Eq. 1 row-
// broadcast, GAT attention GEMVs el = C a_l / er = C a_r, ReLU).
//
// Tensor-core path: persistent (one CTA per SM over 128 x BN
// tiles, BN <= 128; the N tiles of an M tile run back to back so A re-reads hit
// L2), warp-specialised, 18 warps:
//   warp 0       TMA producer: raw A stages (128 x 32 fp32, SWIZZLE_128B) and
//                pre-split B_hi / B_lo stages (BN x 32, K-major)
//   warp 1       TMEM allocator + single-thread MMA issuer: 3 x tcgen05.mma
//                kind::tf32 per 8-wide k step with A read from TMEM
//                (A_hi B_hi + A_hi B_lo + A_lo B_hi -- the 3xTF32 split), into
//                one of two TMEM accumulators (epilogue overlap)
//   warps 2..9   converters: split raw A rows into tf32 hi / lo and tcgen05.st
//                them into TMEM; the raw smem stage is released immediately
//   warps 10..17 epilogue: tcgen05.ld -> row scale / attention GEMVs / ReLU ->
//                smem transpose -> full 128-byte line stores
// B (the weight, <= K1 x K2 floats) is split and transposed once per call into
// the workspace by a tiny prep kernel.
//
// dW = Aᵀ B (reduction over nodes): MN-major tf32 operands (SWIZZLE_128B_BASE32B)
// with split-K and a fixed-order partial sum.  Fallbacks (unaligned lda / ldb):
// fp32 SIMT tiles and a deterministic split-K SIMT kernel.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <mutex>

#include "internal.h"

namespace granii {

// ======================================================================= PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load_2d(const CUtensorMap* map, uint64_t* bar, void* dst, int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::
          "r"(smem_u32(dst)),
      "l"(map), "r"(smem_u32(bar)), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void fence_barrier_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// UMMA shared-memory descriptor, K-major, SWIZZLE_128B (rows of 128 B, 8-row groups 1024 B apart).
__device__ __forceinline__ uint64_t desc_sw128(uint32_t saddr) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr & 0x3FFFFu) >> 4);  // start address  [0,14)
  d |= (uint64_t)1 << 16;                    // leading byte offset (unused for swizzled K-major)
  d |= (uint64_t)(1024 >> 4) << 32;          // stride byte offset = 1024 B
  d |= (uint64_t)1 << 46;                    // descriptor version (sm_100)
  d |= (uint64_t)2 << 61;                    // SWIZZLE_128B
  return d;
}
// instruction descriptor: D fp32, A/B tf32, both K-major, M = 128, N = BN
__host__ __device__ constexpr uint32_t idesc_tf32(int M, int N) {
  return (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}
__device__ __forceinline__ void mma_tf32(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n" ::"r"(tmem_d),
      "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void mma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, float (&v)[16]) {
  uint32_t r[16];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
}
__device__ __forceinline__ float tf32_rna(float x) {
  uint32_t r;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
  return __uint_as_float(r);
}

// The 3xTF32 split of the hot converters: hi = x rounded half-up (on the magnitude) to 10 mantissa
// bits by integer add + mask, lo = x - hi (exact in fp32), passed with all its bits -- the tf32 MMA
// reads the top 19 bits of every operand, so lo is truncated there.  3 instructions per element
// (cvt.rna.tf32.f32 expands to ~5 on sm_100a, and the split needed two of them); finite inputs.
__device__ __forceinline__ void tf32_split(float x, float& hi, float& lo) {
  hi = __uint_as_float((__float_as_uint(x) + 0x1000u) & 0xFFFFE000u);
  lo = x - hi;
}

// lo = x - trunc_tf32(x) (exact in fp32), for an MMA that reads x itself as the truncated hi
__device__ __forceinline__ float4 tf32_lo_trunc(float4 x) {
  float4 l;
  l.x = x.x - __uint_as_float(__float_as_uint(x.x) & 0xFFFFE000u);
  l.y = x.y - __uint_as_float(__float_as_uint(x.y) & 0xFFFFE000u);
  l.z = x.z - __uint_as_float(__float_as_uint(x.z) & 0xFFFFE000u);
  l.w = x.w - __uint_as_float(__float_as_uint(x.w) & 0xFFFFE000u);
  return l;
}

// ======================================================================= tcgen05 kernel
constexpr int TC_BM = 128, TC_BK = 32;  // 32 fp32 = one 128-byte swizzle row

template <int BN>
struct TcCfg {
  static constexpr int A_BYTES = TC_BM * TC_BK * 4;                  // raw A stage: 128 x 32 fp32 = 16 KB
  static constexpr int B_BYTES = BN * TC_BK * 4;                     // one of B_hi / B_lo
  static constexpr int ACC_COLS = BN <= 32 ? 32 : BN <= 64 ? 64 : 128;  // one fp32 accumulator
  static constexpr int TSTAGES = 4;                                  // split A (hi | lo) stages in TMEM
  static constexpr int TMEM_COLS = 512;                              // 2 accumulators + TSTAGES x 64
  static_assert(2 * ACC_COLS + TSTAGES * 64 <= TMEM_COLS, "TMEM budget");
  static constexpr int EPI_BYTES = 8 * 32 * 33 * 4;                  // epilogue staging (8 warps x 32 x 33)
  static constexpr int B_STAGE = 2 * B_BYTES;
  // raw A stages (HBM stream), then B stages (L2, <= 4); 8 A stages measured no faster
  static constexpr int RA = 4;
  static constexpr int SB_FIT = (200 * 1024 - RA * A_BYTES - EPI_BYTES) / B_STAGE;
  static constexpr int SB = SB_FIT > 4 ? 4 : SB_FIT;                 // B (hi, lo) stages in smem
  static_assert(RA >= 2 && SB >= 2, "smem budget");
  static constexpr int SMEM = RA * A_BYTES + SB * B_STAGE + EPI_BYTES + 1024 /*align*/ + 512 /*barriers*/;
};

struct TcEpi {
  float* C;
  int64_t ldc;
  const float* row_scale;
  const float* att_l;
  const float* att_r;
  float* out_l;  // [n_tiles_n][M] partials (or final when one N tile)
  float* out_r;
  int relu;
  int store;
};

__device__ __forceinline__ void mma_tf32_ta(uint32_t tmem_d, uint32_t tmem_a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n}\n" ::"r"(tmem_d),
      "r"(tmem_a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void tmem_st32(uint32_t taddr, const uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,"
      "%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]),
      "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]), "r"(r[16]), "r"(r[17]), "r"(r[18]),
      "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]), "r"(r[24]), "r"(r[25]), "r"(r[26]), "r"(r[27]),
      "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31])
      : "memory");
}

// Persistent, warp-specialised, one CTA per SM looping over 128 x BN output tiles
// (the N tiles of one M tile back to back so A's re-read hits L2).
//   warp 0      TMA producer: raw A (128 x 32 fp32, SWIZZLE_128B) ring of RA stages and
//               the pre-split B_hi / B_lo (BN x 32, K-major) ring of SB stages
//   warps 2..9  converters (two groups alternating k-blocks): each thread takes one row of the raw A stage (conflict-free
//               swizzled 16-byte reads), splits it into tf32 hi / lo and writes both into
//               a TMEM A stage with tcgen05.st; the raw smem stage is released to the TMA
//               right away (it no longer waits for the MMA)
//   warp 1      TMEM allocator + single-thread MMA issuer: tcgen05.mma kind::tf32 with A
//               read from TMEM, 3 per 8-wide k step (A_hi B_hi + A_hi B_lo + A_lo B_hi);
//               tile i accumulates into TMEM buffer i & 1 while the epilogue drains the other
//   warps 10..17 epilogue: tcgen05.ld -> scale / GEMVs / ReLU -> smem transpose -> 128 B stores;
//               two warps per TMEM lane quadrant split the 32-column chunks (latency hiding)
constexpr int TC_THREADS = 576;

template <int BN>
__global__ void __launch_bounds__(TC_THREADS, 1)
    k_gemm_tc(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmBh,
              const __grid_constant__ CUtensorMap tmBl, int M, int N, int K, TcEpi ep) {
  using Cfg = TcCfg<BN>;
  constexpr int RA = Cfg::RA, SB = Cfg::SB, TS = Cfg::TSTAGES;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // 1 KB-aligned base by pointer arithmetic on the __shared__ array (an integer round trip would
  // lose the address space and turn every staging access into a generic LD / ST)
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sA = smem;                                   // RA x 16 KB
  uint8_t* sB = smem + RA * Cfg::A_BYTES;               // SB x (B_hi | B_lo)
  float* stage_out = (float*)(sB + SB * Cfg::B_STAGE);  // epilogue staging
  uint64_t* bars = (uint64_t*)((uint8_t*)stage_out + Cfg::EPI_BYTES);
  uint64_t* a_full = bars;                 // [RA] TMA -> converters
  uint64_t* a_empty = a_full + RA;         // [RA] converters -> TMA
  uint64_t* b_full = a_empty + RA;         // [SB] TMA -> MMA
  uint64_t* b_empty = b_full + SB;         // [SB] MMA commit -> TMA
  uint64_t* t_full = b_empty + SB;         // [TS] converters -> MMA (A in TMEM)
  uint64_t* t_empty = t_full + TS;         // [TS] MMA commit -> converters
  uint64_t* c_full = t_empty + TS;         // [2] MMA commit -> epilogue
  uint64_t* c_empty = c_full + 2;          // [2] epilogue -> MMA
  uint32_t* tmem_slot = (uint32_t*)(c_empty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nk = (K + TC_BK - 1) / TC_BK;
  const int mt = (M + TC_BM - 1) / TC_BM, ntn = (N + BN - 1) / BN;

  if (warp == 0 && lane == 0) {
    for (int s = 0; s < RA; ++s) { mbar_init(&a_full[s], 1); mbar_init(&a_empty[s], 128); }
    for (int s = 0; s < SB; ++s) { mbar_init(&b_full[s], 1); mbar_init(&b_empty[s], 1); }
    for (int s = 0; s < TS; ++s) { mbar_init(&t_full[s], 128); mbar_init(&t_empty[s], 1); }
    for (int b = 0; b < 2; ++b) { mbar_init(&c_full[b], 1); mbar_init(&c_empty[b], 256); }
    fence_barrier_init();
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tmA) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tmBh) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tmBl) : "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(Cfg::TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const uint32_t tA0 = tmem + 2 * Cfg::ACC_COLS;  // first TMEM A stage (hi: +0..31, lo: +32..63)

#define TC_TILE_LOOP for (int mi = blockIdx.x; mi < mt; mi += gridDim.x) for (int ni = 0; ni < ntn; ++ni
  if (warp == 0) {
    if (lane == 0) {
      int it = 0;
      TC_TILE_LOOP) {
        const int m0 = mi * TC_BM, n0 = ni * BN;
        for (int kb = 0; kb < nk; ++kb, ++it) {
          const int ra = it % RA, sb = it % SB;
          mbar_wait(&a_empty[ra], ((it / RA) & 1) ^ 1);
          mbar_expect_tx(&a_full[ra], Cfg::A_BYTES);
          tma_load_2d(&tmA, &a_full[ra], sA + ra * Cfg::A_BYTES, kb * TC_BK, m0);
          mbar_wait(&b_empty[sb], ((it / SB) & 1) ^ 1);
          mbar_expect_tx(&b_full[sb], Cfg::B_STAGE);
          tma_load_2d(&tmBh, &b_full[sb], sB + sb * Cfg::B_STAGE, kb * TC_BK, n0);
          tma_load_2d(&tmBl, &b_full[sb], sB + sb * Cfg::B_STAGE + Cfg::B_BYTES, kb * TC_BK, n0);
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      constexpr uint32_t idesc = idesc_tf32(TC_BM, BN);
      int it = 0, lt = 0;
      TC_TILE_LOOP, ++lt) {
        const int buf = lt & 1;
        const uint32_t acc = tmem + (uint32_t)(buf * Cfg::ACC_COLS);
        mbar_wait(&c_empty[buf], ((lt >> 1) & 1) ^ 1);  // epilogue has drained this accumulator
        tc_fence_after();
        for (int kb = 0; kb < nk; ++kb, ++it) {
          const int ts = it % TS, sb = it % SB;
          mbar_wait(&t_full[ts], (it / TS) & 1);
          mbar_wait(&b_full[sb], (it / SB) & 1);
          tc_fence_after();
          const uint32_t ahi = tA0 + ts * 64, alo = ahi + 32;
          const uint32_t bh = smem_u32(sB + sb * Cfg::B_STAGE), bl = bh + Cfg::B_BYTES;
          // the last k-block of a K that is not a multiple of 32 (K1 = 100, 602) only issues the
          // 8-wide steps that hold data: the rest would multiply TMA zero fill by zero B rows
          const int ksteps = min(TC_BK / 8, (K - kb * TC_BK + 7) / 8);
#pragma unroll
          for (int k = 0; k < TC_BK / 8; ++k) {  // tf32: K = 8 per MMA (8 TMEM columns, 32 B of B rows)
            if (k >= ksteps) break;
            const uint64_t dbh = desc_sw128(bh + k * 32), dbl = desc_sw128(bl + k * 32);
            mma_tf32_ta(acc, ahi + k * 8, dbh, idesc, (kb | k) ? 1u : 0u);
            mma_tf32_ta(acc, ahi + k * 8, dbl, idesc, 1u);
            mma_tf32_ta(acc, alo + k * 8, dbh, idesc, 1u);
          }
          mma_commit(&b_empty[sb]);
          mma_commit(&t_empty[ts]);
        }
        mma_commit(&c_full[buf]);
      }
    }
  } else if (warp < 10) {
    // ---------------- converters: raw A row -> tf32 hi / lo -> TMEM
    const int quad = warp & 3;
    const int cgroup = (warp - 2) >> 2;  // group g converts the k-blocks with it % 2 == g
    const int row = quad * 32 + lane;    // TMEM lane == tile row
    int it = 0;
    TC_TILE_LOOP) {
      for (int kb = 0; kb < nk; ++kb, ++it) {
        if ((it & 1) != cgroup) continue;  // the other converter group takes this k-block
        const int ra = it % RA, ts = it % TS;
        mbar_wait(&a_full[ra], (it / RA) & 1);
        const uint8_t* rowp = sA + ra * Cfg::A_BYTES + row * 128;
        uint32_t hi[32], lo[32];
#pragma unroll
        for (int c = 0; c < 8; ++c) {  // SWIZZLE_128B: 16-byte chunk c of row r sits at chunk c ^ (r & 7)
          const float4 x = *reinterpret_cast<const float4*>(rowp + ((c ^ (row & 7)) << 4));
          const float xs[4] = {x.x, x.y, x.z, x.w};
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            float h, l;
            tf32_split(xs[q], h, l);
            hi[c * 4 + q] = __float_as_uint(h);
            lo[c * 4 + q] = __float_as_uint(l);
          }
        }
        fence_proxy_async();            // our generic reads before the TMA's next async write
        mbar_arrive(&a_empty[ra]);      // raw stage free as soon as it is split
        mbar_wait(&t_empty[ts], ((it / TS) & 1) ^ 1);
        tc_fence_after();
        const uint32_t tb = tA0 + ts * 64 + ((uint32_t)(quad * 32) << 16);
        tmem_st32(tb, hi);
        tmem_st32(tb + 32, lo);
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        tc_fence_before();
        mbar_arrive(&t_full[ts]);
      }
    }
  } else {
    // ---------------- epilogue: TMEM -> registers -> global
    const int quad = warp & 3;          // TMEM lanes [32*quad, 32*quad+32)
    const int half = (warp - 10) >> 2;  // which of the two warps of this quadrant
    int lt = 0;
    TC_TILE_LOOP, ++lt) {
      const int buf = lt & 1;
      const int m0 = mi * TC_BM, n0 = ni * BN, ntile = ni;
      mbar_wait(&c_full[buf], (lt >> 1) & 1);
      tc_fence_after();
      const int rbase = m0 + quad * 32;  // this warp's 32 rows
      const int r = rbase + lane;        // the row this thread holds in registers
      const bool rok = r < M;
      const float rsc = (ep.row_scale && rok) ? __ldg(ep.row_scale + r) : 1.f;
      float el = 0.f, er = 0.f;
      float* stg = stage_out + (warp - 10) * 32 * 33;
#pragma unroll 1
      for (int c0 = 32 * half; c0 < BN; c0 += 64) {  // this warp's 32-column chunks (BN % 16 == 0)
        float v[32];
        tmem_ld16(tmem + (uint32_t)(buf * Cfg::ACC_COLS) + ((uint32_t)(quad * 32) << 16) + c0, *(float(*)[16])v);
        if (c0 + 16 < BN)
          tmem_ld16(tmem + (uint32_t)(buf * Cfg::ACC_COLS) + ((uint32_t)(quad * 32) << 16) + c0 + 16,
                    *(float(*)[16])(v + 16));
        const int cb = n0 + c0;
        if (ep.row_scale)
#pragma unroll
          for (int j = 0; j < 32; ++j) v[j] *= rsc;
        if (ep.att_l || ep.att_r) {
          // lane j holds a_l / a_r of this chunk's column j (one coalesced load per chunk, 0 past N),
          // broadcast by shuffle instead of a uniform global load per element
          const bool cj = cb + lane < N && c0 + lane < BN;
          const float alj = (ep.att_l && cj) ? __ldg(ep.att_l + cb + lane) : 0.f;
          const float arj = (ep.att_r && cj) ? __ldg(ep.att_r + cb + lane) : 0.f;
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            const float a_l = __shfl_sync(0xffffffffu, alj, j), a_r = __shfl_sync(0xffffffffu, arj, j);
            if (c0 + j < BN) {  // v[j] past the tile's columns was never loaded
              el = fmaf(v[j], a_l, el);
              er = fmaf(v[j], a_r, er);
            }
          }
        }
        if (ep.relu)
#pragma unroll
          for (int j = 0; j < 32; ++j) v[j] = fmaxf(v[j], 0.f);
        if (ep.store) {
          // transpose through shared memory so every store instruction writes whole
          // 128-byte lines (8 lanes per row, 4 rows per instruction)
#pragma unroll
          for (int j = 0; j < 32; ++j) stg[lane * 33 + j] = v[j];
          __syncwarp();
          const int cc = (lane & 7) * 4;  // 4 consecutive columns
          const bool cfull = (cb + cc + 4 <= N) && (c0 + cc + 4 <= BN) && ((ep.ldc & 3) == 0);
#pragma unroll 4
          for (int rr = lane >> 3; rr < 32; rr += 4) {
            const int rowo = rbase + rr;
            if (rowo >= M) break;
            float* cp = ep.C + (int64_t)rowo * ep.ldc + cb + cc;
            const float* sp = stg + rr * 33 + cc;
            if (cfull && ((((uintptr_t)cp) & 15) == 0)) {
              *reinterpret_cast<float4*>(cp) = make_float4(sp[0], sp[1], sp[2], sp[3]);
            } else {
#pragma unroll
              for (int q = 0; q < 4; ++q)
                if (cb + cc + q < N && c0 + cc + q < BN) cp[q] = sp[q];
            }
          }
          __syncwarp();
        }
      }
      tc_fence_before();
      mbar_arrive(&c_empty[buf]);  // accumulator drained: the MMA may overwrite it
      if (rok) {
        if (ep.out_l) ep.out_l[(int64_t)(2 * ntile + half) * M + r] = el;  // per-half partials
        if (ep.out_r) ep.out_r[(int64_t)(2 * ntile + half) * M + r] = er;
      }
    }
  }
#undef TC_TILE_LOOP
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(Cfg::TMEM_COLS));
  }
}


// B (K x N, or N x K when transposed) -> Bt_hi / Bt_lo [Npad x Kpad], K-major, zero padded.
__global__ void k_prep_b(int K, int N, const float* __restrict__ B, int64_t ldb, int transB, int Kpad, int Npad,
                         float* __restrict__ hi, float* __restrict__ lo) {
  const int64_t total = (int64_t)Npad * Kpad;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int n = (int)(i / Kpad), k = (int)(i % Kpad);
    float x = 0.f;
    if (n < N && k < K) x = transB ? B[(int64_t)n * ldb + k] : B[(int64_t)k * ldb + n];
    const float h = tf32_rna(x);
    hi[i] = h;
    lo[i] = tf32_rna(x - h);
  }
}

// ======================================================================= Aᵀ·B on tensor cores
// dW = Aᵀ B with A stored R x M, B stored R x N (R = nodes, the reduction).  Both
// MMA operands are MN-major: TMA boxes of 32 elements (one 128-byte swizzle row)
// x 32 reduction rows; an MN atom (32 wide) is 4 KB, atoms are LBO = 4 KB apart,
// 8-row k groups SBO = 1 KB apart, one tf32 MMA (K = 8) consumes one k group.
// Split-K over R (blockIdx.z) into a partial buffer [splits][M][N], summed later
// in fixed order (deterministic).  Converters split A and B into hi / lo.
__device__ __forceinline__ uint64_t desc_sw128_mn(uint32_t saddr, uint32_t lbo, uint32_t sbo = 1024) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr & 0x3FFFFu) >> 4);
  d |= (uint64_t)(((lbo & 0x0FFFFFFFu) >> 4) & 0x3FFF) << 16;  // leading byte offset: stride between MN atoms
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;  // stride byte offset: between 8-row k groups
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)((lbo >> 28) & 7u) << 61;   // layout type (1 = SWIZZLE_128B_BASE32B for MN-major tf32)
  return d;
}
__host__ __device__ constexpr uint32_t idesc_tf32_mn(int M, int N) {
  return idesc_tf32(M, N) | (1u << 15) | (1u << 16);  // a_major = b_major = MN
}

// BK: node rows per k-block.  16 halves a stage (raw A + A_lo + raw B + B_lo: 48 KB at BN = 256)
// so 4 stages fit instead of 2 -- the 2-stage ring left the converters waiting on the TMA (ncu:
// a third of their samples on the full barrier, tensor pipe 61 % active)
template <int BN, int BK = TC_BK>
struct TnCfg {
  static constexpr int A_BYTES = TC_BM * BK * 4;  // 128 (M) x BK (k) fp32 = 4 MN atoms
  static constexpr int B_BYTES = BN * BK * 4;
  static constexpr int STAGE = 2 * A_BYTES + 2 * B_BYTES;
  static constexpr int STAGES_FIT = 200 * 1024 / STAGE;
  static constexpr int STAGES = STAGES_FIT > 6 ? 6 : STAGES_FIT;
  static constexpr int ACC_COLS = BN <= 32 ? 32 : BN <= 64 ? 64 : BN <= 128 ? 128 : 256;
  // The tcgen05 fp32 accumulation loses about one ulp of the accumulator per MMA, in one direction
  // (tools/gemm_tn_err.py: the error grows linearly with the k-blocks summed into one accumulator,
  // 1.05e-5 relative after 512 rows of positive products).  A split's k-blocks are therefore spread
  // over NACC accumulators filling the 512 TMEM columns (one CTA per SM), consecutive sub-ranges,
  // summed by the epilogue in fixed order with round-to-nearest CUDA-core adds.
  static constexpr int NACC = 512 / ACC_COLS;
  static constexpr int TMEM_COLS = 512;
  static constexpr int SMEM = STAGES * STAGE + 1024 + 256;
};

// NCW converter warps (warps 2 .. NCW+1); they are also the epilogue, NCW / 4 warps per TMEM lane
// quadrant splitting the columns
template <int BN, int BK = TC_BK, int NCW = 4>
__global__ void __launch_bounds__(64 + 32 * NCW, 1)
    k_gemm_tn_tc(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB, int M, int N,
                 int kblocks_per_split, int total_kblocks, float* __restrict__ part, uint32_t dlbo, uint32_t dsbo,
                 uint32_t dkstep, int raw_hi) {
  using Cfg = TnCfg<BN, BK>;
  constexpr int NCT = 32 * NCW;  // converter threads
  constexpr int S = Cfg::STAGES;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // 1 KB-aligned base by pointer arithmetic on the __shared__ array (an integer round trip would
  // lose the address space and turn every staging access into a generic LD / ST)
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* bars = (uint64_t*)(smem + S * Cfg::STAGE);
  uint64_t* full = bars;
  uint64_t* conv = bars + S;
  uint64_t* empty = bars + 2 * S;
  uint64_t* accum = bars + 3 * S;
  uint32_t* tmem_slot = (uint32_t*)(bars + 3 * S + 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int m0 = blockIdx.x * TC_BM, n0 = blockIdx.y * BN;
  const int kb0 = blockIdx.z * kblocks_per_split;
  const int nk = max(0, min(kblocks_per_split, total_kblocks - kb0));
  auto a_hi = [&](int s) { return smem + s * Cfg::STAGE; };
  auto a_lo = [&](int s) { return smem + s * Cfg::STAGE + Cfg::A_BYTES; };
  auto b_hi = [&](int s) { return smem + s * Cfg::STAGE + 2 * Cfg::A_BYTES; };
  auto b_lo = [&](int s) { return smem + s * Cfg::STAGE + 2 * Cfg::A_BYTES + Cfg::B_BYTES; };
  if (warp == 0 && lane == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&conv[s], NCT);
      mbar_init(&empty[s], 1);
    }
    mbar_init(accum, 1);
    fence_barrier_init();
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(Cfg::TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  if (warp == 0) {
    if (lane == 0) {
      for (int kb = 0; kb < nk; ++kb) {
        const int s = kb % S;
        const uint32_t ph = (kb / S) & 1;
        mbar_wait(&empty[s], ph ^ 1);
        mbar_expect_tx(&full[s], Cfg::A_BYTES + Cfg::B_BYTES);
        const int r = (kb0 + kb) * BK;
#pragma unroll
        for (int t = 0; t < TC_BM / 32; ++t) tma_load_2d(&tmA, &full[s], a_hi(s) + t * 32 * BK * 4, m0 + 32 * t, r);
#pragma unroll
        for (int t = 0; t < BN / 32; ++t) tma_load_2d(&tmB, &full[s], b_hi(s) + t * 32 * BK * 4, n0 + 32 * t, r);
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && nk > 0) {
      const uint32_t idesc = (idesc_tf32(TC_BM, BN) & ~(3u << 15)) | ((dkstep >> 16) << 15);
      for (int kb = 0; kb < nk; ++kb) {
        const int s = kb % S;
        const uint32_t ph = (kb / S) & 1;
        mbar_wait(&conv[s], ph);
        tc_fence_after();
        const uint32_t ah = smem_u32(a_hi(s)), al = smem_u32(a_lo(s));
        const uint32_t bh = smem_u32(b_hi(s)), bl = smem_u32(b_lo(s));
        // accumulator t takes the k-blocks [ceil(t nk / NACC), ceil((t+1) nk / NACC))
        const int t = (int)((int64_t)kb * Cfg::NACC / nk);
        const bool first = kb == 0 || (int)((int64_t)(kb - 1) * Cfg::NACC / nk) != t;
        const uint32_t acc = tmem + (uint32_t)(t * Cfg::ACC_COLS);
#pragma unroll
        for (int k = 0; k < BK / 8; ++k) {  // one 8-row k group (1 KB) per MMA
          const uint32_t off = k * (dkstep & 0xFFFF);
          const uint64_t dah = desc_sw128_mn(ah + off, dlbo, dsbo), dal = desc_sw128_mn(al + off, dlbo, dsbo);
          const uint64_t dbh = desc_sw128_mn(bh + off, dlbo, dsbo), dbl = desc_sw128_mn(bl + off, dlbo, dsbo);
          mma_tf32(acc, dah, dbh, idesc, (!first || k) ? 1u : 0u);
          mma_tf32(acc, dah, dbl, idesc, 1u);
          mma_tf32(acc, dal, dbh, idesc, 1u);
        }
        mma_commit(&empty[s]);
      }
      mma_commit(accum);
    }
  } else {
    const int ct = threadIdx.x - 64;
    for (int kb = 0; kb < nk; ++kb) {
      const int s = kb % S;
      const uint32_t ph = (kb / S) & 1;
      mbar_wait(&full[s], ph);
      float4* ahp = reinterpret_cast<float4*>(a_hi(s));
      float4* alp = reinterpret_cast<float4*>(a_lo(s));
      float4* bhp = reinterpret_cast<float4*>(b_hi(s));
      float4* blp = reinterpret_cast<float4*>(b_lo(s));
      if (raw_hi) {
        // the raw stage IS the hi operand: the tf32 MMA reads the top 19 bits of each fp32 (truncation),
        // so hi = trunc(x) needs no store and only lo = x - trunc(x) (exact) is written -- half the
        // converters' shared-memory stores (the kernel is shared-memory-bandwidth bound)
#pragma unroll 4
        for (int i = ct; i < Cfg::A_BYTES / 16; i += NCT) alp[i] = tf32_lo_trunc(ahp[i]);
#pragma unroll 4
        for (int i = ct; i < Cfg::B_BYTES / 16; i += NCT) blp[i] = tf32_lo_trunc(bhp[i]);
      } else {
#pragma unroll 4
        for (int i = ct; i < Cfg::A_BYTES / 16; i += NCT) {
          const float4 x = ahp[i];
          float4 h, l;
          tf32_split(x.x, h.x, l.x);
          tf32_split(x.y, h.y, l.y);
          tf32_split(x.z, h.z, l.z);
          tf32_split(x.w, h.w, l.w);
          ahp[i] = h;
          alp[i] = l;
        }
#pragma unroll 4
        for (int i = ct; i < Cfg::B_BYTES / 16; i += NCT) {
          const float4 x = bhp[i];
          float4 h, l;
          tf32_split(x.x, h.x, l.x);
          tf32_split(x.y, h.y, l.y);
          tf32_split(x.z, h.z, l.z);
          tf32_split(x.w, h.w, l.w);
          bhp[i] = h;
          blp[i] = l;
        }
      }
      fence_proxy_async();
      mbar_arrive(&conv[s]);
    }
    // epilogue: this split's partial tile (zeros if the split is empty)
    const int quad = warp & 3, half = (warp - 2) / 4;  // NCW / 4 warps share a quadrant's columns
    constexpr int CPW = BN / (NCW / 4);
    const int r = m0 + quad * 32 + lane;
    float* P = part + (int64_t)blockIdx.z * M * N;
    if (nk > 0) {
      mbar_wait(accum, 0);
      tc_fence_after();
    }
#pragma unroll 1
    for (int c0 = half * CPW; c0 < (half + 1) * CPW; c0 += 16) {
      float v[16];
#pragma unroll
      for (int j = 0; j < 16; ++j) v[j] = 0.f;
#pragma unroll 1
      for (int t = 0; t < Cfg::NACC; ++t) {
        // accumulator t holds k-blocks iff its sub-range is non-empty (nk < NACC leaves some unused)
        const int lo = (int)(((int64_t)t * nk + Cfg::NACC - 1) / Cfg::NACC);
        const int hi = (int)(((int64_t)(t + 1) * nk + Cfg::NACC - 1) / Cfg::NACC);
        if (lo >= hi) continue;
        float w[16];
        tmem_ld16(tmem + ((uint32_t)(quad * 32) << 16) + (uint32_t)(t * Cfg::ACC_COLS + c0), w);
#pragma unroll
        for (int j = 0; j < 16; ++j) v[j] += w[j];
      }
      if (r < M) {
#pragma unroll
        for (int j = 0; j < 16; ++j)
          if (n0 + c0 + j < N) P[(int64_t)r * N + n0 + c0 + j] = v[j];
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(Cfg::TMEM_COLS));
  }
}

// sum the per-N-tile attention partials in fixed tile order
__global__ void k_reduce_partials(int M, int tiles, const float* __restrict__ part, float* __restrict__ out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < M; i += (int64_t)gridDim.x * blockDim.x) {
    float s = 0.f;
    for (int t = 0; t < tiles; ++t) s += part[(int64_t)t * M + i];
    out[i] = s;
  }
}

// ======================================================================= SIMT fallback
// C = op(A) op(B), 64x64 tile / 256 threads, 4x4 per thread.  Deterministic.
template <bool TA, bool TB>
__global__ void __launch_bounds__(256) k_gemm_simt(int M, int N, int K, const float* __restrict__ A, int64_t lda,
                                                   const float* __restrict__ B, int64_t ldb, float* __restrict__ C,
                                                   int64_t ldc, const float* __restrict__ rs, int relu) {
  __shared__ float As[16][64 + 1];
  __shared__ float Bs[16][64 + 1];
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  const int m0 = blockIdx.x * 64, n0 = blockIdx.y * 64;
  float acc[4][4] = {};
  for (int k0 = 0; k0 < K; k0 += 16) {
    for (int i = threadIdx.x; i < 16 * 64; i += 256) {
      const int kk = i / 64, mm = i % 64;
      const int gm = m0 + mm, gk = k0 + kk;
      As[kk][mm] = (gm < M && gk < K) ? (TA ? A[(int64_t)gk * lda + gm] : A[(int64_t)gm * lda + gk]) : 0.f;
      const int gn = n0 + mm;
      Bs[kk][mm] = (gn < N && gk < K) ? (TB ? B[(int64_t)gn * ldb + gk] : B[(int64_t)gk * ldb + gn]) : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < 16; ++kk) {
      float a[4], b[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) a[i] = As[kk][ty * 4 + i];
#pragma unroll
      for (int j = 0; j < 4; ++j) b[j] = Bs[kk][tx * 4 + j];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int gm = m0 + ty * 4 + i;
    if (gm >= M) continue;
    const float s = rs ? rs[gm] : 1.f;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int gn = n0 + tx * 4 + j;
      if (gn < N) {
        float v = acc[i][j] * s;
        if (relu) v = fmaxf(v, 0.f);
        C[(int64_t)gm * ldc + gn] = v;
      }
    }
  }
}

// C[M x N] = Aᵀ B with A stored R x M, B stored R x N (R = reduction, e.g. nodes).
// Split over R into `splits` chunks; partials [splits][M][N] then fixed-order sum.
__global__ void __launch_bounds__(256) k_gemm_tn_part(int M, int N, int64_t R, int64_t chunk, const float* __restrict__ A,
                                                      int64_t lda, const float* __restrict__ B, int64_t ldb,
                                                      float* __restrict__ part) {
  __shared__ float As[32][64 + 1];
  __shared__ float Bs[32][64 + 1];
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  const int m0 = blockIdx.x * 64, n0 = blockIdx.y * 64;
  const int64_t r0 = blockIdx.z * chunk, r1 = min(R, r0 + chunk);
  float acc[4][4] = {};
  for (int64_t k0 = r0; k0 < r1; k0 += 32) {
    for (int i = threadIdx.x; i < 32 * 64; i += 256) {
      const int kk = i / 64, mm = i % 64;
      const int64_t gk = k0 + kk;
      As[kk][mm] = (m0 + mm < M && gk < r1) ? A[gk * lda + m0 + mm] : 0.f;
      Bs[kk][mm] = (n0 + mm < N && gk < r1) ? B[gk * ldb + n0 + mm] : 0.f;
    }
    __syncthreads();
#pragma unroll 8
    for (int kk = 0; kk < 32; ++kk) {
      float a[4], b[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) a[i] = As[kk][ty * 4 + i];
#pragma unroll
      for (int j = 0; j < 4; ++j) b[j] = Bs[kk][tx * 4 + j];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }
  float* P = part + (int64_t)blockIdx.z * M * N;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int gm = m0 + ty * 4 + i;
    if (gm >= M) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int gn = n0 + tx * 4 + j;
      if (gn < N) P[(int64_t)gm * N + gn] = acc[i][j];
    }
  }
}

__global__ void k_sum_splits(int64_t MN, int splits, const float* __restrict__ part, float* __restrict__ C, int M, int N,
                             int64_t ldc) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < MN; i += (int64_t)gridDim.x * blockDim.x) {
    double s = 0.0;  // hundreds of split partials at full size: the fixed-order sum in fp64
    for (int t = 0; t < splits; ++t) s += (double)part[(int64_t)t * MN + i];
    C[(i / N) * ldc + (i % N)] = (float)s;
  }
}

// ======================================================================= host side
static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (PFN_cuTensorMapEncodeTiled_v12000)p;
  });
  return fn;
}

static bool make_map(CUtensorMap* m, const void* base, uint64_t inner, uint64_t outer, uint64_t ld_elems,
                     uint32_t box_inner, uint32_t box_outer, CUtensorMapSwizzle swz = CU_TENSOR_MAP_SWIZZLE_128B) {
  auto enc = get_encode();
  if (!enc) return false;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {ld_elems * 4};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t es[2] = {1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<void*>(base), dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

static int pick_bn(int64_t N) {
  if (N <= 16) return 16;
  if (N <= 32) return 32;
  if (N <= 48) return 48;
  if (N <= 64) return 64;
  if (N <= 96) return 96;
  return 128;  // wider N runs as consecutive 128-column tiles of the same M tile (A re-read hits L2)
}

static bool tc_eligible(int64_t M, int64_t N, int64_t K, const float* A, int64_t lda, uint32_t flags) {
  if (flags & GRANII_GEMM_TRANS_A) return false;
  if (getenv("GRANII_GEMM_SIMT")) return false;
  if (lda % 4 != 0 || ((uintptr_t)A & 15)) return false;
  if (M <= 0 || N <= 0 || K <= 0) return false;
  if (M > INT32_MAX || K > INT32_MAX) return false;
  return true;
}

// Aᵀ·B plan: BN multiple of 32 (TMA boxes of 32), split the reduction so the grid
// fills the 148 SMs (one CTA per SM: ~190 KB smem), >= 8 k-blocks per split.
struct TnPlan {
  int bn, bk;
  int64_t mt, nt, total_kb, kb_per, splits;
};
// 16-row k-blocks (4 stages) when several output tiles share the grid (Reddit dW 602 x 256: 5 tiles,
// 0.765 -> 0.695 ms per step; 602 x 1024: 2.83 -> 2.67); 32-row blocks for one or two tiles over many
// splits (products GAT dW 100 x 256 and 256 x 47: 1.53 -> 1.68 ms with 16).  GRANII_TN_BK overrides.
static int tn_bk(int64_t tiles) {
  if (const char* e = getenv("GRANII_TN_BK")) return atoi(e) == 32 ? 32 : 16;
  return tiles >= 4 ? 16 : 32;
}
// 8 converter / epilogue warps (B200: Reddit dW 0.677 -> 0.662 ms per step, products GAT 1.54 -> 1.52;
// GRANII_TN_NCW=4 for the former 4)
static int tn_ncw() {
  const char* e = getenv("GRANII_TN_NCW");
  return e && atoi(e) == 4 ? 4 : 8;
}
// rows per split (GRANII_TN_SPLIT_ROWS, 0 = no cap): the error of the tensor-core accumulation grows
// linearly with the number of k-blocks summed into one TMEM accumulator (tools/gemm_tn_err.py, B200:
// normwise 5.8e-4 for Reddit-shaped 602 x 256 over 2.45 M rows with 82 k rows per split; 2.8e-5 with
// 4096), so the split count follows the reduction length -- and the error stays bounded at any graph
// size.  The splits are then rounded so that tiles x splits fills whole waves of 148 CTAs.
static int64_t tn_split_rows() {
  const char* e = getenv("GRANII_TN_SPLIT_ROWS");
  return e ? atoll(e) : 4096;
}
static TnPlan tn_plan(int64_t M, int64_t N, int64_t R) {
  TnPlan p;
  p.bn = N <= 32 ? 32 : N <= 64 ? 64 : N <= 128 ? 128 : 256;
  // (a 128-wide N tile for N = 256 -- three pipeline stages instead of two -- measured 0.78 -> 0.95 ms on 602x256)
  p.mt = ceil_div(M, TC_BM);
  p.nt = ceil_div(N, p.bn);
  p.bk = tn_bk(p.mt * p.nt);
  p.total_kb = ceil_div(R, p.bk);
  int64_t splits = std::max<int64_t>(1, ceil_div(148, p.mt * p.nt));
  splits = std::max<int64_t>(1, std::min<int64_t>(splits, p.total_kb / (8 * TC_BK / p.bk)));
  if (const int64_t cap = tn_split_rows()) {
    const int64_t tiles = p.mt * p.nt;
    splits = std::max<int64_t>(splits, ceil_div(R, std::max<int64_t>(cap, p.bk)));
    const int64_t waves = ceil_div(tiles * splits, 148);
    splits = std::max<int64_t>(splits, std::min<int64_t>(waves * 148 / tiles, p.total_kb));
  }
  p.kb_per = ceil_div(p.total_kb, splits);
  p.splits = ceil_div(p.total_kb, p.kb_per);
  return p;
}
static int64_t simt_tn_splits(int64_t R) { return std::max<int64_t>(1, std::min<int64_t>(64, ceil_div(R, 4096))); }

size_t gemm_workspace(int64_t M, int64_t N, int64_t K, uint32_t flags) {
  size_t ws = 0;
  if (flags & GRANII_GEMM_TRANS_A) {
    // split-K partials (tensor-core or SIMT plan, whichever is larger)
    const int64_t splits = std::max(tn_plan(M, N, K).splits, simt_tn_splits(K));
    return (size_t)splits * M * N * 4 + 256;
  }
  const int bn = pick_bn(N);
  const int64_t Npad = round_up(N, bn), Kpad = round_up(K, TC_BK);
  ws += (size_t)2 * Npad * Kpad * 4 + 1024;
  const int64_t tiles = ceil_div(N, bn);
  ws += (size_t)2 * 2 * tiles * M * 4 + 256;  // attention partials: 2 per N tile (epilogue halves)
  return ws;
}

template <int BN>
static granii_status launch_tc_bn(int M, int N, int K, const CUtensorMap& ta, const CUtensorMap& tbh,
                                  const CUtensorMap& tbl, const TcEpi& ep, cudaStream_t st) {
  using Cfg = TcCfg<BN>;
  static bool attr_set = false;
  if (!attr_set) {
    GR_CUDA(cudaFuncSetAttribute(k_gemm_tc<BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM));
    attr_set = true;
  }
  DevInfo di;
  GR_TRY(dev_info(&di));
  const int64_t tiles = ceil_div(M, TC_BM);  // persistent over M tiles; N tiles inside
  const unsigned grid = (unsigned)std::min<int64_t>(tiles, di.sms);  // persistent: one CTA per SM
  k_gemm_tc<BN><<<grid, TC_THREADS, Cfg::SMEM, st>>>(ta, tbh, tbl, M, N, K, ep);
  GR_CHECK_LAUNCH();
  return GRANII_OK;
}

granii_status launch_gemm(int64_t M, int64_t N, int64_t K, const float* A, int64_t lda, const float* B,
                          int64_t ldb, float* C, int64_t ldc, const granii_gemm_epilogue* epi, uint32_t flags,
                          void* ws, size_t ws_bytes, cudaStream_t st) {
  if (M == 0 || N == 0) return GRANII_OK;
  const bool relu = flags & GRANII_GEMM_RELU;
  const bool store = !(flags & GRANII_GEMM_NO_STORE);
  const bool tb = flags & GRANII_GEMM_TRANS_B;
  const float* rs = epi ? epi->row_scale : nullptr;
  const bool att = epi && (epi->att_l || epi->att_r);
  if (ws_bytes < gemm_workspace(M, N, K, flags)) return fail(GRANII_ERR_INVALID_ARG, "gemm workspace too small");
  DevInfo di;
  GR_TRY(dev_info(&di));

  // algorithmic bytes: A and B read once, C written once (fp32); flops 2MNK
  const double gbytes = 4.0 * ((double)M * K + (double)K * N + (store ? (double)M * N : 0.0));
  const double gflops = 2.0 * (double)M * N * K;
  if (flags & GRANII_GEMM_TRANS_A) {
    if (att || rs || relu || tb) return fail(GRANII_ERR_UNSUPPORTED, "TRANS_A supports plain C = A^T B only");
    // here K is the reduction (rows), A stored K x M, B stored K x N
    const bool tc = !getenv("GRANII_GEMM_SIMT") && lda % 4 == 0 && ldb % 4 == 0 && ((uintptr_t)A & 15) == 0 &&
                    ((uintptr_t)B & 15) == 0 && M <= INT32_MAX && N <= INT32_MAX;
    if (tc) {
      const TnPlan p = tn_plan(M, N, K);
      ProfScope ps("gemm_tn_tc", st, gbytes, gflops, 2);
      float* part = (float*)ws;
      // MN-major tf32 operands need the 128B swizzle with 32B atoms (descriptor layout type 1)
      // debug override GRANII_TN_DESC=lbo,sbo,kstep,major,layout,tma_swizzle
      // LBO = the byte stride between 32-wide MN atoms = one TMA box of 32 x bk fp32
      uint32_t dlbo = 32 * p.bk * 4, dsbo = 512, dkstep = 1024, dmaj = 3, dlay = 1, dswz = 4;
      if (const char* e = getenv("GRANII_TN_DESC"))
        sscanf(e, "%u,%u,%u,%u,%u,%u", &dlbo, &dsbo, &dkstep, &dmaj, &dlay, &dswz);
      dkstep = (dkstep & 0xFFFF) | (dmaj << 16);
      dlbo = (dlbo & 0x0FFFFFFFu) | (dlay << 28);
      CUtensorMap ta, tb;
      if (!make_map(&ta, A, (uint64_t)M, (uint64_t)K, (uint64_t)lda, 32, p.bk, (CUtensorMapSwizzle)dswz) ||
          !make_map(&tb, B, (uint64_t)N, (uint64_t)K, (uint64_t)ldb, 32, p.bk, (CUtensorMapSwizzle)dswz))
        return fail(GRANII_ERR_CUDA, "cuTensorMapEncodeTiled failed (TN)");
      dim3 grid((unsigned)p.mt, (unsigned)p.nt, (unsigned)p.splits);
      const char* rh = getenv("GRANII_TN_RAWHI");
      const int raw_hi = rh ? (rh[0] != '0') : 1;
#define GR_TN3(BN, BK, NCW)                                                                             \
  do {                                                                                                  \
    static bool set_ = false;                                                                           \
    if (!set_) {                                                                                        \
      GR_CUDA(cudaFuncSetAttribute(k_gemm_tn_tc<BN, BK, NCW>, cudaFuncAttributeMaxDynamicSharedMemorySize, \
                                   TnCfg<BN, BK>::SMEM));                                               \
      set_ = true;                                                                                      \
    }                                                                                                   \
    k_gemm_tn_tc<BN, BK, NCW><<<grid, 64 + 32 * NCW, TnCfg<BN, BK>::SMEM, st>>>(                         \
        ta, tb, (int)M, (int)N, (int)p.kb_per, (int)p.total_kb, part, dlbo, dsbo, dkstep, raw_hi);       \
  } while (0)
#define GR_TN2(BN, BK)                     \
  do {                                     \
    if (tn_ncw() == 8) GR_TN3(BN, BK, 8);  \
    else GR_TN3(BN, BK, 4);                \
  } while (0)
#define GR_TN(BN)                   \
  do {                              \
    if (p.bk == 16) GR_TN2(BN, 16); \
    else GR_TN2(BN, 32);            \
  } while (0)
      switch (p.bn) {
        case 32: GR_TN(32); break;
        case 64: GR_TN(64); break;
        case 128: GR_TN(128); break;
        default: GR_TN(256); break;
      }
#undef GR_TN
#undef GR_TN2
#undef GR_TN3
      GR_CHECK_LAUNCH();
      const int64_t MN = M * N;
      k_sum_splits<<<(unsigned)std::min<int64_t>(ceil_div(MN, 256), 4096), 256, 0, st>>>(MN, (int)p.splits, part, C,
                                                                                        (int)M, (int)N, ldc);
      GR_CHECK_LAUNCH();
      return GRANII_OK;
    }
    ProfScope ps("gemm_tn", st, gbytes, gflops, 2);
    const int64_t splits = simt_tn_splits(K);
    const int64_t chunk = round_up(ceil_div(K, splits), 32);
    float* part = (float*)ws;
    dim3 grid((unsigned)ceil_div(M, 64), (unsigned)ceil_div(N, 64), (unsigned)splits);
    k_gemm_tn_part<<<grid, 256, 0, st>>>((int)M, (int)N, K, chunk, A, lda, B, ldb, part);
    GR_CHECK_LAUNCH();
    const int64_t MN = M * N;
    k_sum_splits<<<(unsigned)std::min<int64_t>(ceil_div(MN, 256), 4096), 256, 0, st>>>(MN, (int)splits, part, C,
                                                                                      (int)M, (int)N, ldc);
    GR_CHECK_LAUNCH();
    return GRANII_OK;
  }

  if (!tc_eligible(M, N, K, A, lda, flags)) {
    if (att) return fail(GRANII_ERR_UNSUPPORTED, "attention epilogue needs the tensor-core path (lda % 4 == 0)");
    dim3 grid((unsigned)ceil_div(M, 64), (unsigned)ceil_div(N, 64));
    if (!store) return GRANII_OK;
    ProfScope ps("gemm_simt", st, gbytes, gflops, 1);
    if (tb) k_gemm_simt<false, true><<<grid, 256, 0, st>>>((int)M, (int)N, (int)K, A, lda, B, ldb, C, ldc, rs, relu);
    else k_gemm_simt<false, false><<<grid, 256, 0, st>>>((int)M, (int)N, (int)K, A, lda, B, ldb, C, ldc, rs, relu);
    GR_CHECK_LAUNCH();
    return GRANII_OK;
  }

  const int bn = pick_bn(N);
  const int64_t Npad = round_up(N, bn), Kpad = round_up(K, TC_BK);
  ProfScope ps("gemm_tc", st, gbytes, gflops, 2);
  uint8_t* w = (uint8_t*)(((uintptr_t)ws + 1023) & ~(uintptr_t)1023);
  float* bhi = (float*)w;
  float* blo = bhi + Npad * Kpad;
  float* part_l = blo + Npad * Kpad;
  const int64_t tiles = ceil_div(N, bn);
  float* part_r = part_l + 2 * tiles * M;
  k_prep_b<<<(unsigned)std::min<int64_t>(ceil_div(Npad * Kpad, 256), 4096), 256, 0, st>>>(
      (int)K, (int)N, B, ldb, tb ? 1 : 0, (int)Kpad, (int)Npad, bhi, blo);
  GR_CHECK_LAUNCH();

  CUtensorMap ta, tbh, tbl;
  if (!make_map(&ta, A, (uint64_t)K, (uint64_t)M, (uint64_t)lda, TC_BK, TC_BM) ||
      !make_map(&tbh, bhi, (uint64_t)Kpad, (uint64_t)Npad, (uint64_t)Kpad, TC_BK, bn) ||
      !make_map(&tbl, blo, (uint64_t)Kpad, (uint64_t)Npad, (uint64_t)Kpad, TC_BK, bn))
    return fail(GRANII_ERR_CUDA, "cuTensorMapEncodeTiled failed");

  TcEpi ep{C, ldc, rs, epi ? epi->att_l : nullptr, epi ? epi->att_r : nullptr, nullptr, nullptr, relu ? 1 : 0,
           store ? 1 : 0};
  if (epi && epi->att_l && epi->out_l) ep.out_l = part_l;
  if (epi && epi->att_r && epi->out_r) ep.out_r = part_r;
  switch (bn) {
    case 16: GR_TRY(launch_tc_bn<16>((int)M, (int)N, (int)K, ta, tbh, tbl, ep, st)); break;
    case 32: GR_TRY(launch_tc_bn<32>((int)M, (int)N, (int)K, ta, tbh, tbl, ep, st)); break;
    case 48: GR_TRY(launch_tc_bn<48>((int)M, (int)N, (int)K, ta, tbh, tbl, ep, st)); break;
    case 64: GR_TRY(launch_tc_bn<64>((int)M, (int)N, (int)K, ta, tbh, tbl, ep, st)); break;
    case 96: GR_TRY(launch_tc_bn<96>((int)M, (int)N, (int)K, ta, tbh, tbl, ep, st)); break;
    default: GR_TRY(launch_tc_bn<128>((int)M, (int)N, (int)K, ta, tbh, tbl, ep, st)); break;
  }
  if (ep.out_l || ep.out_r) {  // fixed-order sum of the per-(N tile, half) GEMV partials
    ps.add_launches((ep.out_l ? 1 : 0) + (ep.out_r ? 1 : 0));
    const unsigned b = (unsigned)std::min<int64_t>(ceil_div(M, 256), 4096);
    if (ep.out_l) k_reduce_partials<<<b, 256, 0, st>>>((int)M, (int)(2 * tiles), part_l, epi->out_l);
    if (ep.out_r) k_reduce_partials<<<b, 256, 0, st>>>((int)M, (int)(2 * tiles), part_r, epi->out_r);
    GR_CHECK_LAUNCH();
  }
  return GRANII_OK;
}

}  // namespace granii
