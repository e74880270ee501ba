// layer.cu -- one GNN layer under an explicit composition (§III).
//
// GCN (Eq. 2 L115 / Eq. 3), GAT (Eq. 4-6).  Each composition
// is the paper's primitive sequence with the element-wise work fused into the
// primitive that produces or consumes it:
//   PRE_AGG : SDDMM(dinv,dinv)->Ñ ; SpMM_w(Ñ, H)[K1] ; GEMM(·W)+σ
//   PRE_UPD : SDDMM ; GEMM(H W) ; SpMM_w(Ñ, ·)[K2]+σ
//   DYN_AGG : SpMM_u(Ã, H) with the pre-scale D̃^-½ in the gather and the
//             post-scale in the epilogue [K1] ; GEMM(·W)+σ
//   DYN_UPD : GEMM(H W) with the row-broadcast D̃^-½ in its epilogue ;
//             SpMM_u(Ã, ·)[K2] with D̃^-½ in its epilogue +σ
//   GAT_REUSE  : GEMM Θ = H W (+ el = Θ a_l, er = Θ a_r in the epilogue) ;
//                SDDMM(el, er) + LeakyReLU + row softmax -> α ; SpMM_w(α, Θ)[K2]+σ
//   GAT_RECOMP : GEMM (el, er only; Θ is never written) ; SDDMM -> α ;
//                SpMM_w(α, H)[K1] ; GEMM(·W)+σ  (the extra GEMM of L135)
// Multi-GPU (comm != NULL): rows are partitioned; the dense operand of every
// SpMM / SDDMM is produced straight into this rank's slot of a padded gather
// buffer and all-gathered in place with NCCL before the sparse step.
#include <algorithm>
#include <cmath>

#include "internal.h"

namespace granii {

struct Bump {
  uint8_t* base;
  size_t off = 0;
  explicit Bump(void* b) : base((uint8_t*)b) {}
  float* take(size_t floats) {
    off = (size_t)round_up((int64_t)off, 1024);
    float* p = base ? (float*)(base + off) : nullptr;
    off += floats * sizeof(float);
    return p;
  }
  void* take_bytes(size_t bytes) {
    off = (size_t)round_up((int64_t)off, 1024);
    void* p = base ? base + off : nullptr;
    off += bytes;
    return p;
  }
};

// leading dimension of internal dense buffers: 16-byte rows (TMA / float4), and whole
// 32-byte L2 sectors once rows are >= 8 floats (each gathered row touches the fewest sectors)
static inline int64_t ld4(int64_t k) { return k >= 8 ? round_up(k, 8) : round_up(k, 4); }

struct Ctx {
  const granii_graph_s* g;
  granii_comm_s* comm;
  cudaStream_t st;
  bool dist() const { return comm && comm->world > 1; }
};

// dense operand of a sparse step: in the gather buffer (dist) or plain local rows.
struct GatherBuf {
  float* all = nullptr;  // n_cols x ld
  float* mine = nullptr; // this rank's slot (n_rows x ld)
  int64_t ld = 0;
};

static GatherBuf gather_buf(Bump& b, const Ctx& c, int64_t K) {
  GatherBuf gb;
  gb.ld = ld4(K);
  if (c.dist()) {
    gb.all = b.take((size_t)c.g->n_cols * gb.ld);
    gb.mine = gb.all ? gb.all + (int64_t)c.g->rank * c.g->max_rows * gb.ld : nullptr;
  } else {
    gb.all = b.take((size_t)std::max<int64_t>(c.g->n_rows, 1) * gb.ld);
    gb.mine = gb.all;
  }
  return gb;
}

static granii_status allgather(const Ctx& c, GatherBuf& gb) {
  if (!c.dist()) return GRANII_OK;
  const size_t count = (size_t)c.g->max_rows * gb.ld;
  return comm_allgather(c.comm, gb.mine, gb.all, count, c.st);
}

// Aggregation Y = spmm(X) over a dense operand whose own rows are already in gb.mine.
// One GPU: a plain SpMM.  Several GPUs (N1): instead of all-gather -> SpMM, the blocks are
// broadcast one source rank at a time (rank order) on the communicator's side stream while the
// SpMM runs in P phases on the caller's stream: this rank's block first (nothing to wait for),
// then the other G-1 blocks in P-1 chunks, each as soon as its last broadcast has landed -- the
// transfer overlaps the aggregation.  Each row's entries owned by one rank are a contiguous run
// (sorted columns, monotone gather layout: graph owner_off), so a phase is a plain SpMM over
// sub-ranges that continues from the previous phase's raw partial; the epilogue runs in the last
// phase.  P comes from the cost model (select.cpp agg_schedule; P = 1 = all-gather then one
// SpMM); the phase order is fixed, so results are run-to-run bitwise reproducible.
// GRANII_COMM_OVERLAP=0 forces P = 1, GRANII_COMM_PHASES=P forces P.
static bool overlap_enabled() {
  const char* e = getenv("GRANII_COMM_OVERLAP");
  return !(e && e[0] == '0');
}

bool gat_fused_enabled() {
  const char* e = getenv("GRANII_GAT_FUSED");
  return !(e && e[0] == '0');
}

static granii_status gathered_spmm(const Ctx& c, GatherBuf& gb, const float* vals, int64_t K, float* Y, int64_t ldy,
                                   const float* rs, const float* cs, bool relu, const float* B = nullptr,
                                   int64_t ldb = 0, float beta = 0.f) {
  const granii_graph_s* g = c.g;
  // K % 4 != 0: the float4 gathers read the row's last vector whole, padding columns [K, K4) included
  // (they only ever reach Y's padding); nothing writes them, so zero this rank's before anyone reads
  if (K % 4 != 0 && g->n_rows > 0)
    GR_CUDA(cudaMemset2DAsync(gb.mine + K, (size_t)gb.ld * sizeof(float), 0, (size_t)(round_up(K, 4) - K) * sizeof(float),
                              (size_t)g->n_rows, c.st));
  if (!c.dist()) return launch_spmm_ex(g, vals, gb.all, gb.ld, K, Y, ldy, rs, cs, relu, B, ldb, beta, c.st);
  const int P = overlap_enabled() && g->owner_off ? comm_phases(g, K, vals != nullptr, cs != nullptr) : 1;
  if (P <= 1) {
    GR_TRY(allgather(c, gb));
    return launch_spmm_ex(g, vals, gb.all, gb.ld, K, Y, ldy, rs, cs, relu, B, ldb, beta, c.st);
  }
  cudaStream_t side;
  cudaEvent_t* ev;
  GR_TRY(comm_side(c.comm, &side, &ev));
  const int G = g->world, me = g->rank;
  const size_t count = (size_t)g->max_rows * gb.ld;
  GR_CUDA(cudaEventRecord(ev[G], c.st));  // own block produced
  GR_CUDA(cudaStreamWaitEvent(side, ev[G], 0));
  for (int p = 0; p < G; ++p) {  // every rank issues the broadcasts in the same order
    GR_TRY(comm_bcast_block(c.comm, gb.all, count, p, side));
    GR_CUDA(cudaEventRecord(ev[p], side));
  }
  float* partial = nullptr;
  if (g->n_seg > 0)
    GR_CUDA(cudaMallocAsync((void**)&partial, (size_t)g->n_seg * round_up(K, 4) * sizeof(float), c.st));
  SpmmPhase own{me, me + 1, -1, 1, 0, partial};
  GR_TRY(launch_spmm_phase(g, vals, gb.all, gb.ld, K, Y, ldy, rs, cs, relu, B, ldb, beta, own, c.st));
  // the other blocks in rank order ("other" index k -> rank k + (k >= me)), P-1 chunks
  for (int q = 0; q < P - 1; ++q) {
    const int k0 = (G - 1) * q / (P - 1), k1 = (G - 1) * (q + 1) / (P - 1);
    const int r0 = k0 + (k0 >= me), rl = (k1 - 1) + (k1 - 1 >= me);  // first and last rank
    GR_CUDA(cudaStreamWaitEvent(c.st, ev[rl], 0));
    SpmmPhase ph{r0, rl + 1, (r0 < me && me < rl) ? me : -1, 0, q == P - 2, partial};
    GR_TRY(launch_spmm_phase(g, vals, gb.all, gb.ld, K, Y, ldy, rs, cs, relu, B, ldb, beta, ph, c.st));
  }
  GR_CUDA(cudaStreamWaitEvent(c.st, ev[G - 1], 0));  // the side stream is idle (own send included)
  if (partial) GR_CUDA(cudaFreeAsync(partial, c.st));
  return GRANII_OK;
}

// scalar per-row vector (er) gather: one float per row
static float* vec_buf(Bump& b, const Ctx& c) {
  return b.take((size_t)(c.dist() ? c.g->n_cols : std::max<int64_t>(c.g->n_rows, 1)));
}

static granii_status gemm_ws(Bump& b, int64_t M, int64_t N, int64_t K, uint32_t flags, void** p, size_t* n) {
  *n = gemm_workspace(M, N, K, flags);
  *p = b.take_bytes(*n);
  return GRANII_OK;
}

// saved state of a GAT layer: [Θ (REUSE, R x ld4(K2)) | T = α H (RECOMP, R x ld4(K1))][el: R][er: R]
struct GatSaved {
  int64_t ldz, el, er;
  size_t floats;
};
static GatSaved gat_saved_layout(int64_t R, granii_composition comp, int64_t K1, int64_t K2) {
  GatSaved s;
  s.ldz = ld4(comp == GRANII_GAT_REUSE ? K2 : K1);
  s.el = R * s.ldz;
  s.er = s.el + round_up(R, 4);
  s.floats = (size_t)(s.er + round_up(R, 4));
  return s;
}

// ---------------------------------------------------------------- SGC / TAGCN / GIN (N3, reading R23)
// Forward only.  Shared pieces: one hop of S = D̃^-½ Ã D̃^-½ is a weighted SpMM over Ñ (PRE)
// or an unweighted SpMM with both scalings fused (DYN); multi-hop chains ping-pong between two
// gather buffers (all-gathered between hops on several GPUs); the TAGCN Horner step and GIN's
// ε self term are the SpMM's fused dense addend.
static granii_status ext_forward_impl(const Ctx& c, granii_model m, granii_composition comp,
                                      const granii_layer_args* a, float* out, int64_t ldo, void* ws_base,
                                      size_t* ws_size) {
  const granii_graph_s* g = c.g;
  const bool run = ws_base != nullptr;
  Bump b(ws_base);
  const int64_t R = g->n_rows, Rr = std::max<int64_t>(R, 1), K1 = a->K1, K2 = a->K2;
  const bool relu = a->act == GRANII_ACT_RELU;
  const cudaStream_t st = c.st;
  const int base = m == GRANII_SGC ? GRANII_SGC_PRE_AGG : m == GRANII_TAGCN ? GRANII_TAGCN_PRE_AGG : GRANII_GIN_PRE_AGG;
  const int v = (int)comp - base;
  const bool dyn = v >= 2, upd = (v & 1) != 0;
  const int hops = a->hops;

  // SGC DYN: hop inputs are kept pre-scaled by D̃^-½ (the first one by a row-broadcast pass or
  // the GEMM epilogue, the next ones by fusing D̃^-1 = post-scale x next pre-scale into the hop's
  // epilogue) instead of gathering dinv[c] in every hop and K slice -- when that moves fewer
  // bytes (dyn_prescale)
  DevInfo di;
  if (dev_info(&di) != GRANII_OK) di = DevInfo();
  const bool pre = m == GRANII_SGC && dyn && hops > 0 &&
                   dyn_prescale((double)g->local_nnz, (double)R, g->avg_deg(), (double)g->n_cols, upd ? K2 : K1,
                                di.l2_bytes);
  // TAGCN DYN aggregate-first: the same trade -- every hop's input is D̃^-½ X_j from a row-broadcast
  // pass (X_j itself is kept for the concatenated GEMM), the hop SpMM applies only D̃^-½ on rows
  const bool pre_t = m == GRANII_TAGCN && dyn && !upd && hops > 0 &&
                     dyn_prescale((double)g->local_nnz, (double)R, g->avg_deg(), (double)g->n_cols, K1, di.l2_bytes);
  // H: aligned own rows, and (aggregate-first) its gathered copy
  const float* H = a->H;
  int64_t ldh = a->ldh;
  const bool h_aligned = (ldh % 4 == 0) && (((uintptr_t)H & 15) == 0);
  GatherBuf hg;
  const bool h_gather = c.dist() && !upd;
  const bool h_scale = (pre || pre_t) && !upd;
  float* pscaled = nullptr;  // one GPU, TAGCN pre_t: the pre-scaled hop input, rewritten after every hop
  if (h_gather) {
    hg = gather_buf(b, c, K1);
    if (run) {
      if (h_scale) GR_TRY(launch_scale_mask(R, K1, nullptr, 0, a->H, a->ldh, g->dinv_rows, hg.mine, hg.ld, st));
      else GR_TRY(launch_copy_rows(R, K1, a->H, a->ldh, hg.mine, hg.ld, st));
      GR_TRY(allgather(c, hg));
    }
    H = hg.mine;
    ldh = hg.ld;
  } else if (h_scale) {
    float* hp = b.take((size_t)Rr * ld4(K1));
    if (run) GR_TRY(launch_scale_mask(R, K1, nullptr, 0, a->H, a->ldh, g->dinv_rows, hp, ld4(K1), st));
    H = hp;
    ldh = ld4(K1);
    pscaled = hp;
  } else if (!h_aligned) {
    float* hp = b.take((size_t)Rr * ld4(K1));
    if (run) GR_TRY(launch_copy_rows(R, K1, a->H, a->ldh, hp, ld4(K1), st));
    H = hp;
    ldh = ld4(K1);
  }
  const float* H_all = h_gather ? hg.all : H;

  // sparse values of the PRE compositions (recomputed per call, stateless as GCN's Ñ, R13)
  float* vals = nullptr;
  if (!dyn) vals = b.take((size_t)std::max<int64_t>(g->local_nnz, 1));
  if (run && !dyn) {
    if (m == GRANII_GIN) GR_TRY(launch_gin_vals(g, a->eps, vals, st));
    else GR_TRY(launch_sddmm(g, GRANII_SDDMM_DOT, g->dinv_rows, 1, g->dinv_cols, 1, 1, 1.f, vals, st));
  }
  // one hop Y = S X (+ beta B) (+ ReLU); X in the column-id space
  auto hop = [&](const float* X, int64_t ldx, int64_t K, float* Y, int64_t ldy, bool rl, const float* B, int64_t ldb,
                 float beta) -> granii_status {
    if (!dyn) return launch_spmm_ex(g, vals, X, ldx, K, Y, ldy, nullptr, nullptr, rl, B, ldb, beta, st);
    return launch_spmm_ex(g, nullptr, X, ldx, K, Y, ldy, g->dinv_rows, g->dinv_cols, rl, B, ldb, beta, st);
  };
  // SGC hop: with pre-scaled inputs the row scale is D̃^-1 between hops, D̃^-½ after the last
  auto sgc_hop = [&](const float* X, int64_t ldx, int64_t K, float* Y, int64_t ldy, bool rl,
                     bool last) -> granii_status {
    if (!pre) return hop(X, ldx, K, Y, ldy, rl, nullptr, 0, 0.f);
    return launch_spmm_ex(g, nullptr, X, ldx, K, Y, ldy, last ? g->dinv_rows : g->dinv2_rows, nullptr, rl, nullptr,
                          0, 0.f, st);
  };

  if (m == GRANII_SGC) {
    const int64_t K = upd ? K2 : K1;
    GatherBuf pb[2] = {gather_buf(b, c, K), gather_buf(b, c, K)};
    float* T = upd ? nullptr : b.take((size_t)Rr * ld4(K1));  // S^k H (own rows) before the GEMM
    void* gw;
    size_t gn;
    gemm_ws(b, R, K2, K1, relu ? GRANII_GEMM_RELU : 0, &gw, &gn);
    if (run) {
      const float* X = nullptr;
      int64_t ldx = 0;
      if (upd) {  // P = H W, then the hops at K2
        if (hops == 0) {
          GR_TRY(launch_gemm(R, K2, K1, H, ldh, a->W, K2, out, ldo, nullptr, relu ? GRANII_GEMM_RELU : 0, gw, gn, st));
        } else {
          granii_gemm_epilogue ep{pre ? g->dinv_rows : nullptr, nullptr, nullptr, nullptr, nullptr};
          GR_TRY(launch_gemm(R, K2, K1, H, ldh, a->W, K2, pb[0].mine, pb[0].ld, &ep, 0, gw, gn, st));
          GR_TRY(allgather(c, pb[0]));
          X = pb[0].all;
          ldx = pb[0].ld;
        }
      } else {
        X = H_all;
        ldx = ldh;
      }
      for (int h = 0; h < hops; ++h) {
        const bool last = h == hops - 1;
        GatherBuf& nb = pb[(h + 1) & 1];
        if (last && upd) {
          GR_TRY(sgc_hop(X, ldx, K, out, ldo, relu, true));
        } else if (last) {
          GR_TRY(sgc_hop(X, ldx, K, T, ld4(K1), false, true));
        } else {
          GR_TRY(sgc_hop(X, ldx, K, nb.mine, nb.ld, false, false));
          GR_TRY(allgather(c, nb));
          X = nb.all;
          ldx = nb.ld;
        }
      }
      if (!upd) {
        const float* A = hops == 0 ? H : T;
        const int64_t lda = hops == 0 ? ldh : ld4(K1);
        GR_TRY(launch_gemm(R, K2, K1, A, lda, a->W, K2, out, ldo, nullptr, relu ? GRANII_GEMM_RELU : 0, gw, gn, st));
      }
    }
  } else if (m == GRANII_TAGCN) {
    if (!upd) {
      // X_j = S^j H side by side (block stride Kb, 16-byte aligned), one GEMM with the stacked
      // W_j (padded to Kb rows per block: Wc)
      const int64_t Kb = round_up(K1, 4), ldc = ld4((hops + 1) * Kb);
      float* Xc = b.take((size_t)Rr * ldc);
      float* Wc = b.take((size_t)(hops + 1) * Kb * K2);
      GatherBuf pb[2] = {gather_buf(b, c, K1), gather_buf(b, c, K1)};
      void* gw;
      size_t gn;
      gemm_ws(b, R, K2, (hops + 1) * Kb, relu ? GRANII_GEMM_RELU : 0, &gw, &gn);
      if (run) {
        if (Kb != K1) {  // zero the padding columns / rows so the GEMM adds exact zeros
          GR_CUDA(cudaMemset2DAsync(Xc + K1, ldc * sizeof(float), 0, (Kb - K1) * sizeof(float), (size_t)R, st));
          for (int j = 1; j <= hops; ++j)
            GR_CUDA(cudaMemset2DAsync(Xc + j * Kb + K1, ldc * sizeof(float), 0, (Kb - K1) * sizeof(float),
                                      (size_t)R, st));
          GR_CUDA(cudaMemsetAsync(Wc, 0, sizeof(float) * (size_t)(hops + 1) * Kb * K2, st));
        }
        for (int j = 0; j <= hops; ++j)
          GR_CUDA(cudaMemcpyAsync(Wc + (int64_t)j * Kb * K2, a->W + (int64_t)j * K1 * K2,
                                  sizeof(float) * (size_t)K1 * K2, cudaMemcpyDeviceToDevice, st));
        GR_TRY(launch_copy_rows(R, K1, pre_t ? a->H : H, pre_t ? a->ldh : ldh, Xc, ldc, st));  // X_0 = H
        const float* X = H_all;
        int64_t ldx = ldh;
        for (int j = 1; j <= hops; ++j) {
          float* dst = Xc + (int64_t)(j)*Kb;
          if (pre_t) {  // X_j = D̃^-½ Ã (D̃^-½ X_{j-1}); then the next hop's pre-scaled input
            GR_TRY(launch_spmm_ex(g, nullptr, X, ldx, K1, dst, ldc, g->dinv_rows, nullptr, false, nullptr, 0, 0.f,
                                  st));
            if (j == hops) break;
            if (c.dist()) {
              GatherBuf& nb = pb[j & 1];
              GR_TRY(launch_scale_mask(R, K1, nullptr, 0, dst, ldc, g->dinv_rows, nb.mine, nb.ld, st));
              GR_TRY(allgather(c, nb));
              X = nb.all;
              ldx = nb.ld;
            } else {
              GR_TRY(launch_scale_mask(R, K1, nullptr, 0, dst, ldc, g->dinv_rows, pscaled, ld4(K1), st));
              X = pscaled;
              ldx = ld4(K1);
            }
            continue;
          }
          if (c.dist()) {
            GatherBuf& nb = pb[j & 1];
            GR_TRY(hop(X, ldx, K1, nb.mine, nb.ld, false, nullptr, 0, 0.f));
            GR_TRY(launch_copy_rows(R, K1, nb.mine, nb.ld, dst, ldc, st));
            if (j < hops) GR_TRY(allgather(c, nb));
            X = nb.all;
            ldx = nb.ld;
          } else {
            GR_TRY(hop(X, ldx, K1, dst, ldc, false, nullptr, 0, 0.f));
            X = dst;
            ldx = ldc;
          }
        }
        GR_TRY(launch_gemm(R, K2, (hops + 1) * Kb, Xc, ldc, Wc, K2, out, ldo, nullptr,
                           relu ? GRANII_GEMM_RELU : 0, gw, gn, st));
      }
    } else {
      // Horner: P = H [W_0 | ... | W_k] (one GEMM, blocks of stride Kb2), Z = P_k,
      // Z = S Z + P_j for j = k-1..0 (the addend fused in the SpMM epilogue)
      const int64_t Kb2 = round_up(K2, 4), NP = (hops + 1) * Kb2, ldp = ld4(NP);
      float* P = b.take((size_t)Rr * ldp);
      float* Wh = b.take((size_t)K1 * NP);
      GatherBuf pb[2] = {gather_buf(b, c, K2), gather_buf(b, c, K2)};
      void* gw;
      size_t gn;
      gemm_ws(b, R, NP, K1, 0, &gw, &gn);
      void* gw0;
      size_t gn0;
      gemm_ws(b, R, K2, K1, relu ? GRANII_GEMM_RELU : 0, &gw0, &gn0);
      if (run) {
        if (hops == 0) {
          GR_TRY(launch_gemm(R, K2, K1, H, ldh, a->W, K2, out, ldo, nullptr, relu ? GRANII_GEMM_RELU : 0, gw0, gn0,
                             st));
        } else {
          if (Kb2 != K2) GR_CUDA(cudaMemsetAsync(Wh, 0, sizeof(float) * (size_t)K1 * NP, st));
          for (int j = 0; j <= hops; ++j)  // W_j (K1 x K2) into columns [j Kb2, j Kb2 + K2) of Wh
            GR_CUDA(cudaMemcpy2DAsync(Wh + (int64_t)j * Kb2, NP * sizeof(float), a->W + (int64_t)j * K1 * K2,
                                      K2 * sizeof(float), K2 * sizeof(float), (size_t)K1, cudaMemcpyDeviceToDevice,
                                      st));
          GR_TRY(launch_gemm(R, NP, K1, H, ldh, Wh, NP, P, ldp, nullptr, 0, gw, gn, st));
          const float* X = P + (int64_t)hops * Kb2;
          int64_t ldx = ldp;
          if (c.dist()) {
            GR_TRY(launch_copy_rows(R, K2, X, ldp, pb[0].mine, pb[0].ld, st));
            GR_TRY(allgather(c, pb[0]));
            X = pb[0].all;
            ldx = pb[0].ld;
          }
          for (int j = hops - 1; j >= 0; --j) {
            const float* Bj = P + (int64_t)j * Kb2;
            if (j == 0) {
              GR_TRY(hop(X, ldx, K2, out, ldo, relu, Bj, ldp, 1.f));
            } else {
              GatherBuf& nb = pb[(hops - j) & 1];
              GR_TRY(hop(X, ldx, K2, nb.mine, nb.ld, false, Bj, ldp, 1.f));
              GR_TRY(allgather(c, nb));
              X = nb.all;
              ldx = nb.ld;
            }
          }
        }
      }
    }
  } else {  // GIN
    const int64_t Kh = a->Kh;
    GatherBuf pg;
    if (upd) pg = gather_buf(b, c, Kh);
    float* U = b.take((size_t)Rr * ld4(upd ? Kh : K1));
    float* V = upd ? nullptr : b.take((size_t)Rr * ld4(Kh));
    void* gw1;
    size_t gn1;
    gemm_ws(b, R, Kh, K1, GRANII_GEMM_RELU, &gw1, &gn1);
    void* gw2;
    size_t gn2;
    gemm_ws(b, R, K2, Kh, relu ? GRANII_GEMM_RELU : 0, &gw2, &gn2);
    if (run) {
      // agg(X) = Σ_{Ã} X_j + ε X_i: PRE folds ε into the diagonal values, DYN adds ε X_i in the epilogue
      if (!upd) {
        GR_TRY(launch_spmm_ex(g, vals, H_all, ldh, K1, U, ld4(K1), nullptr, nullptr, false, dyn ? H : nullptr, ldh,
                              a->eps, st));
        GR_TRY(launch_gemm(R, Kh, K1, U, ld4(K1), a->W, Kh, V, ld4(Kh), nullptr, GRANII_GEMM_RELU, gw1, gn1, st));
        GR_TRY(launch_gemm(R, K2, Kh, V, ld4(Kh), a->W2, K2, out, ldo, nullptr, relu ? GRANII_GEMM_RELU : 0, gw2, gn2,
                           st));
      } else {
        GR_TRY(launch_gemm(R, Kh, K1, H, ldh, a->W, Kh, pg.mine, pg.ld, nullptr, 0, gw1, gn1, st));
        GR_TRY(allgather(c, pg));
        GR_TRY(launch_spmm_ex(g, vals, pg.all, pg.ld, Kh, U, ld4(Kh), nullptr, nullptr, true, dyn ? pg.mine : nullptr,
                              pg.ld, a->eps, st));
        GR_TRY(launch_gemm(R, K2, Kh, U, ld4(Kh), a->W2, K2, out, ldo, nullptr, relu ? GRANII_GEMM_RELU : 0, gw2, gn2,
                           st));
      }
    }
  }
  if (ws_size) *ws_size = b.off + 1024;
  return GRANII_OK;
}

// ---------------------------------------------------------------- forward (plan + run)
// Running with base == nullptr only sizes the workspace (no launches).
static granii_status forward_impl(const Ctx& c, granii_model m, granii_composition comp, const granii_layer_args* a,
                                  float* out, int64_t ldo, float* saved, void* ws_base, size_t* ws_size,
                                  size_t* saved_floats) {
  const granii_graph_s* g = c.g;
  const bool run = ws_base != nullptr;
  Bump b(ws_base);
  const int64_t R = g->n_rows, K1 = a->K1, K2 = a->K2;
  const bool relu = a->act == GRANII_ACT_RELU;
  const cudaStream_t st = c.st;
  if (saved_floats) *saved_floats = 0;
  if (m == GRANII_SGC || m == GRANII_TAGCN || m == GRANII_GIN)
    return ext_forward_impl(c, m, comp, a, out, ldo, ws_base, ws_size);

  // H with a 16-byte row stride for the TMA GEMM path / vector gathers
  const float* H = a->H;
  int64_t ldh = a->ldh;
  const bool h_aligned = (ldh % 4 == 0) && (((uintptr_t)H & 15) == 0);
  float* hpad = nullptr;
  const bool agg_first_gather = c.dist() && (comp == GRANII_GCN_PRE_AGG || comp == GRANII_GCN_DYN_AGG ||
                                             comp == GRANII_GAT_RECOMP);
  // GCN DYN_AGG: the pre-scale D̃^-½ H as its own row-broadcast pass when that moves fewer bytes
  // than the gather-fused column scale (dyn_prescale; it rides on the gather-slot copy when
  // partitioned)
  DevInfo di;
  if (dev_info(&di) != GRANII_OK) di = DevInfo();
  const bool prescale = m == GRANII_GCN && comp == GRANII_GCN_DYN_AGG &&
                        dyn_prescale((double)g->local_nnz, (double)R, g->avg_deg(), (double)g->n_cols, K1, di.l2_bytes);
  GatherBuf hg;
  if (agg_first_gather) {
    hg = gather_buf(b, c, K1);  // H goes into the gather slot (aligned copy); gathered by the SpMM
    if (run && prescale) GR_TRY(launch_scale_mask(R, K1, nullptr, 0, H, ldh, g->dinv_rows, hg.mine, hg.ld, st));
    else if (run) GR_TRY(launch_copy_rows(R, K1, H, ldh, hg.mine, hg.ld, st));
    H = hg.mine;
    ldh = hg.ld;
  } else if (prescale) {
    hpad = b.take((size_t)std::max<int64_t>(R, 1) * ld4(K1));
    if (run) GR_TRY(launch_scale_mask(R, K1, nullptr, 0, a->H, a->ldh, g->dinv_rows, hpad, ld4(K1), st));
    H = hpad;
    ldh = ld4(K1);
  } else if (!h_aligned) {
    hpad = b.take((size_t)std::max<int64_t>(R, 1) * ld4(K1));
    if (run) GR_TRY(launch_copy_rows(R, K1, a->H, a->ldh, hpad, ld4(K1), st));
    H = hpad;
    ldh = ld4(K1);
  }
  // aggregation source (column-id space): the gather buffer, or this GPU's rows
  GatherBuf xg = agg_first_gather ? hg : GatherBuf{const_cast<float*>(H), const_cast<float*>(H), ldh};

  if (m == GRANII_GCN) {
    float* nval = nullptr;
    if (comp == GRANII_GCN_PRE_AGG || comp == GRANII_GCN_PRE_UPD) {
      nval = b.take((size_t)std::max<int64_t>(g->local_nnz, 1));
      if (run) GR_TRY(launch_sddmm(g, GRANII_SDDMM_DOT, g->dinv_rows, 1, g->dinv_cols, 1, 1, 1.f, nval, st));
    }
    switch (comp) {
      case GRANII_GCN_PRE_AGG:
      case GRANII_GCN_DYN_AGG: {
        // T = (Ñ H) or (D Ã D H), K1 wide; kept for the backward pass
        const int64_t ldt = ld4(K1);
        if (saved_floats) *saved_floats = (size_t)R * ldt;
        float* T = saved ? saved : b.take((size_t)std::max<int64_t>(R, 1) * ldt);
        void* gw;
        size_t gn;
        gemm_ws(b, R, K2, K1, relu ? GRANII_GEMM_RELU : 0, &gw, &gn);
        if (run) {
          if (comp == GRANII_GCN_PRE_AGG)
            GR_TRY(gathered_spmm(c, xg, nval, K1, T, ldt, nullptr, nullptr, false));
          else  // the gathered operand is D̃^-½ H already when pre-scaled
            GR_TRY(gathered_spmm(c, xg, nullptr, K1, T, ldt, g->dinv_rows, prescale ? nullptr : g->dinv_cols, false));
          GR_TRY(launch_gemm(R, K2, K1, T, ldt, a->W, K2, out, ldo, nullptr, relu ? GRANII_GEMM_RELU : 0, gw, gn, st));
        }
        break;
      }
      case GRANII_GCN_PRE_UPD:
      case GRANII_GCN_DYN_UPD: {
        GatherBuf tg = gather_buf(b, c, K2);
        void* gw;
        size_t gn;
        gemm_ws(b, R, K2, K1, 0, &gw, &gn);
        if (run) {
          granii_gemm_epilogue ep{comp == GRANII_GCN_DYN_UPD ? g->dinv_rows : nullptr, nullptr, nullptr, nullptr,
                                  nullptr};
          GR_TRY(launch_gemm(R, K2, K1, H, ldh, a->W, K2, tg.mine, tg.ld, &ep, 0, gw, gn, st));
          if (comp == GRANII_GCN_PRE_UPD)
            GR_TRY(gathered_spmm(c, tg, nval, K2, out, ldo, nullptr, nullptr, relu));
          else
            GR_TRY(gathered_spmm(c, tg, nullptr, K2, out, ldo, g->dinv_rows, nullptr, relu));
        }
        break;
      }
      default:
        return fail(GRANII_ERR_INVALID_ARG, "composition does not belong to GCN");
    }
  } else {  // GAT
    if (comp != GRANII_GAT_REUSE && comp != GRANII_GAT_RECOMP)
      return fail(GRANII_ERR_INVALID_ARG, "composition does not belong to GAT");
    const bool dot = a->attn == GRANII_ATTN_DOT;
    // additive attention on one GPU over a warp-per-row graph: the scores, the row softmax and the
    // aggregation are one fused SpMM (no SDDMM pass, no alpha array); GRANII_GAT_FUSED=0 disables
    // partitioned graphs: when the aggregation's schedule is a single all-gather (P = 1; the same
    // on every rank) the gathered operand feeds the fused SpMM; an overlapped (phased) schedule
    // keeps SDDMM -> phased SpMM
    const bool out_aligned = (ldo % 4 == 0) && (((uintptr_t)out & 15) == 0);  // REUSE aggregates into out
    const int64_t agg_k = comp == GRANII_GAT_REUSE ? K2 : K1;
    const int agg_p = c.dist() && overlap_enabled() && g->owner_off ? comm_phases(g, agg_k, true, false) : 1;
    const bool fused = !dot && agg_p <= 1 && spmm_att_supported(g) && gat_fused_enabled() &&
                       (comp == GRANII_GAT_RECOMP || out_aligned);
    float* alpha = fused ? nullptr : b.take((size_t)std::max<int64_t>(g->local_nnz, 1));
    const bool need_theta = comp == GRANII_GAT_REUSE || dot;
    // state kept for the backward (gat_saved_layout): Θ (REUSE) or T = α H (RECOMP), el, er
    const GatSaved sv = gat_saved_layout(R, comp, K1, K2);
    if (saved_floats) *saved_floats = sv.floats;
    GatherBuf th;
    if (need_theta) {
      if (saved && comp == GRANII_GAT_REUSE && !c.dist()) {
        th.ld = ld4(K2);
        th.all = th.mine = saved;  // Θ goes straight into the saved state
      } else {
        th = gather_buf(b, c, K2);
      }
    }
    float* el = nullptr;
    float* er_all = nullptr;
    if (!dot) {
      el = saved ? saved + sv.el : b.take((size_t)std::max<int64_t>(R, 1));
      er_all = (saved && !c.dist()) ? saved + sv.er : vec_buf(b, c);
    }
    void* gw;
    size_t gn;
    gemm_ws(b, R, K2, K1, 0, &gw, &gn);
    if (run) {
      float* er_mine = er_all ? (c.dist() ? er_all + (int64_t)g->rank * g->max_rows : er_all) : nullptr;
      granii_gemm_epilogue ep{nullptr, dot ? nullptr : a->a_l, dot ? nullptr : a->a_r, el, er_mine};
      uint32_t fl = need_theta ? 0u : GRANII_GEMM_NO_STORE;
      GR_TRY(launch_gemm(R, K2, K1, H, ldh, a->W, K2, need_theta ? th.mine : nullptr, need_theta ? th.ld : K2,
                         &ep, fl, gw, gn, st));
      if (saved && c.dist()) {  // keep this rank's Θ rows and er for the backward
        if (comp == GRANII_GAT_REUSE)
          GR_CUDA(cudaMemcpyAsync(saved, th.mine, sizeof(float) * (size_t)R * th.ld, cudaMemcpyDeviceToDevice, st));
        if (!dot)
          GR_CUDA(cudaMemcpyAsync(saved + sv.er, er_mine, sizeof(float) * (size_t)R, cudaMemcpyDeviceToDevice, st));
      }
      if (dot) GR_TRY(allgather(c, th));  // the dot scores gather Θ; the additive REUSE SpMM gathers it itself
      if (!dot) {
        if (c.dist()) {
          GatherBuf eb{er_all, er_mine, 1};
          GR_TRY(comm_allgather(c.comm, er_mine, er_all, (size_t)g->max_rows, st));
          (void)eb;
        }
        if (!fused)
          GR_TRY(launch_sddmm(g, GRANII_SDDMM_ADD | GRANII_SDDMM_LEAKYRELU | GRANII_SDDMM_ROW_SOFTMAX, el, 1, er_all,
                              1, 1, 1.f, alpha, st));
      } else {
        GR_TRY(launch_sddmm(g, GRANII_SDDMM_DOT | GRANII_SDDMM_ROW_SOFTMAX, th.mine, th.ld, th.all, th.ld, K2,
                            1.f / std::sqrt((float)K2), alpha, st));
      }
    }
    if (comp == GRANII_GAT_REUSE) {
      if (run) {
        if (dot) GR_TRY(launch_spmm(g, alpha, th.all, th.ld, K2, out, ldo, nullptr, nullptr, relu, st));
        else if (fused) {
          GR_TRY(allgather(c, th));
          GR_TRY(launch_spmm_att(g, el, er_all, th.all, th.ld, K2, out, ldo, nullptr, relu, st));
        }
        else GR_TRY(gathered_spmm(c, th, alpha, K2, out, ldo, nullptr, nullptr, relu));
      }
    } else {
      const int64_t ldt = ld4(K1);
      float* T = saved ? saved : b.take((size_t)std::max<int64_t>(R, 1) * ldt);
      void* gw2;
      size_t gn2;
      gemm_ws(b, R, K2, K1, relu ? GRANII_GEMM_RELU : 0, &gw2, &gn2);
      if (run) {
        if (fused) {
          GR_TRY(allgather(c, xg));
          GR_TRY(launch_spmm_att(g, el, er_all, xg.all, xg.ld, K1, T, ldt, nullptr, false, st));
        }
        else GR_TRY(gathered_spmm(c, xg, alpha, K1, T, ldt, nullptr, nullptr, false));
        GR_TRY(launch_gemm(R, K2, K1, T, ldt, a->W, K2, out, ldo, nullptr, relu ? GRANII_GEMM_RELU : 0, gw2, gn2,
                           st));
      }
    }
  }
  if (ws_size) *ws_size = b.off + 1024;
  return GRANII_OK;
}

static granii_status backward_impl(const Ctx& c, granii_composition comp, const granii_layer_args* a,
                                   const float* out, int64_t ldo, const float* dout, int64_t lddo,
                                   const float* saved, float* dH, int64_t lddh, float* dW, void* ws_base,
                                   size_t* ws_size) {
  const granii_graph_s* g = c.g;
  const bool run = ws_base != nullptr;
  Bump b(ws_base);
  const int64_t R = g->n_rows, K1 = a->K1, K2 = a->K2;
  const cudaStream_t st = c.st;
  const bool relu = a->act == GRANII_ACT_RELU;
  // the transposed aggregations (Mᵀ ·) run over Ãᵀ: Ã itself when symmetric, else the kept
  // transpose (GRANII_BUILD_TRANSPOSE); same owned rows, same gather layout, Ã's D̃ (R4)
  const granii_graph_s* gt = g->transposed() ? g->transposed() : g;  // (sizing of a graph without one)
  const Ctx ct{gt, c.comm, c.st};

  // dY = dout ⊙ 1[out > 0]; written into a gather slot when the next sparse step needs it
  const bool dy_gathered = comp == GRANII_GCN_PRE_UPD || comp == GRANII_GCN_DYN_UPD;
  GatherBuf dyg = gather_buf(b, c, K2);
  if (run) {
    // DYN_UPD: dT = D Ãᵀ (D dY) -- the inner D is applied here, so the SpMM has no column scale
    const float* pre = comp == GRANII_GCN_DYN_UPD ? g->dinv_rows : nullptr;
    GR_TRY(launch_scale_mask(R, K2, relu ? out : nullptr, ldo, dout, lddo, pre, dyg.mine, dyg.ld, st));
  }
  const float* dY = dyg.mine;
  const int64_t lddy = dyg.ld;

  // aligned H (needed by the dW GEMM of the *_UPD compositions)
  const float* H = a->H;
  int64_t ldh = a->ldh;
  float* nval = nullptr;
  if (comp == GRANII_GCN_PRE_AGG || comp == GRANII_GCN_PRE_UPD) {
    nval = b.take((size_t)std::max<int64_t>(gt->local_nnz, 1));  // Ñᵀ's values in Ãᵀ's pattern
    if (run) GR_TRY(launch_sddmm(gt, GRANII_SDDMM_DOT, gt->dinv_rows, 1, gt->dinv_cols, 1, 1, 1.f, nval, st));
  }
  void* gwW;
  size_t gnW;
  gemm_ws(b, K1, K2, R, GRANII_GEMM_TRANS_A, &gwW, &gnW);
  void* gwH;
  size_t gnH;
  gemm_ws(b, R, K1, K2, GRANII_GEMM_TRANS_B, &gwH, &gnH);
  GatherBuf dtg;  // gathered operand for the dH SpMM (*_AGG)
  float* dT = nullptr;
  const int64_t ldt1 = ld4(K1), ldt2 = ld4(K2);
  if (comp == GRANII_GCN_PRE_AGG || comp == GRANII_GCN_DYN_AGG) {
    if (dH) dtg = gather_buf(b, c, K1);
  } else {
    dT = b.take((size_t)std::max<int64_t>(R, 1) * ldt2);
  }

  if (run) {
    switch (comp) {
      case GRANII_GCN_PRE_AGG:   // saved T = Ñ H
      case GRANII_GCN_DYN_AGG: { // saved S' = D Ã D H
        if (!saved) return fail(GRANII_ERR_INVALID_ARG, "this composition's backward needs d_saved");
        GR_TRY(launch_gemm(K1, K2, R, saved, ldt1, dY, lddy, dW, K2, nullptr, GRANII_GEMM_TRANS_A, gwW, gnW, st));
        if (dH) {
          granii_gemm_epilogue ep{comp == GRANII_GCN_DYN_AGG ? g->dinv_rows : nullptr, nullptr, nullptr, nullptr,
                                  nullptr};
          GR_TRY(launch_gemm(R, K1, K2, dY, lddy, a->W, K2, dtg.mine, dtg.ld, &ep, GRANII_GEMM_TRANS_B, gwH, gnH, st));
          if (comp == GRANII_GCN_PRE_AGG)
            GR_TRY(gathered_spmm(ct, dtg, nval, K1, dH, lddh, nullptr, nullptr, false));
          else
            GR_TRY(gathered_spmm(ct, dtg, nullptr, K1, dH, lddh, gt->dinv_rows, nullptr, false));
        }
        break;
      }
      case GRANII_GCN_PRE_UPD:
      case GRANII_GCN_DYN_UPD: {
        if (comp == GRANII_GCN_PRE_UPD)
          GR_TRY(gathered_spmm(ct, dyg, nval, K2, dT, ldt2, nullptr, nullptr, false));
        else
          GR_TRY(gathered_spmm(ct, dyg, nullptr, K2, dT, ldt2, gt->dinv_rows, nullptr, false));
        GR_TRY(launch_gemm(K1, K2, R, H, ldh, dT, ldt2, dW, K2, nullptr, GRANII_GEMM_TRANS_A, gwW, gnW, st));
        if (dH) GR_TRY(launch_gemm(R, K1, K2, dT, ldt2, a->W, K2, dH, lddh, nullptr, GRANII_GEMM_TRANS_B, gwH, gnH, st));
        break;
      }
      default:
        return fail(GRANII_ERR_INVALID_ARG, "composition does not belong to GCN");
    }
    if (c.dist()) GR_TRY(comm_allreduce_sum(c.comm, dW, (size_t)K1 * K2, st));
  }
  (void)dy_gathered;
  if (ws_size) *ws_size = b.off + 1024;
  return GRANII_OK;
}

// ---------------------------------------------------------------- GAT backward (N2, reading R22; gat_bwd.cu)
// REUSE  : dY ; pass A (dα = <dY_i, Θ_j>) ; pass B -> dΘ = αᵀ dY + del a_lᵀ + der a_rᵀ ;
//          dW = Hᵀ dΘ ; dH = dΘ Wᵀ
// RECOMP : dY ; dT = dY Wᵀ ; pass A (dα = <dT_i, H_j>) ; pass B -> dH = αᵀ dT + del (W a_l)ᵀ + der (W a_r)ᵀ ;
//          dW = Tᵀ dY + (Hᵀ del) a_lᵀ + (Hᵀ der) a_rᵀ
// both   : da_l = Wᵀ Hᵀ del, da_r = Wᵀ Hᵀ der
// Multi-GPU: the gathered operands are er, Θ or H (pass A) and dY or dT with the 16-byte
// row records in their row tails (pass B); dW and Hᵀ[del, der] are all-reduced.
static GatherBuf local_buf(Bump& b, int64_t R, int64_t K) {
  GatherBuf gb;
  gb.ld = ld4(K);
  gb.all = gb.mine = b.take((size_t)std::max<int64_t>(R, 1) * gb.ld);
  return gb;
}

static granii_status gat_backward_impl(const Ctx& c, granii_composition comp, const granii_layer_args* a,
                                       const float* out, int64_t ldo, const float* dout, int64_t lddo,
                                       const float* saved, float* dH, int64_t lddh, float* dW, void* ws_base,
                                       size_t* ws_size) {
  const granii_graph_s* g = c.g;
  const bool run = ws_base != nullptr;
  Bump b(ws_base);
  const int64_t R = g->n_rows, K1 = a->K1, K2 = a->K2, Rr = std::max<int64_t>(R, 1);
  const cudaStream_t st = c.st;
  const bool relu = a->act == GRANII_ACT_RELU;
  const bool reuse = comp == GRANII_GAT_REUSE;
  const GatSaved sv = gat_saved_layout(R, comp, K1, K2);
  if (run && !saved) return fail(GRANII_ERR_INVALID_ARG, "GAT backward needs d_saved from the forward");
  // pass B walks Ãᵀ (row j lists every i with j in N(i)): Ã when symmetric, else the kept transpose
  const granii_graph_s* gt = g->transposed() ? g->transposed() : g;
  const float* el = saved ? saved + sv.el : nullptr;
  const float* er_own = saved ? saved + sv.er : nullptr;

  // aligned H (own rows) and, for RECOMP on several GPUs, its gathered copy
  const float* H = a->H;
  int64_t ldh = a->ldh;
  const bool h_aligned = (ldh % 4 == 0) && (((uintptr_t)H & 15) == 0);
  GatherBuf hg;
  const bool h_gather = !reuse && c.dist();
  if (h_gather) {
    hg = gather_buf(b, c, K1);
    if (run) {
      GR_TRY(launch_copy_rows(R, K1, a->H, a->ldh, hg.mine, hg.ld, st));
      GR_TRY(allgather(c, hg));
    }
    H = hg.mine;
    ldh = hg.ld;
  } else if (!h_aligned) {
    float* hpad = b.take((size_t)Rr * ld4(K1));
    if (run) GR_TRY(launch_copy_rows(R, K1, a->H, a->ldh, hpad, ld4(K1), st));
    H = hpad;
    ldh = ld4(K1);
  }
  const float* H_all = h_gather ? hg.all : H;

  // dX (dY for REUSE, dT for RECOMP) rows carry pass A's 16-byte record after column rec
  const int64_t rec = round_up(reuse ? K2 : K1, 4);
  GatherBuf dyg = reuse ? gather_buf(b, c, rec + 4) : local_buf(b, R, K2);
  GatherBuf dtg;
  if (!reuse) dtg = gather_buf(b, c, rec + 4);
  // pass A's P rows (<dX_i, P_i> = c_i): REUSE's output Y (16-byte rows: copied when the caller's are
  // not; the sizing pass always reserves the copy), RECOMP's saved T
  const float* Pp = reuse ? out : saved;
  int64_t ldP = reuse ? ldo : sv.ldz;
  if (reuse && (!run || ldo % 4 != 0 || ((uintptr_t)out & 15) != 0)) {
    float* pc = b.take((size_t)Rr * ld4(K2));
    if (run) GR_TRY(launch_copy_rows(R, K2, out, ldo, pc, ld4(K2), st));
    Pp = pc;
    ldP = ld4(K2);
  }
  float* cvec = b.take((size_t)Rr);
  float* del = b.take((size_t)Rr);
  float* der = b.take((size_t)Rr);
  float* er_all = c.dist() ? vec_buf(b, c) : const_cast<float*>(er_own);
  GatherBuf thg;  // REUSE: Θ in the column-id space
  if (reuse) {
    if (c.dist()) {
      thg = gather_buf(b, c, K2);
    } else {
      thg.ld = sv.ldz;
      thg.all = thg.mine = const_cast<float*>(saved);
    }
  }
  // der only (RECOMP input layer on one GPU, no dH wanted): pass B's transposed SpMM feeds only dH, so
  // der comes from pass A's per-entry dα through Ãᵀ's entry map (launch_gat_der) instead; the map is
  // built on first use (not while the stream is being captured: then pass B runs)
  const bool der_only_ok = !reuse && !dH && !c.dist() && g->local_nnz > 0 && !(getenv("GRANII_GAT_DER_ONLY") &&
                                                                            getenv("GRANII_GAT_DER_ONLY")[0] == '0');
  bool der_only = false;
  if (der_only_ok && run) der_only = ensure_tperm(g, st) == GRANII_OK;
  float* tv = der_only_ok ? b.take((size_t)g->local_nnz) : nullptr;
  float* tvb = der_only_ok ? b.take((size_t)g->local_nnz) : nullptr;
  float4* recs = der_only_ok ? reinterpret_cast<float4*>(b.take((size_t)Rr * 4)) : nullptr;
  float* bout = nullptr;  // pass B output
  int64_t ldbo = 0;
  if (reuse) {
    bout = b.take((size_t)Rr * ld4(K2));
    ldbo = ld4(K2);
  } else if (dH) {
    bout = dH;
    ldbo = lddh;
  } else if (!der_only) {  // sizing (run == false) takes it too
    bout = b.take((size_t)Rr * ld4(K1));
    ldbo = ld4(K1);
  }
  float* uv = reuse ? nullptr : b.take((size_t)2 * K1);
  float* pq = b.take((size_t)4 * K1);  // Hᵀ[del, der] as (hi, lo) float pairs
  float* partial = (float*)b.take_bytes(colreduce2_workspace(R, K1));
  void* gwW;
  size_t gnW;
  gemm_ws(b, K1, K2, R, GRANII_GEMM_TRANS_A, &gwW, &gnW);
  void* gwH;
  size_t gnH;
  gemm_ws(b, R, K1, K2, GRANII_GEMM_TRANS_B, &gwH, &gnH);

  if (run) {
    GR_TRY(launch_gat_prep(R, K2, out, ldo, dout, lddo, relu, dyg.mine, dyg.ld, cvec, st));
    if (c.dist()) {
      float* er_slot = er_all + (int64_t)g->rank * g->max_rows;
      GR_CUDA(cudaMemcpyAsync(er_slot, er_own, sizeof(float) * (size_t)R, cudaMemcpyDeviceToDevice, st));
      GR_TRY(comm_allgather(c.comm, er_slot, er_all, (size_t)g->max_rows, st));
      if (reuse) {
        GR_CUDA(cudaMemcpyAsync(thg.mine, saved, sizeof(float) * (size_t)R * sv.ldz, cudaMemcpyDeviceToDevice, st));
        GR_TRY(allgather(c, thg));
      }
    }
    if (!reuse)
      GR_TRY(launch_gemm(R, K1, K2, dyg.mine, dyg.ld, a->W, K2, dtg.mine, dtg.ld, nullptr, GRANII_GEMM_TRANS_B, gwH,
                         gnH, st));
    GatBwdArgs pa;
    pa.n_rows = R;
    pa.row_ptr = g->row_ptr;
    pa.col_idx = g->col_idx;
    pa.order = g->order;
    pa.K = reuse ? K2 : K1;
    pa.dX = reuse ? dyg.mine : dtg.mine;
    pa.ldx = reuse ? dyg.ld : dtg.ld;
    pa.Z = reuse ? thg.all : H_all;
    pa.ldz = reuse ? thg.ld : ldh;
    pa.el = el;
    pa.er = er_all;
    pa.c = cvec;
    pa.P = Pp;  // Y_i (post-activation: dY is 0 where ReLU clipped) or the saved T_i
    pa.ldpp = ldP;
    pa.dXw = reuse ? dyg.mine : dtg.mine;
    pa.rec = rec;
    pa.del = del;
    if (der_only) {
      pa.tout = tv;
      pa.recs = recs;
    }
    GR_TRY(launch_gat_bwd_pass(g, 0, pa, st));
    if (c.dist()) GR_TRY(allgather(c, reuse ? dyg : dtg));  // rows + records
    if (der_only) GR_TRY(launch_gat_der(g, gt, er_own, tv, tvb, recs, der, st));
    if (!reuse && !der_only) GR_TRY(launch_gat_matvec2(K1, K2, a->W, a->a_l, a->a_r, uv, uv + K1, st));
    GatBwdArgs pb;
    pb.n_rows = R;
    pb.row_ptr = gt->row_ptr;
    pb.col_idx = gt->col_idx;
    pb.order = gt->order;
    pb.K = pa.K;
    pb.dX = reuse ? dyg.all : dtg.all;
    pb.ldx = pa.ldx;
    pb.Z = reuse ? saved : H;
    pb.ldz = reuse ? sv.ldz : ldh;
    pb.er = er_own;
    pb.rec = rec;
    pb.del_in = del;
    pb.der = der;
    pb.u = reuse ? a->a_l : uv;
    pb.v = reuse ? a->a_r : uv + K1;
    pb.out = bout;
    pb.ldo = ldbo;
    pb.vec_store = (ldbo % 4 == 0) && (((uintptr_t)bout & 15) == 0);
    if (!der_only) GR_TRY(launch_gat_bwd_pass(gt, 1, pb, st));
    if (reuse) {
      GR_TRY(launch_gemm(K1, K2, R, H, ldh, bout, ldbo, dW, K2, nullptr, GRANII_GEMM_TRANS_A, gwW, gnW, st));
      if (dH)
        GR_TRY(launch_gemm(R, K1, K2, bout, ldbo, a->W, K2, dH, lddh, nullptr, GRANII_GEMM_TRANS_B, gwH, gnH, st));
    } else {
      GR_TRY(launch_gemm(K1, K2, R, saved, sv.ldz, dyg.mine, dyg.ld, dW, K2, nullptr, GRANII_GEMM_TRANS_A, gwW, gnW,
                         st));
    }
    GR_TRY(launch_colreduce2(R, K1, H, ldh, del, der, partial, pq, st));
    if (c.dist()) {
      GR_TRY(comm_allreduce_sum(c.comm, dW, (size_t)K1 * K2, st));
      GR_TRY(comm_allreduce_sum(c.comm, pq, (size_t)4 * K1, st));
    }
    if (!reuse) GR_TRY(launch_gat_rank2(K1, K2, dW, pq, a->a_l, a->a_r, st));
    if (a->d_a_l || a->d_a_r) GR_TRY(launch_gat_mattvec2(K1, K2, a->W, pq, a->d_a_l, a->d_a_r, st));
  }
  if (ws_size) *ws_size = b.off + 1024;
  return GRANII_OK;
}

granii_status layer_workspace(const granii_graph_s* g, granii_model m, granii_composition comp,
                              const granii_layer_args* shape, size_t* ws, size_t* saved_floats) {
  // size for the distributed layout whenever the graph is partitioned
  granii_comm_s fake;
  fake.world = g->world;
  fake.rank = g->rank;
  Ctx c{g, g->world > 1 ? &fake : nullptr, nullptr};
  const int64_t K1 = shape->K1, K2 = shape->K2;
  granii_layer_args a{};
  a.K1 = K1;
  a.K2 = K2;
  a.hops = shape->hops;
  a.Kh = shape->Kh;
  a.ldh = K1;  // worst case: unaligned H needs a padded copy
  a.act = GRANII_ACT_RELU;
  size_t f = 0, f2 = 0, bwd = 0, sf = 0;
  a.attn = GRANII_ATTN_ADDITIVE;
  GR_TRY(forward_impl(c, m, comp, &a, nullptr, K2, nullptr, nullptr, &f, &sf));
  if (m == GRANII_GAT) {
    a.attn = GRANII_ATTN_DOT;
    GR_TRY(forward_impl(c, m, comp, &a, nullptr, K2, nullptr, nullptr, &f2, &sf));
    f = std::max(f, f2);
  }
  if (m == GRANII_GCN)
    GR_TRY(backward_impl(c, comp, &a, nullptr, K2, nullptr, K2, nullptr, (float*)1, K1, nullptr, nullptr, &bwd));
  else if (m == GRANII_GAT)
    GR_TRY(gat_backward_impl(c, comp, &a, nullptr, K2, nullptr, K2, nullptr, nullptr, K1, nullptr, nullptr, &bwd));
  *ws = std::max(f, bwd);
  if (saved_floats) *saved_floats = sf;
  return GRANII_OK;
}

granii_status layer_forward(const granii_graph_s* g, granii_model m, granii_composition comp,
                            const granii_layer_args* a, float* out, int64_t ldo, float* saved, cudaStream_t st) {
  Ctx c{g, a->comm, st};
  size_t need = 0, sf = 0;
  GR_TRY(forward_impl(c, m, comp, a, out, ldo, saved, nullptr, &need, &sf));
  if (a->workspace_bytes < need) return fail(GRANII_ERR_INVALID_ARG, "layer workspace too small");
  return forward_impl(c, m, comp, a, out, ldo, saved, a->workspace, &need, &sf);
}

granii_status layer_backward(const granii_graph_s* g, granii_composition comp, const granii_layer_args* a,
                             const float* out, int64_t ldo, const float* dout, int64_t lddo, const float* saved,
                             float* dH, int64_t lddh, float* dW, cudaStream_t st) {
  Ctx c{g, a->comm, st};
  size_t need = 0;
  auto impl = (comp == GRANII_GAT_REUSE || comp == GRANII_GAT_RECOMP) ? gat_backward_impl : backward_impl;
  GR_TRY(impl(c, comp, a, out, ldo, dout, lddo, saved, dH, lddh, dW, nullptr, &need));
  if (a->workspace_bytes < need) return fail(GRANII_ERR_INVALID_ARG, "layer workspace too small");
  return impl(c, comp, a, out, ldo, dout, lddo, saved, dH, lddh, dW, a->workspace, &need);
}

}  // namespace granii
