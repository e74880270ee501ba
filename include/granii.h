/*
 * granii.h -- C ABI of the B200-native GRANII hot path.
 *
 * GRANII (Lenadora et al., CGO'26; /root/reference/PAPER.md, "Lnnn" = line nnn)
 * executes one GNN layer under one of several matrix re-associations
 * ("compositions") and picks the composition from input attributes.  This
 * library is the data-parallel part of that: the sparse/dense primitives
 * (g-SpMM, g-SDDMM, GEMM, row-broadcast -- L80-L92), the GCN and GAT layers
 * under each composition (Eq. 2-6), their backward (L340), and the
 * input-inspecting selector (L237-L258).
 *
 * Conventions (all entry points):
 *  - Plain pointers and sizes only.  "d_" pointers are CUDA device memory
 *    owned by the caller (the library never frees them); "h_" pointers are
 *    host memory.  Dense matrices are row-major with an explicit leading
 *    dimension (elements).  The library never allocates in the hot path: the
 *    caller passes a workspace sized by the matching *_workspace_size call.
 *  - `stream` is a cudaStream_t passed as void*; everything is stream-ordered
 *    and asynchronous except where noted (graph creation syncs its stream a few times).
 *  - Every call returns a granii_status; C++ exceptions never cross the ABI.
 *    On a non-OK status granii_last_error() returns a thread-local message.
 *    Arguments are validated before any launch (NULL required pointers,
 *    non-positive sizes, unknown ids -> GRANII_ERR_INVALID_ARG).
 *  - There is no CPU fallback: without a CUDA device the compute calls
 *    return GRANII_ERR_CUDA.
 *  - Determinism: no floating-point atomics; for a fixed input and launch
 *    configuration outputs are bitwise reproducible run to run.
 */
#ifndef GRANII_H
#define GRANII_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif
#if defined(__GNUC__)
#pragma GCC visibility push(default)
#endif

typedef enum {
  GRANII_OK = 0,
  GRANII_ERR_INVALID_ARG = 1,
  GRANII_ERR_OOM = 2,
  GRANII_ERR_CUDA = 3,
  GRANII_ERR_NCCL = 4,
  GRANII_ERR_UNSUPPORTED = 5,
  GRANII_ERR_NOT_CALIBRATED = 6
} granii_status;

/* Thread-local description of the last non-OK status of this thread. */
const char* granii_last_error(void);
/* Library version string, e.g. "granii-b200 0.1 sm_100a". */
const char* granii_version(void);

/* ------------------------------------------------------------------------ */
/* Graph handle: Ã = pattern(A ∪ I) in CSR, rows = destinations.            */
/* ------------------------------------------------------------------------ */
typedef struct granii_graph_s* granii_graph;

/* flags of granii_graph_csr_create */
#define GRANII_ADD_SELF_LOOPS 0x1u /* Ã has self-edges (L113)                          */
#define GRANII_SYMMETRIZE 0x2u     /* undirected input (L328): also insert (v,u)        */
/* keep a second CSR, of Ãᵀ (rows = sources), for the backward on a directed graph:
 * the transposed aggregations Mᵀ dY, αᵀ dY run over it.  Ignored
 * (not needed) with SYMMETRIZE, where Ãᵀ = Ã.  Partitioned: this rank's rows of Ãᵀ
 * over the SAME row block [b_r, b_{r+1}) as Ã, columns in the same gather layout. */
#define GRANII_BUILD_TRANSPOSE 0x4u

#define GRANII_NUM_FEATURES 8

typedef struct {
  int64_t num_nodes;       /* global N                                               */
  int64_t nnz;             /* global stored entries of Ã (incl. self-loops)          */
  int64_t row_begin;       /* first global row owned by this rank                    */
  int64_t row_end;         /* one past the last owned row                            */
  int64_t local_nnz;       /* entries in the owned rows                              */
  int64_t max_local_rows;  /* max rows over ranks = row-block height of gather layout */
  int32_t part_rank;       /* this rank                                              */
  int32_t part_world;      /* number of row blocks                                   */
  int32_t symmetric;       /* 1 if Ã = Ãᵀ by construction (SYMMETRIZE)               */
  int32_t has_transpose;   /* 1 if a CSR of Ãᵀ is kept (BUILD_TRANSPOSE, not symmetric)  */
  /* input-featurizer features (L252-L256), integer and exact:
   * [0] N, [1] nnz, [2] sum deg, [3] sum deg^2, [4] max deg, [5] min deg,
   * [6] nnz held by the ceil(N/100) highest-degree rows, [7] rows with deg 0. */
  int64_t features[GRANII_NUM_FEATURES];
} granii_graph_info;

/*
 * Build Ã from a COO edge list (row = dst, col = src: messages flow source ->
 * destination and are summed at the destination, L192), add self-loops
 * (L113) and/or reverse edges, sort by (row, col), drop duplicates (the graphs
 * are unweighted, L328).  Computes deg_i = row nnz, dinv_i = deg_i^{-1/2}
 * (D̃^{-1/2} of Eq. 2/3; 0 when deg_i = 0) and the integer features above.
 *
 * d_src, d_dst: device int32[num_edges], caller-owned, read-only.
 * part_world > 1: keep only rank part_rank's contiguous, nnz-balanced row
 *   block [b_r, b_{r+1}) with b_g = min{ r : row_ptr[r] >= ceil(g*nnz/G) };
 *   local column ids are remapped to the padded gather layout
 *   owner(j)*max_local_rows + (j - b_owner(j)) used by the layer's all-gather.
 * BUILD_TRANSPOSE (directed graphs): the same build over the reversed edges,
 *   with D̃ still Ã's row degrees (R4), kept beside Ã for the backward.
 * Syncs `stream` (validation, nnz, the host-side schedule of hub rows: a few
 * times, at creation only).  Errors: INVALID_ARG for ids outside
 * [0, num_nodes) or bad sizes or unknown flags; OOM; CUDA.
 */
granii_status granii_graph_csr_create(int64_t num_nodes, int64_t num_edges, const int32_t* d_src,
                                      const int32_t* d_dst, uint32_t flags, int32_t part_rank,
                                      int32_t part_world, void* stream, granii_graph* out);
granii_status granii_graph_destroy(granii_graph g);
granii_status granii_graph_query(granii_graph g, granii_graph_info* out);
/* Copy this rank's CSR to host: h_row_ptr int64[local rows + 1] (rebased to 0),
 * h_col_idx int32[local_nnz] (global column ids).  Syncs the device. */
granii_status granii_graph_export_csr(granii_graph g, int64_t* h_row_ptr, int32_t* h_col_idx);
/* Device pointer to dinv of the owned rows (float[local rows]); valid until destroy. */
granii_status granii_graph_dinv(granii_graph g, const float** d_dinv);
/* Host helper (no device work): the nnz-balanced partition bounds above for
 * a host row_ptr; bounds is int64[world + 1].  Used by the distributed layer. */
granii_status granii_partition_bounds(int64_t num_nodes, const int64_t* h_row_ptr, int32_t world,
                                      int64_t* bounds);
/* Host helper (no device work): map global column ids to the padded gather
 * layout, out[i] = owner(j)*max_rows + (j - bounds[owner(j)]) with
 * bounds[owner] <= j < bounds[owner+1].  The device applies the same map at
 * graph creation; tests compare the two. */
granii_status granii_gather_layout_host(int64_t n, const int32_t* h_cols, const int64_t* bounds, int32_t world,
                                        int64_t max_rows, int32_t* h_out);
/* Like export_csr but col ids are returned exactly as stored on the device
 * (gather-layout ids when partitioned). */
granii_status granii_graph_export_local(granii_graph g, int64_t* h_row_ptr, int32_t* h_col_idx);
/* This rank's rows of Ãᵀ (graph built with BUILD_TRANSPOSE, not symmetric), like export_csr:
 * h_row_ptr int64[local rows + 1], h_col_idx int32[*nnz_t] global ids (size it with
 * granii_graph_transpose_nnz).  INVALID_ARG when no transpose is kept. */
granii_status granii_graph_transpose_nnz(granii_graph g, int64_t* nnz_t);
/* Host wall time of graph creation by phase, ms4[0..3] = CSR build (validate, sort, dedupe,
 * row_ptr / col_idx), featurize (degrees, dinv, the integer features: the input inspection
 * whose overhead PAPER L365 quotes), partition + schedule (row blocks, degree order, hub
 * segments), transpose (BUILD_TRANSPOSE).  Each phase ends at a stream sync. */
granii_status granii_graph_timings(granii_graph g, double* ms4);
granii_status granii_graph_export_transpose(granii_graph g, int64_t* h_row_ptr, int32_t* h_col_idx);

/* ------------------------------------------------------------------------ */
/* Primitives (L80-L92).  All operate on this rank's rows of Ã.              */
/* ------------------------------------------------------------------------ */
/* epilogue / scaling flags */
#define GRANII_EPI_RELU 0x1u /* sigma = ReLU on the output (no bias; Eq. 2/3/5)     */

/*
 * g-SpMM (+, x), L88/L92:
 *   Y_i = rs_i * sum_{e in row i} w_e * cs_{c(e)} * X[c(e), :]      (then ReLU if asked)
 * d_vals == NULL: unweighted aggregation (w_e = 1, "copy", L117 / Appendix B).
 * d_row_scale / d_col_scale == NULL: 1.  Row-scales are the row-broadcast of
 * Eq. 1 (L84) fused into the epilogue; column scales fuse the pre-aggregation
 * row-broadcast D̃^{-1/2} H of Eq. 2 into the gather.
 * d_X: rows indexed by column id (n_cols >= every column id, ld = ldx >= K);
 * d_Y: local rows x K (ldy >= K).  X and Y must not alias.
 */
granii_status granii_spmm(granii_graph g, const float* d_vals, const float* d_X, int64_t ldx, int64_t K,
                          float* d_Y, int64_t ldy, const float* d_row_scale, const float* d_col_scale,
                          uint32_t epilogue, void* stream);

/* SDDMM ops */
#define GRANII_SDDMM_DOT 0u         /* e = scale * sum_k U[r,k] V[c,k]      (L88, App. A)   */
#define GRANII_SDDMM_ADD 1u         /* e = scale * (U[r] + V[c]), K = 1 (g-SDDMM, ⊗ = +)     */
#define GRANII_SDDMM_LEAKYRELU 0x10u /* then e = LeakyReLU_0.2(e)                            */
#define GRANII_SDDMM_ROW_SOFTMAX 0x20u /* then alpha = row softmax of e (incl. self-loop)    */
/*
 * g-SDDMM on Ã's pattern (L41, L88, L92): one value per stored entry, in CSR
 * order, written to d_out (float[local_nnz]).  DOT with K = 1 and U = V =
 * dinv computes Ñ = D̃^{-1/2} Ã D̃^{-1/2} (Eq. 3).  ADD |
 * LEAKYRELU | ROW_SOFTMAX with U = el, V = er computes the GAT attention α
 * of Eq. 4 (reading: single-head GAT [25], slope 0.2).
 * U: local rows x K (ldu), V: rows indexed by column id (ldv).
 */
granii_status granii_sddmm(granii_graph g, uint32_t op, const float* d_U, int64_t ldu, const float* d_V,
                           int64_t ldv, int64_t K, float scale, float* d_out, void* stream);

/* GEMM flags */
#define GRANII_GEMM_TRANS_A 0x1u   /* op(A) = Aᵀ, A stored K x M                             */
#define GRANII_GEMM_TRANS_B 0x2u   /* op(B) = Bᵀ, B stored N x K                             */
#define GRANII_GEMM_RELU 0x4u      /* ReLU epilogue                                           */
#define GRANII_GEMM_NO_STORE 0x8u  /* do not write C (only the attention GEMVs)               */

typedef struct {
  const float* row_scale; /* C_i *= row_scale[i] (Eq. 1 row-broadcast fused), or NULL          */
  const float* att_l;     /* float[N]: out_l[i] = sum_j C_ij att_l[j]  (GAT el = Θ a_l), NULL   */
  const float* att_r;     /* float[N]: out_r[i] = sum_j C_ij att_r[j]  (GAT er = Θ a_r), NULL   */
  float* out_l;           /* float[M] or NULL                                                  */
  float* out_r;           /* float[M] or NULL                                                  */
} granii_gemm_epilogue;

/*
 * GEMM (update step, L80-L82, L92): C[M x N] = op(A)[M x K] · op(B)[K x N],
 * fp32 in/out.  Tensor-core path: tcgen05 kind::tf32 with the 3xTF32 split
 * (A = A_hi + A_lo, C = A_hi B_hi + A_hi B_lo + A_lo B_hi), fp32 accumulation
 * in TMEM, A streamed by TMA -- fp32-accurate (<= 1e-4 rel. vs fp64).  Taken
 * when A is not transposed and lda % 4 == 0 (16-byte TMA strides); otherwise
 * an fp32 SIMT kernel computes the same product.  Epilogue order: row scale,
 * attention GEMVs (on the scaled value), ReLU, store.
 * Workspace: granii_gemm_workspace_size bytes of device memory.
 */
granii_status granii_gemm_workspace_size(int64_t M, int64_t N, int64_t K, uint32_t flags, size_t* bytes);
granii_status granii_gemm(int64_t M, int64_t N, int64_t K, const float* d_A, int64_t lda, const float* d_B,
                          int64_t ldb, float* d_C, int64_t ldc, const granii_gemm_epilogue* epi,
                          uint32_t flags, void* d_workspace, size_t workspace_bytes, void* stream);

/* ------------------------------------------------------------------------ */
/* Layers under an explicit composition (§III, Fig. 3 reading R10) */
/* ------------------------------------------------------------------------ */
/* SGC, TAGCN, GIN: the other models of Table III (L67-L69, L307), cited models' definitions
 * (reading R23) with S = D̃^{-1/2} Ã D̃^{-1/2}:
 *   SGC   out = σ(S^k H W)                 TAGCN out = σ(Σ_{j=0..k} S^j H W_j)
 *   GIN   out = σ(ReLU(agg(H) W W2)),  agg(X)_i = (1+ε) X_i + Σ_{j∈N(i)} X_j  (needs self-loops in Ã) */
typedef enum { GRANII_GCN = 0, GRANII_GAT = 1, GRANII_SGC = 2, GRANII_TAGCN = 3, GRANII_GIN = 4 } granii_model;

typedef enum {
  GRANII_GCN_PRE_AGG = 0, /* Eq. 3, aggregate first: SDDMM Ñ ; SpMM_w(Ñ, H) ; GEMM (·W)       */
  GRANII_GCN_PRE_UPD = 1, /* Eq. 3, update first:    SDDMM Ñ ; GEMM (H W) ; SpMM_w(Ñ, ·)      */
  GRANII_GCN_DYN_AGG = 2, /* Eq. 2, aggregate first: SpMM_u(Ã, D̃^-½ H) ; D̃^-½ ; GEMM (·W)  */
  GRANII_GCN_DYN_UPD = 3, /* Eq. 2, update first:    GEMM (H W) ; D̃^-½ ; SpMM_u(Ã, ·) ; D̃^-½ */
  GRANII_GAT_REUSE = 16,  /* Eq. 5: Θ = H W ; α = Atten(Ã, Θ, W_A) ; SpMM_w(α, Θ)             */
  GRANII_GAT_RECOMP = 17, /* Eq. 6: Θ-scores ; α ; SpMM_w(α, H) ; GEMM (·W)                    */
  /* SGC: k hops of S, PRE = Ñ by SDDMM + weighted SpMMs, DYN = unweighted SpMMs with the
   * D̃^-½ scalings fused; AGG = hops at K1 then GEMM, UPD = GEMM then hops at K2 */
  GRANII_SGC_PRE_AGG = 32, GRANII_SGC_PRE_UPD = 33, GRANII_SGC_DYN_AGG = 34, GRANII_SGC_DYN_UPD = 35,
  /* TAGCN: AGG = X_0..X_k = S^j H at K1 side by side, one GEMM against the stacked W_j;
   * UPD = Horner: Z = H W_k ; Z = S Z + H W_j (the addend fused in the SpMM epilogue) */
  GRANII_TAGCN_PRE_AGG = 48, GRANII_TAGCN_PRE_UPD = 49, GRANII_TAGCN_DYN_AGG = 50, GRANII_TAGCN_DYN_UPD = 51,
  /* GIN: PRE = weighted SpMM with 1+ε on the diagonal (values written per call), DYN =
   * unweighted SpMM with + ε X_i fused in its epilogue; AGG = aggregate at K1 then W,
   * UPD = H W then aggregate at Kh (ReLU fused); W2 last */
  GRANII_GIN_PRE_AGG = 64, GRANII_GIN_PRE_UPD = 65, GRANII_GIN_DYN_AGG = 66, GRANII_GIN_DYN_UPD = 67
} granii_composition;

#define GRANII_ACT_NONE 0u
#define GRANII_ACT_RELU 1u
#define GRANII_ATTN_ADDITIVE 0u /* e_ij = LeakyReLU(Θ_i a_l + Θ_j a_r)                 */
#define GRANII_ATTN_DOT 1u      /* e_ij = <Θ_i, Θ_j> / sqrt(K2)   [proposal, DESIGN R9] */

typedef struct granii_comm_s* granii_comm; /* NCCL communicator (multi-GPU row partition) */

typedef struct {
  int64_t K1, K2;          /* input / output embedding sizes (L105)                     */
  const float* H;          /* owned rows x K1, leading dimension ldh                     */
  int64_t ldh;
  const float* W;          /* K1 x K2 row-major (replicated on every rank)               */
  const float* a_l;        /* GAT additive attention weights W_A = [a_l; a_r], K2 each   */
  const float* a_r;
  uint32_t act;            /* GRANII_ACT_*                                               */
  uint32_t attn;           /* GRANII_ATTN_*                                              */
  void* workspace;         /* device, >= granii_layer_workspace_size bytes               */
  size_t workspace_bytes;
  granii_comm comm;        /* NULL: whole graph on this GPU                              */
  float* d_a_l;            /* GAT backward outputs dL/da_l, dL/da_r (K2 floats each,     */
  float* d_a_r;            /*   all-reduced over comm); NULL: not computed               */
  int32_t hops;            /* SGC / TAGCN: k >= 0 (TAGCN: W holds k+1 stacked K1 x K2)   */
  float eps;               /* GIN: ε                                                     */
  int64_t Kh;              /* GIN: MLP hidden width (W: K1 x Kh, W2: Kh x K2)            */
  const float* W2;         /* GIN: second MLP weight                                     */
} granii_layer_args;

/* Workspace bytes and the number of floats of `saved` (state kept for backward).
 * GCN / GAT only; SGC / TAGCN / GIN need their shape parameters: use the _ex form. */
granii_status granii_layer_workspace_size(granii_graph g, granii_model m, granii_composition c, int64_t K1,
                                          int64_t K2, size_t* workspace_bytes, size_t* saved_floats);
/* Same for any model; reads the shape fields of *a (K1, K2, hops, Kh) only. */
granii_status granii_layer_workspace_size_ex(granii_graph g, granii_model m, granii_composition c,
                                             const granii_layer_args* a, size_t* workspace_bytes,
                                             size_t* saved_floats);
/*
 * out = sigma(layer(H)) for the owned rows (out: rows x K2, ld ldo).  Every
 * composition computes the same mathematical value (L192: only semantically
 * equivalent re-associations).  d_saved (nullable) receives the state the
 * backward of this composition needs (granii_layer_workspace_size); it must be
 * 16-byte aligned (its rows are read as float4), else GRANII_ERR_INVALID_ARG.
 * With comm != NULL the dense operand of every SpMM/SDDMM is all-gathered
 * over NCCL inside the call.
 */
granii_status granii_layer_forward(granii_graph g, granii_model m, granii_composition c,
                                   const granii_layer_args* a, float* d_out, int64_t ldo, float* d_saved,
                                   void* stream);
/*
 * Layer backward (training, L340: the forward's composition is kept).
 * GCN: for out = sigma(M H W), M = D̃^{-1/2} Ã D̃^{-1/2}, upstream d_dout = dL/dout:
 *   dY = dout ⊙ 1[out > 0] (ReLU; identity otherwise), dW = (M H)ᵀ dY, dH = Mᵀ dY Wᵀ.
 * GAT (additive attention; chain rule of Eq. 4-6, R22): dW, dH and,
 *   through a->d_a_l / a->d_a_r, the attention-weight gradients; REUSE works at
 *   K2, RECOMP at K1 (dT = dY Wᵀ first), as in their forwards.  d_saved is
 *   required (Θ or T = α H, el, er written by the forward; 16-byte aligned,
 *   else INVALID_ARG).  Dot attention ->
 *   UNSUPPORTED.
 * d_dH may be NULL (input layer).  d_dW (K1 x K2) is all-reduced over comm.
 * The transposed aggregations (Mᵀ dY; GAT pass B: every i with j in N(i)) run over Ã
 * itself when symmetric, else over the CSR of Ãᵀ kept by GRANII_BUILD_TRANSPOSE;
 * a directed graph without it -> INVALID_ARG.
 */
granii_status granii_layer_backward(granii_graph g, granii_model m, granii_composition c,
                                    const granii_layer_args* a, const float* d_out, int64_t ldo,
                                    const float* d_dout, int64_t lddo, const float* d_saved, float* d_dH,
                                    int64_t lddh, float* d_dW, void* stream);

/* ------------------------------------------------------------------------ */
/* Selector (L237-L258)                                                      */
/* ------------------------------------------------------------------------ */
#define GRANII_SELECT_NO_PREFILTER 0x1u /* skip the embedding-size rule (L237-L239)   */
/* Extension (the paper selects on the forward only, L340): add the backward
 * primitives of each GCN composition to its cost; INPUT_LAYER drops dH. */
#define GRANII_SELECT_TRAINING 0x2u
#define GRANII_SELECT_INPUT_LAYER 0x4u
/* Extension: measured tie-break.  When the two best predictions are within 15 % and the best is
 * below 10 ms (near-ties the models' ~12 % median error cannot decide, on layers cheap enough to
 * time once: belgium-shaped TAGCN 256->256 is a 2 % predicted tie at 5.2 ms, 12 % apart measured), the close
 * candidates run once on zero-filled inputs of the layer's shape (forward, + backward with
 * SELECT_TRAINING) on a private stream and the fastest is returned (predicted_ms stays the model's).
 * Allocates and frees device memory, synchronises its own stream.  Ignored on partitioned graphs
 * (every rank must pick the same composition). */
#define GRANII_SELECT_REFINE 0x8u
#define GRANII_MAX_CANDIDATES 8

/*
 * Pick the composition with the least predicted cost for this graph and
 * (K1, K2): first the embedding-size rule (GCN: K1 >= K2 -> update-first,
 * K1 < K2 -> aggregate-first; L226, L237-L239, reading R11), then per-
 * primitive cost models calibrated on this chip (L241, L258; composition cost
 * = sum of primitive costs), argmin with ties to the lowest id (L241, R12).
 * Host-only, microseconds; reads the features cached in the handle.
 * calib_path: text file written by tools/calibrate.py; NULL -> $GRANII_CALIB,
 * else built-in B200 defaults.  Outputs: *out; candidates[i] / predicted_ms[i]
 * for the n_candidates compositions considered (arrays of GRANII_MAX_CANDIDATES).
 */
granii_status granii_select(granii_graph g, granii_model m, int64_t K1, int64_t K2, const char* calib_path,
                            uint32_t flags, granii_composition* out, int32_t* candidates,
                            double* predicted_ms, int32_t* n_candidates);
/* Same for any model (GCN / GAT as above); reads the shape fields of *a (K1, K2, hops, Kh).
 * SGC / TAGCN: the embedding-size rule picks AGG for K1 < K2 and UPD for K1 >= K2 (as GCN),
 * GIN compares K1 with Kh; the cost models then choose PRE vs DYN.  Forward costs only. */
granii_status granii_select_ex(granii_graph g, granii_model m, const granii_layer_args* a, const char* calib_path,
                               uint32_t flags, granii_composition* out, int32_t* candidates,
                               double* predicted_ms, int32_t* n_candidates);
/* Calibration support: the feature vector the cost model of primitive `prim`
 * (0 spmm weighted, 1 spmm unweighted, 2 spmm unweighted + column scale,
 * 3 sddmm K=1, 4 sddmm K=1 + softmax, 5 gemm, 6 gemm without store, 7 gemm Aᵀ·B,
 * 8 elementwise, 9 all-gather, 10 gemm with the GAT attention GEMVs, 11 / 12 GAT backward passes A / B,
 * 13 the der-only pass of a RECOMP input layer's backward)
 * uses for this graph and widths (K1, K2);
 * feats has room for 8 values; model_name (32 bytes) receives the model key
 * the coefficients are stored under in the calibration file. */
granii_status granii_cost_features(granii_graph g, int32_t prim, int64_t K1, int64_t K2, double* feats,
                                   int32_t* n, char* model_name);

/* ------------------------------------------------------------------------ */
/* Multi-GPU (row partition, NCCL over NVLink)                                */
/* ------------------------------------------------------------------------ */
/* Write a 128-byte NCCL unique id (rank 0); ranks exchange it out of band. */
granii_status granii_comm_unique_id(void* h_id128);
granii_status granii_comm_create(const void* h_id128, int32_t rank, int32_t world, granii_comm* out);
/* In-process loopback group: writes `world` handles (ranks 0..world-1) to out[].
 * Each rank is driven by its own host thread on its own stream of ONE device;
 * every collective call blocks its thread until all ranks have entered it
 * (host barrier), then moves data with stream-ordered device copies, ordered
 * across the ranks' streams by events.  All-reduce sums in rank order, so every
 * rank gets bitwise the same result.  Purpose: run and test the partitioned
 * path on a single GPU; it has no NVLink transport.
 * Errors: INVALID_ARG for world outside [1, 16].  Destroy each handle. */
granii_status granii_comm_create_local(int32_t world, granii_comm* out);
/* TIMING STUB, not a transport: a rank-`rank` communicator whose collectives move no
 * data (they only update the statistics below).  Layer outputs on a partitioned graph
 * are WRONG with it.  It exists to time one rank's local work of a G-way partition on a
 * single GPU (tools/scaling_projection.py).  Errors: INVALID_ARG. */
granii_status granii_comm_create_stub(int32_t rank, int32_t world, granii_comm* out);
/* Bytes this rank has received over the communicator's lifetime (all-gather: (G-1)
 * blocks; block broadcast: one block unless root; all-reduce: the ring's 2(G-1)/G of the
 * buffer) and the number of collective calls.  Host-side counters, any transport. */
granii_status granii_comm_stats(granii_comm c, uint64_t* bytes_in, uint64_t* calls);
granii_status granii_comm_destroy(granii_comm c);
/* The communicator's two data collectives, as the layers use them (north_star (4)), for callers
 * that exchange their own buffers (e.g. all-reducing a gradient they computed themselves):
 *   all-gather: recv = [block of rank 0 | ... | block of rank G-1], `count` floats per block,
 *               send may be recv + rank * count (in place);
 *   all-reduce: buf = Σ_ranks buf (fp32 sum, in place).
 * Device pointers, stream-ordered on `stream`; NCCL, loopback or stub transport (the stub moves
 * no data).  Errors: INVALID_ARG (NULL), NCCL (transport failure). */
granii_status granii_comm_allgather(granii_comm c, const float* d_send, float* d_recv, size_t count, void* stream);
granii_status granii_comm_allreduce_sum(granii_comm c, float* d_buf, size_t count, void* stream);
/* What the transport reports: rank count and this rank (NCCL: ncclCommCount / ncclCommUserRank,
 * so a launcher can check that N processes really formed one N-rank communicator) and the NCCL
 * version (0 for loopback / stub).  Errors: NCCL if the communicator was aborted. */
granii_status granii_comm_query(granii_comm c, int32_t* nranks, int32_t* rank, int32_t* nccl_version);
/* The aggregation schedule the planner picks for a K-wide SpMM on this partitioned graph (N1,
 * DESIGN.md §7): phases (1 = all-gather then SpMM; P >= 2 = own block under the transfer, then the
 * other blocks in P-1 chunks as they land) and the modelled times of both (ms).  Host only. */
granii_status granii_comm_plan(granii_graph g, int64_t K, int32_t weighted, int32_t col_scale, int32_t* phases,
                               double* ms_allgather_then_spmm, double* ms_planned);
/* Failure detection.  Starts (timeout_ms > 0) or stops (<= 0) a host watchdog
 * thread for the communicator: every collective the library issues records an event on its
 * stream (except under CUDA-graph capture); every ~20 ms the watchdog polls
 * ncclCommGetAsyncError and the oldest incomplete collective.  An asynchronous error, a device
 * error, or a collective pending longer than timeout_ms (a mismatched or missing collective on
 * another rank hangs rather than fails) aborts the communicator (ncclCommAbort; loopback: marked
 * failed) and every later collective or granii_comm_check on it returns GRANII_ERR_NCCL with the
 * reason in granii_last_error().  The stub transport is never watched. */
granii_status granii_comm_watchdog(granii_comm c, int64_t timeout_ms);
/* GRANII_OK, or GRANII_ERR_NCCL with the watchdog's reason once the communicator was aborted. */
granii_status granii_comm_check(granii_comm c);
/* Register a device buffer that collectives will read / write (e.g. a layer workspace holding
 * the gather buffers) with NCCL (ncclCommRegister), so NCCL can use it directly instead of
 * staging through its own buffers where the algorithm supports it.  *handle is for
 * granii_comm_deregister; NULL (and OK) on loopback / stub transports.  The buffer must stay
 * allocated until deregistered.  Errors: UNSUPPORTED (NCCL without registration), NCCL. */
granii_status granii_comm_register(granii_comm c, void* d_buf, size_t bytes, void** handle);
granii_status granii_comm_deregister(granii_comm c, void* handle);
/* Test support: one kernel that keeps `stream` busy for `us` microseconds (watchdog tests). */
granii_status granii_debug_spin(int64_t us, void* stream);

/* ------------------------------------------------------------------------ */
/* Training-step helpers around the layers (not selected by GRANII)          */
/* ------------------------------------------------------------------------ */
/* Mean softmax cross-entropy over rows: loss_i = logsumexp(Z_i) - Z_i[y_i];
 * writes dZ = (softmax(Z) - onehot(y)) / n_total and, if d_loss != NULL, the
 * per-row losses (float[rows]). */
granii_status granii_softmax_xent(int64_t rows, int64_t C, const float* d_Z, int64_t ldz, const int32_t* d_y,
                                  int64_t n_total, float* d_dZ, int64_t lddz, float* d_loss, void* stream);
/* W -= lr * dW over n floats. */
granii_status granii_sgd(int64_t n, float lr, const float* d_grad, float* d_param, void* stream);

/* ------------------------------------------------------------------------ */
/* Tracing (per-primitive CUDA-event timer; measurement support)             */
/* ------------------------------------------------------------------------ */
typedef struct {
  char name[32];   /* primitive: spmm, sddmm, gemm_tc, gemm_simt, gemm_tn, csr, elementwise */
  int64_t calls;   /* launcher calls recorded                                            */
  int64_t launches;/* CUDA kernels launched by those calls                               */
  double ms;       /* summed device time between events recorded on the launch stream    */
  double bytes;    /* summed ALGORITHMIC bytes (DESIGN.md §6 per-unit figures)            */
  double flops;    /* summed algorithmic flops                                           */
  double compulsory_bytes; /* summed COMPULSORY HBM bytes: every operand read / written once
                              (SpMM: col ids + X + Y once, however often the gathers re-read X) */
  int64_t l2_resident;     /* calls whose gathered operand (one K slice of X) fits the L2, so the
                              gathers are served by L2: the binding roof is L2 bandwidth  */
} granii_prof_entry;

/* Enable (1) / disable (0) event recording around every primitive; resets the table. */
granii_status granii_profile_enable(int32_t on);
/* Sync the device, aggregate the recorded events per primitive into out[0..*n). */
granii_status granii_profile_read(granii_prof_entry* out, int32_t max_entries, int32_t* n);
/* Total CUDA kernels this library has launched in this process (monotonic). */
int64_t granii_launch_count(void);

#if defined(__GNUC__)
#pragma GCC visibility pop
#endif
#ifdef __cplusplus
}
#endif
#endif /* GRANII_H */
