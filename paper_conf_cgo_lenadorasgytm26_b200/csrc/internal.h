// internal.h -- shared declarations of the B200 GRANII library (not part of the ABI).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <atomic>
#include <string>
#include <vector>

#include "../../include/granii.h"

namespace granii {

// ----------------------------------------------------------------- errors
struct Error {
  granii_status st;
  std::string msg;
};
void set_error(const std::string& m);
granii_status fail(granii_status st, const std::string& m);
#define GR_CUDA(call)                                                                      \
  do {                                                                                     \
    cudaError_t e_ = (call);                                                               \
    if (e_ != cudaSuccess)                                                                 \
      return ::granii::fail(GRANII_ERR_CUDA, std::string(#call) + ": " + cudaGetErrorString(e_)); \
  } while (0)
#define GR_CHECK_LAUNCH()                                                                  \
  do {                                                                                     \
    cudaError_t e_ = cudaGetLastError();                                                   \
    if (e_ != cudaSuccess)                                                                 \
      return ::granii::fail(GRANII_ERR_CUDA, std::string("launch: ") + cudaGetErrorString(e_)); \
  } while (0)
#define GR_TRY(x)                                \
  do {                                           \
    granii_status s_ = (x);                      \
    if (s_ != GRANII_OK) return s_;              \
  } while (0)
#define GR_ARG(cond, msg)                                               \
  do {                                                                  \
    if (!(cond)) return ::granii::fail(GRANII_ERR_INVALID_ARG, msg);    \
  } while (0)

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }
inline int64_t round_up(int64_t a, int64_t b) { return ceil_div(a, b) * b; }

// ----------------------------------------------------------------- device info
struct DevInfo {
  int device = -1;
  int sms = 148;
  int64_t l2_bytes = 126ll << 20;
};
granii_status dev_info(DevInfo* out);
// CTAs of `fn` resident per SM at `threads` threads (cudaOccupancyMaxActiveBlocksPerMultiprocessor,
// cached per kernel).  Grid-stride (persistent) kernels launch sms x this many CTAs: a grid of
// 8 CTAs / SM where 6 fit runs in 1.33 waves, the last third on a quarter of the machine.
int resident_ctas(const void* fn, int threads, size_t smem = 0);
template <typename F>
inline int64_t persistent_grid(F* fn, int threads, int sms, int64_t want) {
  const int64_t cap = (int64_t)sms * resident_ctas((const void*)fn, threads);
  return std::max<int64_t>(1, std::min<int64_t>(want, cap));
}

// ----------------------------------------------------------------- tracing
// RAII scope around one launcher call: counts kernel launches always; records
// a pair of CUDA events on the launch stream when profiling is enabled.
// compulsory < 0: the algorithmic bytes are the compulsory bytes (streaming kernels)
struct ProfScope {
  ProfScope(const char* name, cudaStream_t st, double bytes, double flops, int launches, double compulsory = -1.0,
            bool l2_resident = false);
  ~ProfScope();
  void add_launches(int n);
  const char* name;
  cudaStream_t st;
  double bytes, flops, compulsory;
  int launches;
  int slot;
  bool l2_resident;
};

}  // namespace granii

// ----------------------------------------------------------------- graph
struct granii_graph_s {
  int64_t N = 0;            // global nodes
  int64_t nnz = 0;          // global stored entries
  int64_t row_begin = 0, row_end = 0, n_rows = 0;
  int64_t local_nnz = 0;
  int32_t rank = 0, world = 1;
  int64_t max_rows = 0;     // gather-layout block height
  int64_t n_cols = 0;       // size of the column-id space (N, or world*max_rows)
  int32_t symmetric = 0;
  int32_t self_loops = 0;   // every row of Ã holds its diagonal entry (GRANII_ADD_SELF_LOOPS)
  std::vector<int64_t> bounds;
  int64_t* row_ptr = nullptr;     // device, n_rows+1, rebased
  int32_t* col_idx = nullptr;     // device, local_nnz, column-id space
  float* dinv_rows = nullptr;     // device, n_rows
  float* dinv_cols = nullptr;     // device, n_cols (== dinv_rows when world == 1)
  float* dinv2_rows = nullptr;    // device, n_rows: 1 / deg (post-scale of one hop fused with the next pre-scale)
  int32_t* order = nullptr;       // device, n_rows: owned rows by descending degree
  longlong2* ord_rp = nullptr;    // device, n_rows: {row_ptr[order[t]], row_ptr[order[t] + 1]} -- a row's
                                  // entry range in schedule order, one coalesced load (no dependent
                                  // random row_ptr access after order[t])
  int32_t* owner_off = nullptr;   // device, n_rows x (world+1) when world > 1: entries of row i whose
                                  // column is owned by rank p are [rp_i + off[i][p], rp_i + off[i][p+1])
  int32_t* ord_off = nullptr;     // the same rows of owner_off in schedule order (ord_off[t] = owner_off[order[t]]):
                                  // a phase's entry range of schedule position t without a dependent load
  // heavy rows (degree > seg_len) = order[0 .. n_heavy); each is cut into segments of
  // seg_len entries that are scheduled as independent warp-wide work items
  int64_t seg_len = 2048;
  int64_t n_heavy = 0, n_seg = 0;
  int64_t n_seg_global = -1;      // hub segments of the whole graph (partitioned graphs; -1: = n_seg)
  int32_t* seg_ptr = nullptr;     // device, n_heavy+1: segments of heavy row h are [seg_ptr[h], seg_ptr[h+1])
  int64_t* seg_lo = nullptr;      // device, n_seg: entry range of each segment
  int64_t* seg_hi = nullptr;
  int32_t* seg_heavy = nullptr;   // device, n_seg: heavy index h of each segment
  int32_t* seg_row = nullptr;     // device, n_seg: row of each segment (= order[seg_heavy])
  // rows with more than wide_deg entries = order[0 .. n_wide): the sparse (group-per-row)
  // schedules give them a whole warp
  int64_t wide_deg = 32, n_wide = 0;
  // entry tiles of the K = 1 SDDMM (sddmm.cu): tile t = Ã's entries
  // [t·tile_e, (t+1)·tile_e) in CSR order; tile_row[t] = the row holding entry t·tile_e
  static constexpr int64_t tile_e = 4096;
  int64_t n_tiles = 0;
  int32_t* tile_row = nullptr;    // device, n_tiles
  int64_t features[GRANII_NUM_FEATURES] = {0};
  int device = 0;
  // host wall time of the creation phases (ms): CSR build (validate, sort, dedupe, row_ptr / col_idx),
  // featurize (degrees, dinv, integer features), partition + schedule (order, ord_rp, hub segments),
  // transpose (BUILD_TRANSPOSE) -- PAPER L365 quotes the featurizer's overhead on its own
  double create_ms[4] = {0, 0, 0, 0};
  // built on first use (one GPU; ensure_tperm): a column-blocked layout of per-entry arrays (tblk_n
  // blocks of columns, region b = the entries whose column lies in block b, rows ascending)
  int32_t* tblk = nullptr;        // device, local_nnz: blocked position of Ã's entry e
  int32_t* tperm = nullptr;       // device, local_nnz: blocked position of the Ã entry (i, j) behind Ãᵀ's entry e' = (j, i)
  int tblk_n = 0;
  granii_graph_s* T = nullptr;    // Ãᵀ over the same owned rows (GRANII_BUILD_TRANSPOSE, directed graphs);
                                  // its dinv arrays are Ã's (D̃ = Ã's row degrees, R4)
  // the graph the transposed aggregations of the backward run over (Mᵀ = M when symmetric)
  const granii_graph_s* transposed() const { return symmetric ? this : T; }
  float avg_deg() const { return n_rows > 0 ? float(local_nnz) / float(n_rows) : 0.f; }
};

struct granii_comm_s {
  void* nccl = nullptr;  // ncclComm_t
  void* loop = nullptr;  // in-process loopback group (comm.cpp), shared by its G handles
  int stub = 0;          // timing stub: collectives move no data (granii_comm_create_stub)
  uint64_t bytes_in = 0, calls = 0;        // bytes this rank received / collective calls (stats)
  cudaStream_t side = nullptr;             // collectives overlapped with compute (N1)
  cudaEvent_t* ev = nullptr;               // world + 1 events on `side`
  int32_t rank = 0, world = 1;
  void* wd = nullptr;                      // failure-detection watchdog (comm.cpp), NULL when off
  std::atomic<int> failed{0};              // set once the communicator was aborted
};

namespace granii {
// kernels (launchers); all validate nothing -- callers in api.cu validate.
granii_status launch_spmm(const granii_graph_s* g, const float* vals, const float* X, int64_t ldx, int64_t K,
                          float* Y, int64_t ldy, const float* rs, const float* cs, bool relu, cudaStream_t st);
// Y_i = act(rs_i * sum + beta * B_i): SpMM with a dense addend fused in the epilogue
granii_status launch_spmm_ex(const granii_graph_s* g, const float* vals, const float* X, int64_t ldx, int64_t K,
                             float* Y, int64_t ldy, const float* rs, const float* cs, bool relu, const float* B,
                             int64_t ldb, float beta, cudaStream_t st);
// GAT aggregation with the additive attention fused (Eq. 4-6): Y_i = act(rs_i * sum_e alpha_e X_c(e)),
// alpha = row softmax of LeakyReLU(el_i + er_c) computed on the fly (online max / sum per row, no
// SDDMM pass, no alpha array); warp-per-row graphs (spmm_att_supported), single GPU
bool spmm_att_supported(const granii_graph_s* g);
bool gat_fused_enabled();  // GRANII_GAT_FUSED != 0
granii_status launch_spmm_att(const granii_graph_s* g, const float* el, const float* er, const float* X, int64_t ldx,
                              int64_t K, float* Y, int64_t ldy, const float* rs, bool relu, cudaStream_t st);
// one phase of a block-phased aggregation over a partitioned graph (layer.cu gathered_spmm):
// the entries whose column lies in the gather blocks [p0, p1), block `skip` excluded (-1: none);
// partial = heavy-segment scratch [n_seg][round_up(K,4)] kept across the phases (NULL if the
// graph has no segments)
struct SpmmPhase {
  int p0, p1, skip;
  int first, last;
  float* partial;
};
// K slices of a vec4 SpMM and the dynamic-normalisation pre-scale rule (spmm.cu)
int64_t spmm_slices(double avg_deg, double cols, int64_t K, int64_t l2_bytes);
bool dyn_prescale(double nnz, double rows, double avg_deg, double cols, int64_t K, int64_t l2_bytes);
// phases of an overlapped aggregation on a partitioned graph (select.cpp; 1 = all-gather first)
int comm_phases(const granii_graph_s* g, int64_t K, bool weighted, bool col_scale);
int comm_plan(const granii_graph_s* g, int64_t K, bool weighted, bool col_scale, double* t1, double* tp);
granii_status launch_spmm_phase(const granii_graph_s* g, const float* vals, const float* X, int64_t ldx, int64_t K,
                                float* Y, int64_t ldy, const float* rs, const float* cs, bool relu, const float* B,
                                int64_t ldb, float beta, const SpmmPhase& ph, cudaStream_t st);
// GIN's precomputed values: vals_e = 1 + eps on the diagonal entry of each row, 1 elsewhere
granii_status launch_gin_vals(const granii_graph_s* g, float eps, float* vals, cudaStream_t st);
granii_status launch_sddmm(const granii_graph_s* g, uint32_t op, const float* U, int64_t ldu, const float* V,
                           int64_t ldv, int64_t K, float scale, float* out, cudaStream_t st);
size_t gemm_workspace(int64_t M, int64_t N, int64_t K, uint32_t flags);
granii_status launch_gemm(int64_t M, int64_t N, int64_t K, const float* A, int64_t lda, const float* B,
                          int64_t ldb, float* C, int64_t ldc, const granii_gemm_epilogue* epi, uint32_t flags,
                          void* ws, size_t ws_bytes, cudaStream_t st);
granii_status launch_scale_mask(int64_t rows, int64_t K, const float* out, int64_t ldo, const float* g, int64_t ldg,
                                const float* rs, float* dst, int64_t ldd, cudaStream_t st);
granii_status launch_relu_mask(int64_t rows, int64_t K, const float* out, int64_t ldo, const float* g,
                               int64_t ldg, float* dst, int64_t ldd, cudaStream_t st);
granii_status launch_copy_rows(int64_t rows, int64_t K, const float* src, int64_t lds, float* dst, int64_t ldd,
                               cudaStream_t st);
// GAT backward (gat_bwd.cu); pass 0 = rows i (del, stat), pass 1 = rows j (transposed SpMM, der)
struct GatBwdArgs {
  int64_t n_rows = 0;
  const int64_t* row_ptr = nullptr;
  const int32_t* col_idx = nullptr;
  const int32_t* order = nullptr;
  int64_t K = 0;
  const float* dX = nullptr;  // pass 0: own rows; pass 1: column-id space
  int64_t ldx = 0;
  const float* Z = nullptr;   // pass 0: column-id space; pass 1: own rows
  int64_t ldz = 0;
  const float* el = nullptr;  // pass 0: own rows
  const float* er = nullptr;  // pass 0: column-id space; pass 1: own rows
  const float* c = nullptr;   // pass 0: own rows
  const float* P = nullptr;   // pass 0: own rows of the forward's Y (REUSE) or T = αH (RECOMP): <dX_i, P_i> = c_i
  int64_t ldpp = 0;
  float* dXw = nullptr;       // pass 0: dX's own rows, whose tail receives the row record
  int64_t rec = 0;            // column of the 16-byte record {el, m, 1/s, c} in dX rows
  float* del = nullptr;       // pass 0 out
  const float* del_in = nullptr;    // pass 1: own rows
  float* der = nullptr;       // pass 1 out
  const float* u = nullptr;   // pass 1 epilogue vectors (K)
  const float* v = nullptr;
  float* out = nullptr;       // pass 1 out (own rows x K, ld ldo)
  int64_t ldo = 0;
  int vec_store = 0;
  int64_t n_wide = 0;         // order[0 .. n_wide): a warp per row; the rest: a lane group per row
  // hub segments (set by launch_gat_bwd_pass from the graph): warp-wide items scheduled first,
  // merged per heavy row (heavy_rows[0 .. n_heavy)) in fixed order by a combine kernel
  int64_t n_seg = 0, n_heavy = 0, ldp = 0;
  const int64_t* seg_lo = nullptr;
  const int64_t* seg_hi = nullptr;
  const int32_t* seg_row = nullptr;
  const int32_t* seg_ptr = nullptr;
  const int32_t* heavy_rows = nullptr;
  float4* seg_a = nullptr;    // pass 0: online-softmax state {m, S, Cw, D} per segment
  float* seg_b = nullptr;     // pass 1: partial output row per segment (ld ldp)
  float* seg_der = nullptr;   // pass 1: partial der per segment
  float* tout = nullptr;      // pass 0, optional: dα_ij - c_i per entry in Ã's CSR order (the der-only path)
  float4* recs = nullptr;     // pass 0, optional: the row records {el, m, 1/s, c}, one float4 per own row
};
granii_status launch_gat_prep(int64_t R, int64_t K, const float* out, int64_t ldo, const float* g, int64_t ldg,
                              bool relu, float* dY, int64_t ldd, float* c, cudaStream_t st);
granii_status launch_gat_bwd_pass(const granii_graph_s* g, int pass, const GatBwdArgs& a, cudaStream_t st);
// the column-blocked entry layout (g->tblk, g->tperm: Ã's and Ãᵀ's entries -> blocked positions), built
// once (stable radix sort of Ã's column ids, per-(block, row) counts and their scan);
// GRANII_ERR_UNSUPPORTED on a partitioned graph or while `st` is being captured (no allocation)
granii_status ensure_tperm(const granii_graph_s* g, cudaStream_t st);
// der_j = Σ_{i: j ∈ N(i)} α_ij (dα_ij - c_i) s'_ij over the rows j of gt = Ãᵀ from pass A's per-entry dα
// (tv, Ã order; dz written to tvb in the graph's column-blocked layout, then summed through g->tperm) and
// compact row records: the RECOMP input layer's backward, which needs no dH and so no K-wide transposed
// SpMM (pass B)
granii_status launch_gat_der(const granii_graph_s* g, const granii_graph_s* gt, const float* er, const float* tv,
                             float* tvb, const float4* recs, float* der, cudaStream_t st);
size_t colreduce2_workspace(int64_t R, int64_t K);
// out: 4K floats, [Hᵀd0 | Hᵀd1] as (hi, lo) float pairs: out[0 .. 2K) hi, out[2K .. 4K) lo
granii_status launch_colreduce2(int64_t R, int64_t K, const float* H, int64_t ldh, const float* d0, const float* d1,
                                float* partial, float* out, cudaStream_t st);
granii_status launch_gat_matvec2(int64_t K1, int64_t K2, const float* W, const float* a_l, const float* a_r,
                                float* u, float* v, cudaStream_t st);
granii_status launch_gat_mattvec2(int64_t K1, int64_t K2, const float* W, const float* pq, float* da_l, float* da_r,
                                  cudaStream_t st);
granii_status launch_gat_rank2(int64_t K1, int64_t K2, float* dW, const float* pq, const float* a_l, const float* a_r,
                               cudaStream_t st);
// comm
granii_status comm_allgather(granii_comm_s* c, const float* send, float* recv, size_t count, cudaStream_t st);
granii_status comm_allreduce_sum(granii_comm_s* c, float* buf, size_t count, cudaStream_t st);
granii_status comm_create_local(int32_t world, granii_comm_s** out);
granii_status comm_create_stub(int32_t rank, int32_t world, granii_comm_s** out);
// in-place broadcast of block `root` of a gather buffer (buf_all + root*count) to every rank
granii_status comm_bcast_block(granii_comm_s* c, float* buf_all, size_t count, int root, cudaStream_t st);
// the communicator's side stream and per-block events (created on first use on the current device)
granii_status comm_side(granii_comm_s* c, cudaStream_t* side, cudaEvent_t** ev);
granii_status comm_watchdog(granii_comm_s* c, int64_t timeout_ms);
granii_status comm_check(granii_comm_s* c);
granii_status comm_query(granii_comm_s* c, int32_t* nranks, int32_t* rank, int32_t* version);
granii_status comm_register(granii_comm_s* c, void* buf, size_t bytes, void** handle);
granii_status comm_deregister(granii_comm_s* c, void* handle);
// out[i] = sum_{p < n} src[p][i] in rank order (loopback all-reduce)
granii_status launch_rank_sum(int n, const float* const* src, size_t count, float* out, cudaStream_t st);
granii_status launch_spin(int64_t us, cudaStream_t st);  // test support: one thread spins for `us` microseconds
}  // namespace granii
