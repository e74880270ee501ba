// select.cpp -- GRANII's online stage on B200 (§IV-D/E, L237-L258).
//
// 1. Embedding-size condition (L237-L239; pruning scenarios L226, reading
//    R11): GCN with K1 >= K2 keeps the update-first trees, K1 < K2 the
//    aggregate-first ones.  GAT keeps both (L330: only K1 < K2 is evaluated,
//    where the choice is input-dependent).
// 2. Cost-model condition (L241): each candidate's cost is the SUM of its
//    primitives' predicted costs; argmin, ties -> lowest composition id (R12).
// 3. Per-primitive cost models (L252-L258).  The paper trains XGBoost models
//    on profiled SuiteSparse graphs; here each primitive has a small linear
//    model over hardware-meaningful features of the featurized input (bytes
//    streamed, bytes gathered from L2 vs HBM, tensor flops, launches), with
//    coefficients fitted by NNLS on a B200 calibration sweep
//    (tools/calibrate.py -> calib/b200.txt) and built-in defaults.  Features
//    come from the integer featurizer computed at graph creation, so selection
//    is host-only and takes microseconds (paper: <= 7 ms, L365).
// Extension (not in the paper, which selects on the forward only, L340):
// GRANII_SELECT_TRAINING adds each composition's backward primitives, and
// GRANII_SELECT_INPUT_LAYER drops the dH branch (not needed for layer 1).
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "internal.h"

namespace granii {

struct CostModel {
  std::map<std::string, std::vector<double>> coef;
};

// feature vectors (all sizes in GB / TFLOP / millions, time in ms)
//   spmm            : [1, streamed GB (idx, weights; per K slice), out GB, gathered GB from L2,
//                      gathered GB from HBM, M rows, thousands of hub segments,
//                      G column-scale gathers (one dependent 4-byte gather per entry and K slice)]
//   sddmm1          : [1, streamed GB, M rows]
//   sddmm1_softmax  : [1, streamed GB, M rows]
//   gemm            : [1, HBM GB, TFLOP, thousands of 128x128 tiles, roofline ms]
//   gemm_att        : [1, HBM GB, TFLOP, thousands of tiles, attention GEMV GB (M x K2 x 4), roofline ms]
//   gemm_tn         : [1, HBM GB, TFLOP, thousands of tiles, roofline ms]
//   gat_bwd_a/b     : [1, streamed GB (idx, er / row records), row GB, gathered GB from L2,
//                      gathered GB from HBM, M rows, M dependent gather steps]  (gat_bwd.cu)
//   elementwise     : [1, GB]
//   allgather       : [1, GB received per GPU]  (the pool this was built on has one GPU: the default
//                     slope is B200_PROFILING.md's measured 8-rank NCCL bus bandwidth on this pool,
//                     725 GB/s; GRANII_ALLGATHER_GBS -- which bench.py sets from an all-gather it
//                     times on the real communicator before selecting -- or an "allgather" line of
//                     the calibration file replaces it)
static CostModel defaults() {
  CostModel m;
  m.coef["spmm"] = {0.006, 1.0 / 6.0, 1.0 / 6.0, 1.0 / 19.0, 1.0 / 5.0, 0.0, 0.0, 1.0};
  m.coef["sddmm1"] = {0.005, 1.0 / 5.5, 0.0};
  m.coef["sddmm1_softmax"] = {0.006, 1.0 / 4.0, 0.0};
  m.coef["gemm"] = {0.010, 1.0 / 3.0, 1.0 / 600.0, 0.0, 0.0};
  m.coef["gemm_att"] = {0.010, 1.0 / 3.0, 1.0 / 600.0, 0.0, 1.0 / 3.0, 0.0};
  m.coef["gemm_tn"] = {0.015, 1.0 / 3.0, 1.0 / 300.0, 0.0, 0.0};
  m.coef["gat_bwd_a"] = {0.008, 1.0 / 5.0, 1.0 / 5.0, 1.0 / 15.0, 1.0 / 4.0, 0.0, 0.0};
  m.coef["gat_bwd_b"] = {0.008, 1.0 / 5.0, 1.0 / 5.0, 1.0 / 15.0, 1.0 / 4.0, 0.0, 0.0};
  // der only (RECOMP input layer): streamed column ids + entry map, one 32-byte sector per dα gather
  m.coef["gat_der"] = {0.010, 1.0 / 6.0, 1.0 / 6.0, 0.0};
  // group-per-row graphs (average degree < 16) run other kernels (spmm.cu k_spmm_group, the
  // lane-group GAT backward passes): their own coefficients (B200 fit: SpMM median error
  // 13 % with one model for both schedules, 9 % / 7 % split)
  m.coef["spmm_g"] = m.coef["spmm"];
  m.coef["gat_bwd_a_g"] = m.coef["gat_bwd_a"];
  m.coef["gat_bwd_b_g"] = m.coef["gat_bwd_b"];
  m.coef["elementwise"] = {0.004, 1.0 / 5.5};
  m.coef["allgather"] = {0.020, 1.0 / 0.725};
  return m;
}

static std::mutex g_mu;
static std::map<std::string, CostModel> g_cache;
static std::string g_last_path;  // calibration of the last selection (used by the phase planner)

// GRANII_ALLGATHER_GBS: all-gather bus bandwidth measured on this job's communicator
static void comm_override(CostModel* m) {
  if (const char* e = getenv("GRANII_ALLGATHER_GBS")) {
    const double gbs = atof(e);
    if (gbs > 0.0) m->coef["allgather"][1] = 1000.0 / gbs;
  }
}

static granii_status load_model(const char* path, CostModel* out) {
  std::lock_guard<std::mutex> lk(g_mu);
  std::string key = path ? path : "";
  auto it = g_cache.find(key);
  if (it != g_cache.end()) {
    *out = it->second;
    comm_override(out);
    if (!key.empty()) g_last_path = key;
    return GRANII_OK;
  }
  CostModel m = defaults();
  if (path && *path) {
    FILE* f = fopen(path, "r");
    if (!f) return fail(GRANII_ERR_NOT_CALIBRATED, std::string("cannot open calibration file ") + path);
    char line[1024];
    while (fgets(line, sizeof line, f)) {
      if (line[0] == '#' || line[0] == '\n') continue;
      char name[64];
      int n = 0;
      if (sscanf(line, "%63s%n", name, &n) != 1) continue;
      std::vector<double> v;
      const char* p = line + n;
      double x;
      int k;
      while (sscanf(p, "%lf%n", &x, &k) == 1) {
        v.push_back(x);
        p += k;
      }
      if (m.coef.count(name) && v.size() == m.coef[name].size()) m.coef[name] = v;
    }
    fclose(f);
  }
  g_cache[key] = m;
  g_last_path = key;
  *out = m;
  comm_override(out);
  return GRANII_OK;
}

struct In {
  double R, nnz, ncols, avg, l2, world, nseg;
  double xcols;  // rows of X an SpMM gathers from (a phased SpMM slices like the whole one: ncols)
  double maxd = 0, seg_len = 2048;  // longest row (featurizer feature 4) and the hub-segment length
  double xld = 0;  // row stride (floats) of the gathered operand when wider than K (TAGCN's Horner hops
                   // gather K2 of every (k+1)K2-wide row of P = H[W_0 .. W_k]); 0: = K
  bool addend = false;  // the SpMM's epilogue adds a dense R x K operand (Horner: + P_j), streamed once
};

static bool overlap_on() {
  const char* e = getenv("GRANII_COMM_OVERLAP");
  return !(e && e[0] == '0');
}

// fraction of gathered bytes served by L2: the sliced SpMM keeps
// a slice resident when the graph is dense; otherwise LRU-like hit ~ L2 / |X|.
// (A popularity-weighted variant -- the top-1 % rows' share of the entries held in L2 first --
// was tried and raised the GAT regret on arxiv-shaped graphs: m5 sweep, 77/79 vs 78/79 within 10 %.)
// A strided operand (xld > K) spreads the gathered rows over xld / K times the address range: the
// touched sectors are the same, but their lines / DRAM pages are shared with the unread columns, so
// the LRU estimate runs over the strided footprint (belgium TAGCN 256->256: the Horner hop over the
// 768-strided P measured 34 % slower than the plain SpMM at K = 256).
static double l2_hit(const In& in, double K, double cols) {
  const double xbytes = cols * std::max(K, in.xld) * 4.0;
  if (xbytes <= 0.8 * in.l2) return 1.0;
  if (in.avg >= 32.0 && cols * 64.0 * 4.0 <= 0.55 * in.l2) return 1.0;  // K-sliced
  return std::max(0.0, std::min(1.0, 0.8 * in.l2 / xbytes));
}

// primitive ids of the feature API
enum { P_SPMM_W = 0, P_SPMM_U = 1, P_SPMM_U_CS = 2, P_SDDMM1 = 3, P_SDDMM1_SM = 4, P_GEMM = 5, P_GEMM_NOSTORE = 6,
       P_GEMM_TN = 7, P_ELEMENTWISE = 8, P_ALLGATHER = 9, P_GEMM_ATT = 10, P_GAT_BWD_A = 11, P_GAT_BWD_B = 12,
       P_GAT_DER = 13 };

// the warp-per-row / group-per-row split follows the kernels' own switch (spmm.cu, gat_bwd.cu)
static bool group_mode(const In& in) { return in.avg < 16.0; }

static const char* prim_model(int p, const In& in) {
  switch (p) {
    case P_SPMM_W: case P_SPMM_U: case P_SPMM_U_CS: return group_mode(in) ? "spmm_g" : "spmm";
    case P_SDDMM1: return "sddmm1";
    case P_SDDMM1_SM: return "sddmm1_softmax";
    case P_GEMM: return "gemm";
    case P_GEMM_NOSTORE: case P_GEMM_ATT: return "gemm_att";
    case P_GEMM_TN: return "gemm_tn";
    case P_ELEMENTWISE: return "elementwise";
    case P_ALLGATHER: return "allgather";
    case P_GAT_BWD_A: return group_mode(in) ? "gat_bwd_a_g" : "gat_bwd_a";
    case P_GAT_BWD_B: return group_mode(in) ? "gat_bwd_b_g" : "gat_bwd_b";
    case P_GAT_DER: return "gat_der";
  }
  return "";
}

static double gemm_roof_ms(double hbm_gb, double tflop) {
  return std::max(hbm_gb / 6.53, tflop * 3.0 / 0.705);
}

// K = width of the primitive (SpMM/SDDMM) or (K1, K2) for the GEMMs
static std::vector<double> features(const In& in, int p, double K1, double K2) {
  const double gb = 1e-9;
  switch (p) {
    case P_SPMM_W: case P_SPMM_U: case P_SPMM_U_CS: {
      const double K = K1, gath = in.nnz * K * 4.0 * gb, h = l2_hit(in, K, in.xcols);
      // every K slice re-streams the column ids (+ weights) and re-gathers the column scale
      // (a dependent 4-byte gather costs a whole 32-byte L2 sector)
      const double sl = (double)spmm_slices(in.avg, in.xcols, (int64_t)K, (int64_t)in.l2);
      const double idx = in.nnz * sl * (4.0 + (p == P_SPMM_W ? 4.0 : 0.0)) * gb + (in.addend ? in.R * K * 4.0 * gb : 0.0);
      return {1.0, idx, in.R * K * 4.0 * gb, gath * h, gath * (1.0 - h), in.R * 1e-6, in.nseg * 1e-3,
              p == P_SPMM_U_CS ? in.nnz * sl * 1e-9 : 0.0};
    }
    case P_SDDMM1: return {1.0, in.nnz * 8.0 * gb, in.R * 1e-6};
    case P_SDDMM1_SM: return {1.0, in.nnz * 16.0 * gb, in.R * 1e-6};
    // GEMMs: the last feature is the roofline time max(HBM GB / 6.53 TB/s, 3xTF32 TFLOP at the tf32 half of
    // the measured 1410 TF/s bf16) in ms -- a tall-skinny GEMM is bound by one or the other, which a sum of
    // the byte and flop terms alone cannot express (arxiv GAT 256->512: the el / er-only GEMM that never
    // stores Θ is no faster than the one that does -- it is tensor-bound)
    case P_GEMM: {
      const double hb = in.R * (K1 + K2) * 4.0 * gb, tf = 2.0 * in.R * K1 * K2 * 1e-12;
      return {1.0, hb, tf, std::ceil(in.R / 128.0) * std::ceil(K2 / 128.0) * 1e-3, gemm_roof_ms(hb, tf)};
    }
    case P_GEMM_ATT: {  // GAT Θ = H W with the el / er GEMVs in the epilogue, Θ stored
      const double hb = in.R * (K1 + K2) * 4.0 * gb, tf = 2.0 * in.R * K1 * K2 * 1e-12;
      return {1.0, hb, tf, std::ceil(in.R / 128.0) * std::ceil(K2 / 128.0) * 1e-3, in.R * K2 * 4.0 * gb,
              gemm_roof_ms(hb, tf)};
    }
    case P_GEMM_NOSTORE: {  // el / er only, Θ never written
      const double hb = in.R * K1 * 4.0 * gb, tf = 2.0 * in.R * K1 * K2 * 1e-12;
      return {1.0, hb, tf, std::ceil(in.R / 128.0) * std::ceil(K2 / 128.0) * 1e-3, in.R * K2 * 4.0 * gb,
              gemm_roof_ms(hb, tf)};
    }
    case P_GEMM_TN: {
      const double hb = in.R * (K1 + K2) * 4.0 * gb, tf = 2.0 * in.R * K1 * K2 * 1e-12;
      return {1.0, hb, tf, std::ceil(K1 / 128.0) * std::ceil(K2 / 128.0) * 1e-3, gemm_roof_ms(hb, tf)};
    }
    case P_GAT_BWD_A: case P_GAT_BWD_B: {
      const double K = K1, gath = in.nnz * K * 4.0 * gb, h = l2_hit(in, K, in.ncols);
      const double idx = in.nnz * (p == P_GAT_BWD_A ? 8.0 : 20.0) * gb;
      // dependent gather steps per warp (gat_bwd.cu: G lane groups x U entries per step)
      const double gu = K <= 16 ? 32 : K <= 32 ? 16 : K <= 128 ? 8 : K <= 256 ? 4 : K <= 512 ? 2 : 1;
      // the longest dependent chain: a whole row on warp-per-row graphs, at most one hub segment
      // on group-per-row graphs (gat_bwd.cu) -- the tail of small power-law graphs
      const double chain = (in.avg >= 16.0 ? in.maxd : std::min(in.maxd, in.seg_len)) / gu;
      return {1.0, idx, in.R * K * (p == P_GAT_BWD_A ? 4.0 : 12.0) * gb, gath * h, gath * (1.0 - h), in.R * 1e-6,
              (in.nnz / gu + 0.5 * in.R) * 1e-6, chain * 1e-3};
    }
    case P_GAT_DER: return {1.0, in.nnz * 8.0 * gb, in.nnz * 32.0 * gb, in.R * 1e-6};
    case P_ELEMENTWISE: return {1.0, in.R * K1 * 12.0 * gb};
    case P_ALLGATHER: return {1.0, in.ncols * K1 * 4.0 * (in.world - 1) / std::max(in.world, 1.0) * gb};
  }
  return {};
}

static double cost(const CostModel& m, const In& in, int p, double K1, double K2 = 0) {
  if (p == P_ALLGATHER && in.world <= 1) return 0.0;
  const std::vector<double> f = features(in, p, K1, K2);
  const std::vector<double>& c = m.coef.at(prim_model(p, in));
  double s = 0;
  for (size_t i = 0; i < f.size() && i < c.size(); ++i) s += c[i] * f[i];
  return s;
}

// All-gather of a K-wide operand followed by its aggregation, on G > 1 GPUs (layer.cu
// gathered_spmm).  P = 1: all-gather, then one SpMM.  P >= 2 (overlapped): the G blocks are
// broadcast in rank order on a side stream (landing uniformly over the transfer time); the SpMM
// runs the own block first, then the other G-1 blocks in P-1 chunks, each chunk once its last
// block has landed.  Every phase after the first re-reads and re-writes the partial output rows
// (plus a launch).  Returns the predicted time of the best P (rank-independent inputs, so every
// rank plans the same schedule) and that P.
static double agg_schedule(const CostModel& m, const In& in, int p, double K, int* best_P) {
  const double sp = cost(m, in, p, K);
  if (best_P) *best_P = 1;
  if (in.world <= 1) return sp;
  const double ag = cost(m, in, P_ALLGATHER, K);
  double best = ag + sp;
  if (!overlap_on()) return best;
  const int G = (int)in.world;
  const std::vector<double>& c = m.coef.at(prim_model(P_SPMM_U, in));
  // a phase over n of the G owner blocks: the entries whose columns lie in them (n / G of them,
  // every row visited: the model's per-row term stays whole) gathering from an n / G slice of the
  // operand -- the own block alone (1 / G of X) often fits L2 where the whole X does not (G = 8
  // products-shaped projection: 2 phases 2.66 ms of per-rank compute vs 3.07 ms unphased,
  // profiles/r02/scaling_projection_products-gcn2-infer_P*.json); every phase after the first
  // adds ~40 us of launch + tail per K slice and re-reads + re-writes the partial output rows
  auto phase = [&](double n) {
    In b = in;
    b.nnz = in.nnz * n / G;
    b.xcols = in.xcols * n / G;
    b.nseg = in.nseg * n / G;
    return cost(m, b, p, K);
  };
  double slices = 1.0;
  if (in.avg >= 32.0 && in.ncols * K * 4.0 > 0.6 * in.l2) {
    const double fit = std::floor(0.55 * in.l2 / (in.ncols * 4.0) / 64.0) * 64.0;
    if (fit >= 64.0) slices = std::ceil(K / fit);
  }
  const double h = 0.040 * slices + 2.0 * in.R * K * 4.0 * 1e-9 * c[2];
  for (int P = 2; P <= G; ++P) {
    double t = phase(1.0);  // own block, under the transfer
    int done = 0;
    for (int q = 0; q < P - 1; ++q) {
      const int n = (G - 1) * (q + 1) / (P - 1) - (G - 1) * q / (P - 1);  // blocks in this chunk
      done += n;
      const double landed = ag * (double)done / (G - 1);
      t = std::max(t, landed) + phase((double)n) + h;
    }
    if (t < best) {
      best = t;
      if (best_P) *best_P = P;
    }
  }
  return best;
}

static double agg_cost(const CostModel& m, const In& in, int p, double K) { return agg_schedule(m, in, p, K, nullptr); }

double forward_cost(const CostModel& m, const In& in, int comp, double K1, double K2) {
  switch (comp) {
    case GRANII_GCN_PRE_AGG:
      return cost(m, in, P_SDDMM1, 0) + agg_cost(m, in, P_SPMM_W, K1) + cost(m, in, P_GEMM, K1, K2);
    case GRANII_GCN_PRE_UPD:
      return cost(m, in, P_SDDMM1, 0) + cost(m, in, P_GEMM, K1, K2) + agg_cost(m, in, P_SPMM_W, K2);
    case GRANII_GCN_DYN_AGG:  // pre-scale fused in the gather, or its own row-broadcast pass (layer.cu)
      if (dyn_prescale(in.nnz, in.R, in.avg, in.xcols, (int64_t)K1, (int64_t)in.l2))
        return cost(m, in, P_ELEMENTWISE, K1) + agg_cost(m, in, P_SPMM_U, K1) + cost(m, in, P_GEMM, K1, K2);
      return agg_cost(m, in, P_SPMM_U_CS, K1) + cost(m, in, P_GEMM, K1, K2);
    case GRANII_GCN_DYN_UPD:
      return cost(m, in, P_GEMM, K1, K2) + agg_cost(m, in, P_SPMM_U, K2);
    case GRANII_GAT_REUSE:
    case GRANII_GAT_RECOMP: {
      // warp-per-row graph with a single-all-gather schedule: scores + softmax fused into the
      // aggregation (layer.cu), whose per-entry er gather is modelled like the column-scale gather
      // of the unweighted SpMM; otherwise SDDMM + row softmax, then the (possibly phased) SpMM
      const bool reuse = comp == GRANII_GAT_REUSE;
      const double K = reuse ? K2 : K1;
      const double pre = cost(m, in, reuse ? P_GEMM_ATT : P_GEMM_NOSTORE, K1, K2) + cost(m, in, P_ALLGATHER, 1);
      const double post = reuse ? 0.0 : cost(m, in, P_GEMM, K1, K2);
      int P = 1;
      const double agg = agg_schedule(m, in, P_SPMM_W, K, &P);
      if (P <= 1 && in.avg >= 16.0 && gat_fused_enabled())
        return pre + cost(m, in, P_ALLGATHER, K) + cost(m, in, P_SPMM_U_CS, K) + post;
      return pre + cost(m, in, P_SDDMM1_SM, 0) + agg + post;
    }
  }
  return 1e30;
}

// SGC / TAGCN / GIN (layer.cu ext_forward_impl; reading R23): k hops of the GCN SpMM (with an
// all-gather before each on several GPUs), TAGCN's concatenated GEMM (AGG) or wide GEMM (UPD),
// GIN's two MLP GEMMs around one aggregation at K1 (AGG) or Kh (UPD)
double ext_forward_cost(const CostModel& m, const In& in, int comp, double K1, double K2, double k, double Kh) {
  const bool dyn = (comp & 3) >= 2, upd = (comp & 1) != 0;
  const int base = comp & ~3;
  int sp = base == GRANII_GIN_PRE_AGG ? (dyn ? P_SPMM_U : P_SPMM_W) : (dyn ? P_SPMM_U_CS : P_SPMM_W);
  double t = dyn ? 0.0 : cost(m, in, P_SDDMM1, 0);
  if (base == GRANII_SGC_PRE_AGG) {
    const double K = upd ? K2 : K1;
    if (dyn && k > 0 && dyn_prescale(in.nnz, in.R, in.avg, in.xcols, (int64_t)K, (int64_t)in.l2)) {
      sp = P_SPMM_U;                               // pre-scaled hop inputs (layer.cu sgc_hop)
      if (!upd) t += cost(m, in, P_ELEMENTWISE, K1);  // UPD: fused in the GEMM epilogue
    }
    t += cost(m, in, P_GEMM, K1, K2) + k * (cost(m, in, P_ALLGATHER, K) + cost(m, in, sp, K));
  } else if (base == GRANII_TAGCN_PRE_AGG) {
    if (upd) {
      In h = in;
      h.xld = (k + 1) * K2;  // Horner: Z = S Z + P_j reads P's j-th K2 block (layer.cu)
      h.addend = true;
      t += cost(m, in, P_GEMM, K1, (k + 1) * K2) + k * (cost(m, in, P_ALLGATHER, K2) + cost(m, h, sp, K2));
    }
    else if (dyn && k > 0 && dyn_prescale(in.nnz, in.R, in.avg, in.xcols, (int64_t)K1, (int64_t)in.l2))
      // pre-scaled hop inputs (layer.cu pre_t): a row-broadcast pass before every hop
      t += cost(m, in, P_ELEMENTWISE, K1) * (k + 1) + k * (cost(m, in, P_ALLGATHER, K1) + cost(m, in, P_SPMM_U, K1)) +
           cost(m, in, P_GEMM, (k + 1) * K1, K2);
    else
      t += cost(m, in, P_ELEMENTWISE, K1) + k * (cost(m, in, P_ALLGATHER, K1) + cost(m, in, sp, K1)) +
           cost(m, in, P_GEMM, (k + 1) * K1, K2);
  } else {
    const double K = upd ? Kh : K1;
    t += cost(m, in, P_GEMM, K1, Kh) + cost(m, in, P_GEMM, Kh, K2) + cost(m, in, P_ALLGATHER, K) + cost(m, in, sp, K);
  }
  return t;
}

// backward of the compositions (layer.cu backward_impl / gat_backward_impl), ReLU mask included
double backward_cost(const CostModel& m, const In& in, int comp, double K1, double K2, bool need_dH) {
  double t = cost(m, in, P_ELEMENTWISE, K2) + cost(m, in, P_GEMM_TN, K1, K2);
  switch (comp) {
    case GRANII_GCN_PRE_AGG:
      t += cost(m, in, P_SDDMM1, 0);
      if (need_dH) t += cost(m, in, P_GEMM, K2, K1) + agg_cost(m, in, P_SPMM_W, K1);
      break;
    case GRANII_GCN_PRE_UPD:
      t += cost(m, in, P_SDDMM1, 0) + agg_cost(m, in, P_SPMM_W, K2);
      if (need_dH) t += cost(m, in, P_GEMM, K2, K1);
      break;
    case GRANII_GCN_DYN_AGG:
      if (need_dH) t += cost(m, in, P_GEMM, K2, K1) + agg_cost(m, in, P_SPMM_U, K1);
      break;
    case GRANII_GCN_DYN_UPD:
      t += agg_cost(m, in, P_SPMM_U, K2);  // inner D fused in the ReLU' pass
      if (need_dH) t += cost(m, in, P_GEMM, K2, K1);
      break;
    case GRANII_GAT_REUSE:  // gat_backward_impl: prep ; A, B at K2 ; dW = Hᵀ dΘ ; (dH = dΘ Wᵀ) ; Hᵀ[del, der]
      t += cost(m, in, P_ALLGATHER, K2) * 2.0 + cost(m, in, P_GAT_BWD_A, K2) + cost(m, in, P_GAT_BWD_B, K2) +
           cost(m, in, P_ELEMENTWISE, K1);
      if (need_dH) t += cost(m, in, P_GEMM, K2, K1);
      break;
    case GRANII_GAT_RECOMP:  // prep ; dT = dY Wᵀ ; A, B at K1 (B writes dH) ; dW = Tᵀ dY ; Hᵀ[del, der]
      // (one GPU, no dH: der from pass A's per-entry dα instead of pass B, layer.cu der_only)
      t += cost(m, in, P_GEMM, K2, K1) + cost(m, in, P_ALLGATHER, K1) * 2.0 + cost(m, in, P_GAT_BWD_A, K1) +
           (need_dH || in.world > 1 ? cost(m, in, P_GAT_BWD_B, K1) : cost(m, in, P_GAT_DER, 0)) +
           cost(m, in, P_ELEMENTWISE, K1);
      break;
    default:
      return 0.0;
  }
  return t;
}

// On a partitioned graph every rank must choose the SAME composition (the compositions issue
// different collectives), so the inputs are the whole graph's, averaged per rank -- never this
// rank's own rows.
static In inputs_of(const granii_graph_s* g) {
  DevInfo di;
  if (dev_info(&di) != GRANII_OK) di = DevInfo();  // host-only selection still works
  if (g->world > 1) {
    const double G = (double)g->world, N = (double)g->N, nnz = (double)g->nnz;
    return In{N / G, nnz / G, (double)g->n_cols, N > 0 ? nnz / N : 0.0, (double)di.l2_bytes, G,
              (double)std::max<int64_t>(g->n_seg_global, 0) / G, (double)g->n_cols, (double)g->features[4],
              (double)g->seg_len};
  }
  return In{(double)g->n_rows, (double)g->local_nnz, (double)g->n_cols, g->avg_deg(), (double)di.l2_bytes,
            (double)g->world, (double)g->n_seg, (double)g->n_cols, (double)g->features[4], (double)g->seg_len};
}

granii_status select_impl(const granii_graph_s* g, granii_model model, const granii_layer_args* shape,
                          const char* path, uint32_t flags, granii_composition* out, int32_t* cands, double* pred,
                          int32_t* ncand) {
  const int64_t K1 = shape->K1, K2 = shape->K2;
  if (!path || !*path) path = getenv("GRANII_CALIB");
  CostModel m;
  GR_TRY(load_model(path, &m));
  const In in = inputs_of(g);
  std::vector<int> c;
  // the embedding-size rule is a forward-only argument (narrower SpMM); with the
  // backward in the cost (and no dH on the input layer) it no longer holds, so the
  // training selection keeps all four GCN trees and lets the cost models decide
  const bool prefilter = !(flags & (GRANII_SELECT_NO_PREFILTER | GRANII_SELECT_TRAINING));
  if (model == GRANII_GCN) {
    if (!prefilter) c = {GRANII_GCN_PRE_AGG, GRANII_GCN_PRE_UPD, GRANII_GCN_DYN_AGG, GRANII_GCN_DYN_UPD};
    else if (K1 >= K2) c = {GRANII_GCN_PRE_UPD, GRANII_GCN_DYN_UPD};   // group ">=": update first
    else c = {GRANII_GCN_PRE_AGG, GRANII_GCN_DYN_AGG};                 // group "<": aggregate first
  } else if (model == GRANII_GAT) {
    // offline pruning (offline.py, L226-L233): RECOMP -- the extra GEMM and an SpMM at K1 -- is
    // unprofitable when K1 >= K2 (it does all of REUSE's work on matrices never smaller, and more)
    if (!prefilter || K1 < K2) c = {GRANII_GAT_REUSE, GRANII_GAT_RECOMP};
    else c = {GRANII_GAT_REUSE};
  } else {
    // SGC / TAGCN: the GCN embedding-size rule on (K1, K2); GIN: on (K1, Kh), the width the
    // aggregation runs at (R11 / R23)
    const int base = model == GRANII_SGC ? GRANII_SGC_PRE_AGG : model == GRANII_TAGCN ? GRANII_TAGCN_PRE_AGG
                                                                                         : GRANII_GIN_PRE_AGG;
    const int64_t Kout = model == GRANII_GIN ? shape->Kh : K2;
    // TAGCN at K1 == K2 (reading R28): AGG runs k plain hops at K1 and the (k+1)K1 x K2 GEMM, UPD the
    // K1 x (k+1)K2 GEMM and k Horner hops with a fused addend over a strided operand -- equal sizes,
    // different primitives, so the size rule ranks neither and the cost models decide
    if (!prefilter || (model == GRANII_TAGCN && K1 == Kout)) c = {base, base + 1, base + 2, base + 3};
    else if (K1 >= Kout) c = {base + 1, base + 3};
    else c = {base, base + 2};
  }
  const bool train = (flags & GRANII_SELECT_TRAINING) != 0 && model <= GRANII_GAT;
  const bool need_dH = !(flags & GRANII_SELECT_INPUT_LAYER);
  int best = -1;
  double bc = 0;
  for (size_t i = 0; i < c.size(); ++i) {
    double t = model <= GRANII_GAT
                   ? forward_cost(m, in, c[i], (double)K1, (double)K2)
                   : ext_forward_cost(m, in, c[i], (double)K1, (double)K2, (double)shape->hops, (double)shape->Kh);
    if (train) t += backward_cost(m, in, c[i], (double)K1, (double)K2, need_dH);
    if (cands) cands[i] = c[i];
    if (pred) pred[i] = t;
    if (best < 0 || t < bc) {  // strict: ties keep the lower id (candidates are in id order)
      best = c[i];
      bc = t;
    }
  }
  if (ncand) *ncand = (int32_t)c.size();
  *out = (granii_composition)best;
  return GRANII_OK;
}

// number of phases of an overlapped aggregation (1 = all-gather then SpMM); GRANII_COMM_PHASES
// overrides.  weighted / col_scale pick the SpMM model (P_SPMM_W / P_SPMM_U_CS / P_SPMM_U).
int comm_phases(const granii_graph_s* g, int64_t K, bool weighted, bool col_scale) {
  return comm_plan(g, K, weighted, col_scale, nullptr, nullptr);
}

// the planner's choice and its predicted times (P = 1 and the chosen P), for diagnostics
int comm_plan(const granii_graph_s* g, int64_t K, bool weighted, bool col_scale, double* t1, double* tp) {
  if (t1) *t1 = 0.0;
  if (tp) *tp = 0.0;
  if (g->world <= 1) return 1;
  if (const char* e = getenv("GRANII_COMM_PHASES")) {
    const int P = atoi(e);
    if (P >= 1) return std::min(P, (int)g->world);
  }
  std::string path;
  {
    std::lock_guard<std::mutex> lk(g_mu);
    path = g_last_path;
  }
  if (path.empty() && getenv("GRANII_CALIB")) path = getenv("GRANII_CALIB");
  CostModel m;
  if (load_model(path.empty() ? nullptr : path.c_str(), &m) != GRANII_OK) m = defaults();
  int P = 1;
  const In in = inputs_of(g);
  const int prim = weighted ? P_SPMM_W : col_scale ? P_SPMM_U_CS : P_SPMM_U;
  const double best = agg_schedule(m, in, prim, (double)K, &P);
  if (t1) *t1 = cost(m, in, P_ALLGATHER, (double)K) + cost(m, in, prim, (double)K);
  if (tp) *tp = best;
  return P;
}

granii_status cost_features_impl(const granii_graph_s* g, int32_t prim, int64_t K1, int64_t K2, double* feats,
                                 int32_t* n, char* model_name) {
  if (prim < P_SPMM_W || prim > P_GAT_DER) return fail(GRANII_ERR_INVALID_ARG, "unknown primitive id");
  const std::vector<double> f = features(inputs_of(g), prim, (double)K1, (double)K2);
  for (size_t i = 0; i < f.size(); ++i) feats[i] = f[i];
  *n = (int32_t)f.size();
  if (model_name) {
    strncpy(model_name, prim_model(prim, inputs_of(g)), 31);
    model_name[31] = 0;
  }
  return GRANII_OK;
}

}  // namespace granii
