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
//    streamed, bytes gathered from L2 vs HBM, flops, launches), with
//    coefficients fitted by NNLS on a B200 calibration sweep
//    (tools/calibrate.py) and built-in defaults derived from B200 peaks.
//    Features come from the integer featurizer computed at graph creation,
//    so selection is host-only and takes microseconds (paper: <= 7 ms, L365).
#include <cmath>
#include <cstdio>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "internal.h"

namespace granii {

// coefficient vectors (ms per unit); feature order documented in features_*()
struct CostModel {
  std::map<std::string, std::vector<double>> coef;
};

static CostModel defaults() {
  CostModel m;
  // spmm: [launch, idx GB, out GB, gathered GB served by L2, gathered GB served by HBM]
  m.coef["spmm"] = {0.006, 1.0 / 6.0, 1.0 / 6.0, 1.0 / 14.0, 1.0 / 4.5};
  // sddmm1 (Ñ or GAT scores; K = 1): [launch, streamed GB]
  m.coef["sddmm1"] = {0.005, 1.0 / 5.5};
  m.coef["sddmm1_softmax"] = {0.006, 1.0 / 5.0};
  // gemm (3xTF32 tcgen05): [launch, HBM GB, TFLOP]
  m.coef["gemm"] = {0.010, 1.0 / 6.0, 1.0 / 250.0};
  // all-gather over NVLink: [launch, GB received per GPU]
  m.coef["allgather"] = {0.020, 1.0 / 700.0};
  return m;
}

static std::mutex g_mu;
static std::map<std::string, CostModel> g_cache;

static granii_status load_model(const char* path, CostModel* out) {
  std::lock_guard<std::mutex> lk(g_mu);
  std::string key = path ? path : "";
  auto it = g_cache.find(key);
  if (it != g_cache.end()) {
    *out = it->second;
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
  *out = m;
  return GRANII_OK;
}

static double dot(const std::vector<double>& c, std::initializer_list<double> f) {
  double s = 0;
  size_t i = 0;
  for (double x : f) s += c[i++] * x;
  return s;
}

struct In {
  double R, nnz, ncols, avg, l2, world;
};

// fraction of gathered bytes served by L2: sliced SpMM keeps the
// slice resident when the graph is dense; otherwise LRU-like hit ~ L2 / |X|.
static double l2_hit(const In& in, double K) {
  const double xbytes = in.ncols * K * 4.0;
  if (xbytes <= 0.8 * in.l2) return 1.0;
  if (in.avg >= 32.0) return 1.0;  // K-sliced
  return std::max(0.0, std::min(1.0, 0.8 * in.l2 / xbytes));
}

double cost_spmm(const CostModel& m, const In& in, double K, bool weighted) {
  const double gb = 1e-9;
  const double gath = in.nnz * K * 4.0 * gb, h = l2_hit(in, K);
  return dot(m.coef.at("spmm"), {1.0, in.nnz * (weighted ? 8.0 : 4.0) * gb, in.R * K * 4.0 * gb, gath * h,
                                 gath * (1.0 - h)});
}
double cost_sddmm1(const CostModel& m, const In& in, bool softmax) {
  const double gb = 1e-9;
  if (softmax) return dot(m.coef.at("sddmm1_softmax"), {1.0, in.nnz * 12.0 * gb});
  return dot(m.coef.at("sddmm1"), {1.0, in.nnz * 8.0 * gb});
}
double cost_gemm(const CostModel& m, const In& in, double K1, double K2, bool store) {
  const double gb = 1e-9;
  return dot(m.coef.at("gemm"), {1.0, in.R * (K1 + (store ? K2 : 0.0)) * 4.0 * gb, 2.0 * in.R * K1 * K2 * 1e-12});
}
double cost_allgather(const CostModel& m, const In& in, double K) {
  if (in.world <= 1) return 0.0;
  return dot(m.coef.at("allgather"), {1.0, in.ncols * K * 4.0 * (in.world - 1) / in.world * 1e-9});
}

double composition_cost(const CostModel& m, const In& in, int comp, double K1, double K2) {
  switch (comp) {
    case GRANII_GCN_PRE_AGG:
      return cost_sddmm1(m, in, false) + cost_allgather(m, in, K1) + cost_spmm(m, in, K1, true) +
             cost_gemm(m, in, K1, K2, true);
    case GRANII_GCN_PRE_UPD:
      return cost_sddmm1(m, in, false) + cost_gemm(m, in, K1, K2, true) + cost_allgather(m, in, K2) +
             cost_spmm(m, in, K2, true);
    case GRANII_GCN_DYN_AGG:
      return cost_allgather(m, in, K1) + cost_spmm(m, in, K1, false) + cost_gemm(m, in, K1, K2, true);
    case GRANII_GCN_DYN_UPD:
      return cost_gemm(m, in, K1, K2, true) + cost_allgather(m, in, K2) + cost_spmm(m, in, K2, false);
    case GRANII_GAT_REUSE:
      return cost_gemm(m, in, K1, K2, true) + cost_allgather(m, in, K2) + cost_sddmm1(m, in, true) +
             cost_spmm(m, in, K2, true);
    case GRANII_GAT_RECOMP:
      return cost_gemm(m, in, K1, K2, false) + cost_allgather(m, in, K1) + cost_sddmm1(m, in, true) +
             cost_spmm(m, in, K1, true) + cost_gemm(m, in, K1, K2, true);
  }
  return 1e30;
}

granii_status select_impl(const granii_graph_s* g, granii_model model, int64_t K1, int64_t K2, const char* path,
                          uint32_t flags, granii_composition* out, int32_t* cands, double* pred, int32_t* ncand) {
  if (!path || !*path) path = getenv("GRANII_CALIB");
  CostModel m;
  GR_TRY(load_model(path, &m));
  DevInfo di;
  if (dev_info(&di) != GRANII_OK) di = DevInfo();  // host-only selection still works
  In in{(double)g->n_rows, (double)g->local_nnz, (double)g->n_cols, g->avg_deg(), (double)di.l2_bytes,
        (double)g->world};
  std::vector<int> c;
  if (model == GRANII_GCN) {
    if (flags & GRANII_SELECT_NO_PREFILTER) c = {GRANII_GCN_PRE_AGG, GRANII_GCN_PRE_UPD, GRANII_GCN_DYN_AGG, GRANII_GCN_DYN_UPD};
    else if (K1 >= K2) c = {GRANII_GCN_PRE_UPD, GRANII_GCN_DYN_UPD};   // group ">=": update first
    else c = {GRANII_GCN_PRE_AGG, GRANII_GCN_DYN_AGG};                 // group "<": aggregate first
  } else {
    c = {GRANII_GAT_REUSE, GRANII_GAT_RECOMP};
  }
  int best = -1;
  double bc = 0;
  for (size_t i = 0; i < c.size(); ++i) {
    const double t = composition_cost(m, in, c[i], (double)K1, (double)K2);
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

}  // namespace granii
