/*
 * granii_oracle.c -- TEST INFRASTRUCTURE ONLY (not part of the product path).
 *
 * A plain, slow, obviously-correct fp64 CPU implementation of the GRANII hot
 * path (Lenadora et al., "GRANII: Selection and Ordering of Primitives in
 * GRAph Neural Networks using Input Inspection", CGO'26; /root/reference/PAPER.md,
 * cited as Lnnn = line nnn).  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.  It
 * shares no code, header, table or helper with the CUDA library under
 * paper_conf_cgo_lenadorasgytm26_b200/csrc, and neither includes the other.
 *
 * Every function follows the paper's primitive order literally: row-broadcasts
 * (Eq. 1) are separate passes, SDDMM / SpMM / GEMM are the textbook loops, and
 * every sparse reduction runs in CSR order.  OpenMP parallelises over output
 * rows only, so each output element is computed by one thread in one fixed
 * order (results do not depend on the thread count).
 *
 * Readings of the paper where it is silent/garbled are DESIGN.md §2 (R1..R18);
 * they are cited below as [Rn].
 *
 * Parity pins: see tests/test_oracle_pins.py.  Every function here is pinned
 * (brute-force dense products, closed forms, finite differences, invariants);
 * none is "parity unpinned".
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OR_ADD_SELF_LOOPS 0x1u  /* Ã = pattern(A ∪ I), L113 [R2]            */
#define OR_SYMMETRIZE 0x2u      /* undirected input: add (v,u) for (u,v) L328 */

/* composition ids (Fig. 3 is an image, reading [R10]) */
enum { OR_GCN_PRE_AGG = 0, OR_GCN_PRE_UPD = 1, OR_GCN_DYN_AGG = 2, OR_GCN_DYN_UPD = 3,
       OR_GAT_REUSE = 16, OR_GAT_RECOMP = 17 };

/* ------------------------------------------------------------------------ */
/* O1: graph ingest -> CSR of Ã (integer, bit-exact contract)                */
/* L113 "Ã is the adjacency matrix of the input graph with self-edges";      */
/* L192 messages flow source -> destination and are summed at the destination */
/* => row = destination, column = source [R1]; duplicates removed [R3].      */
/* ------------------------------------------------------------------------ */
static int cmp_u64(const void* a, const void* b) {
  uint64_t x = *(const uint64_t*)a, y = *(const uint64_t*)b;
  return (x > y) - (x < y);
}

/* returns 0 on success, 1 on invalid ids, 2 on capacity/alloc failure */
int oracle_csr_build(int64_t N, int64_t E, const int32_t* src, const int32_t* dst, uint32_t flags,
                     int64_t* row_ptr /* N+1 */, int32_t* col_idx, int64_t cap, int64_t* nnz_out) {
  for (int64_t e = 0; e < E; ++e)
    if (src[e] < 0 || src[e] >= N || dst[e] < 0 || dst[e] >= N) return 1;
  int64_t M = E + ((flags & OR_SYMMETRIZE) ? E : 0) + ((flags & OR_ADD_SELF_LOOPS) ? N : 0);
  uint64_t* key = (uint64_t*)malloc((size_t)(M > 0 ? M : 1) * sizeof(uint64_t));
  if (!key) return 2;
  int64_t m = 0;
  for (int64_t e = 0; e < E; ++e) {
    key[m++] = ((uint64_t)(uint32_t)dst[e] << 32) | (uint32_t)src[e];       /* (row=dst, col=src) */
    if (flags & OR_SYMMETRIZE) key[m++] = ((uint64_t)(uint32_t)src[e] << 32) | (uint32_t)dst[e];
  }
  if (flags & OR_ADD_SELF_LOOPS)
    for (int64_t i = 0; i < N; ++i) key[m++] = ((uint64_t)i << 32) | (uint64_t)i;
  qsort(key, (size_t)m, sizeof(uint64_t), cmp_u64);
  for (int64_t i = 0; i <= N; ++i) row_ptr[i] = 0;
  int64_t nnz = 0;
  for (int64_t t = 0; t < m; ++t) {
    if (t > 0 && key[t] == key[t - 1]) continue;                           /* dedupe */
    if (nnz >= cap) { free(key); return 2; }
    int64_t r = (int64_t)(key[t] >> 32);
    col_idx[nnz++] = (int32_t)(key[t] & 0xffffffffu);
    row_ptr[r + 1] += 1;                                                   /* |row r| */
  }
  for (int64_t i = 0; i < N; ++i) row_ptr[i + 1] += row_ptr[i];            /* prefix sum */
  *nnz_out = nnz;
  free(key);
  return 0;
}

/* O2: nnz-balanced contiguous row partition [proposal; the paper is single-device,
 * L266-L270]: b_0 = 0, b_G = N, b_g = min{ r : row_ptr[r] >= ceil(g*nnz/G) }. */
void oracle_partition(int64_t N, const int64_t* row_ptr, int64_t G, int64_t* bounds) {
  int64_t nnz = row_ptr[N];
  bounds[0] = 0;
  bounds[G] = N;
  for (int64_t g = 1; g < G; ++g) {
    int64_t target = (g * nnz + G - 1) / G;
    int64_t r = 0;
    while (r < N && row_ptr[r] < target) ++r;                              /* linear lower_bound */
    bounds[g] = r;
  }
}

/* O8: integer features of the input featurizer (L252-L256; Appendix E absent [R16]).
 * out[0]=N, [1]=nnz, [2]=sum deg, [3]=sum deg^2, [4]=max deg, [5]=min deg,
 * [6]=nnz held by the ceil(N/100) highest-degree rows, [7]=#rows with deg 0. */
void oracle_features(int64_t N, const int64_t* row_ptr, int64_t* out) {
  int64_t s = 0, s2 = 0, mx = 0, mn = N > 0 ? INT64_MAX : 0, z = 0;
  int64_t* deg = (int64_t*)malloc((size_t)(N > 0 ? N : 1) * sizeof(int64_t));
  for (int64_t i = 0; i < N; ++i) {
    int64_t d = row_ptr[i + 1] - row_ptr[i];
    deg[i] = d;
    s += d; s2 += d * d;
    if (d > mx) mx = d;
    if (d < mn) mn = d;
    if (d == 0) z++;
  }
  /* top-1% share: sort the degrees ascending, sum the last ceil(N/100) */
  qsort(deg, (size_t)N, sizeof(int64_t), cmp_u64);   /* degrees are >= 0: unsigned order == signed */
  int64_t k = (N + 99) / 100, top = 0;
  for (int64_t t = 0; t < k && t < N; ++t) top += deg[N - 1 - t];
  free(deg);
  out[0] = N; out[1] = row_ptr[N]; out[2] = s; out[3] = s2; out[4] = mx; out[5] = mn;
  out[6] = top; out[7] = z;
}

/* a3: D̃^{-1/2}: dinv_i = deg_i^{-1/2} (Eq. 2, Eq. 3); deg = row nnz of Ã [R4];
 * dinv = 0 when deg = 0 [R5]. */
void oracle_dinv(int64_t n_rows, const int64_t* row_ptr, double* dinv) {
  for (int64_t i = 0; i < n_rows; ++i) {
    int64_t d = row_ptr[i + 1] - row_ptr[i];
    dinv[i] = d > 0 ? 1.0 / sqrt((double)d) : 0.0;
  }
}

/* Eq. (1) row-broadcast, L82-L84: c_ij = d_i * b_ij */
void oracle_rowbcast(int64_t M, int64_t K, const double* d, const double* B, double* C) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < M; ++i)
    for (int64_t j = 0; j < K; ++j) C[i * K + j] = d[i] * B[i * K + j];
}

/* g-SDDMM (+,x), L88 "a standard matrix multiplication guided by a sparse mask":
 * out_e = sum_k U[r(e),k] * V[c(e),k] for every stored e = (r, c). */
void oracle_sddmm(int64_t n_rows, const int64_t* row_ptr, const int32_t* col_idx, const double* U,
                  const double* V, int64_t K, double* out) {
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t r = 0; r < n_rows; ++r)
    for (int64_t e = row_ptr[r]; e < row_ptr[r + 1]; ++e) {
      double s = 0.0;
      for (int64_t k = 0; k < K; ++k) s += U[r * K + k] * V[(int64_t)col_idx[e] * K + k];
      out[e] = s;
    }
}

/* g-SpMM (+,x), L88/L92: Y_r = sum_{e in row r} w_e * X[c(e)], CSR order.
 * vals == NULL is the unweighted ("copy") aggregation of L117 / Appendix B. */
void oracle_spmm(int64_t n_rows, const int64_t* row_ptr, const int32_t* col_idx, const double* vals,
                 const double* X, int64_t K, double* Y) {
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t r = 0; r < n_rows; ++r) {
    double* y = Y + r * K;
    for (int64_t k = 0; k < K; ++k) y[k] = 0.0;
    for (int64_t e = row_ptr[r]; e < row_ptr[r + 1]; ++e) {
      double w = vals ? vals[e] : 1.0;
      const double* x = X + (int64_t)col_idx[e] * K;
      for (int64_t k = 0; k < K; ++k) y[k] += w * x[k];
    }
  }
}

/* transpose SpMM: Y = Sᵀ X, i.e. Y_c += w_e * X_r for every stored e = (r, c).
 * Written as the scatter it is (used by the backward pass only): every output
 * element receives its terms in stored-entry order; threads own disjoint column
 * ranges k of Y, so the order per element is the serial scatter's. */
void oracle_spmm_t(int64_t n_rows, int64_t n_cols, const int64_t* row_ptr, const int32_t* col_idx,
                   const double* vals, const double* X, int64_t K, double* Y) {
  for (int64_t i = 0; i < n_cols * K; ++i) Y[i] = 0.0;
  const int64_t kc = 8;  /* column range per task */
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t k0 = 0; k0 < K; k0 += kc) {
    const int64_t k1 = k0 + kc < K ? k0 + kc : K;
    for (int64_t r = 0; r < n_rows; ++r)
      for (int64_t e = row_ptr[r]; e < row_ptr[r + 1]; ++e) {
        double w = vals ? vals[e] : 1.0;
        for (int64_t k = k0; k < k1; ++k) Y[(int64_t)col_idx[e] * K + k] += w * X[r * K + k];
      }
  }
}

/* GEMM, L80-L82 / L92: C = op(A) * op(B), plain triple loop, row-major.
 * op(A) is M x K (A stored K x M when ta), op(B) is K x N (B stored N x K when tb).
 * C[i][j] = sum over k = 0..K-1, in that order, of op(A)[i][k] * op(B)[k][j]; the
 * k loop runs outside the j loop (a row of partial sums per i) so that op(B) is
 * read row by row -- the same products summed in the same order. */
void oracle_gemm(int64_t M, int64_t N, int64_t K, const double* A, int ta, const double* B, int tb,
                 double* C) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < M; ++i) {
    double* s = C + i * N;
    for (int64_t j = 0; j < N; ++j) s[j] = 0.0;
    for (int64_t k = 0; k < K; ++k) {
      double a = ta ? A[k * M + i] : A[i * K + k];
      for (int64_t j = 0; j < N; ++j) {
        double b = tb ? B[j * K + k] : B[k * N + j];
        s[j] += a * b;
      }
    }
  }
}

/* sigma [R7]: act = 0 identity, 1 ReLU (no bias: Eq. 2/3/5 have none) */
static void act_inplace(int64_t n, double* y, int act) {
  if (act == 1)
    for (int64_t i = 0; i < n; ++i) y[i] = y[i] > 0.0 ? y[i] : 0.0;
}

/* ------------------------------------------------------------------------ */
/* O3: GCN forward under each composition.  All four reach the same value    */
/* D̃^{-1/2} Ã D̃^{-1/2} H W (L192: only semantically equivalent re-associations). */
/*   PRE_*  : Eq. (3), Ñ = D̃^{-1/2} Ã D̃^{-1/2} by SDDMM (L41, L119)      */
/*   DYN_*  : Eq. (2), two row-broadcasts + unweighted SpMM (L113, L117)  */
/*   *_AGG / *_UPD: aggregate (SpMM) first or update (GEMM) first (L98, L305)  */
/* y_pre receives the pre-activation Y (N x K2), out = sigma(Y).              */
/* ------------------------------------------------------------------------ */
int oracle_gcn_forward(int comp, int64_t N, const int64_t* row_ptr, const int32_t* col_idx,
                       const double* H, int64_t K1, const double* W, int64_t K2, int act,
                       double* y_pre, double* out) {
  int64_t nnz = row_ptr[N];
  double* dinv = (double*)malloc((size_t)(N ? N : 1) * sizeof(double));
  oracle_dinv(N, row_ptr, dinv);
  int64_t Kmax = K1 > K2 ? K1 : K2;
  double* t1 = (double*)malloc((size_t)(N * Kmax + 1) * sizeof(double));
  double* t2 = (double*)malloc((size_t)(N * Kmax + 1) * sizeof(double));
  double* nval = NULL;
  if (comp == OR_GCN_PRE_AGG || comp == OR_GCN_PRE_UPD) {
    nval = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
    oracle_sddmm(N, row_ptr, col_idx, dinv, dinv, 1, nval);                /* Ñ = D Ã D (K = 1) */
  }
  switch (comp) {
    case OR_GCN_PRE_AGG:                                                   /* (Ñ H) W */
      oracle_spmm(N, row_ptr, col_idx, nval, H, K1, t1);
      oracle_gemm(N, K2, K1, t1, 0, W, 0, y_pre);
      break;
    case OR_GCN_PRE_UPD:                                                   /* Ñ (H W) */
      oracle_gemm(N, K2, K1, H, 0, W, 0, t1);
      oracle_spmm(N, row_ptr, col_idx, nval, t1, K2, y_pre);
      break;
    case OR_GCN_DYN_AGG:                                                   /* (D (Ã (D H))) W */
      oracle_rowbcast(N, K1, dinv, H, t1);
      oracle_spmm(N, row_ptr, col_idx, NULL, t1, K1, t2);
      oracle_rowbcast(N, K1, dinv, t2, t1);
      oracle_gemm(N, K2, K1, t1, 0, W, 0, y_pre);
      break;
    case OR_GCN_DYN_UPD:                                                   /* D (Ã (D (H W))) */
      oracle_gemm(N, K2, K1, H, 0, W, 0, t1);
      oracle_rowbcast(N, K2, dinv, t1, t2);
      oracle_spmm(N, row_ptr, col_idx, NULL, t2, K2, t1);
      oracle_rowbcast(N, K2, dinv, t1, y_pre);
      break;
    default:
      free(dinv); free(t1); free(t2); free(nval);
      return 1;
  }
  memcpy(out, y_pre, (size_t)(N * K2) * sizeof(double));
  act_inplace(N * K2, out, act);
  free(dinv); free(t1); free(t2); free(nval);
  return 0;
}

/* Per-row definition of the GCN layer for sampled rows of a large graph:
 * Y_i = (sum_j Ñ_ij H_j) W with Ñ_ij = dinv_i dinv_j (Eq. 3 read row by row).
 * Rows are local indices into (row_ptr, col_idx); H is indexed by column id. */
void oracle_gcn_rows(int64_t n_sample, const int64_t* rows, const int64_t* row_ptr, const int32_t* col_idx,
                     const int64_t* deg_of_col /* deg of every column id */, const double* H, int64_t K1,
                     const double* W, int64_t K2, int act, double* out /* n_sample x K2 */) {
#pragma omp parallel for schedule(dynamic, 4)
  for (int64_t s = 0; s < n_sample; ++s) {
    int64_t r = rows[s];
    int64_t dr = row_ptr[r + 1] - row_ptr[r];
    double di = dr > 0 ? 1.0 / sqrt((double)dr) : 0.0;
    double* agg = (double*)calloc((size_t)K1, sizeof(double));
    for (int64_t e = row_ptr[r]; e < row_ptr[r + 1]; ++e) {
      int64_t c = col_idx[e];
      double dj = deg_of_col[c] > 0 ? 1.0 / sqrt((double)deg_of_col[c]) : 0.0;
      for (int64_t k = 0; k < K1; ++k) agg[k] += di * dj * H[c * K1 + k];
    }
    for (int64_t j = 0; j < K2; ++j) {
      double v = 0.0;
      for (int64_t k = 0; k < K1; ++k) v += agg[k] * W[k * K2 + j];
      out[s * K2 + j] = (act == 1 && v < 0.0) ? 0.0 : v;
    }
    free(agg);
  }
}

/* ------------------------------------------------------------------------ */
/* O4: GAT forward.  Atten() is opaque in the paper (L127, Eq. 4); reading   */
/* [R8] = single-head GAT of [25] (L499):                                    */
/*   Θ = H W ; el_i = Θ_i·a_l ; er_j = Θ_j·a_r                               */
/*   additive: e_ij = LeakyReLU_0.2(el_i + er_j)                             */
/*   dot [R9, proposal]: e_ij = <Θ_i, Θ_j> / sqrt(K2)                        */
/*   α_ij = exp(e_ij - m_i) / Σ_j' exp(e_ij' - m_i)   (row softmax incl. loop) */
/* REUSE (Eq. 5): Y = α Θ.  RECOMP (Eq. 6): Y = (α H) W.          */
/* alpha_out (nullable) receives α.                                          */
/* ------------------------------------------------------------------------ */
void oracle_edge_softmax(int64_t n_rows, const int64_t* row_ptr, const double* e, double* alpha) {
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t r = 0; r < n_rows; ++r) {
    int64_t b = row_ptr[r], t = row_ptr[r + 1];
    if (b == t) continue;
    double m = e[b];
    for (int64_t i = b + 1; i < t; ++i) m = e[i] > m ? e[i] : m;
    double s = 0.0;
    for (int64_t i = b; i < t; ++i) s += exp(e[i] - m);
    for (int64_t i = b; i < t; ++i) alpha[i] = exp(e[i] - m) / s;
  }
}

int oracle_gat_forward(int comp, int attn_dot, int64_t N, const int64_t* row_ptr, const int32_t* col_idx,
                       const double* H, int64_t K1, const double* W, int64_t K2, const double* a_l,
                       const double* a_r, int act, double* out, double* alpha_out) {
  int64_t nnz = row_ptr[N];
  double* theta = (double*)malloc((size_t)(N * K2 + 1) * sizeof(double));
  double* e = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
  double* alpha = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
  oracle_gemm(N, K2, K1, H, 0, W, 0, theta);                              /* Θ = H W (Eq. 4) */
  if (!attn_dot) {
    double* el = (double*)malloc((size_t)(N + 1) * sizeof(double));
    double* er = (double*)malloc((size_t)(N + 1) * sizeof(double));
    oracle_gemm(N, 1, K2, theta, 0, a_l, 0, el);
    oracle_gemm(N, 1, K2, theta, 0, a_r, 0, er);
    for (int64_t r = 0; r < N; ++r)
      for (int64_t i = row_ptr[r]; i < row_ptr[r + 1]; ++i) {
        double s = el[r] + er[col_idx[i]];
        e[i] = s > 0.0 ? s : 0.2 * s;                                      /* LeakyReLU slope 0.2 */
      }
    free(el); free(er);
  } else {
    oracle_sddmm(N, row_ptr, col_idx, theta, theta, K2, e);
    double sc = 1.0 / sqrt((double)K2);
    for (int64_t i = 0; i < nnz; ++i) e[i] *= sc;
  }
  oracle_edge_softmax(N, row_ptr, e, alpha);
  if (comp == OR_GAT_REUSE) {
    oracle_spmm(N, row_ptr, col_idx, alpha, theta, K2, out);              /* α Θ */
  } else if (comp == OR_GAT_RECOMP) {
    double* t = (double*)malloc((size_t)(N * K1 + 1) * sizeof(double));
    oracle_spmm(N, row_ptr, col_idx, alpha, H, K1, t);                    /* α H */
    oracle_gemm(N, K2, K1, t, 0, W, 0, out);                              /* (α H) W */
    free(t);
  } else {
    free(theta); free(e); free(alpha);
    return 1;
  }
  act_inplace(N * K2, out, act);
  if (alpha_out) memcpy(alpha_out, alpha, (size_t)nnz * sizeof(double));
  free(theta); free(e); free(alpha);
  return 0;
}

/* Per-row definition of the GAT layer (Eq. 4/5 read row by row) for sampled rows:
 * Θ_j = H_j W for j in the row (and the row itself), e_ij = LeakyReLU(Θ_i a_l + Θ_j a_r),
 * α = row softmax, Y_i = Σ_j α_ij Θ_j.  Rows are indices into (row_ptr, col_idx). */
void oracle_gat_rows(int64_t n_sample, const int64_t* rows, const int64_t* row_ptr, const int32_t* col_idx,
                     const double* H, int64_t K1, const double* W, int64_t K2, const double* a_l, const double* a_r,
                     int act, double* out /* n_sample x K2 */) {
#pragma omp parallel for schedule(dynamic, 4)
  for (int64_t s = 0; s < n_sample; ++s) {
    int64_t r = rows[s], b = row_ptr[r], t = row_ptr[r + 1], d = t - b;
    double* th = (double*)malloc((size_t)(K2 * (d + 1)) * sizeof(double));  /* Θ of the neighbours, then Θ_r */
    double* e = (double*)malloc((size_t)(d + 1) * sizeof(double));
    for (int64_t q = 0; q <= d; ++q) {
      int64_t j = q < d ? (int64_t)col_idx[b + q] : r;
      for (int64_t c = 0; c < K2; ++c) {
        double v = 0.0;
        for (int64_t k = 0; k < K1; ++k) v += H[j * K1 + k] * W[k * K2 + c];
        th[q * K2 + c] = v;
      }
    }
    double el = 0.0;
    for (int64_t c = 0; c < K2; ++c) el += th[d * K2 + c] * a_l[c];
    double m = -INFINITY;
    for (int64_t q = 0; q < d; ++q) {
      double er = 0.0;
      for (int64_t c = 0; c < K2; ++c) er += th[q * K2 + c] * a_r[c];
      double x = el + er;
      e[q] = x > 0.0 ? x : 0.2 * x;
      if (e[q] > m) m = e[q];
    }
    double ssum = 0.0;
    for (int64_t q = 0; q < d; ++q) ssum += exp(e[q] - m);
    for (int64_t c = 0; c < K2; ++c) {
      double v = 0.0;
      for (int64_t q = 0; q < d; ++q) v += exp(e[q] - m) / ssum * th[q * K2 + c];
      out[s * K2 + c] = (act == 1 && v < 0.0) ? 0.0 : v;
    }
    free(th);
    free(e);
  }
}

/* ------------------------------------------------------------------------ */
/* O6: GCN backward (training, L340: the forward's composition is used;      */
/* backward follows the forward's primitive order reversed [R14]).           */
/* For out = sigma(Y), Y = M H W with M = D Ã D, upstream G = dL/dout:       */
/*   dY = G ⊙ 1[Y > 0] (ReLU'(0) = 0);  dW = (M H)ᵀ dY;  dH = Mᵀ dY Wᵀ.       */
/* Mᵀ is applied as the literal transpose-scatter of the stored entries.     */
/* ------------------------------------------------------------------------ */
int oracle_gcn_backward(int comp, int64_t N, const int64_t* row_ptr, const int32_t* col_idx,
                        const double* H, int64_t K1, const double* W, int64_t K2, int act,
                        const double* G, double* dH /* nullable */, double* dW) {
  int64_t nnz = row_ptr[N];
  int64_t Kmax = K1 > K2 ? K1 : K2;
  double* y = (double*)malloc((size_t)(N * K2 + 1) * sizeof(double));
  double* o = (double*)malloc((size_t)(N * K2 + 1) * sizeof(double));
  if (oracle_gcn_forward(comp, N, row_ptr, col_idx, H, K1, W, K2, act, y, o)) {
    free(y); free(o);
    return 1;
  }
  double* dY = (double*)malloc((size_t)(N * K2 + 1) * sizeof(double));
  for (int64_t i = 0; i < N * K2; ++i) dY[i] = (act == 1 && !(y[i] > 0.0)) ? 0.0 : G[i];
  double* dinv = (double*)malloc((size_t)(N + 1) * sizeof(double));
  oracle_dinv(N, row_ptr, dinv);
  double* a = (double*)malloc((size_t)(N * Kmax + 1) * sizeof(double));
  double* b = (double*)malloc((size_t)(N * Kmax + 1) * sizeof(double));
  double* c = (double*)malloc((size_t)(N * Kmax + 1) * sizeof(double));
  double* nval = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
  oracle_sddmm(N, row_ptr, col_idx, dinv, dinv, 1, nval);
  switch (comp) {
    case OR_GCN_PRE_AGG:       /* fwd: T = Ñ H ; Y = T W */
      oracle_spmm(N, row_ptr, col_idx, nval, H, K1, a);                     /* T       */
      oracle_gemm(K1, K2, N, a, 1, dY, 0, dW);                              /* Tᵀ dY   */
      if (dH) {
        oracle_gemm(N, K1, K2, dY, 0, W, 1, b);                             /* dT = dY Wᵀ */
        oracle_spmm_t(N, N, row_ptr, col_idx, nval, b, K1, dH);             /* Ñᵀ dT   */
      }
      break;
    case OR_GCN_PRE_UPD:       /* fwd: T = H W ; Y = Ñ T */
      oracle_spmm_t(N, N, row_ptr, col_idx, nval, dY, K2, a);               /* dT = Ñᵀ dY */
      oracle_gemm(K1, K2, N, H, 1, a, 0, dW);                               /* Hᵀ dT   */
      if (dH) oracle_gemm(N, K1, K2, a, 0, W, 1, dH);                       /* dT Wᵀ   */
      break;
    case OR_GCN_DYN_AGG:       /* fwd: H'=D H ; S = Ã H' ; S' = D S ; Y = S' W */
      oracle_rowbcast(N, K1, dinv, H, a);
      oracle_spmm(N, row_ptr, col_idx, NULL, a, K1, b);
      oracle_rowbcast(N, K1, dinv, b, a);                                   /* S'      */
      oracle_gemm(K1, K2, N, a, 1, dY, 0, dW);                              /* S'ᵀ dY  */
      if (dH) {
        oracle_gemm(N, K1, K2, dY, 0, W, 1, b);                             /* dS'     */
        oracle_rowbcast(N, K1, dinv, b, c);                                 /* dS      */
        oracle_spmm_t(N, N, row_ptr, col_idx, NULL, c, K1, b);              /* dH' = Ãᵀ dS */
        oracle_rowbcast(N, K1, dinv, b, dH);                                /* dH      */
      }
      break;
    case OR_GCN_DYN_UPD:       /* fwd: T = H W ; T' = D T ; S = Ã T' ; Y = D S */
      oracle_rowbcast(N, K2, dinv, dY, a);                                  /* dS      */
      oracle_spmm_t(N, N, row_ptr, col_idx, NULL, a, K2, b);                /* dT'     */
      oracle_rowbcast(N, K2, dinv, b, c);                                   /* dT      */
      oracle_gemm(K1, K2, N, H, 1, c, 0, dW);                               /* Hᵀ dT   */
      if (dH) oracle_gemm(N, K1, K2, c, 0, W, 1, dH);                       /* dT Wᵀ   */
      break;
    default:
      break;
  }
  free(y); free(o); free(dY); free(dinv); free(a); free(b); free(c); free(nval);
  return 0;
}

/* ------------------------------------------------------------------------ */
/* GAT backward (training; the paper trains GAT, L324/L340, */
/* but gives no backward: this is the chain rule of the forward definition  */
/* above, additive attention only [R22]).  Reverse of the forward's steps:  */
/*   dY   = G ⊙ σ'(Y)                                                        */
/*   REUSE  (Y = α Θ):     dα_ij = <dY_i, Θ_j>,  dΘ  = αᵀ dY                 */
/*   RECOMP (Y = T W, T = α H): dW = Tᵀ dY, dT = dY Wᵀ,                      */
/*                          dα_ij = <dT_i, H_j>,  dH  = αᵀ dT                */
/*   softmax:   de_ij = α_ij (dα_ij - Σ_j' α_ij' dα_ij')                     */
/*   LeakyReLU: dz_ij = de_ij · (z_ij > 0 ? 1 : 0.2),  z_ij = el_i + er_j    */
/*   del_i = Σ_j dz_ij,  der_j = Σ_i dz_ij                                   */
/*   el = Θ a_l, er = Θ a_r:  dΘ_att = del a_lᵀ + der a_rᵀ,                  */
/*       da_l = Θᵀ del,  da_r = Θᵀ der                                       */
/*   Θ = H W:  dW += Hᵀ dΘ_all,  dH += dΘ_all Wᵀ                             */
/* (REUSE: dΘ_all = αᵀ dY + dΘ_att;  RECOMP: dΘ_all = dΘ_att.)               */
/* αᵀ X is the literal transpose-scatter of the stored entries.             */
/* ------------------------------------------------------------------------ */
int oracle_gat_backward(int comp, int64_t N, const int64_t* row_ptr, const int32_t* col_idx, const double* H,
                        int64_t K1, const double* W, int64_t K2, const double* a_l, const double* a_r, int act,
                        const double* G, double* dH /* nullable */, double* dW, double* da_l, double* da_r) {
  int64_t nnz = row_ptr[N];
  if (comp != OR_GAT_REUSE && comp != OR_GAT_RECOMP) return 1;
  double* theta = (double*)malloc((size_t)(N * K2 + 1) * sizeof(double));
  double* el = (double*)malloc((size_t)(N + 1) * sizeof(double));
  double* er = (double*)malloc((size_t)(N + 1) * sizeof(double));
  double* z = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
  double* e = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
  double* alpha = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
  double* y = (double*)malloc((size_t)(N * K2 + 1) * sizeof(double));
  double* dY = (double*)malloc((size_t)(N * K2 + 1) * sizeof(double));
  double* dal = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
  double* dz = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
  double* del = (double*)calloc((size_t)(N + 1), sizeof(double));
  double* der = (double*)calloc((size_t)(N + 1), sizeof(double));
  double* dth = (double*)malloc((size_t)(N * K2 + 1) * sizeof(double));
  double* t = (double*)malloc((size_t)(N * K1 + 1) * sizeof(double));
  double* dT = (double*)malloc((size_t)(N * K1 + 1) * sizeof(double));
  double* tmp = (double*)malloc((size_t)(K1 * K2 + N * K1 + 1) * sizeof(double));
  /* forward (same steps as oracle_gat_forward) */
  oracle_gemm(N, K2, K1, H, 0, W, 0, theta);
  oracle_gemm(N, 1, K2, theta, 0, a_l, 0, el);
  oracle_gemm(N, 1, K2, theta, 0, a_r, 0, er);
  for (int64_t r = 0; r < N; ++r)
    for (int64_t i = row_ptr[r]; i < row_ptr[r + 1]; ++i) {
      z[i] = el[r] + er[col_idx[i]];
      e[i] = z[i] > 0.0 ? z[i] : 0.2 * z[i];
    }
  oracle_edge_softmax(N, row_ptr, e, alpha);
  oracle_spmm(N, row_ptr, col_idx, alpha, H, K1, t);                          /* T = α H */
  if (comp == OR_GAT_REUSE) oracle_spmm(N, row_ptr, col_idx, alpha, theta, K2, y);
  else oracle_gemm(N, K2, K1, t, 0, W, 0, y);
  /* dY = G ⊙ σ'(Y), ReLU'(0) = 0 */
  for (int64_t i = 0; i < N * K2; ++i) dY[i] = (act == 1 && !(y[i] > 0.0)) ? 0.0 : G[i];
  /* dα (SDDMM of the composition's operands) */
  if (comp == OR_GAT_REUSE) {
    oracle_sddmm(N, row_ptr, col_idx, dY, theta, K2, dal);                    /* <dY_i, Θ_j> */
  } else {
    oracle_gemm(K1, K2, N, t, 1, dY, 0, dW);                                  /* dW = Tᵀ dY */
    oracle_gemm(N, K1, K2, dY, 0, W, 1, dT);                                  /* dT = dY Wᵀ */
    oracle_sddmm(N, row_ptr, col_idx, dT, H, K1, dal);                        /* <dT_i, H_j> */
  }
  /* softmax and LeakyReLU backward, row by row */
  for (int64_t r = 0; r < N; ++r) {
    double s = 0.0;
    for (int64_t i = row_ptr[r]; i < row_ptr[r + 1]; ++i) s += alpha[i] * dal[i];
    for (int64_t i = row_ptr[r]; i < row_ptr[r + 1]; ++i)
      dz[i] = alpha[i] * (dal[i] - s) * (z[i] > 0.0 ? 1.0 : 0.2);
  }
  for (int64_t r = 0; r < N; ++r)
    for (int64_t i = row_ptr[r]; i < row_ptr[r + 1]; ++i) {
      del[r] += dz[i];
      der[col_idx[i]] += dz[i];
    }
  /* dΘ_att = del a_lᵀ + der a_rᵀ ; da = Θᵀ [del, der] */
  for (int64_t r = 0; r < N; ++r)
    for (int64_t c = 0; c < K2; ++c) dth[r * K2 + c] = del[r] * a_l[c] + der[r] * a_r[c];
  oracle_gemm(K2, 1, N, theta, 1, del, 0, da_l);
  oracle_gemm(K2, 1, N, theta, 1, der, 0, da_r);
  if (comp == OR_GAT_REUSE) {
    double* sc = (double*)malloc((size_t)(N * K2 + 1) * sizeof(double));
    oracle_spmm_t(N, N, row_ptr, col_idx, alpha, dY, K2, sc);                 /* αᵀ dY */
    for (int64_t i = 0; i < N * K2; ++i) dth[i] += sc[i];
    free(sc);
    oracle_gemm(K1, K2, N, H, 1, dth, 0, dW);                                 /* Hᵀ dΘ */
    if (dH) oracle_gemm(N, K1, K2, dth, 0, W, 1, dH);                         /* dΘ Wᵀ */
  } else {
    oracle_gemm(K1, K2, N, H, 1, dth, 0, tmp);                                /* Hᵀ dΘ_att */
    for (int64_t i = 0; i < K1 * K2; ++i) dW[i] += tmp[i];
    if (dH) {
      oracle_spmm_t(N, N, row_ptr, col_idx, alpha, dT, K1, dH);               /* αᵀ dT */
      double* h2 = tmp + K1 * K2;
      oracle_gemm(N, K1, K2, dth, 0, W, 1, h2);                               /* dΘ_att Wᵀ */
      for (int64_t i = 0; i < N * K1; ++i) dH[i] += h2[i];
    }
  }
  free(theta); free(el); free(er); free(z); free(e); free(alpha); free(y); free(dY); free(dal); free(dz);
  free(del); free(der); free(dth); free(t); free(dT); free(tmp);
  return 0;
}

/* ------------------------------------------------------------------------ */
/* Magnitude of the GAT backward computation (tolerance scale, reading R19/ */
/* R22): the same steps as oracle_gat_backward with every operand replaced  */
/* by its absolute value and every difference by a sum, so each output is   */
/* the sum of the absolute values of the terms that form it.  A fp32 path's */
/* forward error is bounded by a small multiple of eps times this, so the   */
/* parity tests measure error relative to max(|r|, magnitude) per row.      */
/* (The softmax backward dα - c cancels by construction: near-one-hot rows  */
/* have |dα - c| << |dα|.)                                                   */
/* ------------------------------------------------------------------------ */
int oracle_gat_backward_magnitude(int comp, int64_t N, const int64_t* row_ptr, const int32_t* col_idx,
                                  const double* H, int64_t K1, const double* W, int64_t K2, const double* a_l,
                                  const double* a_r, int act, const double* G, double* mdH, double* mdW,
                                  double* mda_l, double* mda_r) {
  int64_t nnz = row_ptr[N];
  if (comp != OR_GAT_REUSE && comp != OR_GAT_RECOMP) return 1;
  double* theta = (double*)malloc((size_t)(N * K2 + 1) * sizeof(double));
  double* el = (double*)malloc((size_t)(N + 1) * sizeof(double));
  double* er = (double*)malloc((size_t)(N + 1) * sizeof(double));
  double* z = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
  double* e = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
  double* alpha = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
  double* y = (double*)malloc((size_t)(N * K2 + 1) * sizeof(double));
  double* t = (double*)malloc((size_t)(N * K1 + 1) * sizeof(double));
  double* aH = (double*)malloc((size_t)(N * K1 + 1) * sizeof(double));
  double* aW = (double*)malloc((size_t)(K1 * K2 + 1) * sizeof(double));
  double* mth = (double*)malloc((size_t)(N * K2 + 1) * sizeof(double));
  double* mdY = (double*)malloc((size_t)(N * K2 + 1) * sizeof(double));
  double* mdT = (double*)malloc((size_t)(N * K1 + 1) * sizeof(double));
  double* mda = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
  double* mdz = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
  double* mdel = (double*)calloc((size_t)(N + 1), sizeof(double));
  double* mder = (double*)calloc((size_t)(N + 1), sizeof(double));
  double* mdth = (double*)malloc((size_t)(N * K2 + 1) * sizeof(double));
  double* tmp = (double*)malloc((size_t)(K1 * K2 + 2 * N * (K1 > K2 ? K1 : K2) + 1) * sizeof(double));
  double* aal = (double*)malloc((size_t)(K2 + 1) * sizeof(double));
  double* aar = (double*)malloc((size_t)(K2 + 1) * sizeof(double));
  /* forward values (α, Y) as in oracle_gat_forward */
  oracle_gemm(N, K2, K1, H, 0, W, 0, theta);
  oracle_gemm(N, 1, K2, theta, 0, a_l, 0, el);
  oracle_gemm(N, 1, K2, theta, 0, a_r, 0, er);
  for (int64_t r = 0; r < N; ++r)
    for (int64_t i = row_ptr[r]; i < row_ptr[r + 1]; ++i) {
      z[i] = el[r] + er[col_idx[i]];
      e[i] = z[i] > 0.0 ? z[i] : 0.2 * z[i];
    }
  oracle_edge_softmax(N, row_ptr, e, alpha);
  oracle_spmm(N, row_ptr, col_idx, alpha, H, K1, t);
  if (comp == OR_GAT_REUSE) oracle_spmm(N, row_ptr, col_idx, alpha, theta, K2, y);
  else oracle_gemm(N, K2, K1, t, 0, W, 0, y);
  /* magnitudes */
  for (int64_t i = 0; i < N * K1; ++i) aH[i] = fabs(H[i]);
  for (int64_t i = 0; i < K1 * K2; ++i) aW[i] = fabs(W[i]);
  for (int64_t i = 0; i < K2; ++i) { aal[i] = fabs(a_l[i]); aar[i] = fabs(a_r[i]); }
  oracle_gemm(N, K2, K1, aH, 0, aW, 0, mth);                                 /* |H||W| >= |Θ| */
  for (int64_t i = 0; i < N * K2; ++i) mdY[i] = (act == 1 && !(y[i] > 0.0)) ? 0.0 : fabs(G[i]);
  if (comp == OR_GAT_REUSE) {
    oracle_sddmm(N, row_ptr, col_idx, mdY, mth, K2, mda);
  } else {
    oracle_gemm(N, K1, K2, mdY, 0, aW, 1, mdT);
    oracle_sddmm(N, row_ptr, col_idx, mdT, aH, K1, mda);
  }
  for (int64_t r = 0; r < N; ++r) {
    double s = 0.0;
    for (int64_t i = row_ptr[r]; i < row_ptr[r + 1]; ++i) s += alpha[i] * mda[i];
    for (int64_t i = row_ptr[r]; i < row_ptr[r + 1]; ++i)
      mdz[i] = alpha[i] * (mda[i] + s) * (z[i] > 0.0 ? 1.0 : 0.2);
  }
  for (int64_t r = 0; r < N; ++r)
    for (int64_t i = row_ptr[r]; i < row_ptr[r + 1]; ++i) {
      mdel[r] += mdz[i];
      mder[col_idx[i]] += mdz[i];
    }
  for (int64_t r = 0; r < N; ++r)
    for (int64_t c = 0; c < K2; ++c) mdth[r * K2 + c] = mdel[r] * aal[c] + mder[r] * aar[c];
  oracle_gemm(K2, 1, N, mth, 1, mdel, 0, mda_l);
  oracle_gemm(K2, 1, N, mth, 1, mder, 0, mda_r);
  if (comp == OR_GAT_REUSE) {
    double* sc = tmp + K1 * K2 + N * K1;
    oracle_spmm_t(N, N, row_ptr, col_idx, alpha, mdY, K2, sc);
    for (int64_t i = 0; i < N * K2; ++i) mdth[i] += sc[i];
    oracle_gemm(K1, K2, N, aH, 1, mdth, 0, mdW);
    if (mdH) oracle_gemm(N, K1, K2, mdth, 0, aW, 1, mdH);
  } else {
    double* at = tmp + K1 * K2 + N * K1;
    oracle_spmm(N, row_ptr, col_idx, alpha, aH, K1, at);                    /* α|H| >= |T| */
    oracle_gemm(K1, K2, N, at, 1, mdY, 0, mdW);
    oracle_gemm(K1, K2, N, aH, 1, mdth, 0, tmp);
    for (int64_t i = 0; i < K1 * K2; ++i) mdW[i] += tmp[i];
    if (mdH) {
      oracle_spmm_t(N, N, row_ptr, col_idx, alpha, mdT, K1, mdH);
      double* h2 = tmp + K1 * K2;
      oracle_gemm(N, K1, K2, mdth, 0, aW, 1, h2);
      for (int64_t i = 0; i < N * K1; ++i) mdH[i] += h2[i];
    }
  }
  free(theta); free(el); free(er); free(z); free(e); free(alpha); free(y); free(t); free(aH); free(aW); free(mth);
  free(mdY); free(mdT); free(mda); free(mdz); free(mdel); free(mder); free(mdth); free(tmp); free(aal); free(aar);
  return 0;
}

/* ======================================================================== */
/* N3: the other models of Table III (L67-L69, L307): SGC [27], TAGCN [28],  */
/* GIN [24].  The paper names them and counts their compositions (L326) but  */
/* gives no formulas; the definitions below are the cited models' [R23]:     */
/*   S    = D̃^{-1/2} Ã D̃^{-1/2} (the GCN normalisation of Eq. 2/3)         */
/*   SGC  : out = σ(S^k H W)                                                 */
/*   TAGCN: out = σ(Σ_{j=0..k} S^j H W_j)   (W_j stacked: W + j*K1*K2)       */
/*   GIN  : out = σ(ReLU(agg(H) W1) W2),  agg(X)_i = (1+ε) X_i + Σ_{j∈N(i)} X_j */
/*          = Σ_{stored (i,j) of Ã} X_j + ε X_i  (Ã holds one self-loop/row) */
/* Compositions (ids base + {0 PRE_AGG, 1 PRE_UPD, 2 DYN_AGG, 3 DYN_UPD}):   */
/*   PRE: precomputed sparse values (Ñ by SDDMM; GIN: 1+ε on the diagonal),  */
/*   DYN: unweighted SpMM with dense row-broadcasts (GIN: + ε X pass);       */
/*   AGG: aggregate at the input width; UPD: GEMM first (TAGCN: Horner form  */
/*   Z = H W_k; Z = S Z + H W_j for j = k-1..0).                             */
/* ======================================================================== */
enum { OR_SGC = 32, OR_TAGCN = 48, OR_GIN = 64 };

/* one hop Y = S X under the composition's normalisation (tmp: N x K scratch) */
static void or_hop(int dyn, int64_t N, const int64_t* row_ptr, const int32_t* col_idx, const double* nval,
                   const double* dinv, const double* X, int64_t K, double* Y, double* tmp) {
  if (!dyn) {
    oracle_spmm(N, row_ptr, col_idx, nval, X, K, Y);                  /* Ñ X */
  } else {
    oracle_rowbcast(N, K, dinv, X, tmp);                               /* D^-1/2 X */
    oracle_spmm(N, row_ptr, col_idx, NULL, tmp, K, Y);                 /* Ã (.)    */
    oracle_rowbcast(N, K, dinv, Y, tmp);                               /* D^-1/2 (.) */
    memcpy(Y, tmp, (size_t)(N * K) * sizeof(double));
  }
}

int oracle_sgc_forward(int comp, int64_t N, const int64_t* row_ptr, const int32_t* col_idx, const double* H,
                       int64_t K1, const double* W, int64_t K2, int hops, int act, double* out) {
  int v = comp - OR_SGC;
  if (v < 0 || v > 3 || hops < 0) return 1;
  int dyn = v >= 2, upd = v & 1;
  int64_t nnz = row_ptr[N], K = upd ? K2 : K1;
  double* dinv = (double*)malloc((size_t)(N + 1) * sizeof(double));
  double* nval = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
  double* x = (double*)malloc((size_t)(N * K + 1) * sizeof(double));
  double* y = (double*)malloc((size_t)(N * K + 1) * sizeof(double));
  double* tmp = (double*)malloc((size_t)(N * K + 1) * sizeof(double));
  oracle_dinv(N, row_ptr, dinv);
  if (!dyn) oracle_sddmm(N, row_ptr, col_idx, dinv, dinv, 1, nval);
  if (upd) oracle_gemm(N, K2, K1, H, 0, W, 0, x);                      /* H W first */
  else memcpy(x, H, (size_t)(N * K1) * sizeof(double));
  for (int h = 0; h < hops; ++h) {
    or_hop(dyn, N, row_ptr, col_idx, nval, dinv, x, K, y, tmp);
    double* t = x; x = y; y = t;
  }
  if (upd) memcpy(out, x, (size_t)(N * K2) * sizeof(double));
  else oracle_gemm(N, K2, K1, x, 0, W, 0, out);                        /* (S^k H) W */
  act_inplace(N * K2, out, act);
  free(dinv); free(nval); free(x); free(y); free(tmp);
  return 0;
}

int oracle_tagcn_forward(int comp, int64_t N, const int64_t* row_ptr, const int32_t* col_idx, const double* H,
                         int64_t K1, const double* W, int64_t K2, int hops, int act, double* out) {
  int v = comp - OR_TAGCN;
  if (v < 0 || v > 3 || hops < 0) return 1;
  int dyn = v >= 2, upd = v & 1;
  int64_t nnz = row_ptr[N], Km = K1 > K2 ? K1 : K2;
  double* dinv = (double*)malloc((size_t)(N + 1) * sizeof(double));
  double* nval = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
  double* x = (double*)malloc((size_t)(N * Km + 1) * sizeof(double));
  double* y = (double*)malloc((size_t)(N * Km + 1) * sizeof(double));
  double* p = (double*)malloc((size_t)(N * K2 + 1) * sizeof(double));
  double* tmp = (double*)malloc((size_t)(N * Km + 1) * sizeof(double));
  oracle_dinv(N, row_ptr, dinv);
  if (!dyn) oracle_sddmm(N, row_ptr, col_idx, dinv, dinv, 1, nval);
  if (!upd) {                                      /* X_0 = H, X_{j+1} = S X_j ; out = Σ_j X_j W_j */
    memcpy(x, H, (size_t)(N * K1) * sizeof(double));
    for (int64_t i = 0; i < N * K2; ++i) out[i] = 0.0;
    for (int j = 0; j <= hops; ++j) {
      oracle_gemm(N, K2, K1, x, 0, W + (int64_t)j * K1 * K2, 0, p);
      for (int64_t i = 0; i < N * K2; ++i) out[i] += p[i];
      if (j < hops) {
        or_hop(dyn, N, row_ptr, col_idx, nval, dinv, x, K1, y, tmp);
        double* t = x; x = y; y = t;
      }
    }
  } else {                                         /* Horner: Z = H W_k ; Z = S Z + H W_j, j = k-1..0 */
    oracle_gemm(N, K2, K1, H, 0, W + (int64_t)hops * K1 * K2, 0, x);
    for (int j = hops - 1; j >= 0; --j) {
      or_hop(dyn, N, row_ptr, col_idx, nval, dinv, x, K2, y, tmp);
      oracle_gemm(N, K2, K1, H, 0, W + (int64_t)j * K1 * K2, 0, p);
      for (int64_t i = 0; i < N * K2; ++i) x[i] = y[i] + p[i];
    }
    memcpy(out, x, (size_t)(N * K2) * sizeof(double));
  }
  act_inplace(N * K2, out, act);
  free(dinv); free(nval); free(x); free(y); free(p); free(tmp);
  return 0;
}

/* GIN aggregation agg(X) = Σ_{stored (i,j)} X_j + ε X_i (every row of Ã holds its self-loop) */
static void or_gin_agg(int dyn, int64_t N, const int64_t* row_ptr, const int32_t* col_idx, double eps,
                       const double* X, int64_t K, double* Y) {
  if (!dyn) {                                      /* precomputed values: 1 + ε on the diagonal */
    int64_t nnz = row_ptr[N];
    double* vals = (double*)malloc((size_t)(nnz + 1) * sizeof(double));
    for (int64_t r = 0; r < N; ++r)
      for (int64_t e = row_ptr[r]; e < row_ptr[r + 1]; ++e) vals[e] = col_idx[e] == r ? 1.0 + eps : 1.0;
    oracle_spmm(N, row_ptr, col_idx, vals, X, K, Y);
    free(vals);
  } else {                                         /* unweighted SpMM, then + ε X */
    oracle_spmm(N, row_ptr, col_idx, NULL, X, K, Y);
    for (int64_t i = 0; i < N * K; ++i) Y[i] += eps * X[i];
  }
}

int oracle_gin_forward(int comp, int64_t N, const int64_t* row_ptr, const int32_t* col_idx, const double* H,
                       int64_t K1, const double* W1, int64_t Kh, const double* W2, int64_t K2, double eps, int act,
                       double* out) {
  int v = comp - OR_GIN;
  if (v < 0 || v > 3) return 1;
  int dyn = v >= 2, upd = v & 1;
  int64_t Km = K1 > Kh ? K1 : Kh;
  double* a = (double*)malloc((size_t)(N * Km + 1) * sizeof(double));
  double* b = (double*)malloc((size_t)(N * Km + 1) * sizeof(double));
  if (!upd) {
    or_gin_agg(dyn, N, row_ptr, col_idx, eps, H, K1, a);                 /* agg(H)      */
    oracle_gemm(N, Kh, K1, a, 0, W1, 0, b);                              /* agg(H) W1   */
  } else {
    oracle_gemm(N, Kh, K1, H, 0, W1, 0, a);                              /* H W1        */
    or_gin_agg(dyn, N, row_ptr, col_idx, eps, a, Kh, b);                 /* agg(H W1)   */
  }
  act_inplace(N * Kh, b, 1);                                             /* MLP ReLU    */
  oracle_gemm(N, K2, Kh, b, 0, W2, 0, out);
  act_inplace(N * K2, out, act);
  free(a); free(b);
  return 0;
}
