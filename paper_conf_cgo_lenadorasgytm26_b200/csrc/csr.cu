// csr.cu -- graph ingest: COO -> CSR of Ã, degrees,
// D̃^{-1/2}, integer featurizer features, degree-ordered schedule, and the
// nnz-balanced row partition with the padded gather layout.
//
// PAPER.md: Ã "with self-edges" (L113); messages flow src -> dst and are summed
// at the destination (L192) => row = dst, col = src; graphs are unweighted
// (L328) => duplicates collapse; D̃ = degree in Ã (L113) => deg = row nnz.
// Degrees come from row_ptr differences: no per-call atomic "binning" (the
// WiseGraph cost the paper singles out, L353).
#include <cub/cub.cuh>

#include <algorithm>
#include <cmath>

#include <chrono>

#include "internal.h"

namespace granii {

static int key_bits(int64_t n) {
  int b = 1;
  while ((int64_t(1) << b) < n) ++b;
  return b;
}

__global__ void k_validate(int64_t E, const int32_t* __restrict__ s, const int32_t* __restrict__ d, int64_t N,
                           int* bad) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < E; e += (int64_t)gridDim.x * blockDim.x) {
    int32_t a = s[e], b = d[e];
    if (a < 0 || a >= N || b < 0 || b >= N) atomicExch(bad, 1);
  }
}

__global__ void k_make_keys(int64_t E, const int32_t* __restrict__ s, const int32_t* __restrict__ d, int64_t N,
                            int cb, int sym, int loops, uint64_t* __restrict__ keys) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t per = sym ? 2 : 1;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < E; e += stride) {
    uint64_t r = (uint32_t)d[e], c = (uint32_t)s[e];
    keys[e * per] = (r << cb) | c;                      // (row = dst, col = src)
    if (sym) keys[e * per + 1] = (c << cb) | r;         // reverse edge
  }
  if (loops)
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N; i += stride)
      keys[E * per + i] = ((uint64_t)i << cb) | (uint64_t)i;
}

// row_ptr[r] = lower_bound(keys, r << cb); col_idx from the low bits.
__global__ void k_row_ptr(int64_t N, const uint64_t* __restrict__ keys, int64_t nnz, int cb,
                          int64_t* __restrict__ row_ptr) {
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r <= N; r += (int64_t)gridDim.x * blockDim.x) {
    if (r == N) { row_ptr[N] = nnz; continue; }
    uint64_t target = (uint64_t)r << cb;
    int64_t lo = 0, hi = nnz;
    while (lo < hi) {
      int64_t mid = (lo + hi) >> 1;
      if (keys[mid] < target) lo = mid + 1; else hi = mid;
    }
    row_ptr[r] = lo;
  }
}

__global__ void k_cols(int64_t nnz, const uint64_t* __restrict__ keys, uint64_t mask, int32_t* __restrict__ col) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x)
    col[i] = (int32_t)(keys[i] & mask);
}

// deg, dinv = deg^{-1/2} (correctly rounded, reading R6), integer feature sums.
__global__ void k_degree(int64_t n, const int64_t* __restrict__ rp, int32_t* __restrict__ deg,
                         float* __restrict__ dinv, unsigned long long* __restrict__ acc /* s2, max, min, zeros */) {
  unsigned long long s2 = 0, mx = 0, mn = ~0ull, z = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t d = rp[i + 1] - rp[i];
    deg[i] = (int32_t)d;
    dinv[i] = d > 0 ? __frsqrt_rn((float)d) : 0.f;
    s2 += (unsigned long long)(d * d);
    mx = max(mx, (unsigned long long)d);
    mn = min(mn, (unsigned long long)d);
    z += (d == 0);
  }
  typedef cub::BlockReduce<unsigned long long, 256> BR;
  __shared__ typename BR::TempStorage t;
  unsigned long long v;
  v = BR(t).Sum(s2); if (threadIdx.x == 0) atomicAdd(acc + 0, v); __syncthreads();
  v = BR(t).Reduce(mx, cub::Max()); if (threadIdx.x == 0) atomicMax(acc + 1, v); __syncthreads();
  v = BR(t).Reduce(mn, cub::Min()); if (threadIdx.x == 0) atomicMin(acc + 2, v); __syncthreads();
  v = BR(t).Sum(z); if (threadIdx.x == 0) atomicAdd(acc + 3, v);
}

__global__ void k_sum_first(int64_t k, const int32_t* __restrict__ v, unsigned long long* out) {
  unsigned long long s = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < k; i += (int64_t)gridDim.x * blockDim.x)
    s += (unsigned long long)v[i];
  typedef cub::BlockReduce<unsigned long long, 256> BR;
  __shared__ typename BR::TempStorage t;
  s = BR(t).Sum(s);
  if (threadIdx.x == 0) atomicAdd(out, s);
}

__global__ void k_deg_only(int64_t n, const int64_t* __restrict__ rp, int32_t* __restrict__ deg) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    deg[i] = (int32_t)(rp[i + 1] - rp[i]);
}

__global__ void k_ord_rp(int64_t n, const int32_t* __restrict__ order, const int64_t* __restrict__ rp,
                         longlong2* __restrict__ out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = order[i];
    out[i] = make_longlong2(rp[r], rp[r + 1]);
  }
}

// tile_row[t] = the row r with row_ptr[r] <= t·TE < row_ptr[r+1] (every tile start lies in one non-empty row)
__global__ void k_tile_rows(int64_t n, const int64_t* __restrict__ rp, int64_t TE, int32_t* __restrict__ tr) {
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
    const int64_t a = rp[r], b = rp[r + 1];
    if (b == a) continue;
    for (int64_t t = (a + TE - 1) / TE; t <= (b - 1) / TE; ++t) tr[t] = (int32_t)r;
  }
}

__global__ void k_permute_off(int64_t n, int G1, const int32_t* __restrict__ order, const int32_t* __restrict__ off,
                              int32_t* __restrict__ out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n * G1; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t t = i / G1, p = i % G1;
    out[i] = off[(int64_t)order[t] * G1 + p];
  }
}

__global__ void k_iota(int64_t n, int32_t* v) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    v[i] = (int32_t)i;
}

// local block: rebased row_ptr, remapped columns (padded gather layout).
__global__ void k_local_rows(int64_t nr, const int64_t* __restrict__ rp, int64_t b0, int64_t* __restrict__ out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= nr; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = rp[b0 + i] - rp[b0];
}

__global__ void k_remap_cols(int64_t n, const int32_t* __restrict__ col, const int64_t* __restrict__ bounds, int G,
                             int64_t max_rows, int32_t* __restrict__ out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t j = col[i];
    int g = 0;
    while (g + 1 < G && bounds[g + 1] <= j) ++g;        // owner(j): bounds[g] <= j < bounds[g+1]
    out[i] = (int32_t)(g * max_rows + (j - bounds[g]));
  }
}

__global__ void k_square(int64_t n, const float* __restrict__ x, float* __restrict__ y) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    y[i] = x[i] * x[i];
}

// owner_off[i][p] = offset in row i of its first entry whose gather-layout column lies in
// block p (columns are sorted and the layout is monotone in the global id, so each owner's
// entries are one contiguous run); owner_off[i][G] = deg_i
__global__ void k_owner_offsets(int64_t R, const int64_t* __restrict__ rp, const int32_t* __restrict__ col, int G,
                                int64_t max_rows, int32_t* __restrict__ off) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < R; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t lo = rp[i], hi = rp[i + 1];
    for (int p = 0; p <= G; ++p) {
      const int64_t key = (int64_t)p * max_rows;
      int64_t a = lo, b = hi;  // lower_bound
      while (a < b) {
        const int64_t m = (a + b) >> 1;
        if ((int64_t)col[m] < key) a = m + 1;
        else b = m;
      }
      off[i * (G + 1) + p] = (int32_t)(a - lo);
    }
  }
}

__global__ void k_gather_layout_dinv(int64_t N, const float* __restrict__ dinv, const int64_t* __restrict__ bounds,
                                     int G, int64_t max_rows, float* __restrict__ out) {
  int64_t total = (int64_t)G * max_rows;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    int g = (int)(i / max_rows);
    int64_t j = bounds[g] + (i - g * max_rows);
    out[i] = j < bounds[g + 1] ? dinv[j] : 0.f;
  }
}

static int grid_for(int64_t n, int per = 256) {
  int64_t b = ceil_div(std::max<int64_t>(n, 1), per);
  return (int)std::min<int64_t>(b, 148 * 16);
}

// host partition: b_0 = 0, b_G = N, b_g = min{ r : row_ptr[r] >= ceil(g*nnz/G) }
void partition_bounds_host(int64_t N, const int64_t* rp, int G, int64_t* b) {
  int64_t nnz = rp[N];
  b[0] = 0;
  b[G] = N;
  for (int g = 1; g < G; ++g) {
    int64_t target = ceil_div((int64_t)g * nnz, G);
    b[g] = std::lower_bound(rp, rp + N + 1, target) - rp;
    if (b[g] > N) b[g] = N;
  }
}

void graph_free(granii_graph_s* g);

granii_status graph_create(int64_t N, int64_t E, const int32_t* d_src, const int32_t* d_dst, uint32_t flags,
                           int32_t rank, int32_t world, cudaStream_t st, granii_graph_s** out,
                           const int64_t* force_bounds) {
  const int sym = (flags & GRANII_SYMMETRIZE) ? 1 : 0, loops = (flags & GRANII_ADD_SELF_LOOPS) ? 1 : 0;
  const int cb = key_bits(std::max<int64_t>(N, 2));
  GR_ARG(2 * cb <= 64, "num_nodes too large");
  const int64_t M = E * (sym ? 2 : 1) + (loops ? N : 0);
  GR_ARG(M < (int64_t(1) << 31), "too many edges for one build (>= 2^31 entries)");

  auto g = new granii_graph_s();
  g->N = N;
  g->rank = rank;
  g->world = world;
  g->symmetric = sym;
  g->self_loops = loops;
  cudaGetDevice(&g->device);
  {
    // the per-call scratch of the hub-segment paths (SpMM partials, segmented softmax) comes
    // from the stream-ordered pool: keep its memory instead of returning it to the driver at
    // every synchronisation, so a steady-state step never maps memory on the host path
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, g->device) == cudaSuccess) {
      uint64_t keep = UINT64_MAX;
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
    }
  }

  using clk = std::chrono::steady_clock;
  auto t_mark = clk::now();
  auto lap = [&](int phase) {  // called right after a stream sync: host time = device time of the phase
    const auto now = clk::now();
    g->create_ms[phase] += std::chrono::duration<double, std::milli>(now - t_mark).count();
    t_mark = now;
  };
  int* d_bad = nullptr;
  unsigned long long* d_acc = nullptr;
  uint64_t *k0 = nullptr, *k1 = nullptr;
  int64_t* d_nsel = nullptr;
  void* tmp = nullptr;
  size_t tmp_bytes = 0;
  int32_t *deg = nullptr, *deg_sorted = nullptr, *iota = nullptr;
  int64_t* rp_full = nullptr;
  int32_t* col_full = nullptr;
  float* dinv_full = nullptr;
  granii_status rc = GRANII_OK;
  auto cleanup = [&]() {
    cudaFreeAsync(d_bad, st); cudaFreeAsync(d_acc, st); cudaFreeAsync(k0, st); cudaFreeAsync(k1, st);
    cudaFreeAsync(d_nsel, st); cudaFreeAsync(tmp, st); cudaFreeAsync(deg, st); cudaFreeAsync(deg_sorted, st);
    cudaFreeAsync(iota, st);
  };
#define CK(call)                                                                        \
  do {                                                                                  \
    cudaError_t e_ = (call);                                                            \
    if (e_ != cudaSuccess) {                                                            \
      rc = fail(e_ == cudaErrorMemoryAllocation ? GRANII_ERR_OOM : GRANII_ERR_CUDA,     \
                std::string(#call) + ": " + cudaGetErrorString(e_));                    \
      cleanup(); delete g; return rc;                                                   \
    }                                                                                   \
  } while (0)

  CK(cudaMallocAsync(&d_bad, sizeof(int), st));
  CK(cudaMemsetAsync(d_bad, 0, sizeof(int), st));
  if (E > 0) k_validate<<<grid_for(E), 256, 0, st>>>(E, d_src, d_dst, N, d_bad);
  int h_bad = 0;
  CK(cudaMemcpyAsync(&h_bad, d_bad, sizeof(int), cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  if (h_bad) {
    cleanup();
    delete g;
    return fail(GRANII_ERR_INVALID_ARG, "edge endpoint outside [0, num_nodes)");
  }

  // 1. keys, 2. radix sort, 3. unique
  CK(cudaMallocAsync(&k0, std::max<int64_t>(M, 1) * sizeof(uint64_t), st));
  CK(cudaMallocAsync(&k1, std::max<int64_t>(M, 1) * sizeof(uint64_t), st));
  CK(cudaMallocAsync(&d_nsel, sizeof(int64_t), st));
  if (M > 0) k_make_keys<<<grid_for(std::max(E, N)), 256, 0, st>>>(E, d_src, d_dst, N, cb, sym, loops, k0);
  size_t b1 = 0, b2 = 0, b3 = 0, b4 = 0;
  cub::DeviceRadixSort::SortKeys(nullptr, b1, k0, k1, (int)M, 0, 2 * cb, st);
  cub::DeviceSelect::Unique(nullptr, b2, k1, k0, d_nsel, (int)M, st);
  cub::DeviceRadixSort::SortKeys(nullptr, b3, (int32_t*)nullptr, (int32_t*)nullptr, (int)N, 0, 32, st);
  cub::DeviceRadixSort::SortPairsDescending(nullptr, b4, (int32_t*)nullptr, (int32_t*)nullptr, (int32_t*)nullptr,
                                            (int32_t*)nullptr, (int)N, 0, 32, st);
  tmp_bytes = std::max(std::max(b1, b2), std::max(b3, b4));
  CK(cudaMallocAsync(&tmp, std::max<size_t>(tmp_bytes, 16), st));
  int64_t nnz = 0;
  if (M > 0) {
    CK(cub::DeviceRadixSort::SortKeys(tmp, b1, k0, k1, (int)M, 0, 2 * cb, st));
    CK(cub::DeviceSelect::Unique(tmp, b2, k1, k0, d_nsel, (int)M, st));
    CK(cudaMemcpyAsync(&nnz, d_nsel, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));   // the single host sync: learn nnz
  }
  g->nnz = nnz;
  CK(cudaMalloc(&rp_full, (N + 1) * sizeof(int64_t)));
  CK(cudaMalloc(&col_full, std::max<int64_t>(nnz, 1) * sizeof(int32_t)));
  CK(cudaMalloc(&dinv_full, std::max<int64_t>(N, 1) * sizeof(float)));
  k_row_ptr<<<grid_for(N + 1), 256, 0, st>>>(N, k0, nnz, cb, rp_full);
  if (nnz > 0) k_cols<<<grid_for(nnz), 256, 0, st>>>(nnz, k0, (uint64_t(1) << cb) - 1, col_full);
  CK(cudaStreamSynchronize(st));
  lap(0);

  // degrees, dinv, features
  CK(cudaMallocAsync(&deg, std::max<int64_t>(N, 1) * sizeof(int32_t), st));
  CK(cudaMallocAsync(&deg_sorted, std::max<int64_t>(N, 1) * sizeof(int32_t), st));
  CK(cudaMallocAsync(&iota, std::max<int64_t>(N, 1) * sizeof(int32_t), st));
  CK(cudaMallocAsync(&d_acc, 8 * sizeof(unsigned long long), st));
  unsigned long long init[8] = {0, 0, ~0ull, 0, 0, 0, 0, 0};
  CK(cudaMemcpyAsync(d_acc, init, sizeof(init), cudaMemcpyHostToDevice, st));
  if (N > 0) {
    k_degree<<<grid_for(N), 256, 0, st>>>(N, rp_full, deg, dinv_full, d_acc);
    CK(cub::DeviceRadixSort::SortKeys(tmp, b3, deg, deg_sorted, (int)N, 0, 32, st));
    int64_t k = ceil_div(N, 100);
    // ascending sort: the top-k are the last k entries
    k_sum_first<<<grid_for(k), 256, 0, st>>>(k, deg_sorted + (N - k), d_acc + 4);
  }
  unsigned long long hacc[8];
  CK(cudaMemcpyAsync(hacc, d_acc, sizeof(hacc), cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  lap(1);
  g->features[0] = N;
  g->features[1] = nnz;
  g->features[2] = nnz;
  g->features[3] = (int64_t)hacc[0];
  g->features[4] = (int64_t)hacc[1];
  g->features[5] = N > 0 ? (int64_t)hacc[2] : 0;
  g->features[6] = (int64_t)hacc[4];
  g->features[7] = (int64_t)hacc[3];
  // hub segment length: a work item must stay short next to the average warp's share of the
  // graph (a 2048-entry segment is ~250 dependent gather steps, a 300 us tail on a graph
  // whose whole SpMM takes 50 us): nnz / (148 SMs x 64 warps), a power of two in [256, 2048],
  // from the GLOBAL nnz so every rank of a partition cuts the same way
  {
    int64_t want = nnz / (148 * 64), sl = 256;
    while (sl < 2048 && sl * 2 <= want) sl *= 2;
    g->seg_len = sl;
  }
  if (const char* e = getenv("GRANII_SEG")) g->seg_len = std::max<int64_t>(64, atoll(e));

  // partition
  if (world <= 1) {
    g->row_begin = 0;
    g->row_end = N;
    g->n_rows = N;
    g->local_nnz = nnz;
    g->max_rows = N;
    g->n_cols = N;
    g->bounds = {0, N};
    g->row_ptr = rp_full;
    g->col_idx = col_full;
    g->dinv_rows = dinv_full;
    g->dinv_cols = dinv_full;
  } else {
    std::vector<int64_t> hrp(N + 1);
    CK(cudaMemcpyAsync(hrp.data(), rp_full, (N + 1) * sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    g->bounds.assign(world + 1, 0);
    if (force_bounds) g->bounds.assign(force_bounds, force_bounds + world + 1);  // Ãᵀ: Ã's row blocks
    else partition_bounds_host(N, hrp.data(), world, g->bounds.data());
    int64_t mr = 0;
    for (int i = 0; i < world; ++i) mr = std::max(mr, g->bounds[i + 1] - g->bounds[i]);
    g->max_rows = std::max<int64_t>(mr, 1);
    g->row_begin = g->bounds[rank];
    g->row_end = g->bounds[rank + 1];
    g->n_rows = g->row_end - g->row_begin;
    g->local_nnz = hrp[g->row_end] - hrp[g->row_begin];
    g->n_cols = (int64_t)world * g->max_rows;
    for (int64_t i = 0; i < N; ++i) {  // hub segments of the whole graph (rank-independent selection)
      const int64_t d = hrp[i + 1] - hrp[i];
      if (d > g->seg_len) g->n_seg_global += ceil_div(d, g->seg_len);
    }
    int64_t* d_bounds = nullptr;
    CK(cudaMallocAsync(&d_bounds, (world + 1) * sizeof(int64_t), st));
    CK(cudaMemcpyAsync(d_bounds, g->bounds.data(), (world + 1) * sizeof(int64_t), cudaMemcpyHostToDevice, st));
    CK(cudaMalloc(&g->row_ptr, (g->n_rows + 1) * sizeof(int64_t)));
    CK(cudaMalloc(&g->col_idx, std::max<int64_t>(g->local_nnz, 1) * sizeof(int32_t)));
    CK(cudaMalloc(&g->dinv_rows, std::max<int64_t>(g->n_rows, 1) * sizeof(float)));
    CK(cudaMalloc(&g->dinv_cols, g->n_cols * sizeof(float)));
    k_local_rows<<<grid_for(g->n_rows + 1), 256, 0, st>>>(g->n_rows, rp_full, g->row_begin, g->row_ptr);
    if (g->local_nnz > 0)
      k_remap_cols<<<grid_for(g->local_nnz), 256, 0, st>>>(g->local_nnz, col_full + hrp[g->row_begin], d_bounds,
                                                           world, g->max_rows, g->col_idx);
    if (g->n_rows > 0)
      CK(cudaMemcpyAsync(g->dinv_rows, dinv_full + g->row_begin, g->n_rows * sizeof(float),
                         cudaMemcpyDeviceToDevice, st));
    k_gather_layout_dinv<<<grid_for(g->n_cols), 256, 0, st>>>(N, dinv_full, d_bounds, world, g->max_rows,
                                                              g->dinv_cols);
    // per-row owner ranges for the block-phased SpMM (layer.cu gathered_spmm, N1)
    CK(cudaMalloc(&g->owner_off, std::max<int64_t>(g->n_rows, 1) * (world + 1) * sizeof(int32_t)));
    if (g->n_rows > 0)
      k_owner_offsets<<<grid_for(g->n_rows), 256, 0, st>>>(g->n_rows, g->row_ptr, g->col_idx, world, g->max_rows,
                                                           g->owner_off);
    CK(cudaFreeAsync(d_bounds, st));
    CK(cudaStreamSynchronize(st));
    cudaFree(rp_full);
    cudaFree(col_full);
    cudaFree(dinv_full);
  }

  // dinv^2 of the owned rows: between two hops the post-scale and the next pre-scale are one
  CK(cudaMalloc(&g->dinv2_rows, std::max<int64_t>(g->n_rows, 1) * sizeof(float)));
  if (g->n_rows > 0) k_square<<<grid_for(g->n_rows), 256, 0, st>>>(g->n_rows, g->dinv_rows, g->dinv2_rows);

  // degree-descending schedule of the owned rows (stable radix sort: deterministic)
  CK(cudaMalloc(&g->order, std::max<int64_t>(g->n_rows, 1) * sizeof(int32_t)));
  if (g->n_rows > 0) {
    k_iota<<<grid_for(g->n_rows), 256, 0, st>>>(g->n_rows, iota);
    k_deg_only<<<grid_for(g->n_rows), 256, 0, st>>>(g->n_rows, g->row_ptr, deg);
    CK(cub::DeviceRadixSort::SortPairsDescending(tmp, b4, deg, deg_sorted, iota, g->order, (int)g->n_rows, 0, 32,
                                                 st));
  }
  CK(cudaMalloc(&g->ord_rp, std::max<int64_t>(g->n_rows, 1) * sizeof(longlong2)));
  if (g->n_rows > 0) k_ord_rp<<<grid_for(g->n_rows), 256, 0, st>>>(g->n_rows, g->order, g->row_ptr, g->ord_rp);
  g->n_tiles = ceil_div(g->local_nnz, granii_graph_s::tile_e);
  CK(cudaMalloc(&g->tile_row, std::max<int64_t>(g->n_tiles, 1) * sizeof(int32_t)));
  if (g->n_tiles > 0)
    k_tile_rows<<<grid_for(g->n_rows), 256, 0, st>>>(g->n_rows, g->row_ptr, granii_graph_s::tile_e, g->tile_row);
  if (g->owner_off) {
    CK(cudaMalloc(&g->ord_off, std::max<int64_t>(g->n_rows, 1) * (world + 1) * sizeof(int32_t)));
    if (g->n_rows > 0)
      k_permute_off<<<grid_for(g->n_rows * (world + 1)), 256, 0, st>>>(g->n_rows, world + 1, g->order, g->owner_off,
                                                                      g->ord_off);
  }
  CK(cudaGetLastError());
  CK(cudaStreamSynchronize(st));

  // heavy-row segments (power-law hubs): rows with more than seg_len entries are cut
  // into seg_len-entry warp-wide work items so a hub cannot set the kernel's tail
  if (g->n_rows > 0 && g->features[4] > g->seg_len) {
    std::vector<int64_t> hrp(g->n_rows + 1);
    CK(cudaMemcpy(hrp.data(), g->row_ptr, (g->n_rows + 1) * sizeof(int64_t), cudaMemcpyDeviceToHost));
    int64_t nh = 0;
    for (int64_t r = 0; r < g->n_rows; ++r) nh += (hrp[r + 1] - hrp[r]) > g->seg_len;
    if (nh > 0) {
      std::vector<int32_t> hrows(nh);
      CK(cudaMemcpy(hrows.data(), g->order, nh * sizeof(int32_t), cudaMemcpyDeviceToHost));  // degree-descending
      std::vector<int32_t> sptr(nh + 1, 0), sh, sr;
      std::vector<int64_t> lo, hi;
      for (int64_t h = 0; h < nh; ++h) {
        const int64_t r = hrows[h];
        for (int64_t b = hrp[r]; b < hrp[r + 1]; b += g->seg_len) {
          lo.push_back(b);
          hi.push_back(std::min(b + g->seg_len, hrp[r + 1]));
          sh.push_back((int32_t)h);
          sr.push_back((int32_t)r);
        }
        sptr[h + 1] = (int32_t)lo.size();
      }
      g->n_heavy = nh;
      g->n_seg = (int64_t)lo.size();
      CK(cudaMalloc(&g->seg_ptr, (nh + 1) * sizeof(int32_t)));
      CK(cudaMalloc(&g->seg_lo, g->n_seg * sizeof(int64_t)));
      CK(cudaMalloc(&g->seg_hi, g->n_seg * sizeof(int64_t)));
      CK(cudaMemcpy(g->seg_ptr, sptr.data(), (nh + 1) * sizeof(int32_t), cudaMemcpyHostToDevice));
      CK(cudaMemcpy(g->seg_lo, lo.data(), g->n_seg * sizeof(int64_t), cudaMemcpyHostToDevice));
      CK(cudaMemcpy(g->seg_hi, hi.data(), g->n_seg * sizeof(int64_t), cudaMemcpyHostToDevice));
      CK(cudaMalloc(&g->seg_heavy, g->n_seg * sizeof(int32_t)));
      CK(cudaMalloc(&g->seg_row, g->n_seg * sizeof(int32_t)));
      CK(cudaMemcpy(g->seg_heavy, sh.data(), g->n_seg * sizeof(int32_t), cudaMemcpyHostToDevice));
      CK(cudaMemcpy(g->seg_row, sr.data(), g->n_seg * sizeof(int32_t), cudaMemcpyHostToDevice));
    }
  }
  // sparse graphs are processed a lane group per row; rows with more than wide_deg entries
  // (a prefix of the degree-descending order) get a whole warp so they cannot set the tail
  if (g->n_rows > 0 && g->features[4] > g->wide_deg) {
    std::vector<int64_t> hrp(g->n_rows + 1);
    CK(cudaMemcpy(hrp.data(), g->row_ptr, (g->n_rows + 1) * sizeof(int64_t), cudaMemcpyDeviceToHost));
    int64_t nw = 0;
    for (int64_t r = 0; r < g->n_rows; ++r) nw += (hrp[r + 1] - hrp[r]) > g->wide_deg;
    g->n_wide = nw;
  }
  cleanup();
  CK(cudaStreamSynchronize(st));
  lap(2);
#undef CK
  if ((flags & GRANII_BUILD_TRANSPOSE) && !sym) {
    // Ãᵀ = the same build over the reversed edges, over Ã's row blocks; D̃ stays Ã's row degrees
    // (R4: Mᵀ = (D̃^-½ Ã D̃^-½)ᵀ = D̃^-½ Ãᵀ D̃^-½), so its dinv arrays are overwritten with Ã's
    granii_graph_s* t = nullptr;
    granii_status rt = graph_create(N, E, d_dst, d_src, flags & GRANII_ADD_SELF_LOOPS, rank, world, st, &t,
                                    g->bounds.data());
    if (rt != GRANII_OK) {
      graph_free(g);
      return rt;
    }
    cudaError_t e = cudaMemcpyAsync(t->dinv_rows, g->dinv_rows, std::max<int64_t>(g->n_rows, 1) * sizeof(float),
                                    cudaMemcpyDeviceToDevice, st);
    if (e == cudaSuccess && t->dinv_cols != t->dinv_rows)
      e = cudaMemcpyAsync(t->dinv_cols, g->dinv_cols, g->n_cols * sizeof(float), cudaMemcpyDeviceToDevice, st);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(t->dinv2_rows, g->dinv2_rows, std::max<int64_t>(g->n_rows, 1) * sizeof(float),
                          cudaMemcpyDeviceToDevice, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) {
      graph_free(t);
      graph_free(g);
      return fail(GRANII_ERR_CUDA, std::string("transpose dinv: ") + cudaGetErrorString(e));
    }
    g->T = t;
    g->create_ms[3] = std::chrono::duration<double, std::milli>(clk::now() - t_mark).count();
  }
  *out = g;
  return GRANII_OK;
}

void graph_free(granii_graph_s* g) {
  if (!g) return;
  graph_free(g->T);
  cudaFree(g->tperm);
  cudaFree(g->tblk);
  cudaFree(g->owner_off);
  cudaFree(g->ord_off);
  cudaFree(g->dinv2_rows);
  if (g->dinv_cols != g->dinv_rows) cudaFree(g->dinv_cols);
  cudaFree(g->dinv_rows);
  cudaFree(g->row_ptr);
  cudaFree(g->col_idx);
  cudaFree(g->order);
  cudaFree(g->ord_rp);
  cudaFree(g->tile_row);
  cudaFree(g->seg_ptr);
  cudaFree(g->seg_lo);
  cudaFree(g->seg_hi);
  cudaFree(g->seg_heavy);
  cudaFree(g->seg_row);
  delete g;
}

// ---------------------------------------------------------------- Ãᵀ -> Ã entry map, column-blocked
// Ã's entries are ordered by (row i, column j); a stable sort of their positions by column gives them
// in (column j, row i) order -- exactly the CSR order of Ãᵀ (row j, columns i ascending), which is the
// order of the kept transpose T of a directed graph and of Ã itself when symmetric.
// A per-entry array in Ã order (the der-only GAT backward's dz) is read in Ãᵀ order through that map:
// 4-byte gathers over 4·nnz bytes, each 32-byte sector holding 8 columns of one row i that rows j far
// apart need.  So the array is laid out COLUMN-BLOCKED instead: B blocks of columns, region b = the
// entries whose column lies in block b, rows i ascending, each row's run in column order; B is chosen
// so that a region (~ L2 / 3) stays in L2 while the rows j of its block -- consecutive in natural order
// -- are summed.  tblk[e] = the blocked position of Ã's entry e (where the producer writes), tperm[e'] =
// the blocked position of the Ã entry behind Ãᵀ's entry e' (where the consumer reads).
__global__ void k_blk_count(int64_t n, const int64_t* __restrict__ rp, const int32_t* __restrict__ col, int64_t bw,
                            int nb, int32_t* __restrict__ cnt) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    for (int b = 0; b < nb; ++b) cnt[(int64_t)b * n + i] = 0;
    for (int64_t e = rp[i]; e < rp[i + 1]; ++e) ++cnt[(int64_t)(col[e] / bw) * n + i];
  }
}

__global__ void k_blk_pos(int64_t n, const int64_t* __restrict__ rp, const int32_t* __restrict__ col, int64_t bw,
                          const int32_t* __restrict__ off, int32_t* __restrict__ pos) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t b = -1, start = 0;
    for (int64_t e = rp[i]; e < rp[i + 1]; ++e) {
      const int64_t be = col[e] / bw;  // non-decreasing along the row (sorted columns)
      if (be != b) {
        b = be;
        start = e;
      }
      pos[e] = off[b * n + i] + (int32_t)(e - start);
    }
  }
}

__global__ void k_compose(int64_t n, const int32_t* __restrict__ perm, const int32_t* __restrict__ pos,
                          int32_t* __restrict__ out) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x)
    out[e] = pos[perm[e]];
}

granii_status ensure_tperm(const granii_graph_s* gc, cudaStream_t st) {
  granii_graph_s* g = const_cast<granii_graph_s*>(gc);
  if (g->tperm) return GRANII_OK;
  if (g->world > 1) return fail(GRANII_ERR_UNSUPPORTED, "transpose entry map: single-GPU graphs only");
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  GR_CUDA(cudaStreamIsCapturing(st, &cs));
  if (cs != cudaStreamCaptureStatusNone) return fail(GRANII_ERR_UNSUPPORTED, "transpose entry map: stream capturing");
  const int64_t n = g->local_nnz, R = g->n_rows;
  if (n > INT32_MAX) return fail(GRANII_ERR_UNSUPPORTED, "transpose entry map: more than 2^31 entries");
  DevInfo di;
  GR_TRY(dev_info(&di));
  int bits = 1;
  while (bits < 31 && (int64_t(1) << bits) < g->n_cols) ++bits;
  // column blocks: regions of ~ L2 / 3 bytes (GRANII_TBLK overrides the count; 1 = Ã order)
  int nb = (int)std::max<int64_t>(1, ceil_div(4 * n, std::max<int64_t>(di.l2_bytes / 3, 1)));
  if (const char* e = getenv("GRANII_TBLK")) nb = std::max(1, atoi(e));
  nb = (int)std::min<int64_t>(nb, std::max<int64_t>(g->n_cols, 1));
  const int64_t bw = ceil_div(std::max<int64_t>(g->n_cols, 1), nb);
  int32_t *perm = nullptr, *iota = nullptr, *keys = nullptr, *cnt = nullptr, *pos = nullptr, *tp = nullptr;
  void* tmp = nullptr;
  size_t tb = 0, tb2 = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, tb, (const int32_t*)nullptr, (int32_t*)nullptr, (const int32_t*)nullptr,
                                  (int32_t*)nullptr, (int)n, 0, bits, st);
  cub::DeviceScan::ExclusiveSum(nullptr, tb2, (const int32_t*)nullptr, (int32_t*)nullptr, (int)(nb * R), st);
  tb = std::max(tb, tb2);
  cudaError_t e = cudaMalloc(&pos, std::max<int64_t>(n, 1) * sizeof(int32_t));
  if (e == cudaSuccess) e = cudaMalloc(&tp, std::max<int64_t>(n, 1) * sizeof(int32_t));
  if (e == cudaSuccess) e = cudaMallocAsync(&perm, std::max<int64_t>(n, 1) * sizeof(int32_t), st);
  if (e == cudaSuccess) e = cudaMallocAsync(&iota, std::max<int64_t>(n, 1) * sizeof(int32_t), st);
  if (e == cudaSuccess) e = cudaMallocAsync(&keys, std::max<int64_t>(n, 1) * sizeof(int32_t), st);
  if (e == cudaSuccess) e = cudaMallocAsync(&cnt, std::max<int64_t>((int64_t)nb * R, 1) * sizeof(int32_t) * 2, st);
  if (e == cudaSuccess) e = cudaMallocAsync(&tmp, std::max<size_t>(tb, 16), st);
  if (e == cudaSuccess && n > 0) {
    k_iota<<<grid_for(n), 256, 0, st>>>(n, iota);
    e = cub::DeviceRadixSort::SortPairs(tmp, tb, g->col_idx, keys, iota, perm, (int)n, 0, bits, st);
    int32_t* off = cnt + (int64_t)nb * R;
    const unsigned gr = (unsigned)std::min<int64_t>(ceil_div(R, 256), (int64_t)di.sms * 8);
    if (e == cudaSuccess) {
      k_blk_count<<<gr, 256, 0, st>>>(R, g->row_ptr, g->col_idx, bw, nb, cnt);
      e = cub::DeviceScan::ExclusiveSum(tmp, tb, cnt, off, (int)(nb * R), st);
    }
    if (e == cudaSuccess) {
      k_blk_pos<<<gr, 256, 0, st>>>(R, g->row_ptr, g->col_idx, bw, off, pos);
      k_compose<<<grid_for(n), 256, 0, st>>>(n, perm, pos, tp);
    }
  }
  if (e == cudaSuccess) e = cudaGetLastError();
  cudaFreeAsync(tmp, st);
  cudaFreeAsync(cnt, st);
  cudaFreeAsync(keys, st);
  cudaFreeAsync(iota, st);
  cudaFreeAsync(perm, st);
  if (e != cudaSuccess) {
    cudaFree(pos);
    cudaFree(tp);
    return fail(GRANII_ERR_CUDA, std::string("transpose entry map: ") + cudaGetErrorString(e));
  }
  g->tblk = pos;
  g->tperm = tp;
  g->tblk_n = nb;
  return GRANII_OK;
}

}  // namespace granii
