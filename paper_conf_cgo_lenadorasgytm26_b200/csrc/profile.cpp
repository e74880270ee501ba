// profile.cpp -- per-primitive tracer: CUDA events on the launching stream
// around each launcher call, aggregated on demand (granii_profile_read), plus a
// process-wide count of kernels launched by this library.
#include <atomic>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <vector>

#include "internal.h"

namespace granii {
namespace {
struct Rec {
  const char* name;
  cudaEvent_t a, b;
  double bytes, flops, compulsory;
  int launches;
  bool l2;
};
std::atomic<bool> g_on{false};
std::atomic<int64_t> g_launches{0};
std::mutex g_mu;
std::vector<Rec> g_recs;
std::vector<std::pair<cudaEvent_t, cudaEvent_t>> g_pool;
size_t g_used = 0;
}  // namespace

ProfScope::ProfScope(const char* n, cudaStream_t s, double by, double fl, int la, double comp, bool l2)
    : name(n), st(s), bytes(by), flops(fl), compulsory(comp < 0.0 ? by : comp), launches(la), slot(-1),
      l2_resident(l2) {
  if (!g_on.load(std::memory_order_relaxed)) return;
  std::lock_guard<std::mutex> lk(g_mu);
  if (g_used == g_pool.size()) {
    cudaEvent_t a, b;
    if (cudaEventCreate(&a) != cudaSuccess || cudaEventCreate(&b) != cudaSuccess) return;
    g_pool.push_back({a, b});
  }
  slot = (int)g_used++;
  cudaEventRecord(g_pool[slot].first, st);
}

void ProfScope::add_launches(int n) { launches += n; }

ProfScope::~ProfScope() {
  g_launches.fetch_add(launches, std::memory_order_relaxed);
  if (slot < 0) return;
  std::lock_guard<std::mutex> lk(g_mu);
  cudaEventRecord(g_pool[slot].second, st);
  g_recs.push_back({name, g_pool[slot].first, g_pool[slot].second, bytes, flops, compulsory, launches, l2_resident});
}

}  // namespace granii

using namespace granii;

extern "C" {

granii_status granii_profile_enable(int32_t on) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_recs.clear();
  g_used = 0;
  g_on.store(on != 0);
  return GRANII_OK;
}

granii_status granii_profile_read(granii_prof_entry* out, int32_t max_entries, int32_t* n) {
  GR_ARG(out && n && max_entries > 0, "bad argument");
  GR_CUDA(cudaDeviceSynchronize());
  std::lock_guard<std::mutex> lk(g_mu);
  std::map<std::string, granii_prof_entry> agg;
  for (const Rec& r : g_recs) {
    float ms = 0.f;
    GR_CUDA(cudaEventElapsedTime(&ms, r.a, r.b));
    granii_prof_entry& e = agg[r.name];
    e.calls += 1;
    e.launches += r.launches;
    e.ms += ms;
    e.bytes += r.bytes;
    e.flops += r.flops;
    e.compulsory_bytes += r.compulsory;
    e.l2_resident += r.l2 ? 1 : 0;
  }
  int32_t k = 0;
  for (auto& kv : agg) {
    if (k >= max_entries) break;
    granii_prof_entry e = kv.second;
    memset(e.name, 0, sizeof(e.name));
    strncpy(e.name, kv.first.c_str(), sizeof(e.name) - 1);
    out[k++] = e;
  }
  *n = k;
  return GRANII_OK;
}

int64_t granii_launch_count(void) { return g_launches.load(); }

}  // extern "C"
