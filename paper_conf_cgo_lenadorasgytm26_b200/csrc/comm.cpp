// comm.cpp -- NCCL communicator for the row-partitioned multi-GPU layer
// (north_star (4): all-gather of dense embeddings over NVLink for the SpMM,
// all-reduce of dW).  NCCL is resolved at run time with dlopen (the copy
// PyTorch already loaded is reused via RTLD_NOLOAD), so the library loads on
// machines without NCCL and only granii_comm_* need it.
//
// A second transport, the in-process loopback group (granii_comm_create_local),
// runs G ranks as threads of one process on one device: the collectives are
// two host barriers plus stream-ordered device copies (cross-stream ordering by
// events).  It exists so the partitioned data path -- gather-layout column ids,
// padded all-gather buffers, dW all-reduce, the overlapped local/remote SpMM --
// runs and is parity-tested on a single GPU.
#include <dlfcn.h>

#include <chrono>
#include <condition_variable>
#include <cstring>
#include <deque>
#include <mutex>
#include <thread>
#include <vector>

#include "internal.h"

namespace {
typedef struct {
  char internal[128];
} nccl_uid;
typedef void* nccl_comm;
typedef int (*fn_get_uid)(nccl_uid*);
typedef int (*fn_init_rank)(nccl_comm*, int, nccl_uid, int);
typedef int (*fn_allgather)(const void*, void*, size_t, int, nccl_comm, cudaStream_t);
typedef int (*fn_allreduce)(const void*, void*, size_t, int, int, nccl_comm, cudaStream_t);
typedef int (*fn_bcast)(const void*, void*, size_t, int, int, nccl_comm, cudaStream_t);
typedef int (*fn_destroy)(nccl_comm);
typedef const char* (*fn_errstr)(int);
typedef int (*fn_async_err)(nccl_comm, int*);
typedef int (*fn_abort)(nccl_comm);
typedef int (*fn_count)(nccl_comm, int*);
typedef int (*fn_version)(int*);
typedef int (*fn_register)(nccl_comm, void*, size_t, void**);
typedef int (*fn_deregister)(nccl_comm, void*);
constexpr int kFloat32 = 7;  // ncclFloat32
constexpr int kSum = 0;      // ncclSum

struct Nccl {
  void* h = nullptr;
  fn_get_uid get_uid = nullptr;
  fn_init_rank init_rank = nullptr;
  fn_allgather allgather = nullptr;
  fn_allreduce allreduce = nullptr;
  fn_bcast bcast = nullptr;
  fn_destroy destroy = nullptr;
  fn_errstr errstr = nullptr;
  fn_async_err async_err = nullptr;  // ncclCommGetAsyncError
  fn_abort abort = nullptr;          // ncclCommAbort
  fn_count count = nullptr, user_rank = nullptr;
  fn_version version = nullptr;
  fn_register reg = nullptr;
  fn_deregister dereg = nullptr;
};

Nccl* nccl() {
  static Nccl n;
  static std::once_flag once;
  std::call_once(once, [] {
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return;
    n.h = h;
    n.get_uid = (fn_get_uid)dlsym(h, "ncclGetUniqueId");
    n.init_rank = (fn_init_rank)dlsym(h, "ncclCommInitRank");
    n.allgather = (fn_allgather)dlsym(h, "ncclAllGather");
    n.allreduce = (fn_allreduce)dlsym(h, "ncclAllReduce");
    n.bcast = (fn_bcast)dlsym(h, "ncclBroadcast");
    n.destroy = (fn_destroy)dlsym(h, "ncclCommDestroy");
    n.errstr = (fn_errstr)dlsym(h, "ncclGetErrorString");
    n.async_err = (fn_async_err)dlsym(h, "ncclCommGetAsyncError");
    n.abort = (fn_abort)dlsym(h, "ncclCommAbort");
    n.count = (fn_count)dlsym(h, "ncclCommCount");
    n.user_rank = (fn_count)dlsym(h, "ncclCommUserRank");
    n.version = (fn_version)dlsym(h, "ncclGetVersion");
    n.reg = (fn_register)dlsym(h, "ncclCommRegister");
    n.dereg = (fn_deregister)dlsym(h, "ncclCommDeregister");
  });
  return (n.h && n.get_uid && n.init_rank && n.allgather && n.allreduce && n.bcast && n.destroy) ? &n : nullptr;
}

granii_status nccl_fail(Nccl* n, int rc, const char* what) {
  return granii::fail(GRANII_ERR_NCCL,
                      std::string(what) + ": " + (n && n->errstr ? n->errstr(rc) : std::to_string(rc)));
}
}  // namespace

namespace granii {

granii_status comm_unique_id(void* id) {
  Nccl* n = nccl();
  if (!n) return fail(GRANII_ERR_NCCL, "libnccl.so.2 not found");
  nccl_uid u;
  int rc = n->get_uid(&u);
  if (rc) return nccl_fail(n, rc, "ncclGetUniqueId");
  memcpy(id, &u, sizeof(u));
  return GRANII_OK;
}

granii_status comm_create(const void* id, int32_t rank, int32_t world, granii_comm_s** out) {
  Nccl* n = nccl();
  if (!n) return fail(GRANII_ERR_NCCL, "libnccl.so.2 not found");
  nccl_uid u;
  memcpy(&u, id, sizeof(u));
  nccl_comm c = nullptr;
  int rc = n->init_rank(&c, world, u, rank);
  if (rc) return nccl_fail(n, rc, "ncclCommInitRank");
  auto* cm = new granii_comm_s();
  cm->nccl = c;
  cm->rank = rank;
  cm->world = world;
  *out = cm;
  return GRANII_OK;
}

// ------------------------------------------------------------------ failure detection
// A host thread per communicator.  Every collective records an event on its stream (not while the
// stream is being captured into a CUDA graph: there is no host-side completion to watch then).
// Every poll the thread (1) asks NCCL for an asynchronous error, (2) retires the completed
// events in order and measures how long the oldest incomplete one has been pending.  An error, or
// a collective pending longer than the timeout (a mismatched collective hangs instead of
// failing), aborts the communicator: ncclCommAbort makes its kernels exit, and every later call
// on the handle returns GRANII_ERR_NCCL with the reason.  The loopback transport is watched the
// same way (its "abort" only marks the handle failed).
struct Watchdog {
  using clock = std::chrono::steady_clock;
  granii_comm_s* c = nullptr;
  int device = 0;
  int64_t timeout_ms = 0;
  std::thread th;
  std::mutex m;
  std::condition_variable cv;
  bool stop = false;
  std::deque<std::pair<cudaEvent_t, clock::time_point>> pending;
  std::vector<cudaEvent_t> spare;
  uint64_t recorded = 0, retired = 0;
  std::string reason;

  void abort_comm(const std::string& why) {  // called with m held
    if (c->failed.exchange(1)) return;
    reason = why;
    Nccl* n = nccl();
    if (c->nccl && n && n->abort) {
      n->abort((nccl_comm)c->nccl);
      c->nccl = nullptr;  // freed by the abort
    }
  }
  void run() {
    cudaSetDevice(device);
    std::unique_lock<std::mutex> lk(m);
    while (!stop) {
      cv.wait_for(lk, std::chrono::milliseconds(20));
      if (stop || c->failed.load()) continue;
      Nccl* n = nccl();
      if (c->nccl && n && n->async_err) {
        int err = 0;
        const int rc = n->async_err((nccl_comm)c->nccl, &err);
        if (rc == 0 && err != 0 && err != 7 /* ncclInProgress */) {
          abort_comm(std::string("NCCL asynchronous error: ") + (n->errstr ? n->errstr(err) : std::to_string(err)));
          continue;
        }
      }
      while (!pending.empty()) {
        const cudaError_t q = cudaEventQuery(pending.front().first);
        if (q == cudaSuccess) {
          spare.push_back(pending.front().first);
          pending.pop_front();
          ++retired;
          continue;
        }
        if (q != cudaErrorNotReady) {
          abort_comm(std::string("collective failed on the device: ") + cudaGetErrorString(q));
          break;
        }
        const auto age = std::chrono::duration_cast<std::chrono::milliseconds>(clock::now() - pending.front().second);
        if (age.count() > timeout_ms)
          abort_comm("collective #" + std::to_string(retired) + " pending for " + std::to_string(age.count()) +
                     " ms > watchdog timeout " + std::to_string(timeout_ms) + " ms (rank " + std::to_string(c->rank) +
                     " of " + std::to_string(c->world) + "): aborted");
        break;
      }
    }
  }
  granii_status track(cudaStream_t st) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    GR_CUDA(cudaStreamIsCapturing(st, &cs));
    if (cs != cudaStreamCaptureStatusNone) return GRANII_OK;
    std::lock_guard<std::mutex> lk(m);
    cudaEvent_t e;
    if (!spare.empty()) {
      e = spare.back();
      spare.pop_back();
    } else {
      GR_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    }
    GR_CUDA(cudaEventRecord(e, st));
    pending.push_back({e, clock::now()});
    ++recorded;
    return GRANII_OK;
  }
  void shutdown() {
    {
      std::lock_guard<std::mutex> lk(m);
      stop = true;
    }
    cv.notify_all();
    if (th.joinable()) th.join();
    for (auto& p : pending) cudaEventDestroy(p.first);
    for (auto e : spare) cudaEventDestroy(e);
  }
};

static granii_status comm_failed(granii_comm_s* c) {
  auto* w = (Watchdog*)c->wd;
  std::string why = "communicator aborted";
  if (w) {
    std::lock_guard<std::mutex> lk(w->m);
    why = w->reason;
  }
  return fail(GRANII_ERR_NCCL, why);
}

static granii_status watch(granii_comm_s* c, cudaStream_t st) {
  return c && c->wd ? ((Watchdog*)c->wd)->track(st) : GRANII_OK;
}

granii_status comm_watchdog(granii_comm_s* c, int64_t timeout_ms) {
  if (c->wd) {
    auto* w = (Watchdog*)c->wd;
    w->shutdown();
    delete w;
    c->wd = nullptr;
  }
  if (timeout_ms <= 0 || c->stub) return GRANII_OK;
  auto* w = new Watchdog();
  w->c = c;
  w->timeout_ms = timeout_ms;
  GR_CUDA(cudaGetDevice(&w->device));
  c->wd = w;
  w->th = std::thread([w] { w->run(); });
  return GRANII_OK;
}

granii_status comm_check(granii_comm_s* c) { return c->failed.load() ? comm_failed(c) : GRANII_OK; }

granii_status comm_query(granii_comm_s* c, int32_t* nranks, int32_t* rank, int32_t* version) {
  *nranks = c->world;
  *rank = c->rank;
  *version = 0;
  if (c->failed.load()) return comm_failed(c);
  if (c->nccl) {  // what NCCL itself reports for the communicator
    Nccl* n = nccl();
    int v = 0, cnt = 0, r = 0;
    if (n && n->version && n->version(&v) == 0) *version = v;
    if (n && n->count && n->user_rank) {
      int rc = n->count((nccl_comm)c->nccl, &cnt);
      if (rc) return nccl_fail(n, rc, "ncclCommCount");
      rc = n->user_rank((nccl_comm)c->nccl, &r);
      if (rc) return nccl_fail(n, rc, "ncclCommUserRank");
      *nranks = cnt;
      *rank = r;
    }
  }
  return GRANII_OK;
}

granii_status comm_register(granii_comm_s* c, void* buf, size_t bytes, void** handle) {
  *handle = nullptr;
  if (!c->nccl || bytes == 0) return GRANII_OK;  // loopback / stub: nothing to register
  Nccl* n = nccl();
  if (!n || !n->reg) return fail(GRANII_ERR_UNSUPPORTED, "this NCCL has no ncclCommRegister");
  const int rc = n->reg((nccl_comm)c->nccl, buf, bytes, handle);
  if (rc) return nccl_fail(n, rc, "ncclCommRegister");
  return GRANII_OK;
}

granii_status comm_deregister(granii_comm_s* c, void* handle) {
  if (!c->nccl || !handle) return GRANII_OK;
  Nccl* n = nccl();
  if (!n || !n->dereg) return GRANII_OK;
  const int rc = n->dereg((nccl_comm)c->nccl, handle);
  if (rc) return nccl_fail(n, rc, "ncclCommDeregister");
  return GRANII_OK;
}

// ------------------------------------------------------------------ loopback group
struct LoopGroup {
  int world;
  std::mutex m;
  std::condition_variable cv;
  int arrived = 0;
  uint64_t gen = 0;
  int refs;
  std::vector<const float*> src;
  std::vector<cudaEvent_t> ready, done;
  std::vector<float*> stage;
  std::vector<size_t> stage_cap;
  explicit LoopGroup(int w) : world(w), refs(w), src(w), ready(w), done(w), stage(w, nullptr), stage_cap(w, 0) {
    for (int r = 0; r < w; ++r) {
      cudaEventCreateWithFlags(&ready[r], cudaEventDisableTiming);
      cudaEventCreateWithFlags(&done[r], cudaEventDisableTiming);
    }
  }
  ~LoopGroup() {
    for (int r = 0; r < world; ++r) {
      cudaEventDestroy(ready[r]);
      cudaEventDestroy(done[r]);
      if (stage[r]) cudaFree(stage[r]);
    }
  }
  void barrier() {
    std::unique_lock<std::mutex> lk(m);
    const uint64_t g = gen;
    if (++arrived == world) {
      arrived = 0;
      ++gen;
      cv.notify_all();
    } else {
      cv.wait(lk, [&] { return gen != g; });
    }
  }
  // every peer's copy out of this rank's buffers is ordered before this rank's later work
  granii_status finish(int rank, cudaStream_t st) {
    GR_CUDA(cudaEventRecord(done[rank], st));
    barrier();
    for (int p = 0; p < world; ++p)
      if (p != rank) GR_CUDA(cudaStreamWaitEvent(st, done[p], 0));
    return GRANII_OK;
  }
};

granii_status comm_create_local(int32_t world, granii_comm_s** out) {
  auto* grp = new LoopGroup(world);
  for (int r = 0; r < world; ++r) {
    auto* cm = new granii_comm_s();
    cm->loop = grp;
    cm->rank = r;
    cm->world = world;
    out[r] = cm;
  }
  return GRANII_OK;
}

static void free_side(granii_comm_s* c) {
  if (c->ev) {
    for (int i = 0; i <= c->world; ++i) cudaEventDestroy(c->ev[i]);
    delete[] c->ev;
  }
  if (c->side) cudaStreamDestroy(c->side);
}

granii_status comm_side(granii_comm_s* c, cudaStream_t* side, cudaEvent_t** ev) {
  if (!c->side) {
    GR_CUDA(cudaStreamCreateWithFlags(&c->side, cudaStreamNonBlocking));
    c->ev = new cudaEvent_t[c->world + 1];
    for (int i = 0; i <= c->world; ++i) GR_CUDA(cudaEventCreateWithFlags(&c->ev[i], cudaEventDisableTiming));
  }
  *side = c->side;
  *ev = c->ev;
  return GRANII_OK;
}

granii_status comm_destroy(granii_comm_s* c) {
  if (!c) return GRANII_OK;
  if (c->wd) {
    auto* w = (Watchdog*)c->wd;
    w->shutdown();
    delete w;
    c->wd = nullptr;
  }
  free_side(c);
  if (c->loop) {
    auto* grp = (LoopGroup*)c->loop;
    bool last;
    {
      std::lock_guard<std::mutex> lk(grp->m);
      last = --grp->refs == 0;
    }
    if (last) delete grp;
    delete c;
    return GRANII_OK;
  }
  Nccl* n = nccl();
  if (n && c->nccl) n->destroy((nccl_comm)c->nccl);
  delete c;
  return GRANII_OK;
}

// recv[p*count ..] = peer p's send (p's slot when in place); collective over the group
static granii_status loop_allgather(granii_comm_s* c, const float* send, float* recv, size_t count,
                                    cudaStream_t st) {
  auto* grp = (LoopGroup*)c->loop;
  const int r = c->rank;
  GR_CUDA(cudaEventRecord(grp->ready[r], st));
  grp->src[r] = send;
  grp->barrier();
  for (int p = 0; p < grp->world; ++p) {
    float* dst = recv + (size_t)p * count;
    if (p != r) GR_CUDA(cudaStreamWaitEvent(st, grp->ready[p], 0));
    if (grp->src[p] != dst && count)
      GR_CUDA(cudaMemcpyAsync(dst, grp->src[p], count * sizeof(float), cudaMemcpyDeviceToDevice, st));
  }
  return grp->finish(r, st);
}

// every rank copies block `root` from the root's buffer into its own (same layout)
static granii_status loop_bcast(granii_comm_s* c, float* buf_all, size_t count, int root, cudaStream_t st) {
  auto* grp = (LoopGroup*)c->loop;
  const int r = c->rank;
  float* slot = buf_all + (size_t)root * count;
  GR_CUDA(cudaEventRecord(grp->ready[r], st));
  grp->src[r] = slot;
  grp->barrier();
  if (r != root && count) {
    GR_CUDA(cudaStreamWaitEvent(st, grp->ready[root], 0));
    GR_CUDA(cudaMemcpyAsync(slot, grp->src[root], count * sizeof(float), cudaMemcpyDeviceToDevice, st));
  }
  return grp->finish(r, st);
}

// buf = sum over ranks in rank order (bitwise identical on every rank)
static granii_status loop_allreduce(granii_comm_s* c, float* buf, size_t count, cudaStream_t st) {
  auto* grp = (LoopGroup*)c->loop;
  const int r = c->rank;
  if (grp->stage_cap[r] < count) {
    GR_CUDA(cudaStreamSynchronize(st));
    if (grp->stage[r]) GR_CUDA(cudaFree(grp->stage[r]));
    GR_CUDA(cudaMalloc(&grp->stage[r], count * sizeof(float)));
    grp->stage_cap[r] = count;
  }
  if (count) GR_CUDA(cudaMemcpyAsync(grp->stage[r], buf, count * sizeof(float), cudaMemcpyDeviceToDevice, st));
  GR_CUDA(cudaEventRecord(grp->ready[r], st));
  grp->barrier();
  for (int p = 0; p < grp->world; ++p)
    if (p != r) GR_CUDA(cudaStreamWaitEvent(st, grp->ready[p], 0));
  GR_TRY(launch_rank_sum(grp->world, (const float* const*)grp->stage.data(), count, buf, st));
  return grp->finish(r, st);
}

granii_status comm_create_stub(int32_t rank, int32_t world, granii_comm_s** out) {
  auto* cm = new granii_comm_s();
  cm->stub = 1;
  cm->rank = rank;
  cm->world = world;
  *out = cm;
  return GRANII_OK;
}

granii_status comm_allgather(granii_comm_s* c, const float* send, float* recv, size_t count, cudaStream_t st) {
  if (c) {
    c->bytes_in += (uint64_t)count * sizeof(float) * (uint64_t)(c->world - 1);
    ++c->calls;
    if (c->stub) return GRANII_OK;
    if (c->failed.load()) return comm_failed(c);
  }
  if (c && c->loop) {
    GR_TRY(loop_allgather(c, send, recv, count, st));
    return watch(c, st);
  }
  Nccl* n = nccl();
  if (!n || !c || !c->nccl) return fail(GRANII_ERR_NCCL, "communicator not initialised");
  int rc = n->allgather(send, recv, count, kFloat32, (nccl_comm)c->nccl, st);
  if (rc) return nccl_fail(n, rc, "ncclAllGather");
  return watch(c, st);
}

granii_status comm_bcast_block(granii_comm_s* c, float* buf_all, size_t count, int root, cudaStream_t st) {
  if (c) {
    if (root != c->rank) c->bytes_in += (uint64_t)count * sizeof(float);
    ++c->calls;
    if (c->stub) return GRANII_OK;
    if (c->failed.load()) return comm_failed(c);
  }
  if (c && c->loop) {
    GR_TRY(loop_bcast(c, buf_all, count, root, st));
    return watch(c, st);
  }
  Nccl* n = nccl();
  if (!n || !c || !c->nccl) return fail(GRANII_ERR_NCCL, "communicator not initialised");
  float* slot = buf_all + (size_t)root * count;
  int rc = n->bcast(slot, slot, count, kFloat32, root, (nccl_comm)c->nccl, st);
  if (rc) return nccl_fail(n, rc, "ncclBroadcast");
  return watch(c, st);
}

granii_status comm_allreduce_sum(granii_comm_s* c, float* buf, size_t count, cudaStream_t st) {
  if (c) {  // ring all-reduce: 2 (G-1)/G of the buffer in, per rank
    c->bytes_in += (uint64_t)(2.0 * count * sizeof(float) * (c->world - 1) / c->world);
    ++c->calls;
    if (c->stub) return GRANII_OK;
    if (c->failed.load()) return comm_failed(c);
  }
  if (c && c->loop) {
    GR_TRY(loop_allreduce(c, buf, count, st));
    return watch(c, st);
  }
  Nccl* n = nccl();
  if (!n || !c || !c->nccl) return fail(GRANII_ERR_NCCL, "communicator not initialised");
  int rc = n->allreduce(buf, buf, count, kFloat32, kSum, (nccl_comm)c->nccl, st);
  if (rc) return nccl_fail(n, rc, "ncclAllReduce");
  return watch(c, st);
}

}  // namespace granii
