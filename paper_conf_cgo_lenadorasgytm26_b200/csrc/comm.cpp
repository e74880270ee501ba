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

#include <condition_variable>
#include <cstring>
#include <mutex>
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
  }
  if (c && c->loop) return loop_allgather(c, send, recv, count, st);
  Nccl* n = nccl();
  if (!n || !c || !c->nccl) return fail(GRANII_ERR_NCCL, "communicator not initialised");
  int rc = n->allgather(send, recv, count, kFloat32, (nccl_comm)c->nccl, st);
  if (rc) return nccl_fail(n, rc, "ncclAllGather");
  return GRANII_OK;
}

granii_status comm_bcast_block(granii_comm_s* c, float* buf_all, size_t count, int root, cudaStream_t st) {
  if (c) {
    if (root != c->rank) c->bytes_in += (uint64_t)count * sizeof(float);
    ++c->calls;
    if (c->stub) return GRANII_OK;
  }
  if (c && c->loop) return loop_bcast(c, buf_all, count, root, st);
  Nccl* n = nccl();
  if (!n || !c || !c->nccl) return fail(GRANII_ERR_NCCL, "communicator not initialised");
  float* slot = buf_all + (size_t)root * count;
  int rc = n->bcast(slot, slot, count, kFloat32, root, (nccl_comm)c->nccl, st);
  if (rc) return nccl_fail(n, rc, "ncclBroadcast");
  return GRANII_OK;
}

granii_status comm_allreduce_sum(granii_comm_s* c, float* buf, size_t count, cudaStream_t st) {
  if (c) {  // ring all-reduce: 2 (G-1)/G of the buffer in, per rank
    c->bytes_in += (uint64_t)(2.0 * count * sizeof(float) * (c->world - 1) / c->world);
    ++c->calls;
    if (c->stub) return GRANII_OK;
  }
  if (c && c->loop) return loop_allreduce(c, buf, count, st);
  Nccl* n = nccl();
  if (!n || !c || !c->nccl) return fail(GRANII_ERR_NCCL, "communicator not initialised");
  int rc = n->allreduce(buf, buf, count, kFloat32, kSum, (nccl_comm)c->nccl, st);
  if (rc) return nccl_fail(n, rc, "ncclAllReduce");
  return GRANII_OK;
}

}  // namespace granii
