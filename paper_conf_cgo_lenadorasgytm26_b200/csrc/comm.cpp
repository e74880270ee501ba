// comm.cpp -- NCCL communicator for the row-partitioned multi-GPU layer
// (north_star (4): all-gather of dense embeddings over NVLink for the SpMM,
// all-reduce of dW).  NCCL is resolved at run time with dlopen (the copy
// PyTorch already loaded is reused via RTLD_NOLOAD), so the library loads on
// machines without NCCL and only granii_comm_* need it.
#include <dlfcn.h>

#include <cstring>
#include <mutex>

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
    n.destroy = (fn_destroy)dlsym(h, "ncclCommDestroy");
    n.errstr = (fn_errstr)dlsym(h, "ncclGetErrorString");
  });
  return (n.h && n.get_uid && n.init_rank && n.allgather && n.allreduce && n.destroy) ? &n : nullptr;
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

granii_status comm_destroy(granii_comm_s* c) {
  if (!c) return GRANII_OK;
  Nccl* n = nccl();
  if (n && c->nccl) n->destroy((nccl_comm)c->nccl);
  delete c;
  return GRANII_OK;
}

granii_status comm_allgather(granii_comm_s* c, const float* send, float* recv, size_t count, cudaStream_t st) {
  Nccl* n = nccl();
  if (!n || !c || !c->nccl) return fail(GRANII_ERR_NCCL, "communicator not initialised");
  int rc = n->allgather(send, recv, count, kFloat32, (nccl_comm)c->nccl, st);
  if (rc) return nccl_fail(n, rc, "ncclAllGather");
  return GRANII_OK;
}

granii_status comm_allreduce_sum(granii_comm_s* c, float* buf, size_t count, cudaStream_t st) {
  Nccl* n = nccl();
  if (!n || !c || !c->nccl) return fail(GRANII_ERR_NCCL, "communicator not initialised");
  int rc = n->allreduce(buf, buf, count, kFloat32, kSum, (nccl_comm)c->nccl, st);
  if (rc) return nccl_fail(n, rc, "ncclAllReduce");
  return GRANII_OK;
}

}  // namespace granii
