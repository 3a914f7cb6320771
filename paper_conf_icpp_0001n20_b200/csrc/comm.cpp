// comm.cpp -- NCCL for the 1-D partitioned multi-GPU path.
// NCCL is dlopen'ed at run time (torch's bundled libnccl.so.2, located by the
// binding through GX_NCCL_LIB) so that single-GPU use never needs it.
#include <dlfcn.h>

#include <cstdlib>
#include <cstring>
#include <vector>

#include "gx_internal.h"

namespace gx {
void set_last_error(const std::string& m);   // capi.cpp
namespace nccl {
typedef struct { char internal[128]; } UniqueId;
typedef void* Comm;
typedef int (*GetUniqueId_t)(UniqueId*);
typedef int (*CommInitRank_t)(Comm*, int, UniqueId, int);
typedef int (*CommDestroy_t)(Comm);
typedef int (*AllReduce_t)(const void*, void*, size_t, int, int, Comm, cudaStream_t);
typedef int (*AllGather_t)(const void*, void*, size_t, int, Comm, cudaStream_t);
typedef int (*ReduceScatter_t)(const void*, void*, size_t, int, int, Comm, cudaStream_t);
typedef int (*Broadcast_t)(const void*, void*, size_t, int, int, Comm, cudaStream_t);
typedef int (*Reduce_t)(const void*, void*, size_t, int, int, int, Comm, cudaStream_t);
typedef int (*Group_t)();
typedef const char* (*GetErrorString_t)(int);
struct Api {
  void* h = nullptr;
  GetUniqueId_t getUniqueId = nullptr;
  CommInitRank_t commInitRank = nullptr;
  CommDestroy_t commDestroy = nullptr;
  AllReduce_t allReduce = nullptr;
  AllGather_t allGather = nullptr;
  ReduceScatter_t reduceScatter = nullptr;
  Broadcast_t broadcast = nullptr;
  Reduce_t reduce = nullptr;
  Group_t groupStart = nullptr, groupEnd = nullptr;
  GetErrorString_t err = nullptr;
};
Api& api() {
  static Api a;
  if (!a.h) {
    const char* p = std::getenv("GX_NCCL_LIB");
    a.h = dlopen(p && *p ? p : "libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!a.h) GX_THROW(GX_E_NCCL, std::string("cannot dlopen NCCL: ") + dlerror());
    a.getUniqueId = (GetUniqueId_t)dlsym(a.h, "ncclGetUniqueId");
    a.commInitRank = (CommInitRank_t)dlsym(a.h, "ncclCommInitRank");
    a.commDestroy = (CommDestroy_t)dlsym(a.h, "ncclCommDestroy");
    a.allReduce = (AllReduce_t)dlsym(a.h, "ncclAllReduce");
    a.allGather = (AllGather_t)dlsym(a.h, "ncclAllGather");
    a.reduceScatter = (ReduceScatter_t)dlsym(a.h, "ncclReduceScatter");
    a.broadcast = (Broadcast_t)dlsym(a.h, "ncclBroadcast");
    a.reduce = (Reduce_t)dlsym(a.h, "ncclReduce");
    a.groupStart = (Group_t)dlsym(a.h, "ncclGroupStart");
    a.groupEnd = (Group_t)dlsym(a.h, "ncclGroupEnd");
    a.err = (GetErrorString_t)dlsym(a.h, "ncclGetErrorString");
    if (!a.getUniqueId || !a.commInitRank || !a.allReduce || !a.allGather || !a.reduceScatter || !a.broadcast ||
        !a.reduce || !a.groupStart || !a.groupEnd)
      GX_THROW(GX_E_NCCL, "NCCL symbols missing");
  }
  return a;
}
void check(int r, const char* what) {
  if (r != 0) GX_THROW(GX_E_NCCL, std::string(what) + ": " + (api().err ? api().err(r) : "error"));
}
}  // namespace nccl

// ncclDataType / ncclRedOp values (nccl.h)
enum { NCCL_INT32 = 2, NCCL_UINT32 = 3, NCCL_FLOAT32 = 7, NCCL_FLOAT64 = 8, NCCL_UINT64 = 5 };
enum { NCCL_SUM = 0, NCCL_MAX = 2, NCCL_MIN = 3 };

void comm_allreduce(Ctx* c, const void* in, void* out, size_t count, int dtype, int op) {
  nccl::check(nccl::api().allReduce(in, out, count, dtype, op, c->nccl, c->stream), "ncclAllReduce");
}

static bool equal_counts(const std::vector<int64_t>& off) {
  for (size_t p = 1; p + 1 < off.size(); p++)
    if (off[p + 1] - off[p] != off[1] - off[0]) return false;
  return true;
}

// in place: rank p's slice [off[p], off[p+1]) of buf reaches every rank.
// Equal slices: one ncclAllGather (in place: sendbuff = recvbuff + rank *
// count); else the allgather-v as one group of P broadcasts, root p sending
// its slice (NCCL has no native allgather-v).
void comm_allgatherv(Ctx* c, void* buf, const std::vector<int64_t>& off, int dtype, size_t esize) {
  auto& A = nccl::api();
  char* b = static_cast<char*>(buf);
  if (equal_counts(off)) {
    const size_t cnt = (size_t)(off[1] - off[0]);
    nccl::check(A.allGather(b + off[c->rank] * esize, b, cnt, dtype, c->nccl, c->stream), "ncclAllGather");
    return;
  }
  nccl::check(A.groupStart(), "ncclGroupStart");
  for (int p = 0; p < c->world; p++) {
    char* sl = b + off[p] * esize;
    nccl::check(A.broadcast(sl, sl, (size_t)(off[p + 1] - off[p]), dtype, p, c->nccl, c->stream), "ncclBroadcast");
  }
  nccl::check(A.groupEnd(), "ncclGroupEnd");
}

// in place: afterwards rank r's slice [off[r], off[r+1]) holds the reduction
// over every rank's copy of that slice; the rest of buf is left as it was.
// Equal slices: one ncclReduceScatter (recvbuff = sendbuff + rank * count);
// else a group of P reduces, root p receiving its slice.
void comm_reduce_scatterv(Ctx* c, void* buf, const std::vector<int64_t>& off, int dtype, int op, size_t esize) {
  auto& A = nccl::api();
  char* b = static_cast<char*>(buf);
  if (equal_counts(off)) {
    const size_t cnt = (size_t)(off[1] - off[0]);
    nccl::check(A.reduceScatter(b, b + off[c->rank] * esize, cnt, dtype, op, c->nccl, c->stream),
                "ncclReduceScatter");
    return;
  }
  nccl::check(A.groupStart(), "ncclGroupStart");
  for (int p = 0; p < c->world; p++) {
    char* sl = b + off[p] * esize;
    nccl::check(A.reduce(sl, sl, (size_t)(off[p + 1] - off[p]), dtype, op, p, c->nccl, c->stream), "ncclReduce");
  }
  nccl::check(A.groupEnd(), "ncclGroupEnd");
}
}  // namespace gx

extern "C" {
void gx_comm_destroy(void* comm) {
  if (comm) gx::nccl::api().commDestroy(comm);
}

gx_status gx_get_nccl_unique_id(uint8_t out[128]) {
  try {
    if (!out) return GX_E_INVALID;
    gx::nccl::UniqueId id;
    gx::nccl::check(gx::nccl::api().getUniqueId(&id), "ncclGetUniqueId");
    std::memcpy(out, id.internal, 128);
    return GX_OK;
  } catch (const gx::Error& e) {
    gx::set_last_error(e.what());
    return e.st;
  }
}

gx_status gx_ctx_create(gx_ctx** out, int device, void* cuda_stream);

gx_status gx_ctx_create_hosted(gx_ctx** out, int device, void* cuda_stream, int rank, int world, gx_coll_fn fn,
                               void* user) {
  if (!out || !fn || world < 1 || rank < 0 || rank >= world) return GX_E_INVALID;
  gx_status s = gx_ctx_create(out, device, cuda_stream);
  if (s != GX_OK) return s;
  (*out)->coll = fn;
  (*out)->coll_user = user;
  (*out)->rank = rank;
  (*out)->world = world;
  return GX_OK;
}

gx_status gx_ctx_create_dist(gx_ctx** out, int device, void* cuda_stream, int rank, int world,
                             const uint8_t id[128]) {
  if (!out || !id || world < 1 || rank < 0 || rank >= world) return GX_E_INVALID;
  gx_status s = gx_ctx_create(out, device, cuda_stream);
  if (s != GX_OK) return s;
  try {
    gx::nccl::UniqueId uid;
    std::memcpy(uid.internal, id, 128);
    void* comm = nullptr;
    gx::nccl::check(gx::nccl::api().commInitRank(&comm, world, uid, rank), "ncclCommInitRank");
    (*out)->nccl = comm;
    (*out)->rank = rank;
    (*out)->world = world;
    return GX_OK;
  } catch (const gx::Error& e) {
    gx::set_last_error(e.what());
    gx_ctx_destroy(*out);
    *out = nullptr;
    return e.st;
  }
}
}
