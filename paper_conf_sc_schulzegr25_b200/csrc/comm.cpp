// comm.cpp — NCCL over NVLink 5 / NVSwitch for pw-dim shards.
// NCCL is dlopen'ed on first use, so libmdh loads (and plans) on machines without it.
// The communicator is created from a unique id the caller broadcasts (through
// torch.distributed); every collective is enqueued on the execute stream.
#include <dlfcn.h>
#include <nccl.h>

#include <cstring>
#include <mutex>

#include "internal.h"

namespace mdh {

namespace {
struct Nccl {
  void* h = nullptr;
  ncclResult_t (*getUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*commInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*allGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*allReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t) = nullptr;
  const char* (*getErrorString)(ncclResult_t) = nullptr;
  ncclResult_t (*send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*groupStart)() = nullptr;
  ncclResult_t (*groupEnd)() = nullptr;
  bool ok = false;
};
Nccl g_nccl;
std::once_flag g_once;

void load() {
  const char* names[] = {"libnccl.so.2", "libnccl.so"};
  for (const char* n : names) {
    g_nccl.h = dlopen(n, RTLD_NOW | RTLD_GLOBAL);
    if (g_nccl.h) break;
  }
  if (!g_nccl.h) return;
#define SYM(field, name) g_nccl.field = reinterpret_cast<decltype(g_nccl.field)>(dlsym(g_nccl.h, name))
  SYM(getUniqueId, "ncclGetUniqueId");
  SYM(commInitRank, "ncclCommInitRank");
  SYM(commDestroy, "ncclCommDestroy");
  SYM(allGather, "ncclAllGather");
  SYM(allReduce, "ncclAllReduce");
  SYM(getErrorString, "ncclGetErrorString");
  SYM(send, "ncclSend");
  SYM(recv, "ncclRecv");
  SYM(groupStart, "ncclGroupStart");
  SYM(groupEnd, "ncclGroupEnd");
#undef SYM
  g_nccl.ok = g_nccl.getUniqueId && g_nccl.commInitRank && g_nccl.commDestroy && g_nccl.allGather &&
              g_nccl.allReduce && g_nccl.getErrorString;
}

mdh_status need() {
  std::call_once(g_once, load);
  if (!g_nccl.ok) {
    set_error("NCCL (libnccl.so.2) could not be loaded");
    return MDH_ERR_NCCL;
  }
  return MDH_OK;
}

mdh_status chk(ncclResult_t r, const char* what) {
  if (r == ncclSuccess) return MDH_OK;
  set_error("NCCL error in %s: %s", what, g_nccl.getErrorString(r));
  return MDH_ERR_NCCL;
}
}  // namespace

mdh_status comm_unique_id(void* id128) {
  if (!id128) { set_error("NULL id"); return MDH_ERR_INVALID_ARG; }
  MDH_TRY(need());
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
  ncclUniqueId id;
  MDH_TRY(chk(g_nccl.getUniqueId(&id), "ncclGetUniqueId"));
  std::memcpy(id128, &id, sizeof(id));
  return MDH_OK;
}

mdh_status comm_init(const void* id128, int world, int rank, int device, void** comm) {
  if (!id128 || !comm || world < 1 || rank < 0 || rank >= world) { set_error("bad comm_init arguments"); return MDH_ERR_INVALID_ARG; }
  MDH_TRY(need());
  MDH_CUDA(cudaSetDevice(device));
  ncclUniqueId id;
  std::memcpy(&id, id128, sizeof(id));
  ncclComm_t c = nullptr;
  MDH_TRY(chk(g_nccl.commInitRank(&c, world, id, rank), "ncclCommInitRank"));
  *comm = c;
  return MDH_OK;
}

mdh_status comm_destroy(void* comm) {
  if (!comm) return MDH_OK;
  MDH_TRY(need());
  return chk(g_nccl.commDestroy((ncclComm_t)comm), "ncclCommDestroy");
}

mdh_status comm_allgather(void* comm, const void* send, void* recv, size_t bytes, cudaStream_t st) {
  MDH_TRY(need());
  return chk(g_nccl.allGather(send, recv, bytes, ncclUint8, (ncclComm_t)comm, st), "ncclAllGather");
}

mdh_status comm_allreduce(void* comm, const void* send, void* recv, size_t count, mdh_dtype dt, mdh_combine op,
                          cudaStream_t st) {
  MDH_TRY(need());
  ncclDataType_t t;
  switch (dt) {
    case MDH_F32: t = ncclFloat32; break;
    case MDH_F64: t = ncclFloat64; break;
    case MDH_BF16: t = ncclBfloat16; break;
    case MDH_I32: t = (op == MDH_PW_ADD) ? ncclUint32 : ncclInt32; break;   // wrap sum (C-12)
    case MDH_U32: t = ncclUint32; break;
    case MDH_I64: t = (op == MDH_PW_ADD) ? ncclUint64 : ncclInt64; break;
    default: set_error("allreduce: bad dtype"); return MDH_ERR_UNSUPPORTED;
  }
  ncclRedOp_t o = op == MDH_PW_ADD ? ncclSum : (op == MDH_PW_MAX ? ncclMax : ncclMin);
  return chk(g_nccl.allReduce(send, recv, count, t, o, (ncclComm_t)comm, st), "ncclAllReduce");
}

// Halo exchange of a z-slab after a sweep (reading C-34): my first owned plane
// (local plane 1) to the lower neighbour, whose copy lands in my plane 0 from it, and my
// last owned plane (nz-2) to the upper neighbour / plane nz-1 from it.  One NCCL group, so
// the four point-to-point transfers proceed together over NVLink.
mdh_status comm_halo_exchange(void* comm, int rank, int world, char* buf, size_t plane_bytes, int64_t nz,
                              cudaStream_t st) {
  MDH_TRY(need());
  if (!g_nccl.send || !g_nccl.recv || !g_nccl.groupStart || !g_nccl.groupEnd) {
    set_error("this NCCL has no ncclSend/ncclRecv (needs >= 2.7)");
    return MDH_ERR_NCCL;
  }
  ncclComm_t c = (ncclComm_t)comm;
  MDH_TRY(chk(g_nccl.groupStart(), "ncclGroupStart"));
  // record the first failure but always close the group: an open group would capture
  // this thread's later NCCL calls
  mdh_status e = MDH_OK;
  auto step = [&e](mdh_status s) { if (e == MDH_OK) e = s; };
  if (rank > 0) {
    step(chk(g_nccl.send(buf + plane_bytes, plane_bytes, ncclUint8, rank - 1, c, st), "ncclSend"));
    step(chk(g_nccl.recv(buf, plane_bytes, ncclUint8, rank - 1, c, st), "ncclRecv"));
  }
  if (rank < world - 1) {
    step(chk(g_nccl.send(buf + (nz - 2) * plane_bytes, plane_bytes, ncclUint8, rank + 1, c, st), "ncclSend"));
    step(chk(g_nccl.recv(buf + (nz - 1) * plane_bytes, plane_bytes, ncclUint8, rank + 1, c, st), "ncclRecv"));
  }
  const mdh_status g = chk(g_nccl.groupEnd(), "ncclGroupEnd");
  return e != MDH_OK ? e : g;
}

}  // namespace mdh
