// comm.cpp — library-owned NCCL communicator for fsm_run_sharded (the C-ABI
// path for callers without torch.distributed).  NCCL is loaded at run time
// (dlopen "libnccl.so.2"; the process's already-loaded copy wins), so the
// library has no link-time NCCL dependency.  The only collective of the
// sharded method is one ncclAllGather of the per-shard state maps.
#include <dlfcn.h>
#include <nccl.h>
#include <nvtx3/nvToolsExt.h>

#include <cstring>
#include <mutex>
#include <string>

#include "gspec.h"
#include "internal.h"

namespace {

struct NcclApi {
  ncclResult_t (*getUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*commInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*allGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
  const char* (*getErrorString)(ncclResult_t) = nullptr;
  bool ok = false;
};

NcclApi& nccl() {
  static NcclApi api;
  static std::once_flag once;
  std::call_once(once, [] {
    void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return;
    api.getUniqueId = (decltype(api.getUniqueId))dlsym(h, "ncclGetUniqueId");
    api.commInitRank = (decltype(api.commInitRank))dlsym(h, "ncclCommInitRank");
    api.allGather = (decltype(api.allGather))dlsym(h, "ncclAllGather");
    api.commDestroy = (decltype(api.commDestroy))dlsym(h, "ncclCommDestroy");
    api.getErrorString = (decltype(api.getErrorString))dlsym(h, "ncclGetErrorString");
    api.ok = api.getUniqueId && api.commInitRank && api.allGather && api.commDestroy;
  });
  return api;
}

}  // namespace

struct fsm_comm_s {
  ncclComm_t comm = nullptr;
  int nranks = 0, rank = 0;
  void* d_local = nullptr;
  void* d_all = nullptr;
  size_t map_bytes = 0;
};

extern "C" {

int gspec_set_error(int code, const char* msg);  // api.cpp

int fsm_comm_unique_id(void* id_out) {
  if (!id_out) return gspec_set_error(FSM_EINVAL, "NULL id");
  NcclApi& a = nccl();
  if (!a.ok) return gspec_set_error(FSM_ENCCL, "libnccl.so.2 not loadable");
  ncclUniqueId id;
  ncclResult_t r = a.getUniqueId(&id);
  if (r != ncclSuccess) return gspec_set_error(FSM_ENCCL, a.getErrorString ? a.getErrorString(r) : "ncclGetUniqueId");
  std::memcpy(id_out, &id, sizeof(id));
  return FSM_OK;
}

int fsm_comm_init(int nranks, int rank, const void* unique_id, fsm_comm_t* out) {
  if (!unique_id || !out || nranks < 1 || rank < 0 || rank >= nranks) return gspec_set_error(FSM_EINVAL, "bad comm args");
  NcclApi& a = nccl();
  if (!a.ok) return gspec_set_error(FSM_ENCCL, "libnccl.so.2 not loadable");
  ncclUniqueId id;
  std::memcpy(&id, unique_id, sizeof(id));
  fsm_comm_s* c = new fsm_comm_s();
  ncclResult_t r = a.commInitRank(&c->comm, nranks, id, rank);
  if (r != ncclSuccess) {
    delete c;
    return gspec_set_error(FSM_ENCCL, a.getErrorString ? a.getErrorString(r) : "ncclCommInitRank");
  }
  c->nranks = nranks;
  c->rank = rank;
  *out = c;
  return FSM_OK;
}

void fsm_comm_free(fsm_comm_t c) {
  if (!c) return;
  if (c->d_local) cudaFree(c->d_local);
  if (c->d_all) cudaFree(c->d_all);
  if (c->comm && nccl().ok) nccl().commDestroy(c->comm);
  delete c;
}

int fsm_run_sharded(fsm_t f, fsm_comm_t c, const uint8_t* d_shard, uint64_t shard_len, const uint8_t* d_lookback,
                    uint32_t lookback_len, const fsm_run_opts* opts, uint32_t* d_chunk_ends_local,
                    fsm_result* out_global) {
  if (!f || !c || !out_global) return gspec_set_error(FSM_EINVAL, "NULL handle/comm/out");
  const size_t mb = fsm_map_bytes(f);
  if (c->map_bytes < mb) {
    if (c->d_local) cudaFree(c->d_local);
    if (c->d_all) cudaFree(c->d_all);
    c->d_local = c->d_all = nullptr;
    c->map_bytes = 0;
    if (cudaMalloc(&c->d_local, mb) != cudaSuccess || cudaMalloc(&c->d_all, mb * c->nranks) != cudaSuccess)
      return gspec_set_error(FSM_ENOMEM, "map buffers");
    c->map_bytes = mb;
  }
  cudaStream_t st = opts ? reinterpret_cast<cudaStream_t>(opts->stream) : nullptr;
  int rc = FSM_OK;
  for (int exact = 0; exact < 2; exact++) {  // speculative map first; FSM_EAGAIN (same on every rank) -> exact
    rc = exact ? fsm_shard_map_exact(f, d_shard, shard_len, d_lookback, lookback_len, opts, c->d_local,
                                     d_chunk_ends_local)
               : fsm_shard_map(f, d_shard, shard_len, d_lookback, lookback_len, opts, c->d_local, d_chunk_ends_local);
    // a failed map is published as an error map (shard.cu k_map_error) and the exchange
    // still runs, so no rank waits in the allgather for one that returned early
    if (rc && f->shard_mode != 4) return rc;
    const int map_rc = rc;
    nvtxRangePushA("ncclAllGather (shard maps)");
    ncclResult_t r = nccl().allGather(c->d_local, c->d_all, mb, ncclUint8, c->comm, st);
    nvtxRangePop();
    if (r != ncclSuccess)
      return gspec_set_error(FSM_ENCCL, nccl().getErrorString ? nccl().getErrorString(r) : "ncclAllGather");
    rc = fsm_shard_finish(f, c->d_all, (uint32_t)c->nranks, (uint32_t)c->rank, opts, d_chunk_ends_local, out_global);
    if (rc == FSM_EAGAIN) continue;  // every rank (a failed one too) redoes the exact map
    if (map_rc) return map_rc;
    break;
  }
  return rc;
}

// Asynchronous step: map + allgather + queued finish; fsm_shard_wait(ticket) collects.  A
// failed map still joins the exchange (error map) and its status reaches every rank's wait.
int fsm_run_sharded_async(fsm_t f, fsm_comm_t c, const uint8_t* d_shard, uint64_t shard_len,
                          const uint8_t* d_lookback, uint32_t lookback_len, const fsm_run_opts* opts,
                          uint32_t* d_chunk_ends_local, uint64_t* ticket) {
  if (!f || !c || !ticket) return gspec_set_error(FSM_EINVAL, "NULL handle/comm/ticket");
  const size_t mb = fsm_map_bytes(f);
  if (c->map_bytes < mb) {
    if (c->d_local) cudaFree(c->d_local);
    if (c->d_all) cudaFree(c->d_all);
    c->d_local = c->d_all = nullptr;
    c->map_bytes = 0;
    if (cudaMalloc(&c->d_local, mb) != cudaSuccess || cudaMalloc(&c->d_all, mb * c->nranks) != cudaSuccess)
      return gspec_set_error(FSM_ENOMEM, "map buffers");
    c->map_bytes = mb;
  }
  cudaStream_t st = opts ? reinterpret_cast<cudaStream_t>(opts->stream) : nullptr;
  const int rc = fsm_shard_map(f, d_shard, shard_len, d_lookback, lookback_len, opts, c->d_local, d_chunk_ends_local);
  if (rc && f->shard_mode != 4) return rc;
  nvtxRangePushA("ncclAllGather (shard maps)");
  ncclResult_t r = nccl().allGather(c->d_local, c->d_all, mb, ncclUint8, c->comm, st);
  nvtxRangePop();
  if (r != ncclSuccess)
    return gspec_set_error(FSM_ENCCL, nccl().getErrorString ? nccl().getErrorString(r) : "ncclAllGather");
  return fsm_shard_finish_async(f, c->d_all, (uint32_t)c->nranks, (uint32_t)c->rank, opts, d_chunk_ends_local,
                                ticket);
}

}  // extern "C"
