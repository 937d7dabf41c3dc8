// comm.cpp — library-owned NCCL communicator for fsm_run_sharded (the C-ABI
// path for callers without torch.distributed).  NCCL is loaded at run time
// (dlopen "libnccl.so.2"; the process's already-loaded copy wins), so the
// library has no link-time NCCL dependency.  The only collective of the
// sharded method is one ncclAllGather of the per-shard state maps.
#include <dlfcn.h>
#include <nccl.h>
#include <nvtx3/nvToolsExt.h>

#include <algorithm>
#include <cstring>
#include <mutex>
#include <vector>
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

int fsm_comm_init(int nranks, int rank, const void* unique_id, int device, fsm_comm_t* out) {
  if (!unique_id || !out || nranks < 1 || rank < 0 || rank >= nranks) return gspec_set_error(FSM_EINVAL, "bad comm args");
  NcclApi& a = nccl();
  if (!a.ok) return gspec_set_error(FSM_ENCCL, "libnccl.so.2 not loadable");
  if (device >= 0 && cudaSetDevice(device) != cudaSuccess) return gspec_set_error(FSM_EINVAL, "bad device");
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

// The SURVEY §8(b) signature: the caller passes its shard's place in the stream and the
// library fetches the lookback bytes itself — every rank's last 16 bytes are gathered with
// one tiny ncclAllGather (17 bytes per rank: bytes + count) and the 16 bytes before this
// shard are taken from the nearest preceding non-empty shards (shard_offset 0: none).
int fsm_run_sharded_at(fsm_t f, fsm_comm_t c, const uint8_t* d_shard, uint64_t shard_offset, uint64_t shard_len,
                       uint64_t total_len, const fsm_run_opts* opts, uint32_t* d_chunk_ends_local,
                       fsm_result* out_global) {
  if (!f || !c || !out_global) return gspec_set_error(FSM_EINVAL, "NULL handle/comm/out");
  const uint32_t B = (opts && opts->chunk_bytes) ? opts->chunk_bytes : 4096;
  if (shard_offset % B != 0 || shard_offset + shard_len > total_len)
    return gspec_set_error(FSM_EINVAL, "shard not chunk-aligned / outside the stream");
  cudaStream_t st = opts ? reinterpret_cast<cudaStream_t>(opts->stream) : nullptr;
  const int G = c->nranks;
  uint8_t *d_tail = nullptr, *d_tails = nullptr;
  if (cudaMalloc(&d_tail, 32) != cudaSuccess || cudaMalloc(&d_tails, 32 * (size_t)G) != cudaSuccess) {
    if (d_tail) cudaFree(d_tail);
    return gspec_set_error(FSM_ENOMEM, "tail buffers");
  }
  const uint32_t n = (uint32_t)(shard_len < 16 ? shard_len : 16);
  cudaMemsetAsync(d_tail, 0, 32, st);
  if (n) cudaMemcpyAsync(d_tail + 16 - n, d_shard + shard_len - n, n, cudaMemcpyDeviceToDevice, st);
  const uint8_t nb = (uint8_t)n;
  cudaMemcpyAsync(d_tail + 16, &nb, 1, cudaMemcpyHostToDevice, st);
  ncclResult_t r = nccl().allGather(d_tail, d_tails, 32, ncclUint8, c->comm, st);
  std::vector<uint8_t> tails(32 * (size_t)G);
  if (r == ncclSuccess)
    cudaMemcpyAsync(tails.data(), d_tails, tails.size(), cudaMemcpyDeviceToHost, st);
  const cudaError_t ce = cudaStreamSynchronize(st);
  cudaFree(d_tail);
  cudaFree(d_tails);
  if (r != ncclSuccess) return gspec_set_error(FSM_ENCCL, "ncclAllGather (tails)");
  if (ce != cudaSuccess) return gspec_set_error(FSM_ECUDA, "tail exchange");
  std::vector<uint8_t> before;  // the stream's bytes before this shard, nearest last
  for (int g = 0; g < c->rank; g++) {
    const uint8_t m = tails[32 * (size_t)g + 16];
    before.insert(before.end(), tails.begin() + 32 * (size_t)g + 16 - m, tails.begin() + 32 * (size_t)g + 16);
  }
  const size_t L = shard_offset == 0 ? 0 : std::min<size_t>(16, before.size());
  uint8_t* d_lb = nullptr;
  if (L) {
    if (cudaMalloc(&d_lb, 16) != cudaSuccess) return gspec_set_error(FSM_ENOMEM, "lookback buffer");
    cudaMemcpy(d_lb, before.data() + before.size() - L, L, cudaMemcpyHostToDevice);
  }
  const int rc = fsm_run_sharded(f, c, d_shard, shard_len, d_lb, (uint32_t)L, opts, d_chunk_ends_local, out_global);
  if (d_lb) cudaFree(d_lb);
  return rc;
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
