// p2p.cu — the state-map exchange of a sharded run without a collective library
// (SURVEY §8(e) "fused alternative"): every rank owns a mailbox in its
// own HBM — two sets (by step parity) of G map slots plus G arrival flags — mapped into
// every peer through CUDA IPC (NVLink / NVSwitch peer memory between GPUs).  A step is
//   map kernels (fsm_shard_map, into this rank's own slot); in the fused mode the last
//      of them, k_map_fused_publish (shard.cu), writes the candidates' map entries AND
//      stores the finished map into slot [rank] of every peer's mailbox, fences
//      system-wide and raises the flag [rank] there — the compute step and the exchange in
//      one kernel, no NCCL launch; the other modes publish with k_publish (the same stores)
//   -> fsm_shard_finish over the own mailbox (compose, fix-up), as after an allgather; its
//      composition kernel (k_compose, shard.cu) first spins (nanosleep, bounded) until every
//      peer's flag for this step has arrived — the wait fused into the receiver's compose.
// Steps alternate between the two sets, so a fast rank's next publish never overwrites
// a map a slow peer is still composing.
#include <cuda_runtime.h>

#include <cstring>
#include <vector>

#include "gspec.h"
#include "internal.h"

namespace gspec {
namespace {

// one CTA: copy this rank's map (mapb bytes, 16-aligned) into slot [rank] of set `set` of
// every peer's mailbox, then raise this rank's flag in each of them
__global__ void __launch_bounds__(1024) k_publish(const uint8_t* __restrict__ own_map, uint64_t mapb,
                                                 uint8_t* const* __restrict__ peers, uint32_t G, uint32_t rank,
                                                 uint32_t set, unsigned long long seq) {
  const uint64_t words = mapb / 16;
  const uint4* src = reinterpret_cast<const uint4*>(own_map);
  for (uint32_t g = 0; g < G; g++) {
    if (g == rank) continue;
    uint4* dst = reinterpret_cast<uint4*>(peers[g] + ((uint64_t)set * G + rank) * mapb);
    for (uint64_t i = threadIdx.x; i < words; i += blockDim.x) dst[i] = __ldcg(src + i);
  }
  __threadfence_system();  // the map bytes are visible system-wide before any flag
  __syncthreads();
  if (threadIdx.x < G && threadIdx.x != rank) {
    unsigned long long* flags = reinterpret_cast<unsigned long long*>(peers[threadIdx.x] + 2ull * G * mapb);
    *reinterpret_cast<volatile unsigned long long*>(flags + (uint64_t)set * G + rank) = seq;
  }
}

}  // namespace

cudaError_t launch_publish(const uint8_t* own_map, uint64_t mapb, uint8_t* const* peers, uint32_t G, uint32_t rank,
                           uint32_t set, unsigned long long seq, cudaStream_t st) {
  k_publish<<<1, 1024, 0, st>>>(own_map, mapb, peers, G, rank, set, seq);
  return cudaGetLastError();
}


}  // namespace gspec

struct fsm_p2p_s {
  int nranks = 0, rank = 0;
  uint64_t mapb = 0;            // slot stride (fsm_map_bytes rounded up to 16)
  uint8_t* box = nullptr;       // own mailbox: [2][G] maps, then [2][G] u64 flags
  size_t box_bytes = 0;
  uint8_t** d_peers = nullptr;  // device [G]: every rank's mailbox as mapped here (own at [rank])
  std::vector<void*> opened;    // peers' mailboxes opened through IPC
  uint32_t* d_status = nullptr;
  uint32_t* h_status = nullptr;  // pinned
  unsigned long long seq = 0;
  bool open = false;
};

extern "C" {

int gspec_set_error(int code, const char* msg);  // api.cpp

int fsm_p2p_create(fsm_t f, int nranks, int rank, void* ipc_handle_out, fsm_p2p_t* out) {
  if (!f || !ipc_handle_out || !out || nranks < 1 || rank < 0 || rank >= nranks)
    return gspec_set_error(FSM_EINVAL, "bad p2p arguments");
  fsm_p2p_s* p = new fsm_p2p_s();
  p->nranks = nranks;
  p->rank = rank;
  p->mapb = (fsm_map_bytes(f) + 15) & ~15ull;
  p->box_bytes = 2ull * nranks * p->mapb + 2ull * nranks * 8;
  cudaIpcMemHandle_t h;
  if (cudaMalloc(&p->box, p->box_bytes) != cudaSuccess || cudaMemset(p->box, 0, p->box_bytes) != cudaSuccess ||
      cudaMalloc(&p->d_peers, sizeof(uint8_t*) * nranks) != cudaSuccess ||
      cudaMalloc(&p->d_status, 16) != cudaSuccess || cudaMallocHost(&p->h_status, 16) != cudaSuccess ||
      cudaIpcGetMemHandle(&h, p->box) != cudaSuccess) {
    fsm_p2p_free(p);
    return gspec_set_error(FSM_ECUDA, "p2p mailbox allocation / IPC handle");
  }
  std::memcpy(ipc_handle_out, &h, sizeof(h));
  *out = p;
  return FSM_OK;
}

int fsm_p2p_open(fsm_p2p_t p, const void* ipc_handles) {
  if (!p || !ipc_handles) return gspec_set_error(FSM_EINVAL, "NULL p2p/handles");
  std::vector<uint8_t*> ptrs(p->nranks, nullptr);
  for (int g = 0; g < p->nranks; g++) {
    if (g == p->rank) {
      ptrs[g] = p->box;
      continue;
    }
    cudaIpcMemHandle_t h;
    std::memcpy(&h, static_cast<const uint8_t*>(ipc_handles) + (size_t)g * sizeof(h), sizeof(h));
    void* q = nullptr;
    if (cudaIpcOpenMemHandle(&q, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess)
      return gspec_set_error(FSM_ECUDA, "cudaIpcOpenMemHandle of a peer's mailbox");
    p->opened.push_back(q);
    ptrs[g] = static_cast<uint8_t*>(q);
  }
  if (cudaMemcpy(p->d_peers, ptrs.data(), sizeof(uint8_t*) * p->nranks, cudaMemcpyHostToDevice) != cudaSuccess)
    return gspec_set_error(FSM_ECUDA, "p2p peer table");
  p->open = true;
  return FSM_OK;
}

void fsm_p2p_free(fsm_p2p_t p) {
  if (!p) return;
  for (void* q : p->opened) cudaIpcCloseMemHandle(q);
  if (p->box) cudaFree(p->box);
  if (p->d_peers) cudaFree(p->d_peers);
  if (p->d_status) cudaFree(p->d_status);
  if (p->h_status) cudaFreeHost(p->h_status);
  delete p;
}

int fsm_run_sharded_p2p(fsm_t f, fsm_p2p_t p, const uint8_t* d_shard, uint64_t shard_len, const uint8_t* d_lookback,
                        uint32_t lookback_len, const fsm_run_opts* opts, uint32_t* d_chunk_ends_local,
                        fsm_result* out_global) {
  if (!f || !p || !out_global) return gspec_set_error(FSM_EINVAL, "NULL handle/p2p/out");
  if (!p->open) return gspec_set_error(FSM_EINVAL, "fsm_p2p_open was not called");
  if (((fsm_map_bytes(f) + 15) & ~15ull) != p->mapb) return gspec_set_error(FSM_EINVAL, "p2p mailbox of another DFA");
  cudaStream_t st = opts ? reinterpret_cast<cudaStream_t>(opts->stream) : nullptr;
  const uint32_t G = (uint32_t)p->nranks, rank = (uint32_t)p->rank;
  int rc = FSM_OK;
  for (int exact = 0; exact < 2; exact++) {  // speculative map first; FSM_EAGAIN (same on every rank) -> exact
    const unsigned long long seq = ++p->seq;
    const uint32_t set = (uint32_t)(seq & 1);
    uint8_t* own_slot = p->box + ((uint64_t)set * G + rank) * p->mapb;
    // the fused-mode map kernel sends the map itself (k_map_fused_publish); the other modes
    // (exact fallbacks, ENUM shards, an error map) publish with k_publish afterwards
    const fsm_s::P2PPub pub{p->mapb, p->d_peers, G, rank, set, seq};
    f->p2p_pub = &pub;
    f->p2p_published = false;
    rc = exact ? fsm_shard_map_exact(f, d_shard, shard_len, d_lookback, lookback_len, opts, own_slot,
                                     d_chunk_ends_local)
               : fsm_shard_map(f, d_shard, shard_len, d_lookback, lookback_len, opts, own_slot, d_chunk_ends_local);
    f->p2p_pub = nullptr;
    if (rc && f->shard_mode != 4) return rc;  // (a failed map publishes its error map like any other)
    const int map_rc = rc;
    const bool sent = f->p2p_published && !rc;
    if (!sent && gspec::launch_publish(own_slot, p->mapb, p->d_peers, G, rank, set, seq, st) != cudaSuccess)
      return gspec_set_error(FSM_ECUDA, "p2p publish launch");
    // the receiver side: fsm_shard_finish's composition kernel waits for the peers' flags of
    // this step before it reads a map (k_compose's wflags) — no separate wait kernel
    const fsm_s::P2PWait wt{reinterpret_cast<const unsigned long long*>(p->box + 2ull * G * p->mapb) +
                                (uint64_t)set * G,
                            seq, p->d_status};
    if (cudaMemsetAsync(p->d_status, 0, 4, st) != cudaSuccess)  // (a finish that fails early leaves it 0)
      return gspec_set_error(FSM_ECUDA, "p2p status reset");
    f->p2p_wait = &wt;
    rc = fsm_shard_finish(f, p->box + (uint64_t)set * G * p->mapb, G, rank, opts, d_chunk_ends_local, out_global);
    f->p2p_wait = nullptr;
    if (cudaMemcpyAsync(p->h_status, p->d_status, 4, cudaMemcpyDeviceToHost, st) != cudaSuccess)
      return gspec_set_error(FSM_ECUDA, "p2p status readback");
    if (cudaStreamSynchronize(st) != cudaSuccess) return gspec_set_error(FSM_ECUDA, "p2p step");
    if (*p->h_status) return gspec_set_error(FSM_ENCCL, "p2p exchange: a peer never published its map");
    if (rc == FSM_EAGAIN) continue;  // every rank redoes the exact map
    if (map_rc) return map_rc;
    break;
  }
  return rc;
}

}  // extern "C"
