"""Multi-GPU contiguous sharding: one process per GPU.

Rank g owns a contiguous, chunk-aligned shard of the stream.  It reduces the
shard to a state map over the transformed states (fsm_shard_map: candidate
starts = lookback image of the bytes before the shard, enumerated with
path fusion, then the speculative pipeline), ONE allgather exchanges the maps
(NCCL over NVLink on GPUs; any torch.distributed backend works), and every
rank composes them from q0 and fixes its chunk ends (fsm_shard_finish).

Map layout (fsm_map_bytes): uint32 end[nt] (0xFFFFFFFF = not a candidate),
padded to 8 bytes, then uint64 count[nt]; nt = nstates + 1 (poison last).
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import FSM, Result, _check, _lib, _run_opts, fsm_num_chunks, fsm_result

FSM_EAGAIN = -7  # fsm_shard_finish: a speculative shard map was invalid (include/gspec.h)

NO_STATE = 0xFFFFFFFF


def map_layout(nt: int):
    off = (nt * 4 + 7) & ~7
    return off, off + nt * 8


def shard_bounds(total_len: int, world: int, rank: int, chunk_bytes: int = 4096):
    """Chunk-aligned contiguous shard [lo, hi) of rank among world."""
    nchunks = fsm_num_chunks(total_len, chunk_bytes)
    c0 = nchunks * rank // world
    c1 = nchunks * (rank + 1) // world
    return min(total_len, c0 * chunk_bytes), min(total_len, c1 * chunk_bytes)


def _all_gather_cat(t, group=None):
    """all_gather of equal-size 1-D tensors, concatenated (NCCL: one in-place
    all_gather_into_tensor on the device; other backends stage through host)."""
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    if dist.get_backend(group) == "nccl":
        out = torch.empty(world * t.numel(), dtype=t.dtype, device=t.device)
        dist.all_gather_into_tensor(out, t, group=group)
        return out
    h = t.cpu()
    parts = [torch.empty_like(h) for _ in range(world)]
    dist.all_gather(parts, h, group=group)
    return torch.cat(parts).to(t.device)


def exchange_lookback(shard, group=None, L: int = 16):
    """The last L (<= 16) bytes of the stream before this rank's shard (tiny allgather of
    every rank's tail).  The shard's candidate start set is the image of all states over
    them; a longer window can only shrink it (delta*(Q, uv) is a subset of
    delta*(Q, v)), so the default takes the 16 bytes fsm_shard_map accepts.  They come from the nearest preceding non-empty shards: a shard
    shorter than L (or empty, when there are fewer chunks than ranks) contributes what it
    has and the ranks before it the rest.  Empty only for a shard that starts the stream."""
    import torch
    import torch.distributed as dist

    assert 0 < L <= 16
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    tail = torch.zeros(17, dtype=torch.uint8, device=shard.device)
    n = min(L, shard.numel())
    if n:
        tail[16 - n:16] = shard[shard.numel() - n:]
    tail[16] = n
    tails = _all_gather_cat(tail, group).view(world, 17).cpu()
    parts = []
    for r in range(rank):
        m = int(tails[r, 16].item())
        parts.append(tails[r, 16 - m:16])
    before = torch.cat(parts) if parts else tail[:0].cpu()
    return before[max(0, before.numel() - L):].contiguous().to(shard.device)


def run_sharded(fsm: FSM, shard, lookback, group=None, scheme="auto", chunk_bytes=4096, spec_k=0,
                chunk_ends=True, stream=None) -> Result:
    """fsm_shard_map -> all_gather_into_tensor(maps) -> fsm_shard_finish."""
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    o = _run_opts(scheme, chunk_bytes, spec_k, stream=stream)
    mb = fsm.map_bytes()
    local = torch.empty(mb, dtype=torch.uint8, device=shard.device)
    n = fsm_num_chunks(shard.numel(), chunk_bytes)
    ce = torch.empty(max(n, 1), dtype=torch.int32, device=shard.device) if chunk_ends else None
    lb = lookback if lookback is not None and lookback.numel() else None
    for exact in (False, True):  # speculative map first; FSM_EAGAIN is seen by every rank alike
        fn = _lib.fsm_shard_map_exact if exact else _lib.fsm_shard_map
        map_rc = fn(fsm.handle, shard.data_ptr() if shard.numel() else None, shard.numel(),
                    lb.data_ptr() if lb is not None else None, lb.numel() if lb is not None else 0,
                    ctypes.byref(o), local.data_ptr(), ce.data_ptr() if ce is not None else None)
        # a failed map is published as an error map (every rank's finish reports it), so
        # this rank still joins the collective the others are waiting in
        gathered = _all_gather_cat(local, group)  # the single data-path collective
        r = fsm_result()
        rc = _lib.fsm_shard_finish(fsm.handle, gathered.data_ptr(), world, rank, ctypes.byref(o),
                                   ce.data_ptr() if ce is not None else None, ctypes.byref(r))
        if rc == FSM_EAGAIN:
            continue
        _check(map_rc, "fsm_shard_map")
        break
    _check(rc, "fsm_shard_finish")
    return Result.from_c(r, ce[:n] if ce is not None else None)


# ---- host-side helpers (CPU process groups, tests) ----------------------------
def pack_map(end: np.ndarray, count: np.ndarray) -> np.ndarray:
    """Pack (end[nt] uint32, count[nt] uint64) into the wire layout."""
    nt = len(end)
    off, total = map_layout(nt)
    buf = np.zeros(total, np.uint8)
    buf[:nt * 4] = np.ascontiguousarray(end, np.uint32).view(np.uint8)
    buf[off:off + nt * 8] = np.ascontiguousarray(count, np.uint64).view(np.uint8)
    return buf


def unpack_map(buf: np.ndarray, nt: int):
    off, total = map_layout(nt)
    b = np.ascontiguousarray(buf[:total])
    return b[:nt * 4].view(np.uint32), b[off:off + nt * 8].view(np.uint64)


def p2p_setup(fsm: FSM, group=None):
    """A peer-memory exchange for this handle (fsm_p2p_*): every rank creates its mailbox,
    the 64-byte IPC handles are exchanged with all_gather_object (host plumbing), and every
    rank maps its peers' mailboxes.  Then P2P.run_sharded(fsm, shard, lookback) runs steps
    without a collective library."""
    import torch.distributed as dist

    from . import P2P

    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    p = P2P(fsm, world, rank)
    handles = [None] * world
    dist.all_gather_object(handles, p.handle, group=group)
    p.open(handles)
    dist.barrier(group)
    return p
