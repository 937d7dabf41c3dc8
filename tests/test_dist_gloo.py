"""World-size-2 gloo tests (CPU) of the multi-GPU host logic: shard bounds,
map wire format, the one allgather of per-shard state maps, and composition
(DESIGN.md §Multi-GPU).  Per-shard maps come from the oracle here (no GPU);
the GPU computes them with fsm_shard_map in tests/test_gpu_shard.py."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import gen
import oracle


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def oracle_shard_map(w, data, lo, hi, B):
    """State map of shard [lo,hi): candidates = lookback image of the 2 bytes before."""
    from paper_conf_ipps_wangwqw22_b200.dist import NO_STATE, pack_map

    perm, inv, _, tt, acc = oracle.transform(w.table, w.accept)
    n = w.nstates
    nt = n + 1
    if lo == 0:
        cands = [int(perm[w.start])]
    else:
        cands, _ = oracle.lookback(tt, n, data[lo - 2:lo], K=nt)
        cands = [int(c) for c in cands]
    end = np.full(nt, NO_STATE, np.uint32)
    cnt = np.zeros(nt, np.uint64)
    for s in cands:
        r = oracle.run(tt, s, acc, data[lo:hi], B)
        end[s] = r["final"] if hi > lo else s
        cnt[s] = r["count"] if hi > lo else 0
    return pack_map(end, cnt), perm, inv


def compose_maps(maps, nt, q0t):
    """Test-side composition of the gathered maps (the library's is k_compose, shard.cu):
    s_0 = q0; s_{g+1} = M_g[s_g]; count = sum_g C_g[s_g]."""
    from paper_conf_ipps_wangwqw22_b200.dist import NO_STATE, unpack_map

    s, total, starts = q0t, 0, [q0t]
    for g in range(maps.shape[0]):
        e, c = unpack_map(maps[g], nt)
        assert int(e[s]) != NO_STATE, f"shard {g}: start state {s} not in its candidate set"
        total += int(c[s])
        s = int(e[s])
        starts.append(s)
    return starts, total


def _worker(rank, world, port, name, length, B, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_wangwqw22_b200.dist import shard_bounds

    w = gen.workload(name, length=length)
    data = w.host()
    lo, hi = shard_bounds(length, world, rank, B)
    buf, perm, inv = oracle_shard_map(w, data, lo, hi, B)
    local = torch.from_numpy(buf)
    gathered = [torch.empty_like(local) for _ in range(world)]
    dist.all_gather(gathered, local)  # the single data-path collective
    maps = torch.stack(gathered).numpy()
    starts, count = compose_maps(maps, w.nstates + 1, int(perm[w.start]))
    q.put((rank, int(inv[starts[-1]]), count, int(inv[starts[rank]]), lo))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("name,length,world", [("c1", 50000, 2), ("c2", 300000, 2), ("c3", 200000, 2),
                                               ("c3", 100000, 3)])
def test_gloo_sharded_compose(name, length, world):
    B = 4096
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, length, B, q)) for r in range(world)]
    for p in procs:
        p.start()
    outs = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    w = gen.workload(name, length=length)
    data = w.host()
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    for rank, fin, count, srank, lo in outs:
        assert fin == ref["final"] and count == ref["count"]
        expect_start = w.start if lo == 0 else int(ref["chunk_end"][lo // B - 1])
        assert srank == expect_start


def test_shard_bounds_and_wire_format():
    from paper_conf_ipps_wangwqw22_b200.dist import map_layout, pack_map, shard_bounds, unpack_map

    for total in (0, 1, 4096, 10**6 + 3):
        for world in (1, 2, 3, 8):
            bs = [shard_bounds(total, world, r) for r in range(world)]
            assert bs[0][0] == 0 and bs[-1][1] == total
            for (a, b), (c, d) in zip(bs, bs[1:]):
                assert b == c and a % 4096 == 0
    end = np.array([3, 0xFFFFFFFF, 1], np.uint32)
    cnt = np.array([5, 0, 2**40], np.uint64)
    buf = pack_map(end, cnt)
    assert len(buf) == map_layout(3)[1]
    e, c = unpack_map(buf, 3)
    assert (e == end).all() and (c == cnt).all()


def _lb_worker(rank, world, port, data, bounds, L, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_wangwqw22_b200.dist import exchange_lookback

    lo, hi = bounds[rank]
    lb = exchange_lookback(torch.from_numpy(data[lo:hi].copy()), L=L)
    q.put((rank, lb.numpy().tobytes()))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("L", [2, 5])
@pytest.mark.parametrize("layout", ["bounds", "ragged"])
def test_exchange_lookback_empty_shards(L, layout):
    """Fewer chunks than ranks: some shards are empty (and some shorter than L); every
    rank still receives the L bytes just before its shard."""
    from paper_conf_ipps_wangwqw22_b200.dist import shard_bounds

    world, B = 8, 16
    data = np.arange(5 * B - 3, dtype=np.uint8)  # 5 chunks over 8 ranks
    if layout == "bounds":
        bounds = [shard_bounds(len(data), world, r, B) for r in range(world)]
    else:  # contiguous, with empty and 1-byte shards
        cuts = [0, 0, 3, 3, 4, 20, 20, 21, len(data)]
        bounds = list(zip(cuts[:-1], cuts[1:]))
    assert any(lo == hi and lo > 0 for lo, hi in bounds)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_lb_worker, args=(r, world, port, data, bounds, L, q)) for r in range(world)]
    for p in procs:
        p.start()
    outs = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for r, (lo, hi) in enumerate(bounds):
        assert outs[r] == data[max(0, lo - L):lo].tobytes(), (r, lo)
