"""dist.run_sharded end to end with real torch.distributed ranks (GPU).

Two/three ranks share cuda:0 (this pool has one GPU per box) over the gloo
backend; the NCCL path differs only in the allgather call."""
import os
import socket

import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, name, length, q):
    import torch.distributed as dist

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_ipps_wangwqw22_b200 as gs
    from paper_conf_ipps_wangwqw22_b200.dist import exchange_lookback, run_sharded, shard_bounds

    torch.cuda.set_device(0)
    w = gen.workload(name, length=length)
    lo, hi = shard_bounds(length, world, rank)
    x = torch.empty(hi - lo, dtype=torch.uint8, device="cuda")
    w.device(x, offset=lo)
    lb = exchange_lookback(x)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    r = run_sharded(fsm, x, lb)
    q.put((rank, r.final_state, r.accept_count, lo, r.chunk_ends.cpu().numpy().view(np.uint32).copy()))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("name,length,world", [("c2", 6 << 20, 2), ("c3", 3 << 20, 3), ("c1", 1 << 20, 2)])
def test_run_sharded_multi_rank(name, length, world):
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, name, length, q)) for r in range(world)]
    for p in ps:
        p.start()
    outs = sorted([q.get(timeout=600) for _ in range(world)], key=lambda t: t[0])
    for p in ps:
        p.join(timeout=120)
        assert p.exitcode == 0
    w = gen.workload(name, length=length)
    ref = oracle.run(w.table, w.start, w.accept, w.host(), 4096)
    for rank, fin, cnt, lo, ce in outs:
        assert fin == ref["final"] and cnt == ref["count"]
    ce_all = np.concatenate([o[4] for o in outs])
    assert (ce_all == ref["chunk_end"]).all()


def _fail_worker(rank, world, port, q):
    import torch.distributed as dist

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_ipps_wangwqw22_b200 as gs
    from paper_conf_ipps_wangwqw22_b200.dist import run_sharded, shard_bounds

    torch.cuda.set_device(0)
    w = gen.workload("c2", length=3 << 20)
    lo, hi = shard_bounds(w.length, world, rank)
    x = torch.empty(hi - lo, dtype=torch.uint8, device="cuda")
    w.device(x, offset=lo)
    lb = torch.zeros(17 if rank == 1 else (2 if rank else 0), dtype=torch.uint8, device="cuda")  # rank 1: bad
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    try:
        run_sharded(fsm, x, lb)
        q.put((rank, 0))
    except gs.GSpecError as e:
        q.put((rank, e.status))
    dist.barrier()
    dist.destroy_process_group()


def test_run_sharded_failed_rank_is_collective():
    """One rank's fsm_shard_map fails: it publishes an error map and still joins the
    allgather, so every rank raises the same status instead of hanging."""
    import paper_conf_ipps_wangwqw22_b200 as gs
    import torch.multiprocessing as mp

    world = 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_fail_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    outs = dict(q.get(timeout=600) for _ in range(world))
    for p in ps:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert outs == {r: gs.FSM_EINVAL for r in range(world)}
