"""The peer-memory state-map exchange (fsm_p2p_*): ranks map each other's
mailboxes through CUDA IPC, publish their shard maps with remote stores + flags and wait
for the peers' flags in a kernel — no collective library.  Here 2 and 3 processes share
cuda:0 (IPC between processes on one device); between GPUs the same code stores over
NVLink peer memory."""
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


def _worker(rank, world, port, name, length, steps, q):
    import torch.distributed as dist

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_ipps_wangwqw22_b200 as gs
    from paper_conf_ipps_wangwqw22_b200.dist import exchange_lookback, p2p_setup, shard_bounds

    torch.cuda.set_device(0)
    w = gen.workload(name, length=length)
    lo, hi = shard_bounds(length, world, rank)
    x = torch.empty(hi - lo, dtype=torch.uint8, device="cuda")
    w.device(x, offset=lo)
    lb = exchange_lookback(x)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    p = p2p_setup(fsm)
    outs = []
    for _ in range(steps):
        r = p.run_sharded(fsm, x, lb)
        outs.append((r.final_state, r.accept_count))
    q.put((rank, outs, lo, r.chunk_ends.cpu().numpy().view(np.uint32).copy()))
    dist.barrier()
    p.close()
    dist.destroy_process_group()


@pytest.mark.parametrize("name,length,world", [("c2", 6 << 20, 2), ("c3", 3 << 20, 3), ("c1", 1 << 20, 2),
                                               ("c4", 4 << 20, 3)])
def test_p2p_exchange(name, length, world):
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    steps = 3  # both mailbox sets, reused
    ps = [ctx.Process(target=_worker, args=(r, world, port, name, length, steps, q)) for r in range(world)]
    for p in ps:
        p.start()
    outs = sorted([q.get(timeout=600) for _ in range(world)], key=lambda t: t[0])
    for p in ps:
        p.join(timeout=120)
        assert p.exitcode == 0
    w = gen.workload(name, length=length)
    ref = oracle.run(w.table, w.start, w.accept, w.host(), 4096)
    for rank, res, lo, ce in outs:
        assert res == [(ref["final"], ref["count"])] * steps, rank
    assert (np.concatenate([o[3] for o in outs]) == ref["chunk_end"]).all()
