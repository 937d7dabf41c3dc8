"""Sharded runs on one GPU with a fake collective:
G shard computations run one after another on cuda:0 and the allgather is a
device copy into the gathered buffer; compose + fix-up are the real code."""
import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def sharded_fake(gs, w, data, G, B=4096, scheme="auto"):
    from paper_conf_ipps_wangwqw22_b200 import _check, _lib, _run_opts, fsm_result
    from paper_conf_ipps_wangwqw22_b200.dist import shard_bounds
    import ctypes

    x = torch.from_numpy(data).cuda()
    fsms = [gs.FSM.load(w.table, w.start, w.accept) for _ in range(G)]
    mb = fsms[0].map_bytes()
    maps = torch.zeros(G * mb, dtype=torch.uint8, device="cuda")
    o = _run_opts(scheme, B)
    bounds = [shard_bounds(len(data), G, g, B) for g in range(G)]
    for exact in (False, True):  # the speculative maps first; FSM_EAGAIN on every rank -> exact maps
        ces = []
        for g, (lo, hi) in enumerate(bounds):
            n = gs.fsm_num_chunks(hi - lo, B)
            ce = torch.full((max(n, 1),), -1, dtype=torch.int32, device="cuda")
            lb = x[max(0, lo - 2):lo] if g else None
            fn = _lib.fsm_shard_map_exact if exact else _lib.fsm_shard_map
            _check(fn(fsms[g].handle, x[lo:].data_ptr() if hi > lo else None, hi - lo,
                      lb.data_ptr() if lb is not None else None, 0 if lb is None else lb.numel(),
                      ctypes.byref(o), maps[g * mb:].data_ptr(), ce.data_ptr()), "shard_map")
            ces.append((ce, n))
        outs, rcs = [], []
        for g in range(G):
            r = fsm_result()
            rcs.append(_lib.fsm_shard_finish(fsms[g].handle, maps.data_ptr(), G, g, ctypes.byref(o),
                                             ces[g][0].data_ptr(), ctypes.byref(r)))
            outs.append(r)
        assert len(set(rcs)) == 1, rcs  # every rank sees the same maps
        if rcs[0] != -7:
            _check(rcs[0], "shard_finish")
            break
    chunk_ends = np.concatenate([ce[:n].cpu().numpy().view(np.uint32) for ce, n in ces])
    return outs, chunk_ends


@pytest.fixture(scope="module")
def gs():
    import paper_conf_ipps_wangwqw22_b200 as m

    return m


@pytest.mark.parametrize("name,length", [("c1", 1 << 20), ("c2", 8 << 20), ("c3", 4 << 20), ("c3s", 2 << 20),
                                         ("c4", 4 << 20), ("rand:40:3:5", 300000), ("rand:300:7:2", 200000)])
@pytest.mark.parametrize("G", [1, 2, 3, 8])
def test_fake_collective(gs, name, length, G):
    w = gen.workload(name, length=length)
    data = w.host()
    ref = oracle.run(w.table, w.start, w.accept, data, 4096)
    outs, ce = sharded_fake(gs, w, data, G)
    for r in outs:
        assert r.final_state == ref["final"] and r.accept_count == ref["count"]
        assert bool(r.accept) == bool(ref["accept"])
    assert (ce == ref["chunk_end"]).all()


def test_single_rank_nccl_group(gs):
    import os
    import torch.distributed as dist
    from paper_conf_ipps_wangwqw22_b200.dist import run_sharded

    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ.setdefault("MASTER_PORT", "29533")
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        w = gen.workload("c2", length=4 << 20)
        data = w.host()
        ref = oracle.run(w.table, w.start, w.accept, data, 4096)
        fsm = gs.FSM.load(w.table, w.start, w.accept)
        r = run_sharded(fsm, torch.from_numpy(data).cuda(), None)
        assert r.final_state == ref["final"] and r.accept_count == ref["count"]
        assert (r.chunk_ends.cpu().numpy().view(np.uint32) == ref["chunk_end"]).all()
    finally:
        dist.destroy_process_group()


def test_library_nccl_single_rank(gs):
    """fsm_comm_init + fsm_run_sharded with a real (1-rank) NCCL communicator."""
    w = gen.workload("c2", length=8 << 20)
    data = w.host()
    ref = oracle.run(w.table, w.start, w.accept, data, 4096)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    comm = gs.Comm(1, 0, gs.Comm.unique_id())
    r = comm.run_sharded(fsm, torch.from_numpy(data).cuda())
    assert r.final_state == ref["final"] and r.accept_count == ref["count"]
    assert (r.chunk_ends.cpu().numpy().view(np.uint32) == ref["chunk_end"]).all()
    comm.close()
