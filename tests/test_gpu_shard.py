"""Sharded runs on one GPU with a fake collective:
G shard computations run one after another on cuda:0 and the allgather is a
device copy into the gathered buffer; compose + fix-up are the real code."""
import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def sharded_fake(gs, w, data, G, B=4096, scheme="auto", L=2):
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
            lb = x[max(0, lo - L):lo] if g else None
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
@pytest.mark.parametrize("G,L", [(1, 2), (2, 2), (3, 2), (8, 2), (3, 16), (8, 16)])
def test_fake_collective(gs, name, length, G, L):
    """L = bytes before each shard whose lookback image is its candidate start set:
    16 gives the smallest sets (a subset of the 2-byte image)."""
    w = gen.workload(name, length=length)
    data = w.host()
    ref = oracle.run(w.table, w.start, w.accept, data, 4096)
    outs, ce = sharded_fake(gs, w, data, G, L=L)
    for r in outs:
        assert r.final_state == ref["final"] and r.accept_count == ref["count"]
        assert bool(r.accept) == bool(ref["accept"])
    assert (ce == ref["chunk_end"]).all()


@pytest.mark.parametrize("name,length,G,B,scheme", [("c3", (48 << 20) + 8192 * 3, 8, 8192, "sre"),
                                                  ("c3s", 40 << 20, 3, 8192, "nf"), ("c2", 24 << 20, 4, 16384, "sre"),
                                                  ("c1", (6 << 20) + 100, 3, 8192, "enum")])
def test_fake_collective_recommended_chunks(gs, name, length, G, B, scheme):
    """The sharded pipeline at the chunk sizes the selector recommends (R29: 8 / 16 KiB), as
    bench.py --config c5 runs it: shard bounds on B, dense SRE / NF rounds inside the shards."""
    w = gen.workload(name, length=length)
    data = w.host()
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    outs, ce = sharded_fake(gs, w, data, G, B=B, scheme=scheme, L=16)
    for r in outs:
        assert r.final_state == ref["final"] and r.accept_count == ref["count"]
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
    """fsm_comm_init + fsm_run_sharded (and the offset form fsm_run_sharded_at) with a real
    (1-rank) NCCL communicator."""
    w = gen.workload("c2", length=8 << 20)
    data = w.host()
    ref = oracle.run(w.table, w.start, w.accept, data, 4096)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    comm = gs.Comm(1, 0, gs.Comm.unique_id(), device=0)
    x = torch.from_numpy(data).cuda()
    for r in (comm.run_sharded(fsm, x), comm.run_sharded_at(fsm, x, 0, x.numel())):
        assert r.final_state == ref["final"] and r.accept_count == ref["count"]
        assert (r.chunk_ends.cpu().numpy().view(np.uint32) == ref["chunk_end"]).all()
    with pytest.raises(gs.GSpecError):
        comm.run_sharded_at(fsm, x[4096:], 100, x.numel())  # not chunk-aligned
    comm.close()


def _maps_and_finish(gs, w, x, G, scheme="auto", B=4096, bad_rank=None, exact=False):
    """Fake-collective round returning the raw status codes: (map rcs, finish rcs, results,
    chunk ends).  bad_rank passes an over-long lookback (17 bytes -> FSM_EINVAL)."""
    import ctypes

    from paper_conf_ipps_wangwqw22_b200 import _lib, _run_opts, fsm_result
    from paper_conf_ipps_wangwqw22_b200.dist import shard_bounds

    L = x.numel()
    fsms = [gs.FSM.load(w.table, w.start, w.accept) for _ in range(G)]
    mb = fsms[0].map_bytes()
    maps = torch.zeros(G * mb, dtype=torch.uint8, device="cuda")
    o = _run_opts(scheme, B)
    ce_all = torch.full((max(1, gs.fsm_num_chunks(L, B)),), -1, dtype=torch.int32, device="cuda")
    map_rc, fin_rc, outs = [], [], []
    for attempt in range(2):
        map_rc = []
        for g in range(G):
            lo, hi = shard_bounds(L, G, g, B)
            lbn = 17 if g == bad_rank else (2 if g else 0)
            lb = x[max(0, lo - lbn):lo] if g else None
            fn = _lib.fsm_shard_map_exact if (exact or attempt) else _lib.fsm_shard_map
            map_rc.append(fn(fsms[g].handle, x[lo:].data_ptr() if hi > lo else None, hi - lo,
                             lb.data_ptr() if lb is not None else None, lbn, ctypes.byref(o),
                             maps[g * mb:].data_ptr(), ce_all[lo // B:].data_ptr()))
        fin_rc, outs = [], []
        for g in range(G):
            r = fsm_result()
            fin_rc.append(_lib.fsm_shard_finish(fsms[g].handle, maps.data_ptr(), G, g, ctypes.byref(o),
                                                ce_all[shard_bounds(L, G, g, B)[0] // B:].data_ptr(), ctypes.byref(r)))
            outs.append(r)
        if fin_rc[0] != -7:
            break
    return map_rc, fin_rc, outs, ce_all


def test_invalid_symbol_in_earlier_shard(gs):
    """An invalid byte (>= nsyms, R4) inside shard 0 of 3: the poison state is a fixed
    entry of every map, so every rank's composition reaches it and reports FSM_ESYMBOL,
    as fsm_run does on one GPU."""
    w = gen.workload("rand:50:7:3", length=3 * 64 * 4096)
    data = w.host()
    data[1000] = 9  # nsyms = 7
    x = torch.from_numpy(data).cuda()
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    with pytest.raises(gs.GSpecError) as e:
        fsm.run(x, scheme="sre")
    assert e.value.status == gs.FSM_ESYMBOL
    for exact in (False, True):
        map_rc, fin_rc, _, _ = _maps_and_finish(gs, w, x, 3, scheme="sre", exact=exact)
        assert map_rc == [0, 0, 0]
        assert fin_rc == [gs.FSM_ESYMBOL] * 3, fin_rc


def test_failed_map_is_collective(gs):
    """A rank whose fsm_shard_map fails publishes an error map; every rank's finish
    returns that rank's status (nobody is left waiting in the exchange)."""
    w = gen.workload("c2", length=6 << 20)
    x = torch.from_numpy(w.host()).cuda()
    map_rc, fin_rc, _, _ = _maps_and_finish(gs, w, x, 3, scheme="sre", bad_rank=1)
    assert map_rc[1] == gs.FSM_EINVAL and map_rc[0] == 0 and map_rc[2] == 0
    assert fin_rc == [gs.FSM_EINVAL] * 3, fin_rc


@pytest.mark.parametrize("n,G", [(100, 3), (40, 2)])
def test_many_nonmerging_paths(gs, n, G):
    """A non-convergent DFA above the ENUM limit (permutation columns, n = 100: 100
    candidate paths that never merge) shards exactly (one pipeline per surviving path)."""
    rng = np.random.default_rng(n)
    t = np.stack([rng.permutation(n) for _ in range(3)], axis=1).astype(np.uint32)
    a = (rng.random(n) < 0.5).astype(np.uint8)
    data = rng.integers(0, 3, 24 * 4096 + 77).astype(np.uint8)
    ref = oracle.run(t, 0, a, data, 4096)

    class W:
        table, start, accept = t, 0, a

    map_rc, fin_rc, outs, ce = _maps_and_finish(gs, W, torch.from_numpy(data).cuda(), G, scheme="sre")
    assert map_rc == [0] * G and fin_rc == [0] * G, (map_rc, fin_rc)
    for r in outs:
        assert r.final_state == ref["final"] and r.accept_count == ref["count"]
    assert (ce[:len(ref["chunk_end"])].cpu().numpy().view(np.uint32) == ref["chunk_end"]).all()


def test_library_nccl_async_steps(gs):
    """fsm_run_sharded_async: several steps queued back to back on one 1-rank NCCL
    communicator, each collected by fsm_shard_wait, every one exact (C2: fused mode; div7:
    the host fix-up ENUM mode, finished inside the async call)."""
    for name, length in (("c2", 8 << 20), ("c1", 1 << 20), ("c3", 4 << 20)):
        w = gen.workload(name, length=length)
        data = w.host()
        ref = oracle.run(w.table, w.start, w.accept, data, 4096)
        fsm = gs.FSM.load(w.table, w.start, w.accept)
        comm = gs.Comm(1, 0, gs.Comm.unique_id())
        x = torch.from_numpy(data).cuda()
        comm.run_sharded(fsm, x)  # warm (selector, speculative-map check)
        ce = torch.empty(gs.fsm_num_chunks(length), dtype=torch.int32, device="cuda")
        tickets = [comm.run_sharded_async(fsm, x, chunk_ends=ce) for _ in range(5)]
        for t in tickets:
            r = gs.Comm.wait(fsm, t)
            assert r.final_state == ref["final"] and r.accept_count == ref["count"], name
        assert (ce.cpu().numpy().view(np.uint32) == ref["chunk_end"]).all()
        with pytest.raises(gs.GSpecError):
            gs.Comm.wait(fsm, tickets[0])  # already collected
        comm.close()
        fsm.close()
