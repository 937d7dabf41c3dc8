"""C5 (BASELINE.json configs[4]): a 16 GiB stream of each of the C1-C4
DFAs, scheme chosen by the selector per DFA, checked bit-exactly against the oracle
at full size — final state, accept flag, u64 accept count and all 4,194,304 chunk
ends — both for one GPU (G = 1) and for the 8-way sharded pipeline (shard maps,
one gathered exchange, compose, fix-up; the allgather replaced by a device copy
because the test box has one GPU).

The oracle walks the same 16 GiB regenerated on the host in 64 MiB blocks
(oracle.run_stream); the four oracle walks start when the module
starts and run in background threads while the GPU works."""
import concurrent.futures
import ctypes

import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

L = 16 << 30
B = 4096
DFAS = ("c1", "c2", "c3", "c4")
_POOL = concurrent.futures.ThreadPoolExecutor(len(DFAS))
_REF = {}


def _oracle_future(name):
    if name not in _REF:
        w = gen.workload(name, length=L)
        _REF[name] = _POOL.submit(oracle.run_stream, w.table, w.start, w.accept, w.host, L, B, 64 << 20, 2)
    return _REF[name]


@pytest.fixture(scope="module", autouse=True)
def _start_oracles():
    for n in DFAS:
        _oracle_future(n)
    yield
    _POOL.shutdown(wait=False, cancel_futures=True)


@pytest.fixture(scope="module")
def gs():
    import paper_conf_ipps_wangwqw22_b200 as m

    return m


def _sharded_fake(gs, w, x, G, scheme):
    from paper_conf_ipps_wangwqw22_b200 import _check, _lib, _run_opts, fsm_result
    from paper_conf_ipps_wangwqw22_b200.dist import shard_bounds

    n_all = x.numel()
    fsms = [gs.FSM.load(w.table, w.start, w.accept) for _ in range(G)]
    mb = fsms[0].map_bytes()
    maps = torch.zeros(G * mb, dtype=torch.uint8, device="cuda")
    o = _run_opts(scheme, B)
    bounds = [shard_bounds(n_all, G, g, B) for g in range(G)]
    ce_all = torch.empty(gs.fsm_num_chunks(n_all, B), dtype=torch.int32, device="cuda")
    for exact in (False, True):
        ces = []
        for g, (lo, hi) in enumerate(bounds):
            ce = ce_all[lo // B:]
            lb = x[lo - 2:lo] if g else None
            fn = _lib.fsm_shard_map_exact if exact else _lib.fsm_shard_map
            _check(fn(fsms[g].handle, x[lo:].data_ptr(), hi - lo, lb.data_ptr() if g else None, 2 if g else 0,
                      ctypes.byref(o), maps[g * mb:].data_ptr(), ce.data_ptr()), "shard_map")
            ces.append(ce)
        outs, rcs = [], []
        for g in range(G):
            r = fsm_result()
            rcs.append(_lib.fsm_shard_finish(fsms[g].handle, maps.data_ptr(), G, g, ctypes.byref(o),
                                             ces[g].data_ptr(), ctypes.byref(r)))
            outs.append(r)
        assert len(set(rcs)) == 1, rcs
        if rcs[0] != -7:
            _check(rcs[0], "shard_finish")
            break
    for f in fsms:
        f.close()
    return outs, ce_all


@pytest.mark.parametrize("name", DFAS)
def test_c5_16gib_every_dfa(gs, name):
    w = gen.workload(name, length=L)
    x = torch.empty(L, dtype=torch.uint8, device="cuda")
    w.device(x)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    scheme, _ = fsm.select_scheme(x[: 1 << 20], chunk_bytes=B)
    assert scheme == {"c1": "enum", "c2": "sre", "c3": "sre", "c4": "sre"}[name]
    single = fsm.run(x, scheme=scheme, chunk_bytes=B)
    ce1 = single.chunk_ends.cpu().numpy().view(np.uint32)
    fsm.close()
    outs, ce8 = _sharded_fake(gs, w, x, 8, scheme)
    ce8 = ce8.cpu().numpy().view(np.uint32)
    del x
    torch.cuda.empty_cache()
    ref = _oracle_future(name).result()
    assert ref["status"] == 0
    assert len(ref["chunk_end"]) == L // B == ce1.size == ce8.size
    for r, ce, tag in [(single, ce1, "G=1")] + [(o, ce8, f"G=8 rank {g}") for g, o in enumerate(outs)]:
        assert r.final_state == ref["final"], tag
        assert bool(r.accept) == bool(ref["accept"]), tag
        assert r.accept_count == ref["count"], tag
    for ce, tag in ((ce1, "G=1"), (ce8, "G=8")):
        bad = np.nonzero(ce != ref["chunk_end"])[0]
        assert bad.size == 0, (tag, bad[:5])
