"""GPU parity of stream-level batching (fsm_run_batch): every stream's
final state, accept count and chunk ends equal the oracle's sequential run of that
stream alone (Alg. 1 L2-3), and the number of re-executed chunks equals the number
of chunks whose lookback-2 prediction (oracle.lookback) differs from the
true start state."""
import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def gs():
    import paper_conf_ipps_wangwqw22_b200 as m

    return m


def make_streams(data, ns, rng, B, maxlen):
    """ns streams carved from data with random gaps (unaligned offsets) and lengths that
    include the edge cases 0, 1, B-1, B, B+1."""
    special = [0, 1, 15, 16, 17, B - 1, B, B + 1, 2 * B + 3]
    lens = [special[i] if i < len(special) else int(rng.integers(0, maxlen)) for i in range(ns)]
    rng.shuffle(lens)
    off = [0]
    pos = 0
    starts = []
    for L in lens:
        pos += int(rng.integers(0, 37))  # gap: streams need not be adjacent or aligned
        starts.append(pos)
        pos += L
    assert pos <= data.size
    return starts, lens


def expected_recoveries(w, tt, perm, seg, ref, B):
    n = 0
    for k in range(1, len(ref["chunk_end"])):
        lo = k * B
        true_start = perm[ref["chunk_end"][k - 1]]
        qs, _ = oracle.lookback(tt, w.nstates, seg[lo - 2:lo], K=16)
        n += int(qs[0] != true_start)
    return n


@pytest.mark.parametrize("name,B", [("c2", 4096), ("c2", 48), ("c3", 4096), ("c4", 4096), ("c1", 16),
                                    ("rand:60:5:11", 64), ("rand:200:256:12", 4096)])
def test_batch_matches_oracle_per_stream(gs, name, B):
    rng = np.random.default_rng(hash(name) % 1000 + B)
    w = gen.workload(name, length=16 << 20)
    data = w.host()
    ns = 300
    starts, lens = make_streams(data, ns, rng, B, min(6 * B, 40000) if B < 4096 else 40000)
    # fsm_run_batch takes contiguous [off[s], off[s+1]) ranges: lay the streams out in order
    # behind a random (unaligned) lead-in of valid symbols
    buf = np.concatenate([data[s:s + L] for s, L in zip(starts, lens)])
    pad = int(rng.integers(0, 16))
    buf = np.concatenate([np.zeros(pad, np.uint8), buf])
    offs = np.cumsum([pad] + lens).astype(np.uint64)
    x = torch.from_numpy(buf).cuda()
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    fin, cnt, ce, st = fsm.run_batch(x, offs, chunk_bytes=B, chunk_ends=True)
    fin, cnt, ce = fin.cpu().numpy().view(np.uint32), cnt.cpu().numpy(), ce.cpu().numpy().view(np.uint32)
    perm, inv, _, tt, acc = oracle.transform(w.table, w.accept)
    c = 0
    rec = 0
    for s in range(ns):
        seg = buf[int(offs[s]):int(offs[s + 1])]
        ref = oracle.run(w.table, w.start, w.accept, seg, B)
        assert fin[s] == ref["final"], s
        assert cnt[s] == ref["count"], s
        k = len(ref["chunk_end"]) if len(seg) else 0
        assert (ce[c:c + k] == ref["chunk_end"][:k]).all(), s
        c += k
        if len(seg):
            rec += expected_recoveries(w, tt, perm, seg, ref, B)
    assert c == st["nchunks"]
    assert st["recoveries"] == rec
    assert st["invalid_streams"] == 0


def test_batch_invalid_symbol_is_loud(gs):
    w = gen.workload("c1", length=1 << 16)
    data = w.host().copy()
    offs = np.array([0, 1000, 5000, 9000], np.uint64)
    data[6000] = 7  # div7 has nsyms = 2: stream 2 is invalid
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    x = torch.from_numpy(data[:9000].copy()).cuda()
    with pytest.raises(gs.GSpecError):
        fsm.run_batch(x, offs, chunk_bytes=64)
    fin = torch.empty(3, dtype=torch.int32, device="cuda")
    # outputs are still written: stream 2 reports nstates, the others their true final state
    import ctypes

    cnt = torch.empty(3, dtype=torch.int64, device="cuda")
    r = gs.fsm_batch_result()
    o = gs._run_opts("sre", 64)
    rc = gs._lib.fsm_run_batch(fsm.handle, x.data_ptr(), offs.ctypes.data, 3, ctypes.byref(o), fin.data_ptr(),
                               cnt.data_ptr(), None, ctypes.byref(r))
    assert rc == -4 and r.invalid_streams == 1
    f = fin.cpu().numpy()
    assert f[2] == 7
    for s in (0, 1):
        ref = oracle.run(w.table, w.start, w.accept, data[int(offs[s]):int(offs[s + 1])], 64)
        assert f[s] == ref["final"]


def test_batch_empty_and_single(gs):
    w = gen.workload("c2", length=1 << 16)
    data = w.host()
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    x = torch.from_numpy(data).cuda()
    fin, cnt, ce, st = fsm.run_batch(x, np.array([0], np.uint64))
    assert st["nstreams"] == 0 and fin.numel() == 0
    fin, cnt, ce, st = fsm.run_batch(x, np.array([0, data.size], np.uint64), chunk_ends=True)
    r = fsm.run(x, scheme="sre")
    assert int(fin[0]) == r.final_state and int(cnt[0]) == r.accept_count
    assert (ce.cpu() == r.chunk_ends.cpu()).all()


def test_fsm_level_batching(gs):
    """FSM-level batching (Alg. 1 L2-3): many (DFA, stream) pairs of mixed
    table formats (u8, u16, u16 delta rows) in one call; every pair's final state and
    accept count equal the oracle's sequential run."""
    rng = np.random.default_rng(7)
    specs = [("c1", 0), ("c2", 0), ("c3", 0), ("c4", 0)] + [(f"rand:{int(rng.integers(1, 300))}:"
                                                             f"{int(rng.integers(1, 257))}:{s}", s) for s in range(10)]
    fsms, xs, refs = [], [], []
    for k, (name, seed) in enumerate(specs * 3):
        length = int(rng.integers(0, 300000))
        w = gen.workload(name, length=length, seed=seed + k)
        h = w.host()
        fsms.append(gs.FSM.load(w.table, w.start, w.accept))
        xs.append(torch.from_numpy(h).cuda() if length else torch.empty(0, dtype=torch.uint8, device="cuda"))
        refs.append(oracle.run(w.table, w.start, w.accept, h, 4096))
    fin, cnt, st = gs.run_multi(fsms, xs, chunk_bytes=4096)
    for i, ref in enumerate(refs):
        assert fin[i] == ref["final"] and cnt[i] == ref["count"], (i, specs[i % len(specs)])
    modes = {f.transform()["mode"] for f in fsms}
    assert len(modes) >= 2, modes  # several table formats in one call
    for f in fsms:
        f.close()


def test_fsm_level_batching_invalid_symbol(gs):
    """A stream with a symbol >= nsyms: its final is 0xFFFFFFFF (R4) and the call raises
    FSM_ESYMBOL after filling every output; the other pairs are still exact."""
    t, s_, a = gen.dfa_div7()
    good = np.array([1, 0, 1, 1] * 5000, np.uint8)
    bad = good.copy()
    bad[777] = 5
    fsm = gs.FSM.load(t, s_, a)
    xs = [torch.from_numpy(good).cuda(), torch.from_numpy(bad).cuda()]
    with pytest.raises(gs.GSpecError):
        gs.run_multi([fsm, fsm], xs)
    ref = oracle.run(t, s_, a, good, 4096)
    fin, cnt, _ = gs.run_multi([fsm], xs[:1])
    assert fin[0] == ref["final"] and cnt[0] == ref["count"]
    fsm.close()
