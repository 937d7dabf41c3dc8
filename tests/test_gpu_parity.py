"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, bit-exact.

Every output of every scheme must equal the sequential result:
final state, accept flag, accept count and every chunk end.  Round
diagnostics must equal the oracle's deterministic round simulator
 exactly.
"""
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


_CACHE = {}


def _wl(name, length, seed=None):
    key = (name, length, seed)
    if key not in _CACHE:
        w = gen.workload(name, length=length, seed=seed)
        _CACHE[key] = (w, w.host())
    return _CACHE[key]


def _fsm(gs, w, **kw):
    key = ("fsm", w.name, tuple(sorted(kw.items())))
    if key not in _CACHE:
        _CACHE[key] = gs.FSM.load(w.table, w.start, w.accept, **kw)
    return _CACHE[key]


def check_equal(res, ref, B, n):
    assert res.final_state == ref["final"]
    assert res.accept == bool(ref["accept"])
    assert res.accept_count == ref["count"]
    ce = res.chunk_ends.cpu().numpy().view(np.uint32)
    assert ce.shape == ref["chunk_end"].shape
    bad = np.nonzero(ce != ref["chunk_end"])[0]
    assert bad.size == 0, f"first mismatching chunk {bad[:5]} of {len(ce)}"


SCHEMES = ["seq", "pm", "sre", "rr", "nf", "cse"]


@pytest.mark.parametrize("scheme", SCHEMES + ["enum", "auto"])
def test_div7_c1(gs, scheme):
    w, data = _wl("c1", 1 << 20)
    ref = oracle.run(w.table, w.start, w.accept, data, 4096)
    fsm = _fsm(gs, w)
    x = torch.from_numpy(data).cuda()
    res = fsm.run(x, scheme=scheme)
    check_equal(res, ref, 4096, w.nstates)
    if scheme == "cse":  # every lookback image is all 7 states (<= 8): exact coverage, no recovery
        assert res.stats["rounds"] == 0 and res.stats["verify_matches"] == res.stats["verify_checks"] == 256
    big_mod = ref["final"]  # pinned separately against int(bits,2) % 7 in the oracle tests
    assert res.accept == (big_mod == 0)


@pytest.mark.parametrize("name,length", [("c2", 4 << 20), ("c3", 4 << 20), ("c3s", 2 << 20), ("c4", 4 << 20)])
@pytest.mark.parametrize("scheme", SCHEMES)
def test_configs_small_with_diagnostics(gs, name, length, scheme):
    w, data = _wl(name, length)
    B = 4096
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    fsm = _fsm(gs, w)
    x = torch.from_numpy(data).cuda()
    res = fsm.run(x, scheme=scheme, chunk_bytes=B)
    check_equal(res, ref, B, w.nstates)
    sim = oracle.simulate(w.table, w.start, w.accept, data, B, scheme=scheme)
    st = res.stats
    for k in ("rounds", "tasks_mustdo", "tasks_sre", "tasks_helper", "reread_bytes", "verify_checks",
              "verify_matches"):
        assert st[k] == sim[k], (k, st[k], sim[k])


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("scheme", SCHEMES + ["enum"])
def test_random_dfas(gs, seed, scheme):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 64 if scheme == "enum" else 300))
    ns = int(rng.integers(1, 257))
    name = f"rand:{n}:{ns}:{seed}"
    length = int(rng.integers(0, 200000))
    w, data = _wl(name, length, seed)
    for B in (16, 48, 4096):
        ref = oracle.run(w.table, w.start, w.accept, data, B)
        fsm = _fsm(gs, w)
        res = fsm.run(torch.from_numpy(data).cuda(), scheme=scheme, chunk_bytes=B)
        check_equal(res, ref, B, n)
        if scheme != "enum":
            sim = oracle.simulate(w.table, w.start, w.accept, data, B, scheme=scheme)
            for k in ("rounds", "tasks_mustdo", "tasks_sre", "tasks_helper", "verify_checks", "verify_matches"):
                assert res.stats[k] == sim[k], (k, B)


@pytest.mark.parametrize("mode", [2, 3])
@pytest.mark.parametrize("budget", [0, 1024])
def test_classed_modes_and_cold_rows(gs, mode, budget):
    """u16/u32 classed tables; a 1 KiB smem budget forces most rows cold (L2)."""
    for name in ("c2", "c3"):
        w, data = _wl(name, 2 << 20)
        ref = oracle.run(w.table, w.start, w.accept, data, 4096)
        fsm = gs.FSM.load(w.table, w.start, w.accept, force_mode=mode, smem_budget=budget)
        tr = fsm.transform()
        assert tr["mode"] == {2: "u16", 3: "u32"}[mode]
        if budget:
            assert tr["hot_rows"] < w.nstates
        for scheme in ("sre", "nf"):
            res = fsm.run(torch.from_numpy(data).cuda(), scheme=scheme)
            check_equal(res, ref, 4096, w.nstates)


@pytest.mark.parametrize("length", [0, 1, 15, 16, 17, 4095, 4096, 4097, 3 * 4096 + 5])
def test_edge_lengths(gs, length):
    for name in ("c1", "c2"):
        w, data = _wl(name, length)
        ref = oracle.run(w.table, w.start, w.accept, data, 4096)
        fsm = _fsm(gs, w)
        for scheme in ("sre", "rr", "pm"):
            x = torch.from_numpy(data).cuda() if length else torch.empty(0, dtype=torch.uint8, device="cuda")
            res = fsm.run(x, scheme=scheme)
            assert res.final_state == ref["final"] and res.accept_count == ref["count"]
            assert res.nchunks == len(ref["chunk_end"])
            if length:
                assert (res.chunk_ends.cpu().numpy().view(np.uint32) == ref["chunk_end"]).all()


def test_unaligned_input(gs):
    w, data = _wl("c2", 1 << 20)
    big = torch.zeros(len(data) + 64, dtype=torch.uint8, device="cuda")
    for off in (1, 3, 8):
        x = big[off:off + len(data)]
        x.copy_(torch.from_numpy(data))
        ref = oracle.run(w.table, w.start, w.accept, data, 4096)
        res = _fsm(gs, w).run(x, scheme="sre")
        check_equal(res, ref, 4096, w.nstates)


def test_invalid_symbol_is_loud(gs):
    t, s, a = gen.dfa_div7()
    fsm = gs.FSM.load(t, s, a)
    data = np.array([1, 0, 1] * 5000 + [9] + [1] * 300, np.uint8)
    for scheme in ("sre", "enum", "nf"):
        with pytest.raises(gs.GSpecError) as e:
            fsm.run(torch.from_numpy(data).cuda(), scheme=scheme, chunk_bytes=64)
        assert e.value.status == gs.FSM_ESYMBOL


@pytest.mark.parametrize("name,length,B", [("c1", (16 << 20) + 5, 4096), ("rand:40:3:2", (12 << 20) + 333, 4096),
                                           ("rand:60:4:7", 10 << 20, 2048), ("rand:9:2:4", (6 << 20) + 17, 1024),
                                           ("c1", 3 << 20, 4096), ("rand:12:3:5", (9 << 20) + 64, 4096),
                                           ("rand:14:30:2", (8 << 20) + 1000, 4096), ("rand:5:4:3", 5 << 20, 512),
                                           ("c1", 1 << 20, 4096), ("rand:9:2:4", 300001, 1024),
                                           ("rand:30:3:8", (1 << 20) + 9, 4096)])
def test_enum_four_symbol_table(gs, name, length, B):
    """ENUM on small alphabets walks 16-byte vectors K symbols per lookup (TK: K = 8 for
    nsyms <= 2, 4 for nsyms <= 4); the unaligned tail and vectors holding a
    byte TK does not cover take the one-symbol step — in the multi-launch walk and in the
    single-launch kernel of streams up to 2 MiB.  Bit-exact against the oracle with TK on and
    off (GSPEC_TK=0), for nt from 6 to 61 (rows padded to 257 words, staged in 16-byte pieces)
    and a 30-symbol DFA that has no TK."""
    import os
    w, data = _wl(name, length)
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    x = torch.from_numpy(data).cuda()
    for flag in ("1", "0"):
        os.environ["GSPEC_TK"] = flag
        try:
            res = fsm.run(x, scheme="enum", chunk_bytes=B)
        finally:
            os.environ.pop("GSPEC_TK", None)
        check_equal(res, ref, B, w.nstates)


@pytest.mark.parametrize("name,nsyms,bad", [("c1", 2, 3), ("c1", 2, 9), ("c1", 2, 255), ("rand:20:3:6", 3, 3),
                                            ("rand:20:3:6", 3, 200)])
def test_enum_four_symbol_table_invalid(gs, name, nsyms, bad):
    """An invalid byte (>= nsyms) inside a TK vector: div7 (K = 8, one-bit symbols) sends any
    such byte through the one-symbol fallback; a 3-symbol DFA (K = 4, two-bit symbols) steps
    the value 3 to the poison state through TK itself and larger values through the fallback
    — FSM_ESYMBOL either way, also when the byte sits in the unaligned tail."""
    w, _ = _wl(name, 1 << 16)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    rng = np.random.default_rng(bad)
    for pos in (5 << 20, (8 << 20) - 3):
        data = rng.integers(0, nsyms, 8 << 20).astype(np.uint8)
        data[pos] = bad
        with pytest.raises(gs.GSpecError) as e:
            fsm.run(torch.from_numpy(data).cuda(), scheme="enum", chunk_bytes=4096)
        assert e.value.status == gs.FSM_ESYMBOL


@pytest.mark.parametrize("policy", [0, 1])
def test_policies_and_transform(gs, policy):
    w, data = _wl("c3", 1 << 20)
    fsm = gs.FSM.load(w.table, w.start, w.accept, freq_policy=policy, profile=data[:65536] if policy else None)
    tr = fsm.transform()
    perm, inv, freq, tt, acc = oracle.transform(w.table, w.accept, policy, data[:65536] if policy else None,
                                                w.start)
    assert (tr["perm"] == perm).all() and (tr["inv"] == inv).all() and (tr["freq"] == freq).all()
    ref = oracle.run(w.table, w.start, w.accept, data, 4096)
    res = fsm.run(torch.from_numpy(data).cuda(), scheme="rr")
    check_equal(res, ref, 4096, w.nstates)


@pytest.mark.parametrize("name", ["c1", "c2", "rand:200:256:7", "rand:120:97:8"])
def test_bank_aware_row_placement(gs, name):
    """A profile sample with freq_policy 0 only moves u8 rows (codes); tids and every
    result stay those of the plain load."""
    w, data = _wl(name, 3 << 20, 7 if name.startswith("rand") else None)
    ref = oracle.run(w.table, w.start, w.accept, data, 4096)
    prof = gen.workload(name, length=1 << 20, seed=99).host()  # disjoint "training" trace
    plain = gs.FSM.load(w.table, w.start, w.accept)
    fsm = gs.FSM.load(w.table, w.start, w.accept, profile=prof)
    tp, tr = plain.transform(), fsm.transform()
    assert tr["mode"] == "u8"
    assert (tp["perm"] == tr["perm"]).all() and (tp["inv"] == tr["inv"]).all()
    x = torch.from_numpy(data).cuda()
    for scheme in SCHEMES:
        res = fsm.run(x, scheme=scheme)
        check_equal(res, ref, 4096, w.nstates)
        assert res.stats == plain.run(x, scheme=scheme).stats | {"ms_spec": res.stats["ms_spec"],
                                                               "ms_verify": res.stats["ms_verify"]}


def test_lookback_table_matches_oracle(gs):
    for name in ("c2", "c3", "c1"):
        w, data = _wl(name, 1 << 16)
        fsm = _fsm(gs, w)
        perm, inv, freq, tt, acc = oracle.transform(w.table, w.accept)
        rng = np.random.default_rng(1)
        pairs = [(int(data[i]), int(data[i + 1])) for i in rng.integers(0, len(data) - 1, 64)]
        for a, b in pairs:
            qs, img = fsm.qs(a, b)
            oq, oimg = oracle.lookback(tt, w.nstates, np.array([a, b], np.uint8), K=16)
            assert list(qs) == list(oq) and img == oimg


def test_selector_features_match_oracle(gs):
    for name, expect in (("c1", {"enum"}), ("c2", {"sre"}), ("c3", {"sre"})):  # R19b
        w, data = _wl(name, 1 << 20)
        fsm = gs.FSM.load(w.table, w.start, w.accept)
        pick, ft = fsm.select_scheme(torch.from_numpy(data).cuda())
        of = oracle.features(w.table, w.start, w.accept, data, B=4096)
        assert ft["acc1"] == pytest.approx(of["acc1"]) and ft["acck"] == pytest.approx(of["acck"])
        assert ft["input_sensitivity"] == pytest.approx(of["sens"]) and ft["uniq10"] == pytest.approx(of["uniq10"])
        assert pick in expect
        assert oracle.select(of, w.nstates) == {"enum": 6, "sre": 3, "rr": 4, "nf": 5, "pm": 2}[pick]


def test_run_host_e2e(gs):
    w, data = _wl("c2", 3 << 20)
    ref = oracle.run(w.table, w.start, w.accept, data, 4096)
    res = _fsm(gs, w).run_host(data, scheme="sre")
    assert res.final_state == ref["final"] and res.accept_count == ref["count"]
    assert (res.chunk_ends == ref["chunk_end"]).all()


def test_device_generator_matches_host():
    for name in ("c1", "c2", "c3s", "c4"):
        w = gen.workload(name, length=(1 << 20) + 12345)
        h = w.host()
        d = torch.empty(len(h), dtype=torch.uint8, device="cuda")
        w.device(d)
        assert gen.bytes_hash(d.cpu().numpy()) == gen.bytes_hash(h)
        # offset slices regenerate identically
        d2 = torch.empty(5000, dtype=torch.uint8, device="cuda")
        w.device(d2, offset=777777)
        assert (d2.cpu().numpy() == h[777777:782777]).all()


@pytest.mark.parametrize("name,length", [("c2", 1 << 30)])
def test_full_size_bench_config(gs, name, length):
    """BASELINE config at full size, in the launch configuration bench.py times."""
    w = gen.workload(name, length=length)
    x = torch.empty(length, dtype=torch.uint8, device="cuda")
    w.device(x)
    h = w.host()
    assert gen.bytes_hash(h[:1 << 24]) == gen.bytes_hash(x[:1 << 24].cpu().numpy())
    ref = oracle.run(w.table, w.start, w.accept, h, 4096)
    fsm = _fsm(gs, w)
    res = fsm.run(x, scheme="auto")
    check_equal(res, ref, 4096, w.nstates)


def test_async_queue(gs):
    """fsm_run_async/fsm_wait: runs queued back to back (different inputs and
    schemes on one handle) each return exactly the sequential result."""
    runs = []
    fsm = None
    for seed in range(6):
        w, data = _wl("c2", (1 << 20) + seed * 4111, 100 + seed)
        fsm = fsm or gs.FSM.load(w.table, w.start, w.accept)
        x = torch.from_numpy(data).cuda()
        ce = torch.empty(gs.fsm_num_chunks(len(data)), dtype=torch.int32, device="cuda")
        scheme = ("sre", "pm", "seq", "rr", "nf", "sre")[seed]
        runs.append((fsm.run_async(x, scheme=scheme, chunk_ends=ce), x, ce, data, w))
    for t, x, ce, data, w in reversed(runs):
        r = fsm.wait(t)
        ref = oracle.run(w.table, w.start, w.accept, data, 4096)
        assert r.final_state == ref["final"] and r.accept_count == ref["count"]
        assert (ce.cpu().numpy().view(np.uint32) == ref["chunk_end"]).all()
    with pytest.raises(gs.GSpecError):
        fsm.wait(runs[0][0])  # already collected


@pytest.mark.parametrize("name,length,B,scheme,vr_oth", [
    ("c3", 32 << 20, 4096, "sre", 16), ("c3", (24 << 20) + 1000, 4096, "sre", 16), ("c3s", 160 << 20, 8192, "sre", 16),
    ("c3", 32 << 20, 4096, "cse", 16), ("c3", 32 << 20, 4096, "rr", 16), ("c3", 32 << 20, 4096, "nf", 16),
    ("c3", (24 << 20) + 1000, 4096, "rr", 16), ("c3", (24 << 20) + 1000, 4096, "nf", 2),
    ("c3s", 160 << 20, 8192, "nf", 16), ("c3", 16 << 20, 4096, "nf", 1), ("c3", 48 << 20, 8192, "sre", 16),
    ("c3", 48 << 20, 8192, "rr", 16), ("c3", (40 << 20) + 4100, 8192, "nf", 4)])
def test_dense_recovery_rounds(gs, name, length, B, scheme, vr_oth):
    """SRE / RR / NF (and CSE's SRE rounds) on a low-accuracy DFA: rounds where many
    chunks re-execute go to the TMA-gather task kernel over the round's task list (RR /
    NF: A-tasks to VR^end, helpers to VR^others at their precomputed ring slots); results
    and round diagnostics stay identical to the oracle's, twice in a row (the second run
    queues as many task-kernel slots as the first used)."""
    w, data = _wl(name, length)
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    sim = oracle.simulate(w.table, w.start, w.accept, data, B, scheme=scheme, vr_oth=vr_oth)
    x = torch.from_numpy(data).cuda()
    for _ in range(2):
        res = fsm.run(x, scheme=scheme, chunk_bytes=B, vr_others=vr_oth)
        check_equal(res, ref, B, w.nstates)
        for k in ("rounds", "tasks_mustdo", "tasks_sre", "tasks_helper", "reread_bytes", "verify_checks",
                  "verify_matches"):
            assert res.stats[k] == sim[k], (k, res.stats[k], sim[k])
    assert res.stats["tasks_sre"] > 2048  # the dense path really ran
    if scheme in ("rr", "nf") and B == 4096:
        assert res.stats["tasks_helper"] > 2048


@pytest.mark.parametrize("scheme", ["sre", "rr", "nf"])
def test_dense_slots_follow_previous_run(gs, scheme):
    """Device-driven dense rounds: a run that needed a dense round but had no task-kernel
    slot queued (the selector's 1 MiB profile run used none) runs it in-kernel and makes
    the next run queue one — for RR / NF as for SRE."""
    w, data = _wl("c3", 48 << 20)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    x = torch.from_numpy(data).cuda()
    fsm.select_scheme(x[: 1 << 20])  # a small profile: no dense round there
    r1 = fsm.run(x, scheme=scheme, chunk_bytes=8192)
    r2 = fsm.run(x, scheme=scheme, chunk_bytes=8192)
    assert r1.stats["kernel_launches"] == 2  # spec + verify (the dense round ran in-kernel)
    assert r2.stats["kernel_launches"] >= 5  # + task kernel, finish, verify per queued slot
    for k in ("rounds", "tasks_sre", "tasks_helper", "verify_matches"):
        assert r1.stats[k] == r2.stats[k]
    assert r1.final_state == r2.final_state and r1.accept_count == r2.accept_count


@pytest.mark.parametrize("name,length,B", [("c1", 1 << 20, 4096), ("c2", 4 << 20, 16384), ("c3", 2 << 20, 8192),
                                           ("c4", 2 << 20, 4096), ("c2", (1 << 20) + 77, 2048), ("c1", 100, 16),
                                           ("c2", 0, 4096)])
def test_paper_literal_sre(gs, name, length, B):
    """The paper-literal single-CTA kernel: bit-exact results, and Alg. 3's
    per-iteration accounting equal to the oracle's literal simulation."""
    w, data = _wl(name, length)
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    fsm = _fsm(gs, w)
    x = torch.from_numpy(data).cuda() if length else torch.empty(0, dtype=torch.uint8, device="cuda")
    res = fsm.run_literal(x, chunk_bytes=B)
    assert res.final_state == ref["final"] and res.accept_count == ref["count"]
    if length:
        assert (res.chunk_ends.cpu().numpy().view(np.uint32) == ref["chunk_end"]).all()
        sim = oracle.simulate_literal_sre(w.table, w.start, w.accept, data, B)
        for k in ("rounds", "tasks_mustdo", "tasks_sre", "reread_bytes", "verify_checks", "verify_matches"):
            assert res.stats[k] == sim[k], (k, res.stats[k], sim[k])
    with pytest.raises(gs.GSpecError):
        fsm.run_literal(torch.zeros(1025 * 16, dtype=torch.uint8, device="cuda"), chunk_bytes=16)
    if name == "c1" and length > 1000:  # an invalid symbol ends on the poison state (R4)
        bad = data.copy()
        bad[length // 2] = 9
        with pytest.raises(gs.GSpecError):
            fsm.run_literal(torch.from_numpy(bad).cuda(), chunk_bytes=B)


@pytest.mark.parametrize("name,length,B", [("c1", 1 << 18, 1024), ("c3", 2 << 20, 8192), ("c2", (1 << 20) + 77, 2048),
                                           ("c4", 2 << 20, 4096), ("rand:40:7:3", 60000, 64), ("rand:200:30:5", 30000, 48)])
@pytest.mark.parametrize("scheme", ["rr", "nf"])
def test_paper_literal_rr_nf(gs, name, length, B, scheme):
    """Paper-literal Alg. 4 (RR) / Alg. 5 (NF) single-CTA kernels: bit-exact
    results, and the per-iteration accounting (must-do, rear re-executions, helpers,
    re-read bytes, checks, matches) equal to the oracle's literal simulation."""
    w, data = _wl(name, length)
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    fsm = _fsm(gs, w)
    for vr in (16, 2):
        res = fsm.run_literal(torch.from_numpy(data).cuda(), chunk_bytes=B, scheme=scheme, vr_end=vr)
        assert res.scheme == scheme
        assert res.final_state == ref["final"] and res.accept_count == ref["count"]
        assert (res.chunk_ends.cpu().numpy().view(np.uint32) == ref["chunk_end"]).all()
        sim = oracle.simulate_literal(w.table, w.start, w.accept, data, B, scheme=scheme, vr_cap=vr)
        for k in ("rounds", "tasks_mustdo", "tasks_sre", "tasks_helper", "reread_bytes", "verify_checks",
                  "verify_matches"):
            assert res.stats[k] == sim[k], (k, vr, res.stats[k], sim[k])
    if name.startswith("rand") or name == "c3":
        assert res.stats["tasks_helper"] > 0


@pytest.mark.parametrize("scheme,B", [("cse", 64), ("cse", 16), ("rr", 64), ("nf", 256)])
def test_chained_verification_passes(gs, scheme, B):
    """div7 with several records per chunk: non-convergent chains that a chaotic pass
    advances one chunk at a time; the chained (Gauss-Seidel) passes cross whole CTA
    ranges (16 K-64 K chunks over many CTAs).  Results and round diagnostics stay exact."""
    w, data = _wl("c1", 1 << 20)
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    fsm = _fsm(gs, w)
    res = fsm.run(torch.from_numpy(data).cuda(), scheme=scheme, chunk_bytes=B)
    check_equal(res, ref, B, w.nstates)
    sim = oracle.simulate(w.table, w.start, w.accept, data, B, scheme=scheme)
    for k in ("rounds", "tasks_mustdo", "tasks_sre", "tasks_helper", "verify_checks", "verify_matches"):
        assert res.stats[k] == sim[k], (k, res.stats[k], sim[k])


@pytest.mark.parametrize("name,length,scheme", [("c3", 1 << 30, "auto"), ("c3", 1 << 30, "sre"), ("c4", 4 << 30, "auto")])
def test_full_size_other_configs(gs, name, length, scheme):
    """BASELINE configs C3 (1 GB) and C4 (4 GB) at full size vs the oracle."""
    w = gen.workload(name, length=length)
    x = torch.empty(length, dtype=torch.uint8, device="cuda")
    w.device(x)
    h = w.host()
    ref = oracle.run(w.table, w.start, w.accept, h, 4096)
    del h
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    res = fsm.run(x, scheme=scheme)
    check_equal(res, ref, 4096, w.nstates)


@pytest.mark.parametrize("name,length,vr_end", [("c2", 16 << 20, 16), ("c4", 16 << 20, 16), ("c4", 8 << 20, 1),
                                                ("rand:40:7:3", 4 << 20, 16)])
def test_inline_round0_recovery(gs, name, length, vr_end):
    """SRE with a high-accuracy profile hint: round 0's verification runs the SRE tasks
    inline (verify_recover.cu, round 0 of SRE); results and round diagnostics must
    equal the listed-task semantics of the oracle's simulator exactly."""
    w, data = _wl(name, length)
    ref = oracle.run(w.table, w.start, w.accept, data, 4096)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    x = torch.from_numpy(data).cuda()
    fsm.select_scheme(x[: 1 << 20])  # sets the accuracy hint: no dense rounds
    res = fsm.run(x, scheme="sre", vr_end=vr_end)
    check_equal(res, ref, 4096, w.nstates)
    sim = oracle.simulate(w.table, w.start, w.accept, data, 4096, scheme="sre", vr_end=vr_end)
    for k in ("rounds", "tasks_mustdo", "tasks_sre", "tasks_helper", "reread_bytes", "verify_checks",
              "verify_matches"):
        assert res.stats[k] == sim[k], (k, res.stats[k], sim[k])
    if name != "c2":
        assert res.stats["tasks_sre"] > 0  # mispredictions really happened


@pytest.mark.parametrize("name,length,budget", [("c4", 4 << 20, 0), ("c4", 2 << 20, 48 * 1024), ("c3", 2 << 20, 0),
                                                ("c2", 2 << 20, 0), ("c2", 1 << 20, 2048),
                                                ("rand:300:60:7", 1 << 20, 8192)])
def test_delta_rows(gs, name, length, budget):
    """u16 table whose cold rows are delta rows in smem (hot base row + <= 2 exceptions,
    the poison row as an extra hot row); when some row does not compress within the
    budget the plain hot/cold split is used — every scheme stays bit-exact."""
    w, data = _wl(name, length)
    ref = oracle.run(w.table, w.start, w.accept, data, 4096)
    fsm = gs.FSM.load(w.table, w.start, w.accept, force_mode=4, smem_budget=budget)
    tr = fsm.transform()
    if tr["mode"] == "u16d":
        assert tr["hot_rows"] < w.nstates + 1
    x = torch.from_numpy(data).cuda()
    for scheme in ("sre", "nf", "pm"):
        res = fsm.run(x, scheme=scheme)
        check_equal(res, ref, 4096, w.nstates)
    res = fsm.run(x[5:], scheme="sre", chunk_bytes=48)  # generic (unaligned) kernel, many tasks
    ref2 = oracle.run(w.table, w.start, w.accept, data[5:], 48)
    check_equal(res, ref2, 48, w.nstates)


def test_c4_auto_picks_delta_rows(gs):
    w, _ = _wl("c4", 1 << 16)
    tr = gs.FSM.load(w.table, w.start, w.accept).transform()
    assert tr["mode"] == "u16d" and tr["hot_rows"] < 2048


def _perm_dfa(n, nsyms, seed):
    """Permutation DFA (every column a permutation): no convergence, uniq10 = n."""
    rng = np.random.default_rng(seed)
    t = np.stack([rng.permutation(n) for _ in range(nsyms)], axis=1).astype(np.uint32)
    a = (rng.random(n) < 0.5).astype(np.uint8)
    return t, 0, a


@pytest.mark.parametrize("n", [31, 32, 63, 64])
def test_selector_enum_bound(gs, n):
    """R19's ENUM leaf: n <= 63 (maps of 32 or 64 entries).  The GPU selector and the
    oracle pick the same scheme on permutation DFAs of 31..64 states, and it is exact."""
    t, s, a = _perm_dfa(n, 3, n)
    rng = np.random.default_rng(n)
    data = rng.integers(0, 3, 1 << 18).astype(np.uint8)
    fsm = gs.FSM.load(t, s, a)
    x = torch.from_numpy(data).cuda()
    pick, ft = fsm.select_scheme(x)
    of = oracle.features(t, s, a, data, B=4096)
    assert ft["uniq10"] == pytest.approx(of["uniq10"]) == n
    assert ft["acc1"] == pytest.approx(of["acc1"]) and ft["acck"] == pytest.approx(of["acck"])
    assert ft["input_sensitivity"] == pytest.approx(of["sens"])
    assert oracle.select(of, n) == gs.SCHEMES[pick]
    assert pick == ("enum" if n <= 63 else "sre")
    ref = oracle.run(t, s, a, data, 4096)
    check_equal(fsm.run(x, scheme="auto"), ref, 4096, n)


def test_selector_features_input_sensitive(gs):
    """GPU features equal the oracle's on inputs whose segments provably differ: the
    designed div7 stream of test_oracle_pins (sens > 0.5) and a C3s slice across a
    region boundary (normal / vowel-free halves)."""
    import test_oracle_pins as pins

    w = gen.workload("c1")
    rng = np.random.default_rng(7)
    B, m = 16, 8
    N = 8 * m + 1
    res = [0] * (N + 1)
    for c in range(1, N):
        res[c] = 0 if (c - 1) // m in (0, 2, 4) and rng.random() < 0.9 else int(rng.integers(1, 7))
    bits = pins._div7_designed_bits(res, B, rng)
    cases = [(w, bits, B)]
    w3 = gen.workload("c3s")
    cases.append((w3, w3.host((1 << 26) - 33 * 4096, 65 * 4096), 4096))
    for wl, data, BB in cases:
        fsm = gs.FSM.load(wl.table, wl.start, wl.accept)
        pick, ft = fsm.select_scheme(torch.from_numpy(data).cuda(), chunk_bytes=BB)
        of = oracle.features(wl.table, wl.start, wl.accept, data, B=BB)
        assert of["sens"] >= 0.2
        assert ft["acc1"] == pytest.approx(of["acc1"]) and ft["acck"] == pytest.approx(of["acck"])
        assert ft["input_sensitivity"] == pytest.approx(of["sens"])
        assert ft["uniq10"] == pytest.approx(of["uniq10"])
        assert gs.SCHEMES[pick] == oracle.select(of, wl.nstates)


@pytest.mark.parametrize("vr_others", [1, 2, 4])
@pytest.mark.parametrize("scheme", ["rr", "nf"])
def test_vr_others_capacity(gs, vr_others, scheme):
    """Helper records go to VR^others; with 1/2/4 slots the FIFO eviction
    (R16) runs on the GPU: results exact, round diagnostics equal the oracle's."""
    w, data = _wl("c3", 4 << 20)
    ref = oracle.run(w.table, w.start, w.accept, data, 4096)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    res = fsm.run(torch.from_numpy(data).cuda(), scheme=scheme, vr_others=vr_others)
    check_equal(res, ref, 4096, w.nstates)
    sim = oracle.simulate(w.table, w.start, w.accept, data, 4096, scheme=scheme, vr_oth=vr_others)
    for k in ("rounds", "tasks_mustdo", "tasks_sre", "tasks_helper", "reread_bytes", "verify_checks",
              "verify_matches"):
        assert res.stats[k] == sim[k], (k, res.stats[k], sim[k])
    assert res.stats["tasks_helper"] > 0


@pytest.mark.parametrize("name,length,B,k", [("c1", 1 << 20, 4096, 4), ("c2", 4 << 20, 4096, 4),
                                             ("c3", 2 << 20, 4096, 4), ("c4", 4 << 20, 4096, 4),
                                             ("c2", (1 << 20) + 77, 2048, 2), ("c3s", 1 << 20, 1024, 8),
                                             ("rand:40:7:3", 200000, 48, 4), ("rand:200:30:5", 100000, 16, 1),
                                             ("c2", 3000, 4096, 4), ("c1", 16, 16, 4)])
def test_pm_tree(gs, name, length, B, k):
    """Faithful PM (FSM_SCHEME_PM_TREE): bit-exact results and every stage
    counter (merge rounds, merge lookups, invalid marks, stage-2 jumps and recoveries,
    re-read bytes) equal to the oracle twin or_simulate_pm_tree."""
    w, data = _wl(name, length)
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    fsm = _fsm(gs, w)
    res = fsm.run(torch.from_numpy(data).cuda(), scheme="pm_tree", chunk_bytes=B, spec_k=k)
    check_equal(res, ref, B, w.nstates)
    assert res.scheme == "pm_tree"
    sim = oracle.simulate_pm_tree(w.table, w.start, w.accept, data, B, k=k)
    st = res.stats
    pairs = [("rounds", "pm_levels"), ("tasks_mustdo", "pm_recoveries"), ("reread_bytes", "pm_reread_bytes"),
             ("pm_merge_checks", "pm_merge_checks"), ("pm_invalid_marks", "pm_invalid_marks"), ("pm_jumps", "pm_jumps"),
             ("verify_checks", "verify_checks"), ("verify_matches", "verify_matches")]
    for a, b in pairs:
        assert st[a] == sim[b], (a, st[a], sim[b])


def _spread_host(w, total):
    """The 1 MiB selector profile of a long stream (reading R20, include/gspec.h): 8
    portions of 128 KiB at floor(i (len - 128 KiB) / 7) rounded down to 4 KiB."""
    S = 128 << 10
    return np.concatenate([w.host((i * (total - S) // 7) & ~4095, S) for i in range(8)])


@pytest.mark.parametrize("name", ["c3s", "c3", "c2"])
def test_selector_spread_profile(gs, name):
    """fsm_select_scheme on a whole 1 GiB stream profiles 8 spread portions of it (R20):
    the GPU features equal the oracle's on the same portions, and on the input-sensitive
    stream the sensitivity feature now sees its normal and vowel-free regions."""
    L = 1 << 30
    w = gen.workload(name, length=L)
    x = torch.empty(L, dtype=torch.uint8, device="cuda")
    w.device(x)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    pick, ft = fsm.select_scheme(x)
    sample = _spread_host(w, L)
    of = oracle.features(w.table, w.start, w.accept, sample, B=4096)
    assert ft["acc1"] == pytest.approx(of["acc1"]) and ft["acck"] == pytest.approx(of["acck"])
    assert ft["input_sensitivity"] == pytest.approx(of["sens"]) and ft["uniq10"] == pytest.approx(of["uniq10"])
    assert gs.SCHEMES[pick] == oracle.select(of, w.nstates)
    if name == "c3s":
        assert of["sens"] >= 0.2
    res = fsm.run(x[:64 << 20], scheme="auto")  # the cached choice
    assert res.scheme == pick
    # R29: convergence fractions of the same spread sample equal the oracle's, and the
    # chunk-size rule (1 GiB on this GPU's SMs) picks 8 KiB for C3 / C3s (one '#' per
    # 8 KiB block: a wrong start re-converges within 8 KiB in >= 3/4 of the windows), 4 KiB for C2
    d = oracle.conv_lengths(w.table, w.start, w.accept, sample, wmax=16384)
    for W, key in ((4096, "conv4k"), (8192, "conv8k"), (16384, "conv16k")):
        assert ft[key] == pytest.approx(float((d <= W).sum()) / d.size, abs=0)
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    assert ft["chunk_bytes"] == oracle.select_chunk(d, L, sms * 768)
    assert ft["chunk_bytes"] == (4096 if name == "c2" else 8192)
    del x
    torch.cuda.empty_cache()


@pytest.mark.parametrize("length", [0, 1, 100, 20000, 21 << 10, 200 << 10])
def test_selector_short_samples(gs, length):
    """Profiles too short for a convergence window (or empty) still select, and recommend the
    default chunk size; the fractions match the oracle's windows (none below 20 KiB)."""
    w, data = _wl("c3", max(length, 1))
    data = data[:length]
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    pick, ft = fsm.select_scheme(torch.from_numpy(data.copy()).cuda())
    assert pick in gs.SCHEMES and ft["chunk_bytes"] == 4096
    d = oracle.conv_lengths(w.table, w.start, w.accept, data, wmax=16384) if length else np.zeros(0, np.uint32)
    assert (d.size == 0) == (length < 4096 + 16384 + 1)  # the first window needs 4 KiB + 16 KiB
    if d.size == 0:
        assert ft["conv4k"] == ft["conv8k"] == ft["conv16k"] == 0.0
    else:
        for W, key in ((4096, "conv4k"), (8192, "conv8k"), (16384, "conv16k")):
            assert ft[key] == pytest.approx(float((d <= W).sum()) / d.size, abs=0)


def test_selector_paper_tree_picks_nf_on_c3s(gs):
    """GSPEC_SELECTOR=paper: the reconstructed Fig. 6 tree without the B200 gate (R19b) —
    on the input-sensitive 1 GiB stream the selector picks NF, as the oracle's
    variant does on the same spread profile; then the NF run is bit-exact on a prefix."""
    import os
    L = 1 << 30
    w = gen.workload("c3s", length=L)
    x = torch.empty(L, dtype=torch.uint8, device="cuda")
    w.device(x)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    os.environ["GSPEC_SELECTOR"] = "paper"
    try:
        pick, ft = fsm.select_scheme(x)
    finally:
        os.environ.pop("GSPEC_SELECTOR", None)
    of = oracle.features(w.table, w.start, w.accept, _spread_host(w, L), B=4096)
    assert gs.SCHEMES[pick] == oracle.select(of, w.nstates, paper_tree=True) == oracle.NF
    assert oracle.select(of, w.nstates) == oracle.SRE  # the default tree (R19b)
    n = 96 << 20
    ref = oracle.run(w.table, w.start, w.accept, x[:n].cpu().numpy(), 8192)
    res = fsm.run(x[:n], scheme="auto", chunk_bytes=8192)
    assert res.scheme == "nf"
    check_equal(res, ref, 8192, w.nstates)
    del x
    torch.cuda.empty_cache()


@pytest.mark.parametrize("name,length", [("c1", 1 << 20), ("c2", 1 << 20), ("c3", 1 << 20), ("c4", 1 << 20),
                                         ("rand:40:7:3", 600000), ("rand:300:4:1", 1 << 20), ("c3s", 900000)])
def test_conv_fractions_match_oracle(gs, name, length):
    """R29: the selector's convergence fractions (k_feat_conv, one warp per window) equal the
    oracle's convergence lengths counted at 4 / 8 / 16 KiB on the same sample, and its chunk
    recommendation equals the oracle's rule for the sample's own length and for a 1 GiB
    and a 16 GiB stream (fsm_chunk_for)."""
    w, data = _wl(name, length)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    _, ft = fsm.select_scheme(torch.from_numpy(data).cuda())
    d = oracle.conv_lengths(w.table, w.start, w.accept, data, wmax=16384)
    assert d.size > 0
    for W, key in ((4096, "conv4k"), (8192, "conv8k"), (16384, "conv16k")):
        assert ft[key] == pytest.approx(float((d <= W).sum()) / d.size, abs=0), key
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    assert ft["chunk_bytes"] == oracle.select_chunk(d, length, sms * 768) == 4096  # too short for larger chunks
    for L in (1 << 30, 16 << 30):
        _, f2 = fsm.select_scheme(torch.from_numpy(data).cuda(), stream_len=L)
        assert f2["chunk_bytes"] == oracle.select_chunk(d, L, sms * 768)
    if name == "c1":
        assert ft["conv16k"] == 0.0  # div7 permutes its states: never converges


@pytest.mark.parametrize("name,length,B", [("c2", 4 << 20, 4096), ("c3", 4 << 20, 4096), ("c4", 2 << 20, 4096),
                                           ("rand:40:7:3", 300000, 48), ("rand:150:3:9", 200000, 64),
                                           ("c1", 1 << 18, 1024), ("c3", (3 << 20) + 555, 2048)])
@pytest.mark.parametrize("scheme,L", [("sre", 3), ("sre", 16), ("rr", 8), ("nf", 5), ("pm", 16), ("cse", 8),
                                      ("pm_tree", 4)])
def test_lookback_long(gs, name, length, B, scheme, L):
    """Lookback over L > 2 symbols (reading R25: per-chunk QS from the pair image
    with multiplicities walked over the extra symbols, k_qs_long): bit-exact results and
    round diagnostics equal to the oracle's simulation with the same lookback."""
    w, data = _wl(name, length)
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    fsm = _fsm(gs, w)
    res = fsm.run(torch.from_numpy(data).cuda(), scheme=scheme, chunk_bytes=B, lookback=L)
    check_equal(res, ref, B, w.nstates)
    if scheme == "pm_tree":
        return
    sim = oracle.simulate(w.table, w.start, w.accept, data, B, scheme=scheme, lookback=L)
    for k in ("rounds", "tasks_mustdo", "tasks_sre", "tasks_helper", "reread_bytes", "verify_checks",
              "verify_matches"):
        assert res.stats[k] == sim[k], (k, res.stats[k], sim[k])


def test_lookback_long_wide_fallback(gs):
    """A permutation DFA (every 2-symbol image has all 100 states > 64): lookback 8 keeps
    the lookback-2 ranking (R25), exactly as the oracle does."""
    t, s, a = _perm_dfa(100, 3, 5)
    rng = np.random.default_rng(5)
    data = rng.integers(0, 3, 20 * 4096).astype(np.uint8)
    ref = oracle.run(t, s, a, data, 1024)
    fsm = gs.FSM.load(t, s, a)
    res = fsm.run(torch.from_numpy(data).cuda(), scheme="sre", chunk_bytes=1024, lookback=8)
    check_equal(res, ref, 1024, 100)
    sim = oracle.simulate(t, s, a, data, 1024, scheme="sre", lookback=8)
    sim2 = oracle.simulate(t, s, a, data, 1024, scheme="sre", lookback=2)
    assert res.stats["verify_matches"] == sim["verify_matches"] == sim2["verify_matches"]


@pytest.mark.parametrize("name,length,B,k", [("c3", 8 << 20, 4096, 16), ("c1", 1 << 20, 4096, 16),
                                             ("c2", 4 << 20, 4096, 12), ("rand:60:5:2", 300000, 64, 16)])
def test_cse_spec16(gs, name, length, B, k):
    """CSE with up to 16 paths per chunk (the whole lookback image of C3's
    16-value counter; the 16-path TMA kernel runs 16 warps of 128 registers): exact, and
    its rounds equal the oracle's simulation with the same spec_k."""
    w, data = _wl(name, length)
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    fsm = _fsm(gs, w)
    res = fsm.run(torch.from_numpy(data).cuda(), scheme="cse", chunk_bytes=B, spec_k=k)
    check_equal(res, ref, B, w.nstates)
    sim = oracle.simulate(w.table, w.start, w.accept, data, B, scheme="cse", spec_k=k)
    for key in ("rounds", "tasks_mustdo", "tasks_sre", "reread_bytes", "verify_checks", "verify_matches"):
        assert res.stats[key] == sim[key], (key, res.stats[key], sim[key])


@pytest.mark.parametrize("name,length,B,scheme", [("c3", 32 << 20, 4096, "rr"), ("c3s", 64 << 20, 4096, "nf"),
                                                  ("rand:40:7:3", 4 << 20, 256, "rr"), ("c1", 1 << 20, 1024, "nf")])
def test_memoized_helpers_match_eager(gs, name, length, B, scheme):
    """R28: memoized RR / NF helpers (opt-in GSPEC_LAZY_HELPERS=1: walked when a
    verification first matches them) give the eager helpers' results and round counters
    exactly; only helper_walks differs.  The memoized run is a child process (the switch is
    read once per process); this process runs the default eager helpers."""
    import json
    import os
    import subprocess
    import sys

    w, data = _wl(name, length)
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    sim = oracle.simulate(w.table, w.start, w.accept, data, B, scheme=scheme)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    x = torch.from_numpy(data).cuda()
    for _ in range(2):  # the second run uses the dense-round slots the first one sized
        res = fsm.run(x, scheme=scheme, chunk_bytes=B)
        check_equal(res, ref, B, w.nstates)
        for k in ("rounds", "tasks_mustdo", "tasks_sre", "tasks_helper", "reread_bytes", "verify_checks",
                  "verify_matches"):
            assert res.stats[k] == sim[k], (k, res.stats[k], sim[k])
    assert res.stats["helper_walks"] == 0  # eager by default
    code = ("import sys, json, torch; sys.path.insert(0, '.'); import gen, paper_conf_ipps_wangwqw22_b200 as gs;"
            f"w = gen.workload({name!r}, length={length}); x = torch.empty({length}, dtype=torch.uint8, device='cuda');"
            "w.device(x); f = gs.FSM.load(w.table, w.start, w.accept);"
            f"r = [f.run(x, scheme={scheme!r}, chunk_bytes={B}) for _ in range(2)][-1];"
            "print(json.dumps([r.final_state, r.accept_count, r.stats['tasks_helper'], r.stats['helper_walks']]))")
    env = dict(os.environ, GSPEC_LAZY_HELPERS="1")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=env, cwd=root, timeout=600)
    assert out.returncode == 0, out.stderr[-2000:]
    fin, cnt, th, hw = json.loads(out.stdout.strip().splitlines()[-1])
    assert (fin, cnt, th) == (res.final_state, res.accept_count, res.stats["tasks_helper"]) and hw <= th


@pytest.mark.parametrize("name,length,B,scheme,ck", [
    ("c3", 32 << 20, 8192, "sre", None), ("c3", (24 << 20) + 1000, 4096, "sre", "64"),
    ("c3s", 96 << 20, 8192, "nf", None), ("c3", 32 << 20, 8192, "rr", "2048"), ("c3", 16 << 20, 4096, "nf", "4096"),
    ("c3", 48 << 20, 16384, "sre", "0")])
def test_checkpointed_dense_rounds(gs, name, length, B, scheme, ck):
    """R30: dense-round tasks stop where their path meets the chunk's round-0 path at a
    checkpoint (every GSPEC_CK bytes of the round-0 walk, default 512; 0 = off).  Results,
    records and round counters equal the oracle's for every interval (the interval is read
    once per process: non-default ones run in a child process); with checkpoints the task
    kernel walks far fewer bytes than the tasks' nominal chunk bytes (C3: the counter part
    of the state converges at the chunk's reset byte)."""
    import json
    import os
    import subprocess
    import sys

    w, data = _wl(name, length)
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    sim = oracle.simulate(w.table, w.start, w.accept, data, B, scheme=scheme)
    keys = ("rounds", "tasks_mustdo", "tasks_sre", "tasks_helper", "reread_bytes", "verify_checks", "verify_matches")
    if ck is None:  # the default interval, in this process
        fsm = gs.FSM.load(w.table, w.start, w.accept)
        x = torch.from_numpy(data).cuda()
        for _ in range(2):  # the second run has the dense-round slots the first one sized
            res = fsm.run(x, scheme=scheme, chunk_bytes=B)
            check_equal(res, ref, B, w.nstates)
            for k in keys:
                assert res.stats[k] == sim[k], (k, res.stats[k], sim[k])
        assert res.stats["tasks_sre"] > 1024
        walked = res.stats["task_walked_bytes"]
        assert 0 < walked < 0.75 * res.stats["reread_bytes"], (walked, res.stats["reread_bytes"])
        return
    code = ("import sys, json, torch, numpy as np; sys.path.insert(0, '.'); import gen, paper_conf_ipps_wangwqw22_b200 as gs;"
            f"w = gen.workload({name!r}, length={length}); x = torch.empty({length}, dtype=torch.uint8, device='cuda');"
            "w.device(x); f = gs.FSM.load(w.table, w.start, w.accept);"
            f"r = [f.run(x, scheme={scheme!r}, chunk_bytes={B}) for _ in range(2)][-1];"
            "ce = r.chunk_ends.cpu().numpy().view(np.uint32);"
            "print(json.dumps([r.final_state, r.accept_count, int(ce.astype(np.uint64).sum()), int(ce[::97].astype(np.uint64).sum()),"
            f" r.stats, {length}]))")
    env = dict(os.environ, GSPEC_CK=ck)
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=env, cwd=root, timeout=600)
    assert out.returncode == 0, out.stderr[-2000:]
    fin, cnt, s_all, s_97, stats, _ = json.loads(out.stdout.strip().splitlines()[-1])
    rce = ref["chunk_end"].astype(np.uint64)
    assert (fin, cnt) == (ref["final"], ref["count"])
    assert (s_all, s_97) == (int(rce.sum()), int(rce[::97].sum()))
    for k in keys:
        assert stats[k] == sim[k], (k, stats[k], sim[k])
    if int(ck) == 0 or B < 2 * int(ck):  # off (or no checkpoint inside a chunk): whole chunks
        assert 0 < stats["task_walked_bytes"] <= stats["reread_bytes"]
        assert stats["task_walked_bytes"] % B == 0
    else:
        assert 0 < stats["task_walked_bytes"] < stats["reread_bytes"]


@pytest.mark.parametrize("name,length,B", [("c1", (16 << 20) + 5, 4096), ("rand:7:2:3", (6 << 20) + 17, 1024),
                                           ("rand:5:2:9", 3 << 20, 4096), ("c1", 1 << 20, 4096)])
def test_enum_packed_maps_on_off(gs, name, length, B):
    """DESIGN.md §5.3 packed maps (K = 8, nt <= 8: one 8-byte lookup per 8 symbols for all
    chains): bit-exact against the oracle with the packed maps (default) and without them
    (GSPEC_TK_PK=0 at load: per-chain TK lookups), in the multi-launch walk and the
    single-launch kernel (<= 2 MiB), with unaligned tails."""
    import os
    w, data = _wl(name, length)
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    x = torch.from_numpy(data).cuda()
    for flag in ("1", "0"):
        os.environ["GSPEC_TK_PK"] = flag
        try:
            fsm = gs.FSM.load(w.table, w.start, w.accept)
        finally:
            os.environ.pop("GSPEC_TK_PK", None)
        res = fsm.run(x, scheme="enum", chunk_bytes=B)
        check_equal(res, ref, B, w.nstates)
        fsm.close()


@pytest.mark.parametrize("exc", ["1", "2"])
@pytest.mark.parametrize("scheme", ["sre", "rr", "cse"])
def test_delta_rows_exception_plans(gs, exc, scheme):
    """C4's delta rows with the one-exception plan (default: the rows needing
    two exceptions are hot, the walk kernels use the one-exception step) and with the
    two-exception plan (GSPEC_DELTA_EXC=2 at load) — both bit-exact against the oracle, round
    counters equal to the oracle's simulation; every other kernel reads either image with the
    two-exception step."""
    import os
    w, data = _wl("c4", 4 << 20)
    B = 4096
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    sim = oracle.simulate(w.table, w.start, w.accept, data, B, scheme=scheme)
    os.environ["GSPEC_DELTA_EXC"] = exc
    try:
        fsm = gs.FSM.load(w.table, w.start, w.accept)
    finally:
        os.environ.pop("GSPEC_DELTA_EXC", None)
    assert fsm.transform()["mode"] == "u16d"
    res = fsm.run(torch.from_numpy(data).cuda(), scheme=scheme, chunk_bytes=B)
    check_equal(res, ref, B, w.nstates)
    for k in ("rounds", "tasks_mustdo", "tasks_sre", "tasks_helper", "verify_checks", "verify_matches"):
        assert res.stats[k] == sim[k], (k, res.stats[k], sim[k])
    lit = fsm.run_literal(torch.from_numpy(data[: 1 << 20]).cuda(), scheme="sre", chunk_bytes=B)
    ref1 = oracle.run(w.table, w.start, w.accept, data[: 1 << 20], B)
    assert lit.final_state == ref1["final"] and lit.accept_count == ref1["count"]
    fsm.close()
