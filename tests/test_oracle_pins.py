"""Pins for the CPU oracle (-m "not gpu").

The oracle (oracle/oracle.c) is checked against things the paper and
mathematics fix, never against itself:
  * div7: big-integer value mod 7, and an independent closed form
    for prefix residues (powers of two mod 7 have period 3);
  * Fig. 4: the worked transformation example (golden file);
  * Aho–Corasick DFAs: brute-force multi-pattern search from first principles;
  * AC x Z16 counter: closed form per component;
  * enumeration / composition: brute force over all starts and chunkings;
  * lookback containment and the div7 closed form of its image.
"""
import os
import random

import numpy as np
import pytest

import gen
import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")


# ---------------------------------------------------------------- div7 ------
def div7_prefix_residues(bits: np.ndarray) -> np.ndarray:
    """value(prefix of length m) mod 7 for m = 1..len, WITHOUT the DFA recurrence:
    value = sum_i b_i 2^(m-1-i);  2^j mod 7 = (1,2,4)[j mod 3]."""
    b = bits.astype(np.int64)
    L = b.size
    i = np.arange(L)
    S = np.zeros((3, L), np.int64)  # S[r][m-1] = sum_{i<m, i%3==r} b_i
    for r in range(3):
        S[r] = np.cumsum(np.where(i % 3 == r, b, 0))
    m = np.arange(1, L + 1)
    pw = np.array([1, 2, 4])
    val = np.zeros(L, np.int64)
    for r in range(3):
        val += S[r] * pw[(m - 1 - r) % 3]
    return val % 7


@pytest.mark.parametrize("seed,length,B", [(1, 1, 16), (2, 1000, 16), (3, 4096, 64), (4, 20000, 4096),
                                          (5, 33333, 48), (0x5EED0001, 1 << 16, 4096)])
def test_div7_closed_form(seed, length, B):
    w = gen.workload("c1", length=length, seed=seed)
    bits = w.host()
    r = oracle.run(w.table, w.start, w.accept, bits, B)
    assert r["status"] == 0
    big = int("".join("01"[x] for x in bits), 2)  # the paper's "binary number"
    assert r["final"] == big % 7
    assert r["accept"] == (big % 7 == 0)
    res = div7_prefix_residues(bits)
    assert r["count"] == int((res == 0).sum())
    nb = oracle.nchunks(length, B)
    ends = [min(length, (c + 1) * B) for c in range(nb)]
    assert list(r["chunk_end"]) == [int(res[e - 1]) for e in ends]
    # spot-check chunk ends with Python big ints as well
    for c in sorted(set([0, nb // 2, nb - 1])):
        assert r["chunk_end"][c] == int("".join("01"[x] for x in bits[:ends[c]]), 2) % 7


def test_div7_empty_and_invalid():
    t, s, a = gen.dfa_div7()
    r = oracle.run(t, s, a, np.zeros(0, np.uint8))
    assert r["status"] == 0 and r["final"] == 0 and r["accept"] == 1 and r["count"] == 0
    assert len(r["chunk_end"]) == 0
    r = oracle.run(t, s, a, np.array([1, 0, 2, 1], np.uint8))
    assert r["status"] == oracle.OR_ESYMBOL


# ---------------------------------------------------------------- Fig. 4 ----
def _fig4():
    orig, trans, mapping, hot = {}, [], {}, None
    for line in open(os.path.join(GOLD, "fig4_transform.txt")):
        if line.startswith("#") or not line.strip():
            continue
        f = line.split()
        if f[0] == "original":
            orig[int(f[1][1:])] = [int(x[1:]) for x in f[2:5]]
        elif f[0] == "transformed":
            trans.append(([int(x[1:-1]) for x in f[2:5]], int(f[5])))
        elif f[0] == "mapping":
            mapping[int(f[1][1:])] = int(f[2][1:-1])
        elif f[0] == "hot":
            hot = int(f[1])
    table = np.array([orig[i] for i in range(4)], np.uint32)
    return table, trans, mapping, hot


def test_fig4_transformation_golden():
    table, trans, mapping, hot = _fig4()
    perm, inv, freq, tt, acc = oracle.transform(table, np.zeros(4, np.uint8))
    assert [int(perm[q]) for q in range(4)] == [mapping[q] for q in range(4)]
    for r, (row, fr) in enumerate(trans):
        assert list(tt[r]) == row
        assert freq[inv[r]] == fr
    # hot test "state ID < 2" selects exactly the two highest-frequency states
    assert sorted(freq, reverse=True)[:hot] == [freq[inv[r]] for r in range(hot)]
    # poison row appended last, absorbing
    assert perm[4] == 4 and inv[4] == 4 and list(tt[4]) == [4, 4, 4]


@pytest.mark.parametrize("seed", range(6))
def test_transform_is_renaming(seed):
    rng = np.random.default_rng(seed)
    n, ns = int(rng.integers(1, 40)), int(rng.integers(1, 20))
    t, s, a = gen.dfa_random(seed, n, ns)
    perm, inv, freq, tt, acc = oracle.transform(t, a)
    assert sorted(perm[:n]) == list(range(n))
    assert all(inv[perm[q]] == q for q in range(n))
    # ranks are non-increasing in frequency; ties ordered by original id
    for r in range(n - 1):
        q1, q2 = inv[r], inv[r + 1]
        assert freq[q1] > freq[q2] or (freq[q1] == freq[q2] and q1 < q2)
    # independent in-degree count
    indeg = np.bincount(t.ravel(), minlength=n)
    assert (freq == indeg).all()
    for q in range(n):
        assert acc[perm[q]] == a[q]
        for c in range(ns):
            assert tt[perm[q], c] == perm[t[q, c]]
    # running the transformed DFA gives the renamed result ("preserve the semantics")
    data = gen.workload(f"rand:{n}:{ns}:{seed}", length=3000, seed=seed).host()
    r1 = oracle.run(t, s, a, data, 64)
    r2 = oracle.run(tt[:n], int(perm[s]), acc[:n], data, 64)
    assert r2["count"] == r1["count"] and inv[r2["final"]] == r1["final"]
    assert (inv[r2["chunk_end"]] == r1["chunk_end"]).all()


def test_transform_profile_policy():
    t, s, a = gen.dfa_random(11, 20, 4)
    data = gen.workload("rand:20:4:11", length=5000).host()
    perm, inv, freq, tt, acc = oracle.transform(t, a, policy=1, profile=data, start=s)
    # visit counts: independent count of states visited by the walk (incl. the start)
    visits = np.zeros(20, np.int64)
    st = s
    visits[st] += 1
    for x in data:
        st = t[st, x]
        visits[st] += 1
    assert (freq == visits).all()
    assert sorted(perm[:20]) == list(range(20))


# ---------------------------------------------------------------- AC --------
def ac_bruteforce(lits, text: bytes):
    """Accept positions = positions where some literal ends (naive search)."""
    ends = set()
    for L in lits:
        if not L:
            continue
        i = text.find(L)
        while i >= 0:
            ends.add(i + len(L))
            i = text.find(L, i + 1)
    return ends


def ac_state_after(table, lits, text: bytes, m: int, maxlen: int):
    """Trie node of the longest suffix of text[:m] that is a prefix of a literal."""
    prefixes = set()
    for L in lits:
        for k in range(len(L) + 1):
            prefixes.add(L[:k])
    for k in range(min(m, maxlen), -1, -1):
        suf = text[m - k:m]
        if suf in prefixes:
            node = 0
            for ch in suf:  # goto edges of the trie (every step stays on the trie)
                node = int(table[node, ch])
            return node
    return 0


@pytest.mark.parametrize("seed,length,B", [(7, 3000, 64), (8, 9000, 512), (0x5EED0002, 1 << 14, 4096)])
def test_ac_bruteforce(seed, length, B):
    w = gen.workload("c2", length=length, seed=seed)
    text = w.host()
    tb = bytes(text)
    r = oracle.run(w.table, w.start, w.accept, text, B)
    ends = ac_bruteforce(w.literals, tb)
    assert r["count"] == len(ends)
    maxlen = max(len(L) for L in w.literals)
    nb = oracle.nchunks(length, B)
    for c in range(nb):
        m = min(length, (c + 1) * B)
        assert r["chunk_end"][c] == ac_state_after(w.table, w.literals, tb, m, maxlen)
    assert r["final"] == ac_state_after(w.table, w.literals, tb, length, maxlen)


def test_ac_counter_closed_form():
    w = gen.workload("c3", length=40000, seed=99)
    text = w.host()
    tb = bytes(text)
    r = oracle.run(w.table, w.start, w.accept, text, 256)
    lb, lo = w.keep
    tac, _, aac = gen.dfa_ac(lb, lo)
    maxlen = max(len(L) for L in w.literals)
    vowels = set(b"aeiou")
    k = 0
    ks = []
    for ch in tb:  # counter: vowels since the last reset, mod 16
        k = 0 if ch == gen.RESET_BYTE else ((k + 1) % 16 if ch in vowels else k)
        ks.append(k)
    ends = ac_bruteforce(w.literals, tb)
    expect_cnt = sum(1 for m in ends if ks[m - 1] == 0)
    assert r["count"] == expect_cnt
    for c in range(0, oracle.nchunks(len(tb), 256), 7):
        m = min(len(tb), (c + 1) * 256)
        a = ac_state_after(tac, w.literals, tb, m, maxlen)
        assert r["chunk_end"][c] == a * 16 + ks[m - 1]


# -------------------------------------------------------- enumeration -------
@pytest.mark.parametrize("seed", range(8))
def test_enum_bruteforce_all_chunkings(seed):
    rng = random.Random(seed)
    n, ns = rng.randint(1, 16), rng.randint(1, 6)
    t, s, a = gen.dfa_random(seed + 100, n, ns)
    data = gen.workload(f"rand:{n}:{ns}:{seed}", length=rng.randint(0, 200), seed=seed).host()
    seq = oracle.run(t, s, a, data, 16)
    # every start, every split point: enum(prefix) then enum(suffix) composes to the run
    for cut in range(0, len(data) + 1, max(1, len(data) // 13)):
        M1, C1 = oracle.enum(t, a, data[:cut])
        M2, C2 = oracle.enum(t, a, data[cut:])
        M, C = oracle.compose(M1, C1, M2, C2)
        for q in range(n):
            rq = oracle.run(t, q, a, data, 16)
            assert M[q] == rq["final"] and C[q] == rq["count"]
        assert M[s] == seq["final"] and C[s] == seq["count"]


def test_enum_composition_invariant_chunks():
    w = gen.workload("c1", length=5000, seed=5)
    data = w.host()
    B = 256
    seq = oracle.run(w.table, w.start, w.accept, data, B)
    M = np.arange(7, dtype=np.uint32)
    C = np.zeros(7, np.uint64)
    starts = []
    for c in range(oracle.nchunks(len(data), B)):
        starts.append(int(M[w.start]))
        Mc, Cc = oracle.enum(w.table, w.accept, data[c * B:(c + 1) * B])
        M, C = oracle.compose(M, C, Mc, Cc)
        assert M[w.start] == seq["chunk_end"][c]
    assert M[w.start] == seq["final"] and C[w.start] == seq["count"]


# ------------------------------------------------------------ lookback ------
def test_lookback_div7_closed_form():
    t, s, a = gen.dfa_div7()
    # delta*(q, ab) = 4q + 2a + b mod 7 is a bijection in q: image = all 7, mult 1 each
    for w in ([0, 0], [0, 1], [1, 0], [1, 1]):
        qs, img = oracle.lookback(t, 7, np.array(w, np.uint8), K=16)
        assert img == 7 and list(qs) == list(range(7))
    qs, img = oracle.lookback(t, 7, np.array([1, 5], np.uint8))
    assert img == 1 and list(qs) == [7]  # invalid symbol -> poison only


@pytest.mark.parametrize("seed", range(5))
def test_lookback_containment(seed):
    """the real start state must be in the produced end state set."""
    rng = random.Random(seed)
    n, ns = rng.randint(2, 30), rng.randint(1, 8)
    t, s, a = gen.dfa_random(seed + 7, n, ns)
    data = gen.workload(f"rand:{n}:{ns}:{seed}", length=2000, seed=seed).host()
    B = 64
    r = oracle.run(t, s, a, data, B)
    for L in (1, 2, 3):
        for c in range(1, oracle.nchunks(len(data), B)):
            qs, img = oracle.lookback(t, n, data[c * B - L:c * B], K=n)
            assert img == len(qs)
            assert r["chunk_end"][c - 1] in set(qs.tolist())
    # ranking by multiplicity: brute-force count
    w = data[62:64]
    qs, img = oracle.lookback(t, n, w, K=n)
    mult = {}
    for q in range(n):
        e = t[t[q, w[0]], w[1]]
        mult[int(e)] = mult.get(int(e), 0) + 1
    expect = sorted(mult, key=lambda e: (-mult[e], e))
    assert list(qs) == expect


@pytest.mark.parametrize("seed", range(4))
def test_lookback_long(seed):
    """Lookback over L in [2, 16] symbols (reading R25): the true start is in the
    image (containment) for every L; the image over the last L symbols is a subset of the
    image over the last 2 (delta*(Q, uv) is a subset of delta*(Q, v)); the ranking is the
    brute-force multiplicity ranking over all states; a DFA whose 2-symbol images exceed 64
    states (a permutation DFA) falls back to the lookback-2 ranking of the last two symbols."""
    rng = random.Random(seed + 100)
    n, ns = rng.randint(2, 40), rng.randint(1, 6)
    t, s, a = gen.dfa_random(seed + 77, n, ns)
    data = gen.workload(f"rand:{n}:{ns}:{seed}", length=4000, seed=seed).host()
    B = 64
    r = oracle.run(t, s, a, data, B)
    for L in (2, 3, 5, 9, 16):
        for c in range(1, oracle.nchunks(len(data), B)):
            w = data[c * B - L:c * B]
            qs, img = oracle.lookback_long(t, n, w, K=n)
            q2, img2 = oracle.lookback(t, n, w[-2:], K=n)
            assert r["chunk_end"][c - 1] in set(qs.tolist())
            assert set(qs.tolist()) <= set(q2.tolist()) and img <= img2
            if c % 7 == 0:  # brute force ranking
                mult = {}
                for q in range(n):
                    e = q
                    for ch in w:
                        e = int(t[e, ch])
                    mult[e] = mult.get(e, 0) + 1
                assert list(qs) == sorted(mult, key=lambda e: (-mult[e], e))
    rng2 = np.random.default_rng(seed)
    nperm = 100
    tp = np.stack([rng2.permutation(nperm) for _ in range(3)], axis=1).astype(np.uint32)
    w = np.array([0, 1, 2, 1, 0, 2], np.uint8)
    qs, img = oracle.lookback_long(tp, nperm, w, K=16)
    q2, img2 = oracle.lookback(tp, nperm, w[-2:], K=16)
    assert list(qs) == list(q2) and img == img2 == nperm


@pytest.mark.parametrize("scheme", ["sre", "rr", "pm", "cse"])
@pytest.mark.parametrize("L", [3, 8, 16])
def test_simulate_lookback_long(scheme, L):
    """Every scheme with a longer lookback still reaches the sequential result."""
    rng = random.Random(L)
    n, ns = rng.randint(2, 30), rng.randint(2, 5)
    t, s, a = gen.dfa_random(L + 3, n, ns)
    data = gen.workload(f"rand:{n}:{ns}:{L}", length=30000, seed=L).host()
    for B in (16, 64):
        r = oracle.run(t, s, a, data, B)
        o = oracle.simulate(t, s, a, data, B, scheme=scheme, lookback=L)
        assert o["status"] == 0 and o["final_state"] == r["final"] and o["accept_count"] == r["count"]
        assert (o["chunk_end"] == r["chunk_end"]).all()


# ----------------------------------------------------------- simulate -------
@pytest.mark.parametrize("scheme", ["seq", "pm", "sre", "rr", "nf", "cse"])
@pytest.mark.parametrize("seed", range(6))
def test_simulate_equals_sequential(scheme, seed):
    rng = random.Random(seed * 31 + len(scheme))
    n, ns = rng.randint(1, 24), rng.randint(1, 5)
    t, s, a = gen.dfa_random(seed + 3, n, ns)
    length = rng.randint(0, 3000)
    data = gen.workload(f"rand:{n}:{ns}:{seed}", length=length, seed=seed).host()
    for B in (16, 48, 256):
        r = oracle.run(t, s, a, data, B)
        o = oracle.simulate(t, s, a, data, B, scheme=scheme, spec_k=rng.randint(1, 4), qs_cap=rng.randint(1, 16),
                            vr_end=rng.randint(1, 16), vr_oth=rng.randint(1, 16))
        assert o["status"] == 0
        assert o["final_state"] == r["final"] and o["accept_count"] == r["count"]
        assert (o["chunk_end"] == r["chunk_end"]).all()
        assert o["accept"] == a[r["final"]]


def test_simulate_seq_is_alg2():
    """SEQ = Alg. 2: one must-do recovery per mismatch of the sequential chain."""
    w = gen.workload("c3", length=60000, seed=4)
    data = w.host()
    B = 1024
    o = oracle.simulate(w.table, w.start, w.accept, data, B, scheme="seq", max_tasks=10000)
    perm, inv, _, tt, acc = oracle.transform(w.table, w.accept)
    r = oracle.run(w.table, w.start, w.accept, data, B)
    # Alg. 2 L9-14 literally: compare end_p with VR_i[0].start
    mism = 0
    endp = int(perm[r["chunk_end"][0]])
    for c in range(1, oracle.nchunks(len(data), B)):
        qs, _ = oracle.lookback(tt, w.nstates, data[c * B - 2:c * B], K=16)
        if endp != qs[0]:
            mism += 1
        endp = int(perm[r["chunk_end"][c]])
    assert o["rounds"] == mism == o["tasks_mustdo"] == o["tasks_total"]
    assert all(k == 0 for (_, _, _, k) in o["tasks"])


def test_simulate_rr_bound_and_nf_order():
    w = gen.workload("c3", length=1 << 16, seed=8)
    data = w.host()
    B = 512
    N = oracle.nchunks(len(data), B)
    for scheme in ("rr", "nf"):
        o = oracle.simulate(w.table, w.start, w.accept, data, B, scheme=scheme, max_tasks=1 << 20)
        assert o["ntasks"] == o["tasks_total"] == o["tasks_mustdo"] + o["tasks_sre"] + o["tasks_helper"]
        rounds = {}
        for (rd, c, st, k) in o["tasks"]:
            rounds.setdefault(rd, []).append((c, st, k))
        for rd, tasks in rounds.items():
            f = [c for (c, _, k) in tasks if k == 0]
            assert len(f) == 1
            f = f[0]
            helpers = [(c, st) for (c, st, k) in tasks if k == 2]
            assert all(c > f for c, _ in helpers)  # no helper on verified chunks
            per = {}
            for c, st in helpers:
                per.setdefault(c, []).append(st)
            for c, sts in per.items():
                assert len(sts) == len(set(sts))  # distinct speculative states
            if scheme == "rr" and helpers:
                # at most 1 + ceil((i-1)/(T-i)) threads per chunk, i = f+1, T = N
                i = f + 1
                bound = 1 + -(-(i - 1) // (N - i)) if N > i else 1
                idle = N - sum(1 for (_, _, k) in tasks if k in (0, 1))
                bound = 1 + -(-idle // (N - f - 1))
                for c, sts in per.items():
                    assert len(sts) + 1 <= bound
            if scheme == "nf" and helpers:
                # nearest first: helper chunks are a contiguous run starting at f+1
                cs = sorted(per)
                assert cs[0] == f + 1 and cs == list(range(cs[0], cs[-1] + 1))
                assert [c for c, _ in helpers] == sorted(c for c, _ in helpers)


def test_simulate_cse_exact_coverage():
    """CSE: when a chunk's lookback-2 image has <= spec_k states, round 0
    ran every state of it, and the true start is in it (pinned by
    test_lookback_containment), so verification needs no recovery there.  div7:
    every 2-symbol image is all 7 states (closed form above) -> zero rounds, every
    check matches.  Tiny random DFAs (n <= 8): every image has <= n states -> zero
    rounds.  C3 (counter images > 8): recovery rounds remain, result still exact."""
    t, s, a = gen.dfa_div7()
    data = gen.workload("c1", length=50000, seed=3).host()
    for B in (16, 256, 4096):
        o = oracle.simulate(t, s, a, data, B, scheme="cse")
        N = oracle.nchunks(len(data), B)
        assert o["rounds"] == 0 and o["tasks_total"] == 0
        assert o["verify_checks"] == o["verify_matches"] == N
        pm = oracle.simulate(t, s, a, data, B, scheme="pm", spec_k=4)  # 4 of 7: must recover
        assert pm["rounds"] > 0
    for seed in range(8):
        rng = random.Random(seed)
        n, ns = rng.randint(1, 8), rng.randint(1, 6)
        t, s, a = gen.dfa_random(seed + 11, n, ns)
        data = gen.workload(f"rand:{n}:{ns}:{seed}", length=20000, seed=seed).host()
        o = oracle.simulate(t, s, a, data, 64, scheme="cse")
        r = oracle.run(t, s, a, data, 64)
        assert o["rounds"] == 0 and o["final_state"] == r["final"] and o["accept_count"] == r["count"]
    w = gen.workload("c3", length=1 << 18, seed=2)
    data = w.host()
    o = oracle.simulate(w.table, w.start, w.accept, data, 4096, scheme="cse")
    r = oracle.run(w.table, w.start, w.accept, data, 4096)
    assert o["rounds"] > 0 and o["final_state"] == r["final"] and (o["chunk_end"] == r["chunk_end"]).all()


@pytest.mark.parametrize("seed", range(6))
def test_simulate_literal_sre(seed):
    """Paper-literal SRE (Alg. 2 L2-6 + Alg. 3 verbatim) reaches the sequential
    result (the invariant of Alg. 3: after the iteration with frontier f every chunk <= f
    holds its true end) on random DFAs and chunkings; Alg. 3's accounting: one must-do per
    iteration whose frontier missed, at most N of them, every re-execution is a task."""
    rng = random.Random(seed * 7 + 1)
    n, ns = rng.randint(1, 24), rng.randint(1, 5)
    t, s, a = gen.dfa_random(seed + 21, n, ns)
    data = gen.workload(f"rand:{n}:{ns}:{seed}", length=rng.randint(0, 4000), seed=seed).host()
    for B in (16, 48, 256):
        r = oracle.run(t, s, a, data, B)
        o = oracle.simulate_literal_sre(t, s, a, data, B, vr_cap=rng.randint(1, 16))
        N = oracle.nchunks(len(data), B)
        assert o["status"] == 0
        assert o["final_state"] == r["final"] and o["accept_count"] == r["count"]
        assert (o["chunk_end"] == r["chunk_end"]).all()
        assert o["rounds"] == o["tasks_mustdo"] <= max(N, 0)
        assert o["tasks_total"] >= o["rounds"] and o["verify_checks"] == N * N
    # a DFA whose lookback always predicts right (one state): no recovery at all
    t1 = np.zeros((1, 3), np.uint32)
    d1 = np.array([0, 1, 2] * 300, np.uint8)
    o = oracle.simulate_literal_sre(t1, 0, np.array([1], np.uint8), d1, 16)
    assert o["rounds"] == 0 and o["accept_count"] == len(d1)


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("scheme", ["sre", "rr", "nf"])
def test_simulate_literal_rr_nf(seed, scheme):
    """Paper-literal Alg. 3 / 4 / 5 on random DFAs and chunkings:
    * results equal the sequential run;
    * N iterations with N checks each; one must-do per iteration whose frontier missed;
    * the literal SRE loop equals the separate literal-SRE simulator exactly;
    * RR: at most 1 + ceil((i-1)/(T-i)) threads work on a chunk in an iteration with
      frontier i (P:195, 1-indexed; here i = fr + 1, T = N);
    * NF: helpers fill QS_{f+1} before QS_{f+2}: in every iteration the helper
      targets are non-decreasing in tid order and every chunk before the last targeted
      one gets all its remaining candidates (counted from the lookback ranking, whose
      ranking is pinned above, and the dequeues logged in earlier iterations)."""
    rng = random.Random(seed * 13 + 5)
    n, ns = rng.randint(2, 24), rng.randint(2, 5)
    t, s, a = gen.dfa_random(seed + 41, n, ns)
    data = gen.workload(f"rand:{n}:{ns}:{seed}", length=rng.randint(1, 6000), seed=seed + 3).host()
    perm, inv, _, tt, acc = oracle.transform(t, a)
    for B in (16, 48, 256):
        vr_cap = rng.randint(1, 16)
        r = oracle.run(t, s, a, data, B)
        o = oracle.simulate_literal(t, s, a, data, B, scheme=scheme, vr_cap=vr_cap, max_tasks=1 << 20)
        N = oracle.nchunks(len(data), B)
        assert o["status"] == 0
        assert o["final_state"] == r["final"] and o["accept_count"] == r["count"]
        assert (o["chunk_end"] == r["chunk_end"]).all()
        assert o["verify_checks"] == N * N and o["rounds"] == o["tasks_mustdo"] <= N
        assert o["tasks_total"] == o["tasks_mustdo"] + o["tasks_sre"] + o["tasks_helper"] == len(o["tasks"])
        if scheme == "sre":
            ls = oracle.simulate_literal_sre(t, s, a, data, B, vr_cap=vr_cap)
            for k in ("rounds", "tasks_total", "tasks_mustdo", "tasks_sre", "reread_bytes", "verify_checks",
                      "verify_matches", "accept_count"):
                assert o[k] == ls[k], k
            assert o["tasks_helper"] == 0
            continue
        qlen = [1] + [len(oracle.lookback(tt, n, data[c * B - 2:c * B], K=16)[0]) for c in range(1, N)]
        taken = [1] * N  # round 0 ran QS.front()
        by_it = {}
        for it, cid, st, kind in o["tasks"]:
            by_it.setdefault(it, []).append((cid, st, kind))
        for it, ts in sorted(by_it.items()):
            fr = [cid for cid, _, k in ts if k == 0]
            assert len(fr) == 1
            fr = fr[0]
            per = {}
            for cid, _, _ in ts:
                per[cid] = per.get(cid, 0) + 1
            if scheme == "rr" and N - fr - 1 > 0:
                bound = 1 + -(-fr // (N - fr - 1))
                assert max(per.values()) <= bound
            helpers = [cid for cid, _, k in ts if k == 2]
            assert all(h > fr for h in helpers)
            if scheme == "nf":
                assert helpers == sorted(helpers)
                if helpers:
                    last = helpers[-1]
                    for d in range(fr + 1, last):
                        assert helpers.count(d) == qlen[d] - taken[d], (it, d)
                    assert len(helpers) == min(fr, sum(qlen[d] - taken[d] for d in range(fr + 1, N)))
            for h in helpers:
                taken[h] += 1
            assert all(taken[d] <= qlen[d] for d in range(N))


@pytest.mark.parametrize("seed", range(8))
def test_simulate_pm_tree(seed):
    """Faithful PM (Eq. 2) on random DFAs and chunkings:
    * results equal the sequential run;
    * ceil(log2 N) merge rounds;
    * stage-2 recoveries = chunks whose true start is not among their k speculated
      states (Eq. 2: P_i^PM = 1 - accu_i^spec-k), counted by brute force from the
      sequential run's chunk ends and the lookback ranking (both pinned above)."""
    rng = random.Random(seed * 31 + 7)
    n, ns = rng.randint(1, 40), rng.randint(1, 6)
    t, s, a = gen.dfa_random(seed + 61, n, ns)
    data = gen.workload(f"rand:{n}:{ns}:{seed}", length=rng.randint(0, 20000), seed=seed + 5).host()
    perm, inv, _, tt, acc = oracle.transform(t, a)
    for B in (16, 48, 256):
        for k in (1, 2, 4):
            r = oracle.run(t, s, a, data, B)
            o = oracle.simulate_pm_tree(t, s, a, data, B, k=k)
            N = oracle.nchunks(len(data), B)
            assert o["status"] == 0
            assert o["final_state"] == r["final"] and o["accept_count"] == r["count"]
            assert (o["chunk_end"] == r["chunk_end"]).all()
            assert o["pm_levels"] == (max(N - 1, 0)).bit_length()
            miss = 0
            for c in range(1, N):
                qs, _ = oracle.lookback(tt, n, data[c * B - 2:c * B], K=16)
                miss += int(perm[r["chunk_end"][c - 1]]) not in [int(q) for q in qs[:k]]
            assert o["pm_recoveries"] == miss
            assert o["pm_reread_bytes"] <= miss * B


def test_simulate_pm_tree_special_cases():
    """div7 (every lookback image is all 7 states): with k = 7 every path merges
    (no invalid mark, one stage-2 jump, no recovery); a one-state DFA likewise."""
    w = gen.workload("c1", length=1 << 14)
    d = w.host()
    o = oracle.simulate_pm_tree(w.table, w.start, w.accept, d, 64, k=7)
    assert o["pm_invalid_marks"] == 0 and o["pm_jumps"] == 1 and o["pm_recoveries"] == 0
    o4 = oracle.simulate_pm_tree(w.table, w.start, w.accept, d, 64, k=4)
    assert o4["pm_invalid_marks"] > 0 and o4["pm_recoveries"] > 0
    assert o4["final_state"] == o["final_state"] and o4["accept_count"] == o["accept_count"]
    t1 = np.zeros((1, 3), np.uint32)
    d1 = np.array([0, 1, 2] * 300, np.uint8)
    o = oracle.simulate_pm_tree(t1, 0, np.array([1], np.uint8), d1, 16, k=4)
    assert o["pm_recoveries"] == 0 and o["pm_jumps"] == 1 and o["accept_count"] == len(d1)


def test_simulate_invalid_symbol():
    t, s, a = gen.dfa_div7()
    data = np.array([1, 0, 1] * 100 + [3] + [1] * 50, np.uint8)
    for scheme in ("seq", "sre", "rr", "nf", "pm", "cse"):
        o = oracle.simulate(t, s, a, data, 16, scheme=scheme)
        assert o["status"] == oracle.OR_ESYMBOL


# ----------------------------------------------------------- features -------
def test_features_closed_forms():
    w = gen.workload("c1", length=1 << 16)
    f = oracle.features(w.table, w.start, w.accept, w.host(), B=4096)
    assert f["uniq10"] == 7.0  # delta*(., 10 bits) is a bijection for div7
    assert 0.0 <= f["acc1"] <= f["acck"] <= 1.0
    assert oracle.select(f, 7) == oracle.ENUM
    w = gen.workload("c2", length=1 << 18)
    f = oracle.features(w.table, w.start, w.accept, w.host(), B=4096)
    assert f["uniq10"] <= 4.0 and oracle.select(f, w.nstates) == oracle.SRE
    w = gen.workload("c3", length=1 << 18)
    data = w.host()
    f = oracle.features(w.table, w.start, w.accept, data, B=4096)
    # product structure: |image| = |AC image| x |counter image|; the Z16 counter
    # keeps all 16 values unless a reset byte falls in the 10-symbol window
    tac, _, _ = gen.dfa_ac(*w.keep)
    L = len(data)
    tot = 0
    for j in range(64):
        p = j * (L - 10) // 64
        win = data[p:p + 10]
        img = set(range(tac.shape[0]))
        for ch in win:
            img = {int(tac[q, ch]) for q in img}
        tot += len(img) * (1 if gen.RESET_BYTE in win else 16)
    assert f["uniq10"] == tot / 64 and f["uniq10"] > 8
    # spec-4 adds ~0.2 accuracy: helpers would mostly miss -> SRE (R19b)
    assert f["acck"] - f["acc1"] < 0.5 and oracle.select(f, w.nstates) == oracle.SRE
    g = dict(f, acc1=0.1, acck=0.7)  # helpers catch most mispredictions -> RR / NF by sensitivity
    assert oracle.select(dict(g, sens=0.0), w.nstates) == oracle.RR
    assert oracle.select(dict(g, sens=0.3), w.nstates) == oracle.NF


def test_features_accuracy_bruteforce():
    t, s, a = gen.dfa_random(5, 12, 3)
    data = gen.workload("rand:12:3:5", length=4000).host()
    B = 64
    perm, inv, _, tt, acc = oracle.transform(t, a)
    r = oracle.run(t, s, a, data, B)
    hit1 = hitk = 0
    N = oracle.nchunks(len(data), B)
    for c in range(1, N):
        qs, _ = oracle.lookback(tt, 12, data[c * B - 2:c * B], K=16)
        truth = int(perm[r["chunk_end"][c - 1]])
        hit1 += int(qs[0] == truth)
        hitk += int(truth in list(qs[:4]))
    f = oracle.features(t, s, a, data, B=B)
    assert f["acc1"] == pytest.approx(hit1 / (N - 1)) and f["acck"] == pytest.approx(hitk / (N - 1))


# ------------------------------------------------ input sensitivity (sens) --
def _div7_designed_bits(residues, B, rng):
    """Bits of a div7 stream whose prefix value at every chunk boundary c*B (c >= 1)
    is residues[c] mod 7: the first B-3 bits of a chunk are random, its last 3 bits
    are chosen so that value(prefix) = 8*v + b = v + b (mod 7) hits the target."""
    N = len(residues) - 1  # residues[0..N]: entry c is the target at boundary c*B
    bits = np.zeros(N * B, np.uint8)
    v = 0
    for c in range(N):
        body = rng.integers(0, 2, B - 3)
        for b in body:
            v = (2 * v + int(b)) % 7
        bits[c * B:c * B + B - 3] = body
        target = residues[c + 1] if c + 1 < N else int(rng.integers(0, 7))
        last = (target - v) % 7  # 0..6 < 8: three bits
        bits[c * B + B - 3:c * B + B] = [(last >> 2) & 1, (last >> 1) & 1, last & 1]
        v = (v + last) % 7
    return bits


@pytest.mark.parametrize("seed", [0, 1, 2, 3])
def test_features_sens_div7_designed(seed):
    """Input sensitivity pinned by construction (R19: max - min of the per-segment
    spec-1 accuracy over 8 equal segments of the profile chunks c >= 1).

    div7's lookback-2 image is every state at multiplicity 1 (a bijection), its static
    in-degrees all equal 2 so the transformation is the identity, hence QS = [0..6] and
    spec-1 hits chunk c iff the big-integer value of the prefix before it is = 0 (mod 7),
    spec-4 iff it is < 4.  The residues are drawn here, per segment, so the expected
    acc1 / acc4 / sens come from the design, not from the oracle."""
    rng = np.random.default_rng(seed)
    B, m = 16, 6 + seed          # N - 1 = 8m profile chunks: 8 equal segments of m chunks
    N = 8 * m + 1
    p_hit = np.roll([0.8, 0.2, 0.7, 0.3, 0.9, 0.1, 0.6, 0.4], seed)  # high / low alternate
    res = [0] * (N + 1)
    for c in range(1, N):
        seg = (c - 1) // m
        res[c] = 0 if rng.random() < p_hit[seg] else int(rng.integers(1, 7))
    # segment edges carry the opposite outcome of their neighbour's majority so that a
    # segment formula off by one chunk changes some segment's accuracy
    for j in range(8):
        first, last = 1 + j * m, (j + 1) * m
        res[first] = 0 if p_hit[j] >= 0.5 else 3
        res[last] = 0 if p_hit[j] >= 0.5 else 5
    bits = _div7_designed_bits(res, B, rng)
    # the construction really produces those residues (Python big integers)
    for c in range(1, N):
        assert int("".join(map(str, bits[:c * B])), 2) % 7 == res[c]
    seg_acc = []
    for j in range(8):
        cs = range(1 + j * m, 1 + (j + 1) * m)
        seg_acc.append(sum(res[c] == 0 for c in cs) / m)
    acc1 = sum(res[c] == 0 for c in range(1, N)) / (N - 1)
    acc4 = sum(res[c] < 4 for c in range(1, N)) / (N - 1)
    w = gen.workload("c1")
    f = oracle.features(w.table, w.start, w.accept, bits, B=B, k=4)
    assert f["acc1"] == pytest.approx(acc1, abs=1e-12)
    assert f["acck"] == pytest.approx(acc4, abs=1e-12)
    assert f["sens"] == pytest.approx(max(seg_acc) - min(seg_acc), abs=1e-12)
    assert f["sens"] > 0.5


def test_features_sens_c3s_region_boundary():
    """Input sensitivity on the input-sensitive C3 stream: a profile slice whose first
    half lies in a normal region and second half in a vowel-free region.
    Expected per-segment accuracy by brute force: true chunk starts from the sequential
    run (pinned above), predictions from the lookback ranking (pinned above), 8 equal
    segments of the N - 1 = 64 profile chunks."""
    w = gen.workload("c3s")
    B, N = 4096, 65
    region = 1 << 26
    lo = region - 33 * B         # chunks 1..32 normal, 33..64 vowel-free
    data = w.host(lo, N * B)
    perm, inv, _, tt, acc = oracle.transform(w.table, w.accept)
    r = oracle.run(w.table, w.start, w.accept, data, B)
    m = (N - 1) // 8
    seg = [0] * 8
    for c in range(1, N):
        qs, _ = oracle.lookback(tt, w.nstates, data[c * B - 2:c * B], K=16)
        seg[(c - 1) // m] += int(qs[0] == perm[r["chunk_end"][c - 1]])
    seg_acc = [s / m for s in seg]
    f = oracle.features(w.table, w.start, w.accept, data, B=B)
    assert f["sens"] == pytest.approx(max(seg_acc) - min(seg_acc), abs=1e-12)
    assert f["acc1"] == pytest.approx(sum(seg) / (N - 1), abs=1e-12)
    assert max(seg_acc[4:]) > min(seg_acc[:4]) and f["sens"] >= 0.2  # the regions really differ


def test_select_enum_bound_63_64():
    """R19: the ENUM leaf needs n <= 63 real states (n + poison = two map entries per lane)."""
    f = {"acc1": 0.0, "acck": 0.0, "sens": 0.0, "uniq10": 31.0}
    assert oracle.select(f, 31) == oracle.ENUM
    assert oracle.select(dict(f, uniq10=32.0), 32) == oracle.ENUM
    assert oracle.select(dict(f, uniq10=63.0), 63) == oracle.ENUM
    assert oracle.select(dict(f, uniq10=31.5), 63) == oracle.ENUM
    assert oracle.select(dict(f, uniq10=31.4), 63) != oracle.ENUM
    assert oracle.select(dict(f, uniq10=64.0), 64) != oracle.ENUM
    assert oracle.select(dict(f, uniq10=64.0), 64) == oracle.SRE  # acck - acc1 < 0.5 (R19b)


def test_run_stream_div7_closed_form():
    """The streamed oracle (blocks folded left) against the div7 closed
    form: every chunk end = prefix value mod 7, final accept = big integer mod 7 == 0."""
    w = gen.workload("c1", length=50000)
    bits = w.host()
    B = 16
    r = oracle.run_stream(w.table, w.start, w.accept, w.host, bits.size, B, block=4096, prefetch=2)
    res = div7_prefix_residues(bits)
    ends = np.minimum(np.arange(1, oracle.nchunks(bits.size, B) + 1) * B, bits.size) - 1
    assert (r["chunk_end"] == res[ends]).all()
    assert r["final"] == int("".join(map(str, bits)), 2) % 7
    assert r["accept"] == int(r["final"] == 0)
    assert r["count"] == int((res == 0).sum())


# ------------------------------------------- convergence lengths (R29) -------
def _conv_windows(length, wmax):
    return [j * 4096 for j in range(1, length) if j * 4096 + wmax <= length and 1 <= j % 32 <= 28]


def test_conv_lengths_reset_closed_form():
    """R29 on C3 (AC x Z16, the counter reset by '#'): the lookback image holds states with
    different counter values (vowels move every path's counter alike, so they cannot meet
    before a reset) and the reset byte sends every AC state to the root and every counter
    to 0 — so all paths meet exactly at the window's first '#': d = that offset + 1
    rounded up to 64 bytes, or 'never' when the window holds no '#'.  Windows whose
    2-byte lookback contains '#' (a counter already known) are left out of the pin."""
    w = gen.workload("c3", length=600 << 10, seed=7)
    data = w.host()
    wmax = 4096  # one '#' per 8 KiB block: about half the windows reach one
    assert all(gen.RESET_BYTE not in lit for lit in w.literals)
    d = oracle.conv_lengths(w.table, w.start, w.accept, data, wmax=wmax)
    wins = _conv_windows(len(data), wmax)
    assert len(d) == len(wins) > 100
    checked = reach = 0
    for p, dw in zip(wins, d):
        if gen.RESET_BYTE in bytes(data[p - 2:p]):
            continue
        seg = bytes(data[p:p + wmax])
        r = seg.find(bytes([gen.RESET_BYTE]))
        expect = 0xFFFFFFFF if r < 0 else -(-(r + 1) // 64) * 64
        assert int(dw) == expect, (p, r, int(dw))
        checked += 1
        reach += r >= 0
    assert checked > 100 and 0 < reach < checked


def test_conv_lengths_permutation_and_constant():
    """div7 (every symbol permutes the states: paths never meet) -> never; a DFA whose
    next state depends on the symbol only (lookback image = one state) -> 0."""
    t, s, a = gen.dfa_div7()
    rng = np.random.default_rng(3)
    bits = rng.integers(0, 2, 300 << 10).astype(np.uint8)
    d = oracle.conv_lengths(t, s, a, bits, wmax=8192)
    assert len(d) == len(_conv_windows(bits.size, 8192)) and (d == 0xFFFFFFFF).all()
    n, ns = 5, 8
    tc = np.tile((np.arange(ns) % n).astype(np.uint32), (n, 1))
    data = rng.integers(0, ns, 200 << 10).astype(np.uint8)
    d = oracle.conv_lengths(tc, 0, np.array([1, 0, 0, 0, 0], np.uint8), data, wmax=4096)
    assert len(d) > 0 and (d == 0).all()


def test_conv_lengths_two_state_merge_bruteforce():
    """A 3-state DFA where symbol 0 sends every state to 0 and other symbols permute
    states 1 <-> 2 (and fix 0): paths from distinct states meet at the first 0 symbol.
    Brute force per window: the image (from the 2 lookback symbols) and the first 0."""
    # row s: symbol 0 -> 0; symbol 1 -> swap 1/2 (0 stays 0); symbol 2 -> identity
    t = np.array([[0, 0, 0], [0, 2, 1], [0, 1, 2]], np.uint32)
    rng = np.random.default_rng(11)
    data = rng.choice(3, size=160 << 10, p=[0.0005, 0.4995, 0.5]).astype(np.uint8)
    d = oracle.conv_lengths(t, 0, np.array([1, 0, 0], np.uint8), data, wmax=8192)
    for p, dw in zip(_conv_windows(data.size, 8192), d):
        img = {int(t[int(t[q, data[p - 2]]), data[p - 1]]) for q in range(3)}
        if len(img) <= 1:
            assert dw == 0
            continue
        r = np.nonzero(data[p:p + 8192] == 0)[0]
        expect = 0xFFFFFFFF if r.size == 0 else -(-(int(r[0]) + 1) // 64) * 64
        assert int(dw) == expect


def test_select_chunk_rule():
    """R29's rule: the smallest W in {4, 8, 16} KiB with >= 3/4 of the windows converged
    within W and >= min_chunks chunks of W (W = 4 KiB always allowed); else 4 KiB."""
    never = 0xFFFFFFFF
    G = 1 << 30
    assert oracle.select_chunk([0] * 8, G, 113664) == 4096
    assert oracle.select_chunk([], G, 113664) == 4096
    assert oracle.select_chunk([never] * 8, G, 113664) == 4096
    d8 = [64, 4096, 5000, 8192, 8000, 7000, 6000, never]  # 2/8 within 4K, 7/8 within 8K
    assert oracle.select_chunk(d8, G, 113664) == 8192
    assert oracle.select_chunk(d8, G, 131073) == 4096        # 1 GiB / 8 KiB = 131072 chunks < 131073
    d16 = [64, 9000, 10000, 12000, 16384, 16000, 5000, never]  # 2/8 within 8K, 7/8 within 16K
    assert oracle.select_chunk(d16, 16 * G, 113664) == 16384
    assert oracle.select_chunk(d16, G, 113664) == 4096
    assert oracle.select_chunk([64, 64, 64, never], G, 113664) == 4096  # exactly 3/4 within 4K


def test_select_paper_tree_variant():
    """R19 without the B200 gate R19b (the paper's Fig. 6 as reconstructed): once ENUM, SRE
    (uniq10 <= 4) and PM are excluded, input sensitivity >= 0.2 -> NF, else RR; the default
    tree sends the same features to SRE while the spec-k gain stays below 0.5."""
    f = {"acc1": 0.2, "acck": 0.6, "sens": 0.3, "uniq10": 16.0}
    assert oracle.select(f, 816, paper_tree=True) == oracle.NF
    assert oracle.select(dict(f, sens=0.1), 816, paper_tree=True) == oracle.RR
    assert oracle.select(f, 816) == oracle.SRE
    assert oracle.select(dict(f, acck=0.75), 816) == oracle.NF  # gain >= 0.5: both trees agree
    assert oracle.select(dict(f, acck=0.95, acc1=0.7), 816, paper_tree=True) == oracle.PM
    assert oracle.select(dict(f, uniq10=3.0), 816, paper_tree=True) == oracle.SRE
    assert oracle.select(dict(f, uniq10=40.0), 63, paper_tree=True) == oracle.ENUM


def test_select_paper_tree_on_c3s_boundary():
    """The input-sensitive stream across a normal / vowel-free region boundary (features
    pinned by brute force above): the paper's tree picks NF."""
    w = gen.workload("c3s")
    B, N = 4096, 65
    data = w.host((1 << 26) - 33 * B, N * B)
    f = oracle.features(w.table, w.start, w.accept, data, B=B)
    assert f["sens"] >= 0.2
    assert oracle.select(f, w.nstates, paper_tree=True) == oracle.NF
