"""Record-level invariants of the hierarchical store (GPU): every live record
of every chunk is a true walk of that chunk (start -> end, accepts), checked
against the oracle's enumeration — so recovery tasks, helpers and
path fusion never store a wrong record.  Memoized RR / NF helper records (R28)
that no verification matched hold their start only."""
import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.mark.parametrize("name,length,B,scheme,seed", [
    ("rand:218:242:4", 176279, 16, "rr", 4), ("rand:218:242:4", 176279, 16, "nf", 4),
    ("rand:218:242:4", 176279, 16, "sre", 4), ("c3", 1 << 20, 4096, "nf", None),
    ("c3", 1 << 20, 4096, "rr", None), ("c3", 1 << 20, 4096, "pm", None), ("c2", 1 << 21, 4096, "sre", None)])
def test_every_live_record_is_a_true_walk(name, length, B, scheme, seed):
    import paper_conf_ipps_wangwqw22_b200 as gs

    w = gen.workload(name, length=length, seed=seed)
    data = w.host()
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    res = fsm.run(torch.from_numpy(data).cuda(), scheme=scheme, chunk_bytes=B)
    N = res.nchunks
    rec = fsm.records(N)
    perm, inv, _, tt, acc = oracle.transform(w.table, w.accept)
    bad, pending, walked = [], 0, 0
    for c in range(N):
        chunk = data[c * B:(c + 1) * B]
        M, C = oracle.enum(tt, acc, chunk)
        slots = list(range(min(rec["n_end"][c], 16))) + [16 + j for j in range(min(rec["n_oth"][c], 16))]
        for s in slots:
            st, en, cn = rec["start"][s, c], rec["end"][s, c], rec["cnt"][s, c]
            if s >= 16 and en == 0xFFFFFFFC:  # a memoized helper never matched (R28): start only
                pending += 1
                continue
            walked += s >= 16
            if M[st] != en or C[st] != cn:
                bad.append((c, s, int(st), int(en), int(M[st]), int(cn), int(C[st])))
    assert not bad, bad[:10]
    ref = oracle.run(w.table, w.start, w.accept, data, B)
    assert res.accept_count == ref["count"]
    if scheme in ("rr", "nf"):  # helper records: every walked one was needed (or helpers are eager)
        assert walked <= res.stats["helper_walks"] or res.stats["helper_walks"] == 0
        assert pending + walked <= res.stats["tasks_helper"]
