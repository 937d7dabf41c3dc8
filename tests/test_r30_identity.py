"""R30: the arithmetic the checkpointed dense rounds rely on, checked with the
oracle's sequential walk (Alg. 1 FSM_PROCESSING) — no GPU.

A recovery task for chunk c from start s may stop at the first checkpoint p where its state
equals the round-0 path's state (start r): by determinism (one next state per (state,
symbol)) the two walks agree from p on, so

    end(s)   = end(r)
    count(s) = count_s[0, p) + (count(r) - count_r[0, p)).

Both sides here are plain oracle.run calls on prefixes and on the whole chunk, so a wrong
sign or a missing term in the identity fails, and so would a checkpoint taken one step off.
"""
import numpy as np
import pytest

import gen
import oracle


def _prefix(w, s, data, p):
    r = oracle.run(w.table, s, w.accept, data[:p], max(p, 1)) if p else {"final": s, "count": 0}
    return int(r["final"]), int(r["count"])


@pytest.mark.parametrize("name,B,cp", [("c3", 8192, 512), ("c3", 4096, 64), ("c2", 4096, 512), ("c4", 4096, 256)])
def test_checkpoint_identity(name, B, cp):
    w = gen.workload(name, length=8 * B)
    data_all = w.host()
    rng = np.random.default_rng(30)
    hits = 0
    for c in range(1, 8):
        data = data_all[c * B:(c + 1) * B]
        r = int(rng.integers(w.nstates))  # the round-0 path's start
        s = int(rng.integers(w.nstates))  # the task's start
        full_r = oracle.run(w.table, r, w.accept, data, B)
        full_s = oracle.run(w.table, s, w.accept, data, B)
        met = None
        for p in range(cp, B, cp):
            qs, cs = _prefix(w, s, data, p)
            qr, cr = _prefix(w, r, data, p)
            if qs == qr:
                met = p
                assert int(full_s["final"]) == int(full_r["final"])
                assert int(full_s["count"]) == cs + (int(full_r["count"]) - cr)
                break
        if met is not None:
            hits += 1
            # determinism: once met, the paths stay together at every later checkpoint
            for p in range(met, B, cp):
                assert _prefix(w, s, data, p)[0] == _prefix(w, r, data, p)[0]
    if name in ("c2", "c4"):
        assert hits == 7  # AC automata: any two starts meet within a few symbols of text
    if name == "c3":
        assert hits >= 1  # the counter part meets at the chunk's reset byte
