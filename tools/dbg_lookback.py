import sys
sys.path.insert(0, ".")
import numpy as np
import torch
import gen
import oracle
import paper_conf_ipps_wangwqw22_b200 as gs

for name, length, B, scheme, L in [("c3", 4 << 20, 4096, "pm_tree", 4), ("c3", (3 << 20) + 555, 2048, "pm_tree", 4),
                                   ("c3", (3 << 20) + 555, 2048, "sre", 3)]:
    w = gen.workload(name, length=length)
    d = w.host()
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    try:
        r = fsm.run(torch.from_numpy(d).cuda(), scheme=scheme, chunk_bytes=B, lookback=L)
        ref = oracle.run(w.table, w.start, w.accept, d, B)
        print(name, length, scheme, L, "ok", r.final_state == ref["final"], r.accept_count == ref["count"], flush=True)
    except Exception as e:
        print(name, length, scheme, L, "ERR", e, flush=True)
rng = np.random.default_rng(5)
n = 100
t = np.stack([rng.permutation(n) for _ in range(3)], axis=1).astype(np.uint32)
a = (rng.random(n) < 0.5).astype(np.uint8)
data = np.random.default_rng(5).integers(0, 3, 20 * 4096).astype(np.uint8)
fsm = gs.FSM.load(t, 0, a)
r = fsm.run(torch.from_numpy(data).cuda(), scheme="sre", chunk_bytes=1024, lookback=8)
print("wide ok", r.final_state == oracle.run(t, 0, a, data, 1024)["final"], flush=True)
