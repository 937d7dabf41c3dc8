import sys
sys.path.insert(0, ".")
import torch
import gen
import oracle
import paper_conf_ipps_wangwqw22_b200 as gs

w4 = gen.workload("c3", length=4 << 20)
wt = gen.workload("c3", length=(3 << 20) + 555)
d4, dt = w4.host(), wt.host()
fsm = gs.FSM.load(w4.table, w4.start, w4.accept)
for scheme, L in [("sre", 3), ("sre", 16), ("rr", 8), ("nf", 5), ("pm", 16), ("cse", 8), ("pm_tree", 4)]:
    for d, B in ((d4, 4096), (dt, 2048)):
        try:
            r = fsm.run(torch.from_numpy(d).cuda(), scheme=scheme, chunk_bytes=B, lookback=L)
            print(scheme, L, len(d), "ok", r.final_state == oracle.run(w4.table, w4.start, w4.accept, d, B)["final"], flush=True)
        except Exception as e:
            print(scheme, L, len(d), "ERR", e, flush=True)
