#!/usr/bin/env python3
"""Run timeline of one config (GSPEC_STAMPS=1): spec kernel, gap, verify kernel, and the
verify phase boundaries, median over 10 runs.  usage: GSPEC_STAMPS=1 python tools/timeline.py c2"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    import gen
    import paper_conf_ipps_wangwqw22_b200 as gs

    name = sys.argv[1] if len(sys.argv) > 1 else "c2"
    w = gen.workload(name)
    x = torch.empty(w.length, dtype=torch.uint8, device="cuda")
    w.device(x)
    prof = torch.empty(1 << 20, dtype=torch.uint8, device="cuda")
    w.device(prof, offset=w.length)
    fsm = gs.FSM.load(w.table, w.start, w.accept, profile=prof.cpu().numpy())
    scheme, _ = fsm.select_scheme(x[: 1 << 20])
    tl, ph, ev = [], [], []
    for i in range(13):
        r = fsm.run(x, scheme=scheme)
        if i >= 3:
            tl.append(fsm.timeline())
            ph.append(fsm.phase_times())
            ev.append((r.stats["ms_spec"] * 1e3, r.stats["ms_verify"] * 1e3))
    tl = np.median(np.array(tl), axis=0)
    print(f"{name} scheme={scheme} rounds={r.stats['rounds']} tasks={r.stats['tasks_total']}")
    print("timeline us: spec %.1f  gap %.1f  verify %.1f" % tuple(tl))
    print("events us: spec %.1f  verify %.1f" % tuple(np.median(np.array(ev), axis=0)))
    n = min(len(p) for p in ph)
    print("verify phases us:", np.round(np.median(np.array([p[:n] for p in ph]), axis=0), 1).tolist())


if __name__ == "__main__":
    main()
