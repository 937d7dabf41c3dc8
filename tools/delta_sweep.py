#!/usr/bin/env python3
"""C4 spec-kernel time vs the u16d hot-row count H (GSPEC_DELTA_H) and smem budget.
usage: python tools/delta_sweep.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    import gen
    import paper_conf_ipps_wangwqw22_b200 as gs

    w = gen.workload("c4")
    x = torch.empty(w.length, dtype=torch.uint8, device="cuda")
    w.device(x)
    for budget, H in ((0, 0), (0, 600), (160 * 1024, 800), (160 * 1024, 1000), (96 * 1024, 0), (2 ** 17 + 2 ** 15, 0)):
        os.environ["GSPEC_DELTA_H"] = str(H)
        fsm = gs.FSM.load(w.table, w.start, w.accept, smem_budget=budget)
        tr = fsm.transform()
        fsm.select_scheme(x[: 1 << 20])
        ts = []
        for _ in range(6):
            r = fsm.run(x, scheme="sre")
            ts.append(r.stats["ms_spec"])
        print(f"budget={budget} H_req={H} mode={tr['mode']} H={tr['hot_rows']} spec_ms={sorted(ts)[3]:.3f} "
              f"verify_ms={r.stats['ms_verify']:.3f}", flush=True)
        fsm.close()


if __name__ == "__main__":
    main()
