"""Debug: C2 on a 16 GiB stream at several chunk sizes — per-run stats (spec / verify ms, rounds, tasks, launches)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import gen
import paper_conf_ipps_wangwqw22_b200 as gs

L = int(sys.argv[1]) if len(sys.argv) > 1 else 16 << 30
name = sys.argv[2] if len(sys.argv) > 2 else "c2"
w = gen.workload(name, length=L)
x = torch.empty(L, dtype=torch.uint8, device="cuda")
w.device(x)
fsm = gs.FSM.load(w.table, w.start, w.accept)
sel = fsm.select_scheme(x, stream_len=L)
print("select", sel[0], sel[1], flush=True)
for B in (4096, 8192):
    for i in range(4):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        r = fsm.run(x, scheme="sre", chunk_bytes=B)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        st = r.stats
        print(B, i, round(dt * 1e3, 3), {k: st[k] for k in ("ms_spec", "ms_verify", "rounds", "tasks_total", "tasks_sre",
                                                         "verify_checks", "verify_matches", "kernel_launches")},
              "phases", [round(float(v), 1) for v in fsm.phase_times()], flush=True)
