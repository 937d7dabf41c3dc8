"""FSM-level batching throughput (fsm_run_multi): P (DFA, stream) pairs in one
call — the C2 / C4 DFAs each over its own 1 MiB stream — vs running the same pairs one by one
with fsm_run.  usage: python tools/bench_multi.py [pairs] [MiB per stream]"""
import json
import sys
import time

sys.path.insert(0, '.')
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_wangwqw22_b200 as gs  # noqa: E402

P = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
L = (int(sys.argv[2]) if len(sys.argv) > 2 else 1) << 20
for cfg in ("c2", "c4"):
    w = gen.workload(cfg, length=P * L)
    x = torch.empty(P * L, dtype=torch.uint8, device="cuda")
    w.device(x)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    xs = [x[i * L:(i + 1) * L] for i in range(P)]
    fsms = [fsm] * P
    for _ in range(2):
        fin, cnt, st = gs.run_multi(fsms, xs)
    best = min(gs.run_multi(fsms, xs)[2]["ms"] for _ in range(3))
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    one = [fsm.run(xs[i], scheme="sre") for i in range(min(P, 64))]
    torch.cuda.synchronize()
    per_run = (time.perf_counter() - t0) / len(one)
    ok = all(one[i].final_state == fin[i] and one[i].accept_count == cnt[i] for i in range(len(one)))
    print(json.dumps({"config": cfg, "pairs": P, "bytes_per_stream": L, "multi_ms": round(best, 3),
                      "multi_GB/s": round(P * L / best / 1e6, 1), "rewalks": st["rewalks"],
                      "one_by_one_ms_per_pair": round(per_run * 1e3, 3),
                      "one_by_one_GB/s": round(L / per_run / 1e9, 1), "agree": ok}))
    fsm.close()
    del x, xs
    torch.cuda.empty_cache()
