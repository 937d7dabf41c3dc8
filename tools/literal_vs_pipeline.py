"""Paper-literal single-CTA kernels (Alg. 3 SRE, Alg. 4 RR, Alg. 5 NF) vs the
batched pipeline and the faithful PM (f2), on the paper's setting: a 10 MiB stream split
into N = 256 chunks.
usage: python tools/literal_vs_pipeline.py [configs...]"""
import json
import sys

sys.path.insert(0, '.')
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_wangwqw22_b200 as gs  # noqa: E402

L = 10 << 20
B = L // 256
for cfg in (sys.argv[1:] or ["c2", "c3", "c4"]):
    w = gen.workload(cfg, length=L)
    x = torch.empty(L, dtype=torch.uint8, device="cuda")
    w.device(x)
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    lit = [fsm.run_literal(x, chunk_bytes=B) for _ in range(3)]
    pip = [fsm.run(x, scheme="sre", chunk_bytes=B) for _ in range(5)]
    tl = min(r.stats["ms_verify"] for r in lit)
    lit_rr = [fsm.run_literal(x, chunk_bytes=B, scheme="rr") for _ in range(3)]
    lit_nf = [fsm.run_literal(x, chunk_bytes=B, scheme="nf") for _ in range(3)]
    pmt = [fsm.run(x, scheme="pm_tree", chunk_bytes=B) for _ in range(3)]
    for r in lit_rr + lit_nf + pmt:
        assert (r.final_state, r.accept_count) == (lit[-1].final_state, lit[-1].accept_count)
    tp = min(r.stats["ms_spec"] + r.stats["ms_verify"] for r in pip)
    p4 = [fsm.run(x, scheme="sre", chunk_bytes=4096) for _ in range(5)]  # the pipeline's own chunking
    t4 = min(r.stats["ms_spec"] + r.stats["ms_verify"] for r in p4)
    assert (lit[-1].final_state, lit[-1].accept_count) == (pip[-1].final_state, pip[-1].accept_count)
    print(json.dumps({"config": cfg, "bytes": L, "chunks": 256, "chunk_bytes": B,
                      "literal_ms": round(tl, 3), "literal_rounds": lit[-1].stats["rounds"],
                      "literal_tasks": lit[-1].stats["tasks_total"],
                      "literal_rr_ms": round(min(r.stats["ms_verify"] for r in lit_rr), 3),
                      "literal_rr_helpers": lit_rr[-1].stats["tasks_helper"],
                      "literal_nf_ms": round(min(r.stats["ms_verify"] for r in lit_nf), 3),
                      "literal_nf_helpers": lit_nf[-1].stats["tasks_helper"],
                      "pm_tree_ms": round(min(r.stats["ms_spec"] + r.stats["ms_verify"] for r in pmt), 3),
                      "pm_tree_recoveries": pmt[-1].stats["tasks_mustdo"],
                      "pipeline_sre_ms": round(tp, 3), "pipeline_rounds": pip[-1].stats["rounds"],
                      "pipeline_tasks": pip[-1].stats["tasks_total"], "speedup": round(tl / tp, 2),
                      "pipeline_sre_4KiB_chunks_ms": round(t4, 3), "speedup_4KiB": round(tl / t4, 2)}))
    fsm.close()
