#!/usr/bin/env python3
"""Throughput of stream-level batching (fsm_run_batch) on a serving-like mix:
many independent streams with lengths drawn log-uniformly in [64 B, 64 KiB], packed
back to back (unaligned), total ~1 GiB of a config's synthetic text.  Prints one JSON
line per config: GB/s over all stream bytes (device time, inputs resident), streams/s,
recoveries, and the single-stream fsm_run rate over the same bytes for context.

usage: python tools/bench_batch.py [c2 c4 ...] [--gib 1] [--reps 5]"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("configs", nargs="*", default=["c2", "c4"])
    ap.add_argument("--gib", type=float, default=1.0)
    ap.add_argument("--reps", type=int, default=5)
    args = ap.parse_args()
    import torch

    import gen
    import paper_conf_ipps_wangwqw22_b200 as gs

    for name in args.configs:
        total = int(args.gib * (1 << 30))
        w = gen.workload(name, length=total)
        x = torch.empty(total, dtype=torch.uint8, device="cuda")
        w.device(x)
        rng = np.random.default_rng(7)
        lens = np.exp(rng.uniform(np.log(64), np.log(65536), size=total // 4096 * 2)).astype(np.int64)
        cs = np.cumsum(lens)
        ns = int(np.searchsorted(cs, total))
        offs = np.concatenate([[0], cs[:ns]]).astype(np.uint64)
        nbytes = int(offs[-1])
        fsm = gs.FSM.load(w.table, w.start, w.accept)
        best = None
        for _ in range(args.reps + 1):
            fin, cnt, _, st = fsm.run_batch(x, offs, chunk_bytes=4096)
            if best is None or st["ms"] < best["ms"]:
                best = st
        r = None
        for _ in range(3):
            r = fsm.run(x[:nbytes], scheme="sre")
        single_ms = r.stats["ms_spec"] + r.stats["ms_verify"]
        print(json.dumps({"config": name, "streams": ns, "bytes": nbytes, "chunks": best["nchunks"],
                          "ms": round(best["ms"], 4), "GB/s": round(nbytes / best["ms"] / 1e6, 1),
                          "Mstreams/s": round(ns / best["ms"] / 1e3, 2), "recoveries": best["recoveries"],
                          "single_stream_GB/s": round(nbytes / single_ms / 1e6, 1)}), flush=True)
        fsm.close()
        del x


if __name__ == "__main__":
    main()
