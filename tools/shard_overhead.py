"""Per-step cost of the multi-GPU shard path on ONE GPU (no collective): fsm_shard_map
of a rank >= 1 shard (lookback image + fusion check + pipeline + map) and fsm_shard_finish
(compose + fix-up + readback) for G ranks' maps, vs a plain fsm_run of the same bytes.
usage: python tools/shard_overhead.py [c2] [G]"""
import ctypes
import sys
import time

sys.path.insert(0, '.')
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ipps_wangwqw22_b200 as gs  # noqa: E402
from paper_conf_ipps_wangwqw22_b200 import _lib, _run_opts, fsm_result, _check  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c2"
G = int(sys.argv[2]) if len(sys.argv) > 2 else 8
w = gen.workload(cfg)
L = w.length
x = torch.empty(L, dtype=torch.uint8, device="cuda")
w.device(x, offset=L)  # rank 1's shard
lb = torch.empty(2, dtype=torch.uint8, device="cuda")
w.device(lb, offset=L - 2)
fsm = gs.FSM.load(w.table, w.start, w.accept)
o = _run_opts("sre", 4096)
mb = fsm.map_bytes()
m = torch.empty(mb, dtype=torch.uint8, device="cuda")
maps = torch.empty(G * mb, dtype=torch.uint8, device="cuda")
ce = torch.empty(L // 4096, dtype=torch.int32, device="cuda")


def t_run(fn, reps=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps):
        fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / reps * 1e3


def plain():
    fsm.run(x, scheme="sre")


def smap():
    _check(_lib.fsm_shard_map(fsm.handle, x.data_ptr(), L, lb.data_ptr(), 2, ctypes.byref(o), m.data_ptr(),
                              ce.data_ptr()), "map")


def smap_rank0():
    _check(_lib.fsm_shard_map(fsm.handle, x.data_ptr(), L, None, 0, ctypes.byref(o), m.data_ptr(), ce.data_ptr()),
           "map0")


def step_rank0():
    smap_rank0()
    r = fsm_result()  # one rank's map (the compose over G maps is G table lookups)
    _check(_lib.fsm_shard_finish(fsm.handle, m.data_ptr(), 1, 0, ctypes.byref(o), ce.data_ptr(), ctypes.byref(r)),
           "finish")


print({"config": cfg, "plain_fsm_run_ms": round(t_run(plain), 4), "shard_map_rank>=1_ms": round(t_run(smap), 4),
       "shard_map_rank0_ms": round(t_run(smap_rank0), 4), "rank0_map+finish_ms": round(t_run(step_rank0), 4)})
