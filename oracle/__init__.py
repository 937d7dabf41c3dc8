"""TEST INFRASTRUCTURE ONLY — ctypes view of the plain-C oracle (oracle.c).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this.  The product package never does; it shares
no code with the oracle.  Every function cites PAPER.md (P:n = line n).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

OR_OK, OR_EINVAL, OR_ESYMBOL, OR_EUNSUPPORTED = 0, -1, -4, -6
SEQ, PM, SRE, RR, NF, ENUM, CSE = 1, 2, 3, 4, 5, 6, 7
SCHEME_IDS = {"seq": SEQ, "pm": PM, "sre": SRE, "rr": RR, "nf": NF, "enum": ENUM, "cse": CSE}

P = ctypes.c_void_p
U32, U64 = ctypes.c_uint32, ctypes.c_uint64


class SimResult(ctypes.Structure):
    _fields_ = [("final_state", U32), ("accept", U32), ("accept_count", U64), ("nchunks", U64),
                ("rounds", U32), ("tasks_total", U64), ("tasks_mustdo", U64), ("tasks_sre", U64),
                ("tasks_helper", U64), ("reread_bytes", U64), ("verify_checks", U64),
                ("verify_matches", U64), ("active_sum", U64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class Task(ctypes.Structure):
    _fields_ = [("round", U32), ("chunk", U32), ("start", U32), ("kind", U32)]


class PmStats(ctypes.Structure):
    _fields_ = [("levels", U32), ("merge_checks", U64), ("invalid_marks", U64), ("jumps", U64),
                ("recoveries", U64), ("reread_bytes", U64)]


class Features(ctypes.Structure):
    _fields_ = [("acc1", ctypes.c_double), ("acck", ctypes.c_double), ("sens", ctypes.c_double),
                ("uniq10", ctypes.c_double)]


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "liboracle.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `python build.py`")
        L = ctypes.CDLL(path)
        L.or_run.argtypes = [P, U32, U32, U32, P, P, U64, U32, P, P, P]
        L.or_transform.argtypes = [P, U32, U32, P, ctypes.c_int, P, U64, U32, P, P, P, P, P]
        L.or_lookback.argtypes = [P, U32, U32, P, U32, U32, P, P]
        L.or_lookback.restype = U32
        L.or_enum.argtypes = [P, U32, U32, P, P, U64, P, P]
        L.or_compose.argtypes = [U32, P, P, P, P, P, P]
        L.or_simulate.argtypes = [P, U32, U32, U32, P, P, P, U64, U32, ctypes.c_int, U32, U32, U32, U32, U32,
                                  P, ctypes.POINTER(SimResult), P, U64, P]
        L.or_lookback_long.argtypes = [P, U32, U32, P, U32, U32, P, P]
        L.or_lookback_long.restype = U32
        L.or_simulate_literal_sre.argtypes = [P, U32, U32, U32, P, P, P, U64, U32, U32, P,
                                              ctypes.POINTER(SimResult)]
        L.or_simulate_literal.argtypes = [P, U32, U32, U32, P, P, P, U64, U32, ctypes.c_int, U32, U32, P,
                                          ctypes.POINTER(SimResult), P, U64, P]
        L.or_simulate_pm_tree.argtypes = [P, U32, U32, U32, P, P, P, U64, U32, U32, U32, P,
                                          ctypes.POINTER(SimResult), ctypes.POINTER(PmStats)]
        L.or_features_compute.argtypes = [P, U32, U32, U32, P, P, U64, U32, U32, U32, ctypes.POINTER(Features)]
        L.or_select.argtypes = [ctypes.POINTER(Features), U32]
        L.or_select_variant.argtypes = [ctypes.POINTER(Features), U32, ctypes.c_int]
        L.or_conv_lengths.argtypes = [P, U32, U32, P, U64, U32, P]
        L.or_conv_lengths.restype = U32
        L.or_select_chunk.argtypes = [P, U32, U64, U64]
        L.or_select_chunk.restype = U32
        _LIB = L
    return _LIB


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


def nchunks(length: int, B: int) -> int:
    return (length + B - 1) // B


def run(table, start, accept, data, B=4096):
    """Alg. 1 FSM_PROCESSING. Returns dict(status, final, accept, count, chunk_end)."""
    t = _c(table, np.uint32)
    a = _c(accept, np.uint8)
    d = _c(data, np.uint8)
    n, ns = t.shape
    ce = np.zeros(max(1, nchunks(d.size, B)), np.uint32)
    fin, cnt = U32(0), U64(0)
    rc = lib().or_run(t.ctypes.data, n, ns, start, a.ctypes.data, d.ctypes.data, d.size, B, ce.ctypes.data,
                      ctypes.byref(fin), ctypes.byref(cnt))
    if rc != OR_OK:
        return {"status": rc}
    if d.size == 0:
        fin = U32(start)
    f = int(fin.value)
    return {"status": 0, "final": f, "accept": int(a[f]), "count": int(cnt.value),
            "chunk_end": ce[:nchunks(d.size, B)]}


def run_stream(table, start, accept, fill, length, B=4096, block=64 << 20, prefetch=2):
    """Alg. 1 FSM_PROCESSING over a stream too large for one host buffer
    (16 GiB in 64 MiB blocks).  Alg. 1 is a left fold over the input,
    so the walk is or_run block after block, each block starting from the previous
    block's final state; block is a multiple of B, so every chunk lies in one block.
    fill(offset, n) -> uint8 array of the stream's bytes [offset, offset + n), e.g. the
    host generator; the next `prefetch` blocks are generated in background threads.
    Returns the same dict as run()."""
    import concurrent.futures

    assert block % B == 0
    t = _c(table, np.uint32)
    a = _c(accept, np.uint8)
    n, ns = t.shape
    ce = np.zeros(max(1, nchunks(length, B)), np.uint32)
    s, total = int(start), 0
    offs = list(range(0, length, block))
    with concurrent.futures.ThreadPoolExecutor(max(1, prefetch)) as ex:
        futs = {}
        for i, off in enumerate(offs):
            for j in range(i, min(len(offs), i + prefetch + 1)):
                if j not in futs:
                    futs[j] = ex.submit(fill, offs[j], min(block, length - offs[j]))
            d = _c(futs.pop(i).result(), np.uint8)
            fin, cnt = U32(0), U64(0)
            rc = lib().or_run(t.ctypes.data, n, ns, s, a.ctypes.data, d.ctypes.data, d.size, B,
                              ce[off // B:].ctypes.data, ctypes.byref(fin), ctypes.byref(cnt))
            if rc != OR_OK:
                return {"status": rc}
            s = int(fin.value)
            total += int(cnt.value)
    return {"status": 0, "final": s, "accept": int(a[s]), "count": total, "chunk_end": ce[:nchunks(length, B)]}


def transform(table, accept, policy=0, profile=None, start=0):
    """Frequency-based transformation. Returns (perm[n+1], inv[n+1], freq[n], tt[n+1,ns], acc_t[n+1])."""
    t = _c(table, np.uint32)
    a = _c(accept, np.uint8)
    n, ns = t.shape
    perm = np.zeros(n + 1, np.uint32)
    inv = np.zeros(n + 1, np.uint32)
    freq = np.zeros(n, np.uint64)
    tt = np.zeros((n + 1, ns), np.uint32)
    acc = np.zeros(n + 1, np.uint8)
    prof = _c(profile if profile is not None else np.zeros(0, np.uint8), np.uint8)
    rc = lib().or_transform(t.ctypes.data, n, ns, a.ctypes.data, policy, prof.ctypes.data, prof.size, start,
                            perm.ctypes.data, inv.ctypes.data, freq.ctypes.data, tt.ctypes.data, acc.ctypes.data)
    assert rc == 0
    return perm, inv, freq, tt, acc


def lookback(t, nq, w, K=16):
    """All-state lookback over the real states 0..nq-1 of table t."""
    t = _c(t, np.uint32)
    w = _c(w, np.uint8)
    qs = np.zeros(max(1, K), np.uint32)
    ql = U32(0)
    img = lib().or_lookback(t.ctypes.data, nq, t.shape[1], w.ctypes.data, w.size, K, qs.ctypes.data,
                            ctypes.byref(ql))
    return qs[:ql.value].copy(), int(img)


def enum(table, accept, data):
    """Enumeration: (M[n], C[n]) or None on an invalid symbol."""
    t = _c(table, np.uint32)
    a = _c(accept, np.uint8)
    d = _c(data, np.uint8)
    n, ns = t.shape
    M = np.zeros(n, np.uint32)
    C = np.zeros(n, np.uint64)
    rc = lib().or_enum(t.ctypes.data, n, ns, a.ctypes.data, d.ctypes.data, d.size, M.ctypes.data, C.ctypes.data)
    return None if rc != 0 else (M, C)


def compose(M1, C1, M2, C2):
    n = len(M1)
    M = np.zeros(n, np.uint32)
    C = np.zeros(n, np.uint64)
    M1, C1, M2, C2 = _c(M1, np.uint32), _c(C1, np.uint64), _c(M2, np.uint32), _c(C2, np.uint64)
    lib().or_compose(n, M1.ctypes.data, C1.ctypes.data, M2.ctypes.data, C2.ctypes.data, M.ctypes.data, C.ctypes.data)
    return M, C


def lookback_long(t, nq, w, K=16):
    """Lookback over the len(w) in [2, 16] symbols w before a chunk (reading R25)."""
    t = _c(t, np.uint32)
    w = _c(w, np.uint8)
    qs = np.zeros(max(1, K), np.uint32)
    ql = U32(0)
    img = lib().or_lookback_long(t.ctypes.data, nq, t.shape[1], w.ctypes.data, w.size, K, qs.ctypes.data,
                                 ctypes.byref(ql))
    return qs[:ql.value].copy(), int(img)


def simulate(table, start, accept, data, B=4096, scheme="sre", spec_k=None, qs_cap=16, vr_end=16, vr_oth=16,
             policy=0, max_tasks=0, lookback=2):
    """Round semantics of Alg. 2-5. Works on the transformed DFA.
    spec_k: round-0 paths per chunk for PM (default 4) and CSE (default 8)."""
    if spec_k is None:
        spec_k = 8 if scheme == "cse" else 4
    perm, inv, _, tt, acc = transform(table, accept, policy, data if policy == 1 else None, start)
    t = _c(table, np.uint32)
    n, ns = t.shape
    d = _c(data, np.uint8)
    ce = np.zeros(max(1, nchunks(d.size, B)), np.uint32)
    res = SimResult()
    tasks = (Task * max(1, max_tasks))()
    nt = U64(0)
    rc = lib().or_simulate(tt.ctypes.data, n, ns, int(perm[start]), acc.ctypes.data, inv.ctypes.data,
                           d.ctypes.data, d.size, B, SCHEME_IDS[scheme], spec_k, qs_cap, lookback, vr_end, vr_oth,
                           ce.ctypes.data, ctypes.byref(res), tasks, max_tasks, ctypes.byref(nt))
    out = res.as_dict()
    out["status"] = rc
    out["chunk_end"] = ce[:nchunks(d.size, B)]
    out["tasks"] = [(tasks[i].round, tasks[i].chunk, tasks[i].start, tasks[i].kind)
                    for i in range(min(nt.value, max_tasks))]
    out["ntasks"] = nt.value
    out["perm"] = perm
    return out


def simulate_literal_sre(table, start, accept, data, B=4096, vr_cap=16, policy=0):
    """Paper-literal SRE: Alg. 2 L2-6 then Alg. 3 verbatim, N iterations."""
    perm, inv, _, tt, acc = transform(table, accept, policy, data if policy == 1 else None, start)
    t = _c(table, np.uint32)
    n, ns = t.shape
    d = _c(data, np.uint8)
    ce = np.zeros(max(1, nchunks(d.size, B)), np.uint32)
    res = SimResult()
    rc = lib().or_simulate_literal_sre(tt.ctypes.data, n, ns, int(perm[start]), acc.ctypes.data, inv.ctypes.data,
                                       d.ctypes.data, d.size, B, vr_cap, ce.ctypes.data, ctypes.byref(res))
    out = res.as_dict()
    out["status"] = rc
    out["chunk_end"] = ce[:nchunks(d.size, B)]
    return out


def simulate_literal(table, start, accept, data, B=4096, scheme="rr", qs_cap=16, vr_cap=16, policy=0,
                     max_tasks=0):
    """Paper-literal SRE / RR / NF (Alg. 3 / 4 / 5 verbatim, N iterations)."""
    perm, inv, _, tt, acc = transform(table, accept, policy, data if policy == 1 else None, start)
    t = _c(table, np.uint32)
    n, ns = t.shape
    d = _c(data, np.uint8)
    ce = np.zeros(max(1, nchunks(d.size, B)), np.uint32)
    res = SimResult()
    tasks = (Task * max(1, max_tasks))()
    nt = U64(0)
    rc = lib().or_simulate_literal(tt.ctypes.data, n, ns, int(perm[start]), acc.ctypes.data, inv.ctypes.data,
                                   d.ctypes.data, d.size, B, SCHEME_IDS[scheme], qs_cap, vr_cap, ce.ctypes.data,
                                   ctypes.byref(res), tasks, max_tasks, ctypes.byref(nt))
    out = res.as_dict()
    out["status"] = rc
    out["chunk_end"] = ce[:nchunks(d.size, B)]
    out["tasks"] = [(tasks[i].round, tasks[i].chunk, tasks[i].start, tasks[i].kind)
                    for i in range(min(nt.value, max_tasks))]
    out["perm"] = perm
    return out


def simulate_pm_tree(table, start, accept, data, B=4096, k=4, qs_cap=16, policy=0):
    """Faithful PM (Eq. 2): spec-k, tree merge with delayed recovery, sequential stage 2."""
    perm, inv, _, tt, acc = transform(table, accept, policy, data if policy == 1 else None, start)
    t = _c(table, np.uint32)
    n, ns = t.shape
    d = _c(data, np.uint8)
    ce = np.zeros(max(1, nchunks(d.size, B)), np.uint32)
    res, pm = SimResult(), PmStats()
    rc = lib().or_simulate_pm_tree(tt.ctypes.data, n, ns, int(perm[start]), acc.ctypes.data, inv.ctypes.data,
                                   d.ctypes.data, d.size, B, k, qs_cap, ce.ctypes.data, ctypes.byref(res),
                                   ctypes.byref(pm))
    out = res.as_dict()
    out.update({"pm_" + k_: getattr(pm, k_) for k_, _ in PmStats._fields_})
    out["status"] = rc
    out["chunk_end"] = ce[:nchunks(d.size, B)]
    return out


def features(table, start, accept, data, B=4096, k=4, qs_cap=16, policy=0):
    """Selector features (reading c.4 #19) on the transformed DFA."""
    perm, inv, _, tt, acc = transform(table, accept, policy, data if policy == 1 else None, start)
    n, ns = _c(table, np.uint32).shape
    d = _c(data, np.uint8)
    f = Features()
    lib().or_features_compute(tt.ctypes.data, n, ns, int(perm[start]), acc.ctypes.data, d.ctypes.data, d.size,
                              B, k, qs_cap, ctypes.byref(f))
    return {"acc1": f.acc1, "acck": f.acck, "sens": f.sens, "uniq10": f.uniq10}


def select(feat: dict, nstates: int, paper_tree: bool = False) -> int:
    """The selector's decision tree (R19); paper_tree: without the B200 gate R19b."""
    f = Features(feat["acc1"], feat["acck"], feat["sens"], feat["uniq10"])
    if paper_tree:
        return int(lib().or_select_variant(ctypes.byref(f), nstates, 1))
    return int(lib().or_select(ctypes.byref(f), nstates))


def conv_lengths(table, start, accept, data, wmax=16384, policy=0):
    """Convergence lengths of the lookback-2 image over 4 KiB-spaced windows (reading
    R29): uint32 per window, 0xFFFFFFFF = not converged within wmax."""
    perm, inv, _, tt, acc = transform(table, accept, policy, data if policy == 1 else None, start)
    n, ns = _c(table, np.uint32).shape
    d = _c(data, np.uint8)
    nwin = lib().or_conv_lengths(tt.ctypes.data, n, ns, d.ctypes.data, d.size, wmax, None)
    out = np.zeros(max(nwin, 1), dtype=np.uint32)
    lib().or_conv_lengths(tt.ctypes.data, n, ns, d.ctypes.data, d.size, wmax, out.ctypes.data)
    return out[:nwin]


def select_chunk(d, length, min_chunks):
    """Chunk size (granularity) from convergence lengths (reading R29)."""
    d = _c(d, np.uint32)
    return int(lib().or_select_chunk(d.ctypes.data if d.size else None, d.size, length, min_chunks))
