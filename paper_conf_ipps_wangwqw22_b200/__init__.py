"""B200-native GSpecPal hot path — thin Python binding over libgspec.so.

Argument marshalling only: every step of the method runs in the sm_100a
kernels behind the C ABI (include/gspec.h).  PyTorch is used for device
memory and streams; there is no CPU fallback — importing this package without
the built library raises.

    import paper_conf_ipps_wangwqw22_b200 as gs
    fsm = gs.FSM.load(table, start, accept)          # numpy uint32 [n, nsyms]
    res = fsm.run(x_cuda_uint8, scheme="auto")       # -> Result
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libgspec.so")
if not os.path.exists(_LIB_PATH):
    raise ImportError(f"{_LIB_PATH} is missing: build it with `python build.py` (no CPU fallback exists)")
_lib = ctypes.CDLL(_LIB_PATH)

FSM_OK, FSM_EINVAL, FSM_ENOMEM, FSM_ECUDA, FSM_ESYMBOL, FSM_ENCCL, FSM_EUNSUPPORTED = 0, -1, -2, -3, -4, -5, -6
FSM_EAGAIN = -7
SCHEMES = {"auto": 0, "seq": 1, "pm": 2, "sre": 3, "rr": 4, "nf": 5, "enum": 6, "cse": 7, "pm_tree": 8}
SCHEME_NAMES = {v: k for k, v in SCHEMES.items()}
MODES = {1: "u8", 2: "u16", 3: "u32", 4: "u16d"}

U32, U64, P = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_void_p


class fsm_load_opts(ctypes.Structure):
    _fields_ = [("freq_policy", U32), ("profile_sample", P), ("profile_len", U64),
                ("smem_budget_bytes", U32), ("force_mode", U32)]


class fsm_run_opts(ctypes.Structure):
    _fields_ = [("scheme", ctypes.c_int), ("chunk_bytes", U32), ("spec_k", U32), ("lookback", U32),
                ("qs_cap", U32), ("vr_end", U32), ("vr_others", U32), ("stream", P)]


class fsm_result(ctypes.Structure):
    _fields_ = [("final_state", U32), ("accept", U32), ("accept_count", U64), ("nchunks", U64),
                ("scheme_used", ctypes.c_int), ("rounds", U32), ("tasks_total", U64), ("tasks_mustdo", U64),
                ("tasks_sre", U64), ("tasks_helper", U64), ("reread_bytes", U64), ("verify_checks", U64),
                ("verify_matches", U64), ("avg_active_workers", ctypes.c_double), ("ms_spec", ctypes.c_double),
                ("ms_verify", ctypes.c_double), ("kernel_launches", U32), ("pm_merge_checks", U64),
                ("pm_invalid_marks", U64), ("pm_jumps", U64), ("helper_walks", U64),
                ("task_walked_bytes", U64)]


class fsm_batch_result(ctypes.Structure):
    _fields_ = [("nstreams", U64), ("nchunks", U64), ("recoveries", U64), ("reread_bytes", U64),
                ("invalid_streams", U64), ("ms", ctypes.c_float)]


class fsm_multi_result(ctypes.Structure):
    _fields_ = [("rewalks", U64), ("rounds", U64), ("ms", ctypes.c_float)]


class fsm_features(ctypes.Structure):
    _fields_ = [("acc1", ctypes.c_double), ("acck", ctypes.c_double), ("input_sensitivity", ctypes.c_double),
                ("uniq10", ctypes.c_double), ("nstates", U32), ("chunk_bytes", U32), ("conv4k", ctypes.c_double),
                ("conv8k", ctypes.c_double), ("conv16k", ctypes.c_double)]


_lib.fsm_load.argtypes = [P, U32, U32, U32, P, ctypes.POINTER(fsm_load_opts), ctypes.POINTER(P)]
_lib.fsm_chunk_for.argtypes = [ctypes.POINTER(fsm_features), U64]
_lib.fsm_chunk_for.restype = U32
_lib.fsm_num_chunks.argtypes = [U64, U32]
_lib.fsm_num_chunks.restype = U64
_lib.fsm_run.argtypes = [P, P, U64, ctypes.POINTER(fsm_run_opts), P, ctypes.POINTER(fsm_result)]
_lib.fsm_run_host.argtypes = [P, P, U64, ctypes.POINTER(fsm_run_opts), P, ctypes.POINTER(fsm_result)]
_lib.fsm_run_literal.argtypes = [P, P, U64, ctypes.POINTER(fsm_run_opts), P, ctypes.POINTER(fsm_result)]
_lib.fsm_run_async.argtypes = [P, P, U64, ctypes.POINTER(fsm_run_opts), P, ctypes.POINTER(U64)]
_lib.fsm_wait.argtypes = [P, U64, ctypes.POINTER(fsm_result)]
_lib.fsm_batch_chunks.argtypes = [P, U32, U32]
_lib.fsm_batch_chunks.restype = U64
_lib.fsm_run_batch.argtypes = [P, P, P, U32, ctypes.POINTER(fsm_run_opts), P, P, P, ctypes.POINTER(fsm_batch_result)]
_lib.fsm_run_multi.argtypes = [P, U32, P, P, ctypes.POINTER(fsm_run_opts), P, P, ctypes.POINTER(fsm_multi_result)]
_lib.fsm_select_scheme.argtypes = [P, P, U64, ctypes.POINTER(fsm_run_opts), ctypes.POINTER(ctypes.c_int),
                                   ctypes.POINTER(fsm_features)]
_lib.fsm_map_bytes.argtypes = [P]
_lib.fsm_map_bytes.restype = U64
_lib.fsm_shard_map.argtypes = [P, P, U64, P, U32, ctypes.POINTER(fsm_run_opts), P, P]
_lib.fsm_shard_map_exact.argtypes = [P, P, U64, P, U32, ctypes.POINTER(fsm_run_opts), P, P]
_lib.fsm_shard_finish.argtypes = [P, P, U32, U32, ctypes.POINTER(fsm_run_opts), P, ctypes.POINTER(fsm_result)]
_lib.fsm_get_transform.argtypes = [P, P, P, P, P, P, P]
_lib.fsm_get_qs.argtypes = [P, ctypes.c_uint8, ctypes.c_uint8, P, P, P]
_lib.fsm_get_records.argtypes = [P, U64, P, P, P, P, P, P]
_lib.fsm_get_phase_times.argtypes = [P, P, ctypes.POINTER(U32)]
_lib.fsm_get_timeline.argtypes = [P, P]
_lib.fsm_comm_unique_id.argtypes = [P]
_lib.fsm_comm_init.argtypes = [ctypes.c_int, ctypes.c_int, P, ctypes.c_int, ctypes.POINTER(P)]
_lib.fsm_run_sharded_at.argtypes = [P, P, P, U64, U64, U64, ctypes.POINTER(fsm_run_opts), P, ctypes.POINTER(fsm_result)]
_lib.fsm_run_sharded.argtypes = [P, P, P, U64, P, U32, ctypes.POINTER(fsm_run_opts), P, ctypes.POINTER(fsm_result)]
_lib.fsm_run_sharded_async.argtypes = [P, P, P, U64, P, U32, ctypes.POINTER(fsm_run_opts), P, ctypes.POINTER(U64)]
_lib.fsm_shard_finish_async.argtypes = [P, P, U32, U32, ctypes.POINTER(fsm_run_opts), P, ctypes.POINTER(U64)]
_lib.fsm_shard_wait.argtypes = [P, U64, ctypes.POINTER(fsm_result)]
_lib.fsm_p2p_create.argtypes = [P, ctypes.c_int, ctypes.c_int, P, ctypes.POINTER(P)]
_lib.fsm_p2p_open.argtypes = [P, P]
_lib.fsm_run_sharded_p2p.argtypes = [P, P, P, U64, P, U32, ctypes.POINTER(fsm_run_opts), P, ctypes.POINTER(fsm_result)]
_lib.fsm_p2p_free.argtypes = [P]
_lib.fsm_p2p_free.restype = None
_lib.fsm_comm_free.argtypes = [P]
_lib.fsm_comm_free.restype = None
_lib.fsm_free.argtypes = [P]
_lib.fsm_free.restype = None
_lib.fsm_strerror.argtypes = [ctypes.c_int]
_lib.fsm_strerror.restype = ctypes.c_char_p
_lib.fsm_last_error.restype = ctypes.c_char_p


class GSpecError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = _lib.fsm_last_error().decode(errors="replace")
        super().__init__(f"{where}: {_lib.fsm_strerror(status).decode()} ({status}): {msg}")


def _check(rc: int, where: str):
    if rc != FSM_OK:
        raise GSpecError(rc, where)


def lib_path() -> str:
    return _LIB_PATH


def fsm_num_chunks(length: int, chunk_bytes: int = 4096) -> int:
    return int(_lib.fsm_num_chunks(length, chunk_bytes))


def run_multi(fsms, inputs, chunk_bytes=4096, stream=None):
    """fsm_run_multi (FSM-level batching): fsms[i] over the uint8 CUDA tensor inputs[i], all
    pairs in one launch per table format.  Returns (finals uint32 [n], counts uint64 [n],
    stats dict); a final of 0xFFFFFFFF marks a stream with an invalid symbol (and raises)."""
    n = len(fsms)
    assert len(inputs) == n
    hs = (ctypes.c_void_p * max(n, 1))(*[f.handle for f in fsms])
    ptrs = (ctypes.c_void_p * max(n, 1))(*[x.data_ptr() if x.numel() else 0 for x in inputs])
    lens = np.array([x.numel() for x in inputs] or [0], np.uint64)
    fin = np.zeros(max(n, 1), np.uint32)
    cnt = np.zeros(max(n, 1), np.uint64)
    o = _run_opts("sre", chunk_bytes, stream=stream)
    r = fsm_multi_result()
    _check(_lib.fsm_run_multi(hs, n, ptrs, lens.ctypes.data, ctypes.byref(o), fin.ctypes.data, cnt.ctypes.data,
                              ctypes.byref(r)), "fsm_run_multi")
    return fin[:n], cnt[:n], {k: getattr(r, k) for k, _ in fsm_multi_result._fields_}


def _run_opts(scheme="auto", chunk_bytes=4096, spec_k=0, qs_cap=16, vr_end=16, vr_others=16, stream=None,
              lookback=2):
    if isinstance(scheme, str):
        scheme = SCHEMES[scheme]
    if stream is None:
        import torch

        stream = torch.cuda.current_stream().cuda_stream if torch.cuda.is_available() else 0
    return fsm_run_opts(scheme=scheme, chunk_bytes=chunk_bytes, spec_k=spec_k, lookback=lookback, qs_cap=qs_cap,
                        vr_end=vr_end, vr_others=vr_others, stream=stream)


@dataclass
class Result:
    final_state: int
    accept: bool
    accept_count: int
    nchunks: int
    scheme: str
    stats: dict = field(default_factory=dict)
    chunk_ends: object = None

    @staticmethod
    def from_c(r: fsm_result, chunk_ends=None) -> "Result":
        stats = {k: getattr(r, k) for k, _ in fsm_result._fields_}
        return Result(int(r.final_state), bool(r.accept), int(r.accept_count), int(r.nchunks),
                      SCHEME_NAMES.get(r.scheme_used, "?"), stats, chunk_ends)


class FSM:
    """A loaded DFA (device image of the frequency-transformed table)."""

    def __init__(self, handle: int, nstates: int, nsyms: int):
        self._h = handle
        self.nstates = nstates
        self.nsyms = nsyms

    @staticmethod
    def load(table, start: int, accept, freq_policy: int = 0, profile=None, smem_budget: int = 0,
             force_mode: int = 0) -> "FSM":
        """fsm_load: table uint32 [n, nsyms] (original ids), accept uint8 [n]."""
        t = np.ascontiguousarray(table, dtype=np.uint32)
        a = np.ascontiguousarray(accept, dtype=np.uint8)
        n, ns = t.shape
        prof = None if profile is None else np.ascontiguousarray(profile, dtype=np.uint8)
        o = fsm_load_opts(freq_policy=freq_policy, profile_sample=None if prof is None else prof.ctypes.data,
                          profile_len=0 if prof is None else prof.size, smem_budget_bytes=smem_budget,
                          force_mode=force_mode)
        h = P()
        _check(_lib.fsm_load(t.ctypes.data, n, ns, start, a.ctypes.data, ctypes.byref(o), ctypes.byref(h)),
               "fsm_load")
        return FSM(h.value, n, ns)

    def close(self):
        if self._h:
            _lib.fsm_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ---- runs -----------------------------------------------------------------
    def run(self, x, scheme="auto", chunk_bytes=4096, spec_k=0, qs_cap=16, vr_end=16, vr_others=16,
            chunk_ends=True, stream=None, lookback=2) -> Result:
        """fsm_run over a uint8 CUDA tensor; chunk_ends -> uint32 chunk end states (a torch.int32
        CUDA tensor); lookback = symbols before each chunk used for its prediction (2..16)."""
        import torch

        assert x.is_cuda and x.dtype == torch.uint8 and x.is_contiguous()
        o = _run_opts(scheme, chunk_bytes, spec_k, qs_cap, vr_end, vr_others, stream, lookback)
        n = fsm_num_chunks(x.numel(), chunk_bytes)
        ce = torch.empty(max(n, 1), dtype=torch.int32, device=x.device) if chunk_ends else None
        r = fsm_result()
        _check(_lib.fsm_run(self._h, x.data_ptr() if x.numel() else None, x.numel(), ctypes.byref(o),
                            ce.data_ptr() if ce is not None else None, ctypes.byref(r)), "fsm_run")
        return Result.from_c(r, ce[:n] if ce is not None else None)

    def run_async(self, x, scheme="auto", chunk_bytes=4096, chunk_ends=None, spec_k=0, stream=None,
                  lookback=2) -> int:
        """fsm_run_async: enqueue a run (stream-ordered) and return a ticket for wait()."""
        o = _run_opts(scheme, chunk_bytes, spec_k, stream=stream, lookback=lookback)
        t = U64(0)
        _check(_lib.fsm_run_async(self._h, x.data_ptr() if x.numel() else None, x.numel(), ctypes.byref(o),
                                  chunk_ends.data_ptr() if chunk_ends is not None else None, ctypes.byref(t)),
               "fsm_run_async")
        return t.value

    def wait(self, ticket: int) -> Result:
        r = fsm_result()
        _check(_lib.fsm_wait(self._h, ticket, ctypes.byref(r)), "fsm_wait")
        return Result.from_c(r)

    def run_literal(self, x, chunk_bytes=4096, vr_end=16, scheme="sre", qs_cap=16, stream=None) -> Result:
        """fsm_run_literal: the paper-literal single-CTA kernel (Alg. 2 L2-6 + Alg. 3 SRE /
        Alg. 4 RR / Alg. 5 NF verbatim, <= 1024 chunks) on a uint8 CUDA tensor."""
        o = _run_opts(scheme, chunk_bytes, qs_cap=qs_cap, vr_end=vr_end, stream=stream)
        n = fsm_num_chunks(x.numel(), chunk_bytes)
        import torch

        ce = torch.empty(max(n, 1), dtype=torch.int32, device=x.device)
        r = fsm_result()
        _check(_lib.fsm_run_literal(self._h, x.data_ptr() if x.numel() else None, x.numel(), ctypes.byref(o),
                                    ce.data_ptr(), ctypes.byref(r)), "fsm_run_literal")
        return Result.from_c(r, ce[:n])

    def run_host(self, data: np.ndarray, scheme="auto", chunk_bytes=4096, chunk_ends=True, stream=None,
                 **kw) -> Result:
        """fsm_run_host: host bytes in, host chunk ends out (H2D/D2H inside the call)."""
        d = np.ascontiguousarray(data, dtype=np.uint8) if not hasattr(data, "data_ptr") else data
        o = _run_opts(scheme, chunk_bytes, stream=stream, **kw)
        n = fsm_num_chunks(len(d) if not hasattr(d, "numel") else d.numel(), chunk_bytes)
        ce = np.zeros(max(n, 1), np.uint32) if chunk_ends else None
        r = fsm_result()
        ptr = d.data_ptr() if hasattr(d, "data_ptr") else d.ctypes.data
        length = d.numel() if hasattr(d, "numel") else d.size
        _check(_lib.fsm_run_host(self._h, ptr if length else None, length, ctypes.byref(o),
                                 ce.ctypes.data if ce is not None else None, ctypes.byref(r)), "fsm_run_host")
        return Result.from_c(r, ce[:n] if ce is not None else None)

    def select_scheme(self, sample, chunk_bytes=4096, spec_k=4, stream=None, stream_len=None):
        """fsm_select_scheme on a uint8 CUDA tensor: (scheme name, features dict).  The
        dict's chunk_bytes is the recommended chunk size (reading R29) for a stream of
        stream_len bytes per GPU (default: the sample's own length; fsm_chunk_for)."""
        o = _run_opts("sre", chunk_bytes, spec_k, stream=stream)
        out = ctypes.c_int(0)
        ft = fsm_features()
        _check(_lib.fsm_select_scheme(self._h, sample.data_ptr() if sample.numel() else None, sample.numel(),
                                      ctypes.byref(o), ctypes.byref(out), ctypes.byref(ft)), "fsm_select_scheme")
        if stream_len is not None:
            ft.chunk_bytes = _lib.fsm_chunk_for(ctypes.byref(ft), stream_len)
        return SCHEME_NAMES[out.value], {k: getattr(ft, k) for k, _ in fsm_features._fields_}

    # ---- introspection --------------------------------------------------------
    def transform(self):
        n = self.nstates
        perm = np.zeros(n + 1, np.uint32)
        inv = np.zeros(n + 1, np.uint32)
        freq = np.zeros(n, np.uint64)
        mode, H, C = U32(0), U32(0), U32(0)
        _check(_lib.fsm_get_transform(self._h, perm.ctypes.data, inv.ctypes.data, freq.ctypes.data,
                                      ctypes.byref(mode), ctypes.byref(H), ctypes.byref(C)), "fsm_get_transform")
        return {"perm": perm, "inv": inv, "freq": freq, "mode": MODES.get(mode.value, "?"), "hot_rows": H.value,
                "nclasses": C.value}

    def qs(self, a: int, b: int):
        q = np.zeros(16, np.uint32)
        ql, im = U32(0), U32(0)
        _check(_lib.fsm_get_qs(self._h, a, b, q.ctypes.data, ctypes.byref(ql), ctypes.byref(im)), "fsm_get_qs")
        return q[:ql.value].copy(), im.value

    def records(self, nchunks: int):
        """Records of the last run (transformed ids): dict of [32, nchunks] arrays + rings + x."""
        a = {k: np.zeros((32, nchunks), np.uint32) for k in ("start", "end", "cnt")}
        ne = np.zeros(nchunks, np.uint32)
        no = np.zeros(nchunks, np.uint32)
        x = np.zeros(nchunks + 1, np.uint32)
        _check(_lib.fsm_get_records(self._h, nchunks, a["start"].ctypes.data, a["end"].ctypes.data,
                                    a["cnt"].ctypes.data, ne.ctypes.data, no.ctypes.data, x.ctypes.data),
               "fsm_get_records")
        a.update(n_end=ne, n_oth=no, x=x)
        return a

    def phase_times(self):
        """Verify/recover phase boundaries (µs from kernel start) of the last collected run."""
        us = np.zeros(24, np.float64)
        n = U32(0)
        _check(_lib.fsm_get_phase_times(self._h, us.ctypes.data, ctypes.byref(n)), "fsm_get_phase_times")
        return us[:n.value].copy()

    def run_batch(self, x, offsets, chunk_bytes=4096, chunk_ends=False, stream=None):
        """fsm_run_batch: independent streams x[offsets[s]:offsets[s+1]] (x: uint8 CUDA tensor,
        offsets: host ints, len nstreams+1).  Returns (final int32 CUDA [ns], count int64 CUDA [ns],
        chunk_ends int32 CUDA or None, stats dict).  final == nstates marks a stream with an
        invalid byte (the call then raises GSpecError after filling the outputs)."""
        import torch

        assert x.is_cuda and x.dtype == torch.uint8 and x.is_contiguous()
        off = np.ascontiguousarray(offsets, dtype=np.uint64)
        ns = off.size - 1
        assert ns >= 0 and (ns == 0 or int(off[-1]) <= x.numel())
        o = _run_opts("sre", chunk_bytes, stream=stream)
        nch = int(_lib.fsm_batch_chunks(off.ctypes.data, ns, chunk_bytes))
        fin = torch.empty(max(ns, 1), dtype=torch.int32, device=x.device)
        cnt = torch.empty(max(ns, 1), dtype=torch.int64, device=x.device)
        ce = torch.empty(max(nch, 1), dtype=torch.int32, device=x.device) if chunk_ends else None
        r = fsm_batch_result()
        rc = _lib.fsm_run_batch(self._h, x.data_ptr() if x.numel() else None, off.ctypes.data, ns, ctypes.byref(o),
                                fin.data_ptr(), cnt.data_ptr(), ce.data_ptr() if ce is not None else None,
                                ctypes.byref(r))
        stats = {k: getattr(r, k) for k, _ in fsm_batch_result._fields_}
        _check(rc, "fsm_run_batch")
        return fin[:ns], cnt[:ns], (ce[:nch] if ce is not None else None), stats

    def timeline(self):
        """(spec kernel, gap, verify kernel) in µs of the last collected run; -1 unless GSPEC_STAMPS=1."""
        us = np.zeros(3, np.float64)
        _check(_lib.fsm_get_timeline(self._h, us.ctypes.data), "fsm_get_timeline")
        return us.copy()

    def map_bytes(self) -> int:
        return int(_lib.fsm_map_bytes(self._h))

    @property
    def handle(self):
        return self._h


class Comm:
    """Library-owned NCCL communicator (fsm_comm_init); one per rank / GPU."""

    def __init__(self, nranks: int, rank: int, unique_id: bytes, device: int = -1):
        h = P()
        buf = ctypes.create_string_buffer(bytes(unique_id), 128)
        _check(_lib.fsm_comm_init(nranks, rank, buf, device, ctypes.byref(h)), "fsm_comm_init")
        self._h = h.value
        self.nranks, self.rank = nranks, rank

    @staticmethod
    def unique_id() -> bytes:
        buf = ctypes.create_string_buffer(128)
        _check(_lib.fsm_comm_unique_id(buf), "fsm_comm_unique_id")
        return buf.raw

    def run_sharded(self, fsm: "FSM", shard, lookback=None, scheme="auto", chunk_bytes=4096, spec_k=0,
                    chunk_ends=True, stream=None) -> Result:
        """fsm_run_sharded: shard map + one ncclAllGather + finish, all inside the library."""
        import torch

        o = _run_opts(scheme, chunk_bytes, spec_k, stream=stream)
        n = fsm_num_chunks(shard.numel(), chunk_bytes)
        ce = torch.empty(max(n, 1), dtype=torch.int32, device=shard.device) if chunk_ends else None
        lb = lookback if lookback is not None and lookback.numel() else None
        r = fsm_result()
        _check(_lib.fsm_run_sharded(fsm.handle, self._h, shard.data_ptr() if shard.numel() else None, shard.numel(),
                                    lb.data_ptr() if lb is not None else None, lb.numel() if lb is not None else 0,
                                    ctypes.byref(o), ce.data_ptr() if ce is not None else None, ctypes.byref(r)),
               "fsm_run_sharded")
        return Result.from_c(r, ce[:n] if ce is not None else None)

    def run_sharded_at(self, fsm: "FSM", shard, shard_offset: int, total_len: int, scheme="auto",
                       chunk_bytes=4096, spec_k=0, chunk_ends=True, stream=None) -> Result:
        """fsm_run_sharded_at: as run_sharded, the lookback bytes fetched by the library."""
        import torch

        o = _run_opts(scheme, chunk_bytes, spec_k, stream=stream)
        n = fsm_num_chunks(shard.numel(), chunk_bytes)
        ce = torch.empty(max(n, 1), dtype=torch.int32, device=shard.device) if chunk_ends else None
        r = fsm_result()
        _check(_lib.fsm_run_sharded_at(fsm.handle, self._h, shard.data_ptr() if shard.numel() else None, shard_offset,
                                       shard.numel(), total_len, ctypes.byref(o),
                                       ce.data_ptr() if ce is not None else None, ctypes.byref(r)),
               "fsm_run_sharded_at")
        return Result.from_c(r, ce[:n] if ce is not None else None)

    def run_sharded_async(self, fsm: "FSM", shard, lookback=None, scheme="auto", chunk_bytes=4096, spec_k=0,
                          chunk_ends=None, stream=None) -> int:
        """fsm_run_sharded_async: queue one sharded step (map, ncclAllGather, finish) without a
        host wait; returns a ticket for wait().  chunk_ends: an int32 CUDA tensor or None."""
        o = _run_opts(scheme, chunk_bytes, spec_k, stream=stream)
        lb = lookback if lookback is not None and lookback.numel() else None
        t = U64(0)
        _check(_lib.fsm_run_sharded_async(fsm.handle, self._h, shard.data_ptr() if shard.numel() else None,
                                          shard.numel(), lb.data_ptr() if lb is not None else None,
                                          lb.numel() if lb is not None else 0, ctypes.byref(o),
                                          chunk_ends.data_ptr() if chunk_ends is not None else None,
                                          ctypes.byref(t)), "fsm_run_sharded_async")
        return t.value

    @staticmethod
    def wait(fsm: "FSM", ticket: int) -> Result:
        """fsm_shard_wait: block until a queued sharded step is done (GSpecError FSM_EAGAIN:
        redo the step with run_sharded on every rank)."""
        r = fsm_result()
        _check(_lib.fsm_shard_wait(fsm.handle, ticket, ctypes.byref(r)), "fsm_shard_wait")
        return Result.from_c(r)

    def close(self):
        if self._h:
            _lib.fsm_comm_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class P2P:
    """Peer-memory state-map exchange (fsm_p2p_*): a mailbox in this GPU's HBM that every
    peer maps through CUDA IPC.  handle -> exchange out of band -> open(all handles)."""

    def __init__(self, fsm: "FSM", nranks: int, rank: int):
        h = P()
        buf = ctypes.create_string_buffer(64)
        _check(_lib.fsm_p2p_create(fsm.handle, nranks, rank, buf, ctypes.byref(h)), "fsm_p2p_create")
        self._h = h.value
        self.handle = buf.raw
        self.nranks, self.rank = nranks, rank

    def open(self, handles):
        """handles: the nranks 64-byte IPC handles, in rank order."""
        assert len(handles) == self.nranks
        blob = ctypes.create_string_buffer(b"".join(bytes(x) for x in handles), 64 * self.nranks)
        _check(_lib.fsm_p2p_open(self._h, blob), "fsm_p2p_open")

    def run_sharded(self, fsm: "FSM", shard, lookback=None, scheme="auto", chunk_bytes=4096, spec_k=0,
                    chunk_ends=True, stream=None) -> Result:
        """fsm_run_sharded_p2p: shard map, publish into every peer's mailbox, wait, finish."""
        import torch

        o = _run_opts(scheme, chunk_bytes, spec_k, stream=stream)
        n = fsm_num_chunks(shard.numel(), chunk_bytes)
        ce = torch.empty(max(n, 1), dtype=torch.int32, device=shard.device) if chunk_ends else None
        lb = lookback if lookback is not None and lookback.numel() else None
        r = fsm_result()
        _check(_lib.fsm_run_sharded_p2p(fsm.handle, self._h, shard.data_ptr() if shard.numel() else None,
                                        shard.numel(), lb.data_ptr() if lb is not None else None,
                                        lb.numel() if lb is not None else 0, ctypes.byref(o),
                                        ce.data_ptr() if ce is not None else None, ctypes.byref(r)),
               "fsm_run_sharded_p2p")
        return Result.from_c(r, ce[:n] if ce is not None else None)

    def close(self):
        if self._h:
            _lib.fsm_p2p_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# C-ABI names (same entry points, argument marshalling only)
def fsm_load(table, start, accept, **kw) -> FSM:
    return FSM.load(table, start, accept, **kw)


def fsm_run(fsm: FSM, x, **kw) -> Result:
    return fsm.run(x, **kw)


def fsm_run_host(fsm: FSM, data, **kw) -> Result:
    return fsm.run_host(data, **kw)


def fsm_select_scheme(fsm: FSM, sample, **kw):
    return fsm.select_scheme(sample, **kw)


def fsm_free(fsm: FSM) -> None:
    fsm.close()
