"""Seeded synthetic workloads (DFAs + input streams) for tests and bench.

Shared by the oracle tests and the CUDA-path tests/bench.  Holds none of the
method's arithmetic (see gen.h).  The recipe is SURVEY.md §8.0 / DESIGN.md
"Inputs": every byte is a pure function of (seed, offset), so any slice can be
regenerated on host (``input_host``) or in HBM (``input_device``) identically.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None
_CUDA_LIB = None

GS_IN_BITS, GS_IN_TEXT, GS_IN_UNIFORM = 0, 1, 2
GIB = 1 << 30
MIB = 1 << 20


class InputParams(ctypes.Structure):
    _fields_ = [
        ("kind", ctypes.c_uint32),
        ("nsyms", ctypes.c_uint32),
        ("seed", ctypes.c_uint64),
        ("plants_per_block", ctypes.c_uint32),
        ("nlit", ctypes.c_uint32),
        ("lit_bytes", ctypes.c_void_p),
        ("lit_off", ctypes.c_void_p),
        ("reset_byte", ctypes.c_int32),
        ("sensitive", ctypes.c_uint32),
    ]


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libgsgen.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `python build.py` first")
        L = ctypes.CDLL(path)
        L.gs_input_fill.argtypes = [ctypes.POINTER(InputParams), ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p]
        L.gs_bytes_hash.argtypes = [ctypes.c_void_p, ctypes.c_uint64]
        L.gs_bytes_hash.restype = ctypes.c_uint64
        L.gs_skew_table.argtypes = [ctypes.c_int, ctypes.c_void_p]
        L.gs_literals.argtypes = [ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32,
                                  ctypes.c_void_p, ctypes.c_void_p]
        L.gs_literals.restype = ctypes.c_uint32
        L.gs_dfa_div7.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
        L.gs_dfa_ac.argtypes = [ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
        L.gs_dfa_ac.restype = ctypes.c_uint32
        L.gs_dfa_ac_counter.argtypes = [ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32,
                                        ctypes.c_void_p, ctypes.c_void_p]
        L.gs_dfa_ac_counter.restype = ctypes.c_uint32
        L.gs_dfa_random.argtypes = [ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p]
        _LIB = L
    return _LIB


def cuda_lib():
    global _CUDA_LIB
    if _CUDA_LIB is None:
        path = os.path.join(_HERE, "libgsgen_cuda.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `python build.py` first")
        L = ctypes.CDLL(path)
        L.gs_input_fill_device.argtypes = [ctypes.POINTER(InputParams), ctypes.c_uint64, ctypes.c_uint64,
                                           ctypes.c_void_p, ctypes.c_void_p]
        L.gs_input_fill_device.restype = ctypes.c_int
        _CUDA_LIB = L
    return _CUDA_LIB


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


def literals(seed: int, nlit: int, lmin: int, lmax: int):
    """Literal set: (bytes uint8[total], offsets uint32[nlit+1])."""
    b = np.zeros(max(1, nlit * min(lmax, 63)), np.uint8)
    o = np.zeros(nlit + 1, np.uint32)
    tot = lib().gs_literals(seed, nlit, lmin, lmax, _ptr(b), _ptr(o))
    return b[:tot].copy(), o


def literal_list(lb: np.ndarray, lo: np.ndarray):
    return [bytes(lb[lo[i]:lo[i + 1]]) for i in range(len(lo) - 1)]


def dfa_div7():
    t = np.zeros((7, 2), np.uint32)
    a = np.zeros(7, np.uint8)
    lib().gs_dfa_div7(_ptr(t), _ptr(a))
    return t, 0, a


def dfa_ac(lb: np.ndarray, lo: np.ndarray):
    nlit = len(lo) - 1
    n = lib().gs_dfa_ac(nlit, _ptr(lb), _ptr(lo), None, None)
    t = np.zeros((n, 256), np.uint32)
    a = np.zeros(n, np.uint8)
    lib().gs_dfa_ac(nlit, _ptr(lb), _ptr(lo), _ptr(t), _ptr(a))
    return t, 0, a


def dfa_ac_counter(lb: np.ndarray, lo: np.ndarray, reset_byte: int):
    nlit = len(lo) - 1
    n = lib().gs_dfa_ac_counter(nlit, _ptr(lb), _ptr(lo), reset_byte, None, None)
    t = np.zeros((n, 256), np.uint32)
    a = np.zeros(n, np.uint8)
    lib().gs_dfa_ac_counter(nlit, _ptr(lb), _ptr(lo), reset_byte, _ptr(t), _ptr(a))
    return t, 0, a


def dfa_random(seed: int, n: int, nsyms: int):
    t = np.zeros((n, nsyms), np.uint32)
    a = np.zeros(n, np.uint8)
    lib().gs_dfa_random(seed, n, nsyms, _ptr(t), _ptr(a))
    return t, 0, a


def skew_table(variant: int = 0) -> np.ndarray:
    out = np.zeros(256, np.uint8)
    lib().gs_skew_table(variant, _ptr(out))
    return out


@dataclass
class Workload:
    """One BASELINE.json config made concrete."""
    name: str
    table: np.ndarray
    start: int
    accept: np.ndarray
    params: InputParams
    length: int
    keep: tuple = ()
    literals: tuple = ()

    @property
    def nstates(self):
        return self.table.shape[0]

    @property
    def nsyms(self):
        return self.table.shape[1]

    def host(self, offset: int = 0, length: int | None = None) -> np.ndarray:
        length = self.length if length is None else length
        out = np.empty(length, np.uint8)
        if length:
            lib().gs_input_fill(ctypes.byref(self.params), offset, length, _ptr(out))
        return out

    def device(self, tensor, offset: int = 0, stream: int = 0) -> None:
        """Fill a uint8 CUDA tensor with bytes offset..offset+numel."""
        n = tensor.numel()
        rc = cuda_lib().gs_input_fill_device(ctypes.byref(self.params), offset, n, tensor.data_ptr(), stream)
        if rc != 0:
            raise RuntimeError(f"gs_input_fill_device failed: {rc}")


def _text_params(seed, lb, lo, ppb, reset=-1, sensitive=0):
    p = InputParams(kind=GS_IN_TEXT, nsyms=256, seed=seed, plants_per_block=ppb, nlit=len(lo) - 1,
                    lit_bytes=lb.ctypes.data if len(lb) else None, lit_off=lo.ctypes.data,
                    reset_byte=reset, sensitive=sensitive)
    return p


RESET_BYTE = ord("#")


def workload(name: str, length: int | None = None, seed: int | None = None) -> Workload:
    """Named workloads: c1 div7, c2 AC-114, c3 ACxZ16, c3s (input-sensitive), c4 AC-9770,
    rand:<n>:<nsyms>:<dfa_seed> (uniform random DFA on uniform symbols)."""
    if name == "c1":
        t, s, a = dfa_div7()
        p = InputParams(kind=GS_IN_BITS, nsyms=2, seed=seed if seed is not None else 0x5EED0001)
        return Workload(name, t, s, a, p, length if length is not None else MIB)
    if name == "c2":
        lb, lo = literals(0xC2, 12, 6, 12)
        t, s, a = dfa_ac(lb, lo)
        p = _text_params(seed if seed is not None else 0x5EED0002, lb, lo, 1)
        return Workload(name, t, s, a, p, length if length is not None else GIB, (lb, lo), literal_list(lb, lo))
    if name in ("c3", "c3s"):
        lb, lo = literals(0xC3, 6, 8, 12)
        t, s, a = dfa_ac_counter(lb, lo, RESET_BYTE)
        p = _text_params(seed if seed is not None else 0x5EED0003, lb, lo, 1, RESET_BYTE, 1 if name == "c3s" else 0)
        return Workload(name, t, s, a, p, length if length is not None else GIB, (lb, lo), literal_list(lb, lo))
    if name == "c4":
        lb, lo = literals(0xC4, 520, 8, 32)
        t, s, a = dfa_ac(lb, lo)
        p = _text_params(seed if seed is not None else 0x5EED0004, lb, lo, 16)
        return Workload(name, t, s, a, p, length if length is not None else 4 * GIB, (lb, lo), literal_list(lb, lo))
    if name.startswith("rand:"):
        _, n, ns, ds = name.split(":")
        t, s, a = dfa_random(int(ds), int(n), int(ns))
        p = InputParams(kind=GS_IN_UNIFORM, nsyms=int(ns), seed=seed if seed is not None else 0x5EED0009)
        return Workload(name, t, s, a, p, length if length is not None else MIB)
    raise KeyError(name)


def bytes_hash(a: np.ndarray) -> int:
    return int(lib().gs_bytes_hash(_ptr(a), a.size))
