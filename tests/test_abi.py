"""C-ABI boundary checks that need no GPU (-m "not gpu")."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "gspec.h")


@pytest.fixture(scope="module")
def lib():
    import build

    build.build_gspec()
    import paper_conf_ipps_wangwqw22_b200 as gs

    return gs


def declared_symbols():
    src = open(HDR).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(fsm_[a-z_0-9]+)\s*\(", src)))


def test_header_declares_the_paper_calls():
    syms = declared_symbols()
    for s in ("fsm_load", "fsm_run", "fsm_select_scheme", "fsm_free", "fsm_run_host", "fsm_shard_map",
              "fsm_shard_finish"):
        assert s in syms


def test_library_exports_every_declared_symbol(lib):
    out = subprocess.run(["nm", "-D", "--defined-only", lib.lib_path()], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (fsm_[a-z_0-9]+)", out))
    missing = [s for s in declared_symbols() if s not in exported]
    assert not missing, missing
    so = ctypes.CDLL(lib.lib_path())
    for s in declared_symbols():
        assert hasattr(so, s)


def test_library_is_sm100a(lib):
    out = subprocess.run(["cuobjdump", "--list-elf", lib.lib_path()], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_host_only_calls(lib):
    assert lib.fsm_num_chunks(0, 4096) == 0
    assert lib.fsm_num_chunks(1, 4096) == 1
    assert lib.fsm_num_chunks(4096, 4096) == 1
    assert lib.fsm_num_chunks(4097, 4096) == 2
    assert lib.fsm_num_chunks(100, 0) == 1  # 0 -> default 4096
    assert lib._lib.fsm_strerror(-4) == b"input symbol out of range"
    import numpy as np

    off = np.array([0, 0, 1, 4096, 4096 + 4097, 9000, 9000], np.uint64)  # empty, 1 B, 1 chunk, 2 chunks, short, empty
    assert lib._lib.fsm_batch_chunks(off.ctypes.data, 6, 4096) == 0 + 1 + 1 + 2 + 1 + 0
    assert lib._lib.fsm_batch_chunks(off.ctypes.data, 6, 16) == sum(
        (int(off[i + 1]) - int(off[i]) + 15) // 16 for i in range(6))


def test_binding_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_wangwqw22_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h", ".cuh")):
                src = open(os.path.join(dirpath, f), errors="replace").read()
                assert "oracle" not in src.replace("oracle/", "").lower() or f.endswith(".md"), f
