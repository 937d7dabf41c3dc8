#!/usr/bin/env python3
"""Build every native artefact in-tree (sm_100a CUDA + host C).

  gen/libgsgen.so               seeded generators (host)            gcc
  gen/libgsgen_cuda.so          generators' device twin             nvcc
  oracle/liboracle.so           the CPU oracle (test infra only)    gcc
  paper_conf_ipps_wangwqw22_b200/libgspec.so   the product (C ABI)  nvcc sm_100a

Usage: python build.py [--force] [--only gen|oracle|gspec]
"""
from __future__ import annotations

import concurrent.futures
import glob
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.abspath(__file__))
PKG = os.path.join(ROOT, "paper_conf_ipps_wangwqw22_b200")
NVCC = shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc"
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVFLAGS = ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O3", "--expt-relaxed-constexpr",
                  "-Xptxas", "-warn-spills"]


def _stale(out, deps):
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    return any(os.path.getmtime(d) > t for d in deps)


def _run(cmd):
    print("+", " ".join(cmd), flush=True)
    subprocess.run(cmd, check=True, cwd=ROOT)


def build_gen(force=False):
    src = ["gen/gen.c"]
    deps = src + ["gen/gen.h", "gen/gs_hash.h"]
    out = "gen/libgsgen.so"
    if force or _stale(os.path.join(ROOT, out), [os.path.join(ROOT, d) for d in deps]):
        _run(["gcc", "-O2", "-fPIC", "-shared", "-std=c11", "-Wall", "-o", out] + src)
    out = "gen/libgsgen_cuda.so"
    deps2 = deps + ["gen/gen_cuda.cu"]
    if force or _stale(os.path.join(ROOT, out), [os.path.join(ROOT, d) for d in deps2]):
        os.makedirs(os.path.join(ROOT, "build"), exist_ok=True)
        _run(["gcc", "-O2", "-fPIC", "-std=c11", "-c", "gen/gen.c", "-o", "build/gen.o"])
        _run([NVCC] + NVFLAGS + ["-shared", "gen/gen_cuda.cu", "build/gen.o", "-o", out])


def build_oracle(force=False):
    src = ["oracle/oracle.c"]
    deps = src + ["oracle/oracle.h"]
    out = "oracle/liboracle.so"
    if force or _stale(os.path.join(ROOT, out), [os.path.join(ROOT, d) for d in deps]):
        _run(["gcc", "-O2", "-fPIC", "-shared", "-std=c11", "-Wall", "-Wno-unused-variable", "-o", out] + src)


def build_gspec(force=False):
    csrc = os.path.join(PKG, "csrc")
    srcs = sorted(glob.glob(os.path.join(csrc, "*.cu")) + glob.glob(os.path.join(csrc, "*.cpp")))
    deps = srcs + glob.glob(os.path.join(csrc, "*.h")) + glob.glob(os.path.join(csrc, "*.cuh")) + \
        [os.path.join(ROOT, "include", "gspec.h")]
    out = os.path.join(PKG, "libgspec.so")
    if not srcs:
        return
    if not (force or _stale(out, deps)):
        return
    objdir = os.path.join(ROOT, "build", "gspec")
    os.makedirs(objdir, exist_ok=True)
    objs, cmds = [], []
    hdrs = glob.glob(os.path.join(csrc, "*.h")) + glob.glob(os.path.join(csrc, "*.cuh")) + \
        [os.path.join(ROOT, "include", "gspec.h")]
    for s in srcs:
        o = os.path.join(objdir, os.path.basename(s) + ".o")
        if force or _stale(o, [s] + hdrs):
            cmds.append([NVCC] + NVFLAGS + ["-I", os.path.join(ROOT, "include"), "-I", csrc, "-rdc=false", "-c", s,
                                            "-o", o])
        objs.append(o)
    # translation units are independent: compile them in parallel
    with concurrent.futures.ThreadPoolExecutor(max_workers=max(1, min(len(cmds), os.cpu_count() or 1))) as ex:
        for fut in [ex.submit(_run, c) for c in cmds]:
            fut.result()
    _run([NVCC] + ARCH + ["-shared", "-o", out] + objs + ["-ldl"])


def build_all(force=False):
    build_gen(force)
    build_oracle(force)
    build_gspec(force)


if __name__ == "__main__":
    force = "--force" in sys.argv
    only = None
    if "--only" in sys.argv:
        only = sys.argv[sys.argv.index("--only") + 1]
    if only in (None, "gen"):
        build_gen(force)
    if only in (None, "oracle"):
        build_oracle(force)
    if only in (None, "gspec"):
        build_gspec(force)
