"""Build libsvb200.so (sm_100a) in-tree with nvcc.  No GPU needed.

Usage: python -m paper_conf_sc_markidis23_b200.build [--force] [--verbose]
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
BUILD = os.path.join(HERE, "_build")
LIB = os.path.join(HERE, "libsvb200.so")
ROOT = os.path.dirname(HERE)
INCLUDE = os.path.join(ROOT, "include")

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
# nvJitLink compiles the PTX of the pass-specialised kernels at circuit creation (rpass_jit.cpp)
LINK: list = []
COMMON = ["-O3", "-std=c++17", "-lineinfo", "-Xcudafe", "--diag_suppress=177", "-Xcompiler", "-fPIC,-O3", "-I", INCLUDE, "-I", CSRC]

SOURCES = ["apply.cu", "apply64.cu", "blocked.cu", "small.cu", "state.cu", "fuser.cpp", "planner.cpp", "rpass_jit.cpp",
           "sv_api.cpp"]
HEADERS = ["kernels.h", "sv_internal.h", "device_util.cuh"]


def _newest_input() -> float:
    paths = [os.path.join(CSRC, f) for f in SOURCES + HEADERS] + [os.path.join(INCLUDE, "sv.h"), __file__]
    return max(os.path.getmtime(p) for p in paths)


def _compile(src: str, verbose: bool) -> str:
    obj = os.path.join(BUILD, src + ".o")
    hdr = max(os.path.getmtime(p) for p in [os.path.join(CSRC, f) for f in HEADERS] + [os.path.join(INCLUDE, "sv.h"), __file__])
    if os.path.exists(obj) and os.path.getmtime(obj) >= max(os.path.getmtime(os.path.join(CSRC, src)), hdr):
        return obj  # up to date
    cmd = [NVCC] + ARCH + COMMON + ["-c", os.path.join(CSRC, src), "-o", obj]
    if src.endswith(".cu"):
        cmd += ["-Xptxas", "-v"] if verbose else []
    else:
        cmd += ["-x", "cu"] if False else []
    if verbose:
        print(" ".join(cmd), flush=True)
    subprocess.check_call(cmd)
    return obj


def build_variant(name: str, defines, csrc: str = CSRC, include: str = INCLUDE) -> str:
    """Build an A/B variant library (extra -D flags, or another source tree,
    e.g. a git ref extracted by tools/ab_ref.py) next to the main one."""
    out = os.path.join(HERE, "_variants", f"libsvb200_{name}.so")
    bdir = os.path.join(HERE, "_variants", name)
    os.makedirs(bdir, exist_ok=True)
    extra = [f"-D{d}" for d in defines]
    common = [c for c in COMMON]
    common[common.index(INCLUDE)] = include
    common[common.index(CSRC)] = csrc

    def comp(src):
        obj = os.path.join(bdir, src + ".o")
        subprocess.check_call([NVCC] + ARCH + common + extra + ["-c", os.path.join(csrc, src), "-o", obj])
        return obj

    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 4)) as ex:
        objs = list(ex.map(comp, SOURCES))
    subprocess.check_call([NVCC] + ARCH + ["-shared", "-o", out] + objs + ["-Xcompiler", "-fPIC"] + LINK)
    return out


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and os.path.exists(LIB) and os.path.getmtime(LIB) >= _newest_input():
        return LIB
    os.makedirs(BUILD, exist_ok=True)
    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 4)) as ex:
        objs = list(ex.map(lambda s: _compile(s, verbose), SOURCES))
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = [NVCC] + ARCH + ["-shared", "-o", tmp] + objs + ["-Xcompiler", "-fPIC"] + LINK
    if verbose:
        print(" ".join(cmd), flush=True)
    subprocess.check_call(cmd)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    if len(sys.argv) > 2 and sys.argv[1] == "--variant":
        print(build_variant(sys.argv[2], sys.argv[3:]))
    else:
        build(force="--force" in sys.argv, verbose="--verbose" in sys.argv)
        print(LIB)
