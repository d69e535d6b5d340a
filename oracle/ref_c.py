"""ctypes loader for oracle/sv_ref.c (TEST INFRASTRUCTURE ONLY).

Compiled by ``build()`` (plain gcc -O2 -fopenmp) into oracle/libsvref.so.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import time

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "sv_ref.c")
LIB = os.path.join(HERE, "libsvref.so")

_lib = None


def build(force: bool = False) -> str:
    """Compile sv_ref.c (no GPU, no product headers)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        tmp = LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c99",
                               "-o", tmp, SRC])
        os.replace(tmp, LIB)
    return LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB)
        dp = ctypes.POINTER(ctypes.c_double)
        ip = ctypes.POINTER(ctypes.c_int)
        L.svref_apply.argtypes = [ctypes.c_int, ctypes.c_int, ip, dp, dp]
        L.svref_apply.restype = ctypes.c_int
        L.svref_run.argtypes = [ctypes.c_int, ctypes.c_int64, ip, ip, dp, dp]
        L.svref_run.restype = ctypes.c_int
        L.svref_zero_state.argtypes = [ctypes.c_int, dp]
        L.svref_threads.restype = ctypes.c_int
        _lib = L
    return _lib


def _dp(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def _ip(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_int))


def threads() -> int:
    return int(lib().svref_threads())


def zero_state(n: int) -> np.ndarray:
    psi = np.empty(1 << n, dtype=np.complex128)
    lib().svref_zero_state(n, _dp(psi.view(np.float64)))
    return psi


def apply(psi: np.ndarray, n: int, qubits, mat: np.ndarray) -> None:
    """In place on a complex128 array."""
    assert psi.dtype == np.complex128 and psi.flags.c_contiguous
    q = np.ascontiguousarray(qubits, dtype=np.int32)
    m = np.ascontiguousarray(mat, dtype=np.complex128)
    rc = lib().svref_apply(n, len(q), _ip(q), _dp(m.view(np.float64)), _dp(psi.view(np.float64)))
    if rc:
        raise ValueError("svref_apply: bad arguments")


def run(n: int, gates, psi: np.ndarray | None = None) -> np.ndarray:
    """Simulate unfused gates (1-2 qubits) from |0..0> (or psi, in place)."""
    from workloads.rqc import gate_arrays
    if psi is None:
        psi = zero_state(n)
    nq, qq, mat = gate_arrays(gates)
    rc = lib().svref_run(n, len(gates), _ip(nq), _ip(np.ascontiguousarray(qq)),
                         _dp(np.ascontiguousarray(mat)), _dp(psi.view(np.float64)))
    if rc:
        raise ValueError("svref_run: bad arguments")
    return psi


def time_gates(n: int, gates, max_seconds: float = 20.0):
    """Bounded timing sample for the CPU baseline: apply gates in order on a
    fresh 2^n state until max_seconds elapse.  Returns (gates_done, seconds)."""
    from workloads.rqc import gate_arrays
    psi = zero_state(n)
    nq, qq, mat = gate_arrays(gates)
    L = lib()
    t0 = time.perf_counter()
    done = 0
    for i in range(len(gates)):
        rc = L.svref_apply(n, int(nq[i]), _ip(np.ascontiguousarray(qq[i])),
                           _dp(np.ascontiguousarray(mat[i])), _dp(psi.view(np.float64)))
        assert rc == 0
        done += 1
        if time.perf_counter() - t0 > max_seconds:
            break
    return done, time.perf_counter() - t0
