"""Python binding of libsvb200 (include/sv.h) -- argument marshalling only.

Every call maps 1:1 onto the C ABI of the same name; every step of the hot
path runs in the library's CUDA kernels.  There is no fallback: if the
shared library is missing or cannot be loaded, importing the binding's
functions raises.  Build it with ``python -m paper_conf_sc_markidis23_b200.build``
(or ``__graft_entry__.build()``).

Arrays are numpy; device buffers may be passed as integers (e.g. a torch
tensor's ``data_ptr()``).  Gates are either a numpy array of dtype
``SV_GATE`` or any sequence of objects with ``.qubits`` and ``.matrix``
(1-2 qubits, complex matrix with bit b of the index <-> qubits[b]).
"""
from __future__ import annotations

import ctypes
import os
from typing import Sequence

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
# SVB200_LIB selects an alternative in-tree build (A/B kernel variants)
LIB_PATH = os.environ.get("SVB200_LIB") or os.path.join(HERE, "libsvb200.so")

SV_OK = 0
SV_EINVAL = -1
SV_ENOMEM = -2
SV_ECUDA = -3
SV_ECOMM = -4
SV_EUNSUPPORTED = -5
SV_EBADSTATE = -6

SV_OPT_BLOCK_BITS = 1
SV_OPT_PASS_JIT = 2
SV_OPT_APPLY_PATH = 3
SV_OPT_TIMING = 4
SV_OPT_DIAG_SKIP = 5
SV_OPT_PASS_PIN = 6
SV_OPT_PASS_SPEC = 7
SV_OPT_PASS_SEARCH = 8
SV_PATH_AUTO = 0
SV_PATH_SIMT = 1
SV_PATH_INT8 = 2

SV_GATE = np.dtype([("nq", "<i4"), ("q", "<i4", (2,)), ("pad", "<i4"), ("m", "<c16", (16,))], align=True)
assert SV_GATE.itemsize == 272


class SVError(RuntimeError):
    def __init__(self, code: int, where: str, msg: str):
        super().__init__(f"{where} failed ({code}): {msg}")
        self.code = code


class sv_stats(ctypes.Structure):
    _fields_ = [
        ("n_fused", ctypes.c_int32),
        ("n_exchanges", ctypes.c_int32),
        ("fused_hist", ctypes.c_int32 * 7),
        ("n_launch_high", ctypes.c_int32),
        ("n_launch_low", ctypes.c_int32),
        ("n_launch_other", ctypes.c_int32),
        ("t_fuse_s", ctypes.c_double),
        ("t_plan_s", ctypes.c_double),
        ("t_upload_s", ctypes.c_double),
        ("t_total_s", ctypes.c_double),
        ("t_apply_high_dev_s", ctypes.c_double),
        ("t_apply_low_dev_s", ctypes.c_double),
        ("t_exchange_dev_s", ctypes.c_double),
        ("t_other_dev_s", ctypes.c_double),
        ("bytes_apply", ctypes.c_uint64),
        ("bytes_exchange", ctypes.c_uint64),
        ("flops_apply", ctypes.c_uint64),
        ("n_passes", ctypes.c_int32),
        ("block_bits", ctypes.c_int32),
        ("fma_apply", ctypes.c_uint64),
        ("bytes_apply_high", ctypes.c_uint64),
        ("bytes_apply_low", ctypes.c_uint64),
        ("n_jit_passes", ctypes.c_int32),
        ("reserved2_", ctypes.c_int32),
    ]

    def as_dict(self):
        d = {f: getattr(self, f) for f, _ in self._fields_}
        d["fused_hist"] = list(self.fused_hist)
        return d


class sv_config(ctypes.Structure):
    _fields_ = [
        ("n_qubits", ctypes.c_int32),
        ("world", ctypes.c_int32),
        ("rank", ctypes.c_int32),
        ("virtual_shards", ctypes.c_int32),
        ("exchange_vmin", ctypes.c_int32),
        ("device", ctypes.c_int32),
        ("dev_buf", ctypes.c_void_p),
        ("buf_bytes", ctypes.c_size_t),
        ("cuda_stream", ctypes.c_void_p),
        ("precision", ctypes.c_int32),
        ("reserved_", ctypes.c_int32),
    ]


_lib = None
_vp = ctypes.c_void_p
_sz = ctypes.c_size_t
_i32p = ctypes.POINTER(ctypes.c_int32)
_u64p = ctypes.POINTER(ctypes.c_uint64)

_SIGS = {
    "sv_create": ([ctypes.c_int, ctypes.POINTER(_vp)], ctypes.c_int),
    "sv_create_ex": ([ctypes.POINTER(sv_config), ctypes.POINTER(_vp)], ctypes.c_int),
    "sv_destroy": ([_vp], ctypes.c_int),
    "sv_reset": ([_vp], ctypes.c_int),
    "sv_apply_fused": ([_vp, ctypes.c_int, _i32p, _vp], ctypes.c_int),
    "sv_apply_fused_c128": ([_vp, ctypes.c_int, _i32p, _vp], ctypes.c_int),
    "sv_apply_controlled": ([_vp, ctypes.c_int, _i32p, ctypes.c_int, _i32p, _vp], ctypes.c_int),
    "sv_run_circuit": ([_vp, _vp, _sz, ctypes.c_int, ctypes.POINTER(sv_stats)], ctypes.c_int),
    "sv_circuit_create": ([_vp, _vp, _sz, ctypes.c_int, ctypes.POINTER(_vp)], ctypes.c_int),
    "sv_circuit_run_device": ([_vp, _vp], ctypes.c_int),
    "sv_circuit_stats": ([_vp, ctypes.POINTER(sv_stats)], ctypes.c_int),
    "sv_circuit_destroy": ([_vp], ctypes.c_int),
    "sv_amplitudes": ([_vp, _u64p, _sz, _vp], ctypes.c_int),
    "sv_amplitudes_c128": ([_vp, _u64p, _sz, _vp], ctypes.c_int),
    "sv_sample": ([_vp, ctypes.c_uint64, _sz, _u64p], ctypes.c_int),
    "sv_sample_device": ([_vp, ctypes.c_uint64, _sz, _vp], ctypes.c_int),
    "sv_set_state": ([_vp, _vp, _sz], ctypes.c_int),
    "sv_get_state": ([_vp, _vp, _sz], ctypes.c_int),
    "sv_set_state_c128": ([_vp, _vp, _sz], ctypes.c_int),
    "sv_get_state_c128": ([_vp, _vp, _sz], ctypes.c_int),
    "sv_device_ptr": ([_vp, ctypes.c_int, ctypes.POINTER(_vp)], ctypes.c_int),
    "sv_fusion_plan": ([_vp, _sz, ctypes.c_int, _i32p, _sz, ctypes.POINTER(_sz)], ctypes.c_int),
    "sv_fused_matrix": ([_vp, _sz, ctypes.c_int, _sz, _vp, _sz], ctypes.c_int),
    "sv_block_plan": ([_vp, _sz, ctypes.c_int, ctypes.c_int, _i32p, _sz, ctypes.POINTER(_sz)], ctypes.c_int),
    "sv_shard_plan": ([_i32p, _sz, ctypes.c_int, ctypes.c_int, ctypes.c_int, _i32p, _sz, ctypes.POINTER(_sz), _i32p],
                      ctypes.c_int),
    "sv_shard_plan_diag": ([_i32p, _sz, _u64p, ctypes.c_int, ctypes.c_int, ctypes.c_int, _i32p, _sz,
                            ctypes.POINTER(_sz), _i32p], ctypes.c_int),
    "sv_fusion_diag_masks": ([_vp, _sz, ctypes.c_int, _u64p, _sz, ctypes.POINTER(_sz)], ctypes.c_int),
    "sv_qubit_map": ([_vp, _i32p], ctypes.c_int),
    "sv_ipc_handle": ([_vp, _vp, _sz, ctypes.POINTER(_sz)], ctypes.c_int),
    "sv_attach_peers": ([_vp, _vp, _sz], ctypes.c_int),
    "sv_set_blocking": ([_vp, ctypes.c_int], ctypes.c_int),
    "sv_set_timing": ([_vp, ctypes.c_int], ctypes.c_int),
    "sv_set_option": ([_vp, ctypes.c_int, ctypes.c_int], ctypes.c_int),
    "sv_pass_kernels": ([_vp, _sz, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_char_p, _sz, ctypes.POINTER(_sz)],
                        ctypes.c_int),
    "sv_jit_stats": ([_u64p, _u64p, ctypes.POINTER(ctypes.c_double)], ctypes.c_int),
    "sv_last_stats": ([_vp, ctypes.POINTER(sv_stats)], ctypes.c_int),
    "sv_last_pass_costs": ([_vp, _u64p, _u64p, _sz, ctypes.POINTER(_sz)], ctypes.c_int),
    "sv_synchronize": ([_vp], ctypes.c_int),
    "sv_last_error": ([], ctypes.c_char_p),
    "sv_version": ([], ctypes.c_char_p),
}
EXPORTED = tuple(_SIGS)


def lib():
    """Load libsvb200.so (raises if it is missing -- no fallback path)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built; run python -m paper_conf_sc_markidis23_b200.build")
        L = ctypes.CDLL(LIB_PATH)
        for name, (args, res) in _SIGS.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = res
        _lib = L
    return _lib


def _check(rc: int, where: str):
    if rc != SV_OK:
        raise SVError(rc, where, lib().sv_last_error().decode(errors="replace"))


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


def as_gates(gates) -> np.ndarray:
    """Marshal gates into an SV_GATE array (fp64 matrices)."""
    if isinstance(gates, np.ndarray) and gates.dtype == SV_GATE:
        return np.ascontiguousarray(gates)
    arr = np.zeros(len(gates), dtype=SV_GATE)
    for i, g in enumerate(gates):
        qs = tuple(g.qubits)
        k = len(qs)
        arr["nq"][i] = k
        arr["q"][i, :k] = qs
        m = np.asarray(g.matrix, dtype=np.complex128).reshape(-1)
        arr["m"][i, : m.size] = m
    return arr


# ---- lifetime -----------------------------------------------------------------
def sv_create(n_qubits: int) -> int:
    h = _vp()
    _check(lib().sv_create(n_qubits, ctypes.byref(h)), "sv_create")
    return h.value


def sv_create_ex(n_qubits: int, world: int = 1, rank: int = 0, virtual_shards: bool = True,
                 exchange_vmin: int = -1, device: int = -1, dev_buf: int = 0, buf_bytes: int = 0,
                 cuda_stream: int = 0, precision: int = 0) -> int:
    """precision: 0 = complex64 (default), 1 = complex128."""
    cfg = sv_config(n_qubits, world, rank, 1 if virtual_shards else 0, exchange_vmin, device,
                    dev_buf or None, buf_bytes, cuda_stream or None, precision, 0)
    h = _vp()
    _check(lib().sv_create_ex(ctypes.byref(cfg), ctypes.byref(h)), "sv_create_ex")
    return h.value


def sv_destroy(h: int) -> None:
    _check(lib().sv_destroy(h), "sv_destroy")


def sv_reset(h: int) -> None:
    _check(lib().sv_reset(h), "sv_reset")


# ---- hot path -----------------------------------------------------------------
def sv_apply_fused(h: int, qubits: Sequence[int], matrix) -> None:
    q = np.ascontiguousarray(qubits, dtype=np.int32)
    m = np.ascontiguousarray(matrix, dtype=np.complex64)
    k = q.size
    if m.size != (1 << (2 * k)):
        raise ValueError("matrix must be 2^k x 2^k")
    _check(lib().sv_apply_fused(h, k, q.ctypes.data_as(_i32p), _ptr(m)), "sv_apply_fused")


def sv_apply_controlled(h: int, controls: Sequence[int], targets: Sequence[int], matrix) -> None:
    c = np.ascontiguousarray(controls, dtype=np.int32)
    t = np.ascontiguousarray(targets, dtype=np.int32)
    m = np.ascontiguousarray(matrix, dtype=np.complex64)
    if m.size != (1 << (2 * t.size)):
        raise ValueError("matrix must be 2^k x 2^k over the targets")
    _check(lib().sv_apply_controlled(h, c.size, c.ctypes.data_as(_i32p), t.size, t.ctypes.data_as(_i32p), _ptr(m)),
           "sv_apply_controlled")


def sv_apply_fused_c128(h: int, qubits: Sequence[int], matrix) -> None:
    q = np.ascontiguousarray(qubits, dtype=np.int32)
    m = np.ascontiguousarray(matrix, dtype=np.complex128)
    if m.size != (1 << (2 * q.size)):
        raise ValueError("matrix must be 2^k x 2^k")
    _check(lib().sv_apply_fused_c128(h, q.size, q.ctypes.data_as(_i32p), _ptr(m)), "sv_apply_fused_c128")


def sv_run_circuit(h: int, gates, max_fused: int) -> dict:
    g = as_gates(gates)
    st = sv_stats()
    _check(lib().sv_run_circuit(h, _ptr(g), len(g), max_fused, ctypes.byref(st)), "sv_run_circuit")
    return st.as_dict()


def sv_circuit_create(h: int, gates, max_fused: int) -> int:
    g = as_gates(gates)
    c = _vp()
    _check(lib().sv_circuit_create(h, _ptr(g), len(g), max_fused, ctypes.byref(c)), "sv_circuit_create")
    return c.value


def sv_circuit_run_device(h: int, c: int) -> None:
    _check(lib().sv_circuit_run_device(h, c), "sv_circuit_run_device")


def sv_circuit_stats(c: int) -> dict:
    st = sv_stats()
    _check(lib().sv_circuit_stats(c, ctypes.byref(st)), "sv_circuit_stats")
    return st.as_dict()


def sv_circuit_destroy(c: int) -> None:
    _check(lib().sv_circuit_destroy(c), "sv_circuit_destroy")


def sv_amplitudes(h: int, idx) -> np.ndarray:
    i = np.ascontiguousarray(idx, dtype=np.uint64)
    out = np.empty(i.size, dtype=np.complex64)
    _check(lib().sv_amplitudes(h, i.ctypes.data_as(_u64p), i.size, _ptr(out)), "sv_amplitudes")
    return out


def sv_amplitudes_c128(h: int, idx) -> np.ndarray:
    i = np.ascontiguousarray(idx, dtype=np.uint64)
    out = np.empty(i.size, dtype=np.complex128)
    _check(lib().sv_amplitudes_c128(h, i.ctypes.data_as(_u64p), i.size, _ptr(out)), "sv_amplitudes_c128")
    return out


def sv_sample(h: int, seed: int, n_samples: int, out=None) -> np.ndarray:
    """n_samples logical bitstrings; `out` (optional): a caller-owned contiguous
    uint64 array of at least n_samples entries (e.g. pinned host memory) to
    receive them."""
    if out is None:
        out = np.empty(n_samples, dtype=np.uint64)
    elif out.dtype != np.uint64 or not out.flags["C_CONTIGUOUS"] or out.size < n_samples:
        raise ValueError("out must be a contiguous uint64 array of at least n_samples entries")
    _check(lib().sv_sample(h, seed, n_samples, out.ctypes.data_as(_u64p)), "sv_sample")
    return out


def sv_sample_device(h: int, seed: int, n_samples: int, dev_out: int) -> None:
    _check(lib().sv_sample_device(h, seed, n_samples, dev_out), "sv_sample_device")


def sv_set_state(h: int, psi) -> None:
    a = np.ascontiguousarray(psi, dtype=np.complex64)
    _check(lib().sv_set_state(h, _ptr(a), a.size), "sv_set_state")


def sv_get_state(h: int, n_qubits: int) -> np.ndarray:
    out = np.empty(1 << n_qubits, dtype=np.complex64)
    _check(lib().sv_get_state(h, _ptr(out), out.size), "sv_get_state")
    return out


def sv_set_state_c128(h: int, psi) -> None:
    a = np.ascontiguousarray(psi, dtype=np.complex128)
    _check(lib().sv_set_state_c128(h, _ptr(a), a.size), "sv_set_state_c128")


def sv_get_state_c128(h: int, n_qubits: int) -> np.ndarray:
    out = np.empty(1 << n_qubits, dtype=np.complex128)
    _check(lib().sv_get_state_c128(h, _ptr(out), out.size), "sv_get_state_c128")
    return out


def sv_device_ptr(h: int, shard: int = 0) -> int:
    p = _vp()
    _check(lib().sv_device_ptr(h, shard, ctypes.byref(p)), "sv_device_ptr")
    return p.value


# ---- pure host ------------------------------------------------------------------
def sv_fusion_plan(gates, max_fused: int) -> np.ndarray:
    g = as_gates(gates)
    need = _sz()
    rc = lib().sv_fusion_plan(_ptr(g), len(g), max_fused, None, 0, ctypes.byref(need))
    if rc != SV_OK and need.value == 0:
        _check(rc, "sv_fusion_plan")
    buf = np.empty(need.value, dtype=np.int32)
    _check(lib().sv_fusion_plan(_ptr(g), len(g), max_fused, buf.ctypes.data_as(_i32p), buf.size,
                                ctypes.byref(need)), "sv_fusion_plan")
    return buf


def sv_block_plan(gates, max_fused: int, tile_bits: int) -> list:
    """Cache-blocked pass plan (pure host): a list of passes, each
    {"S": tile qubits, "fused": fused-gate indices in pass order,
     "phases": [(R tile positions, [indices into "fused"]), ...]}."""
    g = as_gates(gates)
    need = _sz()
    rc = lib().sv_block_plan(_ptr(g), len(g), max_fused, tile_bits, None, 0, ctypes.byref(need))
    if rc != SV_OK and need.value == 0:
        _check(rc, "sv_block_plan")
    buf = np.empty(need.value, dtype=np.int32)
    _check(lib().sv_block_plan(_ptr(g), len(g), max_fused, tile_bits, buf.ctypes.data_as(_i32p), buf.size,
                               ctypes.byref(need)), "sv_block_plan")
    out, i = [], 0
    b = buf.tolist()
    while i < len(b):
        T = b[i]
        S = b[i + 1:i + 1 + T]
        i += 1 + T
        n = b[i]
        fused = b[i + 1:i + 1 + n]
        i += 1 + n
        nph = b[i]
        i += 1
        phases = []
        for _ in range(nph):
            m = b[i]
            R = b[i + 1:i + 1 + m]
            i += 1 + m
            ng = b[i]
            phases.append((R, b[i + 1:i + 1 + ng]))
            i += 1 + ng
        out.append({"S": S, "fused": fused, "phases": phases})
    return out


def sv_fused_matrix(gates, max_fused: int, index: int, k: int) -> np.ndarray:
    g = as_gates(gates)
    out = np.empty((1 << k) * (1 << k), dtype=np.complex128)
    _check(lib().sv_fused_matrix(_ptr(g), len(g), max_fused, index, _ptr(out), out.size), "sv_fused_matrix")
    return out.reshape(1 << k, 1 << k)


def sv_shard_plan(fusion_stream, n_qubits: int, log2_world: int, vmin: int = 5):
    fs = np.ascontiguousarray(fusion_stream, dtype=np.int32)
    need = _sz()
    pos = np.empty(n_qubits, dtype=np.int32)
    lib().sv_shard_plan(fs.ctypes.data_as(_i32p), fs.size, n_qubits, log2_world, vmin, None, 0, ctypes.byref(need),
                        None)
    buf = np.empty(max(need.value, 1), dtype=np.int32)
    _check(lib().sv_shard_plan(fs.ctypes.data_as(_i32p), fs.size, n_qubits, log2_world, vmin,
                               buf.ctypes.data_as(_i32p), buf.size, ctypes.byref(need), pos.ctypes.data_as(_i32p)),
           "sv_shard_plan")
    return buf[: need.value], pos


def sv_fusion_diag_masks(gates, max_fused: int) -> np.ndarray:
    """Per fused gate: mask of the logical qubits its fp64 matrix is block-diagonal in."""
    g = as_gates(gates)
    need = _sz()
    lib().sv_fusion_diag_masks(_ptr(g), len(g), max_fused, None, 0, ctypes.byref(need))
    out = np.zeros(max(need.value, 1), dtype=np.uint64)
    _check(lib().sv_fusion_diag_masks(_ptr(g), len(g), max_fused, out.ctypes.data_as(_u64p), out.size,
                                      ctypes.byref(need)), "sv_fusion_diag_masks")
    return out[: need.value]


def sv_shard_plan_diag(fusion_stream, diag_masks, n_qubits: int, log2_world: int, vmin: int = 5):
    fs = np.ascontiguousarray(fusion_stream, dtype=np.int32)
    dm = np.ascontiguousarray(diag_masks, dtype=np.uint64)
    need = _sz()
    pos = np.empty(n_qubits, dtype=np.int32)
    lib().sv_shard_plan_diag(fs.ctypes.data_as(_i32p), fs.size, dm.ctypes.data_as(_u64p), n_qubits, log2_world, vmin,
                             None, 0, ctypes.byref(need), None)
    buf = np.empty(max(need.value, 1), dtype=np.int32)
    _check(lib().sv_shard_plan_diag(fs.ctypes.data_as(_i32p), fs.size, dm.ctypes.data_as(_u64p), n_qubits, log2_world,
                                    vmin, buf.ctypes.data_as(_i32p), buf.size, ctypes.byref(need),
                                    pos.ctypes.data_as(_i32p)), "sv_shard_plan_diag")
    return buf[: need.value], pos


def sv_qubit_map(h: int, n_qubits: int) -> np.ndarray:
    pos = np.empty(n_qubits, dtype=np.int32)
    _check(lib().sv_qubit_map(h, pos.ctypes.data_as(_i32p)), "sv_qubit_map")
    return pos


# ---- multi-process ----------------------------------------------------------------
def sv_ipc_handle(h: int) -> bytes:
    need = _sz()
    lib().sv_ipc_handle(h, None, 0, ctypes.byref(need))
    buf = ctypes.create_string_buffer(need.value)
    _check(lib().sv_ipc_handle(h, buf, need.value, ctypes.byref(need)), "sv_ipc_handle")
    return buf.raw


def sv_attach_peers(h: int, blobs: Sequence[bytes]) -> None:
    each = len(blobs[0])
    raw = b"".join(blobs)
    buf = ctypes.create_string_buffer(raw, len(raw))
    _check(lib().sv_attach_peers(h, buf, each), "sv_attach_peers")


# ---- misc ----------------------------------------------------------------------------
def sv_set_blocking(h: int, tile_bits: int) -> None:
    _check(lib().sv_set_blocking(h, tile_bits), "sv_set_blocking")


def sv_set_timing(h: int, enable: bool) -> None:
    _check(lib().sv_set_timing(h, 1 if enable else 0), "sv_set_timing")


def sv_set_option(h: int, option: int, value: int) -> None:
    _check(lib().sv_set_option(h, option, value), "sv_set_option")


def sv_pass_kernels(gates, max_fused: int, tile_bits: int, compile: bool = False) -> list:
    """CUDA sources of the pass-specialised kernels of a circuit's register-
    blocked passes (pure host; compile=True also compiles the PTX)."""
    g = as_gates(gates)
    need = _sz()
    _check(lib().sv_pass_kernels(_ptr(g), len(g), max_fused, tile_bits, 1 if compile else 0, None, 0,
                                 ctypes.byref(need)), "sv_pass_kernels")
    buf = ctypes.create_string_buffer(need.value)
    _check(lib().sv_pass_kernels(_ptr(g), len(g), max_fused, tile_bits, 0, buf, need.value, ctypes.byref(need)),
           "sv_pass_kernels")
    return [x for x in buf.value.decode().split("\n//----\n") if x.strip()]


def sv_jit_stats() -> dict:
    c, h, t = ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_double()
    _check(lib().sv_jit_stats(ctypes.byref(c), ctypes.byref(h), ctypes.byref(t)), "sv_jit_stats")
    return {"compiled": c.value, "cache_hits": h.value, "compile_s": t.value}


def sv_last_stats(h: int) -> dict:
    st = sv_stats()
    _check(lib().sv_last_stats(h, ctypes.byref(st)), "sv_last_stats")
    return st.as_dict()


def sv_last_pass_costs(h: int):
    """(bytes, fmas) per register-blocked pass of the last circuit run."""
    need = _sz()
    lib().sv_last_pass_costs(h, None, None, 0, ctypes.byref(need))
    b = np.zeros(max(need.value, 1), dtype=np.uint64)
    f = np.zeros(max(need.value, 1), dtype=np.uint64)
    _check(lib().sv_last_pass_costs(h, b.ctypes.data_as(_u64p), f.ctypes.data_as(_u64p), b.size, ctypes.byref(need)),
           "sv_last_pass_costs")
    return b[: need.value], f[: need.value]


def sv_synchronize(h: int) -> None:
    _check(lib().sv_synchronize(h), "sv_synchronize")


def sv_version() -> str:
    return lib().sv_version().decode()
