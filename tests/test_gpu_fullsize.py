"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (prepared circuit: sv_circuit_create + sv_reset + sv_circuit_run_device).

* 30 q depth 14 (configs[1]): the whole complex128 oracle state (16 GiB,
  oracle/sv_ref.c on all host cores) against the GPU state for max_fused = 1
  and 2 (register-blocked passes: the optimal fusion on B200), 4 (SIMT k=4),
  5 (int8 tensor cores, k=5) and 6 (int8 tensor cores, k=6) -- fidelity and max |delta| against the north-star
  bounds, accumulated in fp64 chunk by chunk.  Sampling at 30 q is bit-exact
  against oracle/sample.py on the GPU's own complex64 state.
* 34 q depth 20 (configs[3], 128 GiB in place; no host oracle fits): the
  properties that hold at any size -- unit norm, and the inverse circuit
  returning |0...0> -- on the same launch configuration.

These are the slow GPU tests (~3 min, ~60 GB of host RAM); they skip when the
host or the GPU is too small.
"""
import os

import numpy as np
import pytest

import paper_conf_sc_markidis23_b200 as sv
from oracle import ref_c
from oracle import sample as osample
from oracle import sv as osv
from workloads import rqc as W

pytestmark = pytest.mark.gpu

CHUNK = 1 << 26


def _host_ram_gb():
    try:
        return os.sysconf("SC_PAGE_SIZE") * os.sysconf("SC_PHYS_PAGES") / 2 ** 30
    except (ValueError, OSError):
        return 0.0


def _gpu_free_gb():
    import torch
    free, _ = torch.cuda.mem_get_info()
    return free / 2 ** 30


def _run_prepared(n, gates, F):
    h = sv.sv_create(n)
    c = sv.sv_circuit_create(h, gates, F)
    sv.sv_reset(h)
    sv.sv_circuit_run_device(h, c)
    sv.sv_synchronize(h)
    st = sv.sv_circuit_stats(c)
    sv.sv_circuit_destroy(c)
    return h, st


def _compare_chunked(got, ref):
    ip = 0j
    err = 0.0
    for i in range(0, got.size, CHUNK):
        g = got[i:i + CHUNK].astype(np.complex128)
        r = ref[i:i + CHUNK]
        ip += np.vdot(g, r)
        err = max(err, float(np.abs(g - r).max()))
    return abs(ip) ** 2, err


@pytest.fixture(scope="module")
def ref30():
    if _host_ram_gb() < 64:
        pytest.skip("needs >= 64 GB host RAM for the 30 q oracle state")
    return ref_c.run(30, W.rqc(30, 14, 2023))


@pytest.mark.parametrize("F,kmax", [(1, 2), (2, 2), (4, 4), (5, 5), (6, 6)])
def test_30q_d14_state_vs_oracle(ref30, F, kmax):
    """F = 1, 2: register-blocked passes (the library default for
    max_fused <= 2, tile qubits 13); F >= 4: one launch per fused gate."""
    n, depth = 30, 14
    gates = W.rqc(n, depth, 2023)
    h, st = _run_prepared(n, gates, F)
    try:
        assert max(k for k, c in enumerate(st["fused_hist"]) if c) == kmax
        assert (st["n_passes"] > 0) == (F <= 2)
        got = sv.sv_get_state(h, n)
    finally:
        sv.sv_destroy(h)
    fid, err = _compare_chunked(got, ref30)
    print(f"FULLSIZE 30q d14 F={F}: 1-fidelity={1 - fid:.3e} max|delta|={err:.3e} "
          f"bound={osv.max_abs_bound(n, depth):.3e}")
    assert fid >= 1 - 1e-5, fid
    assert err <= osv.max_abs_bound(n, depth), (err, osv.max_abs_bound(n, depth))


def test_30q_sampling_bit_exact():
    if _host_ram_gb() < 64:
        pytest.skip("needs >= 64 GB host RAM")
    n = 30
    gates = W.rqc(n, 14, 2023)
    h, _ = _run_prepared(n, gates, 5)
    try:
        got = sv.sv_sample(h, 1, 100000)
        psi = sv.sv_get_state(h, n)
    finally:
        sv.sv_destroy(h)
    ref, _ = osample.sample(psi, 1, 100000)
    assert np.array_equal(np.asarray(got, dtype=np.uint64), ref)


@pytest.mark.parametrize("F", [1, 5])
def test_34q_d20_norm_and_inverse_roundtrip(F):
    """F = 1: register-blocked passes (the default); F = 5: int8 tensor cores."""
    n, depth = 34, 20
    if _gpu_free_gb() < 132:
        pytest.skip("needs a 128 GiB state in HBM")
    gates = W.rqc(n, depth, 2023)
    h = sv.sv_create(n)
    try:
        c = sv.sv_circuit_create(h, gates, F)
        ci = sv.sv_circuit_create(h, W.inverse_circuit(gates), F)
        assert (sv.sv_circuit_stats(c)["n_passes"] > 0) == (F <= 2)
        sv.sv_reset(h)
        sv.sv_circuit_run_device(h, c)
        # norm of the forward state from 2^20 sampled amplitudes (uniform indices)
        idx = np.random.default_rng(0).integers(0, 1 << n, size=1 << 20).astype(np.uint64)
        a = sv.sv_amplitudes(h, idx).astype(np.complex128)
        est = (1 << n) * float(np.mean(np.abs(a) ** 2))
        assert abs(est - 1) < 0.01, est  # Porter-Thomas: relative std of the estimate ~ 2^-10
        sv.sv_circuit_run_device(h, ci)
        a0 = sv.sv_amplitudes(h, np.array([0], dtype=np.uint64))[0]
        print(f"FULLSIZE 34q d20 F={F}: norm estimate {est:.5f}, |<0|U^-1 U|0>|^2 - 1 = {abs(complex(a0)) ** 2 - 1:.3e}")
        # two circuits of the north-star per-depth bound each
        assert abs(abs(complex(a0)) ** 2 - 1) <= 2e-5, a0
        sv.sv_circuit_destroy(c)
        sv.sv_circuit_destroy(ci)
    finally:
        sv.sv_destroy(h)
