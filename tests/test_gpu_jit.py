"""Pass-specialised register-blocked kernels (rpass_jit.cpp) against the
generic apply_rpass kernel and the oracle.

Both kernels run the same phase plan with the same FFMA2 sequence per complex
MAC, so their states must be bit-identical; the JIT path is also checked
against the oracle with the north star's tolerances.
"""
import numpy as np
import pytest

import paper_conf_sc_markidis23_b200 as sv
from oracle import ref_c
from workloads import rqc as W

from test_gpu_circuit import _check, _mixed_circuit, layer_depth

pytestmark = pytest.mark.gpu


def _state(n, gates, F, bits, jit, world=1, lazy_zero=True):
    h = sv.sv_create_ex(n, world=world, virtual_shards=True) if world > 1 else sv.sv_create(n)
    try:
        sv.sv_set_option(h, sv.SV_OPT_PASS_JIT, 1 if jit else 0)
        sv.sv_set_blocking(h, bits)
        c = sv.sv_circuit_create(h, gates, F)
        if not lazy_zero:
            sv.sv_get_state(h, n)  # materialises |0...0>: the first pass loads it
        sv.sv_circuit_run_device(h, c)
        st = sv.sv_last_stats(h)
        sv.sv_synchronize(h)
        got = sv.sv_get_state(h, n)
        sv.sv_circuit_destroy(c)
        return got, st
    finally:
        sv.sv_destroy(h)


@pytest.mark.parametrize("bits", [10, 11, 12, 13])
@pytest.mark.parametrize("F", [1, 2])
def test_jit_bit_identical_to_generic_rqc(bits, F):
    n, d = 21, 12
    gates = W.rqc(n, d, seed=bits + 10 * F)
    a, sa = _state(n, gates, F, bits, jit=True)
    b, sb = _state(n, gates, F, bits, jit=False)
    assert sa["n_jit_passes"] == sa["n_passes"] > 0
    assert sb["n_jit_passes"] == 0
    assert np.array_equal(a.view(np.uint32), b.view(np.uint32))


@pytest.mark.parametrize("bits", [10, 12, 13])
@pytest.mark.parametrize("F", [1, 2])
def test_jit_mixed_kinds_vs_generic_and_oracle(bits, F):
    """Dense, diagonal and CZ-like gates (CZ on register and on thread bits),
    tile bit 0 in and out of the register set, both store paths."""
    n, m = 20, 200
    gates = _mixed_circuit(n, m, seed=7 * bits + F)
    a, sa = _state(n, gates, F, bits, jit=True)
    b, _ = _state(n, gates, F, bits, jit=False)
    assert sa["n_jit_passes"] > 0
    assert np.array_equal(a.view(np.uint32), b.view(np.uint32))
    _check(n, layer_depth(gates), a, ref_c.run(n, gates))


@pytest.mark.parametrize("lazy", [True, False])
def test_jit_first_pass_zero_init_and_loaded(lazy):
    """The first pass synthesises |0...0> (lazy reset) or loads it."""
    n, d = 22, 14
    gates = W.rqc(n, d)
    a, _ = _state(n, gates, 1, 13, jit=True, lazy_zero=lazy)
    b, _ = _state(n, gates, 1, 13, jit=False, lazy_zero=lazy)
    assert np.array_equal(a.view(np.uint32), b.view(np.uint32))
    _check(n, d, a, ref_c.run(n, gates))


@pytest.mark.parametrize("world", [2, 4])
def test_jit_virtual_shards(world):
    n, d = 20, 14
    gates = W.rqc(n, d, seed=world)
    a, sa = _state(n, gates, 1, 11, jit=True, world=world)
    b, _ = _state(n, gates, 1, 11, jit=False, world=world)
    assert sa["n_exchanges"] >= 1 and sa["n_jit_passes"] > 0
    assert np.array_equal(a.view(np.uint32), b.view(np.uint32))
    _check(n, d, a, ref_c.run(n, gates))


def test_jit_kernel_cache_reuses_structure():
    """A second circuit with the same structure (same generator seed: same
    gates) compiles nothing new; a prepared circuit re-runs without compiling."""
    n, d = 20, 10
    gates = W.rqc(n, d, seed=3)
    h = sv.sv_create(n)
    try:
        c1 = sv.sv_circuit_create(h, gates, 1)
        before = sv.sv_jit_stats()
        c2 = sv.sv_circuit_create(h, gates, 1)
        after = sv.sv_jit_stats()
        assert after["compiled"] == before["compiled"]
        assert after["cache_hits"] > before["cache_hits"]
        sv.sv_circuit_destroy(c1)
        sv.sv_circuit_destroy(c2)
    finally:
        sv.sv_destroy(h)


def test_jit_30q_sampled_amplitudes_match_generic():
    """Full size (30q D14, the bench workload): JIT and generic kernels give
    the same amplitudes on a sample of 2^16 indices."""
    n, d = 30, 14
    gates = W.rqc(n, d)
    idx = np.random.default_rng(5).integers(0, 1 << n, size=1 << 16).astype(np.uint64)
    out = []
    for jit in (True, False):
        h = sv.sv_create(n)
        try:
            sv.sv_set_option(h, sv.SV_OPT_PASS_JIT, 1 if jit else 0)
            st = sv.sv_run_circuit(h, gates, 1)
            assert (st["n_jit_passes"] > 0) == jit
            out.append(sv.sv_amplitudes(h, idx))
        finally:
            sv.sv_destroy(h)
    assert np.array_equal(out[0].view(np.uint32), out[1].view(np.uint32))
