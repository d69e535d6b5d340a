"""Pass-specialised register-blocked kernels (rpass_jit.cpp) against the
generic apply_rpass kernel and the oracle.

Both kernels run the same phase plan with the same FFMA2 sequence per complex
MAC, so with SV_OPT_PASS_SPEC = 0 their states must be bit-identical; the
JIT path (with and without the structured-gate arithmetic, R11) is
also checked against the oracle with the north star's tolerances.
"""
import numpy as np
import pytest

import paper_conf_sc_markidis23_b200 as sv
from oracle import ref_c
from workloads import rqc as W

from test_gpu_circuit import _check, _mixed_circuit, layer_depth

pytestmark = pytest.mark.gpu


def _state(n, gates, F, bits, jit, world=1, lazy_zero=True, spec=0):
    h = sv.sv_create_ex(n, world=world, virtual_shards=True) if world > 1 else sv.sv_create(n)
    try:
        sv.sv_set_option(h, sv.SV_OPT_PASS_JIT, 1 if jit else 0)
        sv.sv_set_option(h, sv.SV_OPT_PASS_SPEC, spec)
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
    a, sa = _state(n, gates, F, bits, jit=True, lazy_zero=False)
    b, sb = _state(n, gates, F, bits, jit=False, lazy_zero=False)
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
    a, sa = _state(n, gates, F, bits, jit=True, lazy_zero=False)
    b, _ = _state(n, gates, F, bits, jit=False, lazy_zero=False)
    assert sa["n_jit_passes"] > 0
    assert np.array_equal(a.view(np.uint32), b.view(np.uint32))
    _check(n, layer_depth(gates), a, ref_c.run(n, gates))


def test_jit_first_pass_loads_zero_state():
    """A materialised |0...0>: the first pass loads it (bit-identical)."""
    n, d = 22, 14
    gates = W.rqc(n, d)
    a, _ = _state(n, gates, 1, 13, jit=True, lazy_zero=False)
    b, _ = _state(n, gates, 1, 13, jit=False, lazy_zero=False)
    assert np.array_equal(a.view(np.uint32), b.view(np.uint32))
    _check(n, d, a, ref_c.run(n, gates))


@pytest.mark.parametrize("n,d,F,bits", [(22, 14, 1, 13), (21, 12, 2, 12), (20, 10, 1, 10)])
def test_jit_product_state_start_rqc(n, d, F, bits):
    """A run from the lazy |0...0> folds the first one-qubit gate of every
    qubit into a product-state first pass (R8): parity with the
    oracle, and with the generic kernel (which applies every gate) within
    the same tolerance."""
    gates = W.rqc(n, d, seed=n)
    a, sa = _state(n, gates, F, bits, jit=True, lazy_zero=True)
    b, sb = _state(n, gates, F, bits, jit=False, lazy_zero=True)
    c, sc = _state(n, gates, F, bits, jit=True, lazy_zero=True, spec=1)
    assert sa["n_jit_passes"] == sa["n_passes"] > 0
    assert sa["fma_apply"] < sb["fma_apply"]  # folded gates are not applied
    assert sc["fma_apply"] <= sa["fma_apply"]
    ref = ref_c.run(n, gates)
    _check(n, d, a, ref)
    _check(n, d, b, ref)
    _check(n, d, c, ref)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_jit_product_state_start_mixed(seed):
    """Mixed circuits: some qubits start with a two-qubit gate (not folded),
    some with diagonal or permutation gates, some are never touched."""
    n, m = 20, 120
    gates = _mixed_circuit(n - 2, m, seed=seed)  # qubits 18, 19 untouched
    a, sa = _state(n, gates, 1, 12, jit=True, lazy_zero=True)
    assert sa["n_jit_passes"] > 0
    _check(n, layer_depth(gates), a, ref_c.run(n, gates))


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
    """Full size (30q D14, the bench workload): from a materialised |0...0>
    the JIT and generic kernels give bit-identical amplitudes (2^16 sampled
    indices); from the lazy |0...0> (product-state start, the bench's step)
    they agree within the north-star max-abs bound."""
    n, d = 30, 14
    gates = W.rqc(n, d)
    idx = np.random.default_rng(5).integers(0, 1 << n, size=1 << 16).astype(np.uint64)
    out = {}
    for jit in (True, False):
        for lazy in (True, False):
            h = sv.sv_create(n)
            try:
                sv.sv_set_option(h, sv.SV_OPT_PASS_JIT, 1 if jit else 0)
                sv.sv_set_option(h, sv.SV_OPT_PASS_SPEC, 0)
                sv.sv_set_blocking(h, 13)  # the generic kernel's largest tile
                if not lazy:
                    sv.sv_device_ptr(h)  # writes |0...0> now
                st = sv.sv_run_circuit(h, gates, 1)
                assert (st["n_jit_passes"] > 0) == jit
                out[jit, lazy] = sv.sv_amplitudes(h, idx)
            finally:
                sv.sv_destroy(h)
    assert np.array_equal(out[True, False].view(np.uint32), out[False, False].view(np.uint32))
    assert np.array_equal(out[False, True].view(np.uint32), out[False, False].view(np.uint32))
    err = np.abs(out[True, True].astype(np.complex128) - out[False, False].astype(np.complex128)).max()
    bound = 1e-5 * 2.0 ** (-n / 2) * d
    assert err <= bound, (err, bound)


@pytest.mark.parametrize("bits", [10, 11, 12, 13, 14])
@pytest.mark.parametrize("F", [1, 2])
def test_fused_sampling_bins_bit_exact(bits, F):
    """The circuit's last pass writes the sampler's 16-amplitude S5 bin
    weights (no separate read of the state): samples are bit-identical to
    the oracle sampler on the GPU's final complex64 state, also for a second
    draw (bins recomputed) and after a state change.  RQC and mixed circuits
    cover the three store layouts of the last pass."""
    from oracle import sample as osample
    n = 21
    for gates in (W.rqc(n, 12, seed=bits + F), _mixed_circuit(n, 150, seed=3 * bits + F)):
        h = sv.sv_create(n)
        try:
            sv.sv_set_blocking(h, bits)
            c = sv.sv_circuit_create(h, gates, F)
            sv.sv_circuit_run_device(h, c)
            got1 = sv.sv_sample(h, 11, 4000)
            got2 = sv.sv_sample(h, 12, 4000)
            psi = sv.sv_get_state(h, n)
            sv.sv_apply_fused(h, [5], W.GATE_H.astype(np.complex64))
            got3 = sv.sv_sample(h, 13, 4000)
            psi3 = sv.sv_get_state(h, n)
            sv.sv_circuit_destroy(c)
        finally:
            sv.sv_destroy(h)
        assert np.array_equal(got1, osample.sample(psi, 11, 4000)[0])
        assert np.array_equal(got2, osample.sample(psi, 12, 4000)[0])
        assert np.array_equal(got3, osample.sample(psi3, 13, 4000)[0])


@pytest.mark.parametrize("pin", [3, 5])
@pytest.mark.parametrize("F", [1, 2])
def test_pass_pin_option(pin, F):
    """SV_OPT_PASS_PIN: tiles pinned to qubits 0..pin-1 (64 B / 256 B runs):
    JIT == generic bit for bit from a written |0...0>, oracle parity from the
    lazy one, and sampling bit-exact whether or not the last pass can write
    the 16-amplitude bins (it needs tile bits 0..3 = qubits 0..3)."""
    from oracle import sample as osample
    n, d = 21, 12
    gates = W.rqc(n, d, seed=pin + F)
    out = {}
    for jit, lazy in ((1, False), (0, False), (1, True)):
        h = sv.sv_create(n)
        try:
            sv.sv_set_option(h, sv.SV_OPT_PASS_PIN, pin)
            sv.sv_set_option(h, sv.SV_OPT_PASS_JIT, jit)
            sv.sv_set_option(h, sv.SV_OPT_PASS_SPEC, 0)
            sv.sv_set_blocking(h, 12)
            if not lazy:
                sv.sv_device_ptr(h)
            st = sv.sv_run_circuit(h, gates, F)
            smp = sv.sv_sample(h, 3, 3000)
            psi = sv.sv_get_state(h, n)
        finally:
            sv.sv_destroy(h)
        assert st["n_passes"] > 0
        assert np.array_equal(smp, osample.sample(psi, 3, 3000)[0])
        out[jit, lazy] = psi
    assert np.array_equal(out[1, False].view(np.uint32), out[0, False].view(np.uint32))
    _check(n, d, out[1, True], ref_c.run(n, gates))


# ---------------------------------------------------------------------------
# Structured one-qubit gates (SV_OPT_PASS_SPEC, R11)

def _structured_circuit(n, m, seed):
    """Every one-qubit class the pass kernels specialise -- row form (H,
    sqrt(X), sqrt(Y), with unit and non-unit row-1 factors, T sqrt(X)),
    column form (H T), diagonals with unit (Z, S, S^dag) and non-unit (T)
    ratios -- next to generic one-qubit gates (X, Y: zero diagonal; Haar) and CZ / dense two-qubit gates, with gates applied to
    the same qubit back to back (fused at F = 1) and across tile / thread
    bits."""
    rng = np.random.default_rng(seed)
    w = np.exp(1j * np.pi / 4)
    pool = [W.GATE_H, W.GATE_X_1_2, W.GATE_Y_1_2, W.GATE_T, W.GATE_Z, W.GATE_S, np.conj(W.GATE_S),
            W.GATE_T @ W.GATE_X_1_2, W.GATE_H @ W.GATE_T, W.GATE_X, W.GATE_Y, np.diag([1j, np.exp(0.3j)]),
            np.array([[1, 1j], [1j * w, w]]) / np.sqrt(2), W.haar_unitary(2, rng)]
    gates = []
    for t in range(m):
        r = rng.random()
        if r < 0.7:
            q = int(rng.integers(n if rng.random() < 0.5 else 6))
            M = pool[int(rng.integers(len(pool)))] * np.exp(1j * rng.uniform(0, 2 * np.pi))
            gates.append(W.Gate(t, "u", (q,), np.asarray(M, dtype=np.complex128)))
        elif r < 0.9:
            a, b = (int(x) for x in rng.choice(n, 2, replace=False))
            gates.append(W.Gate(t, "cz", (a, b), W.GATE_CZ))
        else:
            a, b = (int(x) for x in rng.choice(n, 2, replace=False))
            gates.append(W.Gate(t, "u2", (a, b), W.haar_unitary(4, rng)))
    return gates


@pytest.mark.parametrize("bits", [10, 12, 13, 14])
@pytest.mark.parametrize("lazy", [True, False])
def test_spec_structured_gates_vs_oracle(bits, lazy):
    """Structured-gate arithmetic (additions, one scalar per pass applied
    into the start state, a generic gate, a row-form gate or explicitly)
    against the oracle; with SV_OPT_PASS_SPEC = 0 the same circuit runs as
    dense matrices: both within the bound, the structured one with fewer
    operations."""
    n, m = 20, 260
    gates = _structured_circuit(n, m, seed=bits + 7 * lazy)
    ref = ref_c.run(n, gates)
    a, sa = _state(n, gates, 1, bits, jit=True, lazy_zero=lazy, spec=1)
    b, sb = _state(n, gates, 1, bits, jit=True, lazy_zero=lazy, spec=0)
    assert sa["n_jit_passes"] > 0
    assert sa["fma_apply"] < sb["fma_apply"]
    _check(n, layer_depth(gates), a, ref)
    _check(n, layer_depth(gates), b, ref)


def _monomial_circuit(n, m, seed):
    """Two-qubit monomial gates (one nonzero per row and column: fSim(pi/2,
    phi), iSWAP, SWAP, random permutations with unit (i^k) and non-unit
    phases) among structured and dense one-qubit gates and dense two-qubit
    gates, on register and tile bits in every order."""
    rng = np.random.default_rng(seed)
    iswap = np.array([[1, 0, 0, 0], [0, 0, 1j, 0], [0, 1j, 0, 0], [0, 0, 0, 1]])
    swap = np.array([[1, 0, 0, 0], [0, 0, 1, 0], [0, 1, 0, 0], [0, 0, 0, 1]])
    gates = []
    for t in range(m):
        r = rng.random()
        a, b = (int(x) for x in rng.choice(n if rng.random() < 0.5 else 7, 2, replace=False))
        if r < 0.45:
            kind = int(rng.integers(4))
            if kind == 0:
                M = W.gate_fsim(np.pi / 2, rng.uniform(0, 2 * np.pi))
            elif kind == 1:
                M = iswap
            elif kind == 2:
                M = swap
            else:
                P = np.eye(4)[rng.permutation(4)]
                ph = np.where(rng.random(4) < 0.5, 1j ** rng.integers(4, size=4), np.exp(1j * rng.uniform(0, 6.3, 4)))
                M = np.diag(ph) @ P
            gates.append(W.Gate(t, "mono", (a, b), np.asarray(M, dtype=np.complex128)))
        elif r < 0.55:
            gates.append(W.Gate(t, "u2", (a, b), W.haar_unitary(4, rng)))
        else:
            M = [W.GATE_H, W.GATE_X_1_2, W.GATE_T, W.haar_unitary(2, rng)][int(rng.integers(4))]
            gates.append(W.Gate(t, "u", (a,), np.asarray(M, dtype=np.complex128)))
    return gates


@pytest.mark.parametrize("bits", [11, 13, 14])
@pytest.mark.parametrize("lazy", [True, False])
def test_spec_monomial_two_qubit_gates_vs_oracle(bits, lazy):
    """Two-qubit monomial gates as copies, rotations and multiplies (reading
    R11) against the oracle, and fewer operations than the dense form."""
    n, m = 20, 220
    gates = _monomial_circuit(n, m, seed=bits + 3 * lazy)
    ref = ref_c.run(n, gates)
    a, sa = _state(n, gates, 1, bits, jit=True, lazy_zero=lazy, spec=1)
    b, sb = _state(n, gates, 1, bits, jit=True, lazy_zero=lazy, spec=0)
    assert sa["n_jit_passes"] > 0 and sa["fma_apply"] < sb["fma_apply"]
    _check(n, layer_depth(gates), a, ref)
    _check(n, layer_depth(gates), b, ref)


@pytest.mark.parametrize("n,d,bits", [(22, 14, 13), (20, 20, 11), (21, 12, 10), (22, 16, 14)])
def test_spec_rqc_vs_oracle(n, d, bits):
    """The RQC (H, sqrt(X), sqrt(Y), T, CZ) through the structured path,
    from the lazy |0...0> (product start) and a written one; the depth-20
    case has more passes than the pass scalar can hide (explicit multiply)."""
    gates = W.rqc(n, d, seed=3 * n + d)
    ref = ref_c.run(n, gates)
    for lazy in (True, False):
        a, sa = _state(n, gates, 1, bits, jit=True, lazy_zero=lazy, spec=1)
        _check(n, d, a, ref)


def test_spec_virtual_shards_and_sampling():
    """Sharded runs (passes with per-shard matrices stay dense) and the
    fused sampling bins on a structured final state: samples bit-exact to
    the oracle sampler on the GPU's final state."""
    from oracle import sample as osample
    n, d = 20, 14
    gates = W.rqc(n, d, seed=11)
    ref = ref_c.run(n, gates)
    for world in (1, 2, 4):
        a, sa = _state(n, gates, 1, 11, jit=True, world=world, spec=1)
        _check(n, d, a, ref)
    h = sv.sv_create(n)
    try:
        sv.sv_set_blocking(h, 12)
        sv.sv_run_circuit(h, gates, 1)
        got = sv.sv_sample(h, 21, 3000)
        psi = sv.sv_get_state(h, n)
    finally:
        sv.sv_destroy(h)
    assert np.array_equal(got, osample.sample(psi, 21, 3000)[0])
    _check(n, d, psi, ref)


def test_spec_30q_sampled_amplitudes():
    """Full size (30q D14, the bench step): the structured path within the
    north-star max-abs bound of the dense-matrix path on 2^16 sampled
    amplitudes, and with fewer fp32 operations."""
    n, d = 30, 14
    gates = W.rqc(n, d)
    idx = np.random.default_rng(6).integers(0, 1 << n, size=1 << 16).astype(np.uint64)
    out, ops = {}, {}
    for spec in (1, 0):
        h = sv.sv_create(n)
        try:
            sv.sv_set_option(h, sv.SV_OPT_PASS_SPEC, spec)
            st = sv.sv_run_circuit(h, gates, 1)
            out[spec] = sv.sv_amplitudes(h, idx)
            ops[spec] = st["fma_apply"]
        finally:
            sv.sv_destroy(h)
    err = np.abs(out[1].astype(np.complex128) - out[0].astype(np.complex128)).max()
    bound = 1e-5 * 2.0 ** (-n / 2) * d
    assert err <= bound, (err, bound)
    assert ops[1] < 0.6 * ops[0], ops


@pytest.mark.parametrize("pin", [4, 5])
@pytest.mark.parametrize("F", [1, 2])
def test_tile14_vs_oracle(pin, F):
    """14-qubit tiles (512 threads, 128 KB of shared memory; pass-specialised
    kernels only): RQC and mixed circuits from the lazy and a written
    |0...0>, with 128 B and 256 B runs, against the oracle; the generic
    kernel refuses them (sv_set_blocking(14) with SV_OPT_PASS_JIT 0 runs 13)."""
    n, d = 21, 14
    for gates in (W.rqc(n, d, seed=pin + F), _mixed_circuit(n, 160, seed=9 * pin + F)):
        ref = ref_c.run(n, gates)
        for lazy in (True, False):
            h = sv.sv_create(n)
            try:
                sv.sv_set_option(h, sv.SV_OPT_PASS_PIN, pin)
                sv.sv_set_blocking(h, 14)
                if not lazy:
                    sv.sv_device_ptr(h)
                st = sv.sv_run_circuit(h, gates, F)
                psi = sv.sv_get_state(h, n)
            finally:
                sv.sv_destroy(h)
            assert st["block_bits"] == 14 and st["n_jit_passes"] == st["n_passes"] > 0, st
            _check(n, layer_depth(gates), psi, ref)
    h = sv.sv_create(n)
    try:
        sv.sv_set_option(h, sv.SV_OPT_PASS_JIT, 0)
        sv.sv_set_blocking(h, 14)
        st = sv.sv_run_circuit(h, W.rqc(n, d), 1)
        assert st["block_bits"] == 13, st
    finally:
        sv.sv_destroy(h)
