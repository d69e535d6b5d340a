"""GPU parity of whole circuits (fuser + dispatcher + kernels), sampling,
amplitudes and the virtual-shard exchange path, against the oracle.

Tolerances are the north star's (BASELINE.json): fidelity
|<psi_gpu|psi_ref>|^2 >= 1 - 1e-5 and max |psi_gpu - psi_ref| <=
1e-5 * 2^(-n/2) * depth.  Sampling is bit-exact against oracle/sample.py on a
seeded complex64 state (S5 is integer arithmetic).
"""
import numpy as np
import pytest

import paper_conf_sc_markidis23_b200 as sv
from oracle import ref_c
from oracle import sample as osample
from oracle import sv as osv
from workloads import rqc as W

pytestmark = pytest.mark.gpu


def _run(n, gates, F, world=1):
    h = sv.sv_create_ex(n, world=world, virtual_shards=True) if world > 1 else sv.sv_create(n)
    try:
        st = sv.sv_run_circuit(h, gates, F)
        return sv.sv_get_state(h, n), st
    finally:
        sv.sv_destroy(h)


def _check(n, depth, got, ref):
    got = got.astype(np.complex128)
    fid = osv.fidelity(got, ref)
    err = np.abs(got - ref).max()
    assert fid >= 1 - 1e-5, fid
    assert err <= osv.max_abs_bound(n, depth), (err, osv.max_abs_bound(n, depth))


@pytest.mark.parametrize("F", range(7))
def test_rqc12_all_fusion_sizes(F):
    gates = W.rqc(12, 14)
    got, st = _run(12, gates, F)
    _check(12, 14, got, osv.simulate(12, gates))
    assert st["n_fused"] == [121, 85, 34, 19, 15, 11, 8][F]


@pytest.mark.parametrize("n,d,F", [(16, 14, 2), (20, 14, 4), (22, 16, 3), (24, 14, 5), (25, 14, 6), (26, 14, 4)])
def test_rqc_medium(n, d, F):
    gates = W.rqc(n, d, seed=n)
    got, _ = _run(n, gates, F)
    _check(n, d, got, ref_c.run(n, gates))


def test_random_circuit_unsorted_two_qubit_gates():
    n = 18
    gates = W.random_circuit(n, 150, 9, two_qubit_frac=0.5)
    ref = ref_c.run(n, gates)
    for F in (0, 2, 4, 6):
        got, _ = _run(n, gates, F)
        _check(n, 10, got, ref)


@pytest.mark.parametrize("world", [2, 4, 8])
@pytest.mark.parametrize("n,F", [(16, 2), (16, 4), (19, 5), (19, 6)])
def test_virtual_shards_match_oracle(world, n, F):
    """F = 5, 6 at 19 qubits: 16-18 local qubits, so the int8 tensor-core
    apply runs inside the shards between exchanges."""
    gates = W.rqc(n, 14, seed=world)
    got, st = _run(n, gates, F, world=world)
    _check(n, 14, got, ref_c.run(n, gates))
    assert st["n_exchanges"] >= 1


@pytest.mark.parametrize("bits", [0, 10, 12, 13])
@pytest.mark.parametrize("F", [1, 2, 4])
def test_blocked_passes_match_oracle(bits, F):
    """Cache-blocked passes (sv_set_blocking) against the oracle."""
    n, d = 20, 14
    gates = W.rqc(n, d, seed=F + bits)
    h = sv.sv_create(n)
    try:
        sv.sv_set_blocking(h, bits)
        c = sv.sv_circuit_create(h, gates, F)
        sv.sv_circuit_run_device(h, c)
        sv.sv_synchronize(h)
        got = sv.sv_get_state(h, n)
        sv.sv_circuit_destroy(c)
    finally:
        sv.sv_destroy(h)
    _check(n, d, got, ref_c.run(n, gates))


def test_amplitudes_match_state():
    n = 20
    gates = W.rqc(n, 12)
    h = sv.sv_create(n)
    try:
        sv.sv_run_circuit(h, gates, 4)
        full = sv.sv_get_state(h, n)
        idx = np.random.default_rng(0).integers(0, 1 << n, size=1000).astype(np.uint64)
        assert np.array_equal(sv.sv_amplitudes(h, idx), full[idx.astype(np.int64)])
        with pytest.raises(sv.SVError):
            sv.sv_amplitudes(h, np.array([1 << n], dtype=np.uint64))
    finally:
        sv.sv_destroy(h)


@pytest.mark.parametrize("n", [2, 3, 5, 6, 11, 20])
def test_sampler_bit_exact(n):
    psi = W.random_state_c64(n, 50 + n)
    ref, _ = osample.sample(psi, 1234, 5000)
    h = sv.sv_create(n)
    try:
        sv.sv_set_state(h, psi)
        got = sv.sv_sample(h, 1234, 5000)
    finally:
        sv.sv_destroy(h)
    assert np.array_equal(got, ref)


def test_sampler_rqc12_appendix_c_state():
    """Sample the oracle's fp64 RQC-12 state rounded to complex64 (S5 vectors)."""
    psi = osv.simulate(12, W.rqc(12, 14)).astype(np.complex64)
    h = sv.sv_create(12)
    try:
        sv.sv_set_state(h, psi)
        got = sv.sv_sample(h, 1, 8)
    finally:
        sv.sv_destroy(h)
    assert [int(x) for x in got] == [2318, 3050, 3966, 1826, 1826, 3132, 3597, 2133]


@pytest.mark.parametrize("world", [2, 4, 8])
def test_sampler_sharded_bit_exact(world):
    n = 14
    psi = W.random_state_c64(n, 77)
    ref, _ = osample.sample(psi, 99, 3000)
    h = sv.sv_create_ex(n, world=world, virtual_shards=True)
    try:
        sv.sv_set_state(h, psi)
        got = sv.sv_sample(h, 99, 3000)
    finally:
        sv.sv_destroy(h)
    assert np.array_equal(got, ref)


def test_sampler_after_sharded_circuit_statistics():
    n, d = 14, 12
    gates = W.rqc(n, d)
    p = osample.exact_probabilities(ref_c.run(n, gates))
    h = sv.sv_create_ex(n, world=4, virtual_shards=True)
    try:
        sv.sv_run_circuit(h, gates, 4)
        s = sv.sv_sample(h, 5, 200000)
    finally:
        sv.sv_destroy(h)
    cnt = np.bincount(s.astype(np.int64), minlength=1 << n)
    # chi-square on the 64 coarse bins of the top 6 bits
    P = p.reshape(64, -1).sum(1)
    C = cnt.reshape(64, -1).sum(1)
    chi2 = float(np.sum((C - s.size * P) ** 2 / (s.size * P)))
    assert chi2 < 63 + 6 * np.sqrt(2 * 63)


def test_sampler_rejects_zero_state():
    h = sv.sv_create(6)
    try:
        sv.sv_set_state(h, np.zeros(64, np.complex64))
        with pytest.raises(sv.SVError) as e:
            sv.sv_sample(h, 1, 10)
        assert e.value.code == sv.SV_EINVAL
    finally:
        sv.sv_destroy(h)


def test_prepared_circuit_and_reset():
    n = 18
    gates = W.rqc(n, 14)
    ref = ref_c.run(n, gates)
    h = sv.sv_create(n)
    try:
        c = sv.sv_circuit_create(h, gates, 4)
        for _ in range(2):
            sv.sv_reset(h)
            sv.sv_circuit_run_device(h, c)
            sv.sv_synchronize(h)
            _check(n, 14, sv.sv_get_state(h, n), ref)
        sv.sv_circuit_destroy(c)
    finally:
        sv.sv_destroy(h)


def layer_depth(gates):
    """Number of moments of the ASAP schedule (a gate starts after the last
    gate on any of its qubits): the "depth" of the north-star max-abs bound
    for circuits that are not RQC layers."""
    level = {}
    depth = 0
    for g in gates:
        d = 1 + max(level.get(q, 0) for q in g.qubits)
        for q in g.qubits:
            level[q] = d
        depth = max(depth, d)
    return depth


def _mixed_circuit(n, m, seed):
    """Dense 1q/2q Haar gates, diagonal gates (T, S, Z, CP(phi)), CZ and
    permutations (CX, SWAP), biased towards qubits 0..4 so that the
    register-blocked passes see tile bit 0 in and out of the register set,
    all three gate kinds (dense, diagonal, CZ-like) and both store paths."""
    rs = np.random.default_rng(seed)
    fixed = {"t": W.GATE_T, "s": W.GATE_S, "z": W.GATE_Z, "cz": W.GATE_CZ, "cx": W.GATE_CX, "swap": W.GATE_SWAP}
    gates = []
    for i in range(m):
        kind = rs.choice(["u1", "u2", "t", "s", "z", "cz", "cp", "cx", "swap"])
        k = 2 if kind in ("u2", "cz", "cp", "cx", "swap") else 1
        pool = np.arange(n) if rs.random() < 0.5 else np.arange(min(n, 6))
        qs = tuple(int(x) for x in rs.choice(pool, size=k, replace=False))
        if kind in ("u1", "u2"):
            mat = W.haar_unitary(1 << k, rs)
        elif kind == "cp":
            mat = W.gate_cp(float(rs.uniform(0, 2 * np.pi)))
        else:
            mat = fixed[kind]
        gates.append(W.Gate(i, str(kind), qs, mat))
    return gates


@pytest.mark.parametrize("bits", [10, 11, 12, 13])
@pytest.mark.parametrize("F", [1, 2])
def test_register_blocked_mixed_kinds(bits, F):
    """Register-blocked passes (apply_rpass) on a circuit mixing dense,
    diagonal and CZ-like fused gates, against the oracle."""
    n, m = 18, 160
    gates = _mixed_circuit(n, m, seed=100 * F + bits)
    h = sv.sv_create(n)
    try:
        sv.sv_set_blocking(h, bits)
        c = sv.sv_circuit_create(h, gates, F)
        st = sv.sv_circuit_stats(c)
        assert st["n_passes"] > 0 and st["block_bits"] == bits
        sv.sv_circuit_run_device(h, c)
        sv.sv_synchronize(h)
        got = sv.sv_get_state(h, n)
        sv.sv_circuit_destroy(c)
    finally:
        sv.sv_destroy(h)
    _check(n, layer_depth(gates), got, ref_c.run(n, gates))


def test_blocking_auto_default():
    """Default (-1 = auto): blocked passes for max_fused <= 2 at n >= 20,
    one launch per fused gate otherwise."""
    n = 20
    gates = W.rqc(n, 10)
    h = sv.sv_create(n)
    try:
        for F, blocked in [(1, True), (2, True), (3, False), (4, False)]:
            c = sv.sv_circuit_create(h, gates, F)
            assert (sv.sv_circuit_stats(c)["n_passes"] > 0) == blocked
            sv.sv_circuit_destroy(c)
    finally:
        sv.sv_destroy(h)


@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("F", [1, 2])
def test_virtual_shards_blocked_passes(world, F):
    """Register-blocked passes inside every shard between the exchanges."""
    n = 18
    gates = W.rqc(n, 14, seed=7 + world)
    h = sv.sv_create_ex(n, world=world, virtual_shards=True)
    try:
        sv.sv_set_blocking(h, 11)
        st = sv.sv_run_circuit(h, gates, F)
        got = sv.sv_get_state(h, n)
    finally:
        sv.sv_destroy(h)
    assert st["n_exchanges"] >= 1 and st["n_passes"] >= 1
    _check(n, 14, got, ref_c.run(n, gates))


def test_reset_is_exact_for_every_reader():
    """sv_reset writes |0...0> lazily (complex64): every reader sees it --
    get_state, amplitudes, sampling, a per-gate apply, and a circuit whose
    first register-blocked pass synthesises the zero tiles."""
    n = 20
    rs = np.random.default_rng(3)
    h = sv.sv_create(n)
    try:
        e0 = np.zeros(1 << n, dtype=np.complex64)
        e0[0] = 1
        sv.sv_set_state(h, W.random_state_c64(n, 2))
        sv.sv_reset(h)
        assert np.array_equal(sv.sv_get_state(h, n), e0)
        sv.sv_set_state(h, W.random_state_c64(n, 2))
        sv.sv_reset(h)
        assert sv.sv_amplitudes(h, np.array([0, 1, 5], dtype=np.uint64)).tolist() == [1, 0, 0]
        sv.sv_reset(h)
        assert np.all(sv.sv_sample(h, 1, 100) == 0)
        sv.sv_reset(h)
        M = W.haar_unitary(2, rs).astype(np.complex64)
        sv.sv_apply_fused(h, [7], M)
        got = sv.sv_get_state(h, n)
        assert abs(got[0] - M[0, 0]) < 1e-6 and abs(got[1 << 7] - M[1, 0]) < 1e-6
        gates = W.rqc(n, 8)
        sv.sv_set_state(h, W.random_state_c64(n, 4))
        sv.sv_reset(h)
        c = sv.sv_circuit_create(h, gates, 1)
        assert sv.sv_circuit_stats(c)["n_passes"] > 0
        sv.sv_circuit_run_device(h, c)
        sv.sv_synchronize(h)
        got = sv.sv_get_state(h, n)
        sv.sv_circuit_destroy(c)
    finally:
        sv.sv_destroy(h)
    _check(n, 8, got, ref_c.run(n, gates))


# ------------------------------------------------ Sycamore-style RQC (NEXT-4)
@pytest.mark.parametrize("F", range(7))
def test_sycamore_all_fusion_sizes(F):
    """fSim(pi/2, pi/6) + sqrt(X/Y/W) circuits: the default path for each
    fusion size (register-blocked passes for F <= 2 at n >= 20)."""
    n, cyc = 22, 12
    gates = W.sycamore_rqc(n, cyc, seed=F)
    got, st = _run(n, gates, F)
    _check(n, 2 * cyc + 1, got, ref_c.run(n, gates))


@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("F", [1, 4])
def test_sycamore_virtual_shards(world, F):
    n, cyc = 20, 10
    gates = W.sycamore_rqc(n, cyc, seed=world)
    got, st = _run(n, gates, F, world=world)
    assert st["n_exchanges"] >= 1
    _check(n, 2 * cyc + 1, got, ref_c.run(n, gates))


# ------------------------------------ diagonal exchange skip (NEXT-4, R10)
@pytest.mark.parametrize("world", [2, 4, 8])
@pytest.mark.parametrize("F,bits", [(1, 11), (2, 11), (1, 0), (4, 0)])
def test_diag_skip_virtual_shards(world, F, bits):
    """Fused gates block-diagonal in a global qubit (CZ-like at F = 1) run as
    per-shard blocks without an exchange: fewer exchanges, same state as the
    oracle, on register-blocked passes (bits 11) and per-gate launches."""
    n, d = 18, 14
    gates = W.rqc(n, d, seed=world + F)
    ref = ref_c.run(n, gates)
    out = {}
    for skip in (1, 0):
        h = sv.sv_create_ex(n, world=world, virtual_shards=True)
        try:
            sv.sv_set_option(h, sv.SV_OPT_DIAG_SKIP, skip)
            sv.sv_set_blocking(h, bits)
            st = sv.sv_run_circuit(h, gates, F)
            got = sv.sv_get_state(h, n)
        finally:
            sv.sv_destroy(h)
        _check(n, d, got, ref)
        out[skip] = st["n_exchanges"]
    # n_exchanges includes the final canonicalisation exchange (R3)
    assert out[1] <= out[0]
    if F == 1 and world >= 4:
        assert out[1] < out[0], out
