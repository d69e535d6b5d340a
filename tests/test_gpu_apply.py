"""GPU parity of the apply kernels through the C ABI.

Every input is seeded (workloads/); the expected values come only from the
oracle.  A single fused k-qubit apply is compared element by element with
the oracle's complex128 apply of the SAME complex64 matrix to the SAME
complex64 state, against the fp32 error bound of the kernels' arithmetic
|dy_r| <= (4 (2^k + 1) + 2) u sum_c |M_rc||a_c|   (u = 2^-24),
derived in DESIGN.md "Tolerances" for both the 3-multiplication (Gauss) form
used for k <= 5 and the 4-FMA form used for k = 6.  Dense k = 5 (k = 6) gates
on states of >= 13 (14) qubits run on the exact int8-slice tensor-core path, whose
inputs are rounded to 22 bits relative to the group-row / matrix-column
maximum, whose dropped cross products are bounded per real product by
2^-19 of those maxima, and whose per-column norm restoration rescales every
column by at most 2^-22; the bound then adds
2^(k+1) (2^-19 + 2^-20) max_group|a| max|M|.
"""
import numpy as np
import pytest

import paper_conf_sc_markidis23_b200 as sv
from oracle import sv as osv
from workloads import rqc as W

pytestmark = pytest.mark.gpu

U32 = 2.0 ** -24


def _apply_gpu(n, psi, qubits, M):
    h = sv.sv_create(n)
    try:
        sv.sv_set_state(h, psi)
        sv.sv_apply_fused(h, list(qubits), M)
        return sv.sv_get_state(h, n)
    finally:
        sv.sv_destroy(h)


def _check_apply(n, qubits, seed):
    k = len(qubits)
    rs = np.random.default_rng(seed)
    M = W.haar_unitary(1 << k, rs).astype(np.complex64)
    psi = W.random_state_c64(n, seed + 1)
    got = _apply_gpu(n, psi, qubits, M)
    ref = osv.apply_gate(psi.astype(np.complex128), n, list(qubits), M.astype(np.complex128))
    bound = osv.apply_gate(np.abs(psi).astype(np.complex128), n, list(qubits), np.abs(M).astype(np.complex128)).real
    err = np.abs(got.astype(np.complex128) - ref)
    tol = (4.0 * ((1 << k) + 1) + 2.0) * U32 * bound
    if k >= 5:
        t = np.abs(psi).astype(np.float64).reshape((2,) * n)
        gmax = np.broadcast_to(np.max(t, axis=tuple(n - 1 - q for q in qubits), keepdims=True), t.shape).reshape(-1)
        tol = tol + (2 << k) * (2.0 ** -19 + 2.0 ** -20) * gmax * float(np.abs(M).max())
    assert np.all(err <= tol + 1e-30), (qubits, float((err / (tol + 1e-30)).max()))


# qubit classes: all-high, with qubit 0, low in {1,2,3}, mixed, unsorted order
CASES = {
    1: [(5,), (0,), (1,), (2,), (3,), (4,), (11,)],
    2: [(4, 9), (0, 7), (1, 2), (3, 10), (8, 0), (2, 1), (11, 4)],
    3: [(4, 6, 10), (0, 1, 2), (1, 5, 9), (9, 3, 0), (0, 4, 11), (2, 3, 8)],
    4: [(4, 5, 6, 7), (0, 1, 2, 3), (1, 6, 8, 11), (10, 0, 3, 5), (2, 4, 9, 7), (0, 5, 8, 11)],
    5: [(4, 5, 6, 8, 10), (0, 1, 2, 3, 4), (1, 5, 7, 9, 11), (11, 0, 6, 2, 8), (0, 4, 6, 8, 10)],
    6: [(4, 5, 6, 7, 8, 9), (0, 1, 2, 3, 4, 5), (0, 2, 5, 7, 9, 11), (1, 4, 6, 8, 10, 11), (11, 3, 7, 0, 9, 5)],
}


@pytest.mark.parametrize("k", sorted(CASES))
@pytest.mark.parametrize("n", [12, 17])
def test_apply_parity(k, n):
    for i, qs in enumerate(CASES[k]):
        _check_apply(n, qs, seed=100 * k + i + n)


@pytest.mark.parametrize("k", [1, 2, 4, 6])
def test_apply_parity_random_qubits_n22(k):
    rs = np.random.default_rng(k)
    for t in range(3):
        qs = [int(x) for x in rs.choice(22, size=k, replace=False)]
        _check_apply(22, qs, seed=1000 + 10 * k + t)


@pytest.mark.parametrize("n,k", [(1, 1), (2, 2), (3, 1), (3, 3), (4, 2), (5, 5), (6, 6), (7, 6)])
def test_apply_tiny_states(n, k):
    rs = np.random.default_rng(n * 10 + k)
    for t in range(4):
        qs = [int(x) for x in rs.choice(n, size=k, replace=False)]
        _check_apply(n, qs, seed=7 * n + t)


@pytest.mark.parametrize("k", [1, 2, 3, 4, 5, 6])
def test_identity_is_bit_exact(k):
    n = 16
    psi = W.random_state_c64(n, 3)
    for qs in CASES[k][:3]:
        got = _apply_gpu(n, psi, qs, np.eye(1 << k, dtype=np.complex64))
        assert np.array_equal(got, psi)


def test_permutations_are_exact():
    n = 15
    psi = W.random_state_c64(n, 4)
    for qs, M in (((3,), W.GATE_X), ((0, 9), W.GATE_SWAP), ((2, 1), W.GATE_SWAP), ((5, 0), W.GATE_CX),
                  ((1, 3), W.GATE_CX)):
        got = _apply_gpu(n, psi, qs, M.astype(np.complex64))
        ref = osv.apply_gate(psi.astype(np.complex128), n, list(qs), M).astype(np.complex64)
        assert np.array_equal(got, ref), qs


@pytest.mark.parametrize("k", [1, 2, 3, 4, 5, 6])
def test_monomial_matrices_are_exact(k):
    """Diagonal / permuted-diagonal matrices with entries in {+-1, +-i}
    (CZ-like) give exactly permuted, sign/phase-flipped amplitudes."""
    n = 14
    psi = W.random_state_c64(n, 5 + k)
    rs = np.random.default_rng(k)
    D = 1 << k
    for qs in CASES[k][:3]:
        perm = rs.permutation(D)
        ph = np.array([1, -1, 1j, -1j])[rs.integers(0, 4, size=D)]
        M = np.zeros((D, D), np.complex64)
        M[np.arange(D), perm] = ph
        got = _apply_gpu(n, psi, qs, M)
        ref = osv.apply_gate(psi.astype(np.complex128), n, list(qs), M.astype(np.complex128)).astype(np.complex64)
        assert np.array_equal(got, ref), qs


def test_apply_errors():
    h = sv.sv_create(8)
    try:
        with pytest.raises(sv.SVError) as e:
            sv.sv_apply_fused(h, [1, 1], np.eye(4))
        assert e.value.code == sv.SV_EINVAL
        with pytest.raises(sv.SVError) as e:
            sv.sv_apply_fused(h, [8], np.eye(2))
        assert e.value.code == sv.SV_EINVAL
        with pytest.raises(sv.SVError) as e:
            sv.sv_apply_fused(h, list(range(7)), np.eye(128))
        assert e.value.code == sv.SV_EINVAL
    finally:
        sv.sv_destroy(h)
