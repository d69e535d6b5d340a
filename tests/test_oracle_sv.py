"""Pins for the S0 oracle simulator (oracle/sv.py, oracle/sv_ref.c).

Every check here fixes the oracle against something other than itself:
brute-force dense matrices (Fig. 4, L84-92), closed forms (H^n,
GHZ, QFT of a basis state), norm preservation (L76), the inverse circuit,
and the gate-table identities.
"""
import json
import math
import os

import numpy as np
import pytest

from oracle import ref_c, sv
from workloads import rqc as W

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "appendix_c.json")))


# ---------------------------------------------------------------- gate table
@pytest.mark.parametrize("name", ["h", "t", "x_1_2", "y_1_2", "cz", "x", "cx", "swap"])
def test_gate_unitary(name):
    g = W.GATE_TABLE[name]
    assert np.abs(g.conj().T @ g - np.eye(g.shape[0])).max() < 1e-15


def test_gate_identities():
    I2, I4 = np.eye(2), np.eye(4)
    assert np.abs(W.GATE_H @ W.GATE_H - I2).max() < 1e-15
    assert np.abs(W.GATE_X_1_2 @ W.GATE_X_1_2 - W.GATE_X).max() < 1e-15
    assert np.abs(W.GATE_Y_1_2 @ W.GATE_Y_1_2 - W.GATE_Y).max() < 1e-15
    assert np.abs(W.GATE_T @ W.GATE_T - W.GATE_S).max() < 1e-15
    assert np.abs(np.linalg.matrix_power(W.GATE_T, 8) - I2).max() < 1e-14
    assert np.abs(W.GATE_CZ @ W.GATE_CZ - I4).max() == 0


# ------------------------------------------------------------- brute force
def test_two_brute_forces_agree():
    """Fig. 4 built with np.kron equals the element-wise definition."""
    rs = np.random.default_rng(3)
    for n in (1, 3, 5):
        for q in range(n):
            g = W.haar_unitary(2, rs)
            assert np.abs(sv.kron_single_qubit(n, q, g) - sv.full_gate_matrix(n, [q], g)).max() < 1e-15


def test_fig4_three_qubit_structure():
    """PAPER.md Fig. 4: G on the highest qubit (0x4) of 3 is block G (x) I_4;
    on the lowest (0x1) it is block-diagonal I_4 (x) G."""
    g = np.array([[1, 2], [3, 4]], dtype=np.complex128)
    hi = sv.full_gate_matrix(3, [2], g)
    lo = sv.full_gate_matrix(3, [0], g)
    assert np.array_equal(hi, np.kron(g, np.eye(4)))
    assert np.array_equal(lo, np.kron(np.eye(4), g))


def test_cx_convention():
    """CX with qubits (control, target) maps index 1 <-> 3 (bit 0 = control)."""
    for ctrl, tgt in ((0, 1), (1, 0)):
        for basis in range(4):
            psi = np.zeros(4, complex)
            psi[basis] = 1
            out = sv.apply_gate(psi, 2, [ctrl, tgt], W.GATE_CX)
            expect = basis ^ (1 << tgt) if (basis >> ctrl) & 1 else basis
            assert out[expect] == 1 and np.count_nonzero(out) == 1


@pytest.mark.parametrize("n,seed", [(4, 0), (7, 1), (10, 2)])
def test_simulate_vs_brute_force(n, seed):
    gates = W.random_circuit(n, 40, seed)
    psi0 = W.random_state_c64(n, seed + 100).astype(np.complex128)
    u = sv.full_circuit_unitary(n, gates)
    assert np.abs(sv.simulate(n, gates, psi0) - u @ psi0).max() < 1e-12


@pytest.mark.parametrize("k", [1, 2, 3, 4, 5, 6])
def test_apply_k_qubit_vs_brute_force(k):
    rs = np.random.default_rng(10 + k)
    n = 8
    for trial in range(3):
        qs = [int(x) for x in rs.choice(n, size=k, replace=False)]  # unsorted on purpose
        g = W.haar_unitary(1 << k, rs)
        psi = W.random_state_c64(n, trial).astype(np.complex128)
        ref = sv.full_gate_matrix(n, qs, g) @ psi
        assert np.abs(sv.apply_gate(psi, n, qs, g) - ref).max() < 1e-13
        c = psi.copy()
        ref_c.apply(c, n, qs, g)
        assert np.abs(c - ref).max() < 1e-13


def test_rqc12_unitary_brute_force():
    gates = W.rqc(10, 8, seed=5)
    u = sv.full_circuit_unitary(10, gates)
    psi = sv.simulate(10, gates)
    assert np.abs(psi - u[:, 0]).max() < 1e-12
    assert np.abs(u.conj().T @ u - np.eye(1 << 10)).max() < 1e-12


# -------------------------------------------------------- controlled gates
def test_controlled_gate_vs_brute_force():
    rs = np.random.default_rng(21)
    n = 7
    for controls, targets in (([0], [1]), ([3], [0]), ([6, 2], [4]), ([1, 5], [0, 3]), ([0, 1, 2], [6]),
                              ([4], [2, 5, 6])):
        g = W.haar_unitary(1 << len(targets), rs)
        psi = W.random_state_c64(n, 5).astype(np.complex128)
        ref = sv.controlled_full_matrix(n, controls, targets, g) @ psi
        assert np.abs(sv.apply_controlled(psi, n, controls, targets, g) - ref).max() < 1e-14


def test_controlled_x_is_cx_and_controls_commute():
    psi = W.random_state_c64(5, 2).astype(np.complex128)
    # CX (qubits[0] = control) == controlled-X
    assert np.abs(sv.apply_controlled(psi, 5, [1], [3], W.GATE_X) - sv.apply_gate(psi, 5, [1, 3], W.GATE_CX)).max() == 0
    # CZ is symmetric: control 0 target 2 == control 2 target 0
    a = sv.apply_controlled(psi, 5, [0], [2], W.GATE_Z)
    b = sv.apply_controlled(psi, 5, [2], [0], W.GATE_Z)
    assert np.abs(a - b).max() == 0


# ------------------------------------------------------------- closed forms
@pytest.mark.parametrize("n", [1, 5, 12])
def test_hadamard_layer_uniform(n):
    gates = [W.Gate(0, "h", (q,), W.GATE_H) for q in range(n)]
    psi = sv.simulate(n, gates)
    assert np.abs(psi - 2.0 ** (-n / 2)).max() < 1e-14
    assert np.abs(ref_c.run(n, gates) - 2.0 ** (-n / 2)).max() < 1e-14


@pytest.mark.parametrize("n", [2, 6, 13])
def test_ghz(n):
    gates = [W.Gate(0, "h", (0,), W.GATE_H)]
    gates += [W.Gate(i, "cx", (i - 1, i), W.GATE_CX) for i in range(1, n)]
    for psi in (sv.simulate(n, gates), ref_c.run(n, gates)):
        assert abs(psi[0] - 1 / math.sqrt(2)) < 1e-15
        assert abs(psi[-1] - 1 / math.sqrt(2)) < 1e-15
        assert np.count_nonzero(psi) == 2


def _qft_gates(n):
    gates = []
    for j in range(n - 1, -1, -1):
        gates.append(W.Gate(0, "h", (j,), W.GATE_H))
        for k in range(j - 1, -1, -1):
            gates.append(W.Gate(0, "cp", (k, j), W.gate_cp(math.pi / 2 ** (j - k))))
    for j in range(n // 2):
        gates.append(W.Gate(0, "swap", (j, n - 1 - j), W.GATE_SWAP))
    return gates


@pytest.mark.parametrize("n,x", [(3, 5), (6, 37), (9, 300)])
def test_qft_of_basis_state(n, x):
    psi0 = np.zeros(1 << n, complex)
    psi0[x] = 1
    y = np.arange(1 << n)
    expect = np.exp(2j * np.pi * x * y / 2 ** n) / 2 ** (n / 2)
    assert np.abs(sv.simulate(n, _qft_gates(n), psi0) - expect).max() < 1e-13
    c = psi0.copy()
    ref_c.run(n, _qft_gates(n), c)
    assert np.abs(c - expect).max() < 1e-13


# ------------------------------------------------------------- invariants
def test_norm_and_inverse_circuit():
    n = 14
    gates = W.rqc(n, 14, seed=7)
    psi = ref_c.run(n, gates)
    assert abs(np.vdot(psi, psi).real - 1) < 1e-12
    back = ref_c.run(n, W.inverse_circuit(gates), psi.copy())
    assert abs(back[0] - 1) < 1e-12 and np.abs(back[1:]).max() < 1e-12


def test_c_oracle_matches_numpy_oracle():
    for n, d, s in ((12, 14, 2023), (16, 10, 0)):
        gates = W.rqc(n, d, s)
        assert np.abs(ref_c.run(n, gates) - sv.simulate(n, gates)).max() < 1e-13


def test_c_oracle_rejects_bad_args():
    psi = ref_c.zero_state(3)
    with pytest.raises(ValueError):
        ref_c.apply(psi, 3, [0, 0], np.eye(4))
    with pytest.raises(ValueError):
        ref_c.apply(psi, 3, [3], np.eye(2))


# ------------------------------------------------------ regression vectors
def test_appendix_c_rqc12_state():
    g = GOLD["rqc12"]
    psi = sv.simulate(g["n"], W.rqc(g["n"], g["depth"], g["seed"]))
    for i, (re, im) in g["psi"].items():
        assert abs(psi[int(i)] - complex(re, im)) < 1e-15
    assert abs((1 << g["n"]) * np.sum(np.abs(psi) ** 4) - g["two_n_sum_p2"]) < 1e-6


# ------------------------------------------- Sycamore-style gates (NEXT-4)
@pytest.mark.parametrize("name", ["hz_1_2", "fs"])
def test_sycamore_gates_unitary(name):
    g = W.GATE_TABLE[name]
    assert np.abs(g.conj().T @ g - np.eye(g.shape[0])).max() < 1e-15


def test_sycamore_gate_identities():
    """sqrt(W)^2 = W with W = (X + Y)/sqrt(2) (so W^2 = I); the fSim closed
    form: fSim(0, 0) = I, fSim(theta, phi) maps |01> -> cos|01> - i sin|10>,
    |11> -> e^{-i phi}|11> and is symmetric in its two qubits."""
    Wm = (W.GATE_X + W.GATE_Y) / math.sqrt(2)
    assert np.abs(W.GATE_W - Wm).max() < 1e-15
    assert np.abs(W.GATE_W @ W.GATE_W - np.eye(2)).max() < 1e-15
    assert np.abs(W.GATE_SQRT_W @ W.GATE_SQRT_W - W.GATE_W).max() < 1e-15
    assert np.abs(W.gate_fsim(0, 0) - np.eye(4)).max() == 0
    th, ph = 0.7, 1.3
    f = W.gate_fsim(th, ph)
    e01 = np.array([0, 1, 0, 0], complex)
    assert np.abs(f @ e01 - np.array([0, math.cos(th), -1j * math.sin(th), 0])).max() < 1e-15
    assert abs(f[3, 3] - np.exp(-1j * ph)) < 1e-15
    swap = W.GATE_SWAP
    assert np.abs(swap @ f @ swap - f).max() < 1e-15
    # the Sycamore gate: iSWAP-like exchange with a pi/6 conditional phase
    syc = W.GATE_FSIM_SYC
    assert abs(syc[1, 2] + 1j) < 1e-15 and abs(syc[1, 1]) < 1e-15 and abs(syc[3, 3] - np.exp(-1j * np.pi / 6)) < 1e-15


def test_sycamore_circuit_brute_force():
    """A 9-qubit, 6-cycle Sycamore-style circuit: oracle state = first column
    of the brute-force circuit unitary; the C oracle agrees."""
    gates = W.sycamore_rqc(9, 6, seed=4)
    u = sv.full_circuit_unitary(9, gates)
    psi = sv.simulate(9, gates)
    assert np.abs(psi - u[:, 0]).max() < 1e-12
    assert np.abs(ref_c.run(9, gates) - psi).max() < 1e-13
