"""S0 oracle simulator (TEST INFRASTRUCTURE ONLY -- see oracle/__init__.py).

PAPER.md L69 (§2.2): the state of n qubits is a complex vector of length 2^n;
|c_i|^2 is the probability of |i>.  L71-80 (Fig. 3): a gate acts as psi' = G psi.
L84-92 (Fig. 4): the full-system matrix is G tensored with identities, never
stored -- "a matrix-free approach is employed, and the operation is performed
in place".  Index convention: qubit q is bit q of i;
bit b of a gate's matrix index belongs to qubits[b].

Everything is complex128 and unfused: one gate at a time in circuit order.
"""
from __future__ import annotations

from typing import Sequence

import numpy as np


def zero_state(n: int) -> np.ndarray:
    """|0...0>: psi[0] = 1 (PAPER.md L69, L131 'setting states')."""
    psi = np.zeros(1 << n, dtype=np.complex128)
    psi[0] = 1.0
    return psi


def apply_gate(psi: np.ndarray, n: int, qubits: Sequence[int], g: np.ndarray) -> np.ndarray:
    """psi' = (G on `qubits`, identity elsewhere) psi, matrix-free.

    The state is viewed as an n-axis tensor with axis n-1-q for qubit q; the
    gate as a 2k-axis tensor (row bits k-1..0, column bits k-1..0).  The
    contraction over the gate's column axes is exactly
    psi'[.. r ..] = sum_c G[r, c] psi[.. c ..] of L80 / Fig. 3, generalised to k
    qubits.  Returns a new array (complex128).
    """
    k = len(qubits)
    assert len(set(qubits)) == k and all(0 <= q < n for q in qubits)
    g = np.asarray(g, dtype=np.complex128).reshape((2,) * (2 * k))
    t = np.asarray(psi, dtype=np.complex128).reshape((2,) * n)
    col_axes = [k + (k - 1 - b) for b in range(k)]
    st_axes = [n - 1 - qubits[b] for b in range(k)]
    res = np.tensordot(g, t, axes=(col_axes, st_axes))
    res = np.moveaxis(res, [k - 1 - b for b in range(k)], st_axes)
    return np.ascontiguousarray(res).reshape(-1)


def apply_controlled(psi: np.ndarray, n: int, controls: Sequence[int], targets: Sequence[int],
                     g: np.ndarray) -> np.ndarray:
    """Controlled gate (qsim's ApplyControlledGate): G acts
    on `targets` in the subspace where every control qubit is 1; amplitudes
    with any control 0 are unchanged.  Written as that definition: take the
    sub-tensor with the control axes fixed to 1 and apply G to it."""
    controls = list(controls)
    targets = list(targets)
    assert not set(controls) & set(targets)
    t = np.asarray(psi, dtype=np.complex128).reshape((2,) * n).copy()
    idx = [slice(None)] * n
    for c in controls:
        idx[n - 1 - c] = 1
    sub = t[tuple(idx)]  # remaining axes: qubits not in controls, descending
    rest = sorted((q for q in range(n) if q not in controls), reverse=True)
    m = len(rest)
    # qubit q -> position in the sub-state (little-endian over the remaining qubits)
    sub_pos = {q: m - 1 - i for i, q in enumerate(rest)}
    new = apply_gate(sub.reshape(-1), m, [sub_pos[q] for q in targets], g).reshape(sub.shape)
    t[tuple(idx)] = new
    return t.reshape(-1)


def controlled_full_matrix(n: int, controls: Sequence[int], targets: Sequence[int], g: np.ndarray) -> np.ndarray:
    """Brute force: |all-controls-1><..| (x) G + (I - that projector) (x) I as a
    2^n x 2^n matrix (n <= 10)."""
    u = full_gate_matrix(n, list(targets), g)
    idx = np.arange(1 << n)
    on = np.ones(1 << n, dtype=bool)
    for c in controls:
        on &= ((idx >> c) & 1) == 1
    full = np.eye(1 << n, dtype=np.complex128)
    full[np.ix_(on, on)] = u[np.ix_(on, on)]
    return full


def simulate(n: int, gates, psi0: np.ndarray | None = None) -> np.ndarray:
    """U_m ... U_1 |psi0> (default |0..0>), unfused, in circuit order (S0)."""
    psi = zero_state(n) if psi0 is None else np.asarray(psi0, dtype=np.complex128).copy()
    for gt in gates:
        psi = apply_gate(psi, n, gt.qubits, gt.matrix)
    return psi


def full_gate_matrix(n: int, qubits: Sequence[int], g: np.ndarray) -> np.ndarray:
    """Brute force: the explicit 2^n x 2^n matrix of Fig. 4 (n <= 10).

    Entry U[i', i] = G[r, c] when i' and i agree on every non-gate bit, with
    r (c) the bits of i' (i) at the gate's qubits; zero otherwise.
    """
    assert n <= 10
    k = len(qubits)
    dim = 1 << n
    idx = np.arange(dim)
    c = np.zeros(dim, dtype=np.int64)
    rest = idx.copy()
    for b, q in enumerate(qubits):
        c |= ((idx >> q) & 1) << b
        rest &= ~(1 << q)
    u = np.zeros((dim, dim), dtype=np.complex128)
    g = np.asarray(g, dtype=np.complex128)
    for r in range(1 << k):
        ip = rest.copy()
        for b, q in enumerate(qubits):
            ip |= ((r >> b) & 1) << q
        u[ip, idx] = g[r, c]
    return u


def full_circuit_unitary(n: int, gates) -> np.ndarray:
    """Brute force U = U_m ... U_1 as dense matrices (n <= 10)."""
    u = np.eye(1 << n, dtype=np.complex128)
    for gt in gates:
        u = full_gate_matrix(n, gt.qubits, gt.matrix) @ u
    return u


def kron_single_qubit(n: int, q: int, g: np.ndarray) -> np.ndarray:
    """I_{2^(n-1-q)} (x) G (x) I_{2^q}: Fig. 4 built with np.kron (pin only)."""
    return np.kron(np.kron(np.eye(1 << (n - 1 - q)), g), np.eye(1 << q))


def fidelity(a: np.ndarray, b: np.ndarray) -> float:
    """|<a|b>|^2, unnormalised."""
    return float(abs(np.vdot(np.asarray(a, np.complex128), np.asarray(b, np.complex128))) ** 2)


def max_abs_bound(n: int, depth: int) -> float:
    """North-star tolerance: max |psi_gpu - psi_ref| <= 1e-5 * 2^(-n/2) * depth."""
    return 1e-5 * 2.0 ** (-n / 2.0) * depth
