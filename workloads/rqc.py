"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the simulation method (no gate
application, no fusion, no sampling).  It only produces inputs:

* the random-quantum-circuit (RQC) generator (the paper's
  workload is "RQC circuits with 30 qubits ... generated with Cirq",
  PAPER.md L169, §4 Experimental setup);
* the gate table those circuits draw from;
* seeded random states and Haar-random unitaries for kernel tests;
* splitmix64, the counter-based generator every random draw uses
  (SURVEY.md §8c-S1/S5).  The CUDA side re-implements splitmix64 itself in
  its sampler; nothing here is imported by the product library.

Conventions (SURVEY.md §8c readings Q1/Q3): qubit q is bit q of the basis
index (little-endian); a k-qubit gate matrix is row-major 2^k x 2^k and bit b
of the matrix row/column index belongs to ``qubits[b]``.
"""
from __future__ import annotations

import math
from dataclasses import dataclass
from typing import List, Sequence, Tuple

import numpy as np

MASK64 = (1 << 64) - 1
GOLDEN = 0x9E3779B97F4A7C15


def splitmix64_mix(state: int) -> int:
    """The splitmix64 output function applied to an (already advanced) state."""
    z = state & MASK64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31)


class SplitMix64:
    """splitmix64: state += golden; z = mix(state)."""

    def __init__(self, seed: int):
        self.state = seed & MASK64

    def next(self) -> int:
        self.state = (self.state + GOLDEN) & MASK64
        return splitmix64_mix(self.state)


def splitmix64_nth(seed: int, s: int) -> int:
    """Output #(s+1) of splitmix64 started at ``seed`` (counter-based form)."""
    return splitmix64_mix((seed + (s + 1) * GOLDEN) & MASK64)


# --------------------------------------------------------------------------
# Gate table, S2 (fp64, row-major, bit b of the index <-> qubits[b])
# --------------------------------------------------------------------------
_R2 = 1.0 / math.sqrt(2.0)
GATE_H = np.array([[_R2, _R2], [_R2, -_R2]], dtype=np.complex128)
GATE_T = np.array([[1, 0], [0, np.exp(1j * np.pi / 4)]], dtype=np.complex128)
GATE_X_1_2 = 0.5 * np.array([[1 + 1j, 1 - 1j], [1 - 1j, 1 + 1j]], dtype=np.complex128)
GATE_Y_1_2 = 0.5 * np.array([[1 + 1j, -1 - 1j], [1 + 1j, 1 + 1j]], dtype=np.complex128)
GATE_CZ = np.diag([1, 1, 1, -1]).astype(np.complex128)
# test-only gates
GATE_X = np.array([[0, 1], [1, 0]], dtype=np.complex128)
GATE_Y = np.array([[0, -1j], [1j, 0]], dtype=np.complex128)
GATE_Z = np.array([[1, 0], [0, -1]], dtype=np.complex128)
GATE_S = np.array([[1, 0], [0, 1j]], dtype=np.complex128)
# CX with qubits[0] = control, qubits[1] = target: maps index 1 <-> 3 (bit 0 = control)
GATE_CX = np.array([[1, 0, 0, 0], [0, 0, 0, 1], [0, 0, 1, 0], [0, 1, 0, 0]], dtype=np.complex128)
GATE_SWAP = np.array([[1, 0, 0, 0], [0, 0, 1, 0], [0, 1, 0, 0], [0, 0, 0, 1]], dtype=np.complex128)


# Sycamore-style RQC gates (ref [3] of the paper, Arute
# et al. 2019, cited at PAPER.md L145/L169 -- the gate set is [not in paper]):
# sqrt(X), sqrt(Y), sqrt(W) with W = (X + Y)/sqrt(2), each P^(1/2) =
# (1+i)/2 I + (1-i)/2 P for a Pauli-like P (P^2 = I); and fSim(theta, phi)
# on |00>, |01>, |10>, |11>.
GATE_SQRT_X = GATE_X_1_2
GATE_SQRT_Y = GATE_Y_1_2
GATE_W = np.array([[0, np.exp(-1j * np.pi / 4)], [np.exp(1j * np.pi / 4), 0]], dtype=np.complex128)
GATE_SQRT_W = 0.5 * (1 + 1j) * np.eye(2, dtype=np.complex128) + 0.5 * (1 - 1j) * GATE_W


def gate_fsim(theta: float, phi: float) -> np.ndarray:
    c, s_ = math.cos(theta), math.sin(theta)
    return np.array([[1, 0, 0, 0], [0, c, -1j * s_, 0], [0, -1j * s_, c, 0], [0, 0, 0, np.exp(-1j * phi)]],
                    dtype=np.complex128)


GATE_FSIM_SYC = gate_fsim(math.pi / 2, math.pi / 6)


def gate_cp(phi: float) -> np.ndarray:
    """Controlled phase diag(1,1,1,e^{i phi})."""
    return np.diag([1, 1, 1, np.exp(1j * phi)]).astype(np.complex128)


GATE_TABLE = {
    "h": GATE_H,
    "t": GATE_T,
    "x_1_2": GATE_X_1_2,
    "y_1_2": GATE_Y_1_2,
    "cz": GATE_CZ,
    "x": GATE_X,
    "y": GATE_Y,
    "z": GATE_Z,
    "s": GATE_S,
    "cx": GATE_CX,
    "swap": GATE_SWAP,
    "hz_1_2": GATE_SQRT_W,  # qsim's name of sqrt(W)
    "fs": GATE_FSIM_SYC,    # fSim(pi/2, pi/6), the Sycamore two-qubit gate
}


@dataclass
class Gate:
    """One circuit gate: qsim-text 'time name q...' plus its fp64 matrix."""

    time: int
    name: str
    qubits: Tuple[int, ...]
    matrix: np.ndarray  # complex128, (2^k, 2^k), bit b <-> qubits[b]

    @property
    def nq(self) -> int:
        return len(self.qubits)


# --------------------------------------------------------------------------
# RQC generator, S1 (reading of PAPER.md L169/L177: Cirq "v2" supremacy rules)
# --------------------------------------------------------------------------
GRIDS = {
    12: (3, 4, ()),
    20: (4, 5, ()),
    24: (4, 6, ()),
    28: (4, 7, ()),
    30: (5, 6, ()),
    32: (4, 8, ()),
    34: (6, 6, ((5, 4), (5, 5))),
    35: (5, 7, ()),
    36: (6, 6, ()),
}

_LAYER_ORDER = [0, 3, 2, 1, 4, 7, 6, 5]


def grid_sites(n: int) -> List[Tuple[int, int]]:
    """Present (row, col) sites; qubit index = position in row-major order.

    Sizes not in GRIDS use rows = floor(sqrt(n)), cols = ceil(n/rows) with the
    trailing sites of the last row removed (a reading).
    """
    if n in GRIDS:
        rows, cols, missing = GRIDS[n]
    else:
        rows = max(1, int(math.isqrt(n)))
        cols = -(-n // rows)
        extra = rows * cols - n
        missing = tuple((rows - 1, cols - 1 - e) for e in range(extra))
    miss = set(missing)
    sites = [(r, c) for r in range(rows) for c in range(cols) if (r, c) not in miss]
    assert len(sites) == n
    return sites


def _cz_layer(sites, li: int):
    L = _LAYER_ORDER[li % 8]
    dr = L % 2
    dc = 1 - dr
    shift = (L >> 1) % 4
    index = {s: i for i, s in enumerate(sites)}
    pairs = []
    for (r, c) in sites:
        other = (r + dr, c + dc)
        if other in index and (r * (2 - dr) + c * (2 - dc)) % 4 == shift:
            pairs.append((index[(r, c)], index[other]))
    pairs.sort()
    return pairs


def rqc(n: int, depth: int, seed: int = 2023) -> List[Gate]:
    """Generate the synthetic Google-style RQC of SURVEY.md §8c-S1.

    Moment 0: H on all qubits.  Moments 1..depth: one CZ layer, then one
    single-qubit gate per idle qubit (T at moment 1; after a CZ a random X^1/2
    or Y^1/2 from the top bit of splitmix64; after a non-T single-qubit gate a
    T; else nothing).  Moment depth+1: H on all qubits.
    """
    sites = grid_sites(n)
    rng = SplitMix64(seed)
    gates: List[Gate] = []
    prev = ["h"] * n  # op of each qubit at the previous moment ("" = nothing)
    for q in range(n):
        gates.append(Gate(0, "h", (q,), GATE_H))
    li = 0
    for moment in range(1, depth + 1):
        pairs = []
        if n >= 2:
            while True:
                pairs = _cz_layer(sites, li)
                li += 1
                if pairs:
                    break
        in_cz = set()
        for a, b in pairs:
            gates.append(Gate(moment, "cz", (a, b), GATE_CZ))
            in_cz.add(a)
            in_cz.add(b)
        cur = [""] * n
        for q in range(n):
            if q in in_cz:
                cur[q] = "cz"
                continue
            name = ""
            if moment == 1:
                name = "t"
            elif prev[q] == "cz":
                name = "y_1_2" if (rng.next() >> 63) & 1 else "x_1_2"
            elif prev[q] not in ("", "t", "cz"):
                name = "t"
            if name:
                gates.append(Gate(moment, name, (q,), GATE_TABLE[name]))
            cur[q] = name
        prev = cur
    for q in range(n):
        gates.append(Gate(depth + 1, "h", (q,), GATE_H))
    return gates


# --------------------------------------------------------------------------
# Sycamore-style RQC (reading R9)
# --------------------------------------------------------------------------
_SYC_PATTERN = "ABCDCDAB"


def _syc_couplers(sites, letter: str):
    """Coupler pattern on the square grid: A / B = vertical edges from even /
    odd rows, C / D = horizontal edges from even / odd columns (four disjoint
    matchings covering every edge, as Sycamore's four diagonal patterns do)."""
    index = {s: i for i, s in enumerate(sites)}
    pairs = []
    for (r, c) in sites:
        if letter in "AB" and r % 2 == (0 if letter == "A" else 1):
            o = (r + 1, c)
        elif letter in "CD" and c % 2 == (0 if letter == "C" else 1):
            o = (r, c + 1)
        else:
            continue
        if o in index:
            pairs.append((index[(r, c)], index[o]))
    pairs.sort()
    return pairs


def sycamore_rqc(n: int, cycles: int, seed: int = 2023) -> List[Gate]:
    """Sycamore-style RQC on grid_sites(n): every cycle is a layer of random
    single-qubit gates from {sqrt(X), sqrt(Y), sqrt(W)} on all qubits (never
    the gate the qubit had in the previous cycle; choice = candidates[(r *
    len) >> 64] with r the next splitmix64 output, qubits ascending), then
    fSim(pi/2, pi/6) on the couplers of pattern ABCDCDAB[cycle % 8]; a final
    single-qubit layer follows the last cycle."""
    sites = grid_sites(n)
    rng = SplitMix64(seed)
    names = ["x_1_2", "y_1_2", "hz_1_2"]
    prev = [""] * n
    gates: List[Gate] = []

    def one_qubit_layer(t):
        for q in range(n):
            cand = [x for x in names if x != prev[q]]
            name = cand[(rng.next() * len(cand)) >> 64]
            gates.append(Gate(t, name, (q,), GATE_TABLE[name]))
            prev[q] = name

    for cyc in range(cycles):
        one_qubit_layer(2 * cyc)
        for a, b in _syc_couplers(sites, _SYC_PATTERN[cyc % 8]):
            gates.append(Gate(2 * cyc + 1, "fs", (a, b), GATE_FSIM_SYC))
    one_qubit_layer(2 * cycles)
    return gates


def inverse_circuit(gates: Sequence[Gate]) -> List[Gate]:
    """C^dagger: reversed order, conjugate-transposed matrices (test input)."""
    out = []
    t_last = gates[-1].time if gates else 0
    for g in reversed(gates):
        out.append(Gate(t_last + 1 + (t_last - g.time), g.name + "_dag", g.qubits,
                        np.conj(g.matrix.T).copy()))
    return out


def to_qsim_text(n: int, gates: Sequence[Gate]) -> str:
    """qsim circuit text format: first line n, then 'time name q...' (fSim:
    'time fs q0 q1 theta phi')."""
    lines = [str(n)]
    for g in gates:
        extra = [repr(math.pi / 2), repr(math.pi / 6)] if g.name == "fs" else []
        lines.append(" ".join([str(g.time), g.name] + [str(q) for q in g.qubits] + extra))
    return "\n".join(lines) + "\n"


def from_qsim_text(text: str) -> Tuple[int, List[Gate]]:
    """Read the qsim text format for the gate names in GATE_TABLE."""
    lines = [ln.split() for ln in text.strip().splitlines() if ln.strip()]
    n = int(lines[0][0])
    gates = []
    for tok in lines[1:]:
        t, name = int(tok[0]), tok[1]
        if name == "fs":
            qs = (int(tok[2]), int(tok[3]))
            gates.append(Gate(t, name, qs, gate_fsim(float(tok[4]), float(tok[5]))))
            continue
        qs = tuple(int(x) for x in tok[2:])
        gates.append(Gate(t, name, qs, GATE_TABLE[name]))
    return n, gates


def random_circuit(n: int, m: int, seed: int, two_qubit_frac: float = 0.3,
                   three_qubit: bool = False) -> List[Gate]:
    """Random gate list with Haar-random 1/2-qubit unitaries (test input)."""
    rs = np.random.default_rng(seed)
    gates = []
    for i in range(m):
        u = rs.random()
        k = 1
        if n >= 2 and u < two_qubit_frac:
            k = 2
        qs = tuple(int(x) for x in rs.choice(n, size=k, replace=False))
        gates.append(Gate(i, f"u{k}", qs, haar_unitary(1 << k, rs)))
    return gates


# --------------------------------------------------------------------------
# Seeded states and unitaries for kernel tests
# --------------------------------------------------------------------------
def haar_unitary(d: int, rs: np.random.Generator) -> np.ndarray:
    """Haar-random d x d unitary: QR of a complex Gaussian, phases fixed."""
    z = (rs.standard_normal((d, d)) + 1j * rs.standard_normal((d, d))) / math.sqrt(2.0)
    q, r = np.linalg.qr(z)
    ph = np.diag(r) / np.abs(np.diag(r))
    return (q * ph[None, :]).astype(np.complex128)


def random_state_c64(n: int, seed: int) -> np.ndarray:
    """Normalised complex Gaussian state rounded to complex64 (seeded)."""
    rs = np.random.default_rng(seed)
    psi = rs.standard_normal(1 << n) + 1j * rs.standard_normal(1 << n)
    psi /= np.linalg.norm(psi)
    return psi.astype(np.complex64)


def gate_arrays(gates: Sequence[Gate]):
    """Flatten gates into the C-ABI sv_gate layout arrays.

    Returns (nq int32[m], q int32[m,2], mat float64[m,16,2]) where the 2x2
    matrices occupy the first 4 entries.
    """
    m = len(gates)
    nq = np.zeros(m, dtype=np.int32)
    qq = np.zeros((m, 2), dtype=np.int32)
    mat = np.zeros((m, 16, 2), dtype=np.float64)
    for i, g in enumerate(gates):
        k = g.nq
        nq[i] = k
        qq[i, :k] = g.qubits
        flat = np.asarray(g.matrix, dtype=np.complex128).reshape(-1)
        mat[i, : flat.size, 0] = flat.real
        mat[i, : flat.size, 1] = flat.imag
    return nq, qq, mat
