"""S4 qubit-map planner + virtual-shard emulator (TEST INFRASTRUCTURE ONLY).

Multi-GPU is the paper's future work (the qsim CUDA/HIP
backend is single-GPU; cuQuantum has multi-GPU).  The north star shards the
2^n state over P = 2^g GPUs by its top g physical qubits and, before a fused
gate that touches a global qubit, swaps global and local qubits.  The planning
rule (Belady pairing with a victim floor vmin) is the reading of SURVEY.md
§8c-S4, listed in DESIGN.md (Readings).

Diagonal skip (reading R10): with ``diag``
given, a fused gate only forces an exchange for its global qubits in which it
is NOT block-diagonal.  A gate block-diagonal in qubit q (M[r][c] == 0
whenever bit q of r and c differ -- it commutes with Z_q, like CZ or a
control qubit) acts on the shard whose device bit for q is x as the block
G_x over its other qubits, so a global q needs no exchange.  Next use counts
only non-diagonal uses.  APPLY events then list global physical bits for
such qubits.

Events: ("X", [(P_j, p_j), ...])  -- exchange: swap physical bit P_j (global,
          >= l = n-g) with physical bit p_j (local, < l), all j at once;
        ("A", i, [pos[q] for q in sorted(Q_i)]) -- apply fused gate i on those
          physical bits (bit b of the fused matrix <-> the b-th entry).
Final map: pos[q] = physical bit of logical qubit q.
"""
from __future__ import annotations

import math
from typing import List, Sequence

import numpy as np

from .sv import apply_gate

INF = math.inf


DIAG_TOL = 1e-10  # |entry| below this counts as zero (fp64 rounding residue of exact zeros)


def diag_qubits(Q: Sequence[int], M: np.ndarray) -> set:
    """Qubits of a fused gate (matrix M over sorted Q, bit b <-> Q[b]) in
    which M is block-diagonal: every entry between a row and a column that
    differ in bit b is zero (|entry| <= DIAG_TOL: products of the fp64 gate
    table leave ~1e-17 where the exact product has 0; reading R10)."""
    k = len(Q)
    out = set()
    for b in range(k):
        r = np.arange(1 << k)
        differ = ((r[:, None] ^ r[None, :]) >> b) & 1
        if not np.any(np.abs(M[differ.astype(bool)]) > DIAG_TOL):
            out.add(Q[b])
    return out


def plan_sharded(fused_qubits: Sequence[Sequence[int]], n: int, g: int, vmin: int = 5, diag=None):
    """S4 exactly as SURVEY.md §8c-S4 states it (diag: per fused gate the set
    of its block-diagonal qubits, or None).  Returns (events, pos)."""
    l = n - g
    pos = list(range(n))
    inv = list(range(n))
    nf = len(fused_qubits)
    uses = [set(Q) - (set(diag[i]) if diag else set()) for i, Q in enumerate(fused_qubits)]

    def nu(q, i):
        for j in range(i, nf):
            if q in uses[j]:
                return j
        return INF

    events = []
    for i, Qi in enumerate(fused_qubits):
        Qs = set(Qi)
        need = [q for q in Qi if pos[q] >= l and q in uses[i]]
        if need:
            glob = [inv[p] for p in range(l, n)]
            glob.sort(key=lambda q: (nu(q, i), q))
            cand = [inv[p] for p in range(vmin, l) if inv[p] not in Qs]
            if len(cand) < len(need):
                cand = [inv[p] for p in range(0, l) if inv[p] not in Qs]
            # nu descending (infinity first), then physical position descending
            cand.sort(key=lambda q: (-nu(q, i), -pos[q]))
            pairs = []
            for a, b in zip(glob, cand):
                if nu(a, i) < nu(b, i):
                    pairs.append((pos[a], pos[b]))
                else:
                    break
            assert len(pairs) >= len(need), "not enough local qubits to swap"
            for P, p in pairs:
                a, b = inv[P], inv[p]
                pos[a], pos[b] = p, P
                inv[P], inv[p] = b, a
            events.append(("X", pairs))
        events.append(("A", i, [pos[q] for q in sorted(Qi)]))
    return events, pos


def swap_bits(psi: np.ndarray, n: int, pairs) -> np.ndarray:
    """Plain definition of an exchange: permute the index by swapping bits."""
    idx = np.arange(1 << n)
    src = idx.copy()
    for P, p in pairs:
        bP = (idx >> P) & 1
        bp = (idx >> p) & 1
        src = src & ~((1 << P) | (1 << p))
        src |= (bP << p) | (bp << P)
    # new[i] = old[i with bits swapped]; a bit swap is an involution
    return psi[src]


def exchange_shards(shards: List[np.ndarray], l: int, pairs) -> None:
    """The distributed form of one exchange, in place on P shard arrays.

    Device d's chunk c (local offsets whose bits at {p_j} equal c) swaps with
    device e's chunk c_d, e = d with device bits (P_j - l) set to c, c_d = d's
    device bits at (P_j - l) (SURVEY.md §8c-S4 'Exchange semantics').
    """
    s = len(pairs)
    P = len(shards)
    loc = np.arange(1 << l)

    def chunk(c):
        sel = np.ones(1 << l, dtype=bool)
        for j, (_, p) in enumerate(pairs):
            sel &= ((loc >> p) & 1) == ((c >> j) & 1)
        return np.nonzero(sel)[0]

    for d in range(P):
        cd = 0
        for j, (Pj, _) in enumerate(pairs):
            cd |= ((d >> (Pj - l)) & 1) << j
        for c in range(1 << s):
            e = d
            for j, (Pj, _) in enumerate(pairs):
                e = (e & ~(1 << (Pj - l))) | (((c >> j) & 1) << (Pj - l))
            if (d, c) >= (e, cd):
                continue  # each symmetric pair once; c == cd is a self-swap
            ia, ib = chunk(c), chunk(cd)
            tmp = shards[d][ia].copy()
            shards[d][ia] = shards[e][ib]
            shards[e][ib] = tmp


def run_sharded(n: int, g: int, fused, events, psi0: np.ndarray | None = None, emulate_chunks=True):
    """Virtual-shard simulation of a planned circuit; returns the LOGICAL state.

    fused: list of (Q, mem, M); events from plan_sharded.  Each APPLY applies M
    on the given physical bits; each EXCHANGE runs exchange_shards (or the
    plain bit swap when emulate_chunks is False).
    """
    l = n - g
    psi = np.zeros(1 << n, dtype=np.complex128) if psi0 is None else psi0.astype(np.complex128).copy()
    if psi0 is None:
        psi[0] = 1.0
    pos = list(range(n))
    for ev in events:
        if ev[0] == "X":
            if emulate_chunks:
                shards = [psi[d << l:(d + 1) << l].copy() for d in range(1 << g)]
                exchange_shards(shards, l, ev[1])
                psi = np.concatenate(shards)
            else:
                psi = swap_bits(psi, n, ev[1])
            inv = {p: q for q, p in enumerate(pos)}
            for P, p in ev[1]:
                a, b = inv[P], inv[p]
                pos[a], pos[b] = p, P
        else:
            _, i, phys = ev
            if any(p >= l for p in phys):
                # diagonal skip: shard d applies the block of M selected by its
                # device bits at the global positions, on its local bits
                shards = [psi[d << l:(d + 1) << l].copy() for d in range(1 << g)]
                for d in range(1 << g):
                    loc, sub = shard_block(fused[i][2], phys, l, d)
                    if loc:
                        shards[d] = apply_gate(shards[d], l, loc, sub)
                    else:
                        shards[d] = shards[d] * sub[0, 0]
                psi = np.concatenate(shards)
            else:
                psi = apply_gate(psi, n, phys, fused[i][2])
    return to_logical(psi, n, pos), pos


def shard_block(M: np.ndarray, phys: Sequence[int], l: int, d: int):
    """Block of M (bit b <-> phys[b]) on shard d: rows/columns whose global
    bits (phys[b] >= l) equal d's device bits; returns (local phys, block)."""
    k = len(phys)
    gb = [b for b in range(k) if phys[b] >= l]
    lb = [b for b in range(k) if phys[b] < l]
    x = 0
    for b in gb:
        x |= ((d >> (phys[b] - l)) & 1) << b
    idx = []
    for t in range(1 << len(lb)):
        r = x
        for j, b in enumerate(lb):
            r |= ((t >> j) & 1) << b
        idx.append(r)
    return [phys[b] for b in lb], M[np.ix_(idx, idx)]


def to_logical(psi_phys: np.ndarray, n: int, pos: Sequence[int]) -> np.ndarray:
    """Logical index i has qubit q at physical bit pos[q]."""
    idx = np.arange(1 << n)
    phys = np.zeros_like(idx)
    for q in range(n):
        phys |= ((idx >> q) & 1) << pos[q]
    return psi_phys[phys]


def plan_stream(events) -> np.ndarray:
    """Flat int32 encoding used by the C ABI sv_shard_plan: per event
    X: -1, s, P_0, p_0, ..., P_{s-1}, p_{s-1};  A: i, k, phys_0..phys_{k-1}."""
    out = []
    for ev in events:
        if ev[0] == "X":
            out += [-1, len(ev[1])]
            for P, p in ev[1]:
                out += [P, p]
        else:
            out += [ev[1], len(ev[2])] + list(ev[2])
    return np.array(out, dtype=np.int32)
