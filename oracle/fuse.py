"""S3 reference gate fuser (TEST INFRASTRUCTURE ONLY -- see oracle/__init__.py).

PAPER.md L98 (§2.2, Fig. 5): gates on different qubits fuse "in space" by a
tensor product; gates on the same qubits fuse "in time" by a matrix product
"adhering to the order".  L104: the transpiler fuses "given as input the
maximum of fused gates" (reading Q4: max_fused F = max qubits per fused gate;
F = 0 = no fusion).  The greedy order and blocking rule are the reading of
SURVEY.md §8c-S3 (Readings).

Output plan: list of (sorted qubit tuple Q, member gate indices ascending).
Fused matrix: M = E_{mem[-1]} ... E_{mem[0]} in complex128, where E_j is gate j
expanded to the |Q|-qubit space with local bit b <-> sorted(Q)[b].
"""
from __future__ import annotations

from typing import List, Sequence, Tuple

import numpy as np

from .sv import full_gate_matrix


def fuse_plan(gate_qubits: Sequence[Sequence[int]], max_fused: int) -> List[Tuple[Tuple[int, ...], List[int]]]:
    """The integer part of S3: which gates fuse, on which qubits."""
    m = len(gate_qubits)
    if max_fused == 0:
        return [(tuple(sorted(q)), [i]) for i, q in enumerate(gate_qubits)]
    F = max_fused
    done = [False] * m
    plan = []
    for i in range(m):
        if done[i]:
            continue
        done[i] = True
        Q = set(gate_qubits[i])
        mem = [i]
        if len(Q) > F:
            plan.append((tuple(sorted(Q)), mem))
            continue
        B = set()
        for j in range(i + 1, m):
            if done[j]:
                continue
            S = set(gate_qubits[j])
            if S & B:
                B |= S
            elif len(Q | S) <= F:
                Q |= S
                mem.append(j)
                done[j] = True
            else:
                B |= S
            if len(Q) == F and Q <= B:
                break
        plan.append((tuple(sorted(Q)), mem))
    return plan


def expand_to(qs_local: Sequence[int], gate_qubits: Sequence[int], g: np.ndarray) -> np.ndarray:
    """E_j: gate on `gate_qubits` as a 2^|Q| matrix over the sorted set Q."""
    pos = [list(qs_local).index(q) for q in gate_qubits]
    return full_gate_matrix(len(qs_local), pos, g)


def fused_matrix(gates, Q: Sequence[int], mem: Sequence[int]) -> np.ndarray:
    """M(Q, mem) = E_{mem[-1]} ... E_{mem[0]} (complex128)."""
    d = 1 << len(Q)
    m = np.eye(d, dtype=np.complex128)
    for j in mem:
        m = expand_to(Q, gates[j].qubits, gates[j].matrix) @ m
    return m


def fuse(gates, max_fused: int):
    """Full S3: [(Q, mem, M complex128)]."""
    plan = fuse_plan([g.qubits for g in gates], max_fused)
    return [(Q, mem, fused_matrix(gates, Q, mem)) for Q, mem in plan]


def plan_stream(plan) -> np.ndarray:
    """Flat int32 encoding of SURVEY.md §8b sv_fusion_plan:
    per fused gate: k, q_0..q_{k-1}, n_mem, mem_0..mem_{n_mem-1}."""
    out = []
    for Q, mem in plan:
        out.append(len(Q))
        out.extend(Q)
        out.append(len(mem))
        out.extend(mem)
    return np.array(out, dtype=np.int32)
