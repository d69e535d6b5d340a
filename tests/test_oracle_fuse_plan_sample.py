"""Pins for the S3 fuser, S4 planner and S5 sampler in oracle/.

Fuser: fused simulation == unfused (fusion is exact re-association of the
product), Fig. 5's two fusion kinds, hand-worked plans.
Planner: sharded emulation == unsharded; chunk exchange == plain bit swap.
Sampler: the definition min{i : C_i > t} by brute force; exact enumeration;
chi-square against |c_i|^2.
"""
import json
import math
import os

import numpy as np
import pytest

from oracle import fuse, plan, sample, sv
from workloads import rqc as W

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "appendix_c.json")))


def _sim_fused(n, fused, psi0=None):
    psi = sv.zero_state(n) if psi0 is None else psi0.copy()
    for Q, _, M in fused:
        psi = sv.apply_gate(psi, n, list(Q), M)
    return psi


# ------------------------------------------------------------------ fuser
@pytest.mark.parametrize("F", range(7))
def test_fused_equals_unfused_rqc(F):
    n = 12
    gates = W.rqc(n, 14)
    ref = sv.simulate(n, gates)
    assert np.abs(_sim_fused(n, fuse.fuse(gates, F)) - ref).max() < 1e-12


@pytest.mark.parametrize("F", range(7))
def test_fused_equals_unfused_sycamore(F):
    """NEXT-4 workload: fSim gates stand alone at F = 1 and absorb their
    neighbours' single-qubit gates from F = 2 on."""
    n = 10
    gates = W.sycamore_rqc(n, 8, seed=3)
    ref = sv.simulate(n, gates)
    fz = fuse.fuse(gates, F)
    assert np.abs(_sim_fused(n, fz) - ref).max() < 1e-12
    if F == 1:
        assert sum(len(Q) == 2 for Q, _, _ in fz) == sum(x.name == "fs" for x in gates)


@pytest.mark.parametrize("F,seed", [(1, 0), (2, 1), (3, 2), (4, 3), (5, 4), (6, 5)])
def test_fused_equals_unfused_random(F, seed):
    n = 9
    gates = W.random_circuit(n, 80, seed, two_qubit_frac=0.4)
    psi0 = W.random_state_c64(n, seed).astype(np.complex128)
    ref = sv.simulate(n, gates, psi0)
    assert np.abs(_sim_fused(n, fuse.fuse(gates, F), psi0) - ref).max() < 1e-12


@pytest.mark.parametrize("F", range(7))
def test_plan_invariants(F):
    gates = W.random_circuit(10, 120, 7 + F, two_qubit_frac=0.35)
    p = fuse.fuse_plan([g.qubits for g in gates], F)
    seen = sorted(i for _, mem in p for i in mem)
    assert seen == list(range(len(gates)))  # a partition of the gates
    firsts = [mem[0] for _, mem in p]
    assert firsts == sorted(firsts)  # greedy: seeds in circuit order
    for Q, mem in p:
        assert list(Q) == sorted(set(q for i in mem for q in gates[i].qubits))
        assert mem == sorted(mem)
        assert len(Q) <= max(F, len(gates[mem[0]].qubits))
        if F == 0:
            assert len(mem) == 1


def test_plan_hand_worked():
    # g0 H(0), g1 CZ(0,1), g2 T(1), g3 H(2), g4 CZ(1,2); F=2 (worked by hand)
    qs = [(0,), (0, 1), (1,), (2,), (1, 2)]
    assert fuse.fuse_plan(qs, 2) == [((0, 1), [0, 1, 2]), ((1, 2), [3, 4])]
    # blocking: g0 H(0), g1 CZ(1,2), g2 CZ(0,1); g2 may not jump over g1
    qs = [(0,), (1, 2), (0, 1)]
    assert fuse.fuse_plan(qs, 2) == [((0,), [0]), ((1, 2), [1]), ((0, 1), [2])]
    # F=1: a CZ stands alone and absorbs nothing
    qs = [(0,), (0, 1), (0,), (1,)]
    assert fuse.fuse_plan(qs, 1) == [((0,), [0]), ((0, 1), [1]), ((0,), [2]), ((1,), [3])]


def test_fig5_space_and_time_fusion():
    rs = np.random.default_rng(0)
    a, b = W.haar_unitary(2, rs), W.haar_unitary(2, rs)
    gs = [W.Gate(0, "a", (3,), a), W.Gate(0, "b", (1,), b)]
    # space: disjoint qubits -> tensor product, higher qubit = more significant factor
    assert np.abs(fuse.fused_matrix(gs, (1, 3), [0, 1]) - np.kron(a, b)).max() < 1e-15
    # time: same qubit -> ordered matrix product (later gate on the left)
    gt = [W.Gate(0, "a", (2,), a), W.Gate(1, "b", (2,), b)]
    assert np.abs(fuse.fused_matrix(gt, (2,), [0, 1]) - b @ a).max() < 1e-15


def test_appendix_c_plan_and_counts():
    g = GOLD["rqc12"]
    gates = W.rqc(12, 14)
    p = fuse.fuse_plan([x.qubits for x in gates], 4)
    assert [[list(Q), mem] for Q, mem in p[:3]] == g["f4_first3"]
    for key, counts in GOLD["fused_counts"].items():
        n, d = map(int, key.split("_"))
        gq = [x.qubits for x in W.rqc(n, d)]
        assert [len(fuse.fuse_plan(gq, F)) for F in range(7)] == counts


# ---------------------------------------------------------------- planner
@pytest.mark.parametrize("n,g,F,vmin", [(10, 1, 4, 5), (11, 2, 2, 5), (12, 3, 4, 5),
                                         (12, 2, 6, 5), (12, 3, 3, 0), (10, 3, 5, 2)])
def test_sharded_emulation_equals_unsharded(n, g, F, vmin):
    gates = W.rqc(n, 14, seed=n + g)
    fz = fuse.fuse(gates, F)
    ev, pos = plan.plan_sharded([Q for Q, _, _ in fz], n, g, vmin)
    l = n - g
    for e in ev:
        if e[0] == "X":
            assert all(P >= l and p < l for P, p in e[1])
            assert len({P for P, _ in e[1]}) == len(e[1]) == len({p for _, p in e[1]})
        else:
            assert all(p < l for p in e[2])
    out, _ = plan.run_sharded(n, g, fz, ev)
    assert np.abs(out - sv.simulate(n, gates)).max() < 1e-12
    assert sorted(pos) == list(range(n))


def test_chunk_exchange_is_bit_swap():
    rs = np.random.default_rng(1)
    n, g = 9, 3
    l = n - g
    psi = rs.standard_normal(1 << n) + 1j * rs.standard_normal(1 << n)
    for pairs in ([(8, 0)], [(6, 2), (8, 5)], [(6, 0), (7, 3), (8, 1)]):
        shards = [psi[d << l:(d + 1) << l].copy() for d in range(1 << g)]
        plan.exchange_shards(shards, l, pairs)
        assert np.array_equal(np.concatenate(shards), plan.swap_bits(psi, n, pairs))


def test_sharded_exchange_counts_appendix_a():
    for key, bits in GOLD["sharded_f4"].items():
        n, g = map(int, key.split("_"))
        d = 20
        fq = [Q for Q, _ in fuse.fuse_plan([x.qubits for x in W.rqc(n, d)], 4)]
        ev, _ = plan.plan_sharded(fq, n, g)
        assert [len(e[1]) for e in ev if e[0] == "X"] == bits


# ---------------------------------------------------------------- sampler
def _brute_sample(psi_c64, seed, N):
    """The S5 definition with Python integers and a linear scan."""
    w = []
    for a in psi_c64:
        re, im = float(np.float32(a.real)), float(np.float32(a.imag))
        p = re * re + im * im
        w.append(math.floor(p * 2.0 ** 62))
    T = sum(w)
    C, acc = [], 0
    for x in w:
        acc += x
        C.append(acc)
    out = []
    for s in range(N):
        t = (W.splitmix64_nth(seed, s) * T) >> 64
        out.append(next(i for i, c in enumerate(C) if c > t))
    return out, T


@pytest.mark.parametrize("n,seed", [(3, 0), (6, 5), (9, 11)])
def test_sampler_matches_definition(n, seed):
    psi = W.random_state_c64(n, seed)
    got, T = sample.sample(psi, seed, 300)
    ref, Tr = _brute_sample(psi, seed, 300)
    assert T == Tr and [int(x) for x in got] == ref


def test_sampler_complex128_matches_definition():
    """Reading R5: complex128 weights use p = fl(fl(re^2) + fl(im^2)), i.e.
    Python float arithmetic."""
    rs = np.random.default_rng(8)
    n = 7
    psi = rs.standard_normal(1 << n) + 1j * rs.standard_normal(1 << n)
    psi /= np.linalg.norm(psi)
    w_ref = [math.floor((a.real * a.real + a.imag * a.imag) * 2.0 ** 62) for a in psi]
    assert [int(x) for x in sample.weights(psi)] == w_ref
    got, T = sample.sample(psi, 5, 200)
    C = np.cumsum(np.array(w_ref, dtype=object))
    for s_, x in enumerate(got):
        t = (W.splitmix64_nth(5, s_) * sum(w_ref)) >> 64
        assert int(x) == next(i for i, c in enumerate(C) if c > t)


def test_sampler_enumeration_n2():
    # probabilities exactly 1/2, 0, 1/4, 1/4: w = 2^61, 0, 2^60, 2^60
    psi = np.array([0.5 + 0.5j, 0, 0.5, 0.5j], dtype=np.complex64)
    assert [int(x) for x in sample.weights(psi)] == [2 ** 61, 0, 2 ** 60, 2 ** 60]
    out, T = sample.sample(psi, 3, 20000)
    assert 1 not in set(int(x) for x in out)
    frac = np.bincount(out.astype(np.int64), minlength=4) / out.size
    assert abs(frac[0] - 0.5) < 0.02 and abs(frac[2] - 0.25) < 0.02 and abs(frac[3] - 0.25) < 0.02


def test_sampler_chi_square():
    n = 8
    psi = W.random_state_c64(n, 4)
    N = 200000
    out, _ = sample.sample(psi, 99, N)
    p = sample.exact_probabilities(psi)
    p /= p.sum()
    cnt = np.bincount(out.astype(np.int64), minlength=1 << n)
    chi2 = float(np.sum((cnt - N * p) ** 2 / (N * p)))
    dof = (1 << n) - 1
    assert chi2 < dof + 6 * math.sqrt(2 * dof)


def test_sampler_appendix_c():
    g = GOLD["rqc12"]
    psi = sv.simulate(12, W.rqc(12, 14)).astype(np.complex64)
    out, T = sample.sample(psi, 1, 8)
    assert T == g["sampler_T"] and [int(x) for x in out] == g["sampler_seed1_first8"]


# ------------------------------------------- diagonal exchange skip (NEXT-4)
def test_diag_qubits_definition():
    assert plan.diag_qubits((0, 1), W.GATE_CZ) == {0, 1}
    assert plan.diag_qubits((3, 5), W.GATE_CX) == {3}  # control (bit 0) only
    assert plan.diag_qubits((2,), W.GATE_T) == {2}
    assert plan.diag_qubits((2,), W.GATE_H) == set()
    assert plan.diag_qubits((0, 1), W.GATE_FSIM_SYC) == set()


@pytest.mark.parametrize("n,g,F,seed", [(10, 1, 1, 0), (11, 2, 1, 1), (12, 3, 1, 2), (12, 3, 2, 3), (11, 2, 4, 4)])
def test_sharded_diag_skip_equals_unsharded(n, g, F, seed):
    """With the diagonal skip, global qubits a gate is block-diagonal in stay
    global; the per-shard block emulation (shard_block) equals the plain
    unsharded simulation, and the skip never adds exchanges."""
    gates = W.rqc(n, 14, seed=seed)
    fz = fuse.fuse(gates, F)
    dq = [plan.diag_qubits(Q, M) for Q, _, M in fz]
    ev, pos = plan.plan_sharded([Q for Q, _, _ in fz], n, g, 5, diag=dq)
    ev0, _ = plan.plan_sharded([Q for Q, _, _ in fz], n, g, 5)
    nx = sum(e[0] == "X" for e in ev)
    assert nx <= sum(e[0] == "X" for e in ev0)
    l = n - g
    skipped = 0
    for e in ev:
        if e[0] == "A":
            i, phys = e[1], e[2]
            for q, p in zip(sorted(fz[i][0]), phys):
                if p >= l:
                    assert q in dq[i]
                    skipped += 1
    if F == 1:
        assert skipped > 0  # CZ gates on global qubits run in place
    out, _ = plan.run_sharded(n, g, fz, ev)
    assert np.abs(out - sv.simulate(n, gates)).max() < 1e-12
