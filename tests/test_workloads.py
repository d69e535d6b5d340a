"""The seeded input generators (workloads/rqc.py) against SURVEY.md §8c-S1
and its Appendix C regression vectors (tests/golden/appendix_c.json)."""
import json
import os
from collections import Counter

import numpy as np
import pytest

from workloads import rqc as W

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "appendix_c.json")))


def test_splitmix64_known_values():
    r = W.SplitMix64(0)
    assert [hex(r.next()), hex(r.next())] == GOLD["splitmix64_seed0"]
    assert W.splitmix64_nth(0, 0) == int(GOLD["splitmix64_seed0"][0], 16)
    r = W.SplitMix64(12345)
    seq = [r.next() for _ in range(8)]
    assert [W.splitmix64_nth(12345, s) for s in range(8)] == seq


def test_rqc12_matches_spec_vectors():
    g = GOLD["rqc12"]
    gates = W.rqc(g["n"], g["depth"], g["seed"])
    assert len(gates) == g["n_gates"]
    assert dict(Counter(x.name for x in gates)) == g["counts"]
    got = [[x.time, x.name] + list(x.qubits) for x in gates[12:32]]
    assert got == g["gates_12_31"]
    for m, pairs in enumerate(g["cz_moments_1_4"], start=1):
        assert [list(x.qubits) for x in gates if x.time == m and x.name == "cz"] == pairs


@pytest.mark.parametrize("key", ["30_14", "32_20", "34_20", "36_20"])
def test_rqc_gate_counts(key):
    n, d = map(int, key.split("_"))
    assert dict(Counter(x.name for x in W.rqc(n, d))) == GOLD["gate_counts"][key]


@pytest.mark.parametrize("n", [12, 20, 30, 34, 36, 17, 22])
def test_rqc_structure(n):
    """Rules of S1: H layers first/last; each qubit has at most one op per
    moment; CZ on grid neighbours; no two T in a row on a qubit."""
    gates = W.rqc(n, 14)
    sites = W.grid_sites(n)
    D = 14
    assert all(x.name == "h" for x in gates[:n]) and all(x.name == "h" for x in gates[-n:])
    for m in range(1, D + 1):
        used = [q for x in gates if x.time == m for q in x.qubits]
        assert len(used) == len(set(used))
        for x in gates:
            if x.time == m and x.name == "cz":
                (r0, c0), (r1, c1) = sites[x.qubits[0]], sites[x.qubits[1]]
                assert abs(r0 - r1) + abs(c0 - c1) == 1


def test_qsim_text_roundtrip():
    gates = W.rqc(12, 14)
    n, back = W.from_qsim_text(W.to_qsim_text(12, gates))
    assert n == 12 and [(x.time, x.name, x.qubits) for x in back] == [(x.time, x.name, x.qubits) for x in gates]


@pytest.mark.parametrize("n,cycles", [(12, 8), (30, 14), (36, 20)])
def test_sycamore_structure(n, cycles):
    """NEXT-4 generator rules: a single-qubit layer on every qubit each cycle
    and at the end, never the same gate twice in a row on a qubit; fSim on
    grid neighbours of pattern ABCDCDAB[cycle % 8], disjoint within a cycle."""
    gates = W.sycamore_rqc(n, cycles)
    sites = W.grid_sites(n)
    last = {}
    for t in range(2 * cycles + 1):
        layer = [x for x in gates if x.time == t]
        if t % 2 == 0:
            assert sorted(x.qubits[0] for x in layer) == list(range(n))
            for x in layer:
                assert x.name in ("x_1_2", "y_1_2", "hz_1_2") and last.get(x.qubits[0]) != x.name
                last[x.qubits[0]] = x.name
        else:
            letter = "ABCDCDAB"[(t // 2) % 8]
            used = [q for x in layer for q in x.qubits]
            assert len(used) == len(set(used))
            assert [tuple(x.qubits) for x in layer] == W._syc_couplers(sites, letter)
            for x in layer:
                (r0, c0), (r1, c1) = sites[x.qubits[0]], sites[x.qubits[1]]
                assert (r1 - r0, c1 - c0) == ((1, 0) if letter in "AB" else (0, 1))
                assert x.name == "fs"


def test_sycamore_patterns_cover_every_edge_once():
    sites = W.grid_sites(30)
    allp = [p for L in "ABCD" for p in W._syc_couplers(sites, L)]
    assert len(allp) == len(set(allp)) == 5 * 5 + 4 * 6  # 5x6 grid: 25 horizontal, 24 vertical edges


def test_sycamore_qsim_text_roundtrip():
    gates = W.sycamore_rqc(12, 4)
    n, back = W.from_qsim_text(W.to_qsim_text(12, gates))
    assert n == 12 and [(x.name, x.qubits) for x in back] == [(x.name, x.qubits) for x in gates]
    assert all(np.abs(a.matrix - b.matrix).max() < 1e-15 for a, b in zip(gates, back))
