"""Host logic of the cache-blocked passes (no GPU): the pass plan and the
register-phase plan that sv_block_plan exports are checked for the invariants
that make them exact re-associations of the fused circuit (DESIGN.md reading
R7), and the blocked execution order is simulated with the oracle's fused
matrices against the fused plan order."""
import numpy as np
import pytest

import paper_conf_sc_markidis23_b200 as sv
from oracle import fuse as ofuse
from oracle import sv as osv
from workloads import rqc as W


def _fused(gates, F):
    st = sv.sv_fusion_plan(gates, F).tolist()
    out, i = [], 0
    while i < len(st):
        k = st[i]
        q = st[i + 1:i + 1 + k]
        nm = st[i + 1 + k]
        out.append((tuple(q), st[i + 2 + k:i + 2 + k + nm]))
        i += 2 + k + nm
    return out


def _mixed(n, m, seed):
    rs = np.random.default_rng(seed)
    gates = []
    for i in range(m):
        kind = rs.choice(["u1", "u2", "t", "cz", "cp"])
        k = 2 if kind in ("u2", "cz", "cp") else 1
        pool = np.arange(n) if rs.random() < 0.5 else np.arange(min(n, 6))
        qs = tuple(int(x) for x in rs.choice(pool, size=k, replace=False))
        mat = {"u1": None, "u2": None, "t": W.GATE_T, "cz": W.GATE_CZ}.get(str(kind))
        if kind == "cp":
            mat = W.gate_cp(float(rs.uniform(0, 6.28)))
        if mat is None:
            mat = W.haar_unitary(1 << k, rs)
        gates.append(W.Gate(i, str(kind), qs, mat))
    return gates


CASES = [("rqc30", lambda: W.rqc(30, 14), 30), ("rqc24", lambda: W.rqc(24, 20, 5), 24),
         ("mixed22", lambda: _mixed(22, 300, 1), 22)]


def _execution_order(passes):
    """Fused-gate indices in the order the kernels apply them."""
    order = []
    for p in passes:
        if p["phases"]:
            for _, js in p["phases"]:
                order += [p["fused"][j] for j in js]
        else:
            order += p["fused"]
    return order


@pytest.mark.parametrize("name,make,n", CASES)
@pytest.mark.parametrize("F", [1, 2])
@pytest.mark.parametrize("T", [10, 12, 13])
def test_pass_plan_invariants(name, make, n, F, T):
    gates = make()
    fused = _fused(gates, F)
    passes = sv.sv_block_plan(gates, F, T)
    # every fused gate exactly once, in some pass whose tile holds its qubits
    seen = [p_i for p in passes for p_i in p["fused"]]
    assert sorted(seen) == list(range(len(fused)))
    for p in passes:
        S = p["S"]
        assert len(S) == T and S == sorted(S) and set(range(4)) <= set(S)
        for f in p["fused"]:
            assert set(fused[f][0]) <= set(S)
        # register phases: partition of the pass, R = 5 tile positions, every
        # non-CZ gate inside R
        if p["phases"]:
            js = sorted(j for _, g in p["phases"] for j in g)
            assert js == list(range(len(p["fused"])))
            for R, g in p["phases"]:
                assert len(R) == 5 and R == sorted(R) and all(0 <= r < T for r in R)
                for j in g:
                    q = fused[p["fused"][j]][0]
                    pos = {S.index(x) for x in q}
                    m = ofuse.fused_matrix(gates, q, fused[p["fused"][j]][1])
                    cz = len(q) == 2 and np.array_equal(m, np.diag([1, 1, 1, -1]).astype(complex))
                    assert cz or pos <= set(R)
    # the execution order keeps the relative order of every two fused gates
    # that share a qubit unless both are diagonal (they commute), so it is an
    # exact re-association (R7)
    order = _execution_order(passes)
    where = {f: i for i, f in enumerate(order)}
    mats = [ofuse.fused_matrix(gates, q, mem) for q, mem in fused]
    diag = [not np.count_nonzero(m - np.diag(np.diag(m))) for m in mats]
    swapped = 0
    for a in range(len(fused)):
        for b in range(a + 1, len(fused)):
            if set(fused[a][0]) & set(fused[b][0]) and where[a] > where[b]:
                assert diag[a] and diag[b], (a, b)
                swapped += 1


@pytest.mark.parametrize("F", [1, 2])
def test_blocked_order_simulates_like_fused_order(F):
    """Oracle simulation (fp64) of the fused gates in blocked execution order
    equals the fused plan order on a small circuit."""
    n = 14
    gates = _mixed(n, 120, 7)
    fused = _fused(gates, F)
    mats = [ofuse.fused_matrix(gates, q, mem) for q, mem in fused]
    order = _execution_order(sv.sv_block_plan(gates, F, 10))
    a = np.zeros(1 << n, dtype=np.complex128)
    a[0] = 1
    b = a.copy()
    for i, (q, _) in enumerate(fused):
        a = osv.apply_gate(a, n, list(q), mats[i])
    for i in order:
        b = osv.apply_gate(b, n, list(fused[i][0]), mats[i])
    assert np.abs(a - b).max() < 1e-12


def test_block_plan_errors():
    gates = W.rqc(16, 4)
    with pytest.raises(Exception):
        sv.sv_block_plan(gates, 5, 12)
    with pytest.raises(Exception):
        sv.sv_block_plan(gates, 2, 9)
