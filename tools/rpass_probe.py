"""Marginal cost of gates inside one register-blocked pass at 30 qubits.

usage: python tools/rpass_probe.py [n]
Times (CUDA events via sv_set_timing) one pass holding g dense 1-qubit gates
on distinct qubits (g = 0 means one CZ on qubits 0,1: sign flips only) and
one pass of g dense 2-qubit gates."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import paper_conf_sc_markidis23_b200 as sv
from workloads import rqc as W

n = int(sys.argv[1]) if len(sys.argv) > 1 else 30
h = sv.sv_create(n)
sv.sv_set_blocking(h, 12)
sv.sv_set_timing(h, True)
rs = np.random.default_rng(0)
qs = [4, 5, 6, 7, 8, 9, 10, 11]


def timeit(gates, F, reps=5):
    c = sv.sv_circuit_create(h, gates, F)
    st = sv.sv_circuit_stats(c)
    sv.sv_circuit_run_device(h, c)
    sv.sv_synchronize(h)
    sv.sv_last_stats(h)
    t = 0.0
    for _ in range(reps):
        sv.sv_circuit_run_device(h, c)
        s = sv.sv_last_stats(h)
        t += s["t_apply_high_dev_s"] + s["t_apply_low_dev_s"]
    sv.sv_circuit_destroy(c)
    return t / reps / max(st["n_passes"], 1), st["n_passes"]


print("pass with g gates: ms per pass (one pass expected)")
t, p = timeit([W.Gate(0, "cz", (0, 1), W.GATE_CZ)], 1)
print(f"CZ only: {t * 1e3:.3f} ms ({p} passes)")
for g in (1, 2, 4, 8):
    gates = [W.Gate(i, "u1", (qs[i],), W.haar_unitary(2, rs)) for i in range(g)]
    t, p = timeit(gates, 1)
    print(f"{g} dense 1q: {t * 1e3:.3f} ms ({p} passes)")
for g in (1, 2, 4):
    gates = [W.Gate(i, "u2", (qs[2 * i], qs[2 * i + 1]), W.haar_unitary(4, rs)) for i in range(g)]
    t, p = timeit(gates, 2)
    print(f"{g} dense 2q: {t * 1e3:.3f} ms ({p} passes)")
# repeated gates on the same register set (one phase, many gates)
for g in (4, 8, 16):
    gates = [W.Gate(i, "u1", (qs[i % 4],), W.haar_unitary(2, rs)) for i in range(g)]
    t, p = timeit(gates, 1)
    print(f"{g} dense 1q on 4 qubits: {t * 1e3:.3f} ms ({p} passes)")
sv.sv_destroy(h)
