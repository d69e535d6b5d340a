"""Time one register-blocked pass over a given tile qubit set (30 qubits):
9 dense one-qubit gates on the listed qubits (plus 0..3 pinned) form one pass
whose tile is exactly {0..3} + those qubits.

usage: python tools/tile_probe.py "9,10,13,14,16,21,23,27,29" ["6,7,..."]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import paper_conf_sc_markidis23_b200 as sv
from workloads import rqc as W

n = 30
h = sv.sv_create(n)
sv.sv_device_ptr(h)
sv.sv_set_timing(h, True)
rs = np.random.default_rng(0)
for spec in sys.argv[1:]:
    qs = [int(x) for x in spec.split(",")]
    gates = [W.Gate(i, "u", (q,), W.haar_unitary(2, rs)) for i, q in enumerate(qs)]
    c = sv.sv_circuit_create(h, gates, 1)
    st = sv.sv_circuit_stats(c)
    sv.sv_circuit_run_device(h, c)
    sv.sv_synchronize(h)
    sv.sv_last_stats(h)
    t = []
    for _ in range(5):
        sv.sv_circuit_run_device(h, c)
        s = sv.sv_last_stats(h)
        t.append(s["t_apply_high_dev_s"])
    print(f"S = 0..3 + {qs}: passes {st['n_passes']}, {1e3 * np.median(t):.3f} ms per circuit", flush=True)
    sv.sv_circuit_destroy(c)
sv.sv_destroy(h)
