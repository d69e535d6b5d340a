"""Memory-pattern floor of the passes of a circuit: for every pass of the
RQC's register-blocked plan, time one pass over the same tile qubit set S
made of Hadamards only (structured gates: a few additions per amplitude, so
the pass is bound by its HBM access pattern), next to the pass count.

usage: python tools/pass_mem_probe.py [n=30] [depth=14] [tile_bits=13] [pin]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import paper_conf_sc_markidis23_b200 as sv
from workloads import rqc as W

n = int(sys.argv[1]) if len(sys.argv) > 1 else 30
d = int(sys.argv[2]) if len(sys.argv) > 2 else 14
T = int(sys.argv[3]) if len(sys.argv) > 3 else 13
pin = int(sys.argv[4]) if len(sys.argv) > 4 else 4
h = sv.sv_create(n)
sv.sv_set_option(h, sv.SV_OPT_PASS_PIN, pin)
sv.sv_set_blocking(h, T)
sv.sv_device_ptr(h)
sv.sv_set_timing(h, True)
plan = sv.sv_block_plan(W.rqc(n, d), 1, T)
floor = 2 * 8 * 2 ** n / 6548.5e9 * 1e3
tot = 0.0
for p in plan:
    free = [q for q in p["S"] if q >= pin]
    gates = [W.Gate(i, "h", (q,), W.GATE_H) for i, q in enumerate(free)]
    c = sv.sv_circuit_create(h, gates, 1)
    st = sv.sv_circuit_stats(c)
    t = []
    for _ in range(6):
        sv.sv_circuit_run_device(h, c)
        t.append(sv.sv_last_stats(h)["t_apply_high_dev_s"])
    ms = 1e3 * float(np.median(t[1:]))
    tot += ms
    print(f"S = {p['S']}: passes {st['n_passes']}, {ms:.3f} ms ({floor / ms:.2f} of the HBM floor {floor:.3f} ms)",
          flush=True)
    sv.sv_circuit_destroy(c)
print(f"total {tot:.2f} ms over {len(plan)} passes (floor {floor * len(plan):.2f} ms)")
sv.sv_destroy(h)
