"""Launch a few fused-gate applies at bench size for ncu / timing studies.

usage: python tools/prof_apply.py [n] [reps] [case ...]
cases: h4 (k=4 all-high), l4 (k=4 with low qubit), h2, l2, h1, h5, h6, l5
"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import paper_conf_sc_markidis23_b200 as sv
from workloads import rqc as W

CASES = {
    "h1": (20,), "l1": (2,), "h2": (10, 20), "l2": (1, 20), "h3": (5, 12, 25), "l3": (2, 12, 25),
    "h4": (6, 12, 18, 24), "l4": (2, 12, 18, 24), "l4b": (1, 2, 12, 24), "q0": (0, 12, 18, 24),
    "p4": (0, 1, 2, 3), "p4b": (0, 6, 25, 26), "p4c": (0, 2, 6, 8), "r4": (10, 11, 12, 13), "r5": (10, 11, 12, 13, 14), "r6": (12, 13, 14, 15, 16, 17),
    "h5": (4, 8, 12, 18, 24), "l5": (1, 8, 12, 18, 24), "h6": (4, 8, 12, 16, 20, 24), "l6": (1, 3, 8, 12, 20, 24),
}

n = int(sys.argv[1]) if len(sys.argv) > 1 else 30
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
cases = sys.argv[3:] or ["h4", "l4"]
h = sv.sv_create(n)
sv.sv_set_timing(h, True)
rs = np.random.default_rng(0)
for c in cases:
    qs = CASES[c]
    M = W.haar_unitary(1 << len(qs), rs).astype(np.complex64)
    sv.sv_apply_fused(h, qs, M)
    sv.sv_synchronize(h)
    st0 = sv.sv_last_stats(h)
    for _ in range(reps):
        sv.sv_apply_fused(h, qs, M)
    st = sv.sv_last_stats(h)
    t = (st["t_apply_high_dev_s"] + st["t_apply_low_dev_s"]) - (st0["t_apply_high_dev_s"] + st0["t_apply_low_dev_s"])
    print(f"{c:4s} k={len(qs)} q={qs}: {1e3 * t / reps:.3f} ms/launch, {16 * 2 ** n * reps / t / 1e9:.0f} GB/s, "
          f"{(8 * 2 ** len(qs) - 2) * 2 ** n * reps / t / 1e12:.1f} TFLOP/s")
sv.sv_destroy(h)
