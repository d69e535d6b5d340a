"""Norm loss and infidelity of whole RQC circuits against the oracle, per
fusion size (SVB200_TC selects the apply path).

usage: python tools/circuit_drift.py <n> <depth> <F> [<F> ...]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import paper_conf_sc_markidis23_b200 as sv
from oracle import ref_c
from workloads import rqc as W

n, depth = int(sys.argv[1]), int(sys.argv[2])
gates = W.rqc(n, depth, 2023)
ref = ref_c.run(n, gates)
for F in map(int, sys.argv[3:]):
    h = sv.sv_create(n)
    st = sv.sv_run_circuit(h, gates, F)
    g = sv.sv_get_state(h, n).astype(np.complex128)
    sv.sv_destroy(h)
    norm = float(np.vdot(g, g).real)
    ip = np.vdot(g, ref)
    fid = abs(ip) ** 2
    d = g - ref * (ip / abs(ip)).conjugate()
    print(f"n={n} d={depth} F={F} TC={os.environ.get('SVB200_TC', 'auto')} applies={st['n_fused']}: "
          f"1-norm={1 - norm:+.3e} 1-fid={1 - fid:+.3e} |delta_perp|^2={float(np.vdot(d, d).real):.3e} "
          f"max|delta|={float(np.abs(g - ref).max()):.3e}")
