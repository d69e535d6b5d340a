"""Norm loss and infidelity of whole RQC circuits against the oracle, per
fusion size, on the dense-gate path given by APPLY_PATH = auto | i8 | simt
(sv_set_option SV_OPT_APPLY_PATH).

usage: [APPLY_PATH=auto] python tools/circuit_drift.py <n> <depth> <F> [<F> ...]
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
mode = os.environ.get("APPLY_PATH", "auto")
path = {"auto": sv.SV_PATH_AUTO, "i8": sv.SV_PATH_INT8, "simt": sv.SV_PATH_SIMT}[mode]
for F in map(int, sys.argv[3:]):
    h = sv.sv_create(n)
    sv.sv_set_option(h, sv.SV_OPT_APPLY_PATH, path)
    st = sv.sv_run_circuit(h, gates, F)
    g = sv.sv_get_state(h, n).astype(np.complex128)
    sv.sv_destroy(h)
    norm = float(np.vdot(g, g).real)
    ip = np.vdot(g, ref)
    fid = abs(ip) ** 2
    d = g - ref * (ip / abs(ip)).conjugate()
    print(f"n={n} d={depth} F={F} path={mode} applies={st['n_fused']}: "
          f"1-norm={1 - norm:+.3e} 1-fid={1 - fid:+.3e} |delta_perp|^2={float(np.vdot(d, d).real):.3e} "
          f"max|delta|={float(np.abs(g - ref).max()):.3e}")
