"""Norm drift per fused-gate apply (TC vs SIMT): apply R Haar-random k-qubit
unitaries to a random normalised state and report sum |psi|^2 - 1 after each,
plus the fidelity against the complex128 oracle.  usage: norm_drift.py n k R"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import paper_conf_sc_markidis23_b200 as sv
from oracle import sv as osv
from workloads import rqc as W

n = int(sys.argv[1]) if len(sys.argv) > 1 else 18
k = int(sys.argv[2]) if len(sys.argv) > 2 else 4
R = int(sys.argv[3]) if len(sys.argv) > 3 else 20
rs = np.random.default_rng(0)
psi = W.random_state_c64(n, 3)
ref = psi.astype(np.complex128)
h = sv.sv_create(n)
sv.sv_set_state(h, psi)
for i in range(R):
    qs = [int(x) for x in rs.choice(n, size=k, replace=False)]
    U = W.haar_unitary(1 << k, rs)
    M = U.astype(np.complex64)
    sv.sv_apply_fused(h, qs, M)
    ref = osv.apply_gate(ref, n, qs, M.astype(np.complex128))
    if i % 5 == 4 or i == R - 1:
        g = sv.sv_get_state(h, n).astype(np.complex128)
        print(f"k={k} step {i + 1}: norm-1 gpu {np.vdot(g, g).real - 1:+.3e} ref {np.vdot(ref, ref).real - 1:+.3e} "
              f"1-F {1 - osv.fidelity(g, ref):.3e} maxerr {np.abs(g - ref).max():.2e}")
sv.sv_destroy(h)
