"""Opt-in tensor-core path check (run with SVB200_TC=1): single-apply parity
for k = 4, 5 against the oracle with the TF32x3 error bound, and the
measured per-apply norm change (the documented truncation bias)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import paper_conf_sc_markidis23_b200 as sv
from oracle import sv as osv
from workloads import rqc as W

U = 2.0 ** -24
n = 16
worst = 0.0
drift = []
for k, cases in ((4, [(4, 5, 6, 7), (0, 1, 2, 3), (1, 6, 8, 11), (10, 0, 3, 5)]),
                 (5, [(4, 5, 6, 8, 10), (0, 1, 2, 3, 4), (11, 0, 6, 2, 8)])):
    for i, qs in enumerate(cases):
        rs = np.random.default_rng(100 + 10 * k + i)
        M = W.haar_unitary(1 << k, rs).astype(np.complex64)
        psi = W.random_state_c64(n, 7 + i)
        h = sv.sv_create(n)
        sv.sv_set_state(h, psi)
        sv.sv_apply_fused(h, list(qs), M)
        got = sv.sv_get_state(h, n).astype(np.complex128)
        sv.sv_destroy(h)
        ref = osv.apply_gate(psi.astype(np.complex128), n, list(qs), M.astype(np.complex128))
        bound = osv.apply_gate(np.abs(psi).astype(np.complex128), n, list(qs), np.abs(M).astype(np.complex128)).real
        ratio = float((np.abs(got - ref) / (U * bound + 1e-30)).max())
        worst = max(worst, ratio / (4 * ((1 << k) + 1) + 2))
        drift.append(float(np.vdot(got, got).real - np.vdot(ref, ref).real))
print(f"TC_CHECK worst_error_over_bound={worst:.3f} mean_norm_change_per_apply={np.mean(drift):+.3e}")
