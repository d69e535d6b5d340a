"""Tensor-core path check: single apply parity for k = 4, 5, 6 against the
oracle and the per-apply norm change, on the dense-gate path given as the
argument (sv_set_option SV_OPT_APPLY_PATH): auto (k = 5, 6 on int8 tensor
cores), i8 (k = 4..6 on int8 tensor cores) or simt.
usage: python tools/tc_check.py [auto|i8|simt]
The int8 path's slicing error is relative to the group-row / column maximum,
so its bound adds 2^(k+1) 2^-21 max_c|a| max|M| to the SIMT bound."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import paper_conf_sc_markidis23_b200 as sv
from oracle import sv as osv
from workloads import rqc as W

PATH = {"auto": sv.SV_PATH_AUTO, "i8": sv.SV_PATH_INT8, "simt": sv.SV_PATH_SIMT}[sys.argv[1] if len(sys.argv) > 1 else "auto"]
U = 2.0 ** -24
n = 16
worst = 0.0
drift = []
for k, cases in ((4, [(4, 5, 6, 7), (0, 1, 2, 3), (1, 6, 8, 11), (10, 0, 3, 5)]),
                 (5, [(4, 5, 6, 8, 10), (0, 1, 2, 3, 4), (11, 0, 6, 2, 8)]),
                 (6, [(4, 5, 6, 7, 8, 9), (0, 1, 2, 3, 4, 5), (13, 0, 7, 2, 9, 4), (1, 3, 8, 10, 12, 15)])):
    for i, qs in enumerate(cases):
        rs = np.random.default_rng(100 + 10 * k + i)
        M = W.haar_unitary(1 << k, rs).astype(np.complex64)
        psi = W.random_state_c64(n, 7 + i)
        h = sv.sv_create(n)
        sv.sv_set_option(h, sv.SV_OPT_APPLY_PATH, PATH)
        sv.sv_set_state(h, psi)
        sv.sv_apply_fused(h, list(qs), M)
        got = sv.sv_get_state(h, n).astype(np.complex128)
        sv.sv_destroy(h)
        ref = osv.apply_gate(psi.astype(np.complex128), n, list(qs), M.astype(np.complex128))
        bound = osv.apply_gate(np.abs(psi).astype(np.complex128), n, list(qs), np.abs(M).astype(np.complex128)).real
        # per-group maximum |a| broadcast back onto the group's members
        t = np.abs(psi).astype(np.float64).reshape((2,) * n)
        axes = tuple(n - 1 - q for q in qs)
        gmax = np.broadcast_to(t.max(axis=axes, keepdims=True) if False else np.max(t, axis=axes, keepdims=True),
                               t.shape).reshape(-1)
        slack = (4 * ((1 << k) + 1) + 2) * U * bound + (2 << k) * 2.0 ** -21 * gmax * np.abs(M).max()
        worst = max(worst, float((np.abs(got - ref) / (slack + 1e-30)).max()))
        drift.append(float(np.vdot(got, got).real - np.vdot(ref, ref).real))
print(f"TC_CHECK worst_error_over_bound={worst:.3f} mean_norm_change_per_apply={np.mean(drift):+.3e}")

# whole circuits from |0..0> (many all-zero group rows early on) at F = 4..6
from oracle import ref_c

cworst = 0.0
for nq, depth, F in ((20, 14, 5), (20, 14, 4), (18, 20, 5), (20, 14, 6), (18, 20, 6)):
    gates = W.rqc(nq, depth, 2023)
    ref = ref_c.run(nq, gates)
    h = sv.sv_create(nq)
    sv.sv_set_option(h, sv.SV_OPT_APPLY_PATH, PATH)
    sv.sv_run_circuit(h, gates, F)
    got = sv.sv_get_state(h, nq).astype(np.complex128)
    sv.sv_destroy(h)
    fid = osv.fidelity(got, ref)
    err = float(np.abs(got - ref).max())
    cworst = max(cworst, err / osv.max_abs_bound(nq, depth))
    assert np.isfinite(got).all() and fid >= 1 - 1e-5, (nq, F, fid)
print(f"TC_CIRCUIT worst_error_over_northstar_bound={cworst:.3f}")
