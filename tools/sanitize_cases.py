"""Small invocations of every kernel family for compute-sanitizer
(memcheck / racecheck / synccheck; profiles/r2_sanitize_*.txt):

  compute-sanitizer --tool racecheck python tools/sanitize_cases.py

* pass-specialised register-blocked passes (rpj): F = 1, 2 at tile 10 and
  12, from the lazy |0...0> (product-state start) and from a loaded state;
* the generic apply_rpass kernel and the shared-memory pass kernel;
* per-gate applies k = 1..6 on high, low and qubit-0 sets: SIMT tile loops
  (16 B cp.async and bulk/tensor-copy), int8 tensor-core (tcgen05) k = 5, 6;
* controlled gates; virtual shards P = 4 (exchange kernel) with per-gate and
  blocked passes; sampling (bins, scan, resolve); complex128 applies (k = 6,
  virtual shards with 16 B exchanges and bit-swap permutations); 14-qubit tiles.
Each result is checked against the oracle so a silent corruption also fails.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import paper_conf_sc_markidis23_b200 as sv
from oracle import ref_c
from oracle import sv as osv
from workloads import rqc as W

n = 16
bad = []


def check(tag, got, ref, depth=14):
    got = got.astype(np.complex128)
    err = float(np.abs(got - ref).max())
    if not (osv.fidelity(got, ref) >= 1 - 1e-5 and err <= osv.max_abs_bound(n, depth) * 4):
        bad.append((tag, err))
    print(f"{tag}: max_abs {err:.2e}", flush=True)


gates = W.rqc(n, 10, seed=1)
ref = ref_c.run(n, gates)
for jit in (1, 0):
    for T in (10, 12):
        for F in (1, 2):
            for lazy in (True, False):
                h = sv.sv_create(n)
                sv.sv_set_option(h, sv.SV_OPT_PASS_JIT, jit)
                sv.sv_set_blocking(h, T)
                if not lazy:
                    sv.sv_device_ptr(h)
                sv.sv_run_circuit(h, gates, F)
                check(f"blocked jit={jit} T={T} F={F} lazy={lazy}", sv.sv_get_state(h, n), ref, 10)
                sv.sv_destroy(h)
h = sv.sv_create(n)
sv.sv_set_blocking(h, 10)
sv.sv_run_circuit(h, gates, 4)  # shared-memory pass kernel (k = 3, 4)
check("smem pass F=4", sv.sv_get_state(h, n), ref, 10)
sv.sv_destroy(h)
rs = np.random.default_rng(0)
psi = W.random_state_c64(n, 3)
for k, qs in [(1, (9,)), (1, (2,)), (2, (0, 7)), (3, (1, 5, 11)), (4, (4, 6, 9, 12)), (4, (0, 1, 2, 3)),
              (5, (4, 6, 8, 10, 12)), (5, (1, 3, 5, 7, 9)), (6, (4, 5, 6, 7, 8, 9)), (6, (0, 2, 4, 6, 8, 10))]:
    M = W.haar_unitary(1 << k, rs).astype(np.complex64)
    for path in (sv.SV_PATH_AUTO, sv.SV_PATH_SIMT):
        h = sv.sv_create(n)
        sv.sv_set_option(h, sv.SV_OPT_APPLY_PATH, path)
        sv.sv_set_state(h, psi)
        sv.sv_apply_fused(h, list(qs), M)
        got = sv.sv_get_state(h, n)
        sv.sv_destroy(h)
        exp = osv.apply_gate(psi.astype(np.complex128), n, list(qs), M.astype(np.complex128))
        err = float(np.abs(got.astype(np.complex128) - exp).max())
        if err > 1e-5:
            bad.append((f"apply k={k} {qs}", err))
        print(f"apply k={k} q={qs} path={path}: max_abs {err:.2e}", flush=True)
h = sv.sv_create(n)
sv.sv_set_state(h, psi)
M = W.haar_unitary(4, rs).astype(np.complex64)
sv.sv_apply_controlled(h, [3, 10], [5, 12], M)
got = sv.sv_get_state(h, n)
sv.sv_destroy(h)
exp = osv.apply_controlled(psi.astype(np.complex128), n, [3, 10], [5, 12], M.astype(np.complex128))
err = float(np.abs(got.astype(np.complex128) - exp).max())
if err > 1e-5:
    bad.append(("controlled", err))
print(f"controlled: max_abs {err:.2e}", flush=True)
for F in (4, 1):
    h = sv.sv_create_ex(n, world=4, virtual_shards=True)
    sv.sv_set_blocking(h, 10)
    sv.sv_run_circuit(h, gates, F)
    check(f"virtual shards P=4 F={F}", sv.sv_get_state(h, n), ref, 10)
    s1 = sv.sv_sample(h, 7, 2000)
    sv.sv_destroy(h)
h = sv.sv_create_ex(n, precision=1)
sv.sv_run_circuit(h, gates, 4)
check("complex128 F=4", sv.sv_get_state_c128(h, n), ref, 10)
sv.sv_destroy(h)
# 14-qubit tiles (64 amplitudes per thread), complex128 k = 6 (row-split tile
# kernel), sharded complex128 (16 B exchanges, exact bit-swap permutations)
for lazy in (True, False):
    h = sv.sv_create(n)
    sv.sv_set_blocking(h, 14)
    if not lazy:
        sv.sv_device_ptr(h)
    sv.sv_run_circuit(h, gates, 1)
    check(f"blocked T=14 F=1 lazy={lazy}", sv.sv_get_state(h, n), ref, 10)
    sv.sv_destroy(h)
h = sv.sv_create_ex(n, precision=1)
sv.sv_run_circuit(h, gates, 6)
check("complex128 F=6", sv.sv_get_state_c128(h, n), ref, 10)
sv.sv_destroy(h)
for F, T in ((4, -1), (1, 10)):
    h = sv.sv_create_ex(n, world=4, virtual_shards=True, precision=1)
    sv.sv_set_blocking(h, T)
    sv.sv_run_circuit(h, gates, F)
    sv.sv_sample(h, 3, 2000)
    check(f"complex128 virtual shards P=4 F={F}", sv.sv_get_state_c128(h, n), ref, 10)
    sv.sv_destroy(h)
print("SANITIZE_CASES", "FAIL " + str(bad) if bad else "OK", flush=True)
