"""Controlled gates (NEXT-4; qsim ApplyControlledGate)
against the oracle's definition (oracle/sv.py apply_controlled).  Amplitudes
with any control 0 must come back bit-identical (they are not touched)."""
import numpy as np
import pytest

import paper_conf_sc_markidis23_b200 as sv
from oracle import sv as osv
from workloads import rqc as W

pytestmark = pytest.mark.gpu
U32 = 2.0 ** -24

CASES = [
    ([5], [0]), ([12], [3]), ([1], [7]), ([2, 9], [4]), ([13, 6], [0, 11]), ([3, 4, 5], [1, 2]),
    ([10], [0, 1, 2, 3]), ([7, 8], [9, 10, 11, 12, 13]), ([15], [0, 2, 4, 6, 8, 10]),
    ([0], [5]), ([0, 3], [8, 9]),  # control on qubit 0: block-matrix path
]


@pytest.mark.parametrize("controls,targets", CASES)
@pytest.mark.parametrize("n", [16, 20])
def test_controlled_parity(n, controls, targets):
    k = len(targets)
    rs = np.random.default_rng(len(controls) * 10 + k)
    M = W.haar_unitary(1 << k, rs).astype(np.complex64)
    psi = W.random_state_c64(n, 9)
    h = sv.sv_create(n)
    try:
        sv.sv_set_state(h, psi)
        sv.sv_apply_controlled(h, controls, targets, M)
        got = sv.sv_get_state(h, n)
    finally:
        sv.sv_destroy(h)
    ref = osv.apply_controlled(psi.astype(np.complex128), n, controls, targets, M.astype(np.complex128))
    idx = np.arange(1 << n)
    on = np.ones(1 << n, bool)
    for c in controls:
        on &= ((idx >> c) & 1) == 1
    if 0 not in controls:
        assert np.array_equal(got[~on], psi[~on])  # untouched subspace, never read or written
    kk = k + (len(controls) if 0 in controls else 0)  # block path multiplies over the expanded matrix
    if 0 in controls:
        on[:] = True  # block path: every amplitude goes through the (block) matrix
    bound = osv.apply_controlled(np.abs(psi).astype(np.complex128), n, controls, targets,
                                 np.abs(M).astype(np.complex128)).real
    err = np.abs(got.astype(np.complex128) - ref)
    assert np.all(err[on] <= (4 * ((1 << kk) + 1) + 2) * U32 * bound[on] + 1e-30)


def test_controlled_errors():
    h = sv.sv_create(10)
    try:
        with pytest.raises(sv.SVError) as e:
            sv.sv_apply_controlled(h, [3], [3], np.eye(2))
        assert e.value.code == sv.SV_EINVAL
        with pytest.raises(sv.SVError) as e:
            sv.sv_apply_controlled(h, [0, 1, 2], [3, 4, 5, 6], np.eye(16))
        assert e.value.code == sv.SV_EUNSUPPORTED
    finally:
        sv.sv_destroy(h)
