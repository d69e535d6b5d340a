"""C-ABI boundary semantics on the device (include/sv.h):

* every invalid call returns its documented code with ZERO kernel launches
  and no side effect (the lazy |0...0> stays pending: no reset launch);
* caller-owned buffers (sv_config.dev_buf, the PyTorch interop path) are
  written at create / reset, and a state the caller writes into the buffer is
  what the next call reads;
* sv_sample_device checks the total weight on the device (no host round
  trip): invalid totals give UINT64_MAX outputs and SV_EINVAL at the next
  sv_synchronize;
* sv_apply_fused stages k = 6 / int8 inputs through the ring without host
  syncs -- many queued applies give the same state as synchronised ones.
"""
import numpy as np
import pytest

import paper_conf_sc_markidis23_b200 as sv
from oracle import sv as osv
from workloads import rqc as W

pytestmark = pytest.mark.gpu


def _launches(h):
    st = sv.sv_last_stats(h)
    return st["n_launch_high"] + st["n_launch_low"] + st["n_launch_other"]


def _expect(code, fn, *a):
    with pytest.raises(sv.SVError) as e:
        fn(*a)
    assert e.value.code == code, (fn.__name__, e.value.code)


def test_invalid_calls_launch_nothing():
    n = 12
    h = sv.sv_create(n)
    try:
        sv.sv_reset(h)  # lazy: nothing written yet
        base = _launches(h)
        M2 = np.eye(2, dtype=np.complex64)
        _expect(sv.SV_EINVAL, sv.sv_apply_fused, h, [n], M2)            # qubit out of range
        _expect(sv.SV_EINVAL, sv.sv_apply_fused, h, [3, 3], np.eye(4, dtype=np.complex64))  # duplicate
        _expect(sv.SV_EINVAL, sv.sv_apply_controlled, h, [1], [1], M2)  # control == target
        _expect(sv.SV_EINVAL, sv.sv_apply_controlled, h, [n + 1], [0], M2)
        _expect(sv.SV_EINVAL, sv.sv_apply_controlled, h, [1, 2, 3, 4, 5, 6, 7], [0], M2)  # n_ctrl > 6
        _expect(sv.SV_EINVAL, sv.sv_amplitudes, h, np.array([1 << n], dtype=np.uint64))
        _expect(sv.SV_EINVAL, sv.sv_run_circuit, h, W.rqc(n, 4), 7)    # max_fused > 6
        _expect(sv.SV_EINVAL, sv.sv_set_option, h, 99, 1)
        _expect(sv.SV_EINVAL, sv.sv_set_option, h, sv.SV_OPT_PASS_SEARCH, 0)
        _expect(sv.SV_EINVAL, sv.sv_set_option, h, sv.SV_OPT_PASS_SEARCH, 9)
        _expect(sv.SV_EINVAL, sv.sv_set_blocking, h, 9)
        _expect(sv.SV_EINVAL, sv.sv_set_state, h, np.zeros(5, np.complex64))
        assert _launches(h) == base
        # the pending |0...0> survived every failed call
        assert sv.sv_amplitudes(h, np.array([0, 1], dtype=np.uint64)).tolist() == [1, 0]
    finally:
        sv.sv_destroy(h)


def test_caller_owned_buffer_is_written_and_read():
    import torch
    n = 16
    buf = torch.full((1 << n,), 7 + 7j, dtype=torch.complex64, device="cuda")
    h = sv.sv_create_ex(n, dev_buf=buf.data_ptr(), buf_bytes=buf.numel() * 8)
    try:
        sv.sv_synchronize(h)
        e0 = torch.zeros_like(buf)
        e0[0] = 1
        assert torch.equal(buf, e0)  # create wrote |0...0> into the caller's buffer
        psi = torch.from_numpy(W.random_state_c64(n, 9)).cuda()
        buf.copy_(psi)  # the caller writes a state directly
        torch.cuda.synchronize()
        gates = W.rqc(n, 6)
        sv.sv_run_circuit(h, gates, 1)
        got = sv.sv_get_state(h, n).astype(np.complex128)
        ref = osv.simulate(n, gates, psi.cpu().numpy().astype(np.complex128))
        assert np.abs(got - ref).max() < 1e-5
        sv.sv_reset(h)
        sv.sv_synchronize(h)
        assert torch.equal(buf, e0)  # reset writes the caller's buffer too
    finally:
        sv.sv_destroy(h)


def test_sample_device_invalid_total_reports_at_sync():
    import torch
    n = 8
    h = sv.sv_create(n)
    out = torch.zeros(100, dtype=torch.int64, device="cuda")
    try:
        sv.sv_set_state(h, np.zeros(1 << n, np.complex64))
        sv.sv_sample_device(h, 1, 100, out.data_ptr())  # asynchronous: no error yet
        _expect(sv.SV_EINVAL, sv.sv_synchronize, h)
        assert np.all(out.cpu().numpy().view(np.uint64) == np.uint64(2 ** 64 - 1))
        sv.sv_synchronize(h)  # reported once
        sv.sv_reset(h)
        sv.sv_sample_device(h, 1, 100, out.data_ptr())
        sv.sv_synchronize(h)
        assert np.all(out.cpu().numpy() == 0)
    finally:
        sv.sv_destroy(h)


@pytest.mark.parametrize("k,qs", [(6, (1, 3, 5, 8, 10, 12)), (5, (2, 4, 6, 9, 11))])
def test_async_staging_ring(k, qs):
    """20 queued k = 6 / int8 k = 5 applies (more than the 8 ring slots):
    each staged matrix is the one its launch reads."""
    n = 16
    rs = np.random.default_rng(k)
    Ms = [W.haar_unitary(1 << k, rs).astype(np.complex64) for _ in range(20)]
    psi = W.random_state_c64(n, 1)
    h = sv.sv_create(n)
    try:
        sv.sv_set_state(h, psi)
        for M in Ms:
            sv.sv_apply_fused(h, list(qs), M)
        got = sv.sv_get_state(h, n).astype(np.complex128)
    finally:
        sv.sv_destroy(h)
    ref = psi.astype(np.complex128)
    for M in Ms:
        ref = osv.apply_gate(ref, n, list(qs), M.astype(np.complex128))
    assert osv.fidelity(got, ref) >= 1 - 1e-5 and np.abs(got - ref).max() < 1e-5


def test_sample_into_caller_buffer():
    """sv_sample writes into a caller-owned (here pinned) host buffer: the same
    bitstrings as into a fresh array; a short buffer is rejected."""
    import torch
    n = 14
    h = sv.sv_create(n)
    try:
        sv.sv_set_state(h, W.random_state_c64(n, 5))
        ref = sv.sv_sample(h, 9, 5000)
        buf = torch.empty(5000, dtype=torch.int64, pin_memory=True).numpy().view(np.uint64)
        got = sv.sv_sample(h, 9, 5000, out=buf)
        assert got is buf and np.array_equal(buf, ref)
        with pytest.raises(ValueError):
            sv.sv_sample(h, 9, 5000, out=np.empty(10, dtype=np.uint64))
    finally:
        sv.sv_destroy(h)
