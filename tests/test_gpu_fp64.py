"""complex128 (fp64) states -- SURVEY.md §8f NEXT-1, the paper's Fig. 8
experiment (double precision shows no substantial state
differences).  Parity against the complex128 oracle with the fp64 analogue
of the kernel error bound, |dy_r| <= (4 (2^k + 1) + 2) 2^-53 sum_c |M_rc||a_c|;
circuits with fidelity 1 - 1e-12; sampling bit-exact (reading R5)."""
import numpy as np
import pytest

import paper_conf_sc_markidis23_b200 as sv
from oracle import ref_c
from oracle import sample as osample
from oracle import sv as osv
from workloads import rqc as W

pytestmark = pytest.mark.gpu
U64 = 2.0 ** -53


def _state128(n, seed):
    rs = np.random.default_rng(seed)
    psi = rs.standard_normal(1 << n) + 1j * rs.standard_normal(1 << n)
    return psi / np.linalg.norm(psi)


@pytest.mark.parametrize("k,qs_list", [(1, [(0,), (2,), (9,)]), (2, [(0, 5), (1, 2), (7, 3)]),
                                        (3, [(0, 1, 2), (4, 8, 10), (2, 9, 5)]),
                                        (4, [(0, 1, 2, 3), (3, 6, 9, 12), (13, 1, 7, 4)]),
                                        (5, [(0, 2, 4, 6, 8), (5, 9, 10, 11, 13), (1, 3, 12, 7, 0)]),
                                        (6, [(0, 1, 2, 3, 4, 5), (3, 6, 9, 12, 1, 13), (8, 9, 10, 11, 12, 13)])])
@pytest.mark.parametrize("n", [14, 9])
def test_apply_fp64_parity(k, qs_list, n):
    """One fused complex128 gate (k = 6: the row-split tile kernel; n = 9: the
    per-group kernel of tiny states) against the oracle's fp64 apply."""
    qs_list = [qs for qs in qs_list if max(qs) < n] or [tuple(range(n - k, n))]
    for i, qs in enumerate(qs_list):
        rs = np.random.default_rng(10 * k + i)
        M = W.haar_unitary(1 << k, rs)
        psi = _state128(n, 3 + i)
        h = sv.sv_create_ex(n, precision=1)
        try:
            sv.sv_set_state_c128(h, psi)
            sv.sv_apply_fused_c128(h, list(qs), M)
            got = sv.sv_get_state_c128(h, n)
        finally:
            sv.sv_destroy(h)
        ref = osv.apply_gate(psi, n, list(qs), M)
        bound = osv.apply_gate(np.abs(psi).astype(np.complex128), n, list(qs), np.abs(M).astype(np.complex128)).real
        assert np.all(np.abs(got - ref) <= (4 * ((1 << k) + 1) + 2) * U64 * bound + 1e-300), qs


@pytest.mark.parametrize("n,F", [(12, 0), (12, 4), (16, 2), (20, 4), (20, 5), (16, 6), (20, 6)])
def test_rqc_fp64_matches_oracle(n, F):
    gates = W.rqc(n, 14, seed=n)
    ref = ref_c.run(n, gates)
    h = sv.sv_create_ex(n, precision=1)
    try:
        sv.sv_run_circuit(h, gates, F)
        got = sv.sv_get_state_c128(h, n)
    finally:
        sv.sv_destroy(h)
    assert osv.fidelity(got, ref) >= 1 - 1e-12
    assert np.abs(got - ref).max() <= 1e-12 * 2.0 ** (-n / 2) * 14


def test_fp64_vs_fp32_no_substantial_disparity():
    """fp64 and fp32 states agree (here: fidelity 1 - 1e-5)."""
    n = 20
    gates = W.rqc(n, 14)
    out = {}
    for prec in (0, 1):
        h = sv.sv_create_ex(n, precision=prec)
        try:
            sv.sv_run_circuit(h, gates, 4)
            out[prec] = sv.sv_get_state_c128(h, n)
        finally:
            sv.sv_destroy(h)
    assert osv.fidelity(out[0], out[1]) >= 1 - 1e-5


@pytest.mark.parametrize("n", [3, 10, 17])
def test_sampler_fp64_bit_exact(n):
    psi = _state128(n, 40 + n)
    ref, _ = osample.sample(psi, 77, 3000)
    h = sv.sv_create_ex(n, precision=1)
    try:
        sv.sv_set_state_c128(h, psi)
        got = sv.sv_sample(h, 77, 3000)
        idx = np.arange(0, 1 << n, 7, dtype=np.uint64)
        assert np.array_equal(sv.sv_amplitudes_c128(h, idx), psi[idx.astype(np.int64)])
    finally:
        sv.sv_destroy(h)
    assert np.array_equal(got, ref)


def test_fp64_limits():
    h = sv.sv_create_ex(10, precision=1)
    try:
        with pytest.raises(sv.SVError) as e:
            sv.sv_apply_fused_c128(h, list(range(7)), np.eye(128))
        assert e.value.code == sv.SV_EINVAL
    finally:
        sv.sv_destroy(h)


@pytest.mark.parametrize("n,F,bits", [(20, 1, 12), (20, 2, 12), (21, 1, 10), (22, 2, 11), (20, 1, 13)])
@pytest.mark.parametrize("lazy", [True, False])
def test_fp64_register_blocked_passes(n, F, bits, lazy):
    """complex128 pass-specialised kernels (16 amplitudes per thread, wide
    fold swizzle, fp64 FMAs): from the lazy |0...0> (product-state start) and
    from a written one, against the complex128 oracle at fp64 tolerance."""
    from test_gpu_circuit import _mixed_circuit, layer_depth
    for gates, d in ((W.rqc(n, 14, seed=n + F), 14), (_mixed_circuit(n, 120, seed=n), None)):
        d = d or layer_depth(gates)
        ref = ref_c.run(n, gates)
        h = sv.sv_create_ex(n, precision=1)
        try:
            sv.sv_set_blocking(h, bits)
            if not lazy:
                sv.sv_device_ptr(h)
            st = sv.sv_run_circuit(h, gates, F)
            got = sv.sv_get_state_c128(h, n)
        finally:
            sv.sv_destroy(h)
        assert st["n_passes"] > 0 and st["n_jit_passes"] == st["n_passes"], st
        assert osv.fidelity(got, ref) >= 1 - 1e-12
        assert np.abs(got - ref).max() <= 1e-12 * 2.0 ** (-n / 2) * d


# ---- sharded complex128 states (NEXT-1 with the sharded mode of row e) ----------

@pytest.mark.parametrize("world", [2, 4, 8])
@pytest.mark.parametrize("F", [0, 2, 4, 6])
def test_fp64_virtual_shards_match_oracle(world, F):
    """complex128 state split over 2/4/8 virtual shards: per-gate apply64
    launches (F = 0, 4, 6) or fp64 register-blocked passes (F = 2) between
    exchanges of 16 B amplitudes; the full state (canonicalised by exact bit
    swaps) and sampled amplitudes against the complex128 oracle."""
    n = 16 if F != 2 else 22
    gates = W.rqc(n, 12, seed=100 + world + F)
    ref = ref_c.run(n, gates)
    h = sv.sv_create_ex(n, world=world, virtual_shards=True, precision=1)
    try:
        if F == 2:
            sv.sv_set_blocking(h, 12)  # auto blocking needs >= 20 qubits per shard
        st = sv.sv_run_circuit(h, gates, F)
        idx = np.array([0, 1, 5, (1 << n) - 1, 12345 % (1 << n), (1 << (n - 1)) + 7], dtype=np.uint64)
        amps = sv.sv_amplitudes_c128(h, idx)
        got = sv.sv_get_state_c128(h, n)
    finally:
        sv.sv_destroy(h)
    assert st["n_exchanges"] > 0
    if F == 2:
        assert st["n_passes"] > 0 and st["n_jit_passes"] == st["n_passes"], st
    assert np.array_equal(amps, got[idx.astype(np.int64)])
    assert osv.fidelity(got, ref) >= 1 - 1e-12
    assert np.abs(got - ref).max() <= 1e-12 * 2.0 ** (-n / 2) * 12


@pytest.mark.parametrize("world", [2, 4])
def test_fp64_virtual_shards_apply_and_sample(world):
    """Single fused complex128 gates on global qubits (an exchange before each)
    and the sampler on the sharded, permuted state against the oracle's S5."""
    n = 14
    psi = _state128(n, 9)
    ops = [((n - 1, 2), 2), ((0, n - 2, 5), 3), ((n - 1, n - 2, 3, 1, 0, 7), 6)]
    ref = psi.copy()
    h = sv.sv_create_ex(n, world=world, virtual_shards=True, precision=1)
    try:
        sv.sv_set_state_c128(h, psi)
        for i, (qs, k) in enumerate(ops):
            M = W.haar_unitary(1 << k, np.random.default_rng(50 + i))
            sv.sv_apply_fused_c128(h, list(qs), M)
            ref = osv.apply_gate(ref, n, list(qs), M)
        samples = sv.sv_sample(h, 5, 4000)  # canonicalises the permuted map first
        got = sv.sv_get_state_c128(h, n)
    finally:
        sv.sv_destroy(h)
    assert np.abs(got - ref).max() <= 1e-13
    # the oracle's S5 on its own state: equal unless a sample falls within
    # ~1e-13 of a bin boundary
    want, _ = osample.sample(ref, 5, 4000)
    assert np.array_equal(samples, want)
