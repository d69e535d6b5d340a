"""CPU-only checks of the C-ABI library (no GPU needed):

* libsvb200.so loads and exports every function include/sv.h declares;
* the host fuser (sv_fusion_plan) reproduces the oracle's S3 plan bit for bit
  and its fp64 fused matrices (sv_fused_matrix) within 1e-12;
* the host planner (sv_shard_plan) reproduces the oracle's S4 events bit for
  bit;
* argument validation returns the documented error codes before any device
  work.
"""
import os
import re

import numpy as np
import pytest

import paper_conf_sc_markidis23_b200 as sv
from oracle import fuse as ofuse
from oracle import plan as oplan
from workloads import rqc as W

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_sc_markidis23_b200.build import build
    build()


def test_exports_match_header():
    hdr = open(os.path.join(ROOT, "include", "sv.h")).read()
    declared = set(re.findall(r"^(?:int|const char\*)\s+(sv_\w+)\s*\(", hdr, flags=re.M))
    assert declared, "no declarations parsed"
    L = sv.lib()
    for name in declared:
        assert hasattr(L, name), name
    assert declared == set(sv.EXPORTED)
    assert sv.sv_version().startswith("svb200")


def _circuits():
    yield "rqc12", W.rqc(12, 14)
    yield "rqc30", W.rqc(30, 14)
    yield "rqc36", W.rqc(36, 20)
    yield "rand", W.random_circuit(11, 200, 5, two_qubit_frac=0.4)
    yield "syc30", W.sycamore_rqc(30, 14)
    yield "syc36", W.sycamore_rqc(36, 20)


@pytest.mark.parametrize("F", range(7))
def test_fusion_plan_bit_exact(F):
    for name, gates in _circuits():
        got = sv.sv_fusion_plan(gates, F)
        ref = ofuse.plan_stream(ofuse.fuse_plan([g.qubits for g in gates], F))
        assert np.array_equal(got, ref), (name, F)


@pytest.mark.parametrize("F", [1, 2, 4, 6])
def test_fused_matrices_fp64(F):
    gates = W.random_circuit(9, 60, 100 + F, two_qubit_frac=0.4)
    plan = ofuse.fuse(gates, F)
    for i, (Q, mem, M) in enumerate(plan):
        got = sv.sv_fused_matrix(gates, F, i, len(Q))
        assert np.abs(got - M).max() < 1e-12
        # rounding to complex64 agrees to within one ulp
        a, b = got.astype(np.complex64), M.astype(np.complex64)
        assert np.all(np.abs(a - b) <= np.spacing(np.maximum(np.abs(a.real), np.abs(a.imag))).max() + 0)


@pytest.mark.parametrize("n,d,g,F,vmin", [(12, 14, 1, 4, 5), (20, 14, 2, 4, 5), (30, 14, 3, 2, 5),
                                           (34, 20, 1, 4, 5), (34, 20, 2, 4, 5), (36, 20, 3, 4, 5),
                                           (36, 20, 2, 6, 5), (16, 14, 3, 3, 0), (14, 14, 2, 5, 2)])
def test_shard_plan_bit_exact(n, d, g, F, vmin):
    gates = W.rqc(n, d)
    fs = sv.sv_fusion_plan(gates, F)
    fq = [Q for Q, _ in ofuse.fuse_plan([x.qubits for x in gates], F)]
    ev, pos = oplan.plan_sharded(fq, n, g, vmin)
    got, gpos = sv.sv_shard_plan(fs, n, g, vmin)
    assert np.array_equal(got, oplan.plan_stream(ev))
    assert list(gpos) == list(pos)


@pytest.mark.parametrize("F", [1, 2, 4])
def test_diag_masks_match_oracle(F):
    """The C++ block-diagonal test on the fp64 fused matrices equals
    oracle/plan.diag_qubits on the oracle's fused matrices."""
    for name, gates in [("rqc20", W.rqc(20, 14)), ("syc16", W.sycamore_rqc(16, 8)),
                        ("mixed", W.random_circuit(10, 80, 3, two_qubit_frac=0.4))]:
        got = sv.sv_fusion_diag_masks(gates, F)
        ref = [sum(1 << q for q in oplan.diag_qubits(Q, M)) for Q, _, M in ofuse.fuse(gates, F)]
        assert [int(x) for x in got] == ref, name


@pytest.mark.parametrize("n,d,g,F", [(36, 20, 3, 1), (36, 20, 2, 1), (35, 20, 1, 1), (36, 20, 3, 2), (34, 20, 1, 4),
                                     (20, 14, 2, 1), (16, 14, 3, 2)])
def test_shard_plan_diag_skip_bit_exact(n, d, g, F):
    """Diagonal exchange skip (reading R10): the C++ planner equals the
    oracle's bit for bit; it never needs more exchanges than plain S4
    (36q D20 F=1 at P=8: 7 -> 4)."""
    gates = W.rqc(n, d)
    fs = sv.sv_fusion_plan(gates, F)
    fq = [Q for Q, _ in ofuse.fuse_plan([x.qubits for x in gates], F)]
    dm = sv.sv_fusion_diag_masks(gates, F)
    diag = [{q for q in range(n) if (int(m) >> q) & 1} for m in dm]
    ev, pos = oplan.plan_sharded(fq, n, g, 5, diag=diag)
    got, gpos = sv.sv_shard_plan_diag(fs, dm, n, g, 5)
    assert np.array_equal(got, oplan.plan_stream(ev))
    assert list(gpos) == list(pos)
    ev0, _ = oplan.plan_sharded(fq, n, g, 5)
    nx, nx0 = sum(e[0] == "X" for e in ev), sum(e[0] == "X" for e in ev0)
    assert nx <= nx0
    if (n, g, F) == (36, 3, 1):
        assert (nx0, nx) == (7, 4)


def test_error_codes():
    gates = W.rqc(12, 14)
    with pytest.raises(sv.SVError) as e:
        sv.sv_fusion_plan(gates, 7)
    assert e.value.code == sv.SV_EINVAL
    bad = sv.as_gates(gates[:3])
    bad["nq"][1] = 3
    with pytest.raises(sv.SVError) as e:
        sv.sv_fusion_plan(bad, 2)
    assert e.value.code == sv.SV_EINVAL
    bad = sv.as_gates(gates[12:14])
    bad["q"][0] = [5, 5]
    with pytest.raises(sv.SVError) as e:
        sv.sv_fusion_plan(bad, 2)
    assert e.value.code == sv.SV_EINVAL
    with pytest.raises(sv.SVError) as e:
        sv.sv_shard_plan(np.array([2, 0, 40, 1, 0], np.int32), 12, 1)
    assert e.value.code == sv.SV_EINVAL
    # sv_create validates n before touching the device
    with pytest.raises(sv.SVError) as e:
        sv.sv_create(0)
    assert e.value.code == sv.SV_EINVAL
    with pytest.raises(sv.SVError) as e:
        sv.sv_create_ex(20, world=3)
    assert e.value.code == sv.SV_EUNSUPPORTED


def test_gate_struct_layout():
    g = sv.as_gates([W.Gate(0, "cz", (3, 1), W.GATE_CZ)])
    assert g.itemsize == 272 and g["nq"][0] == 2 and list(g["q"][0]) == [3, 1]
    assert g["m"][0][15] == -1 and g["m"][0][0] == 1


PTXAS = "/usr/local/cuda/bin/ptxas"


@pytest.mark.skipif(not os.path.exists(PTXAS), reason="ptxas not installed")
@pytest.mark.parametrize("n,d,F,T", [(30, 14, 1, 13), (24, 14, 2, 12), (20, 10, 1, 10)])
def test_pass_kernels_assemble(n, d, F, T, tmp_path):
    """The PTX of every pass-specialised kernel (one per register-blocked
    pass, plus the |0...0> form of the first) assembles for sm_100a within
    128 registers (ptxas may spill a few loop-invariant thread constants,
    reloaded once per tile); one kernel per pass of the block plan."""
    import subprocess
    gates = W.rqc(n, d)
    srcs = sv.sv_pass_kernels(gates, F, T)
    plan = sv.sv_block_plan(gates, F, T)
    assert len(srcs) == len(plan) + 1
    for i, src in enumerate(srcs[:4] + srcs[-1:]):
        p = tmp_path / f"k{i}.ptx"
        p.write_text(src)
        out = subprocess.run([PTXAS, "-arch=sm_100a", "-v", str(p), "-o", str(tmp_path / f"k{i}.cubin")],
                             capture_output=True, text=True)
        assert out.returncode == 0, out.stderr[-2000:]
        spill = int(re.search(r"(\d+) bytes spill stores", out.stderr).group(1))
        assert spill <= 512, out.stderr[-800:]
    assert "zinit" in srcs[1] and "zinit" not in srcs[0]
    assert " bins" in srcs[-1].split("\n")[1]  # the last pass writes the sampler bins


def test_options_validate():
    with pytest.raises(sv.SVError) as e:
        sv.sv_set_option(0, sv.SV_OPT_PASS_JIT, 1)
    assert e.value.code == sv.SV_EINVAL
