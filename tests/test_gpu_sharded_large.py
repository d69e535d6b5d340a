"""Sharded mode at full shard size on one GPU.

The north-star run is 36 qubits over 8 GPUs: shards of 2^33 amplitudes
(64 GiB).  One B200 holds a 34-qubit state (128 GiB), so:

* 34q D20 as P = 2 virtual shards (2^33 amplitudes each = the 36q/P=8 shard),
  and as P = 4 / 8 virtual shards, against an unsharded 34q run of the same
  circuit on 2^20 sampled amplitudes (north-star max-abs bound), then the
  inverse circuit brings the sharded state back to |0...0> (|<0|psi>|^2 >=
  1 - 2e-5; the oracle cannot hold 2^34 amplitudes, PAPER.md L229 / SURVEY
  §8c "parity not pinnable by the oracle" at >= 32 q);
* 33q D20 in the multi-process mode (2 processes, one 32 GiB shard each,
  CUDA-IPC peer mapping, device barriers, P2P exchange kernel) sharing one
  GPU, against the unsharded 33q state on the same sampled amplitudes.
"""
import os
import subprocess
import sys

import numpy as np
import pytest

import paper_conf_sc_markidis23_b200 as sv
from workloads import rqc as W

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NS_BOUND = lambda n, d: 1e-5 * 2.0 ** (-n / 2) * d  # noqa: E731  north-star max-abs bound


def _free_gib():
    import torch
    free, _ = torch.cuda.mem_get_info()
    return free / 2 ** 30


def _unsharded_amplitudes(n, gates, F, idx):
    h = sv.sv_create(n)
    try:
        st = sv.sv_run_circuit(h, gates, F)
        return sv.sv_amplitudes(h, idx), st
    finally:
        sv.sv_destroy(h)


@pytest.fixture(scope="module")
def ref34():
    n, d, F = 34, 20, 1
    if _free_gib() < 140:
        pytest.skip("needs ~140 GiB of free device memory")
    gates = W.rqc(n, d)
    idx = np.random.default_rng(34).integers(0, 1 << n, size=1 << 20).astype(np.uint64)
    amps, st = _unsharded_amplitudes(n, gates, F, idx)
    return n, d, F, gates, idx, amps


@pytest.mark.parametrize("world", [2, 4, 8])
def test_34q_virtual_shards_match_unsharded_and_invert(ref34, world):
    n, d, F, gates, idx, ref = ref34
    h = sv.sv_create_ex(n, world=world, virtual_shards=True)
    try:
        st = sv.sv_run_circuit(h, gates, F)
        got = sv.sv_amplitudes(h, idx)
        assert st["n_exchanges"] >= 1 and st["n_passes"] > 0, st
        err = float(np.abs(got.astype(np.complex128) - ref.astype(np.complex128)).max())
        assert err <= NS_BOUND(n, d), (err, NS_BOUND(n, d))
        # inverse circuit on the sharded state: back to |0...0>
        sv.sv_run_circuit(h, W.inverse_circuit(gates), F)
        a0 = sv.sv_amplitudes(h, np.array([0, 1, 1 << (n - 1)], dtype=np.uint64))
        assert abs(a0[0]) ** 2 >= 1 - 2e-5, a0
        assert abs(a0[1]) < 1e-3 and abs(a0[2]) < 1e-3, a0
    finally:
        sv.sv_destroy(h)


def test_33q_two_processes_one_gpu(tmp_path):
    """Two processes, one shard each (2^32 amplitudes), through the IPC path."""
    n, d, F = 33, 20, 1
    if _free_gib() < 72:
        pytest.skip("needs ~72 GiB of free device memory")
    gates = W.rqc(n, d, seed=33)
    idx = np.random.default_rng(33).integers(0, 1 << n, size=1 << 20).astype(np.uint64)
    ref, _ = _unsharded_amplitudes(n, gates, F, idx)
    np.save(tmp_path / "idx.npy", idx)
    np.save(tmp_path / "ref.npy", ref)
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr", "127.0.0.1", "--master-port", "29633", os.path.join(ROOT, "tools", "mp_large.py"),
           str(n), str(d), str(F), str(tmp_path)]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT)
    out = r.stdout + r.stderr
    assert r.returncode == 0 and "MP_LARGE_OK" in out, out[-4000:]
