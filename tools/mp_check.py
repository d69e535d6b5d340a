"""Multi-process sharded mode check (one process per shard).

Launched by tests/test_gpu_multiproc.py as
  python -m torch.distributed.run --nproc-per-node P --master-addr 127.0.0.1 ... tools/mp_check.py N
Every rank owns one shard (sv_create_ex(world=P, rank, virtual_shards=0));
the shards are cross-mapped with CUDA IPC handles exchanged through
torch.distributed (gloo all_gather_object -- plumbing only).  Ranks map onto
cuda:(local_rank % device_count), so P processes can share one GPU.

Rank 0 checks the sharded results against the oracle and prints OK.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch
import torch.distributed as dist

import paper_conf_sc_markidis23_b200 as sv
from oracle import ref_c
from oracle import sample as osample
from oracle import sv as osv
from workloads import rqc as W


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 14
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    local = int(os.environ.get("LOCAL_RANK", "0"))
    dev = local % torch.cuda.device_count()
    torch.cuda.set_device(dev)
    h = sv.sv_create_ex(n, world=world, rank=rank, virtual_shards=False, device=dev)
    blobs = [None] * world
    dist.all_gather_object(blobs, sv.sv_ipc_handle(h))
    sv.sv_attach_peers(h, blobs)
    ok = True
    msgs = []
    # 1. circuit through exchanges
    gates = W.rqc(n, 14, seed=3)
    st = sv.sv_run_circuit(h, gates, 4)
    psi = sv.sv_get_state(h, n)
    ref = ref_c.run(n, gates)
    fid = osv.fidelity(psi.astype(np.complex128), ref)
    err = float(np.abs(psi.astype(np.complex128) - ref).max())
    if not (fid >= 1 - 1e-5 and err <= osv.max_abs_bound(n, 14) and st["n_exchanges"] >= 1):
        ok = False
        msgs.append(f"circuit fid={fid} err={err} exch={st['n_exchanges']}")
    # 1c. register-blocked passes inside the shards between exchanges (F = 1, tile 10)
    sv.sv_set_blocking(h, 10)
    sv.sv_reset(h)
    st1 = sv.sv_run_circuit(h, gates, 1)
    psi1 = sv.sv_get_state(h, n)
    sv.sv_set_blocking(h, -1)
    fid1 = osv.fidelity(psi1.astype(np.complex128), ref)
    err1 = float(np.abs(psi1.astype(np.complex128) - ref).max())
    if not (fid1 >= 1 - 1e-5 and err1 <= osv.max_abs_bound(n, 14) and st1["n_passes"] >= 1):
        ok = False
        msgs.append(f"blocked F=1 fid={fid1} err={err1} passes={st1['n_passes']}")
    # 1b. F = 5 (int8 tensor-core apply inside the shards when >= 13 local qubits)
    sv.sv_reset(h)
    st5 = sv.sv_run_circuit(h, gates, 5)
    psi5 = sv.sv_get_state(h, n)
    fid5 = osv.fidelity(psi5.astype(np.complex128), ref)
    err5 = float(np.abs(psi5.astype(np.complex128) - ref).max())
    if not (fid5 >= 1 - 1e-5 and err5 <= osv.max_abs_bound(n, 14)):
        ok = False
        msgs.append(f"circuit F=5 fid={fid5} err={err5} exch={st5['n_exchanges']}")
    # 2. amplitudes
    idx = np.random.default_rng(1).integers(0, 1 << n, size=200).astype(np.uint64)
    amps = sv.sv_amplitudes(h, idx)
    if not np.array_equal(amps, psi5[idx.astype(np.int64)]):
        ok = False
        msgs.append("amplitudes mismatch")
    # 3. sampling on a seeded state: bit-exact vs the oracle
    s0 = W.random_state_c64(n, 11)
    sv.sv_set_state(h, s0)
    got = sv.sv_sample(h, 42, 4000)
    exp, _ = osample.sample(s0, 42, 4000)
    if not np.array_equal(got, exp):
        ok = False
        msgs.append("sampling mismatch")
    # 4. single apply touching a global qubit (exchange inside sv_apply_fused)
    sv.sv_set_state(h, s0)
    M = W.haar_unitary(4, np.random.default_rng(5)).astype(np.complex64)
    sv.sv_apply_fused(h, [n - 1, 2], M)
    got = sv.sv_get_state(h, n).astype(np.complex128)
    exp = osv.apply_gate(s0.astype(np.complex128), n, [n - 1, 2], M.astype(np.complex128))
    if np.abs(got - exp).max() > 1e-6:
        ok = False
        msgs.append(f"apply with global qubit err={np.abs(got - exp).max()}")
    # 5. complex128 shards (NEXT-1): per-gate fp64 applies and fp64 passes
    #    between exchanges of 16 B amplitudes, amplitudes, sampling
    h64 = sv.sv_create_ex(n, world=world, rank=rank, virtual_shards=False, device=dev, precision=1)
    blobs64 = [None] * world
    dist.all_gather_object(blobs64, sv.sv_ipc_handle(h64))
    sv.sv_attach_peers(h64, blobs64)
    for F, bits in ((4, -1), (1, 10)):
        sv.sv_set_blocking(h64, bits)
        sv.sv_reset(h64)
        st64 = sv.sv_run_circuit(h64, gates, F)
        p64 = sv.sv_get_state_c128(h64, n)
        f64 = osv.fidelity(p64, ref)
        e64 = float(np.abs(p64 - ref).max())
        if not (f64 >= 1 - 1e-12 and e64 <= 1e-12 * 2.0 ** (-n / 2) * 14 and st64["n_exchanges"] >= 1):
            ok = False
            msgs.append(f"complex128 F={F} fid={f64} err={e64} exch={st64['n_exchanges']}")
    a64 = sv.sv_amplitudes_c128(h64, idx)
    if not np.array_equal(a64, p64[idx.astype(np.int64)]):
        ok = False
        msgs.append("complex128 amplitudes mismatch")
    s1 = s0.astype(np.complex128)
    sv.sv_set_state_c128(h64, s1)
    got64 = sv.sv_sample(h64, 42, 4000)
    exp64, _ = osample.sample(s1, 42, 4000)
    if not np.array_equal(got64, exp64):
        ok = False
        msgs.append("complex128 sampling mismatch")
    sv.sv_destroy(h64)
    flags = [None] * world
    dist.all_gather_object(flags, (ok, msgs))
    sv.sv_destroy(h)
    dist.barrier()
    if rank == 0:
        if all(f[0] for f in flags):
            print(f"MP_OK world={world} n={n}")
        else:
            print("MP_FAIL", flags)
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
