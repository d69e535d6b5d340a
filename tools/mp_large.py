"""Multi-process sharded mode at large n (tests/test_gpu_sharded_large.py).

  python -m torch.distributed.run --nproc-per-node P ... tools/mp_large.py <n> <depth> <F> <dir>

Every rank owns one shard (sv_create_ex(world=P, rank, virtual_shards=0)),
shards are cross-mapped with CUDA IPC handles (torch.distributed gloo
all_gather_object: plumbing only).  Runs the RQC of <n> qubits, reads the
amplitudes at <dir>/idx.npy and compares them with <dir>/ref.npy (the
unsharded run) within the north-star max-abs bound; then runs the inverse
circuit and checks |<0|psi>|^2 >= 1 - 2e-5.  Rank 0 prints MP_LARGE_OK.
"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch
import torch.distributed as dist

import paper_conf_sc_markidis23_b200 as sv
from workloads import rqc as W


def main():
    n, d, F = (int(x) for x in sys.argv[1:4])
    path = sys.argv[4]
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    dev = int(os.environ.get("LOCAL_RANK", "0")) % torch.cuda.device_count()
    torch.cuda.set_device(dev)
    h = sv.sv_create_ex(n, world=world, rank=rank, virtual_shards=False, device=dev)
    blobs = [None] * world
    dist.all_gather_object(blobs, sv.sv_ipc_handle(h))
    sv.sv_attach_peers(h, blobs)
    idx = np.load(os.path.join(path, "idx.npy"))
    ref = np.load(os.path.join(path, "ref.npy"))
    gates = W.rqc(n, d, seed=33)
    msgs = []
    t0 = time.time()
    st = sv.sv_run_circuit(h, gates, F)
    t1 = time.time()
    got = sv.sv_amplitudes(h, idx)
    err = float(np.abs(got.astype(np.complex128) - ref.astype(np.complex128)).max())
    bound = 1e-5 * 2.0 ** (-n / 2) * d
    if not (err <= bound and st["n_exchanges"] >= 1):
        msgs.append(f"forward err={err} bound={bound} exchanges={st['n_exchanges']}")
    sv.sv_run_circuit(h, W.inverse_circuit(gates), F)
    a0 = sv.sv_amplitudes(h, np.array([0], dtype=np.uint64))
    if not abs(a0[0]) ** 2 >= 1 - 2e-5:
        msgs.append(f"inverse |<0|psi>|^2 = {abs(a0[0]) ** 2}")
    flags = [None] * world
    dist.all_gather_object(flags, (not msgs, msgs, st["n_exchanges"], st["n_passes"], t1 - t0))
    sv.sv_destroy(h)
    dist.barrier()
    if rank == 0:
        if all(f[0] for f in flags):
            print(f"MP_LARGE_OK world={world} n={n} exchanges={flags[0][2]} passes={flags[0][3]} "
                  f"forward_s={flags[0][4]:.2f} max_err={err:.3e} bound={bound:.3e}")
        else:
            print("MP_LARGE_FAIL", flags)
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
