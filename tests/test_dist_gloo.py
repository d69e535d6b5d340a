"""N>1 host logic on CPU: world-size 2/4 gloo process groups execute the C++
planner's sharded event stream (sv_fusion_plan + sv_shard_plan from
libsvb200, host-only calls) with real rank-to-rank chunk exchanges, and the
gathered state must equal the unsharded oracle.

Each rank owns 2^(n-g) amplitudes (physical top g bits = rank).  APPLY
events run the oracle's apply on the local shard; an EXCHANGE(pairs) sends
chunk c to rank e = rank with device bits (P_j - l) := c_j and receives that
rank's chunk c_d (SURVEY.md §8c-S4 exchange semantics), exactly what the P2P
exchange kernel does in place on the GPU.
"""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n, F, q):
    import sys
    sys.path.insert(0, ROOT)
    import torch

    import paper_conf_sc_markidis23_b200 as sv
    from oracle import fuse as ofuse
    from oracle import sv as osv
    from workloads import rqc as W

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        g = world.bit_length() - 1
        l = n - g
        gates = W.rqc(n, 12, seed=7 + world)
        fs = sv.sv_fusion_plan(gates, F)
        stream, pos = sv.sv_shard_plan(fs, n, g)
        # every rank must hold the same plan
        allp = [None] * world
        dist.all_gather_object(allp, (stream.tolist(), pos.tolist()))
        same = all(x == allp[0] for x in allp)
        fused = ofuse.fuse(gates, F)
        psi0 = np.zeros(1 << n, np.complex128)
        psi0[0] = 1
        shard = psi0[rank << l:(rank + 1) << l].copy()
        loc = np.arange(1 << l)
        o = 0
        n_x = 0
        while o < len(stream):
            if stream[o] == -1:
                s = int(stream[o + 1])
                pairs = [(int(stream[o + 2 + 2 * j]), int(stream[o + 3 + 2 * j])) for j in range(s)]
                o += 2 + 2 * s
                n_x += 1
                cd = 0
                for j, (P, _) in enumerate(pairs):
                    cd |= ((rank >> (P - l)) & 1) << j
                new = shard.copy()
                for c in range(1 << s):
                    e = rank
                    for j, (P, _) in enumerate(pairs):
                        e = (e & ~(1 << (P - l))) | (((c >> j) & 1) << (P - l))
                    sel_c = np.ones(1 << l, bool)
                    sel_cd = np.ones(1 << l, bool)
                    for j, (_, p) in enumerate(pairs):
                        sel_c &= ((loc >> p) & 1) == ((c >> j) & 1)
                        sel_cd &= ((loc >> p) & 1) == ((cd >> j) & 1)
                    if e == rank:
                        continue  # c == cd: stays
                    send = torch.from_numpy(shard[sel_c].copy())
                    recv = torch.empty_like(send)
                    # deadlock-free pairwise exchange: lower rank sends first
                    if rank < e:
                        dist.send(send, e)
                        dist.recv(recv, e)
                    else:
                        dist.recv(recv, e)
                        dist.send(send, e)
                    new[sel_c] = recv.numpy()
                shard = new
            else:
                i, k = int(stream[o]), int(stream[o + 1])
                phys = [int(x) for x in stream[o + 2:o + 2 + k]]
                o += 2 + k
                assert all(p < l for p in phys)
                shard = osv.apply_gate(shard, l, phys, fused[i][2])
        allsh = [None] * world
        dist.all_gather_object(allsh, shard)
        full = np.concatenate(allsh)
        # logical index: qubit q at physical bit pos[q]
        idx = np.arange(1 << n)
        ph = np.zeros_like(idx)
        for qq in range(n):
            ph |= ((idx >> qq) & 1) << int(pos[qq])
        logical = full[ph]
        ref = osv.simulate(n, gates)
        err = float(np.abs(logical - ref).max())
        q.put((rank, same, n_x, err))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,n,F", [(2, 10, 4), (4, 11, 3), (2, 12, 2)])
def test_gloo_sharded_plan_execution(world, n, F):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n, F, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, same, n_x, err in res:
        assert same, "ranks computed different plans"
        assert n_x >= 1
        assert err < 1e-12, err
