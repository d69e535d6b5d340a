"""Multi-process sharded mode (one process per shard, CUDA IPC peer mapping,
device-side barriers, P2P exchange kernel) -- exercised with P processes on
however many GPUs the box has (they may share one GPU)."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("world,n", [(2, 14), (4, 14)])
def test_multiprocess_sharded(world, n):
    port = 29611 + world
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.join(ROOT, "tools", "mp_check.py"),
           str(n)]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    out = r.stdout + r.stderr
    assert r.returncode == 0 and f"MP_OK world={world}" in out, out[-4000:]
