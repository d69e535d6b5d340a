"""The opt-in tcgen05 tensor-core path (SVB200_TC=1, k = 4, 5): parity of a
single fused apply against the oracle within the kernel error bound, and the
systematic norm shrinkage that keeps it off by default."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_tc_single_apply_parity_and_bias():
    env = dict(os.environ, SVB200_TC="1")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "tc_check.py")], capture_output=True, text=True,
                       timeout=600, env=env, cwd=ROOT)
    line = [x for x in r.stdout.splitlines() if x.startswith("TC_CHECK")]
    assert r.returncode == 0 and line, r.stdout + r.stderr
    worst = float(line[0].split("worst_error_over_bound=")[1].split()[0])
    drift = float(line[0].split("mean_norm_change_per_apply=")[1])
    assert worst <= 1.0
    assert -5e-6 < drift < 0.0  # documented truncation bias: small and shrinking
