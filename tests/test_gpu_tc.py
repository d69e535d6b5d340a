"""The tcgen05 int8 tensor-core path of the per-gate dense apply (k = 4..6),
selected per handle with sv_set_option(SV_OPT_APPLY_PATH):

* "i8"   -- exact int8-slice path for k = 4, 5 and 6: single apply parity
  within the SIMT bound plus the slicing term, no norm bias, whole circuits
  from |0..0> within the north-star bound;
* "auto" -- the default policy (k = 5, 6 on int8 tensor cores, k <= 4 SIMT).

The TF32x3 path (biased) is quarantined: it exists only in
builds with -DSVB_TF32X3=1 and is not selectable through the C ABI.
"""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(mode):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "tc_check.py"), mode], capture_output=True,
                       text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stdout + r.stderr
    out = {}
    for x in r.stdout.splitlines():
        for tok in x.split()[1:]:
            k, v = tok.split("=")
            out[k] = float(v)
    return out


@pytest.mark.parametrize("mode", ["i8", "auto"])
def test_int8_tc_parity_unbiased(mode):
    r = _run(mode)
    assert r["worst_error_over_bound"] <= 1.0
    assert abs(r["mean_norm_change_per_apply"]) < 1e-7  # no systematic shrinkage
    assert r["worst_error_over_northstar_bound"] <= 1.0
