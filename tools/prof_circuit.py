"""Run a prepared RQC circuit a few times (for ncu captures of single passes).

usage: python tools/prof_circuit.py <n> <depth> <max_fused> [reps] [pass_pin] [jit] [pass_search]
The first run starts from the lazily reset |0...0> (its first pass
synthesises the zero tiles); later runs reset in between the same way."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_markidis23_b200 as sv  # noqa: E402
from workloads import rqc as W  # noqa: E402

n, d, F = (int(x) for x in sys.argv[1:4])
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 1
h = sv.sv_create(n)
if len(sys.argv) > 5:
    sv.sv_set_option(h, sv.SV_OPT_PASS_PIN, int(sys.argv[5]))
if len(sys.argv) > 6:
    sv.sv_set_option(h, sv.SV_OPT_PASS_JIT, int(sys.argv[6]))
if len(sys.argv) > 7:
    sv.sv_set_option(h, sv.SV_OPT_PASS_SEARCH, int(sys.argv[7]))
c = sv.sv_circuit_create(h, W.rqc(n, d), F)
for _ in range(reps):
    sv.sv_reset(h)
    sv.sv_circuit_run_device(h, c)
sv.sv_synchronize(h)
print("passes", sv.sv_circuit_stats(c)["n_passes"])
