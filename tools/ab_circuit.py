"""Interleaved A/B timing of whole circuits across library builds.

usage: python tools/ab_circuit.py <rounds> <n> <depth> <max_fused> <lib.so[:jit=0|1]> [...]

Each round runs every library in its own process (SVB200_LIB selects the
build) and prints the device time of the prepared circuit (sv_circuit_run_device
after a reset, CUDA events inside the library via sv_set_timing; mean of 5) and
the per-launch apply times.  Libraries alternate every round, so drift of the
box affects all of them alike.
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import json, sys, time
sys.path.insert(0, %r)
import paper_conf_sc_markidis23_b200 as sv
from workloads import rqc as W
n, d, F = %d, %d, %d
h = sv.sv_create(n)
if %r is not None:
    sv.sv_set_option(h, sv.SV_OPT_PASS_JIT, %r)
t0 = time.perf_counter()
c = sv.sv_circuit_create(h, W.rqc(n, d), F)
t_create = time.perf_counter() - t0
for _ in range(2):
    sv.sv_reset(h); sv.sv_circuit_run_device(h, c)
sv.sv_synchronize(h)
sv.sv_set_timing(h, True)
ts = []
for _ in range(5):
    sv.sv_reset(h)
    t0 = time.perf_counter()
    sv.sv_circuit_run_device(h, c)
    sv.sv_synchronize(h)
    t1 = time.perf_counter()
    st = sv.sv_last_stats(h)
    ts.append((t1 - t0, st["t_apply_high_dev_s"] + st["t_apply_low_dev_s"] + st["t_other_dev_s"]))
print(json.dumps({"wall": sum(t[0] for t in ts) / len(ts), "dev": sum(t[1] for t in ts) / len(ts),
                  "passes": sv.sv_circuit_stats(c)["n_passes"], "create": t_create,
                  "jit_passes": st.get("n_jit_passes", 0)}))
"""


def main():
    rounds, n, d, F = (int(x) for x in sys.argv[1:5])
    libs = sys.argv[5:]
    res = {spec: [] for spec in libs}
    for r in range(rounds):
        for spec in libs:
            lib, _, opt = spec.partition(":")
            jit = int(opt.split("=")[1]) if opt.startswith("jit=") else None
            env = dict(os.environ, SVB200_LIB=os.path.abspath(lib))
            out = subprocess.run([sys.executable, "-c", CHILD % (ROOT, n, d, F, jit, jit)], env=env, capture_output=True,
                                 text=True, timeout=600)
            line = out.stdout.strip().splitlines()[-1] if out.stdout.strip() else out.stderr[-400:]
            try:
                d_ = json.loads(line)
                res[spec].append(d_["dev"])
                print(f"round {r} {os.path.basename(spec)}: dev {d_['dev'] * 1e3:.2f} ms wall {d_['wall'] * 1e3:.2f} ms "
                      f"passes {d_['passes']} jit {d_.get('jit_passes')} create {d_.get('create', 0):.2f} s", flush=True)
            except Exception:
                print(f"round {r} {os.path.basename(spec)}: FAILED {line}", flush=True)
    for lib, v in res.items():
        if v:
            v = sorted(v)
            print(f"{os.path.basename(lib)}: median {v[len(v) // 2] * 1e3:.2f} ms min {v[0] * 1e3:.2f} ms ({len(v)} runs)")


if __name__ == "__main__":
    main()
