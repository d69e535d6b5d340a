"""Per-kernel measurements for the §8 rows other than the headline step
(apply per k and qubit class, sampling, exchange, launch-bound 12q).

usage: python tools/micro_bench.py [out.json]
All timings are CUDA-event device times (sv_set_timing) or events around the
call on the library stream; rooflines use MEASURED_PEAKS.json hbm_gbs.
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_sc_markidis23_b200 as sv
from workloads import rqc as W

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PEAK = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
    os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
out = {"peak_hbm_gbs": PEAK, "apply": [], "sample": {}, "exchange": [], "small": {}}

# ---- apply sweep (n = 30) -----------------------------------------------------
CASES = {
    1: {"high": (20,), "low": (2,), "q0": (0,)},
    2: {"high": (10, 20), "low": (1, 20), "q0": (0, 20)},
    3: {"high": (5, 12, 25), "low": (2, 12, 25), "q0": (0, 12, 25)},
    4: {"high": (6, 12, 18, 24), "low": (2, 12, 18, 24), "q0": (0, 12, 18, 24), "low2": (1, 2, 12, 24),
        "run2k": (10, 11, 12, 13), "q0123": (0, 1, 2, 3)},
    5: {"high": (4, 8, 12, 18, 24), "low": (1, 8, 12, 18, 24), "q0": (0, 8, 12, 18, 24), "run1k": (10, 11, 12, 13, 14)},
    6: {"high": (4, 8, 12, 16, 20, 24), "low": (1, 3, 8, 12, 20, 24), "q0": (0, 4, 8, 12, 20, 24),
        "run1k": (12, 13, 14, 15, 16, 17)},
}
n = 30
h = sv.sv_create(n)
sv.sv_set_timing(h, True)
rs = np.random.default_rng(0)
reps = 5
for k, cl in CASES.items():
    for name, qs in cl.items():
        M = W.haar_unitary(1 << k, rs).astype(np.complex64)
        sv.sv_apply_fused(h, qs, M)
        sv.sv_synchronize(h)
        st0 = sv.sv_last_stats(h)
        for _ in range(reps):
            sv.sv_apply_fused(h, qs, M)
        st = sv.sv_last_stats(h)
        t = (st["t_apply_high_dev_s"] + st["t_apply_low_dev_s"] - st0["t_apply_high_dev_s"] - st0["t_apply_low_dev_s"]) / reps
        gbs = 16 * 2 ** n / t / 1e9
        rec = {"k": k, "class": name, "qubits": list(qs), "ms": t * 1e3, "GBps": gbs, "frac": gbs / PEAK,
               "TFLOPs": (8 * 2 ** k - 2) * 2 ** n / t / 1e12}
        out["apply"].append(rec)
        print(json.dumps(rec), flush=True)

# ---- sampling (pass 1 reads 8 B / amplitude) -----------------------------------
dev_out = torch.empty(1_000_000, dtype=torch.int64, device="cuda")
sv.sv_reset(h)
sv.sv_apply_fused(h, (0,), W.GATE_H.astype(np.complex64))
for N in (1_000, 1_000_000):
    sv.sv_sample_device(h, 1, N, dev_out.data_ptr())
    sv.sv_synchronize(h)
    st0 = sv.sv_last_stats(h)
    t0 = time.perf_counter()
    for _ in range(reps):
        sv.sv_sample_device(h, 1, N, dev_out.data_ptr())
    st = sv.sv_last_stats(h)
    t_wall = (time.perf_counter() - t0) / reps
    t = (st["t_other_dev_s"] - st0["t_other_dev_s"]) / reps
    out["sample"][str(N)] = {"device_ms": t * 1e3, "wall_ms": t_wall * 1e3, "pass1_GBps_lower_bound": 8 * 2 ** n / t / 1e9,
                             "frac_lower_bound": 8 * 2 ** n / t / 1e9 / PEAK}
    print("sample", N, out["sample"][str(N)], flush=True)
sv.sv_destroy(h)

# ---- exchange, virtual shards on one GPU (local HBM swap) -----------------------
for world in (2, 8):
    hs = sv.sv_create_ex(n, world=world, virtual_shards=True)
    sv.sv_set_timing(hs, True)
    g = world.bit_length() - 1
    for s_bits in range(1, g + 1):
        qs = list(range(n - s_bits, n))  # s global qubits -> one exchange with s pairs
        M = np.eye(1 << s_bits, dtype=np.complex64)
        sv.sv_reset(hs)
        sv.sv_synchronize(hs)
        st0 = sv.sv_last_stats(hs)
        sv.sv_apply_fused(hs, qs, M)
        st = sv.sv_last_stats(hs)
        t = st["t_exchange_dev_s"] - st0["t_exchange_dev_s"]
        moved = (1 - 2.0 ** -s_bits) * 8 * 2 ** n  # bytes that change shard, all shards
        rec = {"world": world, "s": s_bits, "ms": t * 1e3, "moved_GB": moved / 1e9,
               "local_hbm_GBps": 2 * moved / t / 1e9, "frac_hbm": 2 * moved / t / 1e9 / PEAK}
        out["exchange"].append(rec)
        print("exchange", json.dumps(rec), flush=True)
    sv.sv_destroy(hs)

# ---- launch-bound 12q circuit (config 1) ------------------------------------------
gates = W.rqc(12, 14)
h = sv.sv_create(12)
for F in (0, 4):
    c = sv.sv_circuit_create(h, gates, F)
    for _ in range(3):
        sv.sv_reset(h)
        sv.sv_circuit_run_device(h, c)
    sv.sv_synchronize(h)
    t0 = time.perf_counter()
    R = 50
    for _ in range(R):
        sv.sv_reset(h)
        sv.sv_circuit_run_device(h, c)
    sv.sv_synchronize(h)
    dt = (time.perf_counter() - t0) / R
    out["small"][f"12q_d14_f{F}"] = {"us_per_circuit": dt * 1e6, "fused": sv.sv_circuit_stats(c)["n_fused"]}
    print("small", F, out["small"][f"12q_d14_f{F}"], flush=True)
    sv.sv_circuit_destroy(c)
sv.sv_destroy(h)
if len(sys.argv) > 1:
    json.dump(out, open(sys.argv[1], "w"), indent=1)
