#!/usr/bin/env python3
"""Benchmark of the B200 state-vector hot path (BASELINE.json metric).

Metric: RQC circuit time in seconds (lower is better) and the apply kernels'
achieved HBM bandwidth.  N=1 workload: BASELINE.json configs[1], the paper's
30-qubit RQC at depth 14 "with optimal fusion" (north star):
the same device step is first timed for max_fused = 1..6 with the library's
default execution path for each (register-blocked passes for max_fused <= 2,
one launch per fused gate otherwise; `fusion_sweep_s`), and the fastest
max_fused is the timed configuration (`--max-fused F` fixes it instead; the
paper found 4 optimal on its GPUs, L189).  A "step" is one pass of the whole
hot path: |0..0> init, every fused-gate apply of the
circuit, and drawing 10^6 samples.

  value  -- device time per step with the fused circuit already resident
            (sv_circuit_run_device + sv_sample_device), CUDA events on the
            library's stream, max over ranks.
  e2e    -- the same step through the public C ABI with host buffers:
            sv_reset + sv_run_circuit (host gates -> fusion -> upload ->
            kernels) + sv_sample into host memory.

N>1 (torchrun): the multi-process sharded mode (one shard per GPU, P2P
exchanges) on BASELINE configs[4]: 36 qubits at depth 20 over 4 or 8 GPUs
(35 qubits over 2: 36 q needs 256 GiB per GPU there), strong scaling; the
line adds "exchange" (exchange time, bytes each GPU sends, NVLink GB/s and
fraction of 900 GB/s, and an s = 1..log2 N exchange microbenchmark).  --weak:
2^30 amplitudes per GPU (n = 30 + log2 N) at depth 14.

--impl reference: the CPU oracle (oracle/sv_ref.c, complex128, unfused,
OpenMP on the host cores) on a bounded sample of the same workload: a step
is one gate of the circuit; value = seconds per circuit from the per-gate
means.  --cpu-full times the whole circuit on the oracle once.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from workloads import rqc as W  # noqa: E402

N_SAMPLES = 1_000_000
REASON_BITS = {
    0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
    0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
    0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting",
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--qubits", type=int, default=0, help="0: the BASELINE config for this N (workload_size)")
    ap.add_argument("--depth", type=int, default=0, help="0: 14 at N = 1, 20 for the sharded 35/36q runs")
    ap.add_argument("--weak", action="store_true", help="N > 1: 2^30 amplitudes per GPU at depth 14 instead of 36q D20")
    ap.add_argument("--max-fused", type=int, default=-1,
                    help="-1 (default): optimal over 1..6 from the fusion sweep at N = 1; 1 for N > 1")
    ap.add_argument("--seed", type=int, default=2023)
    ap.add_argument("--workload", default="rqc", choices=["rqc", "sycamore"],
                    help="rqc: Boixo-v2 RQC (the paper's workload); sycamore: fSim + sqrt(X/Y/W) RQC (NEXT-4), "
                         "depth = cycles")
    ap.add_argument("--samples", type=int, default=N_SAMPLES)
    ap.add_argument("--block-bits", type=int, default=-1, help="cache-blocked passes: tile qubits (0 = off; -1 = library default)")
    ap.add_argument("--pass-pin", type=int, default=0, help="fix SV_OPT_PASS_PIN (3: 64 B runs, 4: 128 B) instead of sweeping")
    ap.add_argument("--pass-search", type=int, default=0, help="fix SV_OPT_PASS_SEARCH (1: greedy, 5: searched) instead of sweeping")
    ap.add_argument("--precision", type=int, default=32, choices=[32, 64], help="complex64 (32) or complex128 (64) state")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-sweep", action="store_true",
                    help="skip the max_fused = 1..6 sweep (N = 1) that reports the optimal fusion")
    ap.add_argument("--no-exchange-micro", action="store_true", help="N > 1: skip the s = 1..g exchange microbenchmark")
    ap.add_argument("--cpu-seconds", type=float, default=15.0, help="oracle sample length of cpu_baseline")
    ap.add_argument("--cpu-budget", type=float, default=150.0, help="--impl reference: stop after this many seconds")
    ap.add_argument("--cpu-full", action="store_true", help="time the whole circuit on the oracle once and exit")
    return ap.parse_args()


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d.get("hbm_gbs", 6650.0)), "measured"
    return 6650.0, "fallback"


def load_traffic(kernel_class: str):
    """Per-launch dram bytes of the dominant kernel from the committed ncu
    summary (profiles/ncu_summary.json), if present."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        d = json.load(open(p))
        return d.get("traffic_per_launch", {}).get(kernel_class)
    except Exception:
        return None


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index),
                 "--query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.active",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 3:
                try:
                    self.rows.append((float(parts[0]), float(parts[1]), int(parts[2], 16), time.time()))
                except ValueError:
                    pass

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def wait_ready(self, timeout: float = 5.0):
        """Block until nvidia-smi delivers its first sample (its start-up
        takes longer than a short timed region)."""
        t0 = time.time()
        while self.proc and not self.rows and time.time() - t0 < timeout:
            time.sleep(0.02)

    def mark(self, t0: float, t1: float):
        self.window = (t0, t1)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        rows = self.rows
        w = getattr(self, "window", None)
        if w:  # samples taken during the timed region (100 ms period), else the nearest ones
            inside = [r for r in rows if w[0] - 0.05 <= r[3] <= w[1] + 0.15]
            rows = inside or sorted(rows, key=lambda r: min(abs(r[3] - w[0]), abs(r[3] - w[1])))[:2]
        load = [r for r in rows if not (r[2] & 0x1)] or rows
        reasons = set()
        for r in load:
            for bit, name in REASON_BITS.items():
                if r[2] & bit and bit != 0x1:
                    reasons.add(name)
        return {"sm_mhz": statistics.median(r[0] for r in load), "sm_max_mhz": max(r[1] for r in self.rows),
                "reasons": sorted(reasons), "samples": len(load)}


# ----------------------------------------------------------------------------- CPU oracle
def host_info():
    """Cores the oracle uses, CPU model and RAM of this host."""
    import psutil

    from oracle import ref_c
    model = None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"cores": ref_c.threads(), "cpu_model": model, "ram_gib": round(psutil.virtual_memory().total / 2 ** 30, 1),
            "affinity": len(os.sched_getaffinity(0))}


def cpu_oracle_small(reps: int = 5):
    """BASELINE configs[0]: the whole 12q D14 circuit (121 gates, unfused),
    timed `reps` times on the host cores (mean +- sigma)."""
    from oracle import ref_c
    gates = W.rqc(12, 14, 2023)
    ref_c.run(12, gates)  # warm-up
    ts = []
    for _ in range(reps):
        t0 = time.perf_counter()
        ref_c.run(12, gates)
        ts.append(time.perf_counter() - t0)
    return {"workload": "rqc_12q_d14", "gates": len(gates), "value": statistics.mean(ts),
            "std": statistics.stdev(ts) if len(ts) > 1 else 0.0, "reps": reps, "unit": "s", "kind": "oracle",
            "sample": "measured: the whole circuit, every rep"}


def stride_order(m: int, stride: int = 7):
    """Gate order for a bounded sample whose every prefix is spread over the
    whole circuit (all moments, all gate types): 0, 7, 14, ..., 1, 8, ..."""
    return [i for o in range(stride) for i in range(o, m, stride)]


class OracleSampler:
    """The oracle (unfused complex128 C simulator, OpenMP on the host cores)
    applying the workload circuit's gates one at a time on a 2^n state, in
    stride order; per-gate times by gate size extrapolate to seconds per
    circuit: sum over the circuit's gates of the mean time of their size."""

    def __init__(self, n: int, gates):
        from oracle import ref_c
        from workloads.rqc import gate_arrays
        self.n, self.gates = n, gates
        self.L = ref_c
        self.psi = ref_c.zero_state(n)  # first touch on all host threads
        self.nq, self.qq, self.mat = gate_arrays(gates)
        self.order = stride_order(len(gates))
        self.pos = 0
        self.t = {1: [], 2: []}

    def step(self) -> float:
        i = self.order[self.pos % len(self.order)]
        self.pos += 1
        k = int(self.nq[i])
        q = np.ascontiguousarray(self.qq[i])
        m = np.ascontiguousarray(self.mat[i])
        t0 = time.perf_counter()
        rc = self.L.lib().svref_apply(self.n, k, self.L._ip(q), self.L._dp(m), self.L._dp(self.psi.view(np.float64)))
        dt = time.perf_counter() - t0
        assert rc == 0
        self.t[k].append(dt)
        return dt

    def circuit_seconds(self):
        cnt = {1: int(np.sum(self.nq == 1)), 2: int(np.sum(self.nq == 2))}
        mean = {k: (statistics.mean(v) if v else None) for k, v in self.t.items()}
        if mean[1] is None or mean[2] is None:
            allv = self.t[1] + self.t[2]
            m = statistics.mean(allv)
            return m * len(self.gates), cnt, mean
        return cnt[1] * mean[1] + cnt[2] * mean[2], cnt, mean


def cpu_oracle_sample(n: int, gates, seconds: float, make=None):
    """cpu_baseline of the bench line: the oracle on the workload circuit for a
    bounded time (gates in stride order), extrapolated to seconds per circuit
    by gate size, next to the measured 12q D14 circuit (configs[0]) and the
    committed full-circuit measurement of this workload, if any."""
    import psutil
    n_eff = n
    avail = psutil.virtual_memory().available
    while n_eff > 20 and (16 << n_eff) > 0.6 * avail:
        n_eff -= 1
    sub = (make(n_eff) if make else W.rqc(n_eff, 14, 2023)) if n_eff != n else gates
    smp = OracleSampler(n_eff, sub)
    t0 = time.perf_counter()
    while time.perf_counter() - t0 < seconds and smp.pos < len(sub):
        smp.step()
    value, cnt, mean = smp.circuit_seconds()
    scale = 2.0 ** (n - n_eff)
    value *= scale
    sample = (f"{smp.pos} of {len(sub)} unfused gates of the {n_eff}q workload circuit (stride-7 order over the whole "
              f"circuit: {len(smp.t[1])} one-qubit, {len(smp.t[2])} two-qubit) in {time.perf_counter() - t0:.1f} s; "
              f"seconds per circuit = {cnt[1]} x {mean[1] and mean[1] * 1e3:.1f} ms + {cnt[2]} x "
              f"{mean[2] and mean[2] * 1e3:.1f} ms (per-gate means by size)"
              + (f" x{scale:.0f} (2^{n - n_eff}: host RAM too small for 2^{n} complex128)" if scale > 1 else ""))
    del smp
    out = {"value": value, "unit": "s", "kind": "oracle", "sample": sample, "extrapolated": True}
    out.update(host_info())
    out["config0_12q_d14"] = cpu_oracle_small()
    full = os.path.join(ROOT, "profiles", f"cpu_oracle_{n}q.json")
    if os.path.exists(full):
        out["full_circuit_measured"] = json.load(open(full))
    return out


def cpu_oracle_full(n: int, depth: int, seed: int):
    """The whole circuit on the oracle, once (bench.py --cpu-full; minutes at 30 q)."""
    from oracle import ref_c
    gates = W.rqc(n, depth, seed)
    psi = ref_c.zero_state(n)
    t0 = time.perf_counter()
    ref_c.run(n, gates, psi)
    dt = time.perf_counter() - t0
    out = {"workload": f"rqc_{n}q_d{depth}", "gates": len(gates), "value": dt, "unit": "s", "kind": "oracle",
           "sample": "measured: the whole circuit once", "when": time.strftime("%Y-%m-%dT%H:%M:%SZ", time.gmtime())}
    out.update(host_info())
    return out


def run_reference(args):
    """--impl reference: the oracle, as it stands, on the host cores.  A step
    is ONE unfused gate of the workload circuit (stride order over the whole
    circuit) on the 2^n complex128 state; value = seconds per circuit from the
    per-gate means by gate size; ms_per_step is the measured time per step."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import psutil
    n, depth = workload_size(args, int(os.environ.get("WORLD_SIZE", "1")))
    gates = make_gates(args, n, depth)
    # the oracle state is complex128: shrink n until it fits the host RAM
    # (the per-gate times then scale by 2^(n - n_eff): bandwidth-bound)
    n_eff = n
    while n_eff > 20 and (16 << n_eff) > 0.6 * psutil.virtual_memory().available:
        n_eff -= 1
    scale = 2.0 ** (n - n_eff)
    smp = OracleSampler(n_eff, gates if n_eff == n else make_gates(args, n_eff, depth))
    for _ in range(args.warmup):
        smp.step()
    smp.t = {1: [], 2: []}
    t0 = time.perf_counter()
    steps = 0
    while steps < args.steps:
        smp.step()
        steps += 1
        if time.perf_counter() - t0 > args.cpu_budget:  # the run must end within minutes
            break
    wall = time.perf_counter() - t0
    v, cnt, mean = smp.circuit_seconds()
    v *= scale
    cfg = {"workload": f"{args.workload}_{n}q_d{depth}", "n_qubits": n, "depth": depth,
           "max_fused": "none (the oracle applies the gates unfused)", "seed": args.seed,
           "step": "one unfused gate of the circuit on the 2^n complex128 state (stride-7 order)",
           "steps_requested": args.steps}
    cpu = {"value": v, "unit": "s", "kind": "oracle", "extrapolated": True,
           "sample": f"{steps} gates in {wall:.1f} s ({len(smp.t[1])} one-qubit, {len(smp.t[2])} two-qubit); "
                     + (f"{cnt[1]} x {mean[1] * 1e3:.1f} ms + {cnt[2]} x {mean[2] * 1e3:.1f} ms"
                        if mean[1] is not None and mean[2] is not None else
                        f"{cnt[1] + cnt[2]} gates x {v / scale / max(1, cnt[1] + cnt[2]) * 1e3:.1f} ms (mean over both sizes)")
                     + (f" on {n_eff} qubits x{scale:.0f} (2^{n - n_eff}: host RAM too small for 2^{n} complex128)"
                        if scale > 1 else "")}
    cpu.update(host_info())
    out = {"impl": "reference", "metric": f"{args.workload}_circuit_time_{n}q_d{depth}", "value": v, "unit": "s",
           "n_gpus": args.gpus, "steps": steps, "warmup": args.warmup, "ms_per_step": wall / steps * 1e3,
           "higher_is_better": False, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
           "data": "synthetic", "config": cfg, "cpu_baseline": cpu,
           "e2e": {"value": v, "unit": "s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


def make_gates(args, n, depth):
    return W.sycamore_rqc(n, depth, args.seed) if args.workload == "sycamore" else W.rqc(n, depth, args.seed)


def workload_size(args, world: int):
    """N = 1: BASELINE configs[1] (30q, depth 14).  N > 1: configs[4], 36q
    depth 20 sharded over 4 / 8 GPUs and 35q at 2 GPUs (36 q needs 256 GiB
    per GPU there); --weak: 2^30 amplitudes per GPU at depth 14."""
    if args.qubits:
        return args.qubits, args.depth or (14 if world == 1 else 20)
    if world == 1:
        return 30, args.depth or 14
    if args.weak:
        return 30 + (world.bit_length() - 1), args.depth or 14
    return (35 if world == 2 else 36), args.depth or 20


# ----------------------------------------------------------------------------- ours
def exchange_micro(sv, h, n, world, cdev, reps=3):
    """s = 1 .. log2(P) global qubits swapped with local ones: one
    sv_apply_fused of an identity matrix on s currently-global logical qubits
    triggers exactly one exchange of s pairs (then a local apply).  The
    exchange kernel's own CUDA-event time (t_exchange_dev_s) gives GB/s sent
    per GPU = (1 - 2^-s) * 8 * 2^(n - g) bytes / time."""
    import torch
    g = world.bit_length() - 1
    l = n - g
    out = {}
    sv.sv_set_timing(h, True)
    for s_ in range(1, g + 1):
        ts = []
        for _ in range(reps + 1):
            pos = sv.sv_qubit_map(h, n)
            glob = [q for q in range(n) if pos[q] >= l][:s_]
            M = np.eye(1 << s_, dtype=np.complex64)
            sv.sv_last_stats(h)
            sv.sv_apply_fused(h, glob, M)
            st = sv.sv_last_stats(h)
            ts.append(st["t_exchange_dev_s"])
        t = statistics.mean(ts[1:])
        sent = (1 - 2.0 ** -s_) * 8 * 2 ** l
        tt = torch.tensor([t], device=cdev)
        import torch.distributed as dist
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t = float(tt.item())
        out[str(s_)] = {"ms": t * 1e3, "bytes_sent_per_gpu": sent, "gbs": sent / t / 1e9,
                        "nvlink_frac": sent / t / 900e9}
    sv.sv_set_timing(h, False)
    return out


def run_ours(args):
    import torch

    import paper_conf_sc_markidis23_b200 as sv

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # one rank per GPU; more ranks than GPUs (functional checks of the sharded
    # path on a small box) share devices round-robin
    dev = local % max(torch.cuda.device_count(), 1)
    torch.cuda.set_device(dev)
    dist = None
    cdev = "cuda"  # device of the small tensors the collectives carry
    shared = False
    if world > 1:
        import torch.distributed as dist
        shared = world > torch.cuda.device_count()
        # NCCL refuses two ranks on one device: gloo carries the (tiny) control
        # traffic then; the data path is our own P2P kernel either way
        dist.init_process_group("gloo" if shared else "nccl", **({} if shared else {"device_id": torch.device("cuda", dev)}))
        cdev = "cpu" if shared else "cuda"
    n, depth = workload_size(args, world)
    gates = make_gates(args, n, depth)
    stream = torch.cuda.Stream()
    fp64 = args.precision == 64
    elem = 16 if fp64 else 8
    if world == 1:
        h = sv.sv_create_ex(n, cuda_stream=stream.cuda_stream, precision=1 if fp64 else 0)
    else:
        h = sv.sv_create_ex(n, world=world, rank=rank, virtual_shards=False, cuda_stream=stream.cuda_stream)
        blob = sv.sv_ipc_handle(h)
        blobs = [None] * world
        dist.all_gather_object(blobs, blob)
        sv.sv_attach_peers(h, blobs)
    if args.block_bits >= 0:
        sv.sv_set_blocking(h, args.block_bits)
    if args.pass_pin:
        sv.sv_set_option(h, sv.SV_OPT_PASS_PIN, args.pass_pin)
    if args.pass_search:
        sv.sv_set_option(h, sv.SV_OPT_PASS_SEARCH, args.pass_search)
    samples_dev = torch.empty(args.samples, dtype=torch.int64, device="cuda")

    def barrier():
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize()

    # ---- fusion sweep (N = 1): the same device step for max_fused = 1..6,
    # CUDA events on the launching stream, 1 warm-up + 3 timed steps each;
    # the fastest max_fused becomes the timed configuration (max_fused = -1)
    sweep = None
    pin_sweep = None
    beam_sweep = None
    pass_pin = args.pass_pin or 4
    pass_beam = args.pass_search or 5
    if not fp64 and world == 1 and not args.no_sweep:
        sweep = {}
        pin_sweep = {}
        # max_fused 1..6 at the default pass runs (128 B), and F <= 2 (the
        # register-blocked passes) also with 64 B runs (SV_OPT_PASS_PIN 3)
        # and with the greedy pass formation (SV_OPT_PASS_SEARCH 1)
        beam_sweep = {}
        for f, pin, beam in ([(f, 4, 5) for f in range(1, 7)] + [(1, 3, 5), (2, 3, 5)] +
                             [(f, p, 1) for f in (1, 2) for p in (4, 3)]):
            sv.sv_set_option(h, sv.SV_OPT_PASS_PIN, pin)
            sv.sv_set_option(h, sv.SV_OPT_PASS_SEARCH, beam)
            c = sv.sv_circuit_create(h, gates, f)

            def st_f():
                sv.sv_reset(h)
                sv.sv_circuit_run_device(h, c)
                sv.sv_sample_device(h, 1, args.samples, samples_dev.data_ptr())

            st_f()
            barrier()
            a0 = torch.cuda.Event(enable_timing=True)
            a1 = torch.cuda.Event(enable_timing=True)
            a0.record(stream)
            for _ in range(3):
                st_f()
            a1.record(stream)
            barrier()
            t_f = a0.elapsed_time(a1) / 3 / 1e3
            if beam == 1:
                beam_sweep[f"{f},{pin}"] = t_f
            else:
                (sweep if pin == 4 else pin_sweep)[str(f)] = t_f
            sv.sv_circuit_destroy(c)
        sv.sv_set_option(h, sv.SV_OPT_PASS_PIN, pass_pin)
        sv.sv_set_option(h, sv.SV_OPT_PASS_SEARCH, 5)
    if args.max_fused < 0:
        if sweep:
            best = min([(v, int(f), 4, 5) for f, v in sweep.items()] + [(v, int(f), 3, 5) for f, v in pin_sweep.items()] +
                       [(v, int(k.split(",")[0]), int(k.split(",")[1]), 1) for k, v in beam_sweep.items()])
            args.max_fused, pass_pin, pass_beam = best[1], best[2], best[3]
            sv.sv_set_option(h, sv.SV_OPT_PASS_PIN, pass_pin)
            sv.sv_set_option(h, sv.SV_OPT_PASS_SEARCH, pass_beam)
            fusion_choice = ("optimal over max_fused 1..6 (fusion_sweep_s) and, for the register-blocked passes "
                             "(F <= 2), 128 B or 64 B tile runs (pass_pin_sweep_s) and greedy vs searched pass "
                             "formation (pass_search_sweep_s, SV_OPT_PASS_SEARCH 1 vs 5)")
        else:
            args.max_fused = 1 if not fp64 else 4
            fusion_choice = ("1 (the single-GPU optimum: register-blocked passes between the exchanges)" if not fp64
                             else "4 (complex128 default)")
    else:
        fusion_choice = "fixed by --max-fused"

    # ---- device step: fused circuit resident
    t_c0 = time.time()
    circ = sv.sv_circuit_create(h, gates, args.max_fused)
    t_create = time.time() - t_c0
    cst = sv.sv_circuit_stats(circ)

    def device_step():
        sv.sv_reset(h)
        sv.sv_circuit_run_device(h, circ)
        sv.sv_sample_device(h, 1, args.samples, samples_dev.data_ptr())

    for _ in range(max(args.warmup, 1)):
        device_step()
    sv.sv_synchronize(h)
    barrier()
    sv.sv_set_timing(h, True)
    sv.sv_last_stats(h)  # drain
    acc = {k: 0 for k in ("t_apply_high_dev_s", "t_apply_low_dev_s", "t_exchange_dev_s", "t_other_dev_s",
                          "n_launch_high", "n_launch_low", "n_launch_other", "bytes_apply", "bytes_apply_high",
                          "bytes_apply_low", "flops_apply", "bytes_exchange", "fma_apply", "n_exchanges")}
    last = None
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    with ClockSampler(dev) as clk:
        clk.wait_ready()
        start = torch.cuda.Event(enable_timing=True)
        end = torch.cuda.Event(enable_timing=True)
        barrier()
        t_host0 = time.time()
        start.record(stream)
        for i in range(args.steps):
            evs[i][0].record(stream)
            device_step()
            evs[i][1].record(stream)
            last = sv.sv_last_stats(h)  # syncs + collects per-launch event times of this step
            for k in acc:
                acc[k] += last[k]
        end.record(stream)
        barrier()
        clk.mark(t_host0, time.time())
        time.sleep(0.15)  # let the sampler deliver the sample that covers the end of the region
    sv.sv_set_timing(h, False)
    pass_bytes, pass_fma = sv.sv_last_pass_costs(h)  # per pass of the last timed step
    ms = start.elapsed_time(end) / args.steps
    per_step = [a.elapsed_time(b) for a, b in evs]
    t_high, t_low, t_exch = acc["t_apply_high_dev_s"], acc["t_apply_low_dev_s"], acc["t_exchange_dev_s"]
    t_apply = t_high + t_low
    ms_t = torch.tensor([ms] + per_step, device=cdev)
    if dist is not None:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
    ms = float(ms_t[0].item())
    per_step = [float(x) for x in ms_t[1:].tolist()]
    ex_t = torch.tensor([t_exch], device=cdev)
    if dist is not None:
        dist.all_reduce(ex_t, op=dist.ReduceOp.MAX)
    t_exch_max = float(ex_t.item())

    # ---- exchange microbenchmark (N > 1)
    micro = None
    if world > 1 and not args.no_exchange_micro:
        sv.sv_reset(h)
        micro = exchange_micro(sv, h, n, world, cdev)

    # ---- end-to-end through the public API with host buffers
    # the step's result lands in pinned host memory (the D2H of the e2e step)
    host_samples = torch.empty(args.samples, dtype=torch.int64, pin_memory=True).numpy().view(np.uint64)
    g_arr = sv.as_gates(gates)

    def e2e_step():
        sv.sv_reset(h)
        sv.sv_run_circuit(h, g_arr, args.max_fused)
        sv.sv_sample(h, 1, args.samples, out=host_samples)

    e2e_step()
    barrier()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e2e_steps = max(1, min(args.steps, 3))
    e0.record(stream)
    for _ in range(e2e_steps):
        e2e_step()
    e1.record(stream)
    barrier()
    e2e_ms = e0.elapsed_time(e1) / e2e_steps
    et = torch.tensor([e2e_ms], device=cdev)
    if dist is not None:
        dist.all_reduce(et, op=dist.ReduceOp.MAX)
    e2e_ms = float(et.item())
    # host -> device per e2e step: the step's input is the gate list (sv_gate
    # records with fp64 matrices) the library fuses on the host; what crosses
    # to the device is the fused matrices (kernel parameters / one upload),
    # counted as complex64 2^k x 2^k per fused gate; the larger of the two
    h2d = int(max(g_arr.nbytes, sum(8 * (1 << (2 * k)) * c for k, c in enumerate(cst["fused_hist"]))))

    peak, peak_src = load_peaks()
    steps = max(args.steps, 1)
    launches_apply = acc["n_launch_high"] + acc["n_launch_low"]
    g = world.bit_length() - 1
    bytes_per_launch = 2 * elem * (1 << (n - g))
    # algorithmic bytes the library counted for these launches (16 B per
    # amplitude per pass; 8 B for a first pass that synthesises its tiles)
    achieved = acc["bytes_apply"] / t_apply / 1e9 if t_apply > 0 and acc["bytes_apply"] else None
    frac = achieved / peak if achieved else None
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        try:
            cpu = cpu_oracle_sample(n, gates, args.cpu_seconds, lambda m: make_gates(args, m, depth))
        except Exception as ex:  # host RAM / build issues must not kill the bench line
            cpu = {"value": None, "unit": "s", "cores": os.cpu_count(), "kind": "oracle", "sample": f"failed: {ex}"}
    jit = sv.sv_jit_stats()
    if rank == 0:
        sv_fused = cst["n_fused"]
        exch_bytes = acc["bytes_exchange"] / steps
        fma = acc["fma_apply"]
        smax = clk.summary().get("sm_max_mhz") or 1965
        # FP32 ALU peak: 148 SMs x 128 FP32 lanes x 2 flop x max SM clock; the pass kernels'
        # fp32 work is FMAs (FFMA2 = 2 FMAs at half the issue rate)
        alu_peak_tflops = 148 * 128 * 2 * smax * 1e6 / 1e12 / (2 if fp64 else 1)  # fp64 FMA at half rate
        alu_ach = 2 * fma / t_apply / 1e12 if fma and t_apply else None
        alu_frac = alu_ach / alu_peak_tflops if alu_ach else None
        # per-pass roofline floor: every pass bound by max(HBM bytes / HBM peak, FMAs / FMA peak)
        floor = sum(max(float(b) / (peak * 1e9), float(f) / (alu_peak_tflops * 1e12 / 2))
                    for b, f in zip(pass_bytes, pass_fma))
        apply_step = t_apply / steps
        alu_bound = alu_frac is not None and frac is not None and alu_frac > frac
        out = {
            "metric": f"{args.workload}_circuit_time_{n}q_d{depth}" + ("_c128" if fp64 else ""),
            "value": ms / 1e3,
            "unit": "s",
            "n_gpus": world,
            "steps": args.steps,
            "warmup": args.warmup,
            "ms_per_step": ms,
            "value_std": statistics.stdev(per_step) / 1e3 if len(per_step) > 1 else 0.0,
            "step_ms": per_step,
            "higher_is_better": False,
            "scaling": "weak" if (world == 1 or args.weak) else "strong",
            "vs_baseline": None,
            "dtype": "f64" if fp64 else "f32",
            "data": "synthetic",
            "config": {
                "workload": f"{args.workload}_{n}q_d{depth}",
                "n_qubits": n, "depth": depth, "max_fused": args.max_fused, "fusion": fusion_choice,
                "execution": ("register-blocked passes (pass-specialised kernels), tile qubits "
                              f"{cst.get('block_bits', 13)}, runs of {8 << pass_pin} B (SV_OPT_PASS_PIN {pass_pin}), "
                              f"pass formation {'greedy' if pass_beam == 1 else 'searched'} (SV_OPT_PASS_SEARCH {pass_beam})"
                              if cst.get("n_passes", 0) else "one launch per fused gate"),
                "seed": args.seed,
                "gates": len(gates), "n_fused": sv_fused, "fused_hist": cst["fused_hist"],
                "samples_per_step": args.samples,
                "step": "sv_reset + all fused-gate applies (+ exchanges) + sv_sample_device(1e6)",
                "l2": f"inputs larger than L2 (state {elem << n >> 30} GiB per circuit)",
                "parallelism": "single GPU" if world == 1 else
                               f"sharded x{world} by the top {g} physical qubits (P2P exchange kernel over CUDA-IPC"
                               f"-mapped peer memory){' -- ranks SHARE GPUs: timing not meaningful' if shared else ''}",
                "passes_per_step": last["n_passes"] if last else None,
                "jit_passes_per_step": last["n_jit_passes"] if last else None,
                "apply_ms_per_step": 1e3 * t_apply / steps,
                "apply_high_ms_per_step": 1e3 * t_high / steps,
                "apply_low_ms_per_step": 1e3 * t_low / steps,
                "exchange_ms_per_step": 1e3 * t_exch_max / steps,
                "other_ms_per_step": 1e3 * acc["t_other_dev_s"] / steps,
                "apply_gbs_high": acc["bytes_apply_high"] / t_high / 1e9 if t_high else None,
                "apply_gbs_low": acc["bytes_apply_low"] / t_low / 1e9 if t_low else None,
                "apply_tflops": acc["flops_apply"] / t_apply / 1e12 if t_apply else None,
                "fuse_plan_upload_s": cst["t_fuse_s"] + cst["t_plan_s"] + cst["t_upload_s"],
                "circuit_create_s": t_create,
                "pass_kernels_compiled": jit["compiled"], "pass_kernel_compile_s": jit["compile_s"],
                "apply_launches_per_step": launches_apply // steps,
                "block_bits": args.block_bits,
            },
            "roofline": {"bound": "alu" if alu_bound else "hbm",
                         "kernel": ("rpj (pass-specialised register-blocked pass: all gates of a pass per HBM "
                                    "read + write)" if cst["n_passes"] else "apply_high+apply_low (one launch per fused gate)"),
                         "achieved": alu_ach if alu_bound else achieved,
                         "peak": alu_peak_tflops if alu_bound else peak,
                         "peak_source": ("148 SMs x 128 FP32 lanes x 2 flop x max SM clock (FMA pipe; fp64: half)"
                                         if alu_bound
                                         else peak_src),
                         "unit": "TFLOP/s" if alu_bound else "GB/s",
                         "frac": alu_frac if alu_bound else frac,
                         "hbm": {"achieved": achieved, "peak": peak, "unit": "GB/s", "frac": frac,
                                 "frac_of_8tbs": achieved / 8000.0 if achieved else None},
                         "alu": {"achieved": alu_ach, "peak": alu_peak_tflops, "unit": "TFLOP/s", "frac": alu_frac},
                         "pass_floor": ({"passes": len(pass_bytes), "floor_ms": floor * 1e3,
                                         "apply_ms": apply_step * 1e3,
                                         "frac": floor / apply_step if apply_step else None,
                                         "rule": "sum over passes of max(HBM bytes / HBM peak, FMAs / FMA peak)"}
                                        if len(pass_bytes) else None),
                         "algorithmic_bytes_per_launch": bytes_per_launch,
                         "algorithmic_bytes_per_step": acc["bytes_apply"] // steps,
                         "traffic": load_traffic("rpass" if cst["n_passes"] else "apply")},
            "cpu_baseline": cpu,
            "e2e": {"value": e2e_ms / 1e3, "unit": "s", "h2d_bytes_per_step": h2d,
                    "d2h_bytes_per_step": 8 * args.samples},
            "gpu_launches": (acc["n_launch_high"] + acc["n_launch_low"] + acc["n_launch_other"]),
            "fusion_sweep_s": sweep,
            "pass_pin_sweep_s": pin_sweep,
            "pass_search_sweep_s": beam_sweep,
            "optimal_fusion": (None if not sweep else
                               {"max_fused": args.max_fused, "pass_pin": pass_pin,
                                "value": min(list(sweep.values()) + list((pin_sweep or {}).values())), "unit": "s"}),
            "clocks": clk.summary(),
        }
        if world > 1:
            # NVLink: bytes each GPU sends per step over its exchanges' time
            # (kernel CUDA events, max over ranks) against 900 GB/s per direction
            out["exchange"] = {
                "exchanges_per_step": acc["n_exchanges"] / steps,
                "bytes_exchange_per_step": exch_bytes,
                "exchange_ms_per_step": 1e3 * t_exch_max / steps,
                "nvlink_gbs": exch_bytes / (t_exch_max / steps) / 1e9 if t_exch_max else None,
                "nvlink_frac": exch_bytes / (t_exch_max / steps) / 900e9 if t_exch_max else None,
                "nvlink_peak_gbs": 900.0,
                "micro": micro,
            }
        print(json.dumps(out), flush=True)
    sv.sv_circuit_destroy(circ)
    sv.sv_destroy(h)
    if dist is not None:
        dist.barrier()
        dist.destroy_process_group()


def main():
    args = parse()
    if args.cpu_full:
        n, depth = workload_size(args, int(os.environ.get("WORLD_SIZE", "1")))
        print(json.dumps(cpu_oracle_full(n, depth, args.seed)), flush=True)
    elif args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
