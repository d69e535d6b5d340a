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
exchanges), weak scaling with 2^30 amplitudes per GPU (n = 30 + log2 N)
unless --qubits is given (e.g. --qubits 36 for the north star's 36q run).

--impl reference: the CPU oracle (oracle/sv_ref.c, complex128, unfused,
OpenMP on the host cores) on a bounded sample of the same workload.
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
    ap.add_argument("--qubits", type=int, default=0)
    ap.add_argument("--depth", type=int, default=14)
    ap.add_argument("--max-fused", type=int, default=-1,
                    help="-1 (default): optimal over 1..6 from the fusion sweep (N=1; 4 for N>1)")
    ap.add_argument("--seed", type=int, default=2023)
    ap.add_argument("--samples", type=int, default=N_SAMPLES)
    ap.add_argument("--block-bits", type=int, default=-1, help="cache-blocked passes: tile qubits (0 = off; -1 = library default)")
    ap.add_argument("--precision", type=int, default=32, choices=[32, 64], help="complex64 (32) or complex128 (64) state")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-sweep", action="store_true",
                    help="skip the max_fused = 1..6 sweep (N = 1) that reports the optimal fusion")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
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
def cpu_oracle_sample(n: int, gates, seconds: float):
    """Time the oracle (unfused complex128 C simulator) on the first gates of
    the workload circuit; extrapolate to seconds per circuit."""
    import psutil

    from oracle import ref_c
    n_eff = n
    avail = psutil.virtual_memory().available
    while n_eff > 20 and (16 << n_eff) > 0.6 * avail:
        n_eff -= 1
    sub = W.rqc(n_eff, 14, 2023) if n_eff != n else gates
    done, sec = ref_c.time_gates(n_eff, sub, max_seconds=seconds)
    per_gate = sec / done
    scale = 2.0 ** (n - n_eff)
    value = per_gate * len(gates) * scale
    sample = (f"first {done} of {len(sub)} unfused gates of the {n_eff}q depth-14 RQC in {sec:.1f} s "
              f"({per_gate * 1e3:.1f} ms/gate), extrapolated x{len(gates)} gates"
              + (f" x{scale:.0f} (2^{n - n_eff}: host RAM too small for 2^{n} complex128)" if scale > 1 else ""))
    return {"value": value, "unit": "s", "cores": ref_c.threads(), "kind": "oracle", "sample": sample}


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    n = args.qubits or (30 if args.gpus == 1 else 30 + (args.gpus.bit_length() - 1))
    gates = W.rqc(n, args.depth, args.seed)
    vals = []
    last = None
    for _ in range(args.warmup):
        cpu_oracle_sample(n, gates, min(3.0, args.cpu_seconds))
    for _ in range(args.steps):
        last = cpu_oracle_sample(n, gates, args.cpu_seconds)
        vals.append(last["value"])
    v = statistics.mean(vals)
    cfg = {"workload": f"rqc_{n}q_d{args.depth}", "n_qubits": n, "depth": args.depth,
           "max_fused": "none (the oracle applies the gates unfused)", "seed": args.seed}
    last["value"] = v
    out = {"impl": "reference", "metric": f"rqc_circuit_time_{n}q_d{args.depth}", "value": v, "unit": "s",
           "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": v * 1e3,
           "higher_is_better": False, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
           "data": "synthetic", "config": cfg, "cpu_baseline": last,
           "e2e": {"value": v, "unit": "s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


# ----------------------------------------------------------------------------- ours
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
    if world > 1:
        import torch.distributed as dist
        shared = world > torch.cuda.device_count()
        # NCCL refuses two ranks on one device: gloo carries the (tiny) control
        # traffic then; the data path is our own P2P kernel either way
        dist.init_process_group("gloo" if shared else "nccl", **({} if shared else {"device_id": torch.device("cuda", dev)}))
        cdev = "cpu" if shared else "cuda"
    n = args.qubits or (30 if world == 1 else 30 + (world.bit_length() - 1))
    gates = W.rqc(n, args.depth, args.seed)
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
    samples_dev = torch.empty(args.samples, dtype=torch.int64, device="cuda")

    def barrier():
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize()

    # ---- fusion sweep (N = 1): the same device step for max_fused = 1..6,
    # CUDA events on the launching stream, 1 warm-up + 3 timed steps each;
    # the fastest max_fused becomes the timed configuration (max_fused = -1)
    sweep = None
    if not fp64 and (args.max_fused < 0 or (world == 1 and not args.no_sweep)):
        sweep = {}
        for f in range(1, 7):
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
            sweep[str(f)] = a0.elapsed_time(a1) / 3 / 1e3
            sv.sv_circuit_destroy(c)
    if args.max_fused < 0:
        best = torch.tensor([int(min(sweep, key=sweep.get)) if sweep else 4], device=cdev)
        if dist is not None:  # every rank runs rank 0's choice (collective calls)
            dist.broadcast(best, 0)
        args.max_fused = int(best.item())
        fusion_choice = "optimal over max_fused 1..6 (fusion_sweep_s)" if sweep else "4 (complex128 default)"
    else:
        fusion_choice = "fixed by --max-fused"

    # ---- device step: fused circuit resident
    circ = sv.sv_circuit_create(h, gates, args.max_fused)
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
    t_apply = t_high = t_low = t_exch = t_other = 0.0
    n_high = n_low = n_other = 0
    bytes_apply = 0
    flops = 0
    bytes_exch = 0
    fma = 0
    with ClockSampler(dev) as clk:
        clk.wait_ready()
        start = torch.cuda.Event(enable_timing=True)
        end = torch.cuda.Event(enable_timing=True)
        barrier()
        t_host0 = time.time()
        start.record(stream)
        for _ in range(args.steps):
            device_step()
            st = sv.sv_last_stats(h)  # syncs + collects per-launch event times of this step
            t_high += st["t_apply_high_dev_s"]
            t_low += st["t_apply_low_dev_s"]
            t_exch += st["t_exchange_dev_s"]
            t_other += st["t_other_dev_s"]
            n_high += st["n_launch_high"]
            n_low += st["n_launch_low"]
            n_other += st["n_launch_other"]
            bytes_apply += st["bytes_apply"]
            flops += st["flops_apply"]
            bytes_exch += st["bytes_exchange"]
            fma += st["fma_apply"]
        end.record(stream)
        barrier()
        clk.mark(t_host0, time.time())
        time.sleep(0.15)  # let the sampler deliver the sample that covers the end of the region
    sv.sv_set_timing(h, False)
    ms = start.elapsed_time(end) / args.steps
    # the per-step sv_last_stats sync adds a host round trip per step; report
    # the device-side sum of our launches as well
    t_apply = t_high + t_low
    ms_t = torch.tensor([ms], device=cdev)
    if dist is not None:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
    ms = float(ms_t.item())

    # ---- end-to-end through the public API with host buffers
    host_samples = np.empty(args.samples, dtype=np.uint64)
    g_arr = sv.as_gates(gates)

    def e2e_step():
        sv.sv_reset(h)
        sv.sv_run_circuit(h, g_arr, args.max_fused)
        out = sv.sv_sample(h, 1, args.samples)
        host_samples[:] = out

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
    launches_apply = n_high + n_low
    avg_launch = t_apply / max(launches_apply, 1)
    bytes_per_launch = 2 * elem * (1 << (n - (world.bit_length() - 1)))
    # algorithmic bytes the library counted for these launches (16 B per
    # amplitude per pass; 8 B for a first pass that synthesises |0...0>)
    achieved = (bytes_apply / t_apply / 1e9) if t_apply > 0 and bytes_apply else (
        bytes_per_launch / avg_launch / 1e9 if avg_launch > 0 else None)
    frac = achieved / peak if achieved else None
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        try:
            cpu = cpu_oracle_sample(n, gates, args.cpu_seconds)
        except Exception as ex:  # host RAM / build issues must not kill the bench line
            cpu = {"value": None, "unit": "s", "cores": os.cpu_count(), "kind": "oracle",
                   "sample": f"failed: {ex}"}
    if rank == 0:
        sv_fused = cst["n_fused"]
        out = {
            "metric": f"rqc_circuit_time_{n}q_d{args.depth}" + ("_c128" if fp64 else ""),
            "value": ms / 1e3,
            "unit": "s",
            "n_gpus": world,
            "steps": args.steps,
            "warmup": args.warmup,
            "ms_per_step": ms,
            "higher_is_better": False,
            "scaling": "weak",
            "vs_baseline": None,
            "dtype": "f64" if fp64 else "f32",
            "data": "synthetic",
            "config": {
                "workload": f"rqc_{n}q_d{args.depth}",
                "n_qubits": n, "depth": args.depth, "max_fused": args.max_fused, "fusion": fusion_choice,
                "execution": ("register-blocked passes (apply_rpass), tile qubits "
                              f"{cst.get('block_bits', 12)}" if cst.get("n_passes", 0) else "one launch per fused gate"),
                "seed": args.seed,
                "gates": len(gates), "n_fused": sv_fused, "fused_hist": cst["fused_hist"],
                "samples_per_step": args.samples,
                "step": "sv_reset + all fused-gate applies + sv_sample_device(1e6)",
                "l2": f"inputs larger than L2 (state {elem << n >> 30} GiB per circuit)",
                "parallelism": "single GPU" if world == 1 else f"sharded x{world} (P2P exchange)",
                "apply_ms_per_step": 1e3 * t_apply / args.steps,
                "apply_high_ms_per_step": 1e3 * t_high / args.steps,
                "apply_low_ms_per_step": 1e3 * t_low / args.steps,
                "exchange_ms_per_step": 1e3 * t_exch / args.steps,
                "other_ms_per_step": 1e3 * t_other / args.steps,
                "apply_gbs_high": bytes_per_launch * n_high / t_high / 1e9 if t_high else None,
                "apply_gbs_low": bytes_per_launch * n_low / t_low / 1e9 if t_low else None,
                "apply_tflops": flops / t_apply / 1e12 if t_apply else None,
                "fuse_plan_upload_s": cst["t_fuse_s"] + cst["t_plan_s"] + cst["t_upload_s"],
                "apply_launches_per_step": launches_apply // max(args.steps, 1),
                "block_bits": args.block_bits,
            },
            "roofline": {"bound": "hbm",
                         "kernel": ("apply_rpass (register-blocked pass: all gates of a pass per HBM read+write)"
                                    if cst["n_passes"] else "apply_high+apply_low (one launch per fused gate)"),
                         "achieved": achieved, "peak": peak,
                         "peak_source": peak_src, "unit": "GB/s", "frac": frac,
                         "frac_of_8tbs": achieved / 8000.0 if achieved else None,
                         "algorithmic_bytes_per_launch": bytes_per_launch,
                         "algorithmic_bytes_per_step": bytes_apply // max(args.steps, 1),
                         "traffic": load_traffic("rpass" if cst["n_passes"] else "apply"),
                         # the blocked passes are bound by HBM and the FP32 pipe
                         # together: the FMA-pipe share of the same launches
                         # (fp32 FMAs executed / (148 SMs x 128 FMA/clk x max clock))
                         "fma_pipe": ({"achieved_tfma_s": fma / t_apply / 1e12,
                                       "peak_tfma_s": 148 * 128 * (clk.summary().get("sm_max_mhz") or 1965) * 1e6 / 1e12,
                                       "frac": fma / t_apply / (148 * 128 * (clk.summary().get("sm_max_mhz") or 1965) * 1e6)}
                                      if fma and t_apply else None)},
            "cpu_baseline": cpu,
            "e2e": {"value": e2e_ms / 1e3, "unit": "s", "h2d_bytes_per_step": h2d,
                    "d2h_bytes_per_step": 8 * args.samples},
            "gpu_launches": (n_high + n_low + n_other),
            "fusion_sweep_s": sweep,
            "optimal_fusion": (None if not sweep else
                               {"max_fused": int(min(sweep, key=sweep.get)), "value": min(sweep.values()), "unit": "s"}),
            "clocks": clk.summary(),
        }
        print(json.dumps(out), flush=True)
    sv.sv_circuit_destroy(circ)
    sv.sv_destroy(h)
    if dist is not None:
        dist.barrier()
        dist.destroy_process_group()


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
