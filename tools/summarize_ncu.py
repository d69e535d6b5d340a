"""Summarise ncu output into profiles/ (committed evidence).

usage: python tools/summarize_ncu.py <launches.csv> <full_raw.csv>[,<full_raw2.csv>...] <round_tag>

launches.csv : ncu --metrics gpu__time_duration.sum --csv launch list of a
               bench.py run (cold-cache, serialised -> compare shares)
full_raw.csv : ncu -i <full .ncu-rep> --page raw --csv of the apply kernel(s)
               (comma-separated list: the first is the headline kernel)
Writes profiles/ncu_summary.json (read by bench.py for roofline.traffic)
and profiles/<round_tag>_ncu_summary.md.
"""
import csv
import json
import os
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def kclass(name: str) -> str:
    if "apply_rpass" in name or "apply_pass" in name or name.startswith("rpj"):
        return "rpass"
    if "apply_tci" in name or "apply_tc" in name:
        return "apply_tc"
    if "apply_high" in name or "apply_low" in name or "apply_small" in name:
        return "apply"
    if "exchange" in name:
        return "exchange"
    if "bin_weights" in name or "scan" in name or "sample" in name or "shard_offsets" in name:
        return "sample"
    if "reset" in name:
        return "reset"
    return "other"


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = None
    out = []
    for r in rows:
        if "Kernel Name" in r and "Metric Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            if d.get("Metric Name") == "gpu__time_duration.sum":
                v = float(d["Metric Value"].replace(",", ""))
                unit = d.get("Metric Unit", "")
                scale = {"ns": 1e-9, "usecond": 1e-6, "us": 1e-6, "msecond": 1e-3, "ms": 1e-3, "nsecond": 1e-9}.get(unit, 1e-9)
                out.append((d["Kernel Name"], v * scale))
    return out


def full_raw(path):
    rows = list(csv.reader(open(path)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        res.append(d)
    return hdr, units, res


def to_bytes(v, unit):
    v = float(str(v).replace(",", ""))
    return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)


KEEP = ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "smsp__inst_executed.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum", "sm__cycles_elapsed.avg.per_second")
TSCALE = {"nsecond": 1e-9, "ns": 1e-9, "usecond": 1e-6, "us": 1e-6, "msecond": 1e-3, "ms": 1e-3, "second": 1.0, "s": 1.0}


def captures(path):
    hdr, units, res = full_raw(path)
    ui = dict(zip(hdr, units))
    out = []
    for d in res:
        rb = to_bytes(d["dram__bytes_read.sum"], ui["dram__bytes_read.sum"])
        wb = to_bytes(d["dram__bytes_write.sum"], ui["dram__bytes_write.sum"])
        dur = float(d["gpu__time_duration.sum"].replace(",", "")) * TSCALE.get(ui["gpu__time_duration.sum"], 1e-9)
        keep = {k: d[k] for k in KEEP if k in d}
        out.append({"kernel": d.get("Kernel Name", "")[:120], "dram_read_bytes": rb, "dram_write_bytes": wb,
                    "traffic_bytes": rb + wb, "duration_s": dur, "dram_GBps": (rb + wb) / dur / 1e9, **keep})
    return out


def main():
    lp, fp, tag = sys.argv[1], sys.argv[2], sys.argv[3]
    L = launches(lp)
    by = defaultdict(lambda: [0, 0.0])
    names = defaultdict(lambda: [0, 0.0])
    for n, t in L:
        c = kclass(n)
        by[c][0] += 1
        by[c][1] += t
        names[n.split("(")[0][:90]][0] += 1
        names[n.split("(")[0][:90]][1] += t
    ours = {c: v for c, v in by.items() if c != "other"}
    tot_ours = sum(v[1] for v in ours.values())
    summary = {"round": tag, "launch_list": os.path.basename(lp), "classes": {}, "traffic_per_launch": {}}
    for c, (cnt, t) in sorted(by.items()):
        summary["classes"][c] = {"launches": cnt, "time_s": t, "share_of_our_kernels": (t / tot_ours) if c != "other" and tot_ours else None}
    caps = [c for one in fp.split(",") for c in captures(one)]
    if caps:
        summary["full_capture"] = caps
        for c in caps:  # a full (read + write) pass: the largest capture of the class
            k = kclass(c["kernel"])
            summary["traffic_per_launch"][k] = max(summary["traffic_per_launch"].get(k, 0), c["traffic_bytes"])
    old = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if os.path.exists(old):  # keep per-class traffic of kernels not captured this time
        for k, v in json.load(open(old)).get("traffic_per_launch", {}).items():
            summary["traffic_per_launch"].setdefault(k, v)
    json.dump(summary, open(old, "w"), indent=1)
    md = [f"# ncu summary ({tag})", "", f"Launch list: `{os.path.basename(lp)}` (ncu --metrics gpu__time_duration.sum "
          "--clock-control none; cold-cache, serialised: compare shares, not absolutes)", "",
          "| class | launches | time (s) | share of our kernels |", "|---|---|---|---|"]
    for c, v in summary["classes"].items():
        sh = v["share_of_our_kernels"]
        md.append(f"| {c} | {v['launches']} | {v['time_s']:.4f} | {'' if sh is None else f'{100 * sh:.1f} %'} |")
    md += ["", "Per kernel:", "", "| kernel | launches | time (s) |", "|---|---|---|"]
    for n, (cnt, t) in sorted(names.items(), key=lambda x: -x[1][1])[:20]:
        md.append(f"| `{n}` | {cnt} | {t:.4f} |")
    if caps:
        md += ["", "Full captures (--set full, one launch each, 30 qubits): the headline kernel first:", ""]
        for c in caps:
            md.append(f"- `{c['kernel']}`: DRAM read {c['dram_read_bytes'] / 1e9:.3f} GB, write "
                      f"{c['dram_write_bytes'] / 1e9:.3f} GB per launch (algorithmic 16 B x 2^30 = 17.180 GB), "
                      f"{c['duration_s'] * 1e3:.3f} ms -> {c['dram_GBps']:.0f} GB/s")
            for k, v in c.items():
                if k not in ("kernel", "dram_read_bytes", "dram_write_bytes", "traffic_bytes", "duration_s", "dram_GBps"):
                    md.append(f"  - {k} = {v}")
    open(os.path.join(ROOT, "profiles", f"{tag}_ncu_summary.md"), "w").write("\n".join(md) + "\n")
    print("\n".join(md))


if __name__ == "__main__":
    main()
