"""Summarise an ncu --page source --csv (SASS) export: instruction mix and
warp-stall samples by opcode, by stall reason, and the hottest lines with
their dominant stall reasons.

usage: ncu -i rep --page source --csv --print-source sass [--launch-skip i --launch-count 1] > x.csv
       python tools/ncu_source.py x.csv [n_lines]"""
import collections
import csv
import re
import sys

rows = list(csv.reader(open(sys.argv[1])))
ntop = int(sys.argv[2]) if len(sys.argv) > 2 else 30
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
stalls = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
seen = set()
tot_i = tot_s = 0
by_op, s_op = collections.Counter(), collections.Counter()
by_reason = collections.Counter()
lines = []
for r in rows[2:]:
    if len(r) < len(hdr) or not r[ix["Instructions Executed"]].isdigit():
        continue
    key = r[ix["Address"]]
    if key in seen:  # the export repeats every line once per section
        continue
    seen.add(key)
    src = r[ix["Source"]].strip()
    ie = int(r[ix["Instructions Executed"]])
    s = int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    op = re.sub(r"^@!?U?P\w+\s+", "", src).split(" ")[0].split(".")[0]
    by_op[op] += ie
    s_op[op] += s
    tot_i += ie
    tot_s += s
    rs = {h: int(r[ix[h]] or 0) for h in stalls}
    for h, v in rs.items():
        by_reason[h] += v
    lines.append((s, ie, src, rs))
print(f"instructions {tot_i}  stall samples {tot_s}")
print("by reason:", ", ".join(f"{h[6:]} {v / tot_s * 100:.1f}%" for h, v in by_reason.most_common(12)))
for op, c in by_op.most_common(25):
    print(f"{op:10s} inst {c / tot_i * 100:5.1f}%  samples {s_op[op] / tot_s * 100:5.1f}%")
print("hottest lines (samples, executions, top reasons):")
for s, ie, src, rs in sorted(lines, key=lambda x: -x[0])[:ntop]:
    top = sorted(rs.items(), key=lambda kv: -kv[1])[:3]
    print(f"{s:7d} {ie:10d} {src[:70]:70s} " + " ".join(f"{h[6:]}={v}" for h, v in top if v))
