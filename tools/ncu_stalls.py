#!/usr/bin/env python
"""Per-source-line stall breakdown from `ncu -i rep --page source --csv
--print-source cuda,sass` output: the top lines by stall samples, each with
its file, instruction share and leading stall reasons.

    python tools/ncu_stalls.py src.csv [top]
"""
import collections
import csv
import os
import sys

rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
fname, hdr = "?", None
lines = collections.defaultdict(lambda: collections.Counter())
text = {}
for r in rows:
    if r and r[0] in ("File Name", "File Path"):
        fname = os.path.basename(r[1])
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if not hdr or not r or not r[0].isdigit() or r[2] != "-":
        continue
    key = (fname, int(r[0]))
    text[key] = r[1].strip()[:70]
    for i, h in enumerate(hdr):
        if i >= len(r):
            break
        if h in ("Warp Stall Sampling (All Samples)", "Instructions Executed") or (h.startswith("stall_") and "Not Issued" not in h):
            try:
                lines[key][h] += int(r[i])
            except ValueError:
                pass
ts = sum(c["Warp Stall Sampling (All Samples)"] for c in lines.values())
ti = sum(c["Instructions Executed"] for c in lines.values())
print("stall samples %d, warp inst %d" % (ts, ti))
for key, c in sorted(lines.items(), key=lambda kv: -kv[1]["Warp Stall Sampling (All Samples)"])[:top]:
    st = sorted(((v, h[6:]) for h, v in c.items() if h.startswith("stall_") and v), reverse=True)[:3]
    print("%-18s %5d  samples %5.2f%%  inst %5.2f%%  %-40s %s" % (
        key[0][:18], key[1], 100.0 * c["Warp Stall Sampling (All Samples)"] / ts, 100.0 * c["Instructions Executed"] / ti,
        " ".join("%s:%d" % (h, v) for v, h in st), text[key]))
