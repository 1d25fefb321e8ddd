#!/usr/bin/env python
"""Per-CUDA-source-line instruction and stall-sample totals from an ncu report.

    ncu -i rep.ncu-rep --page source --csv --print-source cuda,sass -k regex:NAME -c 1 > src.csv
    python tools/ncu_lines.py src.csv [top]
"""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
hdr = next(r for r in rows if r and r[0] == "Line No")
ii = hdr.index("Instructions Executed"); si = hdr.index("Warp Stall Sampling (All Samples)")
out = []
for r in rows:
    if len(r) > ii and r[0] not in ("", "Line No") and r[0].isdigit():
        try:
            out.append((int(r[ii]), int(r[si]), int(r[0]), r[1][:90]))
        except ValueError:
            pass
ti = sum(o[0] for o in out); ts = sum(o[1] for o in out)
print("total warp inst %d, stall samples %d" % (ti, ts))
for inst, smp, ln, src in sorted(out, key=lambda o: -o[1])[:top]:
    print("%5d  inst %6.2f%%  samples %6.2f%%  %s" % (ln, 100.0 * inst / ti, 100.0 * smp / ts, src))
