#!/usr/bin/env python
"""Per-level ncu DRAM traffic of one timed step (bench.py roofline.traffic).

    python tools/level_traffic.py <out.json> <level>=<ncu.csv> [<level>=<ncu.csv> ...]

Each CSV comes from one ncu run of one bench level with one timed step:
    ncu --nvtx --nvtx-include "mm_timed:<level>/mm_region]" \
        --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
        --clock-control none --csv --log-file <ncu.csv> \
        python bench.py --levels <level> --steps 1 --warmup 3 --no-cpu-baseline --nvtx
so it holds exactly the launches inside the engine's CUDA-event region
(NVTX "mm_region", mm_engine.cu Timer) of that step.  The summary keeps the
summed DRAM bytes, the launch count and the per-kernel split; the output
file is merged (other levels' entries are kept).
"""
import collections
import csv
import json
import os
import sys


def parse(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, vi, ui, mi, ii = (h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit"),
                          h.index("Metric Name"), h.index("ID"))
    launches = collections.OrderedDict()
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        d = launches.setdefault(r[ii], {"name": r[ki].split("(")[0].replace("void ", "").split("<")[0]})
        v = float(r[vi].replace(",", ""))
        unit = r[ui].lower()
        if r[mi].startswith("dram__bytes"):
            v *= {"byte": 1, "kbyte": 1e3, "mbyte": 1e6, "gbyte": 1e9}.get(unit, 1)
            d["dram"] = d.get("dram", 0.0) + v
        elif r[mi] == "gpu__time_duration.sum":
            v *= {"nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3}.get(unit, 1e-3)
            d["us"] = v
    return list(launches.values())


def main():
    out = sys.argv[1]
    doc = json.load(open(out)) if os.path.exists(out) else {}
    for arg in sys.argv[2:]:
        level, path = arg.split("=", 1)
        ls = parse(path)
        per = collections.OrderedDict()
        for d in ls:
            k = per.setdefault(d["name"], {"launches": 0, "dram_bytes": 0.0, "us": 0.0})
            k["launches"] += 1
            k["dram_bytes"] += d.get("dram", 0.0)
            k["us"] += d.get("us", 0.0)
        doc[level] = {
            "region_dram_bytes_per_step": sum(d.get("dram", 0.0) for d in ls),
            "region_launches_per_step": len(ls),
            "region_kernels": per,
            "region_us_serialised": sum(d.get("us", 0.0) for d in ls),
            "source": os.path.basename(path) + " (ncu, one step, NVTX mm_region, cold-cache serialised launches)",
        }
        print("%-16s %3d launches  %.1f MB dram  %s" % (level, len(ls), doc[level]["region_dram_bytes_per_step"] / 1e6,
                                                      ", ".join("%s x%d" % (k, v["launches"]) for k, v in per.items())))
    json.dump(doc, open(out, "w"), indent=1)


if __name__ == "__main__":
    main()
