#!/usr/bin/env python
"""Summarise ncu outputs into profiles/ (run here, on the CPU box).

    python tools/ncu_summary.py launches <launches.csv> <out.md>
    python tools/ncu_summary.py full <prof.ncu-rep> <out.md> [--traffic profiles/kernel_traffic.json] [--key NAME]
    (--key stores the capture's counters under NAME instead of the kernel's
    short name, e.g. k_mpi_fifo_deep for the configs[4] launch)

`launches`: per-kernel launch counts, summed/avg device time and share of the
step (ncu --metrics gpu__time_duration.sum, cold-cache & serialised: shares,
not absolutes).  `full`: per launch the counters that justify the roofline
(dram bytes, throughputs, occupancy, issue efficiency, top stall reasons).
"""
import collections
import csv
import io
import json
import subprocess
import sys

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram read"),
    ("dram__bytes_write.sum", "dram write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram % of peak"),
    ("lts__t_bytes.sum", "L2 bytes"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM % of peak"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__shared_mem_per_block_dynamic", "dyn smem/block"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("launch__occupancy_limit_shared_mem", "occ limit smem"),
    ("launch__occupancy_limit_registers", "occ limit regs"),
]
STALLS = "smsp__average_warps_issue_stalled_"


def launches(path, out):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    mi = h.index("Metric Name") if "Metric Name" in h else None
    agg = collections.OrderedDict()
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        if mi is not None and r[mi] != "gpu__time_duration.sum":
            continue
        name = r[ki].split("(")[0]
        v = float(r[vi].replace(",", ""))
        unit = r[ui]
        v = v * {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(unit, 1e-3)
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += v
    tot = sum(a[1] for a in agg.values())
    lines = ["| kernel | launches | total us | avg us | share |", "|---|---:|---:|---:|---:|"]
    for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        lines.append("| `%s` | %d | %.1f | %.2f | %.1f%% |" % (k[:90], n, t, t / n, 100 * t / tot))
    open(out, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines[:25]))


def full(path, out, traffic=None, key=None):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, units = rows[0], rows[1]
    lines = []
    tr = {}
    for r in rows[2:]:
        name = r[h.index("Kernel Name")]
        short = name.split("(")[0].replace("void ", "").split("<")[0].replace("mm::", "")
        lines.append("### `%s`\n" % name[:160])
        lines.append("| metric | value |\n|---|---:|")
        vals = {}
        for m, label in METRICS:
            if m in h:
                v = r[h.index(m)]
                vals[m] = v
                lines.append("| %s (`%s`) | %s %s |" % (label, m, v, units[h.index(m)]))
        st = []
        for i, c in enumerate(h):
            if c.startswith(STALLS):
                try:
                    st.append((c.replace("_per_issue_active.ratio", ""), float(r[i].replace(",", ""))))
                except ValueError:
                    pass
        st.sort(key=lambda x: -x[1])
        for c, v in st[:6]:
            lines.append("| stall `%s` (warps per issue) | %.2f |" % (c[len(STALLS):], v))
        lines.append("")

        def num(m):
            v = vals.get(m, "0").replace(",", "")
            u = units[h.index(m)] if m in h else ""
            x = float(v or 0)
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
            return x * scale
        b = num("dram__bytes_read.sum") + num("dram__bytes_write.sum")
        d = tr.setdefault(short, {"launches": 0, "dram_bytes": 0.0, "inst": 0.0, "issue": 0.0})
        d["launches"] += 1
        d["dram_bytes"] += b
        d["inst"] += num("smsp__inst_executed.sum")
        d["issue"] += num("smsp__issue_active.avg.pct_of_peak_sustained_active")
    open(out, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines[:60]))
    if traffic:
        old = json.load(open(traffic)) if __import__("os").path.exists(traffic) else {}
        for k, d in tr.items():
            n = d["launches"]
            old[key or k] = {"dram_bytes_per_launch": d["dram_bytes"] / n, "warp_inst_per_launch": d["inst"] / n,
                      "issue_active_pct": d["issue"] / n, "source": path.split("/")[-1]}
        json.dump(old, open(traffic, "w"), indent=1)


if __name__ == "__main__":
    mode = sys.argv[1]
    if mode == "launches":
        launches(sys.argv[2], sys.argv[3])
    else:
        tr = sys.argv[sys.argv.index("--traffic") + 1] if "--traffic" in sys.argv else None
        key = sys.argv[sys.argv.index("--key") + 1] if "--key" in sys.argv else None
        full(sys.argv[2], sys.argv[3], tr, key)
