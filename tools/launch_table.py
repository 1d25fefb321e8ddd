"""Per-launch table from an ncu --metrics csv (gpu__time_duration + dram bytes)."""
import csv, collections, sys
rows = list(csv.reader(open(sys.argv[1])))
last = int(sys.argv[2]) if len(sys.argv) > 2 else 40
hi = [i for i, r in enumerate(rows) if 'Kernel Name' in r][0]
h = rows[hi]; ki = h.index('Kernel Name'); mi = h.index('Metric Name'); vi = h.index('Metric Value'); ui = h.index('Metric Unit'); ii = h.index('ID')
per = collections.OrderedDict()
for r in rows[hi + 1:]:
    if len(r) <= vi: continue
    key = (r[ii], r[ki].split('(')[0][:64])
    v = float(r[vi].replace(',', '')); u = r[ui]
    if r[mi] == 'gpu__time_duration.sum':
        per.setdefault(key, {})['us'] = v * {'nsecond': 1e-3, 'ns': 1e-3, 'usecond': 1, 'us': 1, 'msecond': 1e3, 'ms': 1e3}.get(u, 1e-3)
    else:
        per.setdefault(key, {})[r[mi]] = v * {'byte': 1, 'Kbyte': 1e3, 'Mbyte': 1e6, 'Gbyte': 1e9}.get(u, 1)
for (i, k), d in list(per.items())[-last:]:
    print("%-64s %9.1f us  dram %8.1f MB" % (k, d.get('us', 0), (d.get('dram__bytes_read.sum', 0) + d.get('dram__bytes_write.sum', 0)) / 1e6))
