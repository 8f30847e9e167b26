"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv): per kernel name, launches and the
mean / first per-launch times in microseconds.   python tools/launches.py file.csv [...]"""
import csv
import sys
from collections import defaultdict

for fn in sys.argv[1:]:
    lines = [l for l in open(fn) if l.startswith('"')]
    rows = list(csv.reader(lines))
    hdr = rows[0]
    iv, ik = hdr.index("Metric Value"), hdr.index("Kernel Name")
    d = defaultdict(list)
    for r in rows[1:]:
        if len(r) > iv and r[iv] != "Metric Value":
            d[r[ik].split("(")[0][:48]].append(float(r[iv].replace(",", "")) / 1000)
    print(fn)
    for k, v in sorted(d.items(), key=lambda kv: -sum(kv[1])):
        print(f"  {k:50s} {len(v):4d} {sum(v) / len(v):9.1f} us   {[round(x, 1) for x in v[:6]]}")
