"""Summarise an ncu --csv launch list (gpu__time_duration + dram bytes per launch)."""
import csv
import sys
from collections import defaultdict

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 5]
h = rows[0]
ki, mi, vi, ii = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
per = defaultdict(dict)
names = {}
for r in rows[1:]:
    per[r[ii]][r[mi]] = float(r[vi].replace(",", ""))
    names[r[ii]] = r[ki].split("(")[0]
for i in sorted(per, key=int):
    m = per[i]
    t = m.get("gpu__time_duration.sum", 0)
    rd, wr = m.get("dram__bytes_read.sum", 0), m.get("dram__bytes_write.sum", 0)
    gbs = (rd + wr) / t if t else 0
    print(f"{i:>4} {names[i][:40]:40s} {t/1e6:8.3f} ms  rd {rd/1e9:7.3f} GB  wr {wr/1e9:7.3f} GB  {gbs:7.1f} GB/s")
