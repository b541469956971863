"""Summarise an ncu --csv launch list (per launch: time, DRAM bytes, L2 sectors, L2 hit
rate), then per kernel name: launches, total ms, share of the listed time, DRAM GB."""
import csv
import sys
from collections import defaultdict

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 5]
h = rows[0]
ki, mi, vi, ii = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
per = defaultdict(dict)
names = {}
for r in rows[1:]:
    try:
        per[r[ii]][r[mi]] = float(r[vi].replace(",", ""))
    except ValueError:
        continue
    names[r[ii]] = r[ki].split("(")[0].replace("void ", "")
agg = defaultdict(lambda: [0, 0.0, 0.0, 0.0])
total = 0.0
for i in sorted(per, key=int):
    m = per[i]
    t = m.get("gpu__time_duration.sum", 0)
    rd, wr = m.get("dram__bytes_read.sum", 0), m.get("dram__bytes_write.sum", 0)
    l2 = m.get("lts__t_sectors_srcunit_tex_op_read.sum", 0)
    hit = m.get("lts__t_sector_hit_rate.pct", 0)
    gbs = (rd + wr) / t if t else 0
    print(f"{i:>4} {names[i][:48]:48s} {t/1e6:8.3f} ms  rd {rd/1e9:7.3f} GB  wr {wr/1e9:7.3f} GB  {gbs:7.1f} GB/s"
          f"  L2rd {l2/1e6:9.1f} M sect  L2hit {hit:5.1f}%")
    a = agg[names[i]]
    a[0] += 1
    a[1] += t / 1e6
    a[2] += (rd + wr) / 1e9
    a[3] += l2 / 1e6
    total += t / 1e6
print("\nper kernel: launches, total ms, share of listed time, DRAM GB, L2 read M sectors")
for n, (c, t, gb, l2) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"  {n[:60]:60s} {c:4d} {t:9.3f} ms {100 * t / total if total else 0:5.1f}%  {gb:8.3f} GB  {l2:10.1f}")
