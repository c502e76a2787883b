"""Summarise an ncu --metrics gpu__time_duration.sum,dram__bytes_* --csv launch list."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr, data = None, []
for r in rows:
    if r and r[0] == "ID":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        data.append(dict(zip(hdr, r)))
per = collections.OrderedDict()
for d in data:
    key = (d["ID"], d["Kernel Name"].split("(")[0].replace("void ", "")[:48])
    per.setdefault(key, {})[d["Metric Name"]] = float(d["Metric Value"].replace(",", ""))
tot = sum(v.get("gpu__time_duration.sum", 0) for v in per.values())
agg = collections.OrderedDict()
for (i, k), v in per.items():
    a = agg.setdefault(k, [0, 0.0, 0.0])
    a[0] += 1
    a[1] += v.get("gpu__time_duration.sum", 0)
    a[2] += v.get("dram__bytes_read.sum", 0) + v.get("dram__bytes_write.sum", 0)
print(f"total {tot/1e6:.3f} ms over {len(per)} launches")
for k, (n, t, b) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"{k:48s} n={n:3d} {t/1e6:9.3f} ms {100*t/tot:5.1f}%  dram {b/1e9:8.3f} GB {b/max(t,1):8.1f} GB/s")
if len(sys.argv) > 2:
    for (i, k), v in per.items():
        t = v.get("gpu__time_duration.sum", 0)
        if t > float(sys.argv[2]) * 1e6:
            b = v.get("dram__bytes_read.sum", 0) + v.get("dram__bytes_write.sum", 0)
            print(f"  #{i:>4} {k:48s} {t/1e6:9.3f} ms dram {b/1e9:7.3f} GB")
