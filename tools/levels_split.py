"""Per-level kernel times from an ncu launch list of one hierarchy step
(levels split at each k_span_coords launch, the first kernel of a level).
Usage: python tools/levels_split.py launches.csv [LEVEL ...]"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr, per = None, collections.OrderedDict()
for r in rows:
    if r and r[0] == "ID":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        e = per.setdefault(d["ID"], {"name": d["Kernel Name"].split("(")[0].replace("void ", ""),
                                     "grid": d["Grid Size"], "block": d["Block Size"]})
        e[d["Metric Name"]] = float(d["Metric Value"].replace(",", ""))
show = {int(a) for a in sys.argv[2:]}
lvl, acc, cnt = -1, collections.defaultdict(float), collections.Counter()
for v in per.values():
    if v["name"].startswith("k_span_coords"):
        lvl += 1
    t = v.get("gpu__time_duration.sum", 0.0)
    acc[lvl] += t
    cnt[lvl] += 1
    if lvl in show:
        b = v.get("dram__bytes_read.sum", 0.0) + v.get("dram__bytes_write.sum", 0.0)
        print(f"L{lvl} {v['name'][:46]:46s} grid {v['grid']:>14s} {t/1e3:9.1f} us  {b/1e6:9.1f} MB")
for l in sorted(acc):
    print(f"level {l}: {acc[l]/1e3:9.1f} us over {cnt[l]} launches")
