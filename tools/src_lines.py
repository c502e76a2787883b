"""Aggregate an ncu `--page source --print-source cuda,sass --csv` dump per CUDA
source line, per kernel (functions whose name contains FILTER).
usage: python tools/src_lines.py dump.csv [FILTER] [top]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
filt = sys.argv[2] if len(sys.argv) > 2 else ""
top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
agg, src = {}, {}
fname = func = None
line = None
hdr = None
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split('/')[-1]
        continue
    if r[0] == "Function Name":
        func = r[1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < 8 or filt not in (func or ""):
        continue
    if r[0]:
        line = (fname, int(r[0]))
        src[line] = r[1].strip()[:80]
    if not r[2]:
        continue

    def f(i):
        try:
            return float(r[i].replace(',', ''))
        except ValueError:
            return 0.0
    a = agg.setdefault(line, [0, 0, 0])
    a[0] += f(4)
    a[1] += f(7)
    a[2] += f(8)
tot = [sum(v[i] for v in agg.values()) or 1 for i in range(3)]
print(f"total samples {tot[0]:.0f} inst {tot[1]:.3g}")
for k, v in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    print(f"{k[0][:20]:20s}:{k[1]:4d} samp {v[0] / tot[0] * 100:5.1f}% inst {v[1] / tot[1] * 100:5.1f}% "
          f"thr/inst {v[2] / max(v[1], 1):5.1f} | {src.get(k, '')}")
