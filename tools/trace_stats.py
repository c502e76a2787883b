"""Summarise HEC_TRACE_ROWS dumps (per work block compute / wait cycles)."""
import glob
import sys

import numpy as np

for f in sorted(glob.glob(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/trace_*.bin")):
    a = np.fromfile(f, dtype=np.int64).reshape(-1, 4)
    comp, kind, T = a[:, 0] / 1.965e3, a[:, 2] // 100000, a[:, 3]
    exp_, ins = (a[:, 1] >> 32) / 1.965e3, (a[:, 1] & 0xffffffff) / 1.965e3
    wait = comp - exp_ - ins  # remaining phases (sort + staging)
    print(f, len(a), "compute us: med %.1f p90 %.1f p99 %.1f max %.1f sum %.1f ms" % (
        np.median(comp), np.percentile(comp, 90), np.percentile(comp, 99), comp.max(), comp.sum() / 1e3))
    for nm, x in (("expand", exp_), ("hash", ins), ("sort+stage", wait)):
        print("   %-10s us: med %.1f p90 %.1f sum %.1f ms" % (nm, np.median(x), np.percentile(x, 90), x.sum() / 1e3))
    for k in (0, 1, 2):
        m = kind == k
        if m.any():
            print("   kind", k, "n", m.sum(), "compute med %.1f p99 %.1f max %.1f sum %.1f ms" % (
                np.median(comp[m]), np.percentile(comp[m], 99), comp[m].max(), comp[m].sum() / 1e3),
                "T med", np.median(T[m]), "rows/sub med", np.median(a[m, 2] % 100000))
    idx = np.argsort(-comp)[:6]
    print("   slowest:", [(int(i), round(comp[i], 1), int(a[i, 2]), int(T[i])) for i in idx])
