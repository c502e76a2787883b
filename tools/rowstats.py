"""Row-volume structure of a level (GPU box): distribution of the member-edge
volume U(a) and of the coarse row length |row a| of G_{l+1}, by power-of-two
class (rows, entries).  usage: python tools/rowstats.py CFG"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import paper_conf_ipps_gilbertabmr21_b200 as P  # noqa: E402

cfg = int(sys.argv[1])
g = gg.config(cfg)
dg = P.DeviceGraph.from_host(g)
ctx = P.Context()
h = P.coarsen_hierarchy(ctx, dg, gg.CONFIGS[cfg]["cutoff"], gg.COARSEN_SEED)
cur = dg
for li, lv in enumerate(h.levels[:2]):
    M = lv.M.long()
    deg = (cur.row_ptr[1:] - cur.row_ptr[:-1])
    n_c = lv.graph.n
    U = torch.zeros(n_c, dtype=torch.int64, device=M.device).index_add_(0, M, deg)
    nxt = lv.graph
    L = (nxt.row_ptr[1:] - nxt.row_ptr[:-1])
    mem = torch.bincount(M, minlength=n_c)
    print(f"level {li}: n={cur.n} nnz={cur.nnz} n_c={n_c} nnz_c={nxt.nnz} maxU={int(U.max())} maxmembers={int(mem.max())}")
    for name, x in (("U", U), ("len", L)):
        x = x.cpu().numpy()
        cls = np.where(x > 0, np.floor(np.log2(np.maximum(x, 1))).astype(int), -1)
        tot = x.sum()
        out = []
        for c in range(-1, cls.max() + 1):
            m = cls == c
            if m.any():
                out.append(f"2^{c}:{m.sum()}r/{x[m].sum() / tot * 100:.1f}%")
        print(f"  {name}: " + " ".join(out))
    # key density by coarse-id sixteenths, weighted by U
    Uc = U.cpu().numpy()
    print("  U per row by id sixteenth:", [int(a.sum() // max(len(a), 1)) for a in np.array_split(Uc, 16)])
    cur = nxt
