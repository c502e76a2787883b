"""In-bucket rank cost of the hash-rank items (GPU box, analysis only): for the
rows of G_{l+1} (sorted distinct keys), the mean bucket occupancy seen by a key
(sum s^2 / D) under the linear key-range buckets k_hrank uses, and under a
CDF-balanced mapping at several table resolutions.  usage: rankcost.py CFG"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import graphgen as gg  # noqa: E402
import paper_conf_ipps_gilbertabmr21_b200 as P  # noqa: E402

cfg = int(sys.argv[1])
g = gg.config(cfg)
dg = P.DeviceGraph.from_host(g)
ctx = P.Context()
h = P.coarsen_hierarchy(ctx, dg, gg.CONFIGS[cfg]["cutoff"], gg.COARSEN_SEED)
lv = h.levels[0]
M = lv.M.long()
deg = dg.row_ptr[1:] - dg.row_ptr[:-1]
G = lv.graph
n_c = G.n
U = torch.zeros(n_c, dtype=torch.int64, device=M.device).index_add_(0, M, deg)
rp = G.row_ptr
rows = torch.repeat_interleave(torch.arange(n_c, device=M.device, dtype=torch.int32), rp[1:] - rp[:-1])
keep = (rows % 16) == 3  # a 1/16 sample of the rows
rows = rows[keep].long()
col = G.col[keep].long()
del keep
cum = torch.cumsum(U, 0)
tot = float(cum[-1])
print("volume share of the lowest ids:", {k: round(float(cum[k - 1]) / tot, 4) for k in (10, 100, 1000, 10000, 100000)})
Ur = U[rows]
# items: whole rows with 124 < U <= 4096; bins of the rows above (equal key width, ~1024 entries)
whole = (Ur > 124) & (Ur <= 4096)
nb = torch.clamp((Ur + 1023) // 1024, max=8192)
binid = torch.where(whole, torch.zeros_like(col), (col * nb) // n_c)
lo = torch.where(whole, torch.zeros_like(col), (binid * n_c + nb - 1) // nb)
hi = torch.where(whole, torch.full_like(col, n_c), ((binid + 1) * n_c + nb - 1) // nb)
item_n = torch.where(whole, Ur, Ur // nb)  # entries of the item (approx for bins)
NB = 2 ** torch.ceil(torch.log2(item_n.clamp(min=2).double())).long()
sel = Ur > 124
for name, F in [("linear", None), ("cdf1024", 1024), ("cdf16384", 16384), ("cdf_exact", 0)]:
    if F is None:
        x = (col - lo).double() / (hi - lo).double()
    else:
        if F == 0:
            tab = torch.cat([torch.zeros(1, device=M.device, dtype=torch.float64), cum.double()])
            def f(b):
                return tab[b]
        else:
            idx = (torch.arange(F + 1, device=M.device) * n_c) // F
            tab = torch.cat([torch.zeros(1, device=M.device, dtype=torch.float64), cum.double()])[idx]
            def f(b, idx=idx, tab=tab, F=F):
                x = b.double() * F / n_c
                k = x.floor().long().clamp(max=F - 1)
                return tab[k] + (tab[k + 1] - tab[k]) * (x - k)
        x = (f(col) - f(lo)) / (f(hi) - f(lo)).clamp(min=1e-9)
    bk = (x * NB).floor().long().clamp(max=NB - 1)
    key = ((rows * 9000 + binid) * 16384 + bk)[sel]
    _, inv, cnt = torch.unique(key, return_inverse=True, return_counts=True)
    s = cnt[inv].double()
    print(f"{name:10s} mean bucket size seen by a key: {float(s.mean()):.2f}  (whole rows {float(s[whole[sel]].mean()):.2f}, bins {float(s[~whole[sel]].mean()):.2f})")
