import ctypes, sys
sys.path.insert(0, '/root/repo')
import numpy as np, torch
import graphgen as gg
import paper_conf_ipps_gilbertabmr21_b200 as P
L = P.load()
g = gg.rmat(14, 16)
ctx = P.Context()
dg = P.DeviceGraph.from_host(g); gc = dg.c()
M, nc = P.hec_find_mapping(ctx, dg, 0x5EED, 0)
full = P.build_coarse_graph(ctx, dg, M, nc).graph
print('stats', ctx.stats(), 'n_c', nc)
rp, col, wgt, vw = full.to_host()
for parts in (1, 2, 3):
    bounds = (ctypes.c_int64 * (parts + 1))()
    L.hec_balance_rows(ctx.h, ctypes.byref(gc), M.data_ptr(), nc, parts, bounds)
    b = list(bounds); off = 0
    for r in range(parts):
        a0, a1 = b[r], b[r + 1]; rows = a1 - a0
        k = ctypes.c_int64()
        counts = torch.empty(max(rows, 1), dtype=torch.int64, device='cuda')
        assert L.hec_build_rows_count(ctx.h, ctypes.byref(gc), M.data_ptr(), nc, a0, a1, counts.data_ptr(), ctypes.byref(k)) == 0
        k = k.value
        orp = torch.empty(rows + 1, dtype=torch.int64, device='cuda'); ocol = torch.empty(max(k,1), dtype=torch.int32, device='cuda')
        owgt = torch.empty(max(k,1), dtype=torch.int32, device='cuda'); ovw = torch.empty(max(rows,1), dtype=torch.int32, device='cuda')
        L.hec_build_rows_write(ctx.h, off, orp.data_ptr(), ocol.data_ptr(), owgt.data_ptr(), ovw.data_ptr())
        oc = ocol[:k].cpu().numpy(); ec = col[rp[a0]:rp[a1]]
        bad = np.nonzero(oc != ec)[0]
        print(parts, r, (a0, a1), 'k', k, 'bad', len(bad), 'stats', ctx.stats())
        if len(bad):
            i = bad[0] + rp[a0]
            row = np.searchsorted(rp, i, side='right') - 1
            print('   first bad entry', i, 'row', row, 'U?', 'exp', col[rp[row]:rp[row+1]][:8], 'got', oc[rp[row]-rp[a0]:rp[row+1]-rp[a0]][:8])
        off += k
print('---- targeted')
def run(a0, a1):
    rows = a1 - a0; k = ctypes.c_int64()
    assert L.hec_build_rows_count(ctx.h, ctypes.byref(gc), M.data_ptr(), nc, a0, a1, None, ctypes.byref(k)) == 0
    k = k.value
    orp = torch.empty(rows + 1, dtype=torch.int64, device='cuda'); ocol = torch.empty(max(k,1), dtype=torch.int32, device='cuda')
    owgt = torch.empty(max(k,1), dtype=torch.int32, device='cuda'); ovw = torch.empty(max(rows,1), dtype=torch.int32, device='cuda')
    L.hec_build_rows_write(ctx.h, 0, orp.data_ptr(), ocol.data_ptr(), owgt.data_ptr(), ovw.data_ptr())
    return orp.cpu().numpy(), ocol[:k].cpu().numpy(), owgt[:k].cpu().numpy()
U = np.diff(rp)
for (a0, a1) in [(132, 917), (132, 133), (131, 133), (1, 1574), (0, 133)]:
    orp, oc, ow = run(a0, a1)
    ec = col[rp[a0]:rp[a1]]; ew = wgt[rp[a0]:rp[a1]]
    bad = np.nonzero((oc != ec) | (ow != ew))[0]
    print((a0, a1), 'bad', len(bad), 'rowlens', np.diff(orp)[:3], U[a0:a0+3])
    if len(bad):
        i = bad[0]; row = np.searchsorted(orp - orp[0], i, side='right') - 1 + a0
        print('   row', row, 'exp c', ec[:6], 'w', ew[:6], '\n   got c', oc[:6], 'w', ow[:6])
