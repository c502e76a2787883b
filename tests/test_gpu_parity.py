"""Parity of the CUDA path (through the C-ABI) against the CPU oracle.

Bar: integer work, so everything is bit-exact — H, root
flags, round counts, M, n_c, and every coarse CSR (row_ptr, col, wgt, vwgt).
Small/medium sizes compare element by element with the oracle run on the same
seeded inputs; the full-size configs C3/C4 compare per-level digests against
tests/golden/oracle_digests.json (written by tests/golden/make_digests.py,
which calls only graphgen/ and oracle/)."""
import itertools
import json
import os

import numpy as np
import pytest
import torch

import graphgen as gg
import oracle as o

pytestmark = pytest.mark.gpu

SEED = 0x5EED


@pytest.fixture(scope="module")
def P():
    import subprocess
    subprocess.run(["make", "-C", os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "-s", "hec"],
                   check=True)
    import paper_conf_ipps_gilbertabmr21_b200 as P
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    return P


@pytest.fixture(scope="module")
def ctx(P):
    c = P.Context()
    yield c
    c.close()


def dev(P, g):
    return P.DeviceGraph.from_host(g)


def host_csr(dg):
    rp, col, wgt, vw = dg.to_host()
    return rp, col, wgt, vw


def assert_csr_equal(dg, oc):
    rp, col, wgt, vw = host_csr(dg)
    assert np.array_equal(rp, oc.row_ptr), "row_ptr differs"
    assert np.array_equal(col, oc.col), "col differs"
    assert np.array_equal(wgt, oc.wgt), "wgt differs"
    assert np.array_equal(vw, oc.vwgt), "vwgt differs"


def random_graph(n, rng, p=0.3, wmax=3, isolated=0):
    edges = [(u, v, int(rng.integers(1, wmax + 1)))
             for u in range(n - isolated) for v in range(u + 1, n - isolated) if rng.random() < p]
    return gg.from_edges(n, edges)


def prio_tensor(pr):
    return torch.from_numpy(pr.view(np.int64).copy()).cuda()


# ------------------------------------------------------------------ a1
@pytest.mark.parametrize("path", ["default", "spans"])
@pytest.mark.parametrize("which", ["grid", "mesh27_small", "rmat12", "rmat16", "random"])
def test_heavy_parity(P, ctx, which, path, monkeypatch):
    """default: graphs of <= 2^18 entries take the warp-per-row kernel, larger
    ones the segmented span kernel; spans: the span kernel for all (test hook)."""
    if path == "spans":
        monkeypatch.setenv("HEC_HEAVY_SEG", "1")
    rng = np.random.default_rng(11)
    if which == "grid":
        gs = [gg.grid2d(64, 64), gg.grid2d(1, 7), gg.grid2d(3, 1000)]
    elif which == "mesh27_small":
        gs = [gg.mesh27(20, 21, 22)]
    elif which == "rmat12":
        gs = [gg.rmat(12, 16)]
    elif which == "rmat16":
        gs = [gg.rmat(16, 16)]
    else:
        gs = [random_graph(int(rng.integers(1, 60)), rng, p=0.3, wmax=3, isolated=int(rng.integers(0, 4)))
              for _ in range(30)]
    for g in gs:
        H = P.hec_debug_heavy(ctx, dev(P, g)).cpu().numpy()
        assert np.array_equal(H, o.heavy(g))


def test_heavy_hub_rows_span_tiles(P, ctx):
    """Rows far longer than a tile (4096 items), ties everywhere, weights chosen so
    the maximum sits at the row's end / start / middle."""
    n = 30000
    edges = [(0, v, 1) for v in range(1, n)]                       # hub row 0
    edges += [(1, v, 1 + (v % 7 == 0)) for v in range(2, 20000)]  # max repeated: first wins
    edges += [(2, n - 1, 9)]                                      # heaviest at row end of 2
    g = gg.from_edges(n, edges)
    H = P.hec_debug_heavy(ctx, dev(P, g)).cpu().numpy()
    assert np.array_equal(H, o.heavy(g))


def scattered_isolated_graph(n, rng, deg=6, iso_frac=0.1):
    """Random graph whose isolated (empty) rows sit at the start, in the middle
    and at the end of the vertex range, next to rows far longer than a span."""
    iso = set(rng.choice(n, max(1, int(iso_frac * n)), replace=False).tolist()) | {0, 1, n // 2, n - 1}
    live = np.array(sorted(set(range(n)) - iso))
    edges = {}
    for _ in range(deg * n // 2):
        u, v = rng.choice(live, 2)
        if u != v:
            edges[(min(u, v), max(u, v))] = int(rng.integers(1, 6))
    hub = int(live[len(live) // 3])
    for v in live[::2]:
        if v != hub:
            edges[(min(hub, v), max(hub, v))] = int(rng.integers(1, 6))
    return gg.from_edges(n, [(u, v, w) for (u, v), w in edges.items()])


@pytest.mark.parametrize("path", ["default", "spans", "tiles"])
@pytest.mark.parametrize("phase", [0, 1, 2, 3, "mixed"])
def test_heavy_isolated_and_unaligned(P, ctx, path, phase, monkeypatch):
    """a1 with empty rows anywhere and col/wgt views that start 0-3 int32 past a
    16-byte boundary (default: warp-per-row kernel for the small graphs; spans:
    the segmented span kernel, scalar loads when the phases differ; tiles: the
    merge-path tile kernel; test hooks)."""
    if path == "tiles":
        monkeypatch.setenv("HEC_HEAVY_TILES", "1")
    if path == "spans":
        monkeypatch.setenv("HEC_HEAVY_SEG", "1")
    rng = np.random.default_rng(31 if phase == "mixed" else 31 + phase)
    for n in (6, 700, 20000):
        g = scattered_isolated_graph(n, rng)
        pc, pw = (1, 3) if phase == "mixed" else (phase, phase)
        cbuf = torch.zeros(g.nnz + 8, dtype=torch.int32, device="cuda")
        wbuf = torch.zeros(g.nnz + 8, dtype=torch.int32, device="cuda")
        col = cbuf[pc:pc + g.nnz]
        wgt = wbuf[pw:pw + g.nnz]
        col.copy_(torch.from_numpy(g.col))
        wgt.copy_(torch.from_numpy(g.wgt))
        dg = P.DeviceGraph(torch.from_numpy(g.row_ptr).cuda(), col, wgt, None)
        H = P.hec_debug_heavy(ctx, dg).cpu().numpy()
        assert np.array_equal(H, o.heavy(g))



# ------------------------------------------------------------------ a3
def test_roots_and_rounds_c1(P, ctx, golden_dir):
    ka = json.load(open(os.path.join(golden_dir, "survey_known_answers.json")))["C1"]
    g = gg.config(1)
    H = o.hierarchy(g, 50, SEED, keep_roots=True)
    cur = g
    for level, lv in enumerate(H.levels):
        root, rounds = P.hec_debug_roots(ctx, dev(P, cur), seed=SEED, level=level)
        assert np.array_equal(root.cpu().numpy(), lv.root)
        assert 1 <= rounds <= ka["rounds"][level]  # see test_hierarchy_c1
        cur = lv.graph


# ------------------------------------------------------------- a1-a5 mapping
def test_mapping_hand_examples(P, ctx, golden_dir):
    ex = json.load(open(os.path.join(golden_dir, "hand_examples.json")))
    for name in ("G6", "P4w"):
        e = ex[name]
        g = gg.from_edges(e["n"], e["edges"])
        for run in e["runs"]:
            pr = o.prio_from_order(run["order"])
            M, nc = P.hec_find_mapping_prio(ctx, dev(P, g), prio_tensor(pr))
            assert nc == run["n_c"] and M.cpu().numpy().tolist() == run["M"]


def test_mapping_exhaustive_small(P, ctx):
    """All visit orders of small graphs with ties and an isolated vertex."""
    rng = np.random.default_rng(12)
    for t in range(4):
        g = random_graph(6, rng, p=0.5, wmax=2, isolated=1 if t % 2 else 0)
        dg = dev(P, g)
        for order in itertools.permutations(range(6)):
            pr = o.prio_from_order(order)
            M, nc = P.hec_find_mapping_prio(ctx, dg, prio_tensor(pr))
            Mo, nco, _ = o.mapping(g, pr)
            assert nc == nco and np.array_equal(M.cpu().numpy(), Mo)


def test_mapping_adversarial_path(P, ctx):
    """Reverse-priority path: O(n) resolution rounds; must still be exact."""
    n = 20000
    g = gg.from_edges(n, [(i, i + 1, 1) for i in range(n - 1)])
    for order in (range(n), range(n - 1, -1, -1)):
        pr = o.prio_from_order(order)
        M, nc = P.hec_find_mapping_prio(ctx, dev(P, g), prio_tensor(pr))
        Mo, nco, _ = o.mapping(g, pr)
        assert nc == nco and np.array_equal(M.cpu().numpy(), Mo)


def path_csr(n):
    """Path 0-1-...-(n-1), unit weights, as a CSR (numpy; from_edges is too slow at 2M)."""
    deg = np.full(n, 2, np.int64)
    deg[0] = deg[-1] = 1
    rp = np.zeros(n + 1, np.int64)
    rp[1:] = np.cumsum(deg)
    col = np.empty(rp[-1], np.int32)
    mid = rp[1:n - 1]                                 # rows 1 .. n-2: (u-1, u+1)
    col[mid] = np.arange(0, n - 2, dtype=np.int32)
    col[mid + 1] = np.arange(2, n, dtype=np.int32)
    col[0] = 1                                        # row 0: (1)
    col[-1] = n - 2                                   # row n-1: (n-2)
    return gg.Graph(rp, col, np.ones(rp[-1], np.int32), np.ones(n, np.int32))


def test_mapping_long_chain_identity_path(P, ctx):
    """Identity visit order on a 2M-vertex path: one aggregate (SURVEY §8(c) M1
    closed form, n_c = 1) reached through a single H-chain of length n -- the
    inherit step must not walk it per vertex (pointer jumping, Alg 5 l.17-21)."""
    import time
    n = 2_000_000
    g = path_csr(n)
    assert np.array_equal(o.heavy(g)[:5], [1, 0, 1, 2, 3])
    pr = np.arange(n, dtype=np.uint64)
    dg, pt = dev(P, g), prio_tensor(pr)
    P.hec_find_mapping_prio(ctx, dg, pt)  # warm-up
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    M, nc = P.hec_find_mapping_prio(ctx, dg, pt)
    dt = time.perf_counter() - t0
    assert nc == 1 and int(M.max()) == 0 and int(M.min()) == 0
    assert dt < 1.0, f"{dt:.3f} s"


def test_mapping_long_rounds_reversed_path(P, ctx):
    """Reverse visit order on a 2M-vertex path: Alg 3 pairs {2k, 2k+1} (SURVEY
    §8(c) M1 closed form), but the decision chain is n long -- n/2 plain
    resolution rounds.  The residual compression (pointer jumping with
    parity along unary chains) must resolve it in well under a second."""
    import time
    n = 2_000_000
    g = path_csr(n)
    pr = np.arange(n, dtype=np.uint64)[::-1].copy()
    dg, pt = dev(P, g), prio_tensor(pr)
    P.hec_find_mapping_prio(ctx, dg, pt)  # warm-up
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    M, nc = P.hec_find_mapping_prio(ctx, dg, pt)
    dt = time.perf_counter() - t0
    assert nc == n // 2
    assert np.array_equal(M.cpu().numpy(), np.arange(n) // 2)
    assert dt < 1.0, f"{dt:.3f} s"


@pytest.mark.parametrize("shape", ["broom", "caterpillar", "spiders"])
def test_mapping_adversarial_trees(P, ctx, shape):
    """Trees whose H-forest has long chains with side branches, visited in
    adversarial orders (priority = depth from the far end), against the oracle."""
    rng = np.random.default_rng({"broom": 41, "caterpillar": 42, "spiders": 43}[shape])
    edges = []
    if shape == "broom":      # a 30k path with a 2k-leaf fan at one end
        L = 30000
        edges += [(i, i + 1, 1) for i in range(L - 1)]
        edges += [(L - 1, L + j, 1) for j in range(2000)]
        n = L + 2000
    elif shape == "caterpillar":  # a 20k spine, a pendant leaf at every third vertex
        L = 20000
        edges += [(i, i + 1, 2) for i in range(L - 1)]
        leaves = list(range(0, L, 3))
        edges += [(v, L + j, 1) for j, v in enumerate(leaves)]
        n = L + len(leaves)
    else:                     # 40 paths of random length hanging off a hub
        n, nxt = 1, 1
        for _ in range(40):
            ln = int(rng.integers(100, 3000))
            prev = 0
            for _ in range(ln):
                edges.append((prev, nxt, 1))
                prev, nxt = nxt, nxt + 1
        n = nxt
    g = gg.from_edges(n, edges)
    for order in (np.arange(n), np.arange(n)[::-1], rng.permutation(n)):
        pr = o.prio_from_order(order)
        M, nc = P.hec_find_mapping_prio(ctx, dev(P, g), prio_tensor(pr))
        Mo, nco, _ = o.mapping(g, pr)
        assert nc == nco and np.array_equal(M.cpu().numpy(), Mo)


@pytest.mark.parametrize("which", ["c1", "c2", "rmat16", "random"])
def test_mapping_parity_seeded(P, ctx, which):
    rng = np.random.default_rng(13)
    if which == "c1":
        gs = [gg.config(1)]
    elif which == "c2":
        gs = [gg.config(2)]
    elif which == "rmat16":
        gs = [gg.rmat(16, 16)]
    else:
        gs = [random_graph(int(rng.integers(1, 200)), rng, p=0.05, wmax=4, isolated=int(rng.integers(0, 3)))
              for _ in range(20)]
    for g in gs:
        for level in (0, 3):
            M, nc = P.hec_find_mapping(ctx, dev(P, g), SEED, level)
            Mo, nco, _ = o.mapping(g, o.prio(SEED, level, g.n))
            assert nc == nco and np.array_equal(M.cpu().numpy(), Mo)


# ------------------------------------------------------- a7-a10 construction
def test_construct_random_labels(P, ctx):
    """Random M over random weighted graphs (exercises SMALL rows, duplicates, self entries)."""
    rng = np.random.default_rng(14)
    for t in range(25):
        g = random_graph(int(rng.integers(2, 120)), rng, p=0.2, wmax=50)
        g.vwgt = rng.integers(1, 5, g.n).astype(np.int32)
        nc = int(rng.integers(1, g.n + 1))
        M = rng.integers(0, nc, g.n).astype(np.int32)
        M[:nc] = np.arange(nc)
        cg = P.build_coarse_graph(ctx, dev(P, g), torch.from_numpy(M).cuda(), nc)
        assert_csr_equal(cg.graph, o.coarsen(g, M, nc))


@pytest.mark.parametrize("path", ["rbm", "bins", "wide_index", "one_end"])
@pytest.mark.parametrize("nc", [3, 40, 900, 20000, 70000])
def test_construct_size_classes(P, ctx, nc, path, monkeypatch):
    """R-MAT with random labels into nc aggregates: few labels give huge rows
    (DENSE when nc <= 32768, key-range buckets otherwise), many labels give
    warp-piece and CTA-window rows.  path=bins forces the key-range bin pieces
    instead of the bitmap-rank items (HEC_BUILD_SORT); path=one_end the
    degree-based one-end storage + transpose (HEC_BUILD_ONE_END); path=wide_index
    runs the member walks with 64-bit entry indices (the nnz >= 2^32 build,
    HEC_FORCE_WIDE_INDEX test hook)."""
    method = {"bins": "sort", "one_end": "one_end"}.get(path, "hash")
    if path == "wide_index":
        monkeypatch.setenv("HEC_FORCE_WIDE_INDEX", "1")
    rng = np.random.default_rng(15 + nc)
    g = gg.rmat(14 if nc < 20000 else 17, 16)
    g.wgt = rng.integers(1, 1000, g.nnz).astype(np.int32)
    # symmetric weights: w(u,v) = w(v,u) = f(min, max)
    rows = np.repeat(np.arange(g.n), np.diff(g.row_ptr))
    lo, hi = np.minimum(rows, g.col), np.maximum(rows, g.col)
    g.wgt = ((lo.astype(np.int64) * 7919 + hi * 104729) % 1000 + 1).astype(np.int32)
    nc = min(nc, g.n)
    M = rng.integers(0, nc, g.n).astype(np.int32)
    M[rng.permutation(g.n)[:nc]] = np.arange(nc)
    cg = P.build_coarse_graph(ctx, dev(P, g), torch.from_numpy(M).cuda(), nc, method=method)
    assert_csr_equal(cg.graph, o.coarsen(g, M, nc))


def test_construct_wide_piece_keys(P, ctx, monkeypatch):
    """The 64-bit (row, b) key path of the warp pieces (used when n_c > 2^26),
    forced on small graphs through the library's test hook."""
    monkeypatch.setenv("HEC_FORCE_WIDE_KEYS", "1")
    rng = np.random.default_rng(21)
    for t in range(10):
        g = random_graph(int(rng.integers(2, 300)), rng, p=0.1, wmax=50)
        nc = int(rng.integers(1, g.n + 1))
        M = rng.integers(0, nc, g.n).astype(np.int32)
        M[:nc] = np.arange(nc)
        cg = P.build_coarse_graph(ctx, dev(P, g), torch.from_numpy(M).cuda(), nc)
        assert_csr_equal(cg.graph, o.coarsen(g, M, nc))
    check_hierarchy(P, ctx, gg.config(2), 1000)


@pytest.mark.parametrize("spread", [600, 6000, 60000])
def test_construct_crowded_keys(P, ctx, spread):
    """Whole-row rank items whose keys crowd the low end of [0, n_c) (spread
    600 / 6000) or spread uniformly (60000): the hash-rank buckets, balanced by
    the level's volume CDF, see very uneven key densities."""
    rng = np.random.default_rng(31 + spread)
    n, nc = 200000, 60000
    M = rng.integers(0, nc, n).astype(np.int32)
    M[rng.permutation(n)[:nc]] = np.arange(nc)
    by_label = [np.flatnonzero((M >= 1) & (M < spread))]
    edges = {}
    heads = np.arange(200)  # rows 0..9 of 20 members, each member with ~120 neighbours in the crowded labels
    M[heads] = heads // 20
    for u in heads:
        for v in rng.choice(by_label[0], 120, replace=False):
            if v != u:
                edges[(min(u, v), max(u, v))] = int(rng.integers(1, 5))
    for _ in range(2 * n):
        u, v = rng.integers(0, n, 2)
        if u != v:
            edges[(min(u, v), max(u, v))] = int(rng.integers(1, 9))
    g = gg.from_edges(n, [(u, v, w) for (u, v), w in edges.items()])
    present = np.unique(M)
    remap = np.full(nc, -1, np.int64)
    remap[present] = np.arange(present.size)
    M = remap[M].astype(np.int32)
    nc = int(present.size)
    cg = P.build_coarse_graph(ctx, dev(P, g), torch.from_numpy(M).cuda(), nc)
    assert_csr_equal(cg.graph, o.coarsen(g, M, nc))


@pytest.mark.parametrize("path", ["rbm", "bins", "one_end"])
def test_construct_duplicate_heavy_rows(P, ctx, path):
    """Skewed rows whose entries repeat few keys: key-range buckets far above a
    warp piece (CTA tier) and above a CTA block (fallback), next to ordinary rows."""
    method = {"bins": "sort", "one_end": "one_end"}.get(path, "hash")
    rng = np.random.default_rng(22)
    n = 60000
    hub_targets = rng.integers(0, n, 4000)
    edges = {}
    for h in range(8):  # 8 hubs, each adjacent to the same 4000 targets
        for v in hub_targets:
            if v != h:
                edges[(min(h, v), max(h, v))] = 1 + (h + int(v)) % 7
    for _ in range(3 * n):
        u, v = rng.integers(0, n, 2)
        if u != v:
            edges[(min(u, v), max(u, v))] = int(rng.integers(1, 9))
    g = gg.from_edges(n, [(u, v, w) for (u, v), w in edges.items()])
    nc = 40000  # > kDenseMax: BUCKET mode
    M = rng.integers(0, nc, n).astype(np.int32)
    M[:8] = 0  # all hubs in one coarse row
    M[hub_targets] = rng.integers(1, 40, hub_targets.size)  # targets collapse onto few keys
    M[rng.permutation(np.setdiff1d(np.arange(8, n), hub_targets))[:nc]] = np.arange(nc)
    cg = P.build_coarse_graph(ctx, dev(P, g), torch.from_numpy(M).cuda(), nc, method=method)
    assert_csr_equal(cg.graph, o.coarsen(g, M, nc))


@pytest.mark.parametrize("hot", [False, True])
@pytest.mark.parametrize("path", ["direct", "hash"])
def test_construct_direct_bins(P, ctx, path, hot, monkeypatch):
    """A hub row of 100k entries whose keys fall in [1, 3001): its key-range
    bins are narrow (<= 4096 keys) and hold ~25k entries each, so they take the
    direct-indexed counters (k_drank, several rounds per bin); path=hash forces
    the hash-rank kernels (HEC_NO_DRANK test hook)."""
    if path == "hash":
        monkeypatch.setenv("HEC_NO_DRANK", "1")
    rng = np.random.default_rng(24)
    n, nc = 150000, 40000
    # hot: the hub's 100k entries fall on 30 keys (whole warps of equal keys,
    # sums of ~2.3e8 per key)
    nk, w0 = (30, 70000) if hot else (3000, 1)
    edges = {(0, v): w0 + v % 5 for v in range(1, 100001)}
    for _ in range(2 * n):
        u, v = rng.integers(1, n, 2)
        if u != v:
            edges[(min(u, v), max(u, v))] = int(rng.integers(1, 9))
    g = gg.from_edges(n, [(u, v, w) for (u, v), w in edges.items()])
    M = np.empty(n, np.int32)
    M[0] = 0
    M[1:100001] = 1 + np.arange(1, 100001) % nk
    rest = np.arange(100001, n)
    M[rest] = rng.integers(nk + 1, nc, rest.size)
    M[rest[:nc - nk - 1]] = np.arange(nk + 1, nc)
    cg = P.build_coarse_graph(ctx, dev(P, g), torch.from_numpy(M).cuda(), nc)
    assert_csr_equal(cg.graph, o.coarsen(g, M, nc))


def test_construct_rbm_rank_windows(P, ctx):
    """Bitmap-rank bins with more distinct keys than one rank window (kRbmCap =
    4096): a skewed row whose neighbours map densely into the low key range, so
    its first bins hold ~7000 distinct keys each (several rank windows, staged
    to the fallback scratch), next to whole-row items and warp pieces."""
    rng = np.random.default_rng(23)
    n, nc = 100000, 70000
    edges = {}
    hubs = np.arange(6)
    nbrs = rng.choice(np.arange(6, n), 24000, replace=False)
    for h in hubs:
        for v in nbrs[h * 4000:(h + 1) * 4000]:
            edges[(int(h), int(v))] = 1 + int(v) % 5
    for _ in range(2 * n):
        u, v = rng.integers(0, n, 2)
        if u != v:
            edges[(min(u, v), max(u, v))] = int(rng.integers(1, 9))
    g = gg.from_edges(n, [(u, v, w) for (u, v), w in edges.items()])
    M = np.empty(n, np.int32)
    rest = np.setdiff1d(np.arange(n), np.concatenate([hubs, nbrs]))
    M[hubs] = 0
    M[nbrs] = 1 + np.arange(nbrs.size) % 20000  # hub row: ~20k distinct keys in [1, 20000]
    M[rest] = rng.integers(0, nc, rest.size)
    M[rng.permutation(rest)[:nc]] = np.arange(nc)
    cg = P.build_coarse_graph(ctx, dev(P, g), torch.from_numpy(M).cuda(), nc)
    assert_csr_equal(cg.graph, o.coarsen(g, M, nc))


def test_construct_dense_row_overflow(P, ctx):
    """A DENSE skewed row (a hub whose 6000 leaves collapse onto one coarse
    vertex): a coarse weight above INT32_MAX is reported, one just below is exact."""
    n = 6001
    M = np.ones(n, np.int32)
    M[0] = 0
    M[1] = 2  # a third aggregate keeps the hub row's keys from being a single value
    for w, ok in ((2**20, False), ((2**31 - 1) // 6000, True)):
        g = gg.from_edges(n, [(0, v, w) for v in range(1, n)])
        Mt = torch.from_numpy(M).cuda()
        if ok:
            cg = P.build_coarse_graph(ctx, dev(P, g), Mt, 3)
            assert_csr_equal(cg.graph, o.coarsen(g, M, 3))
        else:
            with pytest.raises(P.HecError) as e:
                P.build_coarse_graph(ctx, dev(P, g), Mt, 3)
            assert e.value.code == P.HEC_EOVERFLOW


def test_construct_overflow_detected(P, ctx):
    big = 2**31 - 1
    g = gg.from_edges(3, [(0, 2, big), (1, 2, big)])
    M = torch.tensor([0, 0, 1], dtype=torch.int32, device="cuda")
    with pytest.raises(P.HecError) as e:
        P.build_coarse_graph(ctx, dev(P, g), M, 2)
    assert e.value.code == P.HEC_EOVERFLOW
    # near the limit but exact: no error
    g = gg.from_edges(3, [(0, 2, big // 2), (1, 2, big // 2)])
    cg = P.build_coarse_graph(ctx, dev(P, g), M, 2)
    assert_csr_equal(cg.graph, o.coarsen(g, M.cpu().numpy(), 2))


def test_construct_rejects_bad_labels(P, ctx):
    g = gg.from_edges(3, [(0, 1, 1), (1, 2, 1)])
    M = torch.tensor([0, 5, 1], dtype=torch.int32, device="cuda")
    with pytest.raises(P.HecError) as e:
        P.build_coarse_graph(ctx, dev(P, g), M, 2)
    assert e.value.code == P.HEC_EINVAL


def test_validate_flags_bad_graph(P):
    c = P.Context(validate=True)
    g = gg.from_edges(4, [(0, 1, 1), (1, 2, 1), (2, 3, 1)])
    dg = dev(P, g)
    P.hec_find_mapping(c, dg, SEED, 0)  # valid graph passes
    bad = P.DeviceGraph(dg.row_ptr.clone(), dg.col.clone(), dg.wgt.clone(), dg.vwgt)
    bad.wgt[0] = 5  # asymmetric weight
    with pytest.raises(P.HecError) as e:
        P.hec_find_mapping(c, bad, SEED, 0)
    assert e.value.code == P.HEC_EINVAL and "asymmetric" in str(e.value)
    c.close()


# ------------------------------------------------------------ hierarchy
def check_hierarchy(P, ctx, g, cutoff):
    Ho = o.hierarchy(g, cutoff, SEED)
    Hg = P.coarsen_hierarchy(ctx, dev(P, g), cutoff, SEED)
    assert len(Hg.levels) == len(Ho.levels)
    assert Hg.stop_reason == Ho.stop_reason
    if Ho.stop_reason == o.STOP_DISCARD:
        assert Hg.discarded_n_c == Ho.discarded_n_c
    for lg, lo in zip(Hg.levels, Ho.levels):
        assert np.array_equal(lg.M.cpu().numpy(), lo.M)
        assert_csr_equal(lg.graph, lo.graph)
    return Hg


def test_hierarchy_c1(P, ctx, golden_dir):
    Hg = check_hierarchy(P, ctx, gg.config(1), 50)
    ka = json.load(open(os.path.join(golden_dir, "survey_known_answers.json")))["C1"]
    # The kernel fuses decide(r) with scatter(r+1); a root flag published in the
    # same round may be seen one round early, so the count can only be lower.
    # The result (M, G_c) is unaffected — compared exactly above.
    rounds = [lv.rounds for lv in Hg.levels]
    assert all(1 <= r <= k for r, k in zip(rounds, ka["rounds"])), rounds


@pytest.mark.parametrize("build", ["sort", "one_end", "auto"])
@pytest.mark.parametrize("which,cutoff", [("c1", 50), ("rmat14", 50), ("mesh27_24", 100)])
def test_hierarchy_build_methods(P, ctx, build, which, cutoff):
    """Every construction method (hash / sort / one-end) gives the
    oracle's hierarchy bit for bit."""
    g = {"c1": lambda: gg.config(1), "rmat14": lambda: gg.rmat(14, 16),
         "mesh27_24": lambda: gg.mesh27(24, 24, 24)}[which]()
    H = P.coarsen_hierarchy(ctx, dev(P, g), cutoff, SEED, build=build)
    ref = o.hierarchy(g, cutoff, SEED)
    assert len(H.levels) == len(ref.levels) and H.stop_reason == ref.stop_reason
    for lv, lo in zip(H.levels, ref.levels):
        assert np.array_equal(lv.M.cpu().numpy(), lo.M)
        assert_csr_equal(lv.graph, lo.graph)
    H.free()


def test_hierarchy_c2(P, ctx):
    check_hierarchy(P, ctx, gg.config(2), 1000)


@pytest.mark.parametrize("which", ["c1", "rmat12", "mesh27_16"])
def test_hierarchy_fused_heavy_small(P, ctx, which, monkeypatch):
    """The fused heavy keys on small graphs: every placement in one slice per
    32-block group and every level fused (HEC_PLACE_ONE_SLICE, HEC_FUSE_HEAVY_ALL
    test hooks), bit-exact vs the oracle."""
    monkeypatch.setenv("HEC_FUSE_HEAVY_ALL", "1")
    monkeypatch.setenv("HEC_PLACE_ONE_SLICE", "1")
    g = {"c1": lambda: gg.config(1), "rmat12": lambda: gg.rmat(12, 16), "mesh27_16": lambda: gg.mesh27(16, 16, 16)}[which]()
    check_hierarchy(P, ctx, g, 50)


def test_hierarchy_c2_fused_heavy_everywhere(P, ctx, monkeypatch):
    """The next level's heavy neighbours computed by the placement (k_place) on
    every large-enough level, also where most entries sit in multi-row piece
    blocks (per-entry row search; HEC_FUSE_HEAVY_ALL test hook; by default only
    levels averaging >= 256 entries per coarse row fuse)."""
    monkeypatch.setenv("HEC_FUSE_HEAVY_ALL", "1")
    check_hierarchy(P, ctx, gg.config(2), 1000)


@pytest.mark.parametrize("scale", [10, 12, 16, 18])
def test_hierarchy_rmat(P, ctx, scale):
    check_hierarchy(P, ctx, gg.rmat(scale, 16), 50)


@pytest.mark.parametrize("fused", [False, True])
def test_hierarchy_edge_cases(P, ctx, fused, monkeypatch):
    """fused: the heavy keys of every level from its placement (test hooks),
    including rows of G_{l+1} left empty by isolated vertices (key 0 -> itself)."""
    if fused:
        monkeypatch.setenv("HEC_FUSE_HEAVY_ALL", "1")
        monkeypatch.setenv("HEC_PLACE_ONE_SLICE", "1")
    empty = gg.Graph(np.zeros(1, np.int64), np.zeros(0, np.int32), np.zeros(0, np.int32), np.zeros(0, np.int32))
    Hg = P.coarsen_hierarchy(ctx, P.DeviceGraph.from_host(empty), 50, SEED)
    assert Hg.levels == [] and Hg.stop_reason == P.STOP_CUTOFF
    iso = gg.Graph(np.zeros(61, np.int64), np.zeros(0, np.int32), np.zeros(0, np.int32), np.ones(60, np.int32))
    Hg = P.coarsen_hierarchy(ctx, P.DeviceGraph.from_host(iso), 50, SEED)
    assert Hg.levels == [] and Hg.stop_reason == P.STOP_STALL
    star = gg.from_edges(60, [(0, i, 1) for i in range(1, 60)])
    Hg = P.coarsen_hierarchy(ctx, dev(P, star), 50, SEED)
    assert Hg.levels == [] and Hg.stop_reason == P.STOP_DISCARD and Hg.discarded_n_c == 1
    Hg = P.coarsen_hierarchy(ctx, dev(P, gg.config(1)), 50, SEED, max_levels=2)
    assert len(Hg.levels) == 2 and Hg.stop_reason == P.STOP_MAX_LEVELS
    # graph with isolated vertices and a disconnected part
    rng = np.random.default_rng(16)
    g = random_graph(500, rng, p=0.01, wmax=3, isolated=7)
    check_hierarchy(P, ctx, g, 20)


def digest_levels(Hg):
    out = []
    for lv in Hg.levels:
        rp, col, wgt, vw = host_csr(lv.graph)
        out.append(dict(n_c=lv.graph.n, nnz_c=lv.graph.nnz, sum_wc=int(wgt.astype(np.int64).sum()),
                        sha_M=gg.sha16(lv.M.cpu().numpy()), sha_G=gg.sha16(rp, col, wgt), sha_vwgt=gg.sha16(vw)))
    return out


@pytest.mark.parametrize("cfg", [2, 3, 4, 5])
def test_hierarchy_full_size_digests(P, ctx, golden_dir, cfg):
    """Whole hierarchy at BASELINE.json's full sizes (C5 = R-MAT s26 ef16, the
    one-GPU launch configuration bench.py --config 5 times) against the oracle's
    per-level digests (tests/golden/make_digests.py, oracle/ only)."""
    dd = json.load(open(os.path.join(golden_dir, "oracle_digests.json")))
    if str(cfg) not in dd:
        pytest.skip(f"no oracle digest for C{cfg} (python tests/golden/make_digests.py {cfg})")
    d = dd[str(cfg)]
    g = gg.config(cfg)
    assert gg.sha16(g.row_ptr, g.col) == d["sha_G0"]
    Hg = P.coarsen_hierarchy(ctx, dev(P, g), d["cutoff"], d["seed"])
    del g
    got = digest_levels(Hg)
    exp = [{k: lv[k] for k in ("n_c", "nnz_c", "sum_wc", "sha_M", "sha_G", "sha_vwgt")} for lv in d["levels"]]
    assert got == exp
    assert Hg.stop_reason == d["stop_reason"]
    if d["discarded_n_c"] is not None:
        assert Hg.discarded_n_c == d["discarded_n_c"]
