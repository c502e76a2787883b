"""Host-side logic of the multi-GPU path on CPU: world_size 2,
gloo backend, 127.0.0.1.  The collectives and range arithmetic used by
paper_conf_ipps_gilbertabmr21_b200.dist, without a GPU."""
import torch
import torch.multiprocessing as mp

from dist_helpers import free_port, init


def test_even_ranges():
    from paper_conf_ipps_gilbertabmr21_b200.dist import even_ranges
    for n in [0, 1, 7, 100, 101]:
        for parts in [1, 2, 3, 8]:
            r = even_ranges(n, parts)
            assert len(r) == parts and r[0][0] == 0 and r[-1][1] == n
            assert all(a[1] == b[0] for a, b in zip(r, r[1:]))
            sizes = [hi - lo for lo, hi in r]
            assert max(sizes) - min(sizes) <= 1


def _worker(rank, world, port, q):
    import torch.distributed as dist
    from paper_conf_ipps_gilbertabmr21_b200.dist import all_gather_scalars, all_gather_uneven, even_ranges
    init(rank, world, port)
    try:
        n = 11
        rng = even_ranges(n, world)
        lo, hi = rng[rank]
        full = torch.arange(n, dtype=torch.int64) * 3 + 1
        mine = full[lo:hi].clone()
        got = all_gather_uneven(mine, [b - a for a, b in rng])
        assert torch.equal(got, full)
        # int32 pieces of very different sizes, one empty
        sizes = [5, 0] if world == 2 else [5] * world
        piece = torch.full((sizes[rank],), rank + 7, dtype=torch.int32)
        got = all_gather_uneven(piece, sizes)
        exp = torch.cat([torch.full((s,), r + 7, dtype=torch.int32) for r, s in enumerate(sizes)])
        assert torch.equal(got, exp)
        sc = all_gather_scalars([rank * 10, rank + 1])
        assert sc == [[r * 10, r + 1] for r in range(world)]
        # global offsets of slices = exclusive prefix of the gathered totals
        totals = [v[0] for v in all_gather_scalars([100 + rank])]
        assert sum(totals[:rank]) == sum(100 + r for r in range(rank))
        q.put((rank, "ok"))
    except Exception as e:  # noqa: BLE001
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_collectives():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert res == {0: "ok", 1: "ok"}, res
