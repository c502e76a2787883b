"""Host side of the multi-GPU path on CPU: world_size 2, gloo,
127.0.0.1.  libhec's dist calls exchange data only through the all-gather
callback of paper_conf_ipps_gilbertabmr21_b200.dist; here that callback (byte
views of raw pointers, equal-block all-gather, rank order) is checked without a
GPU, together with the fine-vertex slice arithmetic."""
import ctypes

import numpy as np
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
    from paper_conf_ipps_gilbertabmr21_b200 import _lib
    from paper_conf_ipps_gilbertabmr21_b200.dist import allgather_bytes
    init(rank, world, port)
    try:
        cpu = torch.device("cpu")
        # equal blocks of raw host bytes, gathered in rank order
        nb = 13
        send = np.full(nb, 40 + rank, np.uint8)
        recv = np.zeros(nb * world, np.uint8)
        allgather_bytes(send.ctypes.data, recv.ctypes.data, nb, None, cpu)
        assert np.array_equal(recv, np.repeat(np.arange(40, 40 + world, dtype=np.uint8), nb))
        # int64 payloads (the slices' entry counts) through the C callback type
        calls = []

        def cb(s, r, n, stream, user):
            calls.append(n)
            allgather_bytes(s, r, int(n), None, cpu)
            return 0
        fn = _lib.ALLGATHER_FN(cb)
        mine = np.array([1000 + rank], np.int64)
        got = np.zeros(world, np.int64)
        assert fn(mine.ctypes.data, got.ctypes.data, 8, None, None) == 0
        assert got.tolist() == [1000 + r for r in range(world)] and calls == [8]
        # zero-length blocks are legal
        allgather_bytes(0, 0, 0, None, cpu)
        q.put((rank, "ok"))
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_allgather_callback():
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
