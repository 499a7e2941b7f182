"""Multi-process host logic on CPU (gloo, world_size 2): the count all-reduce
callback the C library calls for world > 1, and bench.py's max-over-ranks timing."""
import ctypes as C
import os
import socket

import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_icde_hu0o23_b200 as G
        cb = G.make_allreduce_callback(0)
        buf = (C.c_uint64 * 3)(rank + 1, 10 * (rank + 1), 2 ** 40 + rank)
        st = cb(buf, 3, None)
        import bench
        t = bench.max_over_ranks(1.5 + rank, world)
        q.put((rank, st, list(buf), t))
    finally:
        dist.destroy_process_group()


def test_allreduce_callback_and_max_timing():
    world = 2
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, st, buf, t in res:
        assert st == 0
        assert buf == [3, 30, 2 * 2 ** 40 + 1]
        assert t == 2.5
