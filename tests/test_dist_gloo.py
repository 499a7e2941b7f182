"""Multi-process host logic on CPU (gloo, world_size 2): the count all-reduce
callback the C library calls for world > 1, the all-to-all behind gamma_fpm's
domain-bitmap exchange, and bench.py's max-over-ranks timing."""
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
        big = (C.c_uint64 * 1)(2 ** 63 + 5)     # uint64 sums wrap like the library's
        st2 = cb(big, 1, None)
        # all-to-all layout of the FPM exchange: rank r's block g lands in rank g's block r
        send = torch.arange(6, dtype=torch.int32) + 100 * rank
        recv = torch.empty(6, dtype=torch.int32)
        G.alltoall_tensors(send, recv)
        import bench
        t = bench.max_over_ranks(1.5 + rank, world)
        tsum = bench.max_over_ranks(1.5 + rank, world, "sum")
        q.put((rank, st + st2, list(buf) + [big[0]], recv.tolist(), (t, tsum)))
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
    for rank, st, buf, recv, t in res:
        assert st == 0
        assert buf == [3, 30, 2 * 2 ** 40 + 1, 10]
        assert recv == [3 * rank, 3 * rank + 1, 3 * rank + 2, 100 + 3 * rank, 101 + 3 * rank, 102 + 3 * rank]
        assert t == (2.5, 4.0)   # max and sum over ranks (imbalance = max / (sum / world))
