"""Multi-rank runs on one GPU: two processes (gloo process group, both on cuda:0)
through the real collective callbacks.  kCL / SM counts are all-reduced; FPM's last
level is split over the ranks and its MNI domain bitmaps OR-reduced by the
all-to-all exchange.  Every rank must return the oracle's result."""
import os
import socket

import pytest

import gamma_gen as gg

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q, budget):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_icde_hu0o23_b200 as G
        torch.cuda.set_device(0)
        c = G.Context(device=0, hbm_budget_bytes=budget)
        assert c.world == world and c.rank == rank
        n, s, d, _ = gg.config_graph("c4", seed=2, scale=11)
        lab = gg.labels(n, 5, 2)
        g = c.load_edges(n, s, d, lab)
        res = {"fpm3": g.fpm(3, 20), "chunks": c.stats()["chunks"], "fpm2": g.fpm(2, 5), "fpm1": g.fpm(1, 3),
               "k4": g.kclique(4), "multi": g.kclique_multi([3, 4, 5]),
               "c4": g.match(4, gg.QUERIES["c4"][1], [0, 1, 0, 1])[0]}
        q.put((rank, res))
    except Exception as e:   # noqa: BLE001
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("budget", [0, 100 << 10])
def test_two_ranks_gloo(oracle_mod, budget):
    import gc

    import torch
    import torch.multiprocessing as mp
    # the two rank processes share this GPU and size FPM pools from its free memory:
    # hand back what earlier tests of this process hold (contexts of finished modules,
    # the caching allocator's idle blocks)
    gc.collect()
    torch.cuda.empty_cache()
    world = 2
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, budget)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    n, s, d, _ = gg.config_graph("c4", seed=2, scale=11)
    lab = gg.labels(n, 5, 2)
    o = oracle_mod.Graph(n, s, d, lab)
    want = {"fpm3": [r[:5] for r in o.fpm(3, 20, pattern_cap=1 << 20)],
            "fpm2": [r[:5] for r in o.fpm(2, 5, pattern_cap=1 << 20)],
            "fpm1": [r[:5] for r in o.fpm(1, 3, pattern_cap=1 << 20)],
            "k4": o.kclique(4), "multi": [o.kclique(k) for k in (3, 4, 5)],
            "c4": o.match(4, gg.QUERIES["c4"][1], [0, 1, 0, 1])[0]}
    for rank, r in res:
        assert isinstance(r, dict), r
        for key, w in want.items():
            assert r[key] == w, (rank, key)
        if budget:
            assert r["chunks"] > 1   # the distributed level ran in several chunks
