#!/usr/bin/env python3
"""Simulated ranks on one GPU (SURVEY.md §8(e) load balance without an 8-GPU box).

For a workload, run the rank-r share of the root partition for r = 0..world-1 one
after another on cuda:0 (Context(rank=r, world=W, reduce=False): every rank computes
only its partial count, no collective), and report per rank the device time of the
compute kernels (CUDA events, summed over the hot-path kernel classes), the partial
counts (their sum must equal the world-1 count), and max/mean of the rank times --
the imbalance that caps strong scaling at world W to W / (max/mean).

    python tools/sim_ranks.py c2|heavy|c3|c5 [--world 8] [--reps 2] [--out profiles/sim_ranks_r02.jsonl]
"""
import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

HOT = ("extend", "count", "fused", "bitmap", "sm_extend", "sm_count", "fpm", "roots")


def load_graph(ctx, name):
    import torch
    import gamma_gen as gg
    if name == "c5":
        from gamma_gen.torch_gen import config_graph_torch
        n, s, d = config_graph_torch("c5", seed=1)
        g = ctx.load_edges(n, s, d)
        del s, d
        torch.cuda.empty_cache()
        return g, None
    n, s, d, lab = gg.config_graph(name, seed=1)
    return ctx.load_edges(n, torch.from_numpy(s.view(np.int32)).cuda(), torch.from_numpy(d.view(np.int32)).cuda(),
                          None if lab is None else torch.from_numpy(lab.view(np.int32)).cuda()), lab


def work(g, name):
    import gamma_gen as gg
    if name in ("c2", "heavy", "c5"):
        ks = {"c2": [4, 5, 6], "heavy": [4, 5], "c5": [3, 4]}[name]
        return g.kclique_multi(ks)
    out = []
    for q in ("c4", "diamond", "tailed_triangle", "house"):
        nv, e = gg.QUERIES[q]
        for plab in ([0] * nv, [i % 8 for i in range(nv)]):
            out.append(g.match(nv, e, plab)[0])
    return out


def kernel_ms(st):
    return sum(c["ms"] for k, c in st["classes"].items() if k in HOT)


def class_ms(st):
    return {k: round(c["ms"], 3) for k, c in st["classes"].items() if c["launches"]}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("workload", choices=["c2", "heavy", "c3", "c5"])
    ap.add_argument("--world", type=int, default=8)
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    import torch
    import paper_conf_icde_hu0o23_b200 as G

    ctxs = [G.Context(device=0, rank=r, world=args.world, reduce=False, time_kernels=True) for r in range(args.world)]
    base = G.Context(device=0, time_kernels=True)
    # one graph per context (the root order is cached per graph for its (rank, world))
    g1, _ = load_graph(base, args.workload)
    want = work(g1, args.workload)
    t1, w1 = [], []
    for _ in range(args.reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        got = work(g1, args.workload)
        e1.record()
        torch.cuda.synchronize()
        t1.append(kernel_ms(base.stats()) if args.workload != "c3" else None)
        w1.append(e0.elapsed_time(e1))
    if args.workload != "c3":
        print("world 1 classes", class_ms(base.stats()), flush=True)
    g1.free()
    per_rank, parts, per_rank_wall = [], [], []
    for r, c in enumerate(ctxs):
        g, _ = load_graph(c, args.workload)
        times, walls = [], []
        for _ in range(args.reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            if args.workload == "c3":   # 8 calls: sum their kernel times
                import gamma_gen as gg
                ms, res = 0.0, []
                for q in ("c4", "diamond", "tailed_triangle", "house"):
                    nv, e = gg.QUERIES[q]
                    for plab in ([0] * nv, [i % 8 for i in range(nv)]):
                        res.append(g.match(nv, e, plab)[0])
                        ms += kernel_ms(c.stats())
            else:
                res = work(g, args.workload)
                ms = kernel_ms(c.stats())
                cls = class_ms(c.stats())
            e1.record()
            torch.cuda.synchronize()
            times.append(ms)
            walls.append(e0.elapsed_time(e1))
        per_rank.append(min(times))
        per_rank_wall.append(min(walls))
        parts.append(res)
        g.free()
        print(f"rank {r}: kernel ms {min(times):.3f} device wall ms {min(walls):.3f} partial {res} "
              f"classes {cls if args.workload != 'c3' else ''}", flush=True)
    tot = [sum(p[i] for p in parts) for i in range(len(want))]
    assert tot == want, (tot, want)
    mean = statistics.mean(per_rank)
    # device wall time of each rank's call (CUDA events on the calling stream): with the
    # kCL team launches on concurrent streams the summed kernel times overlap
    wmean = statistics.mean(per_rank_wall)
    rec = {"workload": args.workload, "world": args.world, "rank_kernel_ms": [round(x, 3) for x in per_rank],
           "max_over_mean": max(per_rank) / mean, "sum_of_partials_equals_world1": True,
           "rank_wall_ms": [round(x, 3) for x in per_rank_wall], "wall_max_over_mean": max(per_rank_wall) / wmean,
           "world1_wall_ms": min(w1), "speedup_wall": min(w1) / max(per_rank_wall),
           "world1_kernel_ms": min(x for x in t1 if x is not None) if args.workload != "c3" else None,
           "counts": want, "partition": "roots sorted by cost, snake (boustrophedon) over ranks"}
    print(json.dumps(rec), flush=True)
    if args.out:
        with open(args.out, "a") as f:
            f.write(json.dumps(rec) + "\n")


if __name__ == "__main__":
    main()
