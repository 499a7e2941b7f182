#!/usr/bin/env python3
"""Probe C5 (Friendster-shaped R-MAT, scale 26) candidates on the GPU box: draw the raw
samples in HBM (gamma_gen.torch_gen), build, and time triangle / 4-clique counts.

  python tools/c5_probe.py --a 0.55 --samples 2.2e9 [--a 0.57 --samples 2.0e9 ...]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_icde_hu0o23_b200 as G  # noqa: E402
from gamma_gen.torch_gen import rmat_torch  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--a", type=float, action="append", required=True)
    ap.add_argument("--samples", type=float, action="append", required=True)
    ap.add_argument("--scale", type=int, default=26)
    ap.add_argument("--ks", default="3,4")
    args = ap.parse_args()
    ks = [int(x) for x in args.ks.split(",")]
    ctx = G.Context(device=0)
    for a, ns in zip(args.a, args.samples):
        ns = int(ns)
        b = c = round((1 - a - 0.05) / 2, 4)   # d = 0.05 as in Graph500 (0.57, 0.19, 0.19)
        t0 = time.time()
        src, dst = rmat_torch(args.scale, ns, a, b, c, 1)
        torch.cuda.synchronize()
        tg = time.time() - t0
        t0 = time.time()
        g = ctx.load_edges(1 << args.scale, src, dst)
        torch.cuda.synchronize()
        tb = time.time() - t0
        del src, dst
        torch.cuda.empty_cache()
        info = g.info()
        out = {"a": a, "b": b, "c": c, "samples": ns, "gen_s": tg, "build_s": tb, **info,
               "peak_gb": torch.cuda.max_memory_allocated() / 1e9}
        for k in ks:
            t0 = time.time()
            out[f"k{k}"] = g.kclique(k)
            out[f"k{k}_s"] = time.time() - t0
            out[f"k{k}_stats"] = {kk: v for kk, v in ctx.stats().items() if kk in ("chunks", "retries", "spilled_bytes")}
        print(json.dumps(out), flush=True)
        del g
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
