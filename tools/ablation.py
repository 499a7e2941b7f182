"""Ablation and density study on synthetic Kronecker (R-MAT) graphs (
the paper's Figs. 15, 17-18), run on one GPU.

Variants of the same extension primitive, selected by ctx flags (include/gamma.h):
  kCL  default      bitmap DFS below each root (Opt 2 taken to its limit)
       no_split     ... without hub splitting of heavy roots
       et_fused     list-based ET (Opt 1 per-warp blocks + Opt 2 grouping), last two
                    levels fused in shared memory              (GAMMA_FLAG_NO_BITMAP)
       et_levels    list-based ET, every level materialised    (NO_BITMAP | NO_FUSE)
       et_two_pass  ... with the naive count-then-write extension instead of Opt 1's
                    warp memory blocks (NO_BITMAP | NO_FUSE | TWO_PASS)
  SM   default      grouped extension, L_m staged once per group (Opt 2)
       no_group     L_m never staged: every child intersects all backward lists
                    (GAMMA_FLAG_DEBUG_NOSTAGE)
Density: R-MAT scale 18, (0.57, 0.19, 0.19), edge factor 4..32.  Every count is
checked equal across variants; times are CUDA events on the launching stream, median
of 3 after one warm-up.  Writes one JSON line per (task, density, variant).

    python tools/ablation.py > gpurun_out/ablation.jsonl
"""
from __future__ import annotations

import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import gamma_gen as gg  # noqa: E402
import paper_conf_icde_hu0o23_b200 as G  # noqa: E402

KCL = {"default": 0, "no_split": 0x20, "et_fused": 0x10, "et_levels": 0x10 | 0x2, "et_two_pass": 0x10 | 0x2 | 0x200}
SM = {"default": 0, "no_group": 0x8}


def timed(fn, reps=3):
    fn()
    st = torch.cuda.current_stream()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record(st)
        r = fn()
        b.record(st)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return r, float(np.median(ts))


def main():
    scale = int(os.environ.get("ABL_SCALE", 18))
    out = []
    for ef in (4, 8, 16, 32):
        s, d = gg.rmat(scale, ef << scale, 0.57, 0.19, 0.19, seed=1)
        n = 1 << scale
        lab = gg.labels(n, 4, 1)
        ref = {}
        for name, fl in KCL.items():
            ctx = G.Context(device=0, flags=fl)
            g = ctx.load_edges(n, torch.from_numpy(s.view("int32")).cuda(),
                               torch.from_numpy(d.view("int32")).cuda())
            m = g.info()["m"]
            r, ms = timed(lambda: g.kclique_multi([4, 5]))
            ref.setdefault("kcl", r)
            rec = {"task": "kcl k=4,5", "scale": scale, "edge_factor": ef, "m": m, "variant": name,
                   "ms": ms, "counts": r, "agree": r == ref["kcl"],
                   "embeddings_per_s": sum(r) / ms * 1e3}
            print(json.dumps(rec), flush=True)
            out.append(rec)
            g.free()
            ctx.close()
        plab = [0, 1, 0, 1]
        nv, e = gg.QUERIES["c4"]
        for name, fl in SM.items():
            ctx = G.Context(device=0, flags=fl)
            g = ctx.load_edges(n, torch.from_numpy(s.view("int32")).cuda(),
                               torch.from_numpy(d.view("int32")).cuda(), torch.from_numpy(lab.view("int32")).cuda())
            r, ms = timed(lambda: g.match(nv, e, plab)[0])
            ref.setdefault("sm", r)
            rec = {"task": "sm c4 labels (0,1,0,1), L=4", "scale": scale, "edge_factor": ef, "variant": name,
                   "ms": ms, "count": r, "agree": r == ref["sm"], "embeddings_per_s": r / ms * 1e3}
            print(json.dumps(rec), flush=True)
            out.append(rec)
            g.free()
            ctx.close()
    assert all(r["agree"] for r in out), "variants disagree"


if __name__ == "__main__":
    main()
