#!/usr/bin/env python3
"""Algorithmic bytes of the kCL bench workloads, counted by a host
pass over the ORACLE's enumeration (oracle.Graph.kclique_levels) -- independent of
the CUDA path -- and written to profiles/alg_bytes.json for bench.py's roofline.

Per extension step l -> l+1 of the embedding table (level 2 = the DAG edges, the CSR
itself):
    B_l = 12 N_l              read (vid, parent) + stage the sibling run once per group
        + 4 S_l               fetch N+(u) of every level-l entry u (the intersect step)
        + 8 N_{l+1} [l+1 < k] write the next level (the last level is counted, not written)
N_l = #l-cliques, S_l = sum over l-cliques of d+(last vertex).  A multi-k step
(k = 4, 5, 6 from one walk) costs the walk of its largest k.

    python tools/alg_bytes.py [c1 c2 heavy]
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import gamma_gen as gg  # noqa: E402
import oracle  # noqa: E402

KMAX = {"c1": 4, "c2": 6, "heavy": 5}


def main():
    names = sys.argv[1:] or list(KMAX)
    out_path = os.path.join(ROOT, "profiles", "alg_bytes.json")
    res = json.load(open(out_path)) if os.path.exists(out_path) else {}
    for name in names:
        k = KMAX[name]
        n, s, d, lab = gg.config_graph(name, seed=1)
        g = oracle.Graph(n, s, d, lab)
        t0 = time.time()
        N, S = g.kclique_levels(k)
        steps = []
        for l in range(2, k):
            b = 12 * N[l] + 4 * S[l] + (8 * N[l + 1] if l + 1 < k else 0)
            steps.append({"step": f"{l}->{l + 1}", "bytes": b, "adjacency_bytes": 4 * S[l]})
        res[name] = {"kmax": k, "N": N, "S": S, "steps": steps,
                     "bytes_per_step": sum(x["bytes"] for x in steps),
                     "oracle_seconds": round(time.time() - t0, 2),
                     "how": "oracle.Graph.kclique_levels on gamma_gen.config_graph(name, seed=1)"}
        print(name, json.dumps(res[name]), flush=True)
        json.dump(res, open(out_path, "w"), indent=1)


if __name__ == "__main__":
    main()
