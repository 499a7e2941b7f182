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
SM_QUERIES = ("c4", "diamond", "tailed_triangle", "house")


def sm_bytes(name):
    """SM (C3): per query and labeling, the ET steps t -> t+1 of the method's matching
    order with its symmetry breaking (oracle planner plan_r10_r16, R10/R16), counted by
    og_match_levels (O-2b):  B_t = 12 N[t] + 4 (G[t] + C[t]) + 8 N[t+1] [t+1 < nv]
    (G: the group's prefix lists, once per group -- Opt 2; C: each child's own list).
    The last step is the count level (kernel class sm_count), the others sm_extend."""
    n, s, d, lab = gg.config_graph(name, seed=1)
    g = oracle.Graph(n, s, d, lab)
    t0 = time.time()
    runs, ext, cnt = {}, 0, 0
    for q in SM_QUERIES:
        nv, e = gg.QUERIES[q]
        for lname, plab in (("all0", [0] * nv), ("imod8", [i % 8 for i in range(nv)])):
            N, G, C = g.match_levels(nv, e, plab)
            steps = []
            for t in range(1, nv):
                b = 12 * N[t] + 4 * (G[t] + C[t]) + (8 * N[t + 1] if t + 1 < nv else 0)
                steps.append(b)
            ext += sum(steps[:-1])
            cnt += steps[-1]
            runs[f"{q}/{lname}"] = {"N": N, "G": G, "C": C, "step_bytes": steps}
            print(q, lname, N, steps, flush=True)
    return {"runs": runs, "bytes_per_step": ext + cnt, "class_bytes_per_step": {"sm_extend": ext, "sm_count": cnt},
            "oracle_seconds": round(time.time() - t0, 2),
            "how": "oracle.Graph.match_levels (O-2b) with oracle.plan_r10_r16 on gamma_gen.config_graph(name, seed=1)"}


def fpm_bytes(name, l=3):
    """FPM (C4), Alg. 2 with every prefix frequent (minsup = 1: an upper bound of the
    work at a larger minsup, whose pruning can only remove prefixes): level 1 reads the
    edges, level 2 reads N(u) ++ N(v) per edge, level 3 N(u) ++ N(v) ++ N(y) per
    connected 2-edge set, and each recorded embedding costs 32 B (its 16-byte pattern
    table slot + one 4-byte MNI domain word per position, <= 4 positions):
        B = sum_l 4 A_l + 32 N_l,  N_1 = m, N_2 = sum_v C(d_v,2),
        N_3 = T + sum_v C(d_v,3) + sum_(u,v) (d_u-1)(d_v-1) - 3T,
        A_1 = 2m, A_2 = sum_v d_v^2, A_3 = sum over 2-edge sets of the 3 vertices' degrees.
    Computed from the oracle's CSR (O-0) and triangle count (O-1)."""
    import numpy as np
    n, s, d, lab = gg.config_graph(name, seed=1)
    g = oracle.Graph(n, s, d, lab)
    t0 = time.time()
    off, adj = g.csr()
    deg = np.diff(off.astype(np.int64))
    src = np.repeat(np.arange(n, dtype=np.int64), deg)
    und = src < adj
    du, dv = deg[src[und]], deg[adj[und].astype(np.int64)]
    T = g.kclique(3)
    N1 = int(und.sum())
    N2 = int((deg * (deg - 1) // 2).sum())
    N3 = int(T + (deg * (deg - 1) * (deg - 2) // 6).sum() + ((du - 1) * (dv - 1)).sum() - 3 * T)
    # A_3: wedges centred at c with leaves a != b: sum over them of d_c + d_a + d_b
    #    = sum_c [C(d_c,2) d_c + (d_c - 1) sum_{a in N(c)} d_a]
    nbr_deg_sum = np.bincount(src, weights=deg[adj.astype(np.int64)].astype(np.float64), minlength=n)
    A3 = int(round(float((deg * (deg - 1) // 2 * deg).sum() + ((deg - 1) * nbr_deg_sum).sum())))
    A = [2 * N1, int((deg * deg).sum()), A3][:l]
    Nl = [N1, N2, N3][:l]
    steps = [{"level": i + 1, "embeddings": Nl[i], "adjacency_elems": A[i], "bytes": 4 * A[i] + 32 * Nl[i]}
             for i in range(l)]
    return {"l": l, "steps": steps, "bytes_per_step": sum(x["bytes"] for x in steps),
            "oracle_seconds": round(time.time() - t0, 2),
            "how": "closed forms over oracle.Graph.csr() (O-0) and oracle.Graph.kclique(3) (O-1), minsup = 1 "
                   "(upper bound)"}


def main():
    names = sys.argv[1:] or list(KMAX)
    out_path = os.path.join(ROOT, "profiles", "alg_bytes.json")
    res = json.load(open(out_path)) if os.path.exists(out_path) else {}
    for name in names:
        if name == "c3":
            res[name] = sm_bytes(name)
            json.dump(res, open(out_path, "w"), indent=1)
            continue
        if name == "c4":
            res[name] = fpm_bytes(name)
            print(name, json.dumps(res[name]), flush=True)
            json.dump(res, open(out_path, "w"), indent=1)
            continue
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
