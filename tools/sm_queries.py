#!/usr/bin/env python3
"""Per-query SM timing on C3 (GPU box): where the C3 step's time goes, by query,
labelling and extension depth.

    python tools/sm_queries.py [reps]
"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import bench  # noqa: E402
import gamma_gen as gg  # noqa: E402
import paper_conf_icde_hu0o23_b200 as G  # noqa: E402


def main():
    reps = int(sys.argv[1]) if len(sys.argv) > 1 else 3
    n, s, d, lab = gg.config_graph("c3", seed=1)
    c = G.Context(time_kernels=True)
    g = c.load_edges(n, torch.from_numpy(s.view("int32")).cuda(), torch.from_numpy(d.view("int32")).cuda(),
                     torch.from_numpy(lab.view("int32")).cuda())
    for q, tag, nv, e, pl in bench.sm_runs():
        best = None
        for _ in range(reps):
            torch.cuda.synchronize()
            t = time.perf_counter()
            cnt = g.match(nv, e, pl)[0]
            torch.cuda.synchronize()
            ms = 1e3 * (time.perf_counter() - t)
            st = c.stats()
            cur = (ms, cnt, {k: (v["launches"], round(v["ms"], 2)) for k, v in st["classes"].items()
                             if v["launches"]}, st.get("level_entries"))
            if os.environ.get("SMQ_ALL"):
                print(f"  rep {q}/{tag}: {ms:.2f} ms kernels={cur[2]} retries={st['retries']} "
                      f"chunks={st['chunks']}", flush=True)
            if best is None or ms < best[0]:
                best = cur
        print(f"{q}/{tag}: {best[0]:.2f} ms count={best[1]} classes={best[2]} levels={best[3]}", flush=True)


if __name__ == "__main__":
    main()
