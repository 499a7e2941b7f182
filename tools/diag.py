#!/usr/bin/env python3
"""Ad-hoc timing probes run on the GPU box (one case per process, under `timeout`).

    python tools/diag.py fpm_gpu|fpm_oracle|sm <index>
"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gamma_gen as gg  # noqa: E402

PATS = [(3, [(0, 1), (1, 2), (0, 2)]), (3, [(0, 1), (1, 2)]), (4, [(0, 1), (0, 2), (0, 3)]),
        (4, [(0, 1), (0, 2), (0, 3), (1, 2), (1, 3), (2, 3)]), (5, [(0, 1), (1, 2), (2, 3), (3, 4), (4, 0)]),
        (6, [(0, 1), (1, 2), (2, 0), (2, 3), (3, 4), (4, 5), (5, 3)]), (2, [(0, 1)])]


def main():
    what = sys.argv[1]
    if what.startswith("fpm"):
        scale = int(sys.argv[2]) if len(sys.argv) > 2 else 13
        n, s, d, lab = gg.config_graph("c4", seed=1, scale=scale)
        t = time.time()
        if what == "fpm_gpu":
            import paper_conf_icde_hu0o23_b200 as G
            minsup = int(sys.argv[3]) if len(sys.argv) > 3 else 3
            budget = int(float(sys.argv[4]) * 2 ** 30) if len(sys.argv) > 4 else 0   # GiB (ncu: small pool)
            c = G.Context(time_kernels=True, hbm_budget_bytes=budget)
            g = c.load_edges(n, s, d, lab)
            for it in range(2):
                t = time.time()
                r = g.fpm(3, minsup)
                st = c.stats()
                print("gpu", len(r), f"{time.time() - t:.2f}s", st["level_entries"][:4], "retries", st["retries"],
                      "chunks", st["chunks"], "wall_ms", round(st["wall_ms"]),
                      {k: (v["launches"], round(v["ms"])) for k, v in st["classes"].items() if v["launches"]},
                      flush=True)
        else:
            import oracle
            o = oracle.Graph(n, s, d, lab)
            r = o.fpm(3, 3, pattern_cap=1 << 20)
            print("oracle", len(r), time.time() - t, flush=True)
    elif what == "kcl_phases":
        import torch
        import paper_conf_icde_hu0o23_b200 as G
        n, s, d, _ = gg.config_graph(sys.argv[2] if len(sys.argv) > 2 else "c2", seed=1)
        c = G.Context(time_kernels=True)
        sd = torch.from_numpy(s.view("int32")).cuda()
        dd = torch.from_numpy(d.view("int32")).cuda()
        for it in range(3):
            torch.cuda.synchronize()
            t = time.perf_counter()
            g = c.load_edges(n, sd, dd)
            torch.cuda.synchronize()
            line = [f"build {1e3 * (time.perf_counter() - t):.2f}ms"]
            for k in (4, 5, 6):
                t = time.perf_counter()
                cnt = g.kclique(k)
                torch.cuda.synchronize()
                st = c.stats()
                kms = sum(v["ms"] for v in st["classes"].values())
                line.append(f"k{k} wall {1e3 * (time.perf_counter() - t):.2f}ms lib {st['wall_ms']:.2f} "
                            f"kernels {kms:.2f} launches {st['total_launches']}")
            g.free()
            print(" | ".join(line), flush=True)
    elif what == "sm_phases":
        import torch
        import paper_conf_icde_hu0o23_b200 as G
        import bench
        sc = int(sys.argv[2]) if len(sys.argv) > 2 else None
        n, s, d, lab = gg.config_graph("c3", seed=1, scale=sc)
        c = G.Context(time_kernels=True)
        g = c.load_edges(n, torch.from_numpy(s.view("int32")).cuda(), torch.from_numpy(d.view("int32")).cuda(),
                         torch.from_numpy(lab.view("int32")).cuda())
        print("graph", g.info(), flush=True)
        for it in range(2):
            for (q, lname, nv, e, plab) in bench.sm_runs():
                torch.cuda.synchronize()
                t = time.perf_counter()
                cnt = g.match(nv, e, plab)
                torch.cuda.synchronize()
                st = c.stats()
                cl = {k: (v["launches"], round(v["ms"], 2)) for k, v in st["classes"].items() if v["launches"]}
                print(f"{q}/{lname} {cnt[0]} {1e3 * (time.perf_counter() - t):.1f}ms levels "
                      f"{st['level_entries'][:nv + 1]} {cl}", flush=True)
    elif what == "sm":
        i = int(sys.argv[2])
        nv, e = PATS[i]
        n, s, d, _ = gg.config_graph("c1", seed=2, scale=10)
        lab = gg.labels(n, 3, 2)
        import paper_conf_icde_hu0o23_b200 as G
        import oracle
        c = G.Context()
        g = c.load_edges(n, s, d, lab)
        for plab in (None, [(j * 7) % 3 for j in range(nv)]):
            t = time.time()
            got = g.match(nv, e, plab)
            t1 = time.time()
            want = oracle.Graph(n, s, d, lab).match(nv, e, plab)
            print("sm", i, plab, got, want[:2], f"gpu {t1 - t:.2f}s oracle {time.time() - t1:.2f}s", flush=True)


if __name__ == "__main__":
    main()
