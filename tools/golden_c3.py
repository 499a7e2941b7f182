"""Write tests/golden/c3_full_seed1.json: oracle (O-2) counts of the bench's C3 workload
(configs[2], full size, seed 1) for the four queries x two labelings, non-induced
and induced.  Calls only gamma_gen (inputs) and oracle/ (counts); the GPU path is not
involved.  ~7 min on 8 host cores.

    python tools/golden_c3.py
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import gamma_gen as gg  # noqa: E402
import oracle  # noqa: E402


def main():
    n, s, d, lab = gg.config_graph("c3", seed=1)
    o = oracle.Graph(n, s, d, lab)
    out = {"source": "oracle og_match (O-2) via tools/golden_c3.py; gamma_gen.config_graph('c3', seed=1)",
           "n": n, "m": o.m, "counts": {}}
    for q in ("c4", "diamond", "tailed_triangle", "house"):
        nv, e = gg.QUERIES[q]
        for lname, plab in (("all0", [0] * nv), ("imod8", [i % 8 for i in range(nv)])):
            for ind in (False, True):
                t = time.time()
                c = o.match(nv, e, plab, induced=ind)[0]
                key = f"{q}/{lname}" + ("/induced" if ind else "")
                out["counts"][key] = c
                print(key, c, f"{time.time() - t:.1f}s", flush=True)
    with open(os.path.join(ROOT, "tests", "golden", "c3_full_seed1.json"), "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
