"""Write tests/golden/c2_full_seed1.json: oracle (O-1) k-clique counts of the bench's default
workload configs[1] (cit-Patents-shaped R-MAT scale 22, 16.6M samples, seed 1) for k = 3..6.
Calls only gamma_gen (inputs) and oracle/ (counts); the GPU path is not involved.
A few minutes on 8 host cores.

    python tools/golden_c2.py
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
    n, s, d, lab = gg.config_graph("c2", seed=1)
    o = oracle.Graph(n, s, d, lab)
    out = {"source": 'oracle og_kclique (O-1) via tools/golden_c2.py; gamma_gen.config_graph("c2", seed=1)',
           "n": n, "m": o.m, "counts": {}, "seconds": {}}
    for k in (3, 4, 5, 6):
        t = time.time()
        out["counts"][str(k)] = o.kclique(k)
        out["seconds"][str(k)] = round(time.time() - t, 1)
        print(k, out["counts"][str(k)], out["seconds"][str(k)], flush=True)
    with open(os.path.join(ROOT, "tests", "golden", "c2_full_seed1.json"), "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
