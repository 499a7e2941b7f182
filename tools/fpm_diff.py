"""Diff GPU FPM records against the oracle on a scaled C4 graph (debugging aid)."""
import sys, os
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import gamma_gen as gg, oracle
import paper_conf_icde_hu0o23_b200 as G


def oracle_set(o, l, minsup):
    return [r[:5] for r in o.fpm(l, minsup, pattern_cap=1 << 20)]


n, s, d, lab = gg.config_graph("c4", seed=1, scale=11)
lab = gg.labels(n, 5, 1)
ctx = G.Context()
g = ctx.load_edges(n, s, d, lab)
o = oracle.Graph(n, s, d, lab)
for l, ms in ((3, 1), (3, 20)):
    got = g.fpm(l, ms); want = oracle_set(o, l, ms)
    gd = {r[:4]: r[4] for r in got}; wd = {r[:4]: r[4] for r in want}
    diff = [(k, gd.get(k), wd.get(k)) for k in set(gd) | set(wd) if gd.get(k) != wd.get(k)]
    print(l, ms, len(got), len(want), "ndiff", len(diff))
    for x in sorted(diff, key=str)[:12]: print("  ", x)
