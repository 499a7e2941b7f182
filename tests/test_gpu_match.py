"""GPU parity of gamma_match (Alg. 1, labeled SM, non-induced and induced) against
the oracle (O-2), through the C ABI.  Tolerance 0."""
from math import comb

import numpy as np
import pytest

import gamma_gen as gg

pytestmark = pytest.mark.gpu
Q = gg.QUERIES


@pytest.fixture(scope="module")
def G():
    import torch
    assert torch.cuda.is_available()
    import paper_conf_icde_hu0o23_b200 as G
    return G


@pytest.fixture(scope="module")
def ctx(G):
    return G.Context(device=0)


def gcount(g, q, plab=None):
    nv, e = Q[q]
    return g.match(nv, e, plab)


@pytest.mark.parametrize("n", [5, 8, 12])
def test_complete(ctx, n):
    ns, (s, d) = gg.complete(n)
    g = ctx.load_edges(ns, s, d)
    assert gcount(g, "c4")[0] == 3 * comb(n, 4)
    assert gcount(g, "diamond")[0] == 6 * comb(n, 4)
    assert gcount(g, "tailed_triangle")[0] == 12 * comb(n, 4)
    assert gcount(g, "house")[0] == 60 * comb(n, 5)


def test_closed_forms(ctx):
    n, (s, d) = gg.complete_bipartite(5, 7)
    g = ctx.load_edges(n, s, d)
    assert gcount(g, "c4")[0] == comb(5, 2) * comb(7, 2)
    assert gcount(g, "house")[0] == 0
    n, (s, d) = gg.grid(7, 9)
    g = ctx.load_edges(n, s, d)
    assert gcount(g, "c4")[0] == 6 * 8
    n, (s, d) = gg.wheel(11)
    g = ctx.load_edges(n, s, d)
    assert [gcount(g, q)[0] for q in ("c4", "diamond", "tailed_triangle", "house")] == [11, 11, 121, 22]
    n, (s, d) = gg.petersen()
    assert gcount(ctx.load_edges(n, s, d), "c4")[0] == 0


@pytest.mark.parametrize("seed", [1, 2, 3])
@pytest.mark.parametrize("q", ["c4", "diamond", "tailed_triangle", "house"])
def test_rmat_vs_oracle(ctx, oracle_mod, seed, q):
    n, s, d, _ = gg.config_graph("c3", seed=seed, scale=12)
    lab = gg.labels(n, 8, seed)
    g = ctx.load_edges(n, s, d, lab)
    o = oracle_mod.Graph(n, s, d, lab)
    nv, e = Q[q]
    for plab in ([0] * nv, [i % 8 for i in range(nv)], [i % 2 for i in range(nv)]):
        got = g.match(nv, e, plab)
        want = o.match(nv, e, plab)
        assert got == (want[0], want[1]), (q, plab)


@pytest.mark.parametrize("q", ["c4", "diamond", "tailed_triangle", "house"])
def test_er_unlabeled_vs_oracle(ctx, oracle_mod, q):
    n = 1500
    s, d = gg.er(n, 9000, 4)
    g = ctx.load_edges(n, s, d)
    o = oracle_mod.Graph(n, s, d)
    nv, e = Q[q]
    assert g.match(nv, e)[0] == o.match(nv, e)[0]


def test_unstaged_and_budget_paths(G, oracle_mod):
    n, s, d, _ = gg.config_graph("c3", seed=5, scale=11)
    lab = gg.labels(n, 2, 5)
    o = oracle_mod.Graph(n, s, d, lab)
    for c in (G.Context(flags=0x8), G.Context(hbm_budget_bytes=2 << 20)):
        g = c.load_edges(n, s, d, lab)
        for q in ("c4", "house"):
            nv, e = Q[q]
            plab = [i % 2 for i in range(nv)]
            assert g.match(nv, e, plab)[0] == o.match(nv, e, plab)[0]


def test_more_patterns(ctx, oracle_mod):
    """Triangle, path, star, K4, 5-cycle, 6-vertex patterns and a single vertex."""
    pats = [(3, [(0, 1), (1, 2), (0, 2)]), (3, [(0, 1), (1, 2)]), (4, [(0, 1), (0, 2), (0, 3)]),
            (4, [(0, 1), (0, 2), (0, 3), (1, 2), (1, 3), (2, 3)]), (5, [(0, 1), (1, 2), (2, 3), (3, 4), (4, 0)]),
            (6, [(0, 1), (1, 2), (2, 0), (2, 3), (3, 4), (4, 5), (5, 3)]), (2, [(0, 1)])]
    # ER (no hubs) so that the unlabeled 5- and 6-vertex patterns stay small
    n = 600
    s, d = gg.er(n, 2400, 6)
    lab = gg.labels(n, 3, 2)
    g = ctx.load_edges(n, s, d, lab)
    o = oracle_mod.Graph(n, s, d, lab)
    for nv, e in pats:
        assert g.match(nv, e)[0] == o.match(nv, e)[0], (nv, e)
        plab = [(i * 7) % 3 for i in range(nv)]
        assert g.match(nv, e, plab)[0] == o.match(nv, e, plab)[0], (nv, e, plab)
    assert g.match(1, [], [1])[0] == int((lab == 1).sum())


@pytest.mark.parametrize("deg", [900, 1500])
def test_hub_staged_prefix_list(ctx, oracle_mod, deg):
    """A hub whose neighbour list fits the shared-memory L_m but not the 512-entry
    child-run staging (900: long runs go straight to the level), or exceeds the
    shared L_m (1500: L_m goes to the warp's global scratch slice)."""
    rng = np.random.default_rng(11)
    n = 1800
    hub = [(0, i) for i in range(1, deg + 1)]
    extra = [tuple(x) for x in rng.integers(1, n, size=(5000, 2))]
    e = np.array(hub + extra, dtype=np.uint32)
    s, d = e[:, 0].copy(), e[:, 1].copy()
    g = ctx.load_edges(n, s, d)
    o = oracle_mod.Graph(n, s, d)
    for q in ("diamond", "house", "tailed_triangle", "c4"):
        nv, pe = Q[q]
        assert g.match(nv, pe)[0] == o.match(nv, pe)[0], q


def test_simulated_ranks(G, oracle_mod):
    n, s, d, _ = gg.config_graph("c3", seed=2, scale=11)
    lab = gg.labels(n, 4, 2)
    nv, e = Q["diamond"]
    plab = [0, 1, 1, 0]
    want = oracle_mod.Graph(n, s, d, lab).match(nv, e, plab)[0]
    tot = 0
    for r in range(3):
        c = G.Context(rank=r, world=3, reduce=False)
        tot += c.load_edges(n, s, d, lab).match(nv, e, plab)[0]
    assert tot == want


def test_invalid_patterns(G, ctx):
    n, (s, d) = gg.complete(5)
    g = ctx.load_edges(n, s, d)
    with pytest.raises(G.GammaError):
        g.match(4, [(0, 1), (2, 3)])          # disconnected
    assert g.match(3, [(0, 1), (1, 2)], induced=True)[0] == 0   # K5 has no induced path
    with pytest.raises(G.GammaError):
        g.match(9, [(i, i + 1) for i in range(8)])


# ---- induced SM (R17) --------------------------------
K4 = (4, [(0, 1), (0, 2), (0, 3), (1, 2), (1, 3), (2, 3)])
IPATS = [Q["c4"], Q["diamond"], Q["tailed_triangle"], Q["house"], K4, (3, [(0, 1), (1, 2)]),
         (4, [(0, 1), (1, 2), (2, 3)]), (4, [(0, 1), (0, 2), (0, 3)]),
         (5, [(0, 1), (1, 2), (2, 3), (3, 4), (4, 0)])]


def test_induced_closed_forms(ctx):
    n, (s, d) = gg.complete(9)
    g = ctx.load_edges(n, s, d)
    assert [g.match(*Q[q], induced=True)[0] for q in ("c4", "diamond", "tailed_triangle", "house")] == [0] * 4
    assert g.match(*K4, induced=True)[0] == comb(9, 4)
    n, (s, d) = gg.wheel(11)
    g = ctx.load_edges(n, s, d)
    assert [g.match(*Q[q], induced=True)[0] for q in ("c4", "diamond", "tailed_triangle")] == [0, 11, 11 * 7]
    n, (s, d) = gg.complete_bipartite(5, 7)
    assert ctx.load_edges(n, s, d).match(*Q["c4"], induced=True)[0] == comb(5, 2) * comb(7, 2)


@pytest.mark.parametrize("seed", [1, 2])
def test_induced_rmat_vs_oracle(ctx, oracle_mod, seed):
    n, s, d, _ = gg.config_graph("c3", seed=seed, scale=12)
    lab = gg.labels(n, 8, seed)
    g = ctx.load_edges(n, s, d, lab)
    o = oracle_mod.Graph(n, s, d, lab)
    for nv, e in IPATS[:5]:
        for plab in ([0] * nv, [i % 2 for i in range(nv)], [i % 8 for i in range(nv)]):
            got = g.match(nv, e, plab, induced=True)
            want = o.match(nv, e, plab, induced=True)
            assert got == (want[0], want[1]), (nv, e, plab)


def test_induced_er_paths(G, ctx, oracle_mod):
    """Unlabeled ER: every pattern above, default / unstaged (flag 0x8) / small budget."""
    n = 700
    s, d = gg.er(n, 4200, 8)
    o = oracle_mod.Graph(n, s, d)
    for c in (ctx, G.Context(flags=0x8), G.Context(hbm_budget_bytes=2 << 20)):
        g = c.load_edges(n, s, d)
        for nv, e in IPATS:
            assert g.match(nv, e, induced=True)[0] == o.match(nv, e, induced=True)[0], (nv, e)


@pytest.mark.parametrize("deg", [900, 1500])
def test_induced_hub(ctx, oracle_mod, deg):
    rng = np.random.default_rng(12)
    n = 1800
    hub = [(0, i) for i in range(1, deg + 1)]
    extra = [tuple(x) for x in rng.integers(1, n, size=(5000, 2))]
    e = np.array(hub + extra, dtype=np.uint32)
    s, d = e[:, 0].copy(), e[:, 1].copy()
    g = ctx.load_edges(n, s, d)
    o = oracle_mod.Graph(n, s, d)
    for nv, pe in IPATS[:5]:
        assert g.match(nv, pe, induced=True)[0] == o.match(nv, pe, induced=True)[0], (nv, pe)


@pytest.mark.slow
def test_c3_full_size(ctx):
    """configs[2] at full size (LiveJournal-shaped R-MAT scale 23, L = 8, seed 1), in the
    bench's configuration: the four queries x two labelings, non-induced and induced,
    against the oracle's counts stored by tools/golden_c3.py (oracle-only script)."""
    import json
    import os
    gold = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "c3_full_seed1.json")))
    n, s, d, lab = gg.config_graph("c3", seed=1)
    g = ctx.load_edges(n, s, d, lab)
    assert g.info()["m"] == gold["m"]
    batch = []
    for key, want in gold["counts"].items():
        parts = key.split("/")
        q, lname, ind = parts[0], parts[1], len(parts) > 2
        nv, e = Q[q]
        plab = [0] * nv if lname == "all0" else [i % 8 for i in range(nv)]
        assert g.match(nv, e, plab, induced=ind)[0] == want, key
        batch.append(((nv, e, plab, ind), want))
    # the bench's configuration: all runs in one gamma_match_batch (concurrent chains)
    assert [c for c, _ in g.match_many([b[0] for b in batch])] == [b[1] for b in batch]


def test_motifs(ctx, oracle_mod):
    """Motif counts (induced, every connected 3-/4-vertex graph) against the oracle, plus
    the identities sum_v C(d_v, 2) = iWedge + 3 T and sum over 4-motifs of
    (#spanning-subgraph copies) = the non-induced counts of path / star."""
    import paper_conf_icde_hu0o23_b200 as G
    n, s, d, _ = gg.config_graph("c3", seed=3, scale=11)
    g = ctx.load_edges(n, s, d)
    o = oracle_mod.Graph(n, s, d)
    for k in (3, 4):
        got = g.motifs(k)
        for name, e in G.MOTIFS[k].items():
            assert got[name] == o.match(k, e, induced=True)[0], (k, name)
    m3 = g.motifs(3)
    rp, _ = g.csr()
    deg = np.diff(np.asarray(rp, dtype=np.int64))
    assert m3["wedge"] + 3 * m3["triangle"] == int((deg * (deg - 1) // 2).sum())
    m4 = g.motifs(4)
    # non-induced 3-stars: each induced star 1, tailed triangle 1, diamond 2, K4 4
    assert m4["star"] + m4["tailed_triangle"] + 2 * m4["diamond"] + 4 * m4["k4"] == \
        int((deg * (deg - 1) * (deg - 2) // 6).sum())


_SUB = r"""
import json, sys
sys.path.insert(0, sys.argv[1])
import gamma_gen as gg
import paper_conf_icde_hu0o23_b200 as G
n, s, d, lab = gg.config_graph("c3", seed=2, scale=12)
c = G.Context(device=0)
g, g0 = c.load_edges(n, s, d, lab), c.load_edges(n, s, d)
out = {}
for q in ("c4", "diamond", "tailed_triangle", "house"):
    nv, e = gg.QUERIES[q]
    out[q + "/0"] = g0.match(nv, e)[0]
    out[q + "/m"] = g.match(nv, e, [i % 8 for i in range(nv)])[0]
print(json.dumps(out))
"""


@pytest.mark.parametrize("ratio", ["0", "1", "8"])
def test_last_level_long_child_probe(oracle_mod, ratio):
    """Last-level counting over a long staged L_m: hub children (|N(c)| > ratio * |L_m|)
    are probed from L_m's side (binary search into N(c)) instead of streamed; ratio 0
    turns the probe off, 1 sends nearly every child through it.  Same counts as the
    oracle either way (each process reads GAMMA_SM_LONGRATIO once); unlabeled graph
    (hub-heavy L_m and children) and 8 labels."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, GAMMA_SM_LONGRATIO=ratio)
    r = subprocess.run([sys.executable, "-c", _SUB, root], env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    got = json.loads(r.stdout.strip().splitlines()[-1])
    n, s, d, lab = gg.config_graph("c3", seed=2, scale=12)
    o, o0 = oracle_mod.Graph(n, s, d, lab), oracle_mod.Graph(n, s, d)
    for q in ("c4", "diamond", "tailed_triangle", "house"):
        nv, e = Q[q]
        assert got[q + "/0"] == o0.match(nv, e)[0], (ratio, q, "unlabeled")
        assert got[q + "/m"] == o.match(nv, e, [i % 8 for i in range(nv)])[0], (ratio, q, "imod8")


@pytest.mark.parametrize("q", ["c4", "diamond", "tailed_triangle", "house"])
def test_level_sizes_vs_oracle(ctx, oracle_mod, q):
    """Every ET level the GPU builds, not only the final count: the number of partial
    matches at each depth (stats level_entries) equals the oracle's O-2b level counts in
    the same matching order and constraints (oracle planner plan_r10_r16, pinned in
    tests/test_oracle_match_levels.py)."""
    nv, e = Q[q]
    n, s, d, lab = gg.config_graph("c3", seed=3, scale=12)
    g = ctx.load_edges(n, s, d, lab)
    o = oracle_mod.Graph(n, s, d, lab)
    for plab in ([0] * nv, [i % 8 for i in range(nv)], [i % 2 for i in range(nv)]):
        N, _, _ = o.match_levels(nv, e, plab)
        assert g.match(nv, e, plab)[0] == N[nv]
        assert ctx.stats()["level_entries"][1:nv + 1] == N[1:], plab


@pytest.mark.parametrize("q", ["c4", "diamond", "tailed_triangle", "house"])
@pytest.mark.parametrize("induced", [False, True])
def test_edge_join_vs_oracle(G, oracle_mod, q, induced):
    """SM by edge extension (binary join, GAMMA_FLAG_SM_EDGE_JOIN):
    one pattern edge per step, non-tree edges and anti-edges as separate filter passes --
    the same counts as the oracle, and the same final level as the vertex extension."""
    nv, e = Q[q]
    n, s, d, lab = gg.config_graph("c3", seed=2, scale=11)
    c = G.Context(flags=G._native.GAMMA_FLAG_SM_EDGE_JOIN)
    g = c.load_edges(n, s, d, lab)
    o = oracle_mod.Graph(n, s, d, lab)
    for plab in (None, [0] * nv, [i % 3 for i in range(nv)]):
        assert g.match(nv, e, plab, induced=induced) == o.match(nv, e, plab, induced=induced)[:2], plab


def test_edge_join_small_buffer(G, oracle_mod):
    """Row ranges halve at any step whose output overflows its row buffer (2 MiB budget)."""
    n, s, d, lab = gg.config_graph("c3", seed=1, scale=12)
    c = G.Context(flags=G._native.GAMMA_FLAG_SM_EDGE_JOIN, hbm_budget_bytes=2 << 20)
    g = c.load_edges(n, s, d, lab)
    o = oracle_mod.Graph(n, s, d, lab)
    nv, e = Q["house"]
    assert g.match(nv, e)[0] == o.match(nv, e)[0]
    assert c.stats()["chunks"] > 1


def test_match_many(G, oracle_mod):
    """gamma_match_batch: the same counts and mappings as one gamma_match per query,
    in order, with tables small enough that some chains overflow and rerun alone."""
    n, s, d, lab = gg.config_graph("c3", seed=3, scale=12)
    o = oracle_mod.Graph(n, s, d, lab)
    qs = []
    for q in ("c4", "diamond", "tailed_triangle", "house"):
        nv, e = Q[q]
        qs += [(nv, e, [0] * nv, False), (nv, e, [i % 8 for i in range(nv)], False), (nv, e, None, True)]
    want = [o.match(nv, e, pl, induced=ind)[:2] for nv, e, pl, ind in qs]
    for c in (G.Context(), G.Context(hbm_budget_bytes=16 << 20)):
        g = c.load_edges(n, s, d, lab)
        assert g.match_many(qs) == want
        assert g.match_many([]) == []
