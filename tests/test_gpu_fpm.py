"""GPU parity of gamma_fpm (Alg. 2: edge extension, canonical-code aggregation, MNI
support, sup >= minsup filtering) against the oracle (O-3), through the C ABI.
Tolerance 0 on the (pattern, support) sets."""
import numpy as np
import pytest

import gamma_gen as gg

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def G():
    import torch
    assert torch.cuda.is_available()
    import paper_conf_icde_hu0o23_b200 as G
    return G


@pytest.fixture(scope="module")
def ctx(G):
    return G.Context(device=0)


def oracle_set(o, l, minsup):
    return [r[:5] for r in o.fpm(l, minsup, pattern_cap=1 << 20)]


def test_closed_forms(ctx):
    EDGE = (1, 2, (0, 0), ((0, 1),))
    WEDGE = (2, 3, (0, 0, 0), ((0, 1), (0, 2)))
    TRI = (3, 3, (0, 0, 0), ((0, 1), (0, 2), (1, 2)))
    STAR3 = (3, 4, (0, 0, 0, 0), ((0, 1), (0, 2), (0, 3)))
    PATH3 = (3, 4, (0, 0, 0, 0), ((0, 1), (0, 2), (1, 3)))
    n, (s, d) = gg.complete(6)
    res = {r[:4]: r[4] for r in ctx.load_edges(n, s, d).fpm(3, 1)}
    assert res == {EDGE: 6, WEDGE: 6, TRI: 6, STAR3: 6, PATH3: 6}
    n, (s, d) = gg.star(5)
    res = {r[:4]: r[4] for r in ctx.load_edges(n, s, d).fpm(3, 1)}
    assert res == {EDGE: 6, WEDGE: 1, STAR3: 1}
    n, (s, d) = gg.cycle(7)
    res = {r[:4]: r[4] for r in ctx.load_edges(n, s, d).fpm(3, 1)}
    assert res == {EDGE: 7, WEDGE: 7, PATH3: 7}


@pytest.mark.parametrize("seed", [1, 2, 3])
@pytest.mark.parametrize("L", [1, 3])
def test_er_vs_oracle(ctx, oracle_mod, seed, L):
    n = 60
    s, d = gg.er(n, 150, seed)
    lab = gg.labels(n, L, seed) if L > 1 else None
    g = ctx.load_edges(n, s, d, lab)
    o = oracle_mod.Graph(n, s, d, lab)
    for minsup in (1, 2, 4):
        assert g.fpm(3, minsup) == oracle_set(o, 3, minsup), minsup


@pytest.mark.parametrize("seed", [1, 2])
def test_rmat_vs_oracle(ctx, oracle_mod, seed):
    n, s, d, lab = gg.config_graph("c4", seed=seed, scale=11)
    lab = gg.labels(n, 5, seed)
    g = ctx.load_edges(n, s, d, lab)
    o = oracle_mod.Graph(n, s, d, lab)
    for l, minsup in ((1, 1), (2, 5), (3, 20), (3, 60)):
        assert g.fpm(l, minsup) == oracle_set(o, l, minsup), (l, minsup)


def test_c4_shaped_37_labels(ctx, oracle_mod):
    """configs[3]'s generator (a,b,c = 0.40,0.25,0.25, L = 37) at scale 11."""
    n, s, d, lab = gg.config_graph("c4", seed=1, scale=11)
    g = ctx.load_edges(n, s, d, lab)
    o = oracle_mod.Graph(n, s, d, lab)
    for minsup in (3, 8):
        assert g.fpm(3, minsup) == oracle_set(o, 3, minsup)


def test_pattern_table_growth(G, oracle_mod):
    """A deliberately small HBM budget starts the pattern table tiny; it must grow
    (retries) and still give the oracle's answer."""
    n, s, d, lab = gg.config_graph("c4", seed=2, scale=10)
    c = G.Context(hbm_budget_bytes=48 << 20)
    g = c.load_edges(n, s, d, lab)
    o = oracle_mod.Graph(n, s, d, lab)
    assert g.fpm(3, 2) == oracle_set(o, 3, 2)


@pytest.mark.parametrize("budget_kb,nlab,minsup3", [(100, 5, 20), (120, 5, 20), (1024, 12, 2)])
def test_domain_pool_chunks(G, oracle_mod, budget_kb, nlab, minsup3):
    """A budget too small for one level's MNI domains: the first pass carves domains
    only for patterns whose smallest label is below a threshold, the rest are redone
    in chunks (ascending smallest label) whose passes skip every embedding with a
    smaller label; the table may have to grow too."""
    n, s, d, lab = gg.config_graph("c4", seed=1, scale=11)
    lab = gg.labels(n, nlab, 1)
    c = G.Context(hbm_budget_bytes=budget_kb << 10)
    g = c.load_edges(n, s, d, lab)
    o = oracle_mod.Graph(n, s, d, lab)
    assert g.fpm(2, 5) == oracle_set(o, 2, 5)
    assert g.fpm(3, minsup3) == oracle_set(o, 3, minsup3)
    assert c.stats()["chunks"] > 0


def test_invalid(G, ctx):
    n, (s, d) = gg.complete(4)
    g = ctx.load_edges(n, s, d)
    with pytest.raises(G.GammaError) as e:
        g.fpm(4, 1)
    assert e.value.status == -5
    with pytest.raises(G.GammaError):
        g.fpm(2, 0)
    assert g.fpm(3, 100) == []
