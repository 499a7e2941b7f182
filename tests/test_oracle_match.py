"""Pins of oracle O-2 (labeled, non-induced subgraph matching; Alg. 1
L174-182; readings R4-R6, R10).

Closed forms on K_n, K_{a,b}, grids, wheels, Petersen, C_4; |Aut_L| against brute
force; the label-sum identity; brute force over edge subsets on tiny graphs.
"""
from math import comb

import numpy as np
import pytest

import gamma_gen as gg
import brute

Q = gg.QUERIES


def G(oracle_mod, g, labels=None):
    n, (s, d) = g
    return oracle_mod.Graph(n, s, d, labels)


def count(g, name, plab=None):
    nv, e = Q[name]
    return g.match(nv, e, plab)[0]


@pytest.mark.parametrize("n", [4, 5, 6, 8])
def test_complete(oracle_mod, n):
    g = G(oracle_mod, gg.complete(n))
    assert count(g, "c4") == 3 * comb(n, 4)
    assert count(g, "diamond") == 6 * comb(n, 4)
    assert count(g, "tailed_triangle") == 12 * comb(n, 4)
    assert count(g, "house") == 60 * comb(n, 5)


@pytest.mark.parametrize("a,b", [(2, 2), (3, 4), (5, 3)])
def test_complete_bipartite(oracle_mod, a, b):
    g = G(oracle_mod, gg.complete_bipartite(a, b))
    assert count(g, "c4") == comb(a, 2) * comb(b, 2)
    for q in ("diamond", "tailed_triangle", "house"):
        assert count(g, q) == 0


@pytest.mark.parametrize("a,b", [(2, 2), (3, 5), (6, 4)])
def test_grid(oracle_mod, a, b):
    g = G(oracle_mod, gg.grid(a, b))
    assert count(g, "c4") == (a - 1) * (b - 1)
    for q in ("diamond", "tailed_triangle", "house"):
        assert count(g, q) == 0


@pytest.mark.parametrize("n", [5, 6, 9])
def test_wheel(oracle_mod, n):
    g = G(oracle_mod, gg.wheel(n))
    assert count(g, "c4") == n
    assert count(g, "diamond") == n
    assert count(g, "tailed_triangle") == n * n
    assert count(g, "house") == 2 * n


def test_petersen_c4(oracle_mod):
    assert count(G(oracle_mod, gg.petersen()), "c4") == 0
    assert count(G(oracle_mod, gg.cycle(4)), "c4") == 1


def test_aut():
    assert [brute.aut(*Q[q]) for q in ("c4", "diamond", "tailed_triangle", "house")] == [8, 4, 2, 2]
    assert brute.aut(*Q["c4"], plab=[0, 1, 0, 1]) == 4


def test_oracle_aut_and_mappings(oracle_mod):
    g = G(oracle_mod, gg.complete(6))
    for q, a in (("c4", 8), ("diamond", 4), ("tailed_triangle", 2), ("house", 2)):
        nv, e = Q[q]
        c, mp, aut = g.match(nv, e)
        assert aut == a and mp == c * a
    nv, e = Q["c4"]
    assert g.match(nv, e, [0, 1, 0, 1])[2] == 4


def test_single_vertex_pattern(oracle_mod):
    lab = np.array([0, 1, 1, 2, 1], np.uint32)
    g = G(oracle_mod, gg.path(5), lab)
    assert g.match(1, [], [1])[0] == 3
    assert g.match(1, [])[0] == 5


@pytest.mark.parametrize("q", ["c4", "diamond", "tailed_triangle", "house"])
def test_label_sum_identity(oracle_mod, q):
    import itertools
    nv, e = Q[q]
    n = 12
    s, d = gg.er(n, 40, 11)
    lab = gg.labels(n, 2, 5)
    g = oracle_mod.Graph(n, s, d, lab)
    total = sum(g.match(nv, e, list(pl))[1] for pl in itertools.product(range(2), repeat=nv))
    g0 = oracle_mod.Graph(n, s, d)
    assert total == g0.match(nv, e)[1]


@pytest.mark.parametrize("seed", [1, 2, 3])
@pytest.mark.parametrize("q", ["c4", "diamond", "tailed_triangle", "house"])
def test_brute_force_subsets(oracle_mod, seed, q):
    nv, e = Q[q]
    n = 9
    s, d = gg.er(n, 22, seed)
    E = brute.normalise(s, d)
    lab = gg.labels(n, 2, seed).tolist()
    g = oracle_mod.Graph(n, s, d, np.array(lab, np.uint32))
    assert g.match(nv, e)[0] == brute.distinct_subgraphs(n, E, nv, e)
    plab = [i % 2 for i in range(nv)]
    assert g.match(nv, e, plab)[0] == brute.distinct_subgraphs(n, E, nv, e, plab, lab)
    assert g.match(nv, e, plab)[1] == brute.mappings(n, E, nv, e, plab, lab)


@pytest.mark.parametrize("q", ["c4", "house"])
def test_match_roots_partition(oracle_mod, q):
    nv, e = Q[q]
    n = 64
    s, d = gg.er(n, 300, 9)
    lab = gg.labels(n, 2, 9)
    g = oracle_mod.Graph(n, s, d, lab)
    plab = [i % 2 for i in range(nv)]
    per = g.match_roots(nv, e, np.arange(n, dtype=np.uint32), plab)
    assert int(per.sum()) == g.match(nv, e, plab)[1]


def test_disconnected_pattern_rejected(oracle_mod):
    g = G(oracle_mod, gg.complete(5))
    with pytest.raises(ValueError):
        g.match(4, [(0, 1), (2, 3)])


# ---- induced matching (anti-edge checks) ----------
K4 = (4, [(0, 1), (0, 2), (0, 3), (1, 2), (1, 3), (2, 3)])


def icount(g, name, plab=None):
    nv, e = K4 if name == "k4" else Q[name]
    return g.match(nv, e, plab, induced=True)[0]


@pytest.mark.parametrize("n", [4, 5, 7])
def test_induced_complete(oracle_mod, n):
    g = G(oracle_mod, gg.complete(n))
    for q in ("c4", "diamond", "tailed_triangle", "house"):
        assert icount(g, q) == 0
    assert icount(g, "k4") == comb(n, 4)


@pytest.mark.parametrize("a,b", [(2, 2), (3, 4)])
def test_induced_bipartite_grid(oracle_mod, a, b):
    assert icount(G(oracle_mod, gg.complete_bipartite(a, b)), "c4") == comb(a, 2) * comb(b, 2)
    assert icount(G(oracle_mod, gg.grid(a + 1, b + 1)), "c4") == a * b


@pytest.mark.parametrize("n", [5, 6, 9])
def test_induced_wheel(oracle_mod, n):
    """W_n (n >= 5): every C4 has a chord through the hub; the diamonds hub,i-1,i,i+1
    are induced (i-1, i+1 not adjacent for n >= 5); an induced tailed triangle is a
    triangle hub,i,i+1 with the tail j hanging off the hub, j not in {i-1..i+2}:
    n(n-4)."""
    g = G(oracle_mod, gg.wheel(n))
    assert icount(g, "c4") == 0
    assert icount(g, "tailed_triangle") == n * (n - 4)
    assert icount(g, "diamond") == n


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_induced_supergraph_identities(oracle_mod, seed):
    """Non-induced count = sum over the 4-vertex supergraphs H of P of
    (#copies of P in H) x induced(H): C4 = iC4 + iDiamond + 3 iK4,
    tailed triangle = iTT + 4 iDiamond + 12 iK4, diamond = iDiamond + 6 iK4."""
    n = 64
    s, d = gg.er(n, 700, seed)
    g = oracle_mod.Graph(n, s, d)
    ic4, idi, itt, ik4 = (icount(g, q) for q in ("c4", "diamond", "tailed_triangle", "k4"))
    assert ik4 == g.kclique(4) and ik4 > 0 and idi > 0
    assert count(g, "c4") == ic4 + idi + 3 * ik4
    assert count(g, "tailed_triangle") == itt + 4 * idi + 12 * ik4
    assert count(g, "diamond") == idi + 6 * ik4


@pytest.mark.parametrize("seed", [1, 2])
@pytest.mark.parametrize("q", ["c4", "diamond", "tailed_triangle", "house"])
def test_induced_brute_force(oracle_mod, seed, q):
    n = 11
    s, d = gg.er(n, 30, seed)
    E = brute.normalise(s, d)
    lab = [int(x) for x in gg.labels(n, 2, seed)]
    nv, e = Q[q]
    g0 = oracle_mod.Graph(n, s, d)
    g = oracle_mod.Graph(n, s, d, lab)
    assert g0.match(nv, e, induced=True)[0] == brute.induced_subgraphs(n, E, nv, e)
    plab = [i % 2 for i in range(nv)]
    assert g.match(nv, e, plab, induced=True)[0] == brute.induced_subgraphs(n, E, nv, e, plab, lab)


@pytest.mark.parametrize("seed", [4, 5])
def test_induced_degree_identities(oracle_mod, seed):
    """sum_v C(d,2) = iWedge + 3T; sum_v C(d,3) = iStar + iTT + 2 iDiamond + 4 iK4
    (the 3-stars inside each connected 4-vertex graph)."""
    n = 80
    s, d = gg.er(n, 600, seed)
    E = brute.normalise(s, d)
    deg = [0] * n
    for e in E:
        for x in e:
            deg[x] += 1
    g = oracle_mod.Graph(n, s, d)
    iw = g.match(3, [(0, 1), (1, 2)], induced=True)[0]
    t = g.kclique(3)
    assert iw + 3 * t == sum(comb(x, 2) for x in deg)
    ist = g.match(4, [(0, 1), (0, 2), (0, 3)], induced=True)[0]
    assert ist + icount(g, "tailed_triangle") + 2 * icount(g, "diamond") + 4 * icount(g, "k4") == \
        sum(comb(x, 3) for x in deg)
