"""Pins of oracle O-3 (FPM, edge-induced patterns, MNI support; PAPER.md L113, L142,
L144, Alg. 2; readings R1-R3, R7, R8, R11).

Closed forms (stars, K_n, cycles, single labeled edges, connected-subset counts),
pure-Python brute force over edge subsets, agreement of the oracle's two
independent enumerations, and agreement with the matching-based MNI.
"""
import json
import os

import numpy as np
import pytest

import gamma_gen as gg
import brute

HERE = os.path.dirname(os.path.abspath(__file__))


def G(oracle_mod, g, labels=None):
    n, (s, d) = g
    return oracle_mod.Graph(n, s, d, labels)


def strip(res):
    return [r[:5] for r in res]


EDGE = (1, 2, (0, 0), ((0, 1),))
WEDGE = (2, 3, (0, 0, 0), ((0, 1), (0, 2)))
TRI = (3, 3, (0, 0, 0), ((0, 1), (0, 2), (1, 2)))
STAR3 = (3, 4, (0, 0, 0, 0), ((0, 1), (0, 2), (0, 3)))
PATH3 = (3, 4, (0, 0, 0, 0), ((0, 1), (0, 2), (1, 3)))


@pytest.mark.parametrize("s", [3, 4, 6])
def test_star(oracle_mod, s):
    res = {r[:4]: r[4] for r in G(oracle_mod, gg.star(s)).fpm(3, 1)}
    assert res == {EDGE: s + 1, WEDGE: 1, STAR3: 1}


@pytest.mark.parametrize("n", [4, 5, 7])
def test_complete(oracle_mod, n):
    res = {r[:4]: r[4] for r in G(oracle_mod, gg.complete(n)).fpm(3, 1)}
    assert res == {EDGE: n, WEDGE: n, TRI: n, STAR3: n, PATH3: n}


@pytest.mark.parametrize("n", [5, 6, 9])
def test_cycle(oracle_mod, n):
    res = {r[:4]: r[4] for r in G(oracle_mod, gg.cycle(n)).fpm(3, 1)}
    assert res == {EDGE: n, WEDGE: n, PATH3: n}


def test_threshold_is_inclusive(oracle_mod):
    g = G(oracle_mod, gg.star(5))
    assert {r[:4] for r in g.fpm(3, 6)} == {EDGE}          # sup >= minsup
    assert {r[:4] for r in g.fpm(3, 7)} == set()


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_labeled_single_edge(oracle_mod, seed):
    n = 40
    s, d = gg.er(n, 70, seed)
    lab = gg.labels(n, 3, seed)
    g = oracle_mod.Graph(n, s, d, lab)
    E = brute.normalise(s, d)
    res = {r[2]: r[4] for r in g.fpm(1, 1)}
    for A in range(3):
        for B in range(A, 3):
            if A != B:
                a = {x for e in E for x in e if lab[x] == A and any(lab[y] == B for y in e - {x})}
                b = {x for e in E for x in e if lab[x] == B and any(lab[y] == A for y in e - {x})}
                want = min(len(a), len(b))
            else:
                want = len({x for e in E for x in e if all(lab[y] == A for y in e)})
            assert res.get((A, B), 0) == want


@pytest.mark.parametrize("seed", [1, 2, 3, 4])
def test_connected_subset_counts(oracle_mod, seed):
    n = 30
    s, d = gg.er(n, 70, seed)
    E = brute.normalise(s, d)
    res = oracle_mod.Graph(n, s, d).fpm(3, 1)
    two, three = brute.connected_subset_counts(n, E)
    assert sum(r[5] for r in res if r[0] == 1) == len(E)
    assert sum(r[5] for r in res if r[0] == 2) == two
    assert sum(r[5] for r in res if r[0] == 3) == three


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_brute_force_python(oracle_mod, seed):
    n = 9
    s, d = gg.er(n, 16, seed)
    E = brute.normalise(s, d)
    lab = gg.labels(n, 2, seed)
    g = oracle_mod.Graph(n, s, d, lab)
    want = brute.fpm(n, E, 3, 1, lab.tolist())
    assert g.fpm(3, 1) == want


@pytest.mark.parametrize("seed", [1, 2, 3, 4, 5])
def test_two_enumerations_agree(oracle_mod, seed):
    n = 24
    s, d = gg.er(n, 50, seed)
    lab = gg.labels(n, 3, seed)
    g = oracle_mod.Graph(n, s, d, lab)
    for minsup in (1, 2, 3):
        assert g.fpm(3, minsup, "shapes") == g.fpm(3, minsup, "brute")


@pytest.mark.parametrize("seed", [1, 2])
def test_matches_matching_mni(oracle_mod, seed):
    s, d = gg.rmat(8, 1500, 0.45, 0.22, 0.22, seed)
    lab = gg.labels(256, 3, seed)
    g = oracle_mod.Graph(256, s, d, lab)
    for ne, nv, labs, edges, sup, _ in g.fpm(3, 2):
        assert g.pattern_mni(nv, list(edges), list(labs)) == sup


def test_golden_fig2c(oracle_mod):
    """tests/golden/fig2c.json: a labeled graph consistent with PAPER.md L142
    (pattern A-C-B has support 2 with instances (e1,e2) and (e4,e5))."""
    fx = json.load(open(os.path.join(HERE, "golden", "fig2c.json")))
    src = np.array([e[0] for e in fx["edges"]], np.uint32)
    dst = np.array([e[1] for e in fx["edges"]], np.uint32)
    g = oracle_mod.Graph(fx["n"], src, dst, np.array(fx["labels"], np.uint32))
    res = {(r[2], r[3]): (r[4], r[5]) for r in g.fpm(2, 1)}
    key = (tuple(fx["expect"]["labels"]), tuple(tuple(e) for e in fx["expect"]["edges"]))
    assert res[key] == (fx["expect"]["support"], fx["expect"]["instances"])


# ---- 4-edge patterns (FPM length 4) ----
def _shape(nv, edges):
    (labs, es), _ = brute.canon(nv, list(range(nv)), [tuple(e) for e in edges], [0] * nv)
    return (4, nv, labs, es)


C4 = _shape(4, [(0, 1), (1, 2), (2, 3), (3, 0)])
PAW = _shape(4, [(0, 1), (0, 2), (1, 2), (2, 3)])
STAR4 = _shape(5, [(0, 1), (0, 2), (0, 3), (0, 4)])
PATH4 = _shape(5, [(0, 1), (1, 2), (2, 3), (3, 4)])
FORK = _shape(5, [(0, 1), (1, 2), (0, 3), (0, 4)])


@pytest.mark.parametrize("n", [5, 6, 7])
def test_complete_l4(oracle_mod, n):
    """K_n: the five connected 4-edge shapes, each with MNI n; instance counts
    C4 3C(n,4), paw 3(n-3)C(n,3), 4-star n C(n-1,4), 4-path n!/(2(n-5)!),
    fork n(n-1)(n-2)C(n-3,2)."""
    from math import comb, factorial
    res = {r[:4]: (r[4], r[5]) for r in G(oracle_mod, gg.complete(n)).fpm(4, 1) if r[0] == 4}
    assert res == {C4: (n, 3 * comb(n, 4)), PAW: (n, 3 * (n - 3) * comb(n, 3)), STAR4: (n, n * comb(n - 1, 4)),
                   PATH4: (n, factorial(n) // (2 * factorial(n - 5))), FORK: (n, n * (n - 1) * (n - 2) * comb(n - 3, 2))}


@pytest.mark.parametrize("s", [4, 5, 7])
def test_star_l4(oracle_mod, s):
    from math import comb
    res = {r[:4]: (r[4], r[5]) for r in G(oracle_mod, gg.star(s)).fpm(4, 1) if r[0] == 4}
    assert res == {STAR4: (1, comb(s, 4))}


@pytest.mark.parametrize("n", [4, 6, 9])
def test_cycle_l4(oracle_mod, n):
    res = {r[:4]: (r[4], r[5]) for r in G(oracle_mod, gg.cycle(n)).fpm(4, 1) if r[0] == 4}
    assert res == ({C4: (4, 1)} if n == 4 else {PATH4: (n, n)})


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_brute_force_python_l4(oracle_mod, seed):
    n = 8
    s, d = gg.er(n, 13, seed)
    E = brute.normalise(s, d)
    lab = gg.labels(n, 2, seed)
    g = oracle_mod.Graph(n, s, d, lab)
    assert g.fpm(4, 1) == brute.fpm(n, E, 4, 1, lab.tolist())


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_two_enumerations_agree_l4(oracle_mod, seed):
    n = 20
    s, d = gg.er(n, 40, seed)
    lab = gg.labels(n, 3, seed)
    g = oracle_mod.Graph(n, s, d, lab)
    for minsup in (1, 2):
        assert g.fpm(4, minsup, "shapes") == g.fpm(4, minsup, "brute")


def test_matches_matching_mni_l4(oracle_mod):
    s, d = gg.rmat(7, 500, 0.45, 0.22, 0.22, 3)
    lab = gg.labels(128, 2, 3)
    g = oracle_mod.Graph(128, s, d, lab)
    res = [r for r in g.fpm(4, 3) if r[0] == 4]
    assert len(res) > 5
    for ne, nv, labs, edges, sup, _ in res:
        assert g.pattern_mni(nv, list(edges), list(labs)) == sup
