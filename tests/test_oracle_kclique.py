"""Pins of oracle O-0 (graph normalisation) and O-1 (k-clique counting).

Each pin is fixed by mathematics, not by the oracle: closed forms (K_n, Turan,
wheels, cycles, grids, Petersen), brute force over all k-subsets, additivity over
disjoint unions and independence of the orientation order.  (PAPER.md L15, L269,
L449 name kCL; the count is the plain definition -- DESIGN.md reading R9.)
"""
from math import comb

import numpy as np
import pytest

import gamma_gen as gg
import brute


def G(oracle_mod, g, labels=None):
    n, (s, d) = g
    return oracle_mod.Graph(n, s, d, labels)


def test_normalisation_matches_set_definition(oracle_mod):
    src = np.array([0, 1, 1, 2, 2, 3, 3, 4, 0, 5], np.uint32)
    dst = np.array([1, 0, 1, 3, 3, 2, 4, 4, 5, 0], np.uint32)
    g = oracle_mod.Graph(6, src, dst)
    E = brute.normalise(src, dst)
    assert g.m == len(E)
    off, adj = g.csr()
    got = set()
    for v in range(6):
        lst = adj[off[v]:off[v + 1]].tolist()
        assert lst == sorted(set(lst)), "sorted, no duplicates"
        assert v not in lst, "no self-loops"
        got |= {frozenset((v, u)) for u in lst}
    assert got == E
    # symmetric
    for v in range(6):
        for u in adj[off[v]:off[v + 1]]:
            assert v in adj[off[u]:off[u + 1]]


@pytest.mark.parametrize("n,m", [(1 << 18, 2_000_000), ((1 << 18) + 77, 600_000)])
def test_normalisation_bucketed_path(oracle_mod, n, m):
    """O-0 at n > 65,536, where og_build sorts per bucket of the smaller endpoint across
    threads: the CSR equals the set definition computed by numpy
    (symmetrise, drop self-loops, dedup, ascending lists) on raw samples with planted
    duplicates (both directions), self-loops and a hub."""
    rng = np.random.default_rng(n)
    s = rng.integers(0, n, m, dtype=np.uint32)
    d = rng.integers(0, n, m, dtype=np.uint32)
    k = m // 10
    s[:k], d[:k] = d[k:2 * k], s[k:2 * k]          # reversed duplicates
    d[2 * k:2 * k + 1000] = s[2 * k:2 * k + 1000]   # self-loops
    s[3 * k:3 * k + 50_000] = 12345                 # a hub
    g = oracle_mod.Graph(n, s, d)
    lo, hi = np.minimum(s, d).astype(np.uint64), np.maximum(s, d).astype(np.uint64)
    keep = lo != hi
    und = np.unique((lo[keep] << np.uint64(32)) | hi[keep])
    a, b = (und >> np.uint64(32)).astype(np.int64), (und & np.uint64(0xFFFFFFFF)).astype(np.int64)
    assert g.m == und.size
    src = np.concatenate([a, b])
    dst = np.concatenate([b, a])
    order = np.lexsort((dst, src))
    want_off = np.zeros(n + 1, np.uint64)
    np.cumsum(np.bincount(src, minlength=n), out=want_off[1:])
    off, adj = g.csr()
    assert np.array_equal(off, want_off)
    assert np.array_equal(adj.astype(np.int64), dst[order])


@pytest.mark.parametrize("n", range(1, 11))
def test_complete_graph(oracle_mod, n):
    g = G(oracle_mod, gg.complete(n))
    for k in range(1, n + 2):
        assert g.kclique(k) == comb(n, k)


@pytest.mark.parametrize("n,r", [(6, 2), (6, 3), (8, 4), (9, 3), (12, 4), (10, 5)])
def test_turan(oracle_mod, n, r):
    g = G(oracle_mod, gg.turan(n, r))
    for k in range(2, r + 2):
        assert g.kclique(k) == comb(r, k) * (n // r) ** k


@pytest.mark.parametrize("n", [4, 5, 6, 9, 20])
def test_wheel(oracle_mod, n):
    g = G(oracle_mod, gg.wheel(n))
    assert g.kclique(3) == n
    assert g.kclique(4) == 0


def test_triangle_free(oracle_mod):
    assert G(oracle_mod, gg.cycle(3)).kclique(3) == 1
    for n in (4, 5, 7, 30):
        assert G(oracle_mod, gg.cycle(n)).kclique(3) == 0
    assert G(oracle_mod, gg.grid(5, 7)).kclique(3) == 0
    assert G(oracle_mod, gg.petersen()).kclique(3) == 0
    assert G(oracle_mod, gg.complete_bipartite(4, 5)).kclique(3) == 0


def test_k1_k2(oracle_mod):
    n = 50
    s, d = gg.er(n, 200, 3)
    g = oracle_mod.Graph(n, s, d)
    assert g.kclique(1) == 50
    assert g.kclique(2) == len(brute.normalise(s, d))


def test_empty(oracle_mod):
    g = oracle_mod.Graph(5, np.zeros(0, np.uint32), np.zeros(0, np.uint32))
    assert g.m == 0 and g.kclique(3) == 0 and g.kclique(1) == 5


@pytest.mark.parametrize("seed", [1, 2, 3, 4, 5])
def test_brute_force_random(oracle_mod, seed):
    n = 14
    s, d = gg.er(n, 60, seed)
    E = brute.normalise(s, d)
    g = oracle_mod.Graph(n, s, d)
    for k in range(3, 7):
        assert g.kclique(k) == brute.kcliques(n, E, k)


def test_additivity_disjoint_union(oracle_mod):
    parts = [gg.complete(6), gg.wheel(7), gg.turan(8, 4)]
    u = G(oracle_mod, gg.disjoint_union(*parts))
    for k in (3, 4):
        assert u.kclique(k) == sum(G(oracle_mod, p).kclique(k) for p in parts)


@pytest.mark.parametrize("seed", [1, 2])
def test_order_independence_rmat(oracle_mod, seed):
    s, d = gg.rmat(10, 12000, 0.57, 0.19, 0.19, seed)
    g = oracle_mod.Graph(1 << 10, s, d)
    for k in (3, 4, 5):
        assert g.kclique(k, "degree") == g.kclique(k, "id")


def test_roots_partition_total(oracle_mod):
    s, d = gg.rmat(9, 5000, 0.57, 0.19, 0.19, 7)
    g = oracle_mod.Graph(1 << 9, s, d)
    roots = np.arange(1 << 9, dtype=np.uint32)
    for k in (3, 4):
        assert int(g.kclique_roots(k, roots).sum()) == g.kclique(k)


def test_threads_invariance(oracle_mod):
    n, s, d, _ = gg.config_graph("c1", scale=10)
    g = oracle_mod.Graph(n, s, d)
    assert g.kclique(4, threads=1) == g.kclique(4, threads=0)


# ---- O-1b: ET level statistics (SURVEY §8(d) algorithmic bytes) ----
@pytest.mark.parametrize("n", [1, 2, 5, 9])
def test_levels_complete_graph(oracle_mod, n):
    """K_n: the vertex of rank i has d+ = n-1-i and ends C(i, t-1) t-cliques, so
    S[t] = sum_i C(i, t-1) C(n-1-i, 1) = C(n, t+1) (Vandermonde); N[t] = C(n, t)."""
    g = G(oracle_mod, gg.complete(n))
    k = n + 1
    N, S = g.kclique_levels(k)
    for t in range(1, k + 1):
        assert N[t] == comb(n, t)
        assert S[t] == comb(n, t + 1)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_levels_brute_force(oracle_mod, seed):
    """Brute force over all t-subsets of a small random graph: rank (deg, id), last
    vertex = max rank, d+ counted from the edge set."""
    import itertools
    n = 14
    s, d = gg.er(n, 40, seed)
    E = brute.normalise(s, d)
    deg = [sum(1 for e in E if v in e) for v in range(n)]
    rank = lambda v: (deg[v], v)  # noqa: E731
    dplus = [sum(1 for e in E if v in e and rank(next(iter(e - {v}))) > rank(v)) for v in range(n)]
    g = oracle_mod.Graph(n, s, d)
    k = 5
    N, S = g.kclique_levels(k)
    for t in range(1, k + 1):
        bn = bs = 0
        for C in itertools.combinations(range(n), t):
            if all(frozenset(p) in E for p in itertools.combinations(C, 2)):
                bn += 1
                bs += dplus[max(C, key=rank)]
        assert (N[t], S[t]) == (bn, bs), t
