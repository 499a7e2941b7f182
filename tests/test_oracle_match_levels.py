"""Pins of oracle O-2b (og_match_levels: per-level SM statistics in a given matching
order with given order constraints, SURVEY.md §8(d) algorithmic bytes) and of the
oracle's own planner (plan_r10_r16: DESIGN.md readings R10, R16).

Fixed by things other than the function itself: brute force over injective partial
maps on small graphs (every level count and byte sum), the final level equals the
distinct-subgraph count by brute force (the stabilizer chain keeps exactly one mapping
per automorphism class), the K_n closed form of the C4 query, and the planner's
order/constraints equal those of the library's independently written host planner
(gamma_pattern_plan; host code, no GPU)."""
import itertools
from math import comb

import numpy as np
import pytest

import brute
import gamma_gen as gg
import oracle as O

Q = gg.QUERIES


def brute_levels(n, E, nv, edges, plab, glab, plan):
    """Every injective map of positions 0..t-1 that satisfies labels, the pattern edges
    among placed positions, the order constraints and (t < nv) the degree filter."""
    order, lt, gt = plan
    adj = {v: set() for v in range(n)}
    for e in E:
        a, b = tuple(e)
        adj[a].add(b)
        adj[b].add(a)
    pdeg = [sum(1 for a, b in edges if order[t] in (a, b)) for t in range(nv)]
    pos = {v: t for t, v in enumerate(order)}
    back = [sum(1 << pos[u] for a, b in edges for u in ((b,) if a == order[t] else (a,) if b == order[t] else ())
                if pos[u] < t) for t in range(nv)]
    N, G, C = [0] * (nv + 1), [0] * (nv + 1), [0] * (nv + 1)
    for t in range(1, nv + 1):
        for phi in itertools.permutations(range(n), t):
            ok = True
            for i in range(t):
                x = phi[i]
                if plab is not None and glab[x] != plab[order[i]]:
                    ok = False
                if i + 1 < nv and len(adj[x]) < pdeg[i]:
                    ok = False
                for j in range(i):
                    if (back[i] >> j) & 1 and phi[j] not in adj[x]:
                        ok = False
                    if (lt[i] >> j) & 1 and not x > phi[j]:
                        ok = False
                    if (gt[i] >> j) & 1 and not x < phi[j]:
                        ok = False
                if not ok:
                    break
            if not ok:
                continue
            N[t] += 1
            if t < nv and (back[t] >> (t - 1)) & 1:
                C[t] += len(adj[phi[t - 1]])
            if t + 1 < nv:
                G[t + 1] += sum(len(adj[phi[j]]) for j in range(t) if (back[t + 1] >> j) & 1)
    return N, G, C


@pytest.mark.parametrize("q", ["c4", "diamond", "tailed_triangle", "house"])
@pytest.mark.parametrize("labeled", [False, True])
@pytest.mark.parametrize("seed", [1, 2])
def test_levels_brute_force(q, labeled, seed):
    nv, e = Q[q]
    n = 9
    s, d = gg.er(n, 26, seed)
    E = brute.normalise(s, d)
    glab = gg.labels(n, 2, seed)
    plab = [i % 2 for i in range(nv)] if labeled else None
    g = O.Graph(n, s, d, glab if labeled else None)
    plan = O.plan_r10_r16(nv, e, plab)
    got = g.match_levels(nv, e, plab)
    assert got == brute_levels(n, E, nv, e, plab, glab.tolist() if labeled else None, plan)
    assert got[0][nv] == brute.distinct_subgraphs(n, E, nv, e, plab, glab.tolist() if labeled else None)


@pytest.mark.parametrize("q", ["c4", "diamond", "tailed_triangle", "house"])
def test_last_level_is_the_count(q):
    nv, e = Q[q]
    n, s, d, lab = gg.config_graph("c3", seed=2, scale=10)
    g = O.Graph(n, s, d, lab)
    for plab in (None, [0] * nv, [i % 8 for i in range(nv)]):
        N, _, _ = g.match_levels(nv, e, plab)
        assert N[nv] == g.match(nv, e, plab)[0]


def test_complete_graph_c4():
    """K_n, C4 query, plan phi0 < phi1, phi0 < phi2, phi0 < phi3, phi1 < phi3 (order
    0, 1, 2, 3 on the cycle 0-1-2-3): N1 = n, N2 = C(n,2) (phi1 > phi0), N3 = pairs
    above phi0 for phi1 and phi2 = sum_a (n-1-a)(n-2-a), N4 = 3 C(n,4)."""
    n = 12
    s, d = np.triu_indices(n, 1)
    g = O.Graph(n, s.astype(np.uint32), d.astype(np.uint32))
    nv, e = Q["c4"]
    N, _, _ = g.match_levels(nv, e)
    assert N[1:] == [n, comb(n, 2), sum((n - 1 - a) * (n - 2 - a) for a in range(n)), 3 * comb(n, 4)]


@pytest.mark.parametrize("q", ["c4", "diamond", "tailed_triangle", "house"])
@pytest.mark.parametrize("plab", [None, "mod2", "mod3"])
def test_planner_agrees_with_library(q, plab):
    """The oracle planner restates R10/R16; the library's host planner (written
    independently in match.cu) must reach the same order and constraints, so that the
    oracle's level statistics describe the ET levels the GPU path builds."""
    G = pytest.importorskip("paper_conf_icde_hu0o23_b200")
    nv, e = Q[q]
    pl = None if plab is None else [i % (2 if plab == "mod2" else 3) for i in range(nv)]
    order, lt, gt = O.plan_r10_r16(nv, e, pl)
    p = G.pattern_plan(nv, e, pl)
    assert list(p["order"])[:nv] == order
    assert list(p["less_mask"])[:nv] == lt
    assert list(p["greater_mask"])[:nv] == gt
