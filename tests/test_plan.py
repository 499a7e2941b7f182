"""Host-side SM planner (gamma_pattern_plan, no GPU needed): |Aut_L|, the matching
order and the symmetry-breaking constraints.  The constraints are checked against
their defining property by brute force: on a small graph, the injective mappings
that satisfy them are exactly one per distinct subgraph."""
import itertools

import numpy as np
import pytest

import brute
import gamma_gen as gg

Q = gg.QUERIES


@pytest.fixture(scope="module")
def G():
    import paper_conf_icde_hu0o23_b200 as G
    return G


def test_aut_counts(G):
    assert [G.pattern_plan(*Q[q])["aut"] for q in ("c4", "diamond", "tailed_triangle", "house")] == [8, 4, 2, 2]
    assert G.pattern_plan(4, Q["c4"][1], [0, 1, 0, 1])["aut"] == 4
    assert G.pattern_plan(4, [(0, 1), (0, 2), (0, 3), (1, 2), (1, 3), (2, 3)])["aut"] == 24


def test_order_is_connected_and_max_degree_first(G):
    for q, (nv, e) in Q.items():
        p = G.pattern_plan(nv, e)
        deg = [sum(1 for a, b in e if x in (a, b)) for x in range(nv)]
        assert deg[p["order"][0]] == max(deg)
        assert sorted(p["order"]) == list(range(nv))
        for i in range(1, nv):
            assert p["backward_mask"][i] != 0


def constrained_count(plan, n, E, nv, e, plab=None, glab=None):
    order = plan["order"]
    cnt = 0
    for phi in itertools.permutations(range(n), nv):
        if plab is not None and any(glab[phi[i]] != plab[i] for i in range(nv)):
            continue
        if not all(frozenset((phi[a], phi[b])) in E for a, b in e):
            continue
        ok = True
        for i in range(nv):
            for j in range(i):
                if (plan["less_mask"][i] >> j) & 1 and not phi[order[j]] < phi[order[i]]:
                    ok = False
                if (plan["greater_mask"][i] >> j) & 1 and not phi[order[i]] < phi[order[j]]:
                    ok = False
        cnt += ok
    return cnt


@pytest.mark.parametrize("q", ["c4", "diamond", "tailed_triangle", "house"])
@pytest.mark.parametrize("labeled", [False, True])
def test_symmetry_breaking_is_exact(G, q, labeled):
    nv, e = Q[q]
    n = 8
    s, d = gg.er(n, 20, 3)
    E = brute.normalise(s, d)
    glab = gg.labels(n, 2, 3).tolist()
    plab = [i % 2 for i in range(nv)] if labeled else None
    plan = G.pattern_plan(nv, e, plab)
    want = brute.distinct_subgraphs(n, E, nv, e, plab, glab if labeled else None)
    got = constrained_count(plan, n, E, nv, e, plab, glab if labeled else None)
    assert got == want
    assert brute.mappings(n, E, nv, e, plab, glab if labeled else None) == want * plan["aut"]


def test_plan_rejects(G):
    with pytest.raises(G.GammaError):
        G.pattern_plan(4, [(0, 1), (2, 3)])
    with pytest.raises(G.GammaError):
        G.pattern_plan(0, [])
    # induced plans are accepted (same order / Aut_L / constraints as non-induced)
    assert G.pattern_plan(3, [(0, 1), (1, 2)], induced=True) == G.pattern_plan(3, [(0, 1), (1, 2)])
