"""Pure-Python brute force on tiny graphs: independent pins for the oracle.

These are deliberately the most literal possible statements of the definitions
(all k-subsets, all edge subsets, all injective maps) and are only used for
n <= ~16.  They share no code with oracle/ or with the CUDA path.
"""
from __future__ import annotations

import itertools
from math import comb


def normalise(src, dst):
    """O-0 by sets: undirected, no self-loops, no duplicates."""
    return {frozenset((int(u), int(v))) for u, v in zip(src, dst) if int(u) != int(v)}


def kcliques(n, E, k):
    """|{S subset V : |S| = k, every pair adjacent}| over all k-subsets."""
    return sum(1 for S in itertools.combinations(range(n), k)
               if all(frozenset(p) in E for p in itertools.combinations(S, 2)))


def _pattern_edges(edges):
    return {frozenset(e) for e in edges}


def aut(nv, pedges, plab=None):
    PE = _pattern_edges(pedges)
    plab = plab or [0] * nv
    c = 0
    for p in itertools.permutations(range(nv)):
        if all(plab[p[i]] == plab[i] for i in range(nv)) and \
                {frozenset((p[a], p[b])) for a, b in pedges} == PE:
            c += 1
    return c


def mappings(n, E, nv, pedges, plab=None, glab=None):
    """All injective phi: V_P -> V_G with label(phi i) = plab[i] and every pattern
    edge mapped onto a graph edge (non-induced)."""
    c = 0
    for phi in itertools.permutations(range(n), nv):
        if plab is not None and any(glab[phi[i]] != plab[i] for i in range(nv)):
            continue
        if all(frozenset((phi[a], phi[b])) in E for a, b in pedges):
            c += 1
    return c


def distinct_subgraphs(n, E, nv, pedges, plab=None, glab=None):
    """Number of distinct edge subsets S of G (|S| = |E_P|) isomorphic to P, labels
    respected -- counted by enumerating edge subsets, not mappings."""
    El = sorted(tuple(sorted(e)) for e in E)
    ne = len(pedges)
    PE = _pattern_edges(pedges)
    cnt = 0
    for S in itertools.combinations(El, ne):
        W = sorted({x for e in S for x in e})
        if len(W) != nv:
            continue
        Sset = {frozenset(e) for e in S}
        for p in itertools.permutations(W):
            # p[i] = data vertex playing pattern vertex i
            if plab is not None and any(glab[p[i]] != plab[i] for i in range(nv)):
                continue
            if {frozenset((p[a], p[b])) for a, b in pedges} == Sset:
                cnt += 1
                break
    return cnt


def canon(nv, W, S, glab):
    """Min over bijections of (labels, sorted edge-pair list) + all minimizers."""
    best, arg = None, []
    for p in itertools.permutations(W):
        pos = {v: i for i, v in enumerate(p)}
        labs = tuple(glab[v] for v in p)
        es = tuple(sorted(tuple(sorted((pos[a], pos[b]))) for a, b in S))
        key = (labs, es)
        if best is None or key < best:
            best, arg = key, [p]
        elif key == best:
            arg.append(p)
    return best, arg


def fpm(n, E, l, minsup, glab=None):
    """Every connected edge subset with 1..l edges -> canonical pattern -> MNI."""
    glab = glab if glab is not None else [0] * n
    El = sorted(tuple(sorted(e)) for e in E)
    dom = {}
    inst = {}
    for ne in range(1, l + 1):
        for S in itertools.combinations(El, ne):
            W = sorted({x for e in S for x in e})
            # connectivity of the edge set
            comp = {W[0]}
            changed = True
            while changed:
                changed = False
                for a, b in S:
                    if (a in comp) != (b in comp):
                        comp |= {a, b}
                        changed = True
            if len(comp) != len(W):
                continue
            (labs, es), arg = canon(len(W), W, S, glab)
            key = (ne, len(W), labs, es)
            d = dom.setdefault(key, [set() for _ in W])
            inst[key] = inst.get(key, 0) + 1
            for p in arg:
                for i, v in enumerate(p):
                    d[i].add(v)
    out = []
    for key, d in dom.items():
        sup = min(len(x) for x in d)
        if sup >= minsup:
            out.append((key[0], key[1], key[2], key[3], sup, inst[key]))
    out.sort(key=lambda r: r[:4])
    return out


def connected_subset_counts(n, E):
    """Closed forms: #connected 2-edge sets = sum C(d,2);
    #connected 3-edge sets = T + sum C(d,3) + sum_{uv}(d_u-1)(d_v-1) - 3T."""
    deg = [0] * n
    for e in E:
        for x in e:
            deg[x] += 1
    T = kcliques(n, E, 3)
    two = sum(comb(d, 2) for d in deg)
    three = T + sum(comb(d, 3) for d in deg) + sum((deg[a] - 1) * (deg[b] - 1) for a, b in
                                                   (tuple(e) for e in E)) - 3 * T
    return two, three


def induced_subgraphs(n, E, nv, pedges, plab=None, glab=None):
    """Number of vertex subsets W (|W| = nv) whose induced subgraph G[W] is isomorphic
    to P, labels respected (induced matching, counted by vertex subsets)."""
    PE = _pattern_edges(pedges)
    cnt = 0
    for W in itertools.combinations(range(n), nv):
        EW = {e for e in (frozenset(p) for p in itertools.combinations(W, 2)) if e in E}
        if len(EW) != len(PE):
            continue
        for p in itertools.permutations(W):
            if plab is not None and any(glab[p[i]] != plab[i] for i in range(nv)):
                continue
            if {frozenset((p[a], p[b])) for a, b in pedges} == EW:
                cnt += 1
                break
    return cnt
