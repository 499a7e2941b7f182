"""GPU parity of A1 (CSR/DAG build) and kCL (A2-A8) against the oracle, through the
C ABI.  Tolerance 0: every output is an integer (north_star)."""
from math import comb

import numpy as np
import pytest

import gamma_gen as gg

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def G():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_icde_hu0o23_b200 as G
    return G


@pytest.fixture(scope="module")
def ctx(G):
    return G.Context(device=0)


def load(ctx, n, s, d, lab=None):
    return ctx.load_edges(n, s, d, lab)


def test_library_is_in_tree(G):
    import os
    assert os.path.dirname(G.library_path()) == os.path.dirname(G.__file__)


def test_csr_matches_oracle(ctx, oracle_mod):
    for seed in (1, 2, 3):
        n, s, d, _ = gg.config_graph("c1", seed=seed)
        g = load(ctx, n, s, d)
        o = oracle_mod.Graph(n, s, d)
        rp, col = g.csr("sym")
        orp, ocol = o.csr()
        assert g.info()["m"] == o.m
        assert np.array_equal(rp, orp) and np.array_equal(col, ocol)


def test_csr_from_device_tensors(ctx, oracle_mod):
    import torch
    n, s, d, _ = gg.config_graph("c1", seed=4, scale=11)
    g = ctx.load_edges(n, torch.from_numpy(s.view(np.int32)).cuda(), torch.from_numpy(d.view(np.int32)).cuda())
    o = oracle_mod.Graph(n, s, d)
    rp, col = g.csr("sym")
    orp, ocol = o.csr()
    assert np.array_equal(rp, orp) and np.array_equal(col, ocol)


def test_dag_definition(ctx):
    n, s, d, _ = gg.config_graph("c1", seed=1)
    g = load(ctx, n, s, d)
    rp, col = g.csr("sym")
    drp, dcol = g.csr("dag")
    deg = np.diff(rp.astype(np.int64))
    m = g.info()["m"]
    assert drp[-1] == m
    for v in range(0, n, 7):
        out = dcol[drp[v]:drp[v + 1]]
        assert np.all(np.diff(out.astype(np.int64)) > 0)
        nb = col[rp[v]:rp[v + 1]]
        want = [u for u in nb if (deg[v], v) < (deg[u], u)]
        assert out.tolist() == want
    assert g.info()["max_out_degree"] == int(np.diff(drp.astype(np.int64)).max())


def test_closed_forms(ctx):
    cases = [(gg.complete(12), {k: comb(12, k) for k in range(1, 14)}),
             (gg.turan(12, 4), {k: comb(4, k) * 3 ** k for k in range(2, 6)}),
             (gg.wheel(9), {3: 9, 4: 0}),
             (gg.cycle(3), {3: 1}),
             (gg.grid(6, 7), {3: 0}),
             (gg.petersen(), {3: 0})]
    for (n, (s, d)), want in cases:
        g = load(ctx, n, s, d)
        for k, c in want.items():
            assert g.kclique(k) == c, (n, k)


def test_complete_large_k(ctx):
    # K_24 holds 2^24 cliques over all sizes: deep levels without blowing up the test
    n, (s, d) = gg.complete(24)
    g = load(ctx, n, s, d)
    for k in (5, 8, 12, 20, 24, 25, 32):
        assert g.kclique(k) == comb(24, k)
    # one bitmap pass for sizes 3..12; sizes beyond 12 fall back to per-k calls
    ks = list(range(1, 13))
    assert g.kclique_multi(ks) == [comb(24, k) for k in ks]
    assert g.kclique_multi([3, 16, 24]) == [comb(24, 3), comb(24, 16), 1]
    assert g.kclique_multi([]) == []


@pytest.mark.parametrize("seed", [1, 2, 3, 4, 5])
def test_er_vs_oracle(ctx, oracle_mod, seed):
    n = 1 << (10 + seed)
    s, d = gg.er(n, 12 * n, seed)
    g = load(ctx, n, s, d)
    o = oracle_mod.Graph(n, s, d)
    for k in (3, 4, 5):
        assert g.kclique(k) == o.kclique(k)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_c1_vs_oracle(ctx, oracle_mod, seed):
    n, s, d, _ = gg.config_graph("c1", seed=seed)
    g = load(ctx, n, s, d)
    o = oracle_mod.Graph(n, s, d)
    for k in (1, 2, 3, 4, 5, 6):
        assert g.kclique(k) == o.kclique(k), k


def test_per_root_counts(ctx, oracle_mod):
    n, s, d, _ = gg.config_graph("c1", seed=2, scale=11)
    g = load(ctx, n, s, d)
    o = oracle_mod.Graph(n, s, d)
    roots = np.arange(n, dtype=np.uint32)
    for k in (2, 3, 4, 5):
        got = g.kclique_roots(k, roots)
        want = o.kclique_roots(k, roots)
        assert np.array_equal(got, want), k
        assert int(got.sum()) == g.kclique(k)


def test_budget_forced_splits(G, oracle_mod):
    n, s, d, _ = gg.config_graph("c1", seed=1, scale=11)
    o = oracle_mod.Graph(n, s, d)
    c = G.Context(hbm_budget_bytes=3 << 20, flags=0x10)   # ET path, ~3 MB of ET: forces range splits
    g = c.load_edges(n, s, d)
    for k in (4, 5, 6):
        assert g.kclique(k) == o.kclique(k)
    st = c.stats()
    assert st["retries"] > 0


def test_pinned_host_spill(G, oracle_mod):
    """GAMMA_FLAG_SPILL: levels that exceed the HBM budget are parked in pinned host
    memory and streamed back; counts are unchanged."""
    n, s, d, _ = gg.config_graph("c1", seed=2, scale=11)
    o = oracle_mod.Graph(n, s, d)
    c = G.Context(hbm_budget_bytes=3 << 20, host_spill_bytes=1 << 30, flags=0x10 | 0x4 | 0x2)
    g = c.load_edges(n, s, d)
    for k in (4, 5):
        assert g.kclique(k) == o.kclique(k)
    assert c.stats()["spilled_bytes"] > 0
    roots = np.arange(0, n, 5, dtype=np.uint32)
    assert np.array_equal(g.kclique_roots(5, roots), o.kclique_roots(5, roots))
    small = G.Context(hbm_budget_bytes=3 << 20, host_spill_bytes=4096, flags=0x10 | 0x4 | 0x2)
    with pytest.raises(G.GammaError) as e:
        small.load_edges(n, s, d).kclique(5)
    assert e.value.status == -2


def test_simulated_ranks_partition(G, oracle_mod):
    n, s, d, _ = gg.config_graph("c1", seed=3)
    want = oracle_mod.Graph(n, s, d).kclique(5)
    for world in (2, 3, 8):
        tot = 0
        for r in range(world):
            c = G.Context(rank=r, world=world, reduce=False)
            tot += c.load_edges(n, s, d).kclique(5)
        assert tot == want
    # multi-k over the same partition
    o = oracle_mod.Graph(n, s, d)
    want = [o.kclique(k) for k in (3, 4, 5, 6)]
    tot = [0] * 4
    for r in range(3):
        part = G.Context(rank=r, world=3, reduce=False).load_edges(n, s, d).kclique_multi([3, 4, 5, 6])
        tot = [x + y for x, y in zip(tot, part)]
    assert tot == want


def test_load_csr_roundtrip_and_validation(G, ctx, oracle_mod):
    n, s, d, _ = gg.config_graph("c1", seed=5, scale=11)
    o = oracle_mod.Graph(n, s, d)
    rp, col = o.csr()
    g = ctx.load_csr(n, rp, col)
    assert g.kclique(4) == o.kclique(4)
    bad = col.copy()
    i = int(rp[5])
    if rp[6] - rp[5] >= 2:
        bad[i], bad[i + 1] = bad[i + 1], bad[i]      # unsorted list
        with pytest.raises(G.GammaError):
            ctx.load_csr(n, rp, bad)
    # asymmetric: drop one direction
    rp2, col2 = gg.path(3)[1]
    with pytest.raises(G.GammaError):
        ctx.load_csr(3, np.array([0, 1, 1, 1], np.uint64), np.array([1], np.uint32))


def test_edge_cases(G, ctx):
    g = ctx.load_edges(7, np.zeros(0, np.uint32), np.zeros(0, np.uint32))
    assert g.kclique(1) == 7 and g.kclique(2) == 0 and g.kclique(3) == 0
    g = ctx.load_edges(3, np.array([0, 1, 1], np.uint32), np.array([0, 1, 1], np.uint32))  # self-loops only
    assert g.info()["m"] == 0 and g.kclique(3) == 0
    with pytest.raises(G.GammaError):
        ctx.load_edges(3, np.array([0], np.uint32), np.array([5], np.uint32))
    n, (s, d) = gg.complete(5)
    g = ctx.load_edges(n, s, d)
    with pytest.raises(G.GammaError) as e:
        g.kclique(33)
    assert e.value.status == -5
    with pytest.raises(G.GammaError):
        g.kclique(0)


def test_unstaged_long_run_path(G, oracle_mod):
    """Runs longer than the shared-memory staging buffer take the global-memory
    probe and the direct-reservation write path; the debug flag forces that path
    for every group so it is checked on ordinary inputs."""
    c = G.Context(flags=0x8 | 0x10)   # GAMMA_FLAG_DEBUG_NOSTAGE | GAMMA_FLAG_NO_BITMAP
    for seed in (1, 2):
        n, s, d, _ = gg.config_graph("c1", seed=seed)
        g = c.load_edges(n, s, d)
        o = oracle_mod.Graph(n, s, d)
        for k in (3, 4, 5, 6):
            assert g.kclique(k) == o.kclique(k)


@pytest.mark.parametrize("a", [200, 1100, 2500])
def test_hub_out_list_longer_than_staging(G, ctx, oracle_mod, a):
    """A real vertex with a long DAG out-list: v joined to the a vertices of one side
    of K_{a,a+1} (those outrank v), plus a sprinkle of edges among them.  a=200
    takes the CTA-team bitmap path, a=1100 the wide path with 2 words per lane,
    a=2500 the wide path with 8 words per lane."""
    b = a + 1
    U = np.arange(1, 1 + a)
    F = np.arange(1 + a, 1 + a + b)
    e = [(0, u) for u in U] + [(u, f) for u in U for f in F[:b]]
    rng = np.random.default_rng(3)
    extra = rng.choice(U, size=(3000, 2))
    e = np.array(e + [tuple(x) for x in extra], dtype=np.uint32)
    n = 1 + a + b
    g = ctx.load_edges(n, e[:, 0].copy(), e[:, 1].copy())
    assert g.info()["max_out_degree"] >= a
    o = oracle_mod.Graph(n, e[:, 0].copy(), e[:, 1].copy())
    roots = np.array([0], np.uint32)
    for k in (3, 4, 5):
        assert np.array_equal(g.kclique_roots(k, roots), o.kclique_roots(k, roots))
    want = [o.kclique(k) for k in (3, 4, 5)]
    assert [g.kclique(k) for k in (3, 4, 5)] == want
    assert g.kclique_multi([3, 4, 5]) == want
    # the same counts through the ET path
    c = G.Context(flags=0x10)
    assert [c.load_edges(n, e[:, 0].copy(), e[:, 1].copy()).kclique(k) for k in (3, 4)] == want[:2]


def test_wide_runs_closed_forms(ctx):
    """K_n puts a run of length n-1-i under root i: every path (warp, CTA, wide with 2
    and 8 words per lane, and the ET path past 8192) against C(n, k)."""
    def kn(n):
        s, d = np.triu_indices(n, 1)
        return n, (s.astype(np.uint32), d.astype(np.uint32))

    n, (s, d) = kn(2600)
    g = load(ctx, n, s, d)
    assert g.info()["max_out_degree"] == 2599
    assert g.kclique_multi([3, 4]) == [comb(2600, 3), comb(2600, 4)]
    roots = np.array([0, 1, 100, 600, 1000, 2000, 2400, 2599], np.uint32)
    assert list(g.kclique_roots(4, roots)) == [comb(2599 - int(i), 3) for i in roots]
    assert list(g.kclique_roots(5, roots[3:])) == [comb(2599 - int(i), 4) for i in roots[3:]]
    n, (s, d) = kn(8194)   # root 0 has d+ = 8193 > 8192: ET path
    g = load(ctx, n, s, d)
    assert g.kclique(3) == comb(8194, 3)


@pytest.mark.parametrize("flags", [0, 0x10, 0x2 | 0x10, 0x20, 0x40, 0x200 | 0x10, 0x200 | 0x10 | 0x2])
def test_paths_agree(G, oracle_mod, flags):
    """Bitmap DFS (default), ET levels with the fused tail (NO_BITMAP), ET levels
    with every level materialised (NO_FUSE | NO_BITMAP), the bitmap path without hub
    splitting (NO_SPLIT) and with every root split into parts (DEBUG_SPLIT_ALL) all
    equal the oracle."""
    c = G.Context(flags=flags)
    n, s, d, _ = gg.config_graph("c1", seed=4)
    g = c.load_edges(n, s, d)
    o = oracle_mod.Graph(n, s, d)
    want = [o.kclique(k) for k in range(1, 9)]
    for k in (3, 4, 5, 6, 7):
        assert g.kclique(k) == want[k - 1], (flags, k)
    # every size from one multi-k pass (per-k calls under NO_BITMAP)
    assert g.kclique_multi(list(range(1, 9))) == want, flags
    assert g.kclique_multi([6, 4]) == [want[5], want[3]], flags
    roots = np.arange(0, n, 3, dtype=np.uint32)
    assert np.array_equal(g.kclique_roots(5, roots), o.kclique_roots(5, roots))


@pytest.mark.parametrize("cap", [1, 3, 64])
def test_parts_list_overflow(G, oracle_mod, monkeypatch, cap):
    """Hub splitting with a part list too short for every deferred root:
    a root whose parts do not fit is expanded by its own team, the parts kernel reads
    only reserved slots, and every count still equals the oracle."""
    monkeypatch.setenv("GAMMA_KCL_PARTS_CAP", str(cap))
    c = G.Context(flags=0x40)   # GAMMA_FLAG_DEBUG_SPLIT_ALL: every k >= 6 root is deferred
    n, s, d, _ = gg.config_graph("c1", seed=4)
    g = c.load_edges(n, s, d)
    o = oracle_mod.Graph(n, s, d)
    assert g.kclique(6) == o.kclique(6)
    assert g.kclique_multi([4, 5, 6, 7]) == [o.kclique(k) for k in (4, 5, 6, 7)]
    roots = np.arange(0, n, 2, dtype=np.uint32)
    assert np.array_equal(g.kclique_roots(6, roots), o.kclique_roots(6, roots))


@pytest.mark.slow
def test_c2_full_size(ctx, oracle_mod):
    """configs[1] at full size: cit-Patents-shaped R-MAT scale 22, k = 4, 5, 6, both
    per k and through the one multi-k pass bench.py times (gamma_kclique_multi)."""
    n, s, d, _ = gg.config_graph("c2", seed=1)
    g = load(ctx, n, s, d)
    o = oracle_mod.Graph(n, s, d)
    assert g.info()["m"] == o.m
    want = [o.kclique(k) for k in (4, 5, 6)]
    assert [g.kclique(k) for k in (4, 5, 6)] == want
    assert g.kclique_multi([4, 5, 6]) == want


@pytest.mark.parametrize("case", ["c1", "er", "dups", "selfloops", "one"])
def test_builders_agree(G, ctx, oracle_mod, case):
    """A1 has two builders -- the global key sort (default) and counting sort +
    segmented row sort (GAMMA_FLAG_COUNT_SORT_BUILD); both must give the oracle's O-0
    CSR and the same DAG."""
    if case == "c1":
        n, s, d, _ = gg.config_graph("c1", seed=2)
    elif case == "er":
        n = 5000
        s, d = gg.er(n, 40000, 3)
    elif case == "dups":
        n = 64
        s = np.array([1, 2, 1, 2, 3, 3, 5, 1] * 50, np.uint32)
        d = np.array([2, 1, 2, 1, 4, 4, 1, 5] * 50, np.uint32)
    elif case == "selfloops":
        n = 10
        s = np.arange(10, dtype=np.uint32)
        d = s.copy()
    else:
        n = 2
        s, d = np.array([0], np.uint32), np.array([1], np.uint32)
    counting = G.Context(device=0, flags=0x80)   # GAMMA_FLAG_COUNT_SORT_BUILD
    g1, g2 = ctx.load_edges(n, s, d), counting.load_edges(n, s, d)
    o = oracle_mod.Graph(n, s, d)
    orp, ocol = o.csr()
    for g in (g1, g2):
        rp, col = g.csr("sym")
        assert np.array_equal(rp, orp) and np.array_equal(col, ocol)
        assert g.info()["max_degree"] == (int(np.diff(orp.astype(np.int64)).max()) if n else 0)
    d1, d2 = g1.csr("dag"), g2.csr("dag")
    assert np.array_equal(d1[0], d2[0]) and np.array_equal(d1[1], d2[1])
    assert g1.info()["max_out_degree"] == g2.info()["max_out_degree"]


def test_builder_rejects_bad_ids(ctx):
    s = np.array([0, 7], np.uint32)
    d = np.array([1, 2], np.uint32)
    with pytest.raises(Exception):
        ctx.load_edges(4, s, d)


@pytest.mark.slow
def test_heavy_full_size(ctx):
    """The heavy kCL workload (Graph500-skew R-MAT scale 22, 20M samples, seed 1) at full
    size, in the bench's configuration (one multi-k pass) and per k, against the
    oracle's counts stored by tools/golden_heavy.py (oracle-only script)."""
    import json
    import os
    gold = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "heavy_seed1.json")))
    n, s, d, _ = gg.config_graph("heavy", seed=1)
    g = load(ctx, n, s, d)
    assert g.info()["m"] == gold["m"]
    want = [gold["counts"][str(k)] for k in (3, 4, 5)]
    assert g.kclique_multi([3, 4, 5]) == want
    assert g.kclique_multi([4, 5]) == want[1:]
    assert [g.kclique(k) for k in (4, 5)] == want[1:]


@pytest.mark.slow
def test_c2_full_size_spill(G):
    """A8 at full size: configs[1] on the list-based ET path (GAMMA_FLAG_NO_BITMAP |
    GAMMA_FLAG_NO_FUSE) with a 192 MiB HBM budget, so the level tables (the 5-clique
    level alone is 603 MB) are produced in slabs parked in pinned host memory and
    streamed back, double-buffered on the copy stream; the counts
    equal the oracle's (tests/golden/c2_full_seed1.json, oracle-only script)."""
    import json
    import os
    gold = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "c2_full_seed1.json")))
    c = G.Context(hbm_budget_bytes=192 << 20, host_spill_bytes=8 << 30,
                  flags=G._native.GAMMA_FLAG_NO_BITMAP | G._native.GAMMA_FLAG_NO_FUSE | G._native.GAMMA_FLAG_SPILL)
    n, s, d, _ = gg.config_graph("c2", seed=1)
    g = c.load_edges(n, s, d)
    assert g.info()["m"] == gold["m"]
    for k in (5, 6):
        assert g.kclique(k) == gold["counts"][str(k)], k
        assert c.stats()["spilled_bytes"] > 0, k


@pytest.mark.parametrize("cache_kb", [0, 64, 256, 1 << 20])
def test_host_resident_dag(G, oracle_mod, cache_kb):
    """GAMMA_FLAG_HOST_DAG: the DAG columns in pinned host memory
    mapped into the device, the hottest 64 KiB pages cached in HBM (none / a few / all);
    every count equals the oracle's, per root too."""
    n, s, d, _ = gg.config_graph("c1", seed=3, scale=14)
    c = G.Context(flags=G._native.GAMMA_FLAG_HOST_DAG, dag_cache_bytes=cache_kb << 10)
    g = c.load_edges(n, s, d)
    o = oracle_mod.Graph(n, s, d)
    assert g.kclique_multi([3, 4, 5, 6]) == [o.kclique(k) for k in (3, 4, 5, 6)]
    assert g.kclique(5) == o.kclique(5)
    roots = np.arange(0, n, 7, dtype=np.uint32)
    assert np.array_equal(g.kclique_roots(4, roots), o.kclique_roots(4, roots))
    rp, col = g.csr("dag")   # export still in id space
    assert int(rp[-1]) == g.info()["m"]


@pytest.mark.parametrize("scale,samples,world,min_dplus", [(16, 6_000_000, 8, 512), (16, 6_000_000, 3, 512),
                                                            (18, 6_000_000, 8, 128)])
def test_simulated_ranks_wide_runs(G, scale, samples, world, min_dplus):
    """The root partition on graphs whose runs reach the wide (|R| > 512) and CTA-team
    paths (C5's shape family, a = 0.55 at small scale): the partial counts of the
    `world` rank shares sum to the world-1 counts, for the multi-k pass (k = 3, 4, 5)
    and per k (the C5 simulated-rank run of round 2 disagreed)."""
    s, d = gg.rmat(scale, samples, 0.55, 0.20, 0.20, seed=1)
    n = 1 << scale
    g1 = G.Context().load_edges(n, s, d)
    assert g1.info()["max_out_degree"] > min_dplus   # (scale 16, 6M: 651; scale 18: 464)
    want = g1.kclique_multi([3, 4, 5])
    want4 = g1.kclique(4)
    tot, tot4 = [0, 0, 0], 0
    for r in range(world):
        g = G.Context(rank=r, world=world, reduce=False).load_edges(n, s, d)
        tot = [x + y for x, y in zip(tot, g.kclique_multi([3, 4, 5]))]
        tot4 += g.kclique(4)
    assert tot4 == want4
    assert tot == want
