"""The seeded input generators (gamma_gen): determinism and distribution shape."""
import numpy as np

import gamma_gen as gg


def test_rmat_deterministic_and_in_range():
    a = gg.rmat(12, 5000, 0.57, 0.19, 0.19, 1)
    b = gg.rmat(12, 5000, 0.57, 0.19, 0.19, 1)
    c = gg.rmat(12, 5000, 0.57, 0.19, 0.19, 2)
    assert all(np.array_equal(x, y) for x, y in zip(a, b))
    assert not np.array_equal(a[0], c[0])
    assert a[0].max() < 4096 and a[1].max() < 4096


def test_rmat_block_invariance():
    a = gg.rmat(10, 3000, 0.5, 0.2, 0.2, 3, block=1 << 22)
    b = gg.rmat(10, 3000, 0.5, 0.2, 0.2, 3, block=777)
    assert all(np.array_equal(x, y) for x, y in zip(a, b))


def test_rmat_quadrant_probabilities():
    # unpermuted top bit: P(src bit) = c + d, P(dst bit) = b + d
    s, d = gg.rmat(16, 200_000, 0.57, 0.19, 0.19, 5, permute=False)
    top_s = (s >> 15).mean()
    top_d = (d >> 15).mean()
    assert abs(top_s - 0.24) < 0.01 and abs(top_d - 0.24) < 0.01


def test_permutation_is_bijection():
    for bits in (1, 5, 12, 17):
        x = gg.permute_bits(np.arange(1 << bits, dtype=np.uint64), bits, 9)
        assert np.unique(x).size == 1 << bits


def test_labels_uniform():
    lab = gg.labels(1 << 16, 8, 1)
    counts = np.bincount(lab, minlength=8)
    assert counts.min() > 0.9 * (1 << 13) and counts.max() < 1.1 * (1 << 13)


def test_config_graph_small():
    n, s, d, lab = gg.config_graph("c3", scale=10)
    assert n == 1024 and lab is not None and lab.max() < 8
    assert s.size == int(43_500_000 * 2.0 ** (10 - 23))


def test_torch_twin_matches_numpy():
    """gamma_gen.torch_gen (used to draw C5 in device memory) reproduces the numpy
    recipe element by element, across block boundaries and scales up to 31 bits."""
    from gamma_gen.torch_gen import rmat_torch
    for sc, ns, (a, b, c), seed in [(12, 9000, (0.57, 0.19, 0.19), 1), (26, 50_000, (0.55, 0.2, 0.2), 3),
                                    (7, 1000, (0.4, 0.25, 0.25), 2), (31, 5000, (0.5, 0.2, 0.2), 4)]:
        s, d = gg.rmat(sc, ns, a, b, c, seed)
        ts, td = rmat_torch(sc, ns, a, b, c, seed, device="cpu", block=4096)
        assert np.array_equal(s, ts.numpy().view(np.uint32)), sc
        assert np.array_equal(d, td.numpy().view(np.uint32)), sc
