"""Seeded synthetic input generators shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the method (no CSR build, no normalisation, no
intersection, no canonical labelling).  It only draws raw edge samples and vertex
labels, and it builds small closed-form test graphs as raw edge lists.  Both
``oracle/`` and the product path receive exactly these arrays as inputs.

Recipes (stated again in DESIGN.md §Inputs):

* R-MAT(scale, samples, a, b, c; seed): for sample i and recursion level j
  (j = 0 is the most significant bit) a counter-based 32-bit uniform
  ``u = word(i, j)`` picks quadrant 00 / 01 / 10 / 11 with integer thresholds
  ``floor(a*2^32)``, ``floor((a+b)*2^32)``, ``floor((a+b+c)*2^32)``.  The words are the
  two 32-bit halves of ``splitmix64(key + i*ceil(scale/2) + j//2)``.  Both end
  points are then passed through a seeded bijection of ``[0, 2^scale)`` (the vertex
  permutation).  Raw samples keep duplicates and self-loops; normalisation (O-0)
  is part of the method and happens on each side.
* ER ``G(n, m)``-style: m raw samples ``(h mod n, (h >> 32) mod n)`` with
  ``h = splitmix64(key + i)``.
* Labels: ``splitmix64((seed << 32) ^ v) mod L``.
"""
from __future__ import annotations

import numpy as np

__all__ = [
    "splitmix64", "rmat", "er", "labels", "permute_bits",
    "complete", "turan", "wheel", "cycle", "grid", "petersen", "star",
    "complete_bipartite", "path", "disjoint_union", "CONFIGS", "config_graph", "QUERIES",
]

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def splitmix64(x: np.ndarray) -> np.ndarray:
    """Vectorised splitmix64 finaliser on uint64 arrays (wrapping arithmetic)."""
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = x + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def _key(seed: int, salt: int) -> np.uint64:
    return splitmix64(np.array([(int(seed) << 8) ^ salt], dtype=np.uint64))[0]


def permute_bits(x: np.ndarray, bits: int, seed: int) -> np.ndarray:
    """Seeded bijection of [0, 2^bits): xor-key, odd multiply, xorshift, repeated."""
    if bits == 0:
        return np.zeros_like(np.asarray(x, dtype=np.uint64))
    mask = np.uint64((1 << bits) - 1)
    k = splitmix64(np.array([int(seed) * 7 + 3, int(seed) * 7 + 4, int(seed) * 7 + 5],
                            dtype=np.uint64))
    m1 = np.uint64(int(k[1]) | 1)
    m2 = np.uint64(int(k[2]) | 1)
    r = np.uint64(max(1, (bits + 1) // 2))
    y = np.asarray(x, dtype=np.uint64) & mask
    with np.errstate(over="ignore"):
        y = (y ^ (k[0] & mask)) & mask
        y = (y * m1) & mask
        y = y ^ (y >> r)
        y = (y * m2) & mask
        y = y ^ (y >> r)
        y = (y * m1) & mask
    return y


def rmat(scale: int, samples: int, a: float, b: float, c: float, seed: int,
         permute: bool = True, block: int = 1 << 22):
    """Raw R-MAT samples ``(src, dst)`` as uint32 arrays of length ``samples``."""
    assert 1 <= scale <= 31
    ta = np.uint64(int(a * 2 ** 32))
    tb = np.uint64(int((a + b) * 2 ** 32))
    tc = np.uint64(int((a + b + c) * 2 ** 32))
    key = _key(seed, 0x52)
    words = (scale + 1) // 2
    src = np.empty(samples, dtype=np.uint32)
    dst = np.empty(samples, dtype=np.uint32)
    for lo in range(0, samples, block):
        hi = min(samples, lo + block)
        i = np.arange(lo, hi, dtype=np.uint64)
        s = np.zeros(hi - lo, dtype=np.uint64)
        d = np.zeros(hi - lo, dtype=np.uint64)
        with np.errstate(over="ignore"):
            base = key + i * np.uint64(words)
        for w in range(words):
            with np.errstate(over="ignore"):
                h = splitmix64(base + np.uint64(w))
            for half in range(2):
                j = 2 * w + half
                if j >= scale:
                    break
                u = (h >> np.uint64(32 * half)) & np.uint64(0xFFFFFFFF)
                bit = np.uint64(scale - 1 - j)
                sbit = (u >= tb).astype(np.uint64)           # quadrants 10, 11
                dbit = (((u >= ta) & (u < tb)) | (u >= tc)).astype(np.uint64)  # 01, 11
                s |= sbit << bit
                d |= dbit << bit
        if permute:
            s = permute_bits(s, scale, seed)
            d = permute_bits(d, scale, seed)
        src[lo:hi] = s.astype(np.uint32)
        dst[lo:hi] = d.astype(np.uint32)
    return src, dst


def er(n: int, m: int, seed: int):
    """Raw uniform samples ``(src, dst)`` with ``m`` draws over ``n`` vertices."""
    key = _key(seed, 0x45)
    i = np.arange(m, dtype=np.uint64)
    with np.errstate(over="ignore"):
        h = splitmix64(key + i)
    src = (h & np.uint64(0xFFFFFFFF)) % np.uint64(n)
    dst = (h >> np.uint64(32)) % np.uint64(n)
    return src.astype(np.uint32), dst.astype(np.uint32)


def labels(n: int, L: int, seed: int) -> np.ndarray:
    """Uniform vertex labels ``splitmix64((seed << 32) ^ v) mod L`` as uint32."""
    v = np.arange(n, dtype=np.uint64)
    with np.errstate(over="ignore"):
        h = splitmix64((np.uint64(seed) << np.uint64(32)) ^ v)
    return (h % np.uint64(L)).astype(np.uint32)


# ----------------------------------------------------------------------------------
# Closed-form test graphs (raw undirected edge lists, each edge listed once).
# ----------------------------------------------------------------------------------

def _pairs(e):
    if len(e) == 0:
        return np.zeros(0, np.uint32), np.zeros(0, np.uint32)
    a = np.asarray(e, dtype=np.uint32)
    return a[:, 0].copy(), a[:, 1].copy()


def complete(n):
    return n, _pairs([(i, j) for i in range(n) for j in range(i + 1, n)])


def turan(n, r):
    part = [i % r for i in range(n)]
    return n, _pairs([(i, j) for i in range(n) for j in range(i + 1, n) if part[i] != part[j]])


def wheel(n):
    """Hub 0 joined to the cycle 1..n (n >= 3 rim vertices)."""
    e = [(0, i) for i in range(1, n + 1)]
    e += [(i, i % n + 1) for i in range(1, n + 1)]
    return n + 1, _pairs(e)


def cycle(n):
    return n, _pairs([(i, (i + 1) % n) for i in range(n)])


def path(n):
    return n, _pairs([(i, i + 1) for i in range(n - 1)])


def grid(a, b):
    e = []
    for i in range(a):
        for j in range(b):
            v = i * b + j
            if j + 1 < b:
                e.append((v, v + 1))
            if i + 1 < a:
                e.append((v, v + b))
    return a * b, _pairs(e)


def petersen():
    e = [(i, (i + 1) % 5) for i in range(5)]
    e += [(5 + i, 5 + (i + 2) % 5) for i in range(5)]
    e += [(i, i + 5) for i in range(5)]
    return 10, _pairs(e)


def star(s):
    return s + 1, _pairs([(0, i) for i in range(1, s + 1)])


def complete_bipartite(a, b):
    return a + b, _pairs([(i, a + j) for i in range(a) for j in range(b)])


def disjoint_union(*graphs):
    n0 = 0
    ss, dd = [], []
    for n, (s, d) in graphs:
        ss.append(s.astype(np.uint64) + n0)
        dd.append(d.astype(np.uint64) + n0)
        n0 += n
    s = np.concatenate(ss).astype(np.uint32) if ss else np.zeros(0, np.uint32)
    d = np.concatenate(dd).astype(np.uint32) if dd else np.zeros(0, np.uint32)
    return n0, (s, d)


# ----------------------------------------------------------------------------------
# SM query graphs (SURVEY.md §8(c) reading 5: Fig. 13 is missing from PAPER.md, so the
# four north_star queries are used).  (nv, edge list).
# ----------------------------------------------------------------------------------

QUERIES = {
    "c4": (4, [(0, 1), (1, 2), (2, 3), (3, 0)]),
    "diamond": (4, [(0, 1), (0, 2), (1, 2), (1, 3), (2, 3)]),          # K4 minus {0,3}
    "tailed_triangle": (4, [(0, 1), (0, 2), (1, 2), (2, 3)]),          # triangle + tail at 2
    "house": (5, [(0, 1), (0, 2), (1, 3), (2, 3), (2, 4), (3, 4)]),    # square 0-1-3-2 + roof 4
}


# ----------------------------------------------------------------------------------
# The paper-shaped workloads; parameters restated in DESIGN.md.
# ----------------------------------------------------------------------------------

CONFIGS = {
    # name: (scale, samples, a, b, c, L)
    "c1": (12, 90_000, 0.57, 0.19, 0.19, 1),            # 4-clique, oracle in seconds
    "c2": (22, 16_600_000, 0.53, 0.20, 0.20, 1),        # cit-Patents-shaped kCL k=4,5,6
    "heavy": (22, 20_000_000, 0.57, 0.19, 0.19, 1),     # Graph500-skew kCL scaling workload
    "c3": (23, 43_500_000, 0.50, 0.20, 0.20, 8),        # LiveJournal-shaped labeled SM
    "c4": (22, 16_600_000, 0.40, 0.25, 0.25, 37),       # cit-Patents-shaped FPM, 37 labels
    # Friendster-shaped (2^26 vertices, ~1.97e9 unique edges); a = 0.55 chosen on the box
    # (tools/c5_probe.py) so that the level-3 table (1.08e11 triangles x 8 B = 864 GB)
    # exceeds one GPU's HBM.  Drawn on the device (gamma_gen.torch_gen.config_graph_torch).
    "c5": (26, 2_000_000_000, 0.55, 0.20, 0.20, 1),
}


def config_graph(name: str, seed: int = 1, scale: int | None = None, samples: int | None = None):
    """Raw samples + labels for a named config; ``scale``/``samples`` override for small cases."""
    sc, ns, a, b, c, L = CONFIGS[name]
    if scale is not None:
        ns = max(1, int(ns * 2.0 ** (scale - sc))) if samples is None else samples
        sc = scale
    elif samples is not None:
        ns = samples
    src, dst = rmat(sc, ns, a, b, c, seed)
    lab = labels(1 << sc, L, seed) if L > 1 else None
    return 1 << sc, src, dst, lab
