"""ctypes wrapper of the CPU oracle (oracle/oracle.c).

TEST INFRASTRUCTURE, NOT PRODUCT CODE: only tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / ``--impl reference`` legs may import this package.  It
never imports the product package and the product package never imports it.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

REC = 17  # uint64 words per FPM result record (see oracle.c)


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (-O2 -fopenmp); returns its path."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-g", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-Wall", "-Wno-unused-function", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            L = C.CDLL(build())
            u32p = np.ctypeslib.ndpointer(np.uint32, flags="C_CONTIGUOUS")
            u64p = np.ctypeslib.ndpointer(np.uint64, flags="C_CONTIGUOUS")
            L.og_build.restype = C.c_void_p
            L.og_build.argtypes = [C.c_uint32, C.c_uint64, u32p, u32p, C.c_void_p]
            L.og_free.argtypes = [C.c_void_p]
            L.og_n.restype = C.c_uint32; L.og_n.argtypes = [C.c_void_p]
            L.og_m.restype = C.c_uint64; L.og_m.argtypes = [C.c_void_p]
            L.og_csr.argtypes = [C.c_void_p, u64p, u32p]
            L.og_kclique.restype = C.c_uint64
            L.og_kclique.argtypes = [C.c_void_p, C.c_uint32, C.c_int, C.c_int]
            L.og_kclique_roots.argtypes = [C.c_void_p, C.c_uint32, C.c_uint64, u32p, u64p, C.c_int]
            L.og_kclique_levels.argtypes = [C.c_void_p, C.c_uint32, u64p, u64p, C.c_int]
            L.og_match.restype = C.c_int
            L.og_match.argtypes = [C.c_void_p, C.c_uint32, C.c_uint32, u32p, C.c_void_p, C.c_int, C.c_int,
                                   C.POINTER(C.c_uint64), C.POINTER(C.c_uint64), C.POINTER(C.c_uint64)]
            L.og_match_roots.restype = C.c_int
            L.og_match_roots.argtypes = [C.c_void_p, C.c_uint32, C.c_uint32, u32p, C.c_void_p, C.c_int, C.c_uint64,
                                         u32p, u64p, C.c_int]
            L.og_match_levels.restype = C.c_int
            L.og_match_levels.argtypes = [C.c_void_p, C.c_uint32, C.c_uint32, u32p, C.c_void_p, u32p, u32p, u32p,
                                          C.c_int, u64p, u64p, u64p]
            L.og_fpm.restype = C.c_int64
            L.og_fpm.argtypes = [C.c_void_p, C.c_uint32, C.c_uint64, C.c_int, C.c_int, C.c_uint64,
                                 u64p, C.c_uint64]
            L.og_pattern_mni.restype = C.c_int
            L.og_pattern_mni.argtypes = [C.c_void_p, C.c_uint32, C.c_uint32, u32p, C.c_void_p, C.c_int,
                                         C.POINTER(C.c_uint64)]
            _lib = L
    return _lib


class Graph:
    """O-0 normalised undirected simple graph held by the oracle."""

    def __init__(self, n: int, src, dst, labels=None):
        L = lib()
        src = np.ascontiguousarray(src, dtype=np.uint32)
        dst = np.ascontiguousarray(dst, dtype=np.uint32)
        assert src.shape == dst.shape
        self._labels = None if labels is None else np.ascontiguousarray(labels, dtype=np.uint32)
        lp = None if self._labels is None else self._labels.ctypes.data
        self._h = L.og_build(int(n), int(src.size), src, dst, lp)
        if not self._h:
            raise ValueError("oracle: invalid edge list (vertex id >= n)")

    def __del__(self):
        h = getattr(self, "_h", None)
        if h:
            lib().og_free(h)
            self._h = None

    @property
    def n(self) -> int:
        return lib().og_n(self._h)

    @property
    def m(self) -> int:
        return lib().og_m(self._h)

    def csr(self):
        off = np.empty(self.n + 1, np.uint64)
        adj = np.empty(2 * self.m, np.uint32)
        lib().og_csr(self._h, off, adj)
        return off, adj

    def kclique(self, k: int, order: str = "degree", threads: int = 0) -> int:
        return int(lib().og_kclique(self._h, k, 0 if order == "degree" else 1, threads))

    def kclique_roots(self, k: int, roots, threads: int = 0) -> np.ndarray:
        roots = np.ascontiguousarray(roots, dtype=np.uint32)
        out = np.zeros(roots.size, np.uint64)
        lib().og_kclique_roots(self._h, k, roots.size, roots, out, threads)
        return out

    def kclique_levels(self, k: int, threads: int = 0):
        """(N, S): N[t] = #t-cliques, S[t] = sum over t-cliques of d+(last vertex),
        t = 0..k (index 0 is 0).  Feeds SURVEY §8(d)'s algorithmic bytes."""
        N = np.zeros(k + 1, np.uint64)
        S = np.zeros(k + 1, np.uint64)
        lib().og_kclique_levels(self._h, k, N, S, threads)
        return [int(x) for x in N], [int(x) for x in S]

    def match(self, nv: int, edges, plabels=None, threads: int = 0, induced: bool = False):
        """Return (count, mappings, |Aut_L|); induced=True also maps non-edges to non-edges."""
        e = np.ascontiguousarray(np.asarray(edges, dtype=np.uint32).reshape(-1))
        pl = None if plabels is None else np.ascontiguousarray(plabels, dtype=np.uint32)
        c, mp, a = C.c_uint64(), C.c_uint64(), C.c_uint64()
        st = lib().og_match(self._h, nv, e.size // 2, e, None if pl is None else pl.ctypes.data,
                            int(bool(induced)), threads, C.byref(c), C.byref(mp), C.byref(a))
        if st != 0:
            raise ValueError(f"oracle og_match status {st}")
        return int(c.value), int(mp.value), int(a.value)

    def match_roots(self, nv: int, edges, roots, plabels=None, threads: int = 0,
                    induced: bool = False) -> np.ndarray:
        """Mappings whose image of pattern vertex 0 is each given root."""
        e = np.ascontiguousarray(np.asarray(edges, dtype=np.uint32).reshape(-1))
        pl = None if plabels is None else np.ascontiguousarray(plabels, dtype=np.uint32)
        roots = np.ascontiguousarray(roots, dtype=np.uint32)
        out = np.zeros(roots.size, np.uint64)
        st = lib().og_match_roots(self._h, nv, e.size // 2, e, None if pl is None else pl.ctypes.data,
                                  int(bool(induced)), roots.size, roots, out, threads)
        if st != 0:
            raise ValueError(f"oracle og_match_roots status {st}")
        return out

    def match_levels(self, nv: int, edges, plabels=None, plan=None, threads: int = 0):
        """Per-level SM statistics (O-2b) in the matching order and with the order
        constraints of ``plan`` (default: this oracle's own R10/R16 planner,
        plan_r10_r16): (N, G, C) lists indexed by the number t of placed positions,
        N[nv] = the match count.  Feeds SURVEY §8(d)'s algorithmic bytes of SM."""
        order, lt, gt = plan if plan is not None else plan_r10_r16(nv, edges, plabels)
        e = np.ascontiguousarray(np.asarray(edges, dtype=np.uint32).reshape(-1))
        pl = None if plabels is None else np.ascontiguousarray(plabels, dtype=np.uint32)
        N = np.zeros(nv + 1, np.uint64)
        G = np.zeros(nv + 1, np.uint64)
        Cc = np.zeros(nv + 1, np.uint64)
        st = lib().og_match_levels(self._h, nv, e.size // 2, e, None if pl is None else pl.ctypes.data,
                                   np.asarray(order, np.uint32), np.asarray(lt, np.uint32),
                                   np.asarray(gt, np.uint32), threads, N, G, Cc)
        if st != 0:
            raise ValueError(f"oracle og_match_levels status {st}")
        return [int(x) for x in N], [int(x) for x in G], [int(x) for x in Cc]

    def fpm(self, l: int, minsup: int, method: str = "shapes", threads: int = 0,
            pattern_cap: int = 1 << 16):
        """Frequent patterns as a sorted list of (ne, nv, labels, edges, support, instances).

        ``instances`` is the number of connected edge sets mapped to the pattern."""
        cap = 1 << 14
        while True:
            out = np.zeros(cap * REC, np.uint64)
            n = lib().og_fpm(self._h, l, minsup, 0 if method == "shapes" else 1, threads, cap, out,
                             pattern_cap)
            if n < 0:
                raise ValueError(f"oracle og_fpm status {n}")
            if n <= cap:
                break
            cap = n
        res = []
        for i in range(n):
            r = out[i * REC:(i + 1) * REC]
            ne, nv = int(r[0]), int(r[1])
            res.append((ne, nv, tuple(int(x) for x in r[2:2 + nv]),
                        tuple((int(r[7 + 2 * e]), int(r[8 + 2 * e])) for e in range(ne)), int(r[15]),
                        int(r[16])))
        return res

    def pattern_mni(self, nv: int, edges, plabels=None, threads: int = 0) -> int:
        e = np.ascontiguousarray(np.asarray(edges, dtype=np.uint32).reshape(-1))
        pl = None if plabels is None else np.ascontiguousarray(plabels, dtype=np.uint32)
        s = C.c_uint64()
        st = lib().og_pattern_mni(self._h, nv, e.size // 2, e, None if pl is None else pl.ctypes.data,
                                  threads, C.byref(s))
        if st != 0:
            raise ValueError(f"oracle og_pattern_mni status {st}")
        return int(s.value)


def automorphisms(nv: int, edges, plabels=None):
    """Aut_L(P): every label- and edge-preserving permutation (brute force over nv!)."""
    import itertools
    E = {frozenset(e) for e in edges}
    lab = list(plabels) if plabels is not None else [0] * nv
    return [p for p in itertools.permutations(range(nv))
            if all(lab[p[i]] == lab[i] for i in range(nv)) and {frozenset((p[a], p[b])) for a, b in edges} == E]


def plan_r10_r16(nv: int, edges, plabels=None):
    """The oracle's own statement of the method's matching order and symmetry breaking
    (readings R10, R16; PAPER.md L176 leaves the order open):
      order: the max-degree pattern vertex first (ties: lower id), then repeatedly the
             unplaced vertex with the most placed neighbours (ties: higher degree, then
             lower id), among those with at least one placed neighbour;
      constraints: stabilizer chain of Aut_L(P) along the order -- for the vertex v at
             position t, every other u in v's orbit under the automorphisms fixing the
             vertices of positions < t must satisfy phi(v) < phi(u).
    Returns (order, lt, gt): lt[t] / gt[t] = bitmask of earlier positions j with
    phi(j) < phi(t) / phi(t) < phi(j)."""
    deg = [0] * nv
    adj = [set() for _ in range(nv)]
    for a, b in edges:
        adj[a].add(b)
        adj[b].add(a)
    for v in range(nv):
        deg[v] = len(adj[v])
    order = [max(range(nv), key=lambda v: (deg[v], -v))]
    while len(order) < nv:
        placed = set(order)
        cand = [v for v in range(nv) if v not in placed and adj[v] & placed]
        order.append(max(cand, key=lambda v: (len(adj[v] & placed), deg[v], -v)))
    pos = {v: t for t, v in enumerate(order)}
    auts = automorphisms(nv, edges, plabels)
    lt, gt = [0] * nv, [0] * nv
    fixed = []
    group = auts
    for t, v in enumerate(order):
        group = [p for p in group if all(p[x] == x for x in fixed)]
        orbit = {p[v] for p in group}
        for u in orbit - {v}:
            # phi(v) < phi(u): recorded at the later of the two positions
            if pos[u] > t:
                lt[pos[u]] |= 1 << t
            else:
                gt[t] |= 1 << pos[u]
        fixed.append(v)
    return order, lt, gt
