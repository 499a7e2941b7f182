"""B200-native GAMMA hot path: embedding-table extension for graph pattern mining.

Thin Python binding over the C ABI in ``include/gamma.h`` (libgamma.so, built
in-tree for sm_100a).  This module only marshals arguments: every step of the
path (CSR build, extension, intersection, filtering, compaction, aggregation)
runs in the library's CUDA kernels.  PyTorch supplies the device allocator, the
stream and (for world > 1) the process group; there is no CPU fallback -- if the
library or a CUDA device is missing, calls raise ``GammaError``/``ImportError``.

The C names are re-exported 1:1 (``gamma_ctx_create``, ``gamma_load_edges``,
``gamma_kclique``, ``gamma_match``, ``gamma_fpm`` ...) and wrapped by
:class:`Context` / :class:`Graph`.
"""
from __future__ import annotations

import ctypes as C
import os
import sys
import weakref
from typing import Optional

import numpy as np

from . import _native as N

_lib = N.load()

# 1:1 C entry points
for _name, _res, _args in N.SIGNATURES:
    globals()[_name] = getattr(_lib, _name)

__all__ = ["Context", "Graph", "GammaError", "library_path", "pattern_plan"] + [s[0] for s in N.SIGNATURES]


def library_path() -> str:
    return N.LIB_PATH


# The connected graphs on 3 and 4 vertices (up to isomorphism), for Graph.motifs.
MOTIFS = {
    3: {"wedge": [(0, 1), (1, 2)], "triangle": [(0, 1), (1, 2), (0, 2)]},
    4: {"path": [(0, 1), (1, 2), (2, 3)], "star": [(0, 1), (0, 2), (0, 3)],
        "c4": [(0, 1), (1, 2), (2, 3), (3, 0)], "tailed_triangle": [(0, 1), (0, 2), (1, 2), (2, 3)],
        "diamond": [(0, 1), (0, 2), (1, 2), (1, 3), (2, 3)],
        "k4": [(0, 1), (0, 2), (0, 3), (1, 2), (1, 3), (2, 3)]},
}


class GammaError(RuntimeError):
    def __init__(self, status: int, where: str):
        msg = (_lib.gamma_last_error() or b"").decode(errors="replace")
        super().__init__(f"{where}: status {status}: {msg}")
        self.status = status


def _check(st: int, where: str):
    if st != N.GAMMA_OK:
        raise GammaError(st, where)


def _ptr(x, dtype):
    """(pointer, keepalive, length) for a numpy array or torch tensor (host or CUDA)."""
    if x is None:
        return None, None, 0
    try:
        import torch
        if isinstance(x, torch.Tensor):
            want = {np.uint32: (torch.int32, torch.uint32), np.uint64: (torch.int64, torch.uint64)}[dtype]
            assert x.dtype in want, f"expected {dtype.__name__}-compatible tensor, got {x.dtype}"
            x = x.contiguous()
            return x.data_ptr(), x, x.numel()
    except ImportError:
        pass
    a = np.ascontiguousarray(x, dtype=dtype)
    return a.ctypes.data, a, a.size


def _pattern(nv, edges, labels=None, induced=False):
    e = np.ascontiguousarray(np.asarray(edges, dtype=np.uint32).reshape(-1))
    p = N.gamma_pattern()
    p.nv = nv
    p.ne = e.size // 2
    p.edges = e.ctypes.data_as(C.POINTER(C.c_uint32))
    keep = [e]
    if labels is not None:
        lab = np.ascontiguousarray(labels, dtype=np.uint32)
        p.labels = lab.ctypes.data_as(C.POINTER(C.c_uint32))
        keep.append(lab)
    p.induced = 1 if induced else 0
    return p, keep


def pattern_plan(nv: int, edges, labels=None, induced: bool = False) -> dict:
    """Host-only planner output: matching order, |Aut_L|, symmetry constraints."""
    p, keep = _pattern(nv, edges, labels, induced)
    info = N.gamma_plan_info()
    _check(_lib.gamma_pattern_plan(C.byref(p), C.byref(info)), "gamma_pattern_plan")
    return {"nv": info.nv, "order": [info.order[i] for i in range(nv)],
            "backward_mask": [info.backward_mask[i] for i in range(nv)],
            "less_mask": [info.less_mask[i] for i in range(nv)],
            "greater_mask": [info.greater_mask[i] for i in range(nv)], "aut": int(info.aut)}


def allreduce_sum_inplace(arr: np.ndarray) -> None:
    """SUM all-reduce of a host uint64 array over the default process group (a CUDA
    int64 tensor for NCCL, a CPU one for gloo); wrapping int64 sums equal uint64 sums."""
    import torch
    import torch.distributed as dist
    t = torch.from_numpy(arr.view(np.int64).copy())
    if dist.get_backend() == "nccl":
        t = t.cuda()
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    arr[:] = t.cpu().numpy().view(np.uint64)


def alltoall_tensors(send, recv) -> None:
    """all_to_all_single over the default group; gloo goes through host copies."""
    import torch.distributed as dist
    if dist.get_backend() == "nccl" or not send.is_cuda:
        dist.all_to_all_single(recv, send)
    else:
        rc = send.new_empty(send.shape, device="cpu")
        dist.all_to_all_single(rc, send.cpu())
        recv.copy_(rc)


def make_allreduce_callback(device: int = 0):
    """The ctx's ``allreduce_sum_u64`` callback: an in-place SUM of n uint64 values
    held in host memory.  Returns the ctypes function."""

    def _allreduce(buf, n, user):
        try:
            if n:
                allreduce_sum_inplace(np.ctypeslib.as_array(buf, shape=(n,)))
            return 0
        except Exception:   # noqa: BLE001 -- reported as a gamma_status
            return N.GAMMA_E_CUDA

    return N.ALLREDUCE_FN(_allreduce)


class _DeviceView:
    """Zero-copy int32 view of a library-owned device buffer (CUDA array interface)."""

    def __init__(self, ptr: int, n: int):
        self.__cuda_array_interface__ = {"shape": (int(n),), "typestr": "<i4", "data": (int(ptr), False),
                                         "version": 3, "strides": None}


def make_alltoall_callback(device: int = 0):
    """The ctx's ``alltoall_u32`` callback (gamma_fpm's domain-bitmap exchange): device
    buffers of world * n_per_rank words, exchanged with all_to_all_single."""
    import torch
    import torch.distributed as dist

    def _alltoall(send, recv, n, user):
        try:
            total = dist.get_world_size() * int(n)
            if total:
                s = torch.as_tensor(_DeviceView(send, total), device=torch.device("cuda", device))
                r = torch.as_tensor(_DeviceView(recv, total), device=torch.device("cuda", device))
                alltoall_tensors(s, r)
                torch.cuda.synchronize(device)
            return 0
        except Exception:   # noqa: BLE001 -- reported as a gamma_status
            return N.GAMMA_E_CUDA

    return N.ALLTOALL_FN(_alltoall)


class Context:
    """A gamma_ctx bound to one CUDA device, its stream and allocator.

    ``rank``/``world`` partition root chunks across processes; with a
    ``torch.distributed`` process group initialised and ``world > 1`` the counts are
    all-reduced (SUM) through it inside the C call (callback), else partial.
    """

    def __init__(self, device: int = 0, rank: Optional[int] = None, world: Optional[int] = None,
                 use_torch: bool = True, hbm_budget_bytes: int = 0, host_spill_bytes: int = 0,
                 time_kernels: bool = False, flags: int = 0, reduce: bool = True,
                 torch_alloc: Optional[bool] = None, dag_cache_bytes: int = 0):
        self._keep = []
        if torch_alloc is None:   # GAMMA_ALLOC=native: the library's stream-ordered pool
            torch_alloc = os.environ.get("GAMMA_ALLOC", "torch") != "native"
        self._graphs = weakref.WeakSet()
        d = N.gamma_ctx_desc()
        d.device = device
        self._torch = None
        if use_torch:
            import torch
            self._torch = torch
        dist_ok = False
        if self._torch is not None:
            import torch.distributed as dist
            dist_ok = dist.is_available() and dist.is_initialized()
            if rank is None and dist_ok:
                rank, world = dist.get_rank(), dist.get_world_size()
        d.rank = rank or 0
        d.world = world or 1
        if self._torch is not None and self._torch.cuda.is_available():
            torch = self._torch
            stream = torch.cuda.current_stream(device)
            d.stream = C.c_void_p(stream.cuda_stream)
        if self._torch is not None and self._torch.cuda.is_available() and torch_alloc:
            torch = self._torch
            dev = device

            def _alloc(size, strm, user):
                try:
                    return torch.cuda.caching_allocator_alloc(int(size), dev, int(strm or 0))
                except Exception:   # noqa: BLE001 -- reported as E_NOMEM by the library
                    return None

            def _free(p, user):
                torch.cuda.caching_allocator_delete(int(p))

            fa, ff = N.ALLOC_FN(_alloc), N.FREE_FN(_free)
            d.dev_alloc, d.dev_free = fa, ff
            self._keep += [fa, ff]
        if reduce and d.world > 1 and dist_ok:
            fr = make_allreduce_callback(device)
            d.allreduce_sum_u64 = fr
            self._keep.append(fr)
            if self._torch is not None and self._torch.cuda.is_available():
                fa2a = make_alltoall_callback(device)
                d.alltoall_u32 = fa2a
                self._keep.append(fa2a)
        d.hbm_budget_bytes = hbm_budget_bytes
        d.host_spill_bytes = host_spill_bytes
        d.dag_cache_bytes = dag_cache_bytes
        d.flags = flags | (N.GAMMA_FLAG_TIME_KERNELS if time_kernels else 0)
        self.desc = d
        h = C.c_void_p()
        _check(_lib.gamma_ctx_create(C.byref(d), C.byref(h)), "gamma_ctx_create")
        self._h = h
        self.device, self.rank, self.world = device, d.rank, d.world

    @property
    def handle(self):
        return self._h

    def close(self):
        """Free every live graph of this context, then the context itself (a graph
        must never outlive its context, whatever order the garbage collector picks)."""
        if getattr(self, "_h", None):
            for g in list(getattr(self, "_graphs", ())):
                g.free()
            _lib.gamma_ctx_destroy(self._h)
            self._h = None

    def __del__(self, _finalizing=sys.is_finalizing):   # bound at definition: globals may be gone
        # at interpreter shutdown the allocator callbacks (into torch) may already be
        # gone: leak instead of calling back into a half-finalised interpreter
        if _finalizing():
            return
        try:
            self.close()
        except Exception:   # noqa: BLE001
            pass

    def load_edges(self, n: int, src, dst, labels=None) -> "Graph":
        ps, ks, m = _ptr(src, np.uint32)
        pd, kd, m2 = _ptr(dst, np.uint32)
        assert m == m2, "src and dst differ in length"
        pl, kl, _ = _ptr(labels, np.uint32)
        g = C.c_void_p()
        _check(_lib.gamma_load_edges(self._h, int(n), ps, pd, int(m), pl, C.byref(g)), "gamma_load_edges")
        return Graph(self, g)

    def load_csr(self, n: int, row_ptr, col, labels=None) -> "Graph":
        pr, kr, _ = _ptr(row_ptr, np.uint64)
        pc, kc, _ = _ptr(col, np.uint32)
        pl, kl, _ = _ptr(labels, np.uint32)
        g = C.c_void_p()
        _check(_lib.gamma_load_csr(self._h, int(n), pr, pc, pl, C.byref(g)), "gamma_load_csr")
        return Graph(self, g)

    def stats(self) -> dict:
        s = N.gamma_run_stats()
        _check(_lib.gamma_get_stats(self._h, C.byref(s)), "gamma_get_stats")
        classes = {}
        for i in range(s.n_classes):
            name = bytes(s.name[i]).split(b"\0")[0].decode()
            classes[name] = {"launches": int(s.launches[i]), "ms": float(s.ms[i]),
                             "alg_bytes": int(s.alg_bytes[i])}
        return {"classes": classes, "level_entries": [int(x) for x in s.level_entries],
                "list_elems": int(s.list_elems), "chunks": int(s.chunks), "retries": int(s.retries),
                "spilled_bytes": int(s.spilled_bytes), "total_launches": int(s.total_launches),
                "wall_ms": float(s.wall_ms)}


class Graph:
    """A gamma_graph (symmetric CSR + degree-ordered DAG + labels) in HBM."""

    def __init__(self, ctx: Context, h):
        self.ctx = ctx
        self._h = h
        ctx._graphs.add(self)

    def free(self):
        if getattr(self, "_h", None):
            if getattr(self.ctx, "_h", None):   # the context still exists
                _lib.gamma_graph_free(self._h)
            self._h = None

    def __del__(self, _finalizing=sys.is_finalizing):
        if _finalizing():
            return
        try:
            self.free()
        except Exception:   # noqa: BLE001
            pass

    def info(self) -> dict:
        i = N.gamma_graph_info()
        _check(_lib.gamma_graph_get_info(self._h, C.byref(i)), "gamma_graph_get_info")
        return {"n": i.n, "m": i.m, "max_degree": i.max_degree, "max_out_degree": i.max_out_degree,
                "device_bytes": i.device_bytes, "build_ms": i.build_ms}

    def csr(self, which: str = "sym"):
        inf = self.info()
        w = 0 if which == "sym" else 1
        ne = 2 * inf["m"] if w == 0 else inf["m"]
        rp = np.empty(inf["n"] + 1, np.uint64)
        col = np.empty(max(ne, 1), np.uint32)
        _check(_lib.gamma_graph_copy_csr(self._h, w, rp.ctypes.data, col.ctypes.data), "gamma_graph_copy_csr")
        return rp, col[:ne]

    def kclique(self, k: int) -> int:
        c = C.c_uint64()
        _check(_lib.gamma_kclique(self._h, int(k), C.byref(c)), "gamma_kclique")
        return int(c.value)

    def kclique_multi(self, ks) -> list:
        """Counts for several clique sizes from one call (one bitmap pass when possible)."""
        ka = np.ascontiguousarray(ks, dtype=np.uint32)
        out = np.zeros(len(ka), np.uint64)
        _check(_lib.gamma_kclique_multi(self._h, len(ka), ka.ctypes.data, out.ctypes.data), "gamma_kclique_multi")
        return [int(x) for x in out]

    def kclique_roots(self, k: int, roots) -> np.ndarray:
        pr, kr, nr = _ptr(roots, np.uint32)
        out = np.zeros(nr, np.uint64)
        _check(_lib.gamma_kclique_roots(self._h, int(k), nr, pr, out.ctypes.data), "gamma_kclique_roots")
        return out

    def match(self, nv: int, edges, labels=None, induced: bool = False):
        """(count of distinct subgraphs, mappings = count * |Aut_L|)."""
        p, keep = _pattern(nv, edges, labels, induced)
        c, mp = C.c_uint64(), C.c_uint64()
        _check(_lib.gamma_match(self._h, C.byref(p), C.byref(c), C.byref(mp)), "gamma_match")
        return int(c.value), int(mp.value)

    def match_many(self, queries) -> list:
        """Several queries in one call (gamma_match_batch: level chains on concurrent
        streams): queries = [(nv, edges, labels or None, induced), ...] ->
        [(count, mappings), ...] in order."""
        qs = list(queries)
        if not qs:
            return []
        arr = (N.gamma_pattern * len(qs))()
        keep = []
        for i, q in enumerate(qs):
            nv, e = q[0], q[1]
            lab = q[2] if len(q) > 2 else None
            ind = bool(q[3]) if len(q) > 3 else False
            p, k = _pattern(nv, e, lab, ind)
            arr[i] = p
            keep.append(k)
        counts = np.zeros(len(qs), np.uint64)
        maps = np.zeros(len(qs), np.uint64)
        _check(_lib.gamma_match_batch(self._h, len(qs), arr, counts.ctypes.data, maps.ctypes.data),
               "gamma_match_batch")
        return [(int(c), int(m)) for c, m in zip(counts, maps)]

    def motifs(self, k: int) -> dict:
        """Motif counts: induced counts of every connected unlabeled k-vertex pattern
        (k = 3, 4), one gamma_match(induced=1) call each."""
        if k not in MOTIFS:
            raise ValueError("motifs: k must be 3 or 4")
        return {name: self.match(k, e, induced=True)[0] for name, e in MOTIFS[k].items()}

    def fpm_array(self, max_edges: int, minsup: int) -> np.ndarray:
        """Frequent patterns as a numpy structured array (fields nv, ne, labels[8],
        edges[8][2], support, instances), one record per pattern in the library's order --
        one copy of the result, no per-pattern Python objects."""
        t = self.ctx._torch
        if t is not None and t.cuda.is_available():
            # the MNI domain pool is sized from free HBM: return the context's kept
            # buffers to the caching allocator, then its idle blocks (e.g. the previous
            # call's pool) to the device
            _check(_lib.gamma_ctx_trim(self.ctx._h), "gamma_ctx_trim")
            t.cuda.empty_cache()
        r = C.POINTER(N.gamma_fpm_result)()
        _check(_lib.gamma_fpm(self._h, int(max_edges), int(minsup), C.byref(r)), "gamma_fpm")
        try:
            res = r.contents
            dt = np.dtype([("nv", np.uint32), ("ne", np.uint32), ("labels", np.uint32, 8),
                           ("edges", np.uint8, (8, 2)), ("support", np.uint64), ("instances", np.uint64)],
                          align=True)
            assert dt.itemsize == C.sizeof(N.gamma_fpm_pattern)
            if res.n == 0:
                return np.zeros(0, dt)
            buf = (C.c_char * (res.n * dt.itemsize)).from_address(C.addressof(res.pats.contents))
            return np.frombuffer(buf, dtype=dt).copy()
        finally:
            _lib.gamma_fpm_result_free(r)

    def fpm(self, max_edges: int, minsup: int, instances: bool = False):
        """Frequent patterns: sorted list of (ne, nv, labels, edges, support); with
        ``instances`` (needs a Context created with GAMMA_FLAG_FPM_INSTANCES) each
        tuple also carries the pattern's instance count (connected edge sets)."""
        arr = self.fpm_array(max_edges, minsup)
        out = []
        for pt in arr:
            nv, ne = int(pt["nv"]), int(pt["ne"])
            out.append((ne, nv, tuple(int(x) for x in pt["labels"][:nv]),
                        tuple((int(pt["edges"][e][0]), int(pt["edges"][e][1])) for e in range(ne)),
                        int(pt["support"])) + ((int(pt["instances"]),) if instances else ()))
        return out
