"""The R-MAT recipe of ``gamma_gen.rmat`` evaluated with torch int64 tensors, so that
graphs too large for a host-side numpy pass (C5: 2^26 vertices, ~2·10^9 samples) can
be drawn directly in device memory.  Same counter-based words, thresholds and vertex
bijection as the numpy version; ``tests/test_gen.py`` checks the two agree element by
element (torch on CPU).  Like the rest of ``gamma_gen`` it holds no arithmetic of the
method, only input drawing.

int64 arithmetic wraps like uint64 for +, * and xor; the logical right shifts of the
unsigned recipe are an arithmetic shift followed by a mask of the top bits.
"""
from __future__ import annotations

import numpy as np
import torch

from . import _key, splitmix64

_GOLD = 0x9E3779B97F4A7C15
_M1 = 0xBF58476D1CE4E5B9
_M2 = 0x94D049BB133111EB


def _s64(x: int) -> int:
    """uint64 constant -> the int64 with the same bits."""
    x &= (1 << 64) - 1
    return x - (1 << 64) if x >= 1 << 63 else x


def _srl(x: torch.Tensor, r: int) -> torch.Tensor:
    """Logical right shift of int64 bit patterns."""
    return (x >> r) & ((1 << (64 - r)) - 1)


def splitmix64_t(x: torch.Tensor) -> torch.Tensor:
    z = x + _s64(_GOLD)
    z = (z ^ _srl(z, 30)) * _s64(_M1)
    z = (z ^ _srl(z, 27)) * _s64(_M2)
    return z ^ _srl(z, 31)


def permute_bits_t(y: torch.Tensor, bits: int, seed: int) -> torch.Tensor:
    """Twin of ``gamma_gen.permute_bits`` (bits <= 31, so every product is masked)."""
    if bits == 0:
        return torch.zeros_like(y)
    mask = (1 << bits) - 1
    k = [int(v) for v in splitmix64(np.array([int(seed) * 7 + 3, int(seed) * 7 + 4, int(seed) * 7 + 5],
                                             dtype=np.uint64))]
    m1, m2 = (k[1] | 1) & mask, (k[2] | 1) & mask   # only the low bits survive the mask
    r = max(1, (bits + 1) // 2)
    y = (y ^ (k[0] & mask)) & mask
    y = (y * m1) & mask
    y = y ^ (y >> r)
    y = (y * m2) & mask
    y = y ^ (y >> r)
    y = (y * m1) & mask
    return y


def rmat_torch(scale: int, samples: int, a: float, b: float, c: float, seed: int,
               device="cuda", permute: bool = True, block: int = 1 << 26):
    """Raw R-MAT samples as two int32 tensors (uint32 bit patterns) on ``device``."""
    assert 1 <= scale <= 31
    ta, tb, tc = int(a * 2 ** 32), int((a + b) * 2 ** 32), int((a + b + c) * 2 ** 32)
    key = int(_key(seed, 0x52))
    words = (scale + 1) // 2
    src = torch.empty(samples, dtype=torch.int32, device=device)
    dst = torch.empty(samples, dtype=torch.int32, device=device)
    for lo in range(0, samples, block):
        hi = min(samples, lo + block)
        i = torch.arange(lo, hi, dtype=torch.int64, device=device)
        base = i * words + _s64(key)
        s = torch.zeros(hi - lo, dtype=torch.int64, device=device)
        d = torch.zeros_like(s)
        for w in range(words):
            h = splitmix64_t(base + w)
            for half in range(2):
                j = 2 * w + half
                if j >= scale:
                    break
                u = _srl(h, 32 * half) & 0xFFFFFFFF
                bit = scale - 1 - j
                sbit = (u >= tb).to(torch.int64)
                dbit = (((u >= ta) & (u < tb)) | (u >= tc)).to(torch.int64)
                s |= sbit << bit
                d |= dbit << bit
            del h
        if permute:
            s = permute_bits_t(s, scale, seed)
            d = permute_bits_t(d, scale, seed)
        src[lo:hi] = s.to(torch.int32)
        dst[lo:hi] = d.to(torch.int32)
        del s, d, i, base
    return src, dst


def config_graph_torch(name: str, seed: int = 1, device="cuda"):
    """``gamma_gen.config_graph`` drawn with torch on ``device`` (unlabeled configs):
    (n, src, dst) with int32 tensors holding the uint32 bit patterns."""
    from . import CONFIGS
    sc, ns, a, b, c, L = CONFIGS[name]
    assert L == 1, "labeled configs are drawn on the host"
    src, dst = rmat_torch(sc, ns, a, b, c, seed, device=device)
    return 1 << sc, src, dst
