// device_common.cuh -- warp-level building blocks shared by the extension kernels
// (kclique.cu, match.cu, fpm.cu): in-order warp compaction, sorted-list probes and
// the Opt 1 per-warp memory-block pool.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

namespace gamma_impl {

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// Branch-free lower-bound membership test in a sorted array of len >= 1 entries.
template <class P>
__device__ __forceinline__ bool sorted_contains(P s, uint32_t len, uint32_t y) {
  uint32_t base = 0, n = len;
  while (n > 1) {
    uint32_t half = n >> 1;
    base = (s[base + half] <= y) ? base + half : base;
    n -= half;
  }
  return s[base] == y;
}

// Copies of sorted_contains per global-memory call-site kind, so ncu's source page
// attributes them separately: a hub child's list probed from the short side, and the
// (child, L_m element) pair probes of a short L_m.
template <class P>
__device__ __forceinline__ bool contains_hub(P s, uint32_t len, uint32_t y) {
  uint32_t base = 0, n = len;
  while (n > 1) {
    uint32_t half = n >> 1;
    base = (s[base + half] <= y) ? base + half : base;
    n -= half;
  }
  return s[base] == y;
}
template <class P>
__device__ __forceinline__ bool contains_pair(P s, uint32_t len, uint32_t y) {
  uint32_t base = 0, n = len;
  while (n > 1) {
    uint32_t half = n >> 1;
    base = (s[base + half] <= y) ? base + half : base;
    n -= half;
  }
  return s[base] == y;
}

// First index i in [0, len) with s[i] > y (upper bound), len if none.
template <class P>
__device__ __forceinline__ uint32_t upper_bound_idx(P s, uint32_t len, uint32_t y) {
  uint32_t lo = 0, hi = len;
  while (lo < hi) {
    uint32_t mid = (lo + hi) >> 1;
    if (s[mid] <= y) lo = mid + 1; else hi = mid;
  }
  return lo;
}

// Opt 1: a warp owns one block of the level's vid array and one block of its group
// table at a time; a fresh block is taken from the pool with one atomicAdd on the
// level cursor.  All functions are warp-uniform (every lane calls them).
struct BlockPool {
  unsigned long long *cursor;   // level cursor (device)
  unsigned long long *overflow; // set to 1 when the pool is exhausted
  uint64_t cap;                 // capacity in slots
  uint32_t block;               // block size in slots
};

struct WarpBlock {
  uint64_t b = 0, e = 0;
};

// Reserve f contiguous slots (f <= pool.block) in the warp's current block.
__device__ __forceinline__ bool wb_reserve(WarpBlock &w, const BlockPool &p, uint32_t f, int lane,
                                           uint64_t &pos) {
  if (w.b + f > w.e) {
    unsigned long long nb = 0;
    if (lane == 0) nb = atomicAdd(p.cursor, (unsigned long long)p.block);
    nb = __shfl_sync(0xffffffffu, nb, 0);
    if (nb + p.block > p.cap) {
      if (lane == 0) atomicExch(p.overflow, 1ull);
      return false;
    }
    w.b = nb;
    w.e = nb + p.block;
  }
  pos = w.b;
  w.b += f;
  return true;
}

// Group tables are read densely by the next level, so slots a warp abandons when
// it moves to a fresh block must be marked empty first.  Call before wb_reserve;
// empty(slot) writes the "empty group" marker of one slot.
template <class F>
__device__ __forceinline__ void wb_retire_tail(const WarpBlock &w, uint32_t f, int lane, F empty) {
  if (w.b + f > w.e)
    for (uint64_t s = w.b + lane; s < w.e; s += 32) empty(s);
}

// Reserve ub slots directly from the pool (outputs that may exceed a block).
__device__ __forceinline__ bool pool_reserve(const BlockPool &p, uint64_t ub, int lane, uint64_t &pos) {
  unsigned long long nb = 0;
  if (lane == 0) nb = atomicAdd(p.cursor, (unsigned long long)ub);
  nb = __shfl_sync(0xffffffffu, nb, 0);
  if (nb + ub > p.cap) {
    if (lane == 0) atomicExch(p.overflow, 1ull);
    return false;
  }
  pos = nb;
  return true;
}

}  // namespace gamma_impl
