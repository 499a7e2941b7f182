// kclique_bitmap.cu -- k-clique counting, local-bitmap fast path (DFS inside a root).
//
// Opt 2 of PAPER.md (L269-278) computes L_m, the intersection of the prefix's
// lists, once per group and intersects every child's list with it.  Under the
// degree-ordered DAG, every candidate set below a root v is a subset of the root's
// run R = N+(v): C(v, c1, ..., ct) = R ∩ N+(c1) ∩ ... ∩ N+(ct).  So this path
// intersects each child's list with R exactly once (the depth-2 extension, the only
// step that reads adjacency lists) and stores the result as a bitmap row over R's
// positions; every deeper extension is then a W-word AND of rows, and the last one
// is a popcount (the last extension is counted, not stored).  The
// embedding table below the root is held as these bitmaps, in shared memory, and
// walked depth-first (BFS across roots, DFS inside a root).
//
// Teams: one warp per root for |R| <= 128 (rows of <= 4 words), one CTA per root for
// 128 < |R| <= 512 (<= 16 words).  Work inside a root is split into the root's
// triangles (v, R[j1], R[j2]) so the team stays balanced.  Roots whose 4-clique
// count exceeds a cut (k >= 6 only, where the DFS below a triangle is deep) are not
// expanded by their team: they are cut into parts that separate CTAs take from a
// work list in a second launch (hub splitting, SURVEY.md §7 "skew").  Longer runs
// (and k > 12) use the ET-level path in kclique.cu.
#include <algorithm>
#include <cstdlib>

#include "device_common.cuh"
#include "internal.cuh"

namespace gamma_impl {

namespace {

// Min resident CTAs per SM for the team kernels with k <= 6 (KM = 6).  Shared memory
// (8 warp teams x 6.2 KB, or one CTA team) already limits residency to 4 CTAs, so 4
// leaves the registers uncapped (64); round 1's 5 (51 registers) predates the 4-slot
// bucket table and now only spilled (C2 same box: 7.48 ms at 5, 6.46 at 4).
// Tuning knob: nvcc -DGAMMA_BM_MINB=n.
#ifndef GAMMA_BM_MINB
#define GAMMA_BM_MINB 4
#endif
#define GAMMA_BM_BOUNDS(KM) __launch_bounds__(256, (KM) <= 6 ? GAMMA_BM_MINB : 1)

// Compile-time variants (A/B builds, build.py tag=...; B200 r02 same-box A/B in
// profiles/kcl_ab_r02.md): GAMMA_KCL_LEAF_BAL balanced lane-group leaf walk (default:
// per-word walk -- faster with id-ordered runs, whose bits spread over the words),
// GAMMA_KCL_NO_PAIRS stream the lists of runs <= 32 too (default: pair probes there).
// (The slot-pair hash probe lost to the 4-slot bucket, session g, and was removed.)
#ifndef GAMMA_KCL_LEAF_BAL
#define GAMMA_KCL_LEAF_BAL 0
#endif
#ifndef GAMMA_KCL_TILES   // streamed row build: 32-element tiles whose loads are in flight together
                          // (C2 same box: 2 tiles 5.65 ms/step, 4 5.59, 8 5.83)
#define GAMMA_KCL_TILES 4
#endif
#ifndef GAMMA_KCL_PAIR_U   // rows per lane group whose pair searches run in lock step
#define GAMMA_KCL_PAIR_U 2
#endif
// GAMMA_KCL_PAIR_SORT: runs <= 32 sorted by (degree, id) in the warp, only the pairs above
// the diagonal searched (half the searches, one more gather round trip and the sort;
// C2 same box 6.20 vs 6.14 ms/step, heavy 40.2 vs 40.5: off)
#ifndef GAMMA_KCL_PAIR_SORT
#define GAMMA_KCL_PAIR_SORT 0
#endif
#ifndef GAMMA_KCL_SM_DFS   // warp teams, k <= 6: state-machine DFS (0: nested loops per item)
#define GAMMA_KCL_SM_DFS 1
#endif
#ifndef GAMMA_KCL_NO_PAIRS
#define GAMMA_KCL_NO_PAIRS 0
#endif

constexpr int kMaxStack = 10;        // DFS levels below the first child: k <= 12
constexpr uint32_t kPartCost = 4096; // 4-cliques per heavy-root part (k >= 6; x4 at k = 5)
constexpr uint32_t kMaxParts = 4096;
constexpr uint32_t kSlotB = 520;     // root-rows slot: header 4 + P (<= 513) -> B at 520
constexpr uint32_t kSlotWords = kSlotB + 512 * 17;

// The DAG columns: HBM-resident (base) or, GAMMA_FLAG_HOST_DAG, paged (pages[p] = the
// device address of page p: an HBM cache frame or mapped pinned host memory)
// (PAGED is a kernel template parameter: the HBM path pays nothing for the host mode)
struct DagCol {
  const uint32_t *base;
  const uint64_t *pages;
  template <bool PAGED>
  __device__ __forceinline__ uint32_t at(uint64_t i) const {
    if constexpr (PAGED)
      return __ldg(reinterpret_cast<const uint32_t *>(pages[i >> kDagPageShift]) + (i & ((1u << kDagPageShift) - 1u)));
    else
      return __ldg(base + i);
  }
};

// lower-bound membership of y in col[b, b + len) (len >= 1)
template <bool PAGED>
__device__ __forceinline__ bool col_contains(const DagCol &col, uint64_t b, uint32_t len, uint32_t y) {
  uint32_t base = 0, n = len;
  while (n > 1) {
    const uint32_t half = n >> 1;
    base = (col.at<PAGED>(b + base + half) <= y) ? base + half : base;
    n -= half;
  }
  return col.at<PAGED>(b + base) == y;
}

struct BmArgs {
  const uint64_t *dag_ptr;
  DagCol dag_col;
  const uint32_t *roots;
  uint64_t nroots;
  uint32_t k;
  uint32_t len_lo, len_hi;    // this launch handles roots with len_lo < |R| <= len_hi
  unsigned long long *ctrl;
  unsigned long long *per_root;
  // hub splitting (k >= 6): roots with more than heavy_cut 4-cliques are deferred
  uint64_t heavy_cut;         // 0: never defer
  uint2 *parts;               // (root-rows slot, part | nparts << 16)
  uint32_t parts_cap;
  uint32_t part_cost;         // 4-cliques per part
  // the deferred roots' rows, kept by the team that built them (the parts read them
  // instead of rebuilding): slot = {L, W, BS, root index} + P[0..L] at 4 + B at kSlotB
  uint32_t *root_rows;
  uint32_t root_rows_cap;     // slots
  uint64_t root_base;         // index of roots[0] in the full root list (parts are absolute)
  uint32_t multi;             // count every clique size kmin..k at once (gamma_kclique_multi)
  uint32_t kmin;              // multi: smallest size asked for (>= 3); shorter runs are skipped
  uint32_t trim;              // trim each child's list at the run's largest id (GAMMA_KCL_NO_TRIM: off)
  uint32_t *wide_rows;        // wide runs: per-CTA global row scratch (wide_stride words each)
  uint64_t wide_stride;
  const uint64_t *row_ptr;    // symmetric CSR offsets (degrees of the orientation order);
                              // nullptr in rank space, where the id order is that order
  unsigned long long *work;   // this launch's work cursor (its own word when launches run concurrently)
};

__device__ __forceinline__ uint32_t excl_scan32(uint32_t x, int lane, uint32_t &total) {
  uint32_t s = x;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, s, o);
    if (lane >= o) s += y;
  }
  total = __shfl_sync(0xffffffffu, s, 31);
  return s - x;
}

template <int TW>
__device__ __forceinline__ int next_bit(const uint32_t (&bm)[TW], uint32_t pos, uint32_t W) {
#pragma unroll
  for (int w = 0; w < TW; w++) {
    if (w < (int)W && (uint32_t)(w + 1) * 32 > pos) {
      uint32_t word = bm[w];
      if ((uint32_t)w * 32 < pos) word &= ~0u << (pos & 31);
      if (word) return w * 32 + __ffs(word) - 1;
    }
  }
  return -1;
}

template <int TW>
__device__ __forceinline__ uint32_t popc_and(const uint32_t (&x)[TW], const uint32_t *row, uint32_t W,
                                             uint32_t (&out)[TW]) {
  uint32_t c = 0;
#pragma unroll
  for (int w = 0; w < TW; w++) {
    out[w] = (w < (int)W) ? (x[w] & row[w]) : 0u;
    c += __popc(out[w]);
  }
  return c;
}

// Count the k-cliques that extend a clique of `chosen` vertices whose common
// candidates (a subset of R) are the bitmap `cur`: DFS over the rows B (stride W).
template <int TW>
__device__ uint64_t dfs_count(const uint32_t *B, uint32_t W, const uint32_t (&cur)[TW], uint32_t chosen,
                              uint32_t k) {
  uint32_t c0 = 0;
#pragma unroll
  for (int w = 0; w < TW; w++) c0 += __popc(cur[w]);
  if (chosen + 1 == k) return c0;   // each candidate completes one k-clique
  if (c0 < k - chosen) return 0;
  uint64_t cnt = 0;
  if (chosen + 2 == k) {   // sum over j in cur of |cur ∩ B_j|
    uint32_t pos = 0;
    for (;;) {
      const int j = next_bit<TW>(cur, pos, W);
      if (j < 0) break;
      pos = j + 1;
      uint32_t nx[TW];
      cnt += popc_and<TW>(cur, B + j * W, W, nx);
    }
    return cnt;
  }
  uint32_t stk[kMaxStack][TW];
  uint32_t pos[kMaxStack];
#pragma unroll
  for (int w = 0; w < TW; w++) stk[0][w] = cur[w];
  pos[0] = 0;
  int s = 0;
  while (s >= 0) {
    uint32_t top[TW];
#pragma unroll
    for (int w = 0; w < TW; w++) top[w] = stk[s][w];
    const int j = next_bit<TW>(top, pos[s], W);
    if (j < 0) {
      s--;
      continue;
    }
    pos[s] = j + 1;
    const uint32_t t = s + chosen + 1;   // vertices chosen after taking j
    uint32_t nx[TW];
    const uint32_t c = popc_and<TW>(top, B + j * W, W, nx);
    if (t == k - 1) {
      cnt += c;
      continue;
    }
    if (c < k - t) continue;             // cannot complete a k-clique
    s++;
#pragma unroll
    for (int w = 0; w < TW; w++) stk[s][w] = nx[w];
    pos[s] = 0;
  }
  return cnt;
}

// Multi-size variant: every visited node with `chosen` vertices and candidates cur
// contributes popc(cur) cliques of size chosen+1; the walk goes down to size kmax
// (no size pruning: a branch that cannot reach kmax still holds smaller cliques).
template <int TW>
__device__ void dfs_multi(const uint32_t *B, uint32_t W, const uint32_t (&cur)[TW], uint32_t chosen, uint32_t kmax,
                          uint64_t (&mc)[kMaxStack + 3]) {
  uint32_t c0 = 0;
#pragma unroll
  for (int w = 0; w < TW; w++) c0 += __popc(cur[w]);
  mc[chosen + 1] += c0;
  if (chosen + 1 >= kmax || c0 == 0) return;
  uint32_t stk[kMaxStack][TW];
  uint32_t pos[kMaxStack];
#pragma unroll
  for (int w = 0; w < TW; w++) stk[0][w] = cur[w];
  pos[0] = 0;
  int s = 0;
  while (s >= 0) {
    uint32_t top[TW];
#pragma unroll
    for (int w = 0; w < TW; w++) top[w] = stk[s][w];
    const int j = next_bit<TW>(top, pos[s], W);
    if (j < 0) {
      s--;
      continue;
    }
    pos[s] = j + 1;
    const uint32_t t = s + chosen + 1;   // vertices chosen after taking j
    uint32_t nx[TW];
    const uint32_t c = popc_and<TW>(top, B + j * W, W, nx);
    mc[t + 1] += c;
    if (t + 1 >= kmax || c == 0) continue;
    s++;
#pragma unroll
    for (int w = 0; w < TW; w++) stk[s][w] = nx[w];
    pos[s] = 0;
  }
}

// ---- register-resident DFS (warp teams, rows of TW <= 4 words, stride TW) ----------
// The DFS below a triangle item is unrolled into nested loops by template recursion
// over the number S of chosen vertices (S < SM, a compile-time bound on k), so the
// candidate bitmaps of every level, the set bits still to visit and the per-size
// counters all live in registers (no local-memory stack); a row is one 16-byte
// shared-memory load.
template <int TW>
__device__ __forceinline__ void load_row(const uint32_t *B, uint32_t j, uint32_t (&r)[TW]) {
  if constexpr (TW == 4) {
    const uint4 x = *reinterpret_cast<const uint4 *>(B + j * 4);
    r[0] = x.x; r[1] = x.y; r[2] = x.z; r[3] = x.w;
  } else {
#pragma unroll
    for (int w = 0; w < TW; w++) r[w] = B[j * TW + w];
  }
}

// lowest set bit of rem (cleared), or -1
template <int TW>
__device__ __forceinline__ int pop_next(uint32_t (&rem)[TW]) {
  int wi = -1;
#pragma unroll
  for (int w = TW - 1; w >= 0; w--)
    if (rem[w]) wi = w;
  if (wi < 0) return -1;
  uint32_t word = 0;
#pragma unroll
  for (int w = 0; w < TW; w++)
    if (w == wi) word = rem[w];
#pragma unroll
  for (int w = 0; w < TW; w++)
    if (w == wi) rem[w] = word & (word - 1u);
  return wi * 32 + __ffs(word) - 1;
}

template <int TW>
__device__ __forceinline__ uint32_t popc_n(const uint32_t (&x)[TW]) {
  uint32_t c = 0;
#pragma unroll
  for (int w = 0; w < TW; w++) c += __popc(x[w]);
  return c;
}

// multi-size: node with S chosen vertices adds popc(cur) (S+1)-cliques; expands while
// S + 1 < kmax
template <int TW, int S, int SM, int N>
__device__ __forceinline__ void rdfs_multi(const uint32_t *B, const uint32_t (&cur)[TW], uint32_t kmax,
                                           uint64_t (&mc)[N]) {
  static_assert(SM < N, "counter array too short");
  const uint32_t c = popc_n<TW>(cur);
  mc[S + 1] += c;
  if constexpr (S + 1 < SM) {
    if (S + 1 >= kmax || c == 0) return;
    uint32_t rem[TW];
#pragma unroll
    for (int w = 0; w < TW; w++) rem[w] = cur[w];
    for (;;) {
      const int j = pop_next<TW>(rem);
      if (j < 0) break;
      uint32_t nx[TW];
      load_row<TW>(B, (uint32_t)j, nx);
#pragma unroll
      for (int w = 0; w < TW; w++) nx[w] &= cur[w];
      rdfs_multi<TW, S + 1, SM, N>(B, nx, kmax, mc);
    }
  }
}

// single k: k-cliques below a node with S chosen vertices (prunes nodes that cannot
// reach k)
template <int TW, int S, int SM>
__device__ __forceinline__ uint64_t rdfs_count(const uint32_t *B, const uint32_t (&cur)[TW], uint32_t k) {
  const uint32_t c = popc_n<TW>(cur);
  if (S + 1 == k) return c;
  uint64_t cnt = 0;
  if constexpr (S + 1 < SM) {
    if (c < k - S) return 0;
    uint32_t rem[TW];
#pragma unroll
    for (int w = 0; w < TW; w++) rem[w] = cur[w];
    for (;;) {
      const int j = pop_next<TW>(rem);
      if (j < 0) break;
      uint32_t nx[TW];
      load_row<TW>(B, (uint32_t)j, nx);
#pragma unroll
      for (int w = 0; w < TW; w++) nx[w] &= cur[w];
      cnt += rdfs_count<TW, S + 1, SM>(B, nx, k);
    }
  }
  return cnt;
}

// ---- lane-group DFS (CTA teams and heavy-root parts, rows of W <= 16 words) -------
// A thread-per-item DFS over 16-word rows diverges badly (the subtree sizes of the
// triangles of one hub differ by orders of magnitude; ncu: < 5 active threads per
// warp instruction).  Here a group of aligned lanes walks one item, lane gl holding
// word gl of every candidate bitmap: a node is one conflict-free row load, an AND and a
// popcount per lane; the next child is one group ballot + shuffle.  The counts stay per
// lane (summed by the final warp reduction).  Template recursion over the number S of
// chosen vertices keeps every level in registers.  The group is 8 lanes for rows of
// <= 8 words (|R| <= 256: C2's CTA teams have <= 6) and 16 above: a 16-lane group on
// 6-word rows idled 10 lanes in every word-parallel step.
constexpr int kGroup = 16;   // largest group

struct LaneGroup {
  uint32_t mask;   // the group's lanes in the warp
  int base;        // first lane of the group
  int gl;          // this lane's index inside the group
  int lane;
  int size;        // 8 or 16
};

__device__ __forceinline__ LaneGroup lane_group(int lane, int size) {
  LaneGroup g;
  g.size = size;
  g.base = lane & ~(size - 1);
  g.gl = lane - g.base;
  g.mask = ((1u << size) - 1u) << g.base;
  g.lane = lane;
  return g;
}

#ifndef GAMMA_KCL_GROUP16   // A/B: always 16-lane groups (round 1)
#define GAMMA_KCL_GROUP16 0
#endif
__device__ __forceinline__ int group_size_for(uint32_t W) { return (W <= 8 && !GAMMA_KCL_GROUP16) ? 8 : kGroup; }

// next child of the group's remaining-bits word set (cleared), or -1
__device__ __forceinline__ int group_next(const LaneGroup &g, uint32_t &rem) {
  const uint32_t bal = __ballot_sync(g.mask, rem != 0u);
  if (bal == 0) return -1;
  const int src = __ffs(bal) - 1;
  const uint32_t word = __shfl_sync(g.mask, rem, src);
  if (g.lane == src) rem &= rem - 1u;
  return (src - g.base) * 32 + __ffs(word) - 1;
}

// A node whose children are leaves only needs sum over children j of popc(cur & B[j])
// (the edges inside cur): the group broadcasts cur to all its lanes and each lane
// walks the children in its own word, reading whole rows (odd row stride: no bank
// conflicts between lanes), so no per-child ballot/shuffle is needed.
template <int WW>   // compile-time word bound (>= W): predicated-off words still issue
__device__ __forceinline__ uint32_t group_leaf_sum_w(const uint32_t *B, uint32_t BS, uint32_t W, uint32_t curw,
                                                     const LaneGroup &g) {
  uint32_t cur[WW];
#pragma unroll
  for (int w = 0; w < WW; w++) cur[w] = __shfl_sync(g.mask, curw, g.base + w);
  uint32_t acc = 0, bits = curw;
  while (bits) {
    const uint32_t j = (uint32_t)g.gl * 32 + __ffs(bits) - 1;
    bits &= bits - 1u;
    const uint32_t *row = B + j * BS;
#pragma unroll
    for (int w = 0; w < WW; w++)
      if (w < (int)W) acc += __popc(cur[w] & row[w]);
  }
  return acc;
}

// Balanced variant: the group's set bits of cur are dealt to its lanes by rank (bit r
// to lane r mod 16), each lane summing whole rows -- the per-word walk above gives a
// lane the bits of its own word, and with the run sorted by rank the candidates of a
// deep node crowd into its last words (ncu c2 r02: 2.4 threads per instruction on the
// leaf loop of the CTA-team kernel).
template <int WW>
__device__ __forceinline__ uint32_t group_leaf_sum_bal(const uint32_t *B, uint32_t BS, uint32_t W, uint32_t curw,
                                                       const LaneGroup &g) {
  uint32_t s = __popc(curw);
  for (int o = 1; o < g.size; o <<= 1) {
    const uint32_t y = __shfl_up_sync(g.mask, s, o);
    if (g.gl >= o) s += y;
  }
  uint32_t cur[WW], inc[WW];
#pragma unroll
  for (int w = 0; w < WW; w++) {
    cur[w] = __shfl_sync(g.mask, curw, g.base + w);
    inc[w] = __shfl_sync(g.mask, s, g.base + w);   // bits in words 0..w (W <= WW: the rest are 0)
  }
  const uint32_t total = inc[WW - 1];
  uint32_t acc = 0;
  for (uint32_t r = g.gl; r < total; r += (uint32_t)g.size) {
    uint32_t wsel = 0, before = 0;
#pragma unroll
    for (int w = 0; w < WW; w++)
      if (inc[w] <= r) {
        wsel = w + 1;
        before = inc[w];
      }
    uint32_t word = 0;
#pragma unroll
    for (int w = 0; w < WW; w++)
      if (w == (int)wsel) word = cur[w];
    const uint32_t j = wsel * 32 + __fns(word, 0, r - before + 1);
    const uint32_t *row = B + j * BS;
#pragma unroll
    for (int w = 0; w < WW; w++)
      if (w < (int)W) acc += __popc(cur[w] & row[w]);
  }
  return acc;
}

__device__ __forceinline__ uint32_t group_leaf_sum(const uint32_t *B, uint32_t BS, uint32_t W, uint32_t curw,
                                                   const LaneGroup &g) {
  if (!GAMMA_KCL_LEAF_BAL) {
    if (W <= 4) return group_leaf_sum_w<4>(B, BS, W, curw, g);
    if (W <= 8) return group_leaf_sum_w<8>(B, BS, W, curw, g);
    return group_leaf_sum_w<kGroup>(B, BS, W, curw, g);
  }
  if (W <= 4) return group_leaf_sum_bal<4>(B, BS, W, curw, g);
  if (W <= 8) return group_leaf_sum_bal<8>(B, BS, W, curw, g);
  return group_leaf_sum_bal<kGroup>(B, BS, W, curw, g);
}

template <int S, int SM, int N>
__device__ __forceinline__ void gdfs_multi(const uint32_t *B, uint32_t BS, uint32_t W, uint32_t curw, uint32_t kmax,
                                           uint64_t (&mc)[N], const LaneGroup &g) {
  static_assert(SM < N, "counter array too short");
  mc[S + 1] += __popc(curw);
  if constexpr (S + 1 < SM) {
    if (S + 1 >= kmax) return;
    if (S + 2 == kmax) {   // children are leaves
      mc[S + 2] += group_leaf_sum(B, BS, W, curw, g);
      return;
    }
    uint32_t rem = curw;
    for (;;) {
      const int j = group_next(g, rem);
      if (j < 0) break;
      const uint32_t row = g.gl < (int)W ? B[(uint32_t)j * BS + g.gl] : 0u;
      gdfs_multi<S + 1, SM, N>(B, BS, W, curw & row, kmax, mc, g);
    }
  }
}

template <int S, int SM>
__device__ __forceinline__ uint64_t gdfs_count(const uint32_t *B, uint32_t BS, uint32_t W, uint32_t curw, uint32_t k,
                                               const LaneGroup &g) {
  if (S + 1 == k) return __popc(curw);
  uint64_t cnt = 0;
  if constexpr (S + 1 < SM) {
    if (S + 2 == k) return group_leaf_sum(B, BS, W, curw, g);
    const uint32_t c = __reduce_add_sync(g.mask, __popc(curw));
    if (c < k - S) return 0;
    uint32_t rem = curw;
    for (;;) {
      const int j = group_next(g, rem);
      if (j < 0) break;
      const uint32_t row = g.gl < (int)W ? B[(uint32_t)j * BS + g.gl] : 0u;
      cnt += gdfs_count<S + 1, SM>(B, BS, W, curw & row, k, g);
    }
  }
  return cnt;
}

// j1 = the last row with P[j1] <= q, found from the previous item's row (a caller's
// items only move forward): a short forward scan, then a binary search over the rest
// (the per-item binary search from row 0 was ~12 % of the CTA-team kernel's
// instructions, ncu heavy r02).
__device__ __forceinline__ uint32_t advance_row(const uint32_t *P, uint32_t L, uint32_t q, uint32_t j1) {
#pragma unroll
  for (int s = 0; s < 4; s++)
    if (j1 + 1 < L && P[j1 + 1] <= q) j1++;
  if (j1 + 1 < L && P[j1 + 1] <= q) {
    uint32_t lo = j1 + 1, hi = L;
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (P[mid] <= q) lo = mid; else hi = mid;
    }
    j1 = lo;
  }
  return j1;
}

// Item q -> this lane's word of the candidates of the triangle (v, R[j1], R[j2]); j1
// carries the row of the caller's previous item (0 for the first).
__device__ __forceinline__ uint32_t group_item_cur(const uint32_t *B, const uint32_t *P, uint32_t L, uint32_t W,
                                                   uint32_t BS, uint32_t q, const LaneGroup &g, uint32_t &j1) {
  j1 = advance_row(P, L, q, j1);
  const uint32_t r = q - P[j1];
  const uint32_t w1 = g.gl < (int)W ? B[j1 * BS + g.gl] : 0u;
  // the r-th set bit of row j1: inclusive scan of the word popcounts over the group
  const uint32_t pc = __popc(w1);
  uint32_t inc = pc;
  for (int o = 1; o < g.size; o <<= 1) {
    const uint32_t y = __shfl_up_sync(g.mask, inc, o);
    if (g.gl >= o) inc += y;
  }
  const bool mine = r < inc && r >= inc - pc;
  const uint32_t bal = __ballot_sync(g.mask, mine);
  const int src = __ffs(bal) - 1;
  const uint32_t j2b = mine ? (uint32_t)g.gl * 32 + __fns(w1, 0, r - (inc - pc) + 1) : 0u;
  const uint32_t j2 = __shfl_sync(g.mask, j2b, src);
  const uint32_t w2 = g.gl < (int)W ? B[j2 * BS + g.gl] : 0u;
  return w1 & w2;
}

// ---- warp teams, k <= 6: the DFS as a per-lane state machine ----------------------
// The nested-loop DFS (rdfs_*) gives each lane whole triangle items, and the subtrees
// below the triangles of one root differ by orders of magnitude: ncu c2 r02b put the
// DFS at 7.1 active threads per warp instruction.  Here every lane does exactly one
// node per step -- the next child of its deepest open node, else a fresh triangle item
// -- so the warp stays converged until the root's items run out.  Below a triangle
// (S = 3 chosen vertices, candidates X) the open nodes are X (S = 3) and Y (S = 4):
// a step pops a child j of Y (leaf: popc(Y & B[j]) (S+2)-cliques), else of X (node
// Y = X & B[j]), else takes an item (X = B[j1] & B[j2]).  Items come from a per-warp
// queue refilled 32 at a time (one item -> (j1, j2) mapping per lane).
// Counts per size: multi (kmin..kmax, kmax <= 6) adds popc of every node; single k
// adds only size k and prunes nodes that cannot reach it (as rdfs_count).
__device__ __forceinline__ bool any4(const uint32_t (&x)[4]) { return (x[0] | x[1] | x[2] | x[3]) != 0u; }

template <bool MULTI>
__device__ __forceinline__ void warp_dfs_sm(const uint32_t *B, const uint32_t *P, uint32_t L, uint32_t W,
                                            uint32_t items, uint32_t k, int lane, uint32_t *Q,
                                            uint64_t &c3, uint64_t &c4, uint64_t &c5, uint64_t &c6, uint64_t &cnt) {
  constexpr uint32_t kFull = 0xffffffffu;
  const uint32_t lt = (1u << lane) - 1u;
  uint32_t X[4] = {0, 0, 0, 0}, rX[4] = {0, 0, 0, 0}, Y[4] = {0, 0, 0, 0}, rY[4] = {0, 0, 0, 0};
  uint32_t filled = 0, taken = 0, jq = 0;
  uint32_t a3 = 0, a4 = 0, a5 = 0, a6 = 0;   // this root's counts (< 2^32 for |R| <= 128)
  // expand a node of S chosen vertices (children add size S + 2 below it)?
  const bool exp3 = MULTI ? k > 4 : k > 4, exp4 = MULTI ? k > 5 : k > 5;
  for (;;) {
    const bool useY = any4(rY), useX = !useY && any4(rX);
    const bool busy = useY || useX;
    const uint32_t need = __ballot_sync(kFull, !busy);
    const uint32_t nneed = __popc(need);
    if (filled < items && filled - taken < nneed) {   // warp-uniform refill
      const uint32_t q = filled + lane;
      if (q < items) {
        jq = advance_row(P, L, q, jq);
        uint32_t r = q - P[jq], j2 = 0;
#pragma unroll
        for (uint32_t w = 0; w < 4; w++) {
          const uint32_t word = w < W ? B[jq * 4 + w] : 0u;
          const uint32_t pc = __popc(word);
          if (r < pc) {
            j2 = w * 32 + __fns(word, 0, r + 1);
            r = 0xffffffffu;   // found: no later word matches (r < pc fails)
          } else if (r != 0xffffffffu) {
            r -= pc;
          }
        }
        Q[q & 63] = (jq << 16) | j2;
      }
      filled = min(items, filled + 32);
      __syncwarp();
    }
    const uint32_t avail = filled - taken, rank = __popc(need & lt);
    const bool got = !busy && rank < avail;
    const uint32_t it = got ? Q[(taken + rank) & 63] : 0u;
    taken += min(nneed, avail);
    if (!__any_sync(kFull, busy || got)) break;
    // the node of this step: its parent's candidates (src) and the child row j
    uint32_t src[4], j = 0;
    if (busy) {
      uint32_t rr[4];
#pragma unroll
      for (int w = 0; w < 4; w++) rr[w] = useY ? rY[w] : rX[w];
      const int wi = rr[0] ? 0 : rr[1] ? 1 : rr[2] ? 2 : 3;
      const uint32_t word = wi == 0 ? rr[0] : wi == 1 ? rr[1] : wi == 2 ? rr[2] : rr[3];
      j = (uint32_t)wi * 32 + __ffs(word) - 1;
      const uint32_t nw = word & (word - 1u);
#pragma unroll
      for (int w = 0; w < 4; w++) {
        if (w == wi) {
          if (useY) rY[w] = nw; else rX[w] = nw;
        }
        src[w] = useY ? Y[w] : X[w];
      }
    } else if (got) {
      j = it & 0xffffu;
      const uint4 r1 = *reinterpret_cast<const uint4 *>(B + (it >> 16) * 4);
      src[0] = r1.x; src[1] = r1.y; src[2] = r1.z; src[3] = r1.w;
    } else {
      src[0] = src[1] = src[2] = src[3] = 0u;
    }
    const uint4 rj = *reinterpret_cast<const uint4 *>(B + j * 4);
    const uint32_t n0 = src[0] & rj.x, n1 = src[1] & rj.y, n2 = src[2] & rj.z, n3 = src[3] & rj.w;
    const uint32_t c = __popc(n0) + __popc(n1) + __popc(n2) + __popc(n3);
    if (useY) {            // leaf below Y: (S = 5)-node, c = (S + 1 = 6)-cliques
      a6 += c;
    } else if (useX) {     // Y = X & B[j]: S = 4 node, c = 5-cliques
      a5 += c;
      const bool e = exp4 && (MULTI || c >= k - 4);
      Y[0] = n0; Y[1] = n1; Y[2] = n2; Y[3] = n3;
      rY[0] = e ? n0 : 0u; rY[1] = e ? n1 : 0u; rY[2] = e ? n2 : 0u; rY[3] = e ? n3 : 0u;
    } else if (got) {      // X = B[j1] & B[j2]: S = 3 node (a triangle), c = 4-cliques
      a3 += 1;
      a4 += c;
      const bool e = exp3 && (MULTI || c >= k - 3);
      X[0] = n0; X[1] = n1; X[2] = n2; X[3] = n3;
      rX[0] = e ? n0 : 0u; rX[1] = e ? n1 : 0u; rX[2] = e ? n2 : 0u; rX[3] = e ? n3 : 0u;
    }
  }
  if (MULTI) {
    c3 += a3; c4 += a4; c5 += a5; c6 += a6;
  } else {
    cnt += k == 4 ? a4 : k == 5 ? a5 : a6;
  }
}

template <int TEAM_WARPS>
__device__ __forceinline__ void team_sync() {
  if (TEAM_WARPS == 1) __syncwarp();
  else __syncthreads();
}

// Shared words per team: run R (32 TW), bitmap rows B (32 TW x TW), position hash:
// positions H (4 x 32 TW u16 = 64 TW words) and the vertex ids of the slots Hv
// (4 x 32 TW words), row offsets P (32 TW + 1, padded to +2), two broadcast slots
// (8-byte aligned: every region starts at an even word).
template <int TW>
constexpr int row_words_max() {   // largest row stride (see row_stride)
  return TW == 4 ? 4 : TW + 1;
}

template <int TW>
constexpr int team_words() {
  return TW * 32 + TW * 32 * row_words_max<TW>() + 2 * TW * 32 + 4 * TW * 32 + TW * 32 + 2 + 2;
}

template <int TW>
struct TeamMem {
  uint32_t *R, *B, *P, *slot, *Hv;
  unsigned short *H;
  __device__ TeamMem(uint32_t *base) {
    R = base;
    B = R + TW * 32;
    H = reinterpret_cast<unsigned short *>(B + TW * 32 * row_words_max<TW>());
    Hv = B + TW * 32 * row_words_max<TW>() + 2 * TW * 32;
    P = Hv + 4 * TW * 32;
    slot = P + TW * 32 + 2;
  }
};

// Depth-2 extension of root v: R = N+(v), rows B[i] = positions of R ∩ N+(R[i]).
// Flattened windows of 32 children; each list element is located in R through a
// shared-memory open-addressing position table.  Returns Σ|N+(c)| (for the bytes).
// R and H live in shared memory; B in shared memory (<= 512-long runs) or in a
// global scratch slice (wide runs).
// With Hv (team kernels) the slot's vertex id is stored beside its position, so a
// probe compares ids directly and checks two slots without branching; only when both
// are taken by other ids (rare at load <= 1/4) does it walk the chain.  Without Hv
// (wide runs, whose tables would not fit) the position table alone is probed.
constexpr uint32_t kEmptyId = 0xffffffffu;   // vertex ids are < n <= 2^32 - 1

template <int TEAM_WARPS, bool PAGED>
__device__ uint64_t build_rows_p(const BmArgs &a, uint32_t *R, unsigned short *H, uint32_t *B, uint64_t b0,
                                 uint32_t L, int tid, int lane, uint32_t stride, uint32_t *Hv = nullptr) {
  constexpr int kTeamThreads = TEAM_WARPS * 32;
  const int wit = tid >> 5;
  const uint32_t W = stride;   // row stride in words (>= the row's (L + 31) / 32 words)
  // Short runs (warp teams, |R| <= 32, one-word rows): probe the pairs instead of the
  // lists.  Bit j of row i is R[j] in N+(R[i]): one binary search of R[j] in the child's
  // sorted list per ordered pair -- |R|(|R|-1) probes where streaming the lists would
  // probe sum |N+(c)| elements (C2, |R| <= 32: 1.2e8 pairs vs 5.7e8 elements,
  // scratch/pair_cost.py) -- and no hash table.  The rows of 32 / |R|' consecutive
  // lanes (|R|' = |R| rounded up to a power of two) come out of one ballot.
  if (GAMMA_KCL_PAIR_SORT && TEAM_WARPS == 1 && L <= 32 && !GAMMA_KCL_NO_PAIRS) {
    // The run sorted by the orientation order (degree, id) first (a warp bitonic sort
    // of 64-bit keys): then bit j of row i can only be set for j > i, so only the
    // |R|(|R|-1)/2 pairs above the diagonal are searched -- rows i and |R|-2-i share a
    // lane group (their |R|-1-i and i+1 candidates fill |R| lanes).  The DFS does not
    // care how R is ordered.
    constexpr uint32_t kFull = 0xffffffffu;
    uint32_t x = kEmptyId, dlx = 0, dgx = 0;
    uint64_t cbx = 0;
    if (lane < (int)L) x = a.dag_col.at<PAGED>(b0 + lane);
    if (lane < (int)L) {
      cbx = a.dag_ptr[x];
      dlx = (uint32_t)(a.dag_ptr[x + 1] - cbx);
      if (a.row_ptr) dgx = (uint32_t)(a.row_ptr[x + 1] - a.row_ptr[x]);
    }
    uint64_t key = lane < (int)L ? ((uint64_t)dgx << 32 | x) : ~0ull;
    uint32_t src = lane;
#pragma unroll
    for (uint32_t k = 2; k <= 32; k <<= 1)
#pragma unroll
      for (uint32_t jj = k >> 1; jj > 0; jj >>= 1) {
        const uint64_t ok = __shfl_xor_sync(kFull, key, jj);
        const uint32_t os = __shfl_xor_sync(kFull, src, jj);
        const bool keep_min = ((lane & k) == 0) == ((lane & jj) == 0);
        if (keep_min ? ok < key : ok > key) {
          key = ok;
          src = os;
        }
      }
    const uint64_t cbs = __shfl_sync(kFull, cbx, src);
    const uint32_t dls = __shfl_sync(kFull, dlx, src);
    const uint32_t xs = (uint32_t)key;   // lane p: the p-th vertex of the sorted run
    if (lane < (int)L) R[lane] = xs;
    uint64_t elems = lane < (int)L ? dls : 0u;
    const uint32_t lg = L <= 2 ? 1u : L <= 4 ? 2u : L <= 8 ? 3u : L <= 16 ? 4u : 5u;
    const uint32_t t = lane & ((1u << lg) - 1u), groups = 32u >> lg, gbase = lane & ~((1u << lg) - 1u);
    const uint32_t npairs = L / 2;   // row pairs (p, |R|-2-p); row |R|-1 has no candidate
    constexpr int kU = GAMMA_KCL_PAIR_U;
    for (uint32_t p0 = 0; p0 < npairs; p0 += groups * kU) {
      uint64_t cb[kU];
      uint32_t base[kU], len[kU], yv[kU];
#pragma unroll
      for (int u = 0; u < kU; u++) {
        const uint32_t pp = p0 + u * groups + (lane >> lg);
        const uint32_t first = L - 1 - pp;   // candidates of row pp (j = pp + 1 + t)
        const uint32_t r = t < first ? pp : L - 2 - pp;
        const uint32_t j = t < first ? pp + 1 + t : t;
        const bool on = pp < npairs && t < L && (t < first || r != pp);
        const uint64_t cr = __shfl_sync(kFull, cbs, r & 31);
        const uint32_t dr = __shfl_sync(kFull, dls, r & 31);
        yv[u] = __shfl_sync(kFull, xs, j & 31);
        cb[u] = cr;
        base[u] = 0;
        len[u] = on ? dr : 0u;
      }
      for (;;) {
        bool more = false;
#pragma unroll
        for (int u = 0; u < kU; u++) {
          if (len[u] > 1) {
            const uint32_t half = len[u] >> 1;
            base[u] = a.dag_col.at<PAGED>(cb[u] + base[u] + half) <= yv[u] ? base[u] + half : base[u];
            len[u] -= half;
            more |= len[u] > 1;
          }
        }
        if (!__any_sync(kFull, more)) break;
      }
#pragma unroll
      for (int u = 0; u < kU; u++) {
        const uint32_t pp = p0 + u * groups + (lane >> lg);
        const bool hit = len[u] == 1 && a.dag_col.at<PAGED>(cb[u] + base[u]) == yv[u];
        const uint32_t bal = __ballot_sync(kFull, hit);
        const uint32_t gb = lg == 5 ? bal : (bal >> gbase) & ((1u << (1u << lg)) - 1u);
        if (t == 0 && pp < npairs) {
          const uint32_t first = L - 1 - pp, r = L - 2 - pp;
          const uint32_t lowm = (1u << first) - 1u;
          B[pp * W] = (gb & lowm) << (pp + 1);
          if (r != pp) B[r * W] = gb & ~lowm;
#pragma unroll
          for (uint32_t w = 1; w < 4; w++)   // the state-machine DFS reads whole 4-word rows
            if (w < W) {
              B[pp * W + w] = 0u;
              B[r * W + w] = 0u;
            }
        }
      }
    }
    if (lane == 0) {   // the last row: no candidate after it
      B[(L - 1) * W] = 0u;
#pragma unroll
      for (uint32_t w = 1; w < 4; w++)
        if (w < W) B[(L - 1) * W + w] = 0u;
    }
    __syncwarp();
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) elems += __shfl_down_sync(kFull, elems, off);
    return lane == 0 ? elems : 0u;
  }
  if (TEAM_WARPS == 1 && L <= 32 && !GAMMA_KCL_NO_PAIRS) {
    if (lane < (int)L) R[lane] = a.dag_col.at<PAGED>(b0 + lane);
    __syncwarp();
    const uint32_t lg = L <= 2 ? 1u : L <= 4 ? 2u : L <= 8 ? 3u : L <= 16 ? 4u : 5u;
    const uint32_t j = lane & ((1u << lg) - 1u), rows_per = 32u >> lg;
    const uint32_t rj = j < L ? R[j] : 0u;
    uint64_t elems = 0;
    // kU rows per lane group at once: their binary searches advance in lock step, so a
    // lane keeps kU independent L2 loads in flight (a run of 17..32 took |R| rounds of
    // ~log2 d+ dependent loads one row at a time; C2 same box: kU = 1 6.57 ms/step,
    // 2 6.12, 4 6.44 -- more rows in flight cost registers the DFS needs)
    constexpr int kU = GAMMA_KCL_PAIR_U;
    for (uint32_t i0 = 0; i0 < L; i0 += rows_per * kU) {
      uint64_t cb[kU];
      uint32_t base[kU], len[kU];
#pragma unroll
      for (int u = 0; u < kU; u++) {
        const uint32_t i = i0 + (u * rows_per) + (lane >> lg);
        cb[u] = 0;
        len[u] = 0;
        base[u] = 0;
        if (i < L) {
          const uint32_t c = R[i];
          cb[u] = a.dag_ptr[c];
          const uint32_t dl = (uint32_t)(a.dag_ptr[c + 1] - cb[u]);
          if (j == 0) elems += dl;
          len[u] = (j < L && j != i) ? dl : 0u;
        }
      }
      // lower-bound search of rj in each list (len 0: no search, no hit)
      for (;;) {
        bool more = false;
#pragma unroll
        for (int u = 0; u < kU; u++) {
          if (len[u] > 1) {
            const uint32_t half = len[u] >> 1;
            base[u] = a.dag_col.at<PAGED>(cb[u] + base[u] + half) <= rj ? base[u] + half : base[u];
            len[u] -= half;
            more |= len[u] > 1;
          }
        }
        if (!__any_sync(0xffffffffu, more)) break;
      }
#pragma unroll
      for (int u = 0; u < kU; u++) {
        const uint32_t i = i0 + (u * rows_per) + (lane >> lg);
        const bool hit = len[u] == 1 && a.dag_col.at<PAGED>(cb[u] + base[u]) == rj;
        // one ballot holds every row of this step: row i's bits are its lane group's
        const uint32_t bal = __ballot_sync(0xffffffffu, hit);
        const uint32_t bits = lg == 5 ? bal : (bal >> (lane & ~((1u << lg) - 1u))) & ((1u << (1u << lg)) - 1u);
        if (j == 0 && i < L) {
          B[i * W] = bits;
#pragma unroll
          for (uint32_t w = 1; w < 4; w++)   // the state-machine DFS reads whole 4-word rows
            if (w < W) B[i * W + w] = 0u;
        }
      }
    }
    __syncwarp();
    return elems;
  }
  uint32_t hbits = 2;
  while ((1u << hbits) < 4 * L) hbits++;
  const uint32_t hmask = (1u << hbits) - 1u;
  for (uint32_t i = tid; i < L; i += kTeamThreads) R[i] = a.dag_col.at<PAGED>(b0 + i);
  for (uint32_t i = tid; i < L * W; i += kTeamThreads) B[i] = 0u;
  if (Hv) {
    for (uint32_t i = tid; i <= hmask; i += kTeamThreads) Hv[i] = kEmptyId;
  } else {
    for (uint32_t i = tid; i <= hmask / 2; i += kTeamThreads) reinterpret_cast<uint32_t *>(H)[i] = 0u;
  }
  team_sync<TEAM_WARPS>();
  for (uint32_t i = tid; i < L; i += kTeamThreads) {
    const uint32_t x = R[i];
    uint32_t h = (x * 0x9E3779B1u) >> (32 - hbits);
    if (Hv) {
      h &= ~3u;   // probing starts at a 4-slot bucket read in one load
      while (atomicCAS(&Hv[h], kEmptyId, x) != kEmptyId) h = (h + 1) & hmask;
      H[h] = (unsigned short)i;
    } else {
      while (atomicCAS(&H[h], (unsigned short)0, (unsigned short)(i + 1)) != 0) h = (h + 1) & hmask;
    }
  }
  team_sync<TEAM_WARPS>();
  const uint32_t rmin = R[0], rmax = R[L - 1];
  uint64_t elems = 0;
  for (uint32_t w0 = wit * 32; w0 < L; w0 += TEAM_WARPS * 32) {
    const uint32_t i = w0 + lane;
    uint32_t beg = 0, dl = 0;
    if (i < L) {
      const uint32_t c = R[i];
      const uint64_t cb = a.dag_ptr[c];
      dl = (uint32_t)(a.dag_ptr[c + 1] - cb);
      beg = (uint32_t)cb;
      // rank space: lists ascend by rank, so the part of N+(c) above the run's largest
      // rank cannot meet the run -- trim it (one binary search; ~19 % of the C2 row-build
      // elements, scratch/rank_cut.py)
      if (a.trim && dl && a.dag_col.at<PAGED>(cb + dl - 1) > rmax) {
        uint32_t lo = 0, hi = dl - 1;   // first index with dag_col > rmax, in [0, dl - 1]
        while (lo < hi) {
          const uint32_t mid = (lo + hi) >> 1;
          if (a.dag_col.at<PAGED>(cb + mid) > rmax) hi = mid; else lo = mid + 1;
        }
        dl = lo;
      }
    }
    elems += dl;
    // compact the children with non-empty lists to lanes 0..nnz-1 (every list then
    // has a distinct start offset) and exclusive-scan their lengths
    const uint32_t nz = __ballot_sync(0xffffffffu, dl > 0);
    const uint32_t nnz = __popc(nz);
    const uint32_t src = lane < (int)nnz ? __fns(nz, 0, lane + 1) : 0;
    const uint32_t cbeg = __shfl_sync(0xffffffffu, beg, src);
    const uint32_t sdl = __shfl_sync(0xffffffffu, dl, src);
    const uint32_t cdl = lane < (int)nnz ? sdl : 0u;
    const uint32_t crow = w0 + src;
    uint32_t T;
    const uint32_t o = excl_scan32(cdl, lane, T);
    const uint32_t upto = lane == 31 ? 0xffffffffu : ((2u << lane) - 1u);
    // element t of the window (t in list i: o_i <= t < o_i + len_i) is
    // dag_col[cofs_i + t] with cofs_i = beg_i - o_i (mod 2^32; offsets < m < 2^32)
    const uint32_t cofs = cbeg - o;
    uint32_t nb = 0;   // lists that started before this tile
    // kTiles tiles of 32 elements per step: their loads are issued back to back
    // before any probe, so each lane keeps several L2 gathers in flight
    constexpr int kTiles = GAMMA_KCL_TILES;
    for (uint32_t t0 = 0; t0 < T; t0 += 32 * kTiles) {
      // tiles that hold elements (warp-uniform): a short window runs 1-3 tiles, not 4
      // (the padded tiles were ~half the row-build instructions on C2's small roots)
      const uint32_t nt = (T - t0 + 31) >> 5;
      uint32_t y[kTiles], rj[kTiles];
#pragma unroll
      for (int u = 0; u < kTiles; u++) {
        if ((uint32_t)u >= nt) {
          y[u] = kEmptyId;
          rj[u] = 0;
          continue;
        }
        const uint32_t tb = t0 + 32 * u;
        const uint32_t t = tb + lane;
        // lane t's list = the last list starting at or before t: one OR-reduction of
        // the start offsets that fall in this tile (lanes past the compacted lists hold
        // o = T: a bit at or above every valid t, so it moves no valid lane's list)
        const uint32_t d = o - tb;
        const uint32_t S = __reduce_or_sync(0xffffffffu, d < 32u ? 1u << d : 0u);
        const uint32_t j = (nb + __popc(S & upto) - 1u) & 31u;
        nb += __popc(S);
        const uint32_t off = __shfl_sync(0xffffffffu, cofs, j);
        rj[u] = __shfl_sync(0xffffffffu, crow, j);
        y[u] = t < T ? a.dag_col.at<PAGED>((uint64_t)(uint32_t)(off + t)) : kEmptyId;
      }
#pragma unroll
      for (int u = 0; u < kTiles; u++) {
        if ((uint32_t)u >= nt) break;
        const uint32_t yy = y[u];
        if (Hv) {
          // one 16-byte load of the 4-slot bucket where y's probe sequence starts.  The
          // slots of a bucket are claimed in order (every insertion enters a bucket at
          // its first slot and moves on only past a taken one), so a free last slot
          // ends the probe; only a full bucket without y (rare at load <= 1/4) walks on.
          // The padding id kEmptyId matches the free slots: it is excluded by yy != kEmptyId.
          const uint32_t h0 = ((yy * 0x9E3779B1u) >> (32 - hbits)) & ~3u;
          const uint4 vv = *reinterpret_cast<const uint4 *>(Hv + h0);
          bool hit = (vv.x == yy || vv.y == yy || vv.z == yy || vv.w == yy) && yy != kEmptyId;
          uint32_t hw = 0;   // slot found by the walk
          if (!hit && vv.w != kEmptyId && yy != kEmptyId) {
            for (uint32_t h = (h0 + 4) & hmask;; h = (h + 1) & hmask) {
              const uint32_t vh = Hv[h];
              if (vh == yy) {
                hit = true;
                hw = h;
                break;
              }
              if (vh == kEmptyId) break;
            }
          }
          if (hit) {
            const uint32_t hh = vv.x == yy ? h0 : vv.y == yy ? h0 + 1 : vv.z == yy ? h0 + 2 : vv.w == yy ? h0 + 3 : hw;
            const uint32_t e = H[hh];
            atomicOr(&B[rj[u] * W + (e >> 5)], 1u << (e & 31));
          }
          continue;
        }
        if (yy >= rmin && yy <= rmax) {   // (the padding kEmptyId is above every rmax < n)
          uint32_t h = (yy * 0x9E3779B1u) >> (32 - hbits);
          for (;;) {
            const uint32_t e = H[h];
            if (e == 0) break;
            if (R[e - 1] == yy) {
              atomicOr(&B[rj[u] * W + ((e - 1) >> 5)], 1u << ((e - 1) & 31));
              break;
            }
            h = (h + 1) & hmask;
          }
        }
      }
    }
  }
  team_sync<TEAM_WARPS>();   // (a CTA barrier also orders the global-memory rows)
  return elems;
}

// Row stride in shared memory: TW words for warp teams (16-byte rows, one vector
// load each); for CTA teams the row's own W words rounded up to an odd count, so that
// lanes reading the same word of different rows hit different banks (the
// lane-parallel leaf loop of the group DFS).
template <int TEAM_WARPS, int TW>
__device__ __forceinline__ uint32_t row_stride(uint32_t L) {
  return TEAM_WARPS == 1 ? (uint32_t)TW : (((L + 31) >> 5) | 1u);
}

template <int TEAM_WARPS, int TW, bool PAGED>
__device__ __forceinline__ uint64_t build_rows(const BmArgs &a, const TeamMem<TW> &m, uint64_t b0, uint32_t L,
                                               int tid, int lane) {
  return build_rows_p<TEAM_WARPS, PAGED>(a, m.R, m.H, m.B, b0, L, tid, lane, row_stride<TEAM_WARPS, TW>(L), m.Hv);
}

// P[r] = exclusive scan of the row popcounts (the triangle items), P[L] = total.
template <int TEAM_WARPS, int TW>
__device__ void scan_rows(const TeamMem<TW> &m, uint32_t L, int tid, int lane) {
  const uint32_t W = (L + 31) >> 5, BS = row_stride<TEAM_WARPS, TW>(L);
  if ((tid >> 5) == 0) {
    uint32_t carry = 0;
    for (uint32_t r0 = 0; r0 < L; r0 += 32) {
      const uint32_t r = r0 + lane;
      uint32_t c = 0;
      if (r < L)
        for (uint32_t w = 0; w < W; w++) c += __popc(m.B[r * BS + w]);
      uint32_t tot;
      const uint32_t ex = excl_scan32(c, lane, tot);
      if (r < L) m.P[r] = carry + ex;
      carry += tot;
    }
    if (lane == 0) m.P[L] = carry;
  }
  team_sync<TEAM_WARPS>();
}

// Item q -> candidates of the triangle (v, R[j1], R[j2]); j1 carries the row of the
// caller's previous item (0 for the first).
template <int TW>
__device__ __forceinline__ void item_cur(const TeamMem<TW> &m, uint32_t L, uint32_t W, uint32_t BS, uint32_t q,
                                         uint32_t (&cur)[TW], uint32_t &j1) {
  j1 = advance_row(m.P, L, q, j1);
  uint32_t r = q - m.P[j1], j2 = 0;
  for (uint32_t w = 0; w < W; w++) {
    const uint32_t word = m.B[j1 * BS + w];
    const uint32_t pc = __popc(word);
    if (r < pc) {
      j2 = w * 32 + __fns(word, 0, r + 1);
      break;
    }
    r -= pc;
  }
#pragma unroll
  for (int w = 0; w < TW; w++) cur[w] = (w < (int)W) ? (m.B[j1 * BS + w] & m.B[j2 * BS + w]) : 0u;
}

template <int TEAM_WARPS>
__device__ __forceinline__ uint64_t team_sum(uint64_t x, int lane, uint32_t *slot) {
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) x += __shfl_down_sync(0xffffffffu, x, off);
  x = __shfl_sync(0xffffffffu, x, 0);
  if (TEAM_WARPS == 1) return x;
  unsigned long long *s64 = reinterpret_cast<unsigned long long *>(slot);   // 8-byte aligned slot pair
  if (threadIdx.x == 0) *s64 = 0;
  __syncthreads();
  if (lane == 0) atomicAdd(s64, (unsigned long long)x);
  __syncthreads();
  const uint64_t r = *s64;
  __syncthreads();
  return r;
}

__device__ __forceinline__ void flush_multi(uint64_t (&mc)[kMaxStack + 3], const BmArgs &a, int lane) {
#pragma unroll
  for (uint32_t sz = 3; sz < kMaxStack + 3; sz++) {   // unrolled: mc stays in registers
    if (sz > a.k) break;
    uint64_t x = mc[sz];
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) x += __shfl_down_sync(0xffffffffu, x, off);
    if (lane == 0 && x) atomicAdd(&a.ctrl[CTRL_MULTI + sz], (unsigned long long)x);
  }
}

// KM: compile-time bound on k for the register-resident DFS of warp teams (6 or 12;
// the deeper instantiation needs more registers, so k <= 6 gets its own kernel).
template <int TEAM_WARPS, int TW, bool PER_ROOT, int KM, bool PAGED>
__global__ void GAMMA_BM_BOUNDS(KM) kcl_bitmap_kernel(BmArgs a) {
  extern __shared__ uint32_t smem[];
  constexpr int kTeamThreads = TEAM_WARPS * 32;
  const int lane = threadIdx.x & 31;
  const int team = threadIdx.x / kTeamThreads;
  const int tid = threadIdx.x % kTeamThreads;
  const TeamMem<TW> m(smem + team * team_words<TW>());
  uint64_t total = 0, elems = 0, entries = 0;
  uint64_t mc[kMaxStack + 3] = {};   // multi mode: cliques per size

  // warp teams take roots in batches of 4 (one atomic per batch); CTA teams one
  // root at a time (their roots are the long, costly ones)
  constexpr unsigned long long kBatch = TEAM_WARPS == 1 ? 4 : 1;
  unsigned long long next = 0, end = 0;
  // warp teams: lane t < kBatch holds root base + t of the batch and its DAG offsets,
  // all loaded when the batch is taken (one round trip chain per batch, not per root)
  uint32_t bv = 0;
  uint64_t bb0 = 0, bb1 = 0;
  for (;;) {
    if (next == end) {
      unsigned long long base = 0;
      if (tid == 0) base = atomicAdd(a.work, kBatch);
      if (TEAM_WARPS == 1) {
        base = __shfl_sync(0xffffffffu, base, 0);
        if ((unsigned long long)lane < kBatch && base + lane < a.nroots) {
          bv = a.roots[base + lane];
          bb0 = a.dag_ptr[bv];
          bb1 = a.dag_ptr[bv + 1];
        }
      } else {
        if (tid == 0) m.slot[0] = base < 0xffffffffull ? (uint32_t)base : 0xffffffffu;
        __syncthreads();
        base = m.slot[0];
        __syncthreads();
      }
      next = base;
      end = base + kBatch;
    }
    if (next >= a.nroots) break;
    const unsigned long long gi = next++;
    uint32_t v;
    uint64_t b0;
    uint32_t L;
    if (TEAM_WARPS == 1) {
      const int t = (int)(gi - (end - kBatch));
      v = __shfl_sync(0xffffffffu, bv, t);
      b0 = __shfl_sync(0xffffffffu, bb0, t);
      L = (uint32_t)(__shfl_sync(0xffffffffu, bb1, t) - b0);
    } else {
      v = a.roots[gi];
      b0 = a.dag_ptr[v];
      L = (uint32_t)(a.dag_ptr[v + 1] - b0);
    }
    if (L <= a.len_lo || L > a.len_hi || L < (a.multi ? a.kmin - 1 : a.k - 1)) continue;   // uniform across the team
    const uint32_t W = (L + 31) >> 5, BS = row_stride<TEAM_WARPS, TW>(L);
    if (tid == 0) entries += L;
    elems += build_rows<TEAM_WARPS, TW, PAGED>(a, m, b0, L, tid, lane);
    // ---- deeper extensions: bitmap DFS.  k = 3: one row per thread (its popcount).
    // k >= 4: the work items are the triangles (v, R[j1], R[j2]), j2 in row j1 ----
    uint64_t cnt = 0;
    if (a.k == 3) {
      for (uint32_t j1 = tid; j1 < L; j1 += kTeamThreads) {
        uint32_t c = 0;
        for (uint32_t w = 0; w < W; w++) c += __popc(m.B[j1 * BS + w]);
        cnt += c;
      }
      if (a.multi) mc[3] += cnt;
    } else {
      scan_rows<TEAM_WARPS, TW>(m, L, tid, lane);
      const uint32_t items = m.P[L];
      bool deferred = false;
      // hub splitting: estimate the DFS by the 4-clique count (skipped when even
      // items x |R| -- an upper bound of it -- is below the cut: most roots)
      if (a.heavy_cut && (uint64_t)items * L > a.heavy_cut) {
        uint64_t est = 0;
        uint32_t jr = 0;
        for (uint32_t q = tid; q < items; q += kTeamThreads) {
          uint32_t cur[TW];
          item_cur<TW>(m, L, W, BS, q, cur, jr);
          uint32_t c = 0;
#pragma unroll
          for (int w = 0; w < TW; w++) c += __popc(cur[w]);
          est += c;
        }
        est = team_sum<TEAM_WARPS>(est, lane, m.slot);
        if (est > a.heavy_cut) {
          const uint64_t want = est / a.part_cost + 1;
          const uint32_t nparts = want < kMaxParts ? (uint32_t)want : kMaxParts;
          // keep the rows: one root-rows slot (none left: expand here)
          if (tid == 0) {
            const unsigned long long sl = atomicAdd(&a.ctrl[CTRL_AUX2], 1ull);
            m.slot[0] = sl < a.root_rows_cap ? (uint32_t)sl : 0xffffffffu;
          }
          team_sync<TEAM_WARPS>();
          const uint32_t slot = m.slot[0];
          team_sync<TEAM_WARPS>();
          if (slot != 0xffffffffu) {
            uint32_t *dst = a.root_rows + (uint64_t)slot * kSlotWords;
            if (tid == 0) {
              dst[0] = L;
              dst[1] = W;
              dst[2] = BS;
              dst[3] = (uint32_t)(a.root_base + gi);
            }
            for (uint32_t i = tid; i <= L; i += kTeamThreads) dst[4 + i] = m.P[i];
            for (uint32_t i = tid; i < L * BS; i += kTeamThreads) dst[kSlotB + i] = m.B[i];
            __threadfence();
            team_sync<TEAM_WARPS>();
          }
          if (tid == 0 && slot != 0xffffffffu) {
            // reserve [at, at + nparts) only if it fits: the cursor never passes
            // parts_cap, so every slot below it has been written by its reserver
            // (the parts kernel reads exactly [0, cursor))
            unsigned long long at = *(volatile unsigned long long *)&a.ctrl[CTRL_AUX1];
            bool ok = false;
            while (at + nparts <= a.parts_cap) {
              const unsigned long long seen = atomicCAS(&a.ctrl[CTRL_AUX1], at, at + nparts);
              if (seen == at) {
                ok = true;
                break;
              }
              at = seen;
            }
            if (ok) {
              for (uint32_t p = 0; p < nparts; p++) a.parts[at + p] = make_uint2(slot, p | (nparts << 16));
              m.slot[0] = 1;
            } else {
              m.slot[0] = 0;   // list full: expand here
            }
          } else if (tid == 0) {
            m.slot[0] = 0;     // no root-rows slot: expand here
          }
          team_sync<TEAM_WARPS>();
          deferred = m.slot[0] == 1;
          team_sync<TEAM_WARPS>();
        }
      }
      uint32_t jr = 0;
      if constexpr (TEAM_WARPS == 1 && KM == 6 && GAMMA_KCL_SM_DFS) {   // state-machine DFS
        if (!deferred) {
          if (a.multi)
            warp_dfs_sm<true>(m.B, m.P, L, W, items, a.k, lane, m.Hv, mc[3], mc[4], mc[5], mc[6], cnt);
          else
            warp_dfs_sm<false>(m.B, m.P, L, W, items, a.k, lane, m.Hv, mc[3], mc[4], mc[5], mc[6], cnt);
        }
      } else if (TEAM_WARPS == 1 && !deferred)
        for (uint32_t q = tid; q < items; q += kTeamThreads) {
          uint32_t cur[TW];
          item_cur<TW>(m, L, W, BS, q, cur, jr);
          if constexpr (TEAM_WARPS == 1) {   // register-resident nested loops
            if (a.multi) {
              mc[3] += 1;   // the item is one triangle
              rdfs_multi<TW, 3, KM, kMaxStack + 3>(m.B, cur, a.k, mc);
            } else {
              cnt += rdfs_count<TW, 3, KM>(m.B, cur, a.k);
            }
          }
        }
      if constexpr (TEAM_WARPS > 1) {   // lane groups: one triangle item per 16-lane group
        if (!deferred) {
          const int gsz = group_size_for(W);
          const LaneGroup g = lane_group(lane, gsz);
          const uint32_t ngroups = kTeamThreads / gsz;
          uint32_t jg = 0;
          for (uint32_t q = tid / gsz; q < items; q += ngroups) {
            const uint32_t curw = group_item_cur(m.B, m.P, L, W, BS, q, g, jg);
            if (a.multi) {
              if (g.gl == 0) mc[3] += 1;   // the item is one triangle
              gdfs_multi<3, KM, kMaxStack + 3>(m.B, BS, W, curw, a.k, mc, g);
            } else {
              cnt += gdfs_count<3, KM>(m.B, BS, W, curw, a.k, g);
            }
          }
        }
      }
    }
    total += cnt;
    if (PER_ROOT) {
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) cnt += __shfl_down_sync(0xffffffffu, cnt, off);
      if (lane == 0 && cnt) atomicAdd(&a.per_root[gi], (unsigned long long)cnt);
    }
    team_sync<TEAM_WARPS>();   // R/B are rewritten by the next root
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    total += __shfl_down_sync(0xffffffffu, total, off);
    elems += __shfl_down_sync(0xffffffffu, elems, off);
    entries += __shfl_down_sync(0xffffffffu, entries, off);
  }
  if (lane == 0) {
    if (total) atomicAdd(&a.ctrl[CTRL_COUNT], (unsigned long long)total);
    atomicAdd(&a.ctrl[CTRL_ELEMS], (unsigned long long)elems);
    atomicAdd(&a.ctrl[CTRL_AUX0], (unsigned long long)entries);
  }
  if (a.multi) flush_multi(mc, a, lane);
}

// Second launch for the deferred heavy roots: one CTA per (root, part); the part
// rebuilds the root's rows (cheap next to the DFS) and takes every nparts-th item.
template <bool PER_ROOT, int KM>
__global__ void GAMMA_BM_BOUNDS(KM) kcl_bitmap_parts_kernel(BmArgs a) {
  extern __shared__ uint32_t smem[];
  constexpr int TW = 16;
  const int lane = threadIdx.x & 31;
  const int tid = threadIdx.x;
  const TeamMem<TW> m(smem);
  uint64_t total = 0;
  uint64_t mc[kMaxStack + 3] = {};
  for (;;) {
    if (tid == 0) {
      // the part list was filled by the previous launch; its length (<= parts_cap,
      // every slot below it written) sits in ctrl
      const unsigned long long nparts_total = *(volatile unsigned long long *)&a.ctrl[CTRL_AUX1];
      const unsigned long long w = atomicAdd(a.work, 1ull);
      m.slot[0] = w < nparts_total ? (uint32_t)w : 0xffffffffu;
    }
    __syncthreads();
    const uint32_t wi = m.slot[0];
    __syncthreads();
    if (wi == 0xffffffffu) break;
    const uint2 pt = a.parts[wi];
    const uint32_t part = pt.y & 0xffff, nparts = pt.y >> 16;
    // the root's rows as its team built them (no rebuild): one coalesced copy from L2
    const uint32_t *src = a.root_rows + (uint64_t)pt.x * kSlotWords;
    const uint32_t L = src[0], W = src[1], BS = src[2], gi = src[3];
    for (uint32_t i = tid; i <= L; i += 256) m.P[i] = src[4 + i];
    for (uint32_t i = tid; i < L * BS; i += 256) m.B[i] = src[kSlotB + i];
    __syncthreads();
    const uint32_t items = m.P[L];
    uint64_t cnt = 0;
    const int gsz = group_size_for(W);
    const LaneGroup g = lane_group(lane, gsz);
    const uint32_t ngroups = 256 / gsz;
    uint32_t jg = 0;
    for (uint32_t q = part + (tid / gsz) * nparts; q < items; q += ngroups * nparts) {
      const uint32_t curw = group_item_cur(m.B, m.P, L, W, BS, q, g, jg);
      if (a.multi) {
        if (g.gl == 0) mc[3] += 1;
        gdfs_multi<3, KM, kMaxStack + 3>(m.B, BS, W, curw, a.k, mc, g);
      } else {
        cnt += gdfs_count<3, KM>(m.B, BS, W, curw, a.k, g);
      }
    }
    total += cnt;
    if (PER_ROOT) {
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) cnt += __shfl_down_sync(0xffffffffu, cnt, off);
      if (lane == 0 && cnt) atomicAdd(&a.per_root[gi], (unsigned long long)cnt);
    }
    __syncthreads();
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) total += __shfl_down_sync(0xffffffffu, total, off);
  if (lane == 0 && total) atomicAdd(&a.ctrl[CTRL_COUNT], (unsigned long long)total);
  if (a.multi) flush_multi(mc, a, lane);
}

// ---- wide runs (kBitmapMaxRun < |R| <= kWideMaxRun): one CTA per root ------------
// The rows (|R| x W words, W <= 32 WL) do not fit shared memory: they go to the CTA's
// slice of a global scratch (L2-resident for the run of one root), R and the position
// hash stay in shared memory.  A warp takes one row i at a time (candidates of the
// edge (v, R[i])) and walks the DFS below it with every candidate bitmap spread over
// its lanes (lane l holds words l, l+32, ...): the next candidate is found with one
// ballot per word slice, the AND with a row is a coalesced 128-byte load per slice,
// and every lane accumulates the popcounts of its own words.
constexpr int kWideThreads = 512;

template <int WL>
__device__ __forceinline__ int wide_pop_next(uint32_t (&rem)[WL], int lane) {
#pragma unroll
  for (int t = 0; t < WL; t++) {
    const uint32_t bal = __ballot_sync(0xffffffffu, rem[t] != 0u);
    if (bal) {
      const int l = __ffs(bal) - 1;
      const uint32_t w = __shfl_sync(0xffffffffu, rem[t], l);
      if (lane == l) rem[t] &= rem[t] - 1u;
      return (l + 32 * t) * 32 + __ffs(w) - 1;
    }
  }
  return -1;
}

// DFS below the candidates `cur` of a clique of `chosen` vertices (lane-distributed);
// returns this lane's share of the k-clique count (multi: adds to mc per size).
template <int WL>
__device__ uint64_t wide_dfs(const uint32_t *B, uint32_t W, const uint32_t (&cur0)[WL], uint32_t chosen,
                             uint32_t k, bool multi, uint64_t (&mc)[kMaxStack + 3], int lane) {
  uint32_t cur[kMaxStack][WL], rem[kMaxStack][WL];
#pragma unroll
  for (int t = 0; t < WL; t++) cur[0][t] = rem[0][t] = cur0[t];
  uint64_t cnt = 0;
  int s = 0;
  while (s >= 0) {
    uint32_t r[WL];
#pragma unroll
    for (int t = 0; t < WL; t++) r[t] = rem[s][t];
    const int j = wide_pop_next<WL>(r, lane);
#pragma unroll
    for (int t = 0; t < WL; t++) rem[s][t] = r[t];
    if (j < 0) {
      s--;
      continue;
    }
    const uint32_t tk = chosen + s + 1;   // vertices chosen after taking j
    uint32_t nx[WL];
    uint32_t c = 0;
#pragma unroll
    for (int t = 0; t < WL; t++) {
      const uint32_t w = lane + 32 * t;
      nx[t] = w < W ? (cur[s][t] & B[(uint64_t)j * W + w]) : 0u;
      c += __popc(nx[t]);
    }
    if (multi) mc[tk + 1] += c;
    if (tk + 1 >= k) {
      cnt += c;
      continue;
    }
    // prune: fewer candidates than vertices still missing (single-k only)
    if (!multi && __reduce_add_sync(0xffffffffu, c) < k - tk - 1) continue;
    if (multi && __reduce_add_sync(0xffffffffu, c) == 0) continue;
    s++;
#pragma unroll
    for (int t = 0; t < WL; t++) cur[s][t] = rem[s][t] = nx[t];
  }
  return cnt;
}

// Register-resident variants of wide_dfs (template recursion over the chosen-vertex
// count S; SM = compile-time bound on k): the per-level candidate slices and the bits
// still to visit stay in registers instead of a local-memory stack.
template <int WL, int S, int SM, int N>
__device__ __forceinline__ void wdfs_multi(const uint32_t *B, uint32_t W, const uint32_t (&cur)[WL], uint32_t kmax,
                                           uint64_t (&mc)[N], int lane) {
  static_assert(SM < N, "counter array too short");
  uint32_t c = 0;
#pragma unroll
  for (int t = 0; t < WL; t++) c += __popc(cur[t]);
  mc[S + 1] += c;
  if constexpr (S + 1 < SM) {
    if (S + 1 >= kmax) return;
    uint32_t rem[WL];
#pragma unroll
    for (int t = 0; t < WL; t++) rem[t] = cur[t];
    for (;;) {
      const int j = wide_pop_next<WL>(rem, lane);
      if (j < 0) break;
      uint32_t nx[WL];
#pragma unroll
      for (int t = 0; t < WL; t++) {
        const uint32_t w = lane + 32 * t;
        nx[t] = w < W ? (cur[t] & B[(uint64_t)j * W + w]) : 0u;
      }
      wdfs_multi<WL, S + 1, SM, N>(B, W, nx, kmax, mc, lane);
    }
  }
}

template <int WL, int S, int SM>
__device__ __forceinline__ uint64_t wdfs_count(const uint32_t *B, uint32_t W, const uint32_t (&cur)[WL], uint32_t k,
                                               int lane) {
  uint32_t c = 0;
#pragma unroll
  for (int t = 0; t < WL; t++) c += __popc(cur[t]);
  if (S + 1 == k) return c;   // this lane's share
  uint64_t cnt = 0;
  if constexpr (S + 1 < SM) {
    if (__reduce_add_sync(0xffffffffu, c) < k - S) return 0;
    uint32_t rem[WL];
#pragma unroll
    for (int t = 0; t < WL; t++) rem[t] = cur[t];
    for (;;) {
      const int j = wide_pop_next<WL>(rem, lane);
      if (j < 0) break;
      uint32_t nx[WL];
#pragma unroll
      for (int t = 0; t < WL; t++) {
        const uint32_t w = lane + 32 * t;
        nx[t] = w < W ? (cur[t] & B[(uint64_t)j * W + w]) : 0u;
      }
      cnt += wdfs_count<WL, S + 1, SM>(B, W, nx, k, lane);
    }
  }
  return cnt;
}

template <int WL, bool PER_ROOT, int KM, bool PAGED>
__global__ void __launch_bounds__(kWideThreads) kcl_wide_kernel(BmArgs a) {
  extern __shared__ uint32_t smem[];
  constexpr int kMaxL = 1024 * WL;
  uint32_t *R = smem;                                                   // kMaxL
  unsigned short *H = reinterpret_cast<unsigned short *>(smem + kMaxL); // 4 kMaxL u16
  uint32_t *slot = smem + kMaxL + 2 * kMaxL;                            // 4 words
  uint32_t *B = a.wide_rows + (uint64_t)blockIdx.x * a.wide_stride;
  const int tid = threadIdx.x, lane = tid & 31;
  uint64_t total = 0, elems = 0, entries = 0;
  uint64_t mc[kMaxStack + 3] = {};
  for (;;) {
    if (tid == 0) {
      const unsigned long long w = atomicAdd(a.work, 1ull);
      slot[0] = w < a.nroots ? (uint32_t)w : 0xffffffffu;
      slot[1] = 0;   // row cursor
    }
    __syncthreads();
    const uint32_t gi = slot[0];
    if (gi == 0xffffffffu) break;
    const uint32_t v = a.roots[gi];
    const uint64_t b0 = a.dag_ptr[v];
    const uint32_t L = (uint32_t)(a.dag_ptr[v + 1] - b0);
    if (L <= a.len_lo || L > a.len_hi || L < (a.multi ? a.kmin - 1 : a.k - 1)) {
      __syncthreads();
      continue;
    }
    const uint32_t W = (L + 31) >> 5;
    if (tid == 0) entries += L;
    elems += build_rows_p<kWideThreads / 32, PAGED>(a, R, H, B, b0, L, tid, lane, W);
    uint64_t cnt = 0;
    for (;;) {
      uint32_t i = 0;
      if (lane == 0) i = atomicAdd(&slot[1], 1u);
      i = __shfl_sync(0xffffffffu, i, 0);
      if (i >= L) break;
      uint32_t cur[WL];
      uint32_t c = 0;
#pragma unroll
      for (int t = 0; t < WL; t++) {
        const uint32_t w = lane + 32 * t;
        cur[t] = w < W ? B[(uint64_t)i * W + w] : 0u;
        c += __popc(cur[t]);
      }
      if (a.k == 3) {
        if (a.multi) mc[3] += c;
        cnt += c;
        continue;
      }
      if (a.multi)
        wdfs_multi<WL, 2, KM, kMaxStack + 3>(B, W, cur, a.k, mc, lane);   // adds mc[3] += c itself
      else
        cnt += wdfs_count<WL, 2, KM>(B, W, cur, a.k, lane);
    }
    total += cnt;
    if (PER_ROOT) {
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) cnt += __shfl_down_sync(0xffffffffu, cnt, off);
      if (lane == 0 && cnt) atomicAdd(&a.per_root[gi], (unsigned long long)cnt);
    }
    __syncthreads();   // R, H, B and the slots are rewritten by the next root
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    total += __shfl_down_sync(0xffffffffu, total, off);
    elems += __shfl_down_sync(0xffffffffu, elems, off);
    entries += __shfl_down_sync(0xffffffffu, entries, off);
  }
  if (lane == 0) {
    if (total) atomicAdd(&a.ctrl[CTRL_COUNT], (unsigned long long)total);
    atomicAdd(&a.ctrl[CTRL_ELEMS], (unsigned long long)elems);
    atomicAdd(&a.ctrl[CTRL_AUX0], (unsigned long long)entries);
  }
  if (a.multi) flush_multi(mc, a, lane);
}

template <int WL>
constexpr size_t wide_smem() {
  return (size_t)(1024 * WL + 2 * 1024 * WL + 4) * sizeof(uint32_t);
}

// rows scratch: grid x (run length x words) for the longest run of the launch
template <int WL, int KM, bool PAGED>
void enqueue_wide_km(gamma_ctx *ctx, BmArgs a, bool per_root, uint32_t max_len, DevBuf<uint32_t> &rows) {
  static bool attr = false;
  if (!attr) {
    GAMMA_CUDA(cudaFuncSetAttribute(kcl_wide_kernel<WL, false, KM, PAGED>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    (int)wide_smem<WL>()));
    GAMMA_CUDA(cudaFuncSetAttribute(kcl_wide_kernel<WL, true, KM, PAGED>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    (int)wide_smem<WL>()));
    attr = true;
  }
  static int grid = 0;
  if (!grid)
    grid = ctx->num_sms *
           occupancy_blocks((const void *)kcl_wide_kernel<WL, false, KM, PAGED>, kWideThreads, wide_smem<WL>());
  const uint64_t L = std::min<uint64_t>(max_len, 1024u * WL);
  a.wide_stride = L * ((L + 31) / 32);
  const uint64_t g = std::min<uint64_t>(grid, a.nroots);
  rows = DevBuf<uint32_t>(ctx, g * a.wide_stride);
  a.wide_rows = rows.p;
  GAMMA_CUDA(cudaMemsetAsync(a.work, 0, sizeof(uint64_t), ctx->stream));
  ctx->launch(KC_BITMAP, [&] {
    if (per_root)
      kcl_wide_kernel<WL, true, KM, PAGED><<<(unsigned)g, kWideThreads, wide_smem<WL>(), ctx->stream>>>(a);
    else
      kcl_wide_kernel<WL, false, KM, PAGED><<<(unsigned)g, kWideThreads, wide_smem<WL>(), ctx->stream>>>(a);
  });
}

template <int WL>
void enqueue_wide(gamma_ctx *ctx, BmArgs a, bool per_root, uint32_t max_len, DevBuf<uint32_t> &rows) {
  const bool paged = a.dag_col.pages != nullptr;
  if (a.k <= 6) {
    if (paged) enqueue_wide_km<WL, 6, true>(ctx, a, per_root, max_len, rows);
    else enqueue_wide_km<WL, 6, false>(ctx, a, per_root, max_len, rows);
  } else {
    if (paged) enqueue_wide_km<WL, kBitmapMaxK, true>(ctx, a, per_root, max_len, rows);
    else enqueue_wide_km<WL, kBitmapMaxK, false>(ctx, a, per_root, max_len, rows);
  }
}

template <int TEAM_WARPS, int TW>
constexpr size_t bm_smem() {
  return (size_t)(256 / (TEAM_WARPS * 32)) * team_words<TW>() * sizeof(uint32_t);
}

// Enqueue one team kind over a root range (no host round trip: the work counter is
// reset on the stream, the counts accumulate in ctrl and are read once at the end).
template <int TEAM_WARPS, int TW, int KM, bool PAGED>
void enqueue_bitmap_km(gamma_ctx *ctx, const BmArgs &a0, bool per_root, cudaStream_t st) {
  static bool attr = false;
  if (!attr) {
    GAMMA_CUDA(cudaFuncSetAttribute(kcl_bitmap_kernel<TEAM_WARPS, TW, false, KM, PAGED>,
                                    cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bm_smem<TEAM_WARPS, TW>()));
    GAMMA_CUDA(cudaFuncSetAttribute(kcl_bitmap_kernel<TEAM_WARPS, TW, true, KM, PAGED>,
                                    cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bm_smem<TEAM_WARPS, TW>()));
    attr = true;
  }
  const size_t smem = bm_smem<TEAM_WARPS, TW>();
  static int grid = 0;
  if (!grid)
    grid = ctx->num_sms * occupancy_blocks((const void *)kcl_bitmap_kernel<TEAM_WARPS, TW, false, KM, PAGED>, 256, smem);
  GAMMA_CUDA(cudaMemsetAsync(a0.work, 0, sizeof(uint64_t), st));
  ctx->launch_on(KC_BITMAP, st, [&] {
    if (per_root)
      kcl_bitmap_kernel<TEAM_WARPS, TW, true, KM, PAGED><<<grid, 256, smem, st>>>(a0);
    else
      kcl_bitmap_kernel<TEAM_WARPS, TW, false, KM, PAGED><<<grid, 256, smem, st>>>(a0);
  });
}

template <int TEAM_WARPS, int TW>
void enqueue_bitmap(gamma_ctx *ctx, const BmArgs &a0, bool per_root, cudaStream_t st) {
  const bool paged = a0.dag_col.pages != nullptr;
  if (a0.k <= 6) {
    if (paged) enqueue_bitmap_km<TEAM_WARPS, TW, 6, true>(ctx, a0, per_root, st);
    else enqueue_bitmap_km<TEAM_WARPS, TW, 6, false>(ctx, a0, per_root, st);
  } else {
    if (paged) enqueue_bitmap_km<TEAM_WARPS, TW, kBitmapMaxK, true>(ctx, a0, per_root, st);
    else enqueue_bitmap_km<TEAM_WARPS, TW, kBitmapMaxK, false>(ctx, a0, per_root, st);
  }
}

template <int KM>
void enqueue_parts_km(gamma_ctx *ctx, const BmArgs &a0, bool per_root) {
  static bool attr = false;
  if (!attr) {
    GAMMA_CUDA(cudaFuncSetAttribute(kcl_bitmap_parts_kernel<false, KM>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    (int)bm_smem<8, 16>()));
    GAMMA_CUDA(cudaFuncSetAttribute(kcl_bitmap_parts_kernel<true, KM>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    (int)bm_smem<8, 16>()));
    attr = true;
  }
  static int pgrid = 0;
  if (!pgrid)
    pgrid = ctx->num_sms * occupancy_blocks((const void *)kcl_bitmap_parts_kernel<false, KM>, 256, bm_smem<8, 16>());
  GAMMA_CUDA(cudaMemsetAsync(a0.work, 0, sizeof(uint64_t), ctx->stream));
  ctx->launch(KC_BITMAP, [&] {
    if (per_root)
      kcl_bitmap_parts_kernel<true, KM><<<pgrid, 256, bm_smem<8, 16>(), ctx->stream>>>(a0);
    else
      kcl_bitmap_parts_kernel<false, KM><<<pgrid, 256, bm_smem<8, 16>(), ctx->stream>>>(a0);
  });
}

void enqueue_parts(gamma_ctx *ctx, const BmArgs &a0, bool per_root) {
  if (a0.k <= 6)
    enqueue_parts_km<6>(ctx, a0, per_root);
  else
    enqueue_parts_km<kBitmapMaxK>(ctx, a0, per_root);
}

}  // namespace

// Count k-cliques rooted at roots[0..nroots) whose run length is <= kWideMaxRun
// (k <= 12); longer runs are left to the ET path.  per_root (nullable) indexed like
// roots.  Sorted roots (d+ descending): [0, n_xl) ET path, [n_xl, n_long) wide CTA,
// [n_long, n_mid) CTA teams, [n_mid, nroots) warp teams.
uint64_t kclique_bitmap(gamma_graph *g, uint32_t k, const uint32_t *roots, uint64_t nroots,
                        unsigned long long *per_root, bool sorted, uint64_t n_xl, uint64_t n_long, uint64_t n_mid,
                        uint64_t *multi_out, uint32_t kmin) {
  gamma_ctx *ctx = g->ctx;
  BmArgs a{};
  a.dag_ptr = g->dag_ptr;
  a.row_ptr = g->rank_space ? nullptr : g->row_ptr;
  a.dag_col = DagCol{g->dag_col, g->dag_pages};
  a.roots = roots;
  a.nroots = nroots;
  a.k = k;
  a.ctrl = (unsigned long long *)ctx->ctrl;
  a.per_root = per_root;
  a.multi = multi_out != nullptr;
  a.kmin = std::max<uint32_t>(3, std::min(kmin, k));
  {
    // the list trim pays only in rank space (ids in degree order); GAMMA_KCL_NO_TRIM off
    const char *e = getenv("GAMMA_KCL_NO_TRIM");
    a.trim = g->rank_space && !(e && *e && *e != '0');
  }
  // hub splitting only pays when the DFS below a triangle is deep (k >= 6)
  // (GAMMA_KCL_SPLIT_MINK: the smallest k that splits; default 6 on one GPU, 5 with
  // world > 1: a rank holds 1/world of the roots, so a hub's single CTA becomes the
  // critical path -- heavy, simulated 8 ranks on B200: 17.8 -> 9.3 ms per rank, while
  // at world 1 splitting k = 5 cost 13 %, profiles/sim_ranks_r02.jsonl)
  const char *mk_env = getenv("GAMMA_KCL_SPLIT_MINK");
  const uint32_t split_mink = mk_env && *mk_env ? (uint32_t)std::max(3ul, strtoul(mk_env, nullptr, 10))
                                                : (ctx->desc.world > 1 ? 5u : 6u);
  const bool split = k >= split_mink && (ctx->desc.flags & GAMMA_FLAG_NO_SPLIT) == 0;
  DevBuf<uint2> parts;
  DevBuf<uint32_t> root_rows;
  if (split) {
    // GAMMA_KCL_PARTS_CAP (tests): a small part list forces the "list full, expand
    // here" fallback
    const char *cap_env = getenv("GAMMA_KCL_PARTS_CAP");
    a.parts_cap = cap_env && *cap_env ? (uint32_t)std::max(1ul, std::min(strtoul(cap_env, nullptr, 10), 1ul << 24))
                                      : 1u << 20;
    parts = DevBuf<uint2>(ctx, a.parts_cap);
    a.parts = parts.p;
    a.part_cost = k >= 6 ? kPartCost : 4 * kPartCost;
    {   // GAMMA_KCL_PART_COST: 4-cliques per hub part (A/B knob)
      const char *pc = getenv("GAMMA_KCL_PART_COST");
      if (pc && *pc) a.part_cost = (uint32_t)std::max(64ul, std::min(strtoul(pc, nullptr, 10), 1ul << 24));
    }
    a.heavy_cut = (ctx->desc.flags & GAMMA_FLAG_DEBUG_SPLIT_ALL) ? 1 : 4ull * a.part_cost;
    a.root_rows_cap = std::min<uint32_t>(a.parts_cap, 2048);
    root_rows = DevBuf<uint32_t>(ctx, (uint64_t)a.root_rows_cap * kSlotWords);
    a.root_rows = root_rows.p;
  }
  // Roots sorted by d+ descending fall into three contiguous classes: [0, n_long) ET
  // path, [n_long, n_mid) CTA teams, [n_mid, nroots) warp teams; each team kind runs
  // on its own range.  Unsorted (per-root mode) roots: every launch filters the list.
  if (sorted) {
    n_xl = std::min(n_xl, nroots);
    n_long = std::min(n_long, nroots);
    n_mid = std::min(n_mid, nroots);
  }
  ctrl_reset(ctx);
  a.work = reinterpret_cast<unsigned long long *>(ctx->ctrl) + CTRL_WORK;
  const bool cta = g->max_out_degree > 128 && (!sorted || n_mid > n_long);
  const bool warp = !sorted || nroots > n_mid;
  const char *bands = getenv("GAMMA_KCL_BANDS");   // diagnostics: one warp-team launch per |R| band
  const bool banded = sorted && bands && *bands && *bands != '0' && g->root_order == roots;
  // The warp-team launch runs on a side stream beside the CTA-team launch (their tails
  // overlap), taking its roots from its own work cursor; the hub parts follow both.
  // (GAMMA_KCL_SERIAL=1: one stream.  Warp teams expanding their heavy roots themselves
  // so that the parts could overlap them too cost C2 6.1 -> 9.2 ms/step; a separate
  // launch for runs of 65..128, so that the parts could overlap the runs <= 64, 7.15:
  // the light runs no longer filled the heavy runs' tail.)
  static const bool serial_env = [] {
    const char *e = getenv("GAMMA_KCL_SERIAL");
    return e && *e && *e != '0';
  }();
  const bool conc = cta && warp && !banded && !serial_env;
  cudaEvent_t fork = nullptr, join = nullptr;
  cudaStream_t wst = ctx->stream;
  if (conc) {
    ctx->side_init();
    wst = ctx->side_streams[0];
    GAMMA_CUDA(cudaEventCreateWithFlags(&fork, cudaEventDisableTiming));
    GAMMA_CUDA(cudaEventCreateWithFlags(&join, cudaEventDisableTiming));
    GAMMA_CUDA(cudaEventRecord(fork, ctx->stream));   // after the control block reset
    GAMMA_CUDA(cudaStreamWaitEvent(wst, fork, 0));
  }
  // wide runs, [n_xl, n_long): 512 < |R| <= 2048 with 2 words per lane, longer with 8
  DevBuf<uint32_t> rows_a, rows_b;
  if (g->max_out_degree > kBitmapMaxRun && (!sorted || n_long > n_xl)) {
    a.roots = roots + (sorted ? n_xl : 0);
    a.nroots = sorted ? n_long - n_xl : nroots;
    if (g->max_out_degree > 2048) {
      a.len_lo = 2048;
      a.len_hi = kWideMaxRun;
      enqueue_wide<8>(ctx, a, per_root != nullptr, g->max_out_degree, rows_a);
    }
    a.len_lo = kBitmapMaxRun;
    a.len_hi = 2048;
    enqueue_wide<2>(ctx, a, per_root != nullptr, std::min<uint32_t>(g->max_out_degree, 2048), rows_b);
    a.roots = roots;
    a.nroots = nroots;
  }
  a.len_lo = 128;
  a.len_hi = 512;
  if (cta) {
    a.roots = roots + (sorted ? n_long : 0);
    a.root_base = sorted ? n_long : 0;
    a.nroots = sorted ? n_mid - n_long : nroots;
    enqueue_bitmap<8, 16>(ctx, a, per_root != nullptr, ctx->stream);
  }
  a.len_lo = 0;
  a.len_hi = 128;
  if (warp) {
    BmArgs aw = a;
    aw.roots = roots + (sorted ? n_mid : 0);
    aw.root_base = sorted ? n_mid : 0;
    aw.nroots = sorted ? nroots - n_mid : nroots;
    if (conc) aw.work = reinterpret_cast<unsigned long long *>(ctx->ctrl) + CTRL_WORK2;
    if (banded) {
      const uint32_t thr[] = {129, 65, 33, 17, 9, 0};
      for (int b = 0; b + 1 < 6; b++) {
        const uint64_t lo = std::max<uint64_t>(n_mid, thr[b] < g->root_ge.size() ? g->root_ge[thr[b]] : 0);
        const uint64_t hi = std::min<uint64_t>(nroots, thr[b + 1] < g->root_ge.size() ? g->root_ge[thr[b + 1]] : 0);
        if (hi <= lo) continue;
        BmArgs ab = aw;
        ab.roots = roots + lo;
        ab.root_base = lo;
        ab.nroots = hi - lo;
        enqueue_bitmap<1, 4>(ctx, ab, per_root != nullptr, ctx->stream);
      }
    } else {
      enqueue_bitmap<1, 4>(ctx, aw, per_root != nullptr, wst);
    }
  }
  if (conc) {   // join: the parts read the part lists of both team launches
    GAMMA_CUDA(cudaEventRecord(join, wst));
    GAMMA_CUDA(cudaStreamWaitEvent(ctx->stream, join, 0));
    cudaEventDestroy(fork);
    cudaEventDestroy(join);
  }
  if (split) {
    // parts carry absolute indices into the full root list
    a.roots = roots;
    a.root_base = 0;
    a.nroots = nroots;
    enqueue_parts(ctx, a, per_root != nullptr);
  }
  ctrl_fetch(ctx);
  const uint64_t *h = ctx->ctrl_host;
  ctx->stats.list_elems += h[CTRL_ELEMS];
  ctx->stats.level_entries[2] += h[CTRL_AUX0];
  ctx->stats.alg_bytes[KC_BITMAP] += 4 * h[CTRL_AUX0] + 4 * h[CTRL_ELEMS];
  if (split) ctx->stats.chunks += std::min<uint64_t>(h[CTRL_AUX1], a.parts_cap);
  if (multi_out)
    for (uint32_t sz = 0; sz <= k && sz < 32; sz++) multi_out[sz] = sz >= a.kmin ? h[CTRL_MULTI + sz] : 0;
  return h[CTRL_COUNT];
}

}  // namespace gamma_impl
