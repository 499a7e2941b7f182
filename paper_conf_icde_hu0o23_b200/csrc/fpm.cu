// fpm.cu -- frequent pattern mining, Alg. 2: edge extension
// (Def. 3.1 Ext_e, L131-139), aggregation by canonical label into the pattern
// table (L142), filtering by sup >= minsup (L144) with removal of the instances of
// infrequent patterns before the next extension (Alg. 2 line 4).
// Readings: R1 support = MNI (orbits merged), R2 length = #edges,
// R3 edge-induced, R7 canonical code = min over vertex orders of (labels, sorted
// edge-pair list), R8 sup >= minsup, R11 each connected edge set generated once.
//
// B200 design:
//  * e-ET root = every edge e1 (generated from its smaller endpoint); one warp per
//    root vertex u, lanes over u's edges / over the candidate second edges.  Each
//    connected edge set S = {e1 < e2 < e3} (edge order = (min,max) lexicographic) is
//    produced exactly once: from its minimum edge e1; the second generated edge is
//    the smallest edge of S adjacent to e1's... (see gen rule in fpm_enum_kernel).
//  * The levels < l are regenerated per level rather than stored (DFS per root
//    edge); Alg. 2's pruning is applied at every generated prefix by looking its
//    pattern up in the pattern table (infrequent prefix => no extension).
//  * Canonical code: a 5-comparator sorting network puts the <= 4 vertex labels in
//    order (the minimal label sequence); the minimal sorted edge-pair list and the
//    set of minimizing vertex orders then depend only on the edge mask in sorted
//    positions and on which neighbouring sorted labels tie, read from a 512-entry
//    shared-memory table built on the host by enumerating the 24 orders (no per-
//    embedding permutation loop, all in registers).  Every minimizing order is an
//    automorphic placement, so OR-ing the vertex of each position into that
//    position's domain merges orbits (MNI).
//  * Pattern table: lock-free open-addressing hash (one-word code -> slot, claimed
//    by a single atomicCAS; key and domain offset share one 16-byte slot) in HBM, sized from the number of label combinations so
//    probe chains stay short; the claimer carves the slot's MNI domains from a pool:
//    one bitmap per position over the vertices of that position's label class (bit
//    index = rank of the vertex inside its class), so memory follows the patterns
//    that occur.  Support = min over positions of popcount (one warp per slot).
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_select.cuh>

#include <algorithm>
#include <thread>
#include <cstdio>
#include <cstdlib>
#include <array>
#include <tuple>
#include <chrono>
#include <unordered_map>
#include <vector>

#include "device_common.cuh"
#include "internal.cuh"

namespace gamma_impl {

namespace {

constexpr int kThreads = 256;
#ifndef GAMMA_FPM_MEMO   // level-3 per-warp memo of (prefix, edge mask, new label) -> domains (0: off)
#define GAMMA_FPM_MEMO 1
#endif

// Pattern code packed in one word (0 = empty slot):
//   bits 0..47 four 12-bit labels (canonical order), 48..50 nv, 51..52 ne,
//   53..61 sorted edge-pair key, 63 always set.
constexpr uint64_t kKeyTag = 1ull << 63;

// Positions p < q of a <= 4-vertex pattern index its 6 vertex pairs as
// (0,1)(0,2)(0,3)(1,2)(1,3)(2,3) -> 0..5; kPid holds that index (15 on the diagonal)
// in 4-bit fields at 4(4p+q).  kPairA/kPairB: the endpoints of pair i, 2 bits each.
constexpr uint64_t kPid = 0xf5425f3143f0210full;
constexpr uint32_t kPairA = 0u | 0u << 2 | 0u << 4 | 1u << 6 | 1u << 8 | 2u << 10;
constexpr uint32_t kPairB = 1u | 2u << 2 | 3u << 4 | 2u << 6 | 3u << 8 | 3u << 10;
constexpr int kCanonEntries = 512;   // (sorted-position edge mask M: 6 bits) x (tie mask: 3 bits)

__host__ __device__ __forceinline__ uint32_t pid(uint32_t p, uint32_t q) {
  return (uint32_t)(kPid >> (4 * (4 * p + q))) & 15u;
}

struct Table {
  unsigned long long *slots;  // 2 words per slot: key (0 = empty; claimed with one atomicCAS)
                              // and dom = 1 + pool offset of its domains (0: being carved, ~0: no room)
  unsigned long long *support;
  uint32_t *freq;             // 1 if support >= minsup (set after the slot's level)
  uint64_t cap;               // power of two
  uint32_t *pool;             // per-slot domains, one bitmap per position over its label class
  uint64_t pool_words;
  unsigned long long *pool_cur;
  unsigned long long *inst;   // per-slot instance counts (GAMMA_FLAG_FPM_INSTANCES), nullable
};

__host__ __device__ __forceinline__ uint32_t key_nv(uint64_t k) { return (uint32_t)((k >> 48) & 7); }
__host__ __device__ __forceinline__ uint32_t key_ne(uint64_t k) { return (uint32_t)((k >> 51) & 3); }
__host__ __device__ __forceinline__ uint32_t key_edges(uint64_t k) { return (uint32_t)((k >> 53) & 511); }
__host__ __device__ __forceinline__ uint32_t key_label(uint64_t k, uint32_t p) {
  return (uint32_t)((k >> (12 * p)) & 0xfff);
}

struct FpmArgs {
  const uint64_t *rp;
  const uint32_t *col;
  const uint32_t *lab;       // nullable
  const uint32_t *lrank;     // rank of v inside its label class
  const uint32_t *cwords;    // words of one domain bitmap of each label class
  const uint2 *canon_tab;    // kCanonEntries: {best edge key, minimizing sigma set}
  const uint32_t *perm_tab;  // 24 rows: sigma[c] in bits 2c..2c+1 (c_perm order)
  uint32_t n;
  uint32_t level;            // edges per recorded embedding
  uint32_t rank, world;      // root partition: this rank takes edge batches b = rank (mod world)
  uint32_t claim_only;       // claim pattern slots without carving domains (distributed level)
  uint32_t carve_below;      // carve domains only for patterns whose smallest label is below this
  uint32_t walk_lo;          // last-level chunk pass: skip every embedding with a label < walk_lo
  Table T;
  unsigned long long *ctrl;
};

__device__ __forceinline__ uint32_t labof(const FpmArgs &a, uint32_t v) { return a.lab ? __ldg(a.lab + v) : 0u; }

__device__ __forceinline__ uint64_t ekey(uint32_t x, uint32_t y) {
  const uint32_t lo = x < y ? x : y, hi = x < y ? y : x;
  return ((uint64_t)lo << 32) | hi;
}

__device__ __forceinline__ bool shares(uint64_t e, uint64_t f) {
  const uint32_t a = (uint32_t)(e >> 32), b = (uint32_t)e, c = (uint32_t)(f >> 32), d = (uint32_t)f;
  return a == c || a == d || b == c || b == d;
}

__device__ __forceinline__ uint64_t mix64(uint64_t x) {
  x ^= x >> 33;
  x *= 0xff51afd7ed558ccdull;
  x ^= x >> 33;
  x *= 0xc4ceb9fe1a85ec53ull;
  x ^= x >> 33;
  return x;
}

// Lookup (insert = false) or lookup-or-insert a pattern code; returns the slot (or -1)
// and its dom word.  Lock-free: a slot is claimed by one atomicCAS of its key word; the
// claimer then carves the slot's domains from the pool (dom stays 0 until then).  Key
// and dom share 16 bytes, read with one L1-bypassing vector load.
__device__ int64_t table_slot(const FpmArgs &a, uint64_t key, bool insert, unsigned long long &dom) {
  const Table &T = a.T;
  uint64_t h = mix64(key) & (T.cap - 1);
  // a long probe chain means the table is (nearly) full: report it and let the host
  // grow the table instead of degrading to a linear scan
  const uint64_t max_probe = T.cap < 4096 ? T.cap : 4096;
  for (uint64_t probe = 0; probe < max_probe; probe++, h = (h + 1) & (T.cap - 1)) {
    const ulonglong2 kd = __ldcg(reinterpret_cast<const ulonglong2 *>(T.slots) + h);
    if (kd.x == key) {
      dom = kd.y;
      return (int64_t)h;
    }
    if (kd.x == 0) {
      if (!insert) return -1;
      const unsigned long long k = atomicCAS(&T.slots[2 * h], 0ull, (unsigned long long)key);
      if (k == 0) {
        // the claimer carves the slot's domains: one bitmap per position, sized to the
        // position's label class
        unsigned long long d = ~0ull;
        if (!a.claim_only && key_label(key, 0) >= a.carve_below) {
          atomicExch(&a.ctrl[CTRL_OVF], 1ull);   // left for a later, label-pruned pass
        } else if (!a.claim_only) {
          const uint32_t nv = key_nv(key);
          uint64_t words = 0;
          for (uint32_t p = 0; p < nv; p++) words += __ldg(a.cwords + key_label(key, p));
          const unsigned long long off = atomicAdd(T.pool_cur, (unsigned long long)words);
          d = off + 1;
          if (off + words > T.pool_words) {
            atomicExch(&a.ctrl[CTRL_OVF], 1ull);
            d = ~0ull;
          }
        }
        __threadfence();
        atomicExch(&T.slots[2 * h + 1], d);
        dom = d;
        return (int64_t)h;
      }
      if (k == key) {
        dom = __ldcg(&T.slots[2 * h + 1]);
        return (int64_t)h;
      }
    }
  }
  if (insert) atomicExch(&a.ctrl[CTRL_ERR], 1ull);   // table full
  return -1;
}

// Canonical code (reading R7: min over vertex orders of (labels in order, sorted
// edge-pair list)) of a connected edge set on nv <= 4 local vertices with labels
// l0..l3 and local edge mask em (bit pid(a, b) per edge).  The minimal label sequence
// is the sorted labels, so the minimizing orders are (stable label sort) o sigma with
// sigma permuting positions of equal labels only; which sigmas minimise the edge list
// depends only on the edge mask in sorted positions and on which neighbouring sorted
// labels are equal -- a 512-entry table (canon_tab, built on the host by enumerating
// the 24 sigmas, fpm_canon_tables).  ordw: local index at sorted position s in bits 2s.
struct Canon {
  uint64_t key;
  uint32_t minmask;   // minimizing sigmas (rows of perm_tab)
  uint32_t ordw;
};

__device__ __forceinline__ Canon canonical(const uint2 *tab, uint32_t l0, uint32_t l1, uint32_t l2, uint32_t l3,
                                           uint32_t nv, uint32_t em) {
  // composite (label, local index); the padding positions sort last, in local order
  uint32_t c0 = l0 << 2, c1 = ((nv > 1 ? l1 : 4096u) << 2) | 1u;
  uint32_t c2 = ((nv > 2 ? l2 : 4096u) << 2) | 2u, c3 = ((nv > 3 ? l3 : 4096u) << 2) | 3u;
#define GAMMA_CX(x, y)                 \
  {                                    \
    const uint32_t t_ = min(x, y);     \
    y = max(x, y);                     \
    x = t_;                            \
  }
  GAMMA_CX(c0, c1);
  GAMMA_CX(c2, c3);
  GAMMA_CX(c0, c2);
  GAMMA_CX(c1, c3);
  GAMMA_CX(c1, c2);
#undef GAMMA_CX
  const uint32_t ordw = (c0 & 3u) | (c1 & 3u) << 2 | (c2 & 3u) << 4 | (c3 & 3u) << 6;
  const uint32_t posw = (1u << (2 * (c1 & 3u))) | (2u << (2 * (c2 & 3u))) | (3u << (2 * (c3 & 3u)));
  uint32_t M = 0;
#pragma unroll
  for (uint32_t i = 0; i < 6; i++)
    if ((em >> i) & 1u) {
      const uint32_t pa = (posw >> (2 * ((kPairA >> (2 * i)) & 3u))) & 3u;
      const uint32_t pb = (posw >> (2 * ((kPairB >> (2 * i)) & 3u))) & 3u;
      M |= 1u << pid(pa, pb);
    }
  const uint32_t s0 = c0 >> 2, s1 = c1 >> 2, s2 = c2 >> 2, s3 = c3 >> 2;
  const uint32_t tie = (uint32_t)(s0 == s1) | (uint32_t)(nv > 2 && s1 == s2) << 1 | (uint32_t)(nv > 3 && s2 == s3) << 2;
  const uint2 e = tab[(M << 3) | tie];
  uint64_t key = kKeyTag | ((uint64_t)nv << 48) | ((uint64_t)__popc(M) << 51) | ((uint64_t)e.x << 53);
  key |= (uint64_t)(s0 & 0xfffu) | (uint64_t)(s1 & 0xfffu) << 12;
  if (nv > 2) key |= (uint64_t)(s2 & 0xfffu) << 24;
  if (nv > 3) key |= (uint64_t)(s3 & 0xfffu) << 36;
  return Canon{key, e.y, ordw};
}

__device__ __forceinline__ uint32_t pick4(uint32_t i, uint32_t v0, uint32_t v1, uint32_t v2, uint32_t v3) {
  return i == 0 ? v0 : i == 1 ? v1 : i == 2 ? v2 : v3;
}

// Aggregation: OR the vertex of every position of every minimizing order into the
// position's domain bitmap (read-before-atomic: most bits are already set).  Memory-level
// parallelism (ncu c4s20 r02: 40 % of the kernel's stalls waited on these reads one by
// one): the local vertices' in-class ranks are loaded before the slot lookup returns,
// and all positions' domain words of one minimizing order are read before any atomic.
// k0..k3: the in-class ranks (lrank) of the local vertices -- the enumeration loads the
// root edge's once per edge, a prefix's third once per prefix, only a new fourth vertex
// per embedding.
// OR the bits of the local vertices in `only` (bit i: local vertex i) into the domains
// (base offset d) at every position a minimizing order gives them.
__device__ __forceinline__ void record_bits(const FpmArgs &a, const uint32_t *prm, const Canon &cn,
                                            unsigned long long d, uint32_t k0, uint32_t k1, uint32_t k2, uint32_t k3,
                                            uint32_t nv, uint32_t only) {
  uint64_t off[4];
  off[0] = d - 1;
  off[1] = off[0] + __ldg(a.cwords + key_label(cn.key, 0));
  off[2] = off[1] + __ldg(a.cwords + key_label(cn.key, 1));
  off[3] = off[2] + (nv > 2 ? __ldg(a.cwords + key_label(cn.key, 2)) : 0u);
  uint32_t m = cn.minmask;
  while (m) {
    const int r = __ffs(m) - 1;
    m &= m - 1;
    const uint32_t sg = prm[r];
    uint32_t *w[4];
    uint32_t bb[4], x[4];
    bool on[4];
#pragma unroll
    for (uint32_t c = 0; c < 4; c++) {
      const uint32_t sp = (sg >> (2 * c)) & 3u;            // sorted position placed at canonical c
      const uint32_t lv = (cn.ordw >> (2 * sp)) & 3u;      // its local vertex
      const uint32_t bit = pick4(lv, k0, k1, k2, k3);
      w[c] = a.T.pool + off[c] + (bit >> 5);
      bb[c] = 1u << (bit & 31);
      on[c] = c < nv && ((only >> lv) & 1u);
    }
#pragma unroll
    for (uint32_t c = 0; c < 4; c++) x[c] = on[c] ? __ldcg(w[c]) : ~0u;
#pragma unroll
    for (uint32_t c = 0; c < 4; c++)
      if (!(x[c] & bb[c])) atomicOr(w[c], bb[c]);
  }
}

// Record one embedding: its canonical code, the pattern slot (claimed on first sight),
// then the domain bits of every local vertex.  Returns the slot's domain offset d
// (0: no slot, the table is full; ~0: no domains in this pass).
__device__ unsigned long long record(const FpmArgs &a, const uint2 *tab, const uint32_t *prm, uint32_t k0,
                                     uint32_t k1, uint32_t k2, uint32_t k3, uint32_t l0, uint32_t l1, uint32_t l2,
                                     uint32_t l3, uint32_t nv, uint32_t em) {
  const Canon cn = canonical(tab, l0, l1, l2, l3, nv, em);
  unsigned long long d = 0;
  const int64_t s = table_slot(a, cn.key, true, d);
  if (s < 0) return 0;
  // the claimer may still be carving this slot's domains (a few instructions away);
  // the wait yields with nanosleep so a claiming lane of the same warp progresses.
  // (No fence: the pool words were zeroed before the launch; the claimer only
  // publishes an offset.)
  while (d == 0) {
    __nanosleep(32);
    d = __ldcg(&a.T.slots[2 * s + 1]);
  }
  if (d == ~0ull) return d;   // no domains in this pass (pool exhausted / another chunk)
  // instances: counted in the one pass that carves the slot's domains
  if (a.T.inst) atomicAdd(&a.T.inst[s], 1ull);
  record_bits(a, prm, cn, d, k0, k1, k2, k3, nv, 0xfu);
  return d;
}

// Level-3 memo (per warp, per window of prefixes): (prefix j, edge mask, label of the
// new vertex) -> the slot's domain offset.  Two embeddings with the same key have the
// same labels and edges, hence the same canonical code, slot and minimizing orders:
// the prefix's vertices u, v, y land on the same positions, so the later one only adds
// its new vertex z -- no slot lookup and three of four domain words skipped (a hub
// prefix has hundreds of z, its labels repeat).  Entry: key << 40 | d (d < 2^40; the
// all-ones low part stands for "no domains in this pass"); one 64-bit word, so a
// concurrent overwrite by a colliding key never tears.
constexpr int kMemoBits = 7;   // 128 entries (1 KB) per warp
constexpr uint64_t kMemoD = (1ull << 40) - 1;

__device__ __forceinline__ uint32_t memo_key(uint32_t j, uint32_t em, uint32_t l3) {
  return 1u | (j << 1) | (em << 6) | (l3 << 12);   // 24 bits (labels < 4096, em < 64, j < 32)
}

// Is the pattern of this (prefix) edge set frequent?  (Alg. 2 line 4 pruning)
__device__ __forceinline__ bool frequent(const FpmArgs &a, const uint2 *tab, uint32_t l0, uint32_t l1, uint32_t l2,
                                         uint32_t nv, uint32_t em) {
  const Canon cn = canonical(tab, l0, l1, l2, 0u, nv, em);
  unsigned long long d;
  const int64_t s = table_slot(a, cn.key, false, d);
  return s >= 0 && a.T.freq[s];
}

// One warp per batch of root edges e1 = (u, v), v > u.
//   level 1: record e1.
//   level 2: e2 > e1 adjacent to e1 (an edge at u or v), prefix {e1} frequent.
//   level 3: from each frequent 2-edge prefix (a, b), a < b adjacent, add c with
//            (c > b, c adjacent to a or b)  or  (a < c < b, c adjacent to b, not to a).
//            Every connected {e1<e2<e3} arises exactly once: if e1~e2 from (e1,e2)+e3,
//            else (e3 joins them) from (e1,e3)+e2.
// Local vertices: 0 = u, 1 = v, 2 = the new end y of e2, 3 = the new end of e3.
__global__ void __launch_bounds__(kThreads) fpm_enum_kernel(FpmArgs a) {
  __shared__ uint2 s_tab[kCanonEntries];
  __shared__ uint32_t s_prm[24];
  __shared__ unsigned long long s_memo[kThreads / 32][1 << kMemoBits];
  for (int i = threadIdx.x; i < kCanonEntries; i += blockDim.x) s_tab[i] = a.canon_tab[i];
  if (threadIdx.x < 24) s_prm[threadIdx.x] = a.perm_tab[threadIdx.x];
  __syncthreads();
  const int lane = threadIdx.x & 31;
  unsigned long long *memo = s_memo[threadIdx.x >> 5];
  const bool use_memo = a.level == 3 && a.T.inst == nullptr && GAMMA_FPM_MEMO;   // (instance counts need every record)
  uint64_t emb = 0, elems = 0;       // embeddings recorded; adjacency elements streamed (lane 0)
  const uint64_t ndir = a.rp[a.n];   // directed edges: the roots are the (u, v > u) ones
  constexpr uint64_t kBatch = 8;
  for (;;) {
    // work unit = a batch of root edges (not a root vertex: a hub's edges spread
    // over many warps)
    unsigned long long b = 0;
    if (lane == 0) b = atomicAdd(&a.ctrl[CTRL_WORK], 1ull);
    b = __shfl_sync(0xffffffffu, b, 0);
    const uint64_t i0 = (b * a.world + a.rank) * kBatch;   // this rank's share of the batches
    if (i0 >= ndir) break;
    // u = row of directed edge i0 (binary search of row_ptr)
    uint32_t u;
    {
      uint32_t lo = 0, hi = a.n;
      while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (a.rp[mid] <= i0) lo = mid; else hi = mid;
      }
      u = lo;
    }
    const uint64_t iend = i0 + kBatch < ndir ? i0 + kBatch : ndir;
    for (uint64_t i1 = i0; i1 < iend; i1++) {
      while (a.rp[u + 1] <= i1) u++;   // the batch may cross rows
      const uint32_t v = a.col[i1];
      if (v < u) continue;             // each undirected edge once, from its smaller end
      const uint64_t us = a.rp[u], ue = a.rp[u + 1];
      const uint64_t e1 = ekey(u, v);
      const uint32_t lu = labof(a, u), lv = labof(a, v);
      if (lu < a.walk_lo || lv < a.walk_lo) continue;   // uniform; 0 except in chunk passes
      const uint32_t ku = __ldg(a.lrank + u), kv = __ldg(a.lrank + v);   // in-class ranks of the root edge
      if (a.level == 1) {
        if (lane == 0) {
          record(a, s_tab, s_prm, ku, kv, 0u, 0u, lu, lv, 0u, 0u, 2, 1u << pid(0, 1));
          emb++;
        }
        continue;
      }
      if (!frequent(a, s_tab, lu, lv, 0u, 2, 1u << pid(0, 1))) continue;   // uniform: same e1 in all lanes
      // candidate second edges: incident to u or v (lists of u then v), e2 > e1
      const uint64_t vs = a.rp[v], ve = a.rp[v + 1];
      const uint64_t nu = ue - us, ncand = nu + (ve - vs);
      if (lane == 0) elems += ncand;
      for (uint64_t c0 = 0; c0 < ncand; c0 += 32) {
        if (use_memo) {   // the memo's prefix indices are this window's
          __syncwarp();   // every lane is done with the previous window's entries
#pragma unroll
          for (int q = 0; q < (1 << kMemoBits) / 32; q++) memo[lane + 32 * q] = 0ull;
          __syncwarp();
        }
        const uint64_t ci = c0 + lane;
        // lane's second edge e2 = (x, y), x in {u, v}: a candidate prefix {e1, e2}
        bool valid = ci < ncand;
        uint64_t e2 = 0;
        uint32_t y = 0, ly = 0, em2 = 0;
        if (valid) {
          const bool at_u = ci < nu;
          y = at_u ? a.col[us + ci] : a.col[vs + (ci - nu)];
          e2 = ekey(at_u ? u : v, y);
          valid = e2 > e1;   // also drops e1 itself (y is then u or v)
          em2 = (1u << pid(0, 1)) | (1u << pid(at_u ? 0 : 1, 2));
        }
        if (valid) {
          ly = labof(a, y);
          valid = ly >= a.walk_lo;
        }
        if (valid) {
          if (a.level == 2) {
            record(a, s_tab, s_prm, ku, kv, __ldg(a.lrank + y), 0u, lu, lv, ly, 0u, 3, em2);
            emb++;
            valid = false;
          } else {
            valid = frequent(a, s_tab, lu, lv, ly, 3, em2);   // Alg. 2 line 4
          }
        }
        if (a.level == 2) continue;   // uniform
        // third edges: incident to the 3 vertices u, v, y of a frequent prefix.  The
        // candidate lists N(u) ++ N(v) ++ N(y) of the valid prefixes are concatenated
        // and streamed by all 32 lanes (flattened windows; prefix found by an
        // OR-reduction of the start offsets), so a hub prefix does not serialise on
        // one lane.  N(u), N(v) are the same for every prefix of this e1.
        const uint32_t du = (uint32_t)nu, dv = (uint32_t)(ve - vs);
        uint32_t by = 0, dy = 0, ky = 0;
        if (valid) {
          by = (uint32_t)a.rp[y];
          dy = (uint32_t)(a.rp[y + 1] - by);
          ky = __ldg(a.lrank + y);
        }
        const uint32_t tl = valid ? du + dv + dy : 0u;
        const uint32_t nz = __ballot_sync(0xffffffffu, tl > 0);
        const uint32_t nnz = __popc(nz);
        const uint32_t src = lane < (int)nnz ? __fns(nz, 0, lane + 1) : 0;
        // compacted prefix data (lane k = k-th valid prefix); em2 travels in the top
        // bits of the label word (labels < 4096)
        const uint32_t cy = __shfl_sync(0xffffffffu, y, src);
        const uint32_t cl = __shfl_sync(0xffffffffu, ly | (em2 << 16), src);
        const uint32_t cby = __shfl_sync(0xffffffffu, by, src);
        const uint32_t cky = __shfl_sync(0xffffffffu, ky, src);
        const uint32_t stl = __shfl_sync(0xffffffffu, tl, src);
        const uint32_t ctl = lane < (int)nnz ? stl : 0u;
        uint32_t sc = ctl;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t yv = __shfl_up_sync(0xffffffffu, sc, o);
          if (lane >= o) sc += yv;
        }
        const uint32_t T = __shfl_sync(0xffffffffu, sc, 31);
        if (lane == 0) elems += T;
        const uint32_t ost = sc - ctl;
        const uint32_t upto = lane == 31 ? 0xffffffffu : ((2u << lane) - 1u);
        uint32_t nb = 0;
        for (uint32_t t0 = 0; t0 < T; t0 += 32) {
          const uint32_t t = t0 + lane;
          const uint32_t mine = (lane < (int)nnz && ost >= t0 && ost < t0 + 32) ? (1u << (ost - t0)) : 0u;
          const uint32_t S = __reduce_or_sync(0xffffffffu, mine);
          const int j = ((int)(nb + __popc(S & upto)) - 1) & 31;
          nb += __popc(S);
          const uint32_t py = __shfl_sync(0xffffffffu, cy, j);
          const uint32_t pl = __shfl_sync(0xffffffffu, cl, j);
          const uint32_t pby = __shfl_sync(0xffffffffu, cby, j);
          const uint32_t pky = __shfl_sync(0xffffffffu, cky, j);
          const uint32_t oj = __shfl_sync(0xffffffffu, ost, j);
          if (t >= T) continue;
          const uint32_t r = t - oj;
          uint32_t w, zi, lw;
          if (r < du) { w = u; zi = (uint32_t)us + r; lw = 0; }
          else if (r < du + dv) { w = v; zi = (uint32_t)vs + (r - du); lw = 1; }
          else { w = py; zi = pby + (r - du - dv); lw = 2; }
          const uint32_t z = a.col[zi];
          // an edge joining two prefix vertices is seen from both ends: keep the smaller
          const uint32_t lz = z == u ? 0u : z == v ? 1u : z == py ? 2u : 3u;
          if (lz < 3 && z < w) continue;
          const uint64_t pe2 = ekey((pl >> 16) & (1u << pid(1, 2)) ? v : u, py);
          const uint64_t e3 = ekey(w, z);
          if (e3 == e1 || e3 == pe2) continue;
          const bool ok = (e3 > pe2) || (e3 > e1 && shares(e3, pe2) && !shares(e3, e1));
          if (!ok) continue;
          const uint32_t em3 = (pl >> 16) | (1u << pid(lw, lz));
          const uint32_t l3 = lz == 3 ? labof(a, z) : 0u;
          if (lz == 3 && l3 < a.walk_lo) continue;
          const uint32_t kz = lz == 3 ? __ldg(a.lrank + z) : 0u;
          emb++;
          if (use_memo) {
            const uint32_t mk = memo_key((uint32_t)j, em3, l3);
            const uint32_t mh = (mk * 0x9E3779B1u) >> (32 - kMemoBits);
            const unsigned long long me = memo[mh];
            if ((uint32_t)(me >> 40) == mk) {   // seen: only the new vertex's bits
              const unsigned long long dd = me & kMemoD;
              if (dd != kMemoD && lz == 3)
                record_bits(a, s_prm, canonical(s_tab, lu, lv, pl & 0xffffu, l3, 4, em3), dd, 0u, 0u, 0u, kz, 4,
                            0x8u);
              continue;
            }
            const unsigned long long dd = record(a, s_tab, s_prm, ku, kv, pky, kz, lu, lv, pl & 0xffffu, l3,
                                                 lz == 3 ? 4 : 3, em3);
            if (dd) memo[mh] = ((unsigned long long)mk << 40) | (dd == ~0ull ? kMemoD : dd);
            continue;
          }
          record(a, s_tab, s_prm, ku, kv, pky, kz, lu, lv, pl & 0xffffu, l3, lz == 3 ? 4 : 3, em3);
        }
      }
    }
  }
  for (int off = 16; off > 0; off >>= 1) emb += __shfl_down_sync(0xffffffffu, emb, off);
  if (lane == 0 && emb) atomicAdd(&a.ctrl[CTRL_ENTRIES], (unsigned long long)emb);
  if (lane == 0 && elems) atomicAdd(&a.ctrl[CTRL_ELEMS], (unsigned long long)elems);
}

// Support of every slot of the given level: min over positions of popcount; one
// warp per slot.
__global__ void fpm_support_kernel(FpmArgs a, uint32_t level, uint64_t minsup) {
  const int lane = threadIdx.x & 31;
  const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t s = warp; s < a.T.cap; s += nwarps) {
    const uint64_t key = a.T.slots[2 * s];
    if (key == 0) continue;
    const uint32_t nv = key_nv(key), ne = key_ne(key);
    if (ne != level) continue;
    // no domains in this pass (pool exhausted, or another chunk of a split level):
    // a later pass computes this slot
    const unsigned long long d = a.T.slots[2 * s + 1];
    if (d == 0 || d == ~0ull) continue;
    uint64_t sup = ~0ull;
    for (uint32_t p = 0; p < nv; p++) {
      const uint32_t lp = key_label(key, p);
      const uint64_t words = a.cwords[lp];
      uint64_t off = d - 1;
      for (uint32_t i = 0; i < p; i++) off += a.cwords[key_label(key, i)];
      uint64_t c = 0;
      for (uint64_t w = lane; w < words; w += 32) c += __popc(a.T.pool[off + w]);
      for (int o = 16; o > 0; o >>= 1) c += __shfl_down_sync(0xffffffffu, c, o);
      c = __shfl_sync(0xffffffffu, c, 0);
      sup = c < sup ? c : sup;
    }
    if (lane == 0) {
      a.T.support[s] = sup;
      a.T.freq[s] = sup >= minsup ? 1u : 0u;
    }
  }
}

// frequent slots -> compact (key, support, instances) arrays; dist_level: slots of this
// level come from the distributed path instead (skipped)
__global__ void collect_kernel(const unsigned long long *slots, const unsigned long long *sup, const uint32_t *freq,
                               const unsigned long long *inst, uint64_t cap, uint32_t dist_level,
                               unsigned long long *ok, unsigned long long *os, unsigned long long *oi,
                               unsigned long long *cursor) {
  for (uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; s < cap; s += (uint64_t)gridDim.x * blockDim.x) {
    const unsigned long long k = slots[2 * s];
    if (k == 0 || !freq[s] || (dist_level && key_ne(k) == dist_level)) continue;
    const unsigned long long i = atomicAdd(cursor, 1ull);
    ok[i] = k;
    os[i] = sup[s];
    if (inst) oi[i] = inst[s];
  }
}

__global__ void label_hist_kernel(const uint32_t *lab, uint32_t n, uint32_t *csize, uint32_t *lrank_tmp) {
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
    atomicAdd(&csize[lab ? lab[v] : 0u], 1u);
}

__global__ void label_keys_kernel(const uint32_t *lab, uint32_t n, uint64_t *keys) {
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
    keys[v] = ((uint64_t)(lab ? lab[v] : 0u) << 32) | v;
}

// sorted (label, v) keys -> rank of v inside its label class
__global__ void label_rank_kernel(const uint64_t *sorted, uint32_t n, uint32_t *lrank) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t l = (uint32_t)(sorted[i] >> 32);
    // class start: binary search for the first key with this label
    uint64_t lo = 0, hi = i;
    while (lo < hi) {
      const uint64_t mid = (lo + hi) >> 1;
      if ((uint32_t)(sorted[mid] >> 32) < l) lo = mid + 1; else hi = mid;
    }
    lrank[(uint32_t)sorted[i]] = (uint32_t)(i - lo);
  }
}

__global__ void max_label_kernel(const uint32_t *lab, uint32_t n, unsigned long long *out) {
  unsigned long long m = 0;
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
    m = lab[v] > m ? lab[v] : m;
  for (int o = 16; o > 0; o >>= 1) {
    const unsigned long long x = __shfl_down_sync(0xffffffffu, m, o);
    m = x > m ? x : m;
  }
  if ((threadIdx.x & 31) == 0) atomicMax(out, m);
}

// ---- distributed last level (world > 1) ----
// this rank's pattern codes of one level, in any order
__global__ void level_keys_kernel(const unsigned long long *key, uint64_t cap, uint32_t level,
                                  unsigned long long *out, unsigned long long *cursor) {
  for (uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; s < cap; s += (uint64_t)gridDim.x * blockDim.x) {
    const unsigned long long k = key[2 * s];   // slots: (key, dom) pairs
    if (k && key_ne(k) == level) out[atomicAdd(cursor, 1ull)] = k;
  }
}

// after the all-to-all, recv holds G shards of this rank's word range: OR them into
// the first one
__global__ void or_shards_kernel(uint32_t *recv, uint32_t G, uint64_t shard) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < shard; i += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t x = recv[i];
    for (uint32_t g = 1; g < G; g++) x |= recv[g * shard + i];
    recv[i] = x;
  }
}

// popcount of the part of each domain bitmap (global word range [off, off + w)) that
// lies in this rank's range [lo, lo + shard); one warp per bitmap
__global__ void seg_popc_kernel(const uint32_t *buf, uint64_t lo, uint64_t shard, const uint64_t *seg_off,
                                const uint32_t *seg_w, uint64_t nseg, unsigned long long *cnt) {
  const int lane = threadIdx.x & 31;
  const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t q = warp; q < nseg; q += nwarps) {
    const uint64_t b = seg_off[q] > lo ? seg_off[q] : lo;
    const uint64_t e0 = seg_off[q] + seg_w[q], e1 = lo + shard;
    const uint64_t e = e0 < e1 ? e0 : e1;
    unsigned long long c = 0;
    for (uint64_t x = b + lane; x < e; x += 32) c += __popc(buf[x - lo]);
    for (int o = 16; o > 0; o >>= 1) c += __shfl_down_sync(0xffffffffu, c, o);
    if (lane == 0) cnt[q] = c;
  }
}

#include "fpm4_device.cuh"

inline unsigned g1d(uint64_t n) {
  const uint64_t b = (n + 255) / 256;
  return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(b, 148u * 32u));
}

}  // namespace

// Canonical-code tables for the device (reading R7), by enumeration of the 24 vertex
// orders sigma of the sorted positions: entry (M << 3 | tie) = {min over valid sigma of
// the sorted edge-pair key of the edge mask M under sigma, set of sigmas reaching it}.
// sigma is valid iff it only permutes positions of equal labels (tie bit i: sorted
// labels i and i+1 equal).  perm rows in lexicographic order, sigma[c] in bits 2c.
static void fpm_canon_tables(std::vector<uint2> &tab, std::vector<uint32_t> &prm) {
  std::vector<std::array<uint32_t, 4>> perms;
  std::array<uint32_t, 4> p{0, 1, 2, 3};
  do perms.push_back(p);
  while (std::next_permutation(p.begin(), p.end()));
  prm.assign(24, 0);
  for (int r = 0; r < 24; r++)
    for (int c = 0; c < 4; c++) prm[r] |= perms[r][c] << (2 * c);
  tab.assign(kCanonEntries, make_uint2(0, 0));
  for (uint32_t M = 0; M < 64; M++)
    for (uint32_t tie = 0; tie < 8; tie++) {
      uint32_t grp[4] = {0, 0, 0, 0};
      for (int i = 0; i < 3; i++) grp[i + 1] = grp[i] + (((tie >> i) & 1) ? 0 : 1);
      uint32_t best = 0xffffffffu, mask = 0;
      for (int r = 0; r < 24; r++) {
        const auto &sg = perms[r];
        bool ok = true;
        for (int c = 0; c < 4; c++) ok = ok && grp[sg[c]] == grp[c];
        if (!ok) continue;
        uint32_t inv[4];
        for (uint32_t c = 0; c < 4; c++) inv[sg[c]] = c;
        uint32_t idx[3] = {7, 7, 7}, ne = 0;
        for (uint32_t q = 0; q < 4; q++)
          for (uint32_t pp = 0; pp < q; pp++)
            if ((M >> pid(pp, q)) & 1u) {
              const uint32_t x = inv[pp], y = inv[q];
              if (ne < 3) idx[ne] = pid(std::min(x, y), std::max(x, y));
              ne++;
            }
        if (ne > 3) continue;   // not a pattern of <= 3 edges
        std::sort(idx, idx + 3);
        const uint32_t key = idx[0] * 64 + idx[1] * 8 + idx[2];
        if (key < best) {
          best = key;
          mask = 1u << r;
        } else if (key == best) {
          mask |= 1u << r;
        }
      }
      tab[(M << 3) | tie] = make_uint2(best == 0xffffffffu ? 0u : best, mask);
    }
}

// one column (0 = key, 1 = dom) of the (key, dom) slot pairs <-> a dense host array
static void slots_get(gamma_ctx *ctx, std::vector<unsigned long long> &h, const unsigned long long *slots,
                      uint64_t cap, int colm) {
  h.resize(cap);
  GAMMA_CUDA(cudaMemcpy2DAsync(h.data(), 8, slots + colm, 16, 8, cap, cudaMemcpyDeviceToHost, ctx->stream));
}
static void slots_put(gamma_ctx *ctx, unsigned long long *slots, const std::vector<unsigned long long> &h,
                      uint64_t cap, int colm) {
  GAMMA_CUDA(cudaMemcpy2DAsync(slots + colm, 16, h.data(), 8, 8, cap, cudaMemcpyHostToDevice, ctx->stream));
}

// Host-side parallel helpers for the result (C4: 1.2e6 patterns; one thread took 280 ms
// to decode and sort them).  f(i0, i1) over [0, n) in contiguous chunks.
static unsigned host_threads(size_t n) {
  const unsigned hw = std::max(1u, std::thread::hardware_concurrency());
  return n < (1u << 15) ? 1u : std::min(16u, hw);
}

template <class F>
static void par_for(size_t n, F &&f) {
  const unsigned T = host_threads(n);
  if (T <= 1) {
    f(0, n);
    return;
  }
  std::vector<std::thread> th;
  for (unsigned t = 0; t < T; t++) th.emplace_back([&, t] { f(n * t / T, n * (t + 1) / T); });
  for (auto &x : th) x.join();
}

// sort = chunk sorts on host threads, then pairwise merges
template <class V>
static void par_sort(V &v) {
  const size_t n = v.size();
  unsigned P = 1;
  while (P * 2 <= host_threads(n)) P *= 2;
  if (P <= 1) {
    std::sort(v.begin(), v.end());
    return;
  }
  std::vector<size_t> b(P + 1);
  for (unsigned i = 0; i <= P; i++) b[i] = n * i / P;
  {
    std::vector<std::thread> th;
    for (unsigned i = 0; i < P; i++) th.emplace_back([&, i] { std::sort(v.begin() + b[i], v.begin() + b[i + 1]); });
    for (auto &x : th) x.join();
  }
  for (unsigned w = 1; w < P; w *= 2) {
    std::vector<std::thread> th;
    for (unsigned i = 0; i + w < P; i += 2 * w)
      th.emplace_back([&, i, w] {
        std::inplace_merge(v.begin() + b[i], v.begin() + b[i + w], v.begin() + b[std::min(i + 2 * w, P)]);
      });
    for (auto &x : th) x.join();
  }
}

static gamma_fpm_pattern decode_pattern(uint64_t key, uint64_t support, uint64_t instances = 0) {
  static const uint8_t pairs[6][2] = {{0, 1}, {0, 2}, {0, 3}, {1, 2}, {1, 3}, {2, 3}};
  gamma_fpm_pattern p{};
  p.nv = key_nv(key);
  p.ne = key_ne(key);
  const uint32_t ek = key_edges(key);
  const uint32_t idx[3] = {ek / 64, (ek / 8) % 8, ek % 8};
  for (uint32_t i = 0; i < p.nv; i++) p.labels[i] = key_label(key, i);
  for (uint32_t e = 0; e < p.ne; e++) {
    const uint32_t id = idx[e];   // sorted pair indices first, unused slots hold 7
    p.edges[e][0] = pairs[id][0];
    p.edges[e][1] = pairs[id][1];
  }
  p.support = support;
  p.instances = instances;
  return p;
}

// Algorithmic bytes of one enumeration pass (FPM): 4 B per adjacency
// element streamed by the extension, 32 B per recorded embedding (its 16-byte
// pattern-table slot + one 4-byte domain word per position, <= 4 positions).
static void count_fpm_bytes(gamma_ctx *ctx) {
  ctx->stats.alg_bytes[KC_FPM] += 4 * ctx->ctrl_host[CTRL_ELEMS] + 32 * ctx->ctrl_host[CTRL_ENTRIES];
}

static void coll_allreduce(gamma_ctx *ctx, uint64_t *v, size_t n) {
  const gamma_status st = ctx->desc.allreduce_sum_u64(v, n, ctx->desc.coll_user);
  GAMMA_REQUIRE(st == GAMMA_OK, st, "allreduce_sum_u64 callback failed");
}

static void coll_alltoall(gamma_ctx *ctx, const uint32_t *send, uint32_t *recv, uint64_t n_per_rank) {
  ctx->sync();   // the callback may run on another stream
  const gamma_status st = ctx->desc.alltoall_u32(send, recv, n_per_rank, ctx->desc.coll_user);
  GAMMA_REQUIRE(st == GAMMA_OK, st, "alltoall_u32 callback failed");
}

// The last level of a multi-GPU FPM run: every rank enumerates only its
// share of the root-edge batches, so a pattern's MNI domains are spread over the
// ranks and must be OR-ed.  1. claim pass: the rank's level-l pattern codes enter its
// table (no domains); 2. the codes are all-to-all exchanged, sorted and deduplicated
// into the same global list U on every rank; 3. U is cut into chunks whose domains fit
// half the pool, laid out identically on every rank; per chunk each rank re-runs its
// share of the enumeration recording into that layout, the bitmaps are all-to-all
// exchanged in G shards (NCCL has no bitwise-OR reduction), each rank ORs the shards
// of its word range and popcounts the pieces of every domain in it, and one SUM
// all-reduce of those pieces gives every rank the same |domain| per (pattern,
// position), hence the same supports and output.  Returns false when some rank's
// table overflowed (all ranks then grow it and retry together).
static bool fpm_dist_level(gamma_ctx *ctx, FpmArgs &a, int grid_enum, uint32_t l, uint64_t minsup,
                           const std::vector<uint32_t> &hsize, uint64_t cap, unsigned long long *slots_d,
                           uint32_t *pool_d, uint64_t pool_words,
                           unsigned long long *pcur_d, std::vector<gamma_fpm_pattern> &found) {
  const uint32_t G = (uint32_t)ctx->desc.world, R = (uint32_t)ctx->desc.rank;
  a.level = l;
  a.rank = R;
  a.world = G;
  // ---- 1. claim pass ----
  a.claim_only = 1;
  ctrl_reset(ctx);
  ctx->launch(KC_FPM, [&] { fpm_enum_kernel<<<grid_enum, kThreads, 0, ctx->stream>>>(a); });
  a.claim_only = 0;
  DevBuf<unsigned long long> mine(ctx, cap);
  ctx->launch(KC_MISC, [&] {
    level_keys_kernel<<<g1d(cap), 256, 0, ctx->stream>>>(slots_d, cap, l, mine.p,
                                                         (unsigned long long *)ctx->ctrl + CTRL_AUX0);
  });
  ctrl_fetch(ctx);
  // agree on: table overflow anywhere, every rank's code count, the smallest pool,
  // and the level's embedding count
  std::vector<uint64_t> v(2 * G + 2, 0);
  v[R] = ctx->ctrl_host[CTRL_AUX0];
  v[G + R] = pool_words;
  v[2 * G] = ctx->ctrl_host[CTRL_ERR] != 0;
  v[2 * G + 1] = ctx->ctrl_host[CTRL_ENTRIES];
  coll_allreduce(ctx, v.data(), v.size());
  if (v[2 * G]) return false;
  ctx->stats.level_entries[l] = v[2 * G + 1];
  uint64_t maxc = 1, half = ~0ull;
  for (uint32_t r = 0; r < G; r++) {
    maxc = std::max<uint64_t>(maxc, v[r]);
    half = std::min<uint64_t>(half, v[G + r] / 2);
  }
  const uint64_t nmine = v[R];
  // ---- 2. global code list U ----
  uint64_t nU = 0;
  std::vector<unsigned long long> U;
  {
    DevBuf<unsigned long long> send(ctx, G * maxc), recv(ctx, G * maxc), sorted(ctx, G * maxc);
    GAMMA_CUDA(cudaMemsetAsync(send.p, 0, G * maxc * 8, ctx->stream));
    for (uint32_t r = 0; r < G; r++)
      if (nmine)
        GAMMA_CUDA(cudaMemcpyAsync(send.p + r * maxc, mine.p, nmine * 8, cudaMemcpyDeviceToDevice, ctx->stream));
    coll_alltoall(ctx, (const uint32_t *)send.p, (uint32_t *)recv.p, 2 * maxc);
    const uint64_t tot = G * maxc;
    size_t t1 = 0, t2 = 0;
    GAMMA_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, t1, recv.p, sorted.p, tot, 0, 64, ctx->stream));
    GAMMA_CUDA(cub::DeviceSelect::Unique(nullptr, t2, sorted.p, send.p, (unsigned long long *)ctx->ctrl + CTRL_AUX1,
                                         tot, ctx->stream));
    DevBuf<uint8_t> tmp(ctx, std::max(t1, t2));
    ctx->launch(KC_MISC, [&] {
      GAMMA_CUDA(cub::DeviceRadixSort::SortKeys(tmp.p, t1, recv.p, sorted.p, tot, 0, 64, ctx->stream));
    });
    ctx->cub_sort_launched(KC_MISC, tot, 64);
    ctx->launch(KC_MISC, [&] {
      GAMMA_CUDA(cub::DeviceSelect::Unique(tmp.p, t2, sorted.p, send.p, (unsigned long long *)ctx->ctrl + CTRL_AUX1,
                                           tot, ctx->stream));
    });
    ctx->cub_select_launched(KC_MISC);
    ctrl_fetch(ctx);
    nU = ctx->ctrl_host[CTRL_AUX1];
    U.resize(nU);
    if (nU) GAMMA_CUDA(cudaMemcpyAsync(U.data(), send.p, nU * 8, cudaMemcpyDeviceToHost, ctx->stream));
    ctx->sync();
    if (nU && U[0] == 0) U.erase(U.begin());   // padding
  }
  // ---- 3. chunks of U ----
  std::vector<unsigned long long> hkey, hdom(cap);
  slots_get(ctx, hkey, slots_d, cap, 0);
  ctx->sync();
  std::unordered_map<uint64_t, uint64_t> slot_of;
  slot_of.reserve(nmine * 2 + 1);
  for (uint64_t s = 0; s < cap; s++)
    if (hkey[s] && key_ne(hkey[s]) == l) slot_of.emplace(hkey[s], s);
  uint32_t *dom_buf = pool_d, *recv_buf = pool_d + half;
  std::vector<uint64_t> seg_off;
  std::vector<uint32_t> seg_w;
  size_t next = 0;
  while (next < U.size()) {
    std::fill(hdom.begin(), hdom.end(), ~0ull);
    seg_off.clear();
    seg_w.clear();
    uint64_t used = 0;
    const size_t j0 = next;
    for (; next < U.size(); next++) {
      const uint64_t k = U[next];
      uint64_t words = 0;
      for (uint32_t p = 0; p < key_nv(k); p++) words += (hsize[key_label(k, p)] + 31) / 32;
      GAMMA_REQUIRE(words + G <= half, GAMMA_E_NOMEM, "gamma_fpm: one pattern's domains exceed the HBM budget");
      if (used + words + G > half) break;
      auto it = slot_of.find(k);
      if (it != slot_of.end()) hdom[it->second] = 1 + used;
      for (uint32_t p = 0; p < key_nv(k); p++) {
        const uint32_t w = (hsize[key_label(k, p)] + 31) / 32;
        seg_off.push_back(used);
        seg_w.push_back(w);
        used += w;
      }
    }
    const size_t j1 = next;
    const uint64_t shard = (used + G - 1) / G;
    slots_put(ctx, slots_d, hdom, cap, 1);
    GAMMA_CUDA(cudaMemsetAsync(dom_buf, 0, shard * G * 4, ctx->stream));
    GAMMA_CUDA(cudaMemcpyAsync(pcur_d, &pool_words, 8, cudaMemcpyHostToDevice, ctx->stream));
    ctrl_reset(ctx);
    ctx->launch(KC_FPM, [&] { fpm_enum_kernel<<<grid_enum, kThreads, 0, ctx->stream>>>(a); });
    ctrl_fetch(ctx);
    count_fpm_bytes(ctx);
    GAMMA_REQUIRE(ctx->ctrl_host[CTRL_ERR] == 0 && ctx->ctrl_host[CTRL_OVF] == 0, GAMMA_E_CUDA,
                  "gamma_fpm: a distributed chunk pass met an unclaimed pattern");
    coll_alltoall(ctx, dom_buf, recv_buf, shard);
    const uint64_t nseg = seg_off.size();
    DevBuf<uint64_t> soff = to_device(ctx, seg_off.data(), nseg);
    DevBuf<uint32_t> sw = to_device(ctx, seg_w.data(), nseg);
    DevBuf<unsigned long long> cnt(ctx, nseg);
    ctx->launch(KC_FPM_SUPPORT, [&] { or_shards_kernel<<<g1d(shard), 256, 0, ctx->stream>>>(recv_buf, G, shard); });
    ctx->launch(KC_FPM_SUPPORT, [&] {
      seg_popc_kernel<<<g1d(nseg * 32), 256, 0, ctx->stream>>>(recv_buf, R * shard, shard, soff.p, sw.p, nseg, cnt.p);
    });
    // per-segment popcounts, then (instance counting) each chunk pattern's instances
    std::vector<uint64_t> hc(nseg + (a.T.inst ? j1 - j0 : 0), 0);
    GAMMA_CUDA(cudaMemcpyAsync(hc.data(), cnt.p, nseg * 8, cudaMemcpyDeviceToHost, ctx->stream));
    std::vector<unsigned long long> hinst;
    if (a.T.inst) {
      hinst.resize(cap);
      GAMMA_CUDA(cudaMemcpyAsync(hinst.data(), a.T.inst, cap * 8, cudaMemcpyDeviceToHost, ctx->stream));
    }
    ctx->sync();
    if (a.T.inst)
      for (size_t j = j0; j < j1; j++) {
        auto it = slot_of.find(U[j]);
        if (it != slot_of.end()) hc[nseg + (j - j0)] = hinst[it->second];
      }
    coll_allreduce(ctx, hc.data(), hc.size());
    size_t q = 0;
    for (size_t j = j0; j < j1; j++) {
      uint64_t sup = ~0ull;
      for (uint32_t p = 0; p < key_nv(U[j]); p++, q++) sup = std::min<uint64_t>(sup, hc[q]);
      if (sup >= minsup) found.push_back(decode_pattern(U[j], sup, a.T.inst ? hc[nseg + (j - j0)] : 0));
    }
    if (a.T.inst) GAMMA_CUDA(cudaMemsetAsync(a.T.inst, 0, cap * 8, ctx->stream));
    ctx->stats.chunks++;
  }
  a.rank = 0;
  a.world = 1;
  return true;
}

// Worst-case MNI domain words of the level-l patterns, by the pattern's smallest label
// (every label combination of every shape occurring; shapes: edge; wedge; triangle,
// 3-star, 3-path).  Used to pick the label threshold below which the first pass of a
// level carves domains, so that the patterns left for the chunk passes all have large
// smallest labels -- and a chunk pass with smallest label lo skips every root edge,
// prefix and new vertex labelled below lo (few embeddings have only large labels).
static std::vector<double> fpm_words_by_min_label(uint32_t l, const std::vector<uint32_t> &cw) {
  const uint32_t L = (uint32_t)cw.size();
  std::vector<double> W(L, 0.0);
  if (l == 1) {
    for (uint32_t a = 0; a < L; a++)
      for (uint32_t b = a; b < L; b++) W[a] += cw[a] + cw[b];
  } else if (l == 2) {
    for (uint32_t c = 0; c < L; c++)
      for (uint32_t x = 0; x < L; x++)
        for (uint32_t y = x; y < L; y++) W[std::min(c, x)] += cw[c] + cw[x] + cw[y];
  } else if (l == 3) {
    for (uint32_t a = 0; a < L; a++)
      for (uint32_t b = a; b < L; b++)
        for (uint32_t c = b; c < L; c++) W[a] += cw[a] + cw[b] + cw[c];   // triangles
    for (uint32_t c = 0; c < L; c++)                                         // 3-stars
      for (uint32_t x = 0; x < L; x++)
        for (uint32_t y = x; y < L; y++)
          for (uint32_t z = y; z < L; z++) W[std::min(c, x)] += cw[c] + cw[x] + cw[y] + cw[z];
    for (uint32_t a = 0; a < L; a++)                                         // 3-paths a-b-c-d
      for (uint32_t b = 0; b < L; b++)
        for (uint32_t c = 0; c < L; c++)
          for (uint32_t d = 0; d < L; d++) {
            if (std::make_tuple(a, b, c, d) > std::make_tuple(d, c, b, a)) continue;   // one per reversal
            W[std::min(std::min(a, b), std::min(c, d))] += cw[a] + cw[b] + cw[c] + cw[d];
          }
  }
  return W;
}

// The MNI domain pool (most of free HBM) is taken with cudaMalloc and returned with
// cudaFree, not through the context's allocator: a caching allocator (PyTorch's)
// keeps a freed block reserved, and the next call would see a fraction of the HBM.
struct PoolBuf {
  uint32_t *p = nullptr;
  void alloc(uint64_t words) {
    reset();
    const cudaError_t e = cudaMalloc(&p, words * sizeof(uint32_t));
    if (e != cudaSuccess) {
      cudaGetLastError();
      p = nullptr;
      throw Fail{GAMMA_E_NOMEM, "gamma_fpm: cudaMalloc of the domain pool failed: " +
                                    std::string(cudaGetErrorString(e))};
    }
  }
  void reset() {
    if (p) cudaFree(p);
    p = nullptr;
  }
  ~PoolBuf() { reset(); }
};


// ---- level 4 (4-edge patterns, Opt 3 out-of-core aggregation), host side ----------
// Canonical-code table of <= 5-vertex, <= 4-edge patterns (reading R7), by enumeration
// of the 120 orders sigma of the sorted positions (sigma[c] = sorted position placed at
// canonical position c; valid iff it only permutes positions of equal labels): entry
// (M << 4 | tie) = {smallest sorted pair-index key of the edge mask M under sigma,
// the first minimizing sigma (3 bits per position) | the orbit representative of every
// canonical position under Aut_L of the canonical pattern << 15}.  The orbit of c is
// {c' : some minimizing sigma places at c' what the first one places at c}.
static void fpm_canon5_table(std::vector<uint2> &tab) {
  for (uint32_t x = 0; x < 3125; x++) {   // the sorting network, checked exhaustively
    uint32_t d[5], t = x;
    for (int i = 0; i < 5; i++) { d[i] = t % 5; t /= 5; }
    sort5(d[0], d[1], d[2], d[3], d[4]);
    for (int i = 0; i < 4; i++)
      GAMMA_REQUIRE(d[i] <= d[i + 1], GAMMA_E_CUDA, "gamma_fpm: 5-element sorting network is wrong");
  }
  std::vector<std::array<uint32_t, 5>> perms;
  std::array<uint32_t, 5> p{0, 1, 2, 3, 4};
  do perms.push_back(p);
  while (std::next_permutation(p.begin(), p.end()));
  tab.assign(kCanon5Entries, make_uint2(0, 0));
  for (uint32_t M = 0; M < 1024; M++) {
    if (__builtin_popcount(M) > 4) continue;
    for (uint32_t tie = 0; tie < 16; tie++) {
      uint32_t grp[5] = {0, 0, 0, 0, 0};
      for (int i = 0; i < 4; i++) grp[i + 1] = grp[i] + (((tie >> i) & 1) ? 0 : 1);
      uint32_t best = 0xffffffffu;
      std::vector<int> mins;
      for (int r = 0; r < 120; r++) {
        const auto &sg = perms[r];
        bool ok = true;
        for (int c = 0; c < 5; c++) ok = ok && grp[sg[c]] == grp[c];
        if (!ok) continue;
        uint32_t inv[5];
        for (uint32_t c = 0; c < 5; c++) inv[sg[c]] = c;
        uint32_t idx[4] = {15, 15, 15, 15}, ne = 0;
        for (uint32_t i = 0; i < 10; i++)
          if ((M >> i) & 1u) idx[ne++] = pid5u(inv[(kA5 >> (3 * i)) & 7u], inv[(kB5 >> (3 * i)) & 7u]);
        std::sort(idx, idx + ne);
        const uint32_t key = idx[0] << 12 | idx[1] << 8 | idx[2] << 4 | idx[3];
        if (key < best) {
          best = key;
          mins.assign(1, r);
        } else if (key == best) {
          mins.push_back(r);
        }
      }
      const auto &s0 = perms[mins[0]];
      uint32_t y = 0;
      for (uint32_t c = 0; c < 5; c++) {
        y |= s0[c] << (3 * c);
        uint32_t rep = c;
        for (int r : mins)
          for (uint32_t c2 = 0; c2 < 5; c2++)
            if (perms[r][c2] == s0[c] && c2 < rep) rep = c2;
        y |= rep << (15 + 3 * c);
      }
      tab[(M << 4) | tie] = make_uint2(best, y);
    }
  }
}

static gamma_fpm_pattern decode_pattern5(uint64_t key, uint64_t support, uint64_t instances) {
  gamma_fpm_pattern p{};
  p.nv = key5_nv(key);
  p.ne = key5_ne(key);
  const uint32_t ek = key5_edges(key);
  for (uint32_t i = 0; i < p.nv; i++) p.labels[i] = key5_label(key, i);
  for (uint32_t e = 0; e < p.ne; e++) {
    const uint32_t id = (ek >> (4 * (3 - e))) & 15u;
    p.edges[e][0] = (kA5 >> (3 * id)) & 7u;
    p.edges[e][1] = (kB5 >> (3 * id)) & 7u;
  }
  p.support = support;
  p.instances = instances;
  return p;
}

// Sort + unique of n tuples in the double buffer db (result at db.Current()); returns
// the unique count.
static uint64_t sort_unique(gamma_ctx *ctx, cub::DoubleBuffer<unsigned long long> &db, uint64_t n, int end_bit,
                            DevBuf<uint8_t> &tmp, unsigned long long *nsel) {
  if (n == 0) return 0;
  size_t t1 = 0, t2 = 0;
  GAMMA_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, t1, db, n, 0, end_bit, ctx->stream));
  GAMMA_CUDA(cub::DeviceSelect::Unique(nullptr, t2, db.Current(), db.Alternate(), nsel, n, ctx->stream));
  if (std::max(t1, t2) > tmp.n) tmp = DevBuf<uint8_t>(ctx, std::max(t1, t2));
  ctx->launch(KC_FPM_SUPPORT, [&] {
    GAMMA_CUDA(cub::DeviceRadixSort::SortKeys(tmp.p, t1, db, n, 0, end_bit, ctx->stream));
  });
  ctx->cub_sort_launched(KC_FPM_SUPPORT, n, end_bit);
  ctx->launch(KC_FPM_SUPPORT, [&] {
    GAMMA_CUDA(cub::DeviceSelect::Unique(tmp.p, t2, db.Current(), db.Alternate(), nsel, n, ctx->stream));
  });
  ctx->cub_select_launched(KC_FPM_SUPPORT);
  db.selector ^= 1;
  uint64_t r = 0;
  GAMMA_CUDA(cudaMemcpyAsync(&r, nsel, 8, cudaMemcpyDeviceToHost, ctx->stream));
  ctx->sync();
  return r;
}

struct Run4 {
  unsigned long long *dev = nullptr;   // in the device run area, or
  unsigned long long *host = nullptr;  // spilled to pinned host memory
  uint64_t len = 0;
};

// Level 4: passes of root-edge batches emit (slot, orbit, vertex) tuples; each pass's
// tuples are segment-sorted and deduplicated into a run (Opt 3's segment sort); runs
// live in an HBM run area and are spilled to pinned host memory when it fills; the runs
// are then multi-merged by key range, each range's slice of every run located by its
// matched index (Def. 5.1, Alg. 3), sorted, deduplicated and counted per
// (slot, orbit); support = min over orbits (MNI).
static void fpm_level4(gamma_graph *g, FpmArgs a, int grid4, uint64_t minsup, bool want_inst,
                       std::vector<gamma_fpm_pattern> &out) {
  gamma_ctx *ctx = g->ctx;
  std::vector<uint2> htab5;
  fpm_canon5_table(htab5);
  DevBuf<uint2> tab5 = to_device(ctx, htab5.data(), htab5.size());
  size_t fr = 0, tot = 0;
  GAMMA_CUDA(cudaMemGetInfo(&fr, &tot));
  const uint64_t budget = ctx->desc.hbm_budget_bytes ? ctx->desc.hbm_budget_bytes : (uint64_t)(fr * 0.8);
  const uint64_t ndir = 2 * g->m;
  const uint64_t nb_total = (ndir + 8 * (uint64_t)a.world - 1) / (8 * (uint64_t)a.world);
  uint64_t cap4 = 1ull << 14;
  while (cap4 < (1ull << 26) && cap4 * 48 * 8 < budget) cap4 <<= 1;   // table + counts <= 1/8 of the budget
  // test knobs: a small tuple buffer / run area forces many passes, spilled runs and a
  // multi-range merge (GAMMA_FPM4_TUPLES, GAMMA_FPM4_AREA, in tuples)
  const char *env_t = getenv("GAMMA_FPM4_TUPLES"), *env_a = getenv("GAMMA_FPM4_AREA");
  DevBuf<unsigned long long> flags(ctx, 4), nsel(ctx, 1);
  for (int attempt = 0;; attempt++) {
    GAMMA_REQUIRE(attempt < 4 && cap4 <= (1ull << 28), GAMMA_E_NOMEM, "gamma_fpm: level-4 pattern table overflow");
    const uint64_t fixed = cap4 * (8 + 32 + 8 + (want_inst ? 16 : 0));
    GAMMA_REQUIRE(fixed * 2 < budget, GAMMA_E_NOMEM, "gamma_fpm: level-4 pattern table exceeds the HBM budget");
    // tuple buffers (double buffer for the sort) and the run area share the rest
    const uint64_t rest = (budget - fixed) / 8;
    uint64_t T = std::max<uint64_t>(1 << 16, (uint64_t)(rest * 0.22));
    uint64_t Rcap = std::max<uint64_t>(1 << 16, rest - 2 * T - (rest / 16));   // keep slack for CUB temp
    if (env_t && *env_t) T = std::max<uint64_t>(256, strtoull(env_t, nullptr, 10));
    if (env_a && *env_a) Rcap = std::max<uint64_t>(256, strtoull(env_a, nullptr, 10));
    DevBuf<unsigned long long> key4(ctx, cap4), inst4(ctx, want_inst ? cap4 : 1), inst_pass(ctx, want_inst ? cap4 : 1);
    DevBuf<uint32_t> cnt(ctx, cap4 * 8);
    DevBuf<unsigned long long> sup4(ctx, cap4);
    DevBuf<unsigned long long> tA(ctx, T), tB(ctx, T), area(ctx, Rcap);
    DevBuf<uint8_t> tmp;
    GAMMA_CUDA(cudaMemsetAsync(key4.p, 0, cap4 * 8, ctx->stream));
    GAMMA_CUDA(cudaMemsetAsync(cnt.p, 0, cap4 * 32, ctx->stream));
    if (want_inst) GAMMA_CUDA(cudaMemsetAsync(inst4.p, 0, cap4 * 8, ctx->stream));
    Fpm4Args b{};
    b.tab5 = tab5.p;
    b.key4 = key4.p;
    b.inst4 = want_inst ? inst_pass.p : nullptr;
    b.cap4 = cap4;
    b.tup = tA.p;
    b.tup_cap = T;
    b.flags = flags.p;
    int slot_bits = 0;
    while ((1ull << slot_bits) < cap4) slot_bits++;
    const int end_bit = 35 + slot_bits;
    std::vector<Run4> runs;
    std::vector<void *> pinned;
    uint64_t area_top = 0, entries = 0;
    bool full = false;
    uint64_t b0 = 0, span = nb_total;
    const auto spill_area = [&] {   // device runs -> pinned host memory
      for (auto &r : runs) {
        if (!r.dev) continue;
        void *h = nullptr;
        GAMMA_CUDA(cudaMallocHost(&h, std::max<uint64_t>(r.len, 1) * 8));
        pinned.push_back(h);
        GAMMA_CUDA(cudaMemcpyAsync(h, r.dev, r.len * 8, cudaMemcpyDeviceToHost, ctx->stream));
        ctx->stats.spilled_bytes += r.len * 8;
        r.host = (unsigned long long *)h;
        r.dev = nullptr;
      }
      ctx->sync();
      area_top = 0;
    };
    while (b0 < nb_total) {
      const uint64_t b1 = std::min(nb_total, b0 + span);
      b.b_begin = b0;
      b.b_end = b1;
      GAMMA_CUDA(cudaMemsetAsync(flags.p, 0, 32, ctx->stream));
      GAMMA_CUDA(cudaMemsetAsync(ctx->ctrl + CTRL_WORK, 0, 8, ctx->stream));
      if (want_inst) GAMMA_CUDA(cudaMemsetAsync(inst_pass.p, 0, cap4 * 8, ctx->stream));
      ctx->launch(KC_FPM, [&] { fpm_enum4_kernel<<<grid4, kThreads, 0, ctx->stream>>>(a, b); });
      uint64_t hf[4];
      GAMMA_CUDA(cudaMemcpyAsync(hf, flags.p, 32, cudaMemcpyDeviceToHost, ctx->stream));
      ctx->sync();
      if (hf[2]) {
        full = true;
        break;
      }
      if (hf[1]) {   // the pass's tuples overflowed the buffer: halve the batch range
        GAMMA_REQUIRE(span > 1, GAMMA_E_NOMEM, "gamma_fpm: one root-edge batch overflows the level-4 tuple buffer");
        span = std::max<uint64_t>(1, span / 2);
        ctx->stats.retries++;
        continue;
      }
      entries += hf[3];
      if (want_inst)
        ctx->launch(KC_MISC, [&] { add_u64_kernel<<<g1d(cap4), 256, 0, ctx->stream>>>(inst4.p, inst_pass.p, cap4); });
      cub::DoubleBuffer<unsigned long long> db(tA.p, tB.p);
      const uint64_t r = sort_unique(ctx, db, hf[0], end_bit, tmp, nsel.p);
      if (r) {
        if (area_top + r > Rcap) spill_area();
        if (r > Rcap) {   // a run larger than the area goes straight to the host
          void *h = nullptr;
          GAMMA_CUDA(cudaMallocHost(&h, r * 8));
          pinned.push_back(h);
          GAMMA_CUDA(cudaMemcpyAsync(h, db.Current(), r * 8, cudaMemcpyDeviceToHost, ctx->stream));
          ctx->stats.spilled_bytes += r * 8;
          runs.push_back(Run4{nullptr, (unsigned long long *)h, r});
        } else {
          GAMMA_CUDA(cudaMemcpyAsync(area.p + area_top, db.Current(), r * 8, cudaMemcpyDeviceToDevice, ctx->stream));
          runs.push_back(Run4{area.p + area_top, nullptr, r});
          area_top += r;
        }
      }
      ctx->stats.chunks++;
      b0 = b1;
      if (hf[0] < T / 4 && span < nb_total) span *= 2;
    }
    if (full) {
      ctx->sync();
      for (void *h : pinned) cudaFreeHost(h);
      ctx->stats.retries++;
      cap4 *= 4;
      continue;
    }
    ctx->stats.level_entries[4] = entries;
    ctx->stats.alg_bytes[KC_FPM] += 40 * entries;   // <= 5 tuples of 8 B per level-4 embedding
    // ---- multi-merge of the runs by key range (matched indices) + count ----
    uint64_t total = 0;
    for (auto &r : runs) total += r.len;
    const uint64_t M = T;   // merge buffer: one tuple buffer (the other is the sort's alternate)
    std::vector<unsigned long long> splits;   // range boundaries (exclusive upper bounds)
    if (runs.size() == 1 && runs[0].dev) {
      ctx->launch(KC_FPM_SUPPORT, [&] {
        count_tuples_kernel<<<g1d((runs[0].len + 31) / 32), 256, 0, ctx->stream>>>(runs[0].dev, runs[0].len, cnt.p);
      });
    } else if (total) {
      // splitters from a sample of every run
      std::vector<unsigned long long> sample;
      for (auto &r : runs) {
        const uint64_t stride = std::max<uint64_t>(1, r.len / 256);
        const uint64_t ns = (r.len + stride - 1) / stride;
        std::vector<unsigned long long> s(ns);
        if (r.dev)
          GAMMA_CUDA(cudaMemcpy2DAsync(s.data(), 8, r.dev, stride * 8, 8, ns, cudaMemcpyDeviceToHost, ctx->stream));
        else
          for (uint64_t i = 0; i < ns; i++) s[i] = r.host[i * stride];
        ctx->sync();
        sample.insert(sample.end(), s.begin(), s.end());
      }
      std::sort(sample.begin(), sample.end());
      const uint64_t nranges = std::max<uint64_t>(1, (2 * total + M - 1) / M);
      for (uint64_t i = 1; i < nranges; i++) splits.push_back(sample[i * sample.size() / nranges]);
      splits.push_back(~0ull);
      std::sort(splits.begin(), splits.end());
      splits.erase(std::unique(splits.begin(), splits.end()), splits.end());
      DevBuf<unsigned long long> qk(ctx, 2);
      DevBuf<uint64_t> qi(ctx, 2);
      // matched index of `key` in run r (Def. 5.1: the first position holding a key >= it)
      const auto matched = [&](const Run4 &r, unsigned long long lo, unsigned long long hi, uint64_t &ilo,
                               uint64_t &ihi) {
        if (r.host) {
          ilo = std::lower_bound(r.host, r.host + r.len, lo) - r.host;
          ihi = hi == ~0ull ? r.len : (uint64_t)(std::lower_bound(r.host, r.host + r.len, hi) - r.host);
          return;
        }
        const unsigned long long k2[2] = {lo, hi};
        GAMMA_CUDA(cudaMemcpyAsync(qk.p, k2, 16, cudaMemcpyHostToDevice, ctx->stream));
        ctx->launch(KC_MISC, [&] { lower_bound_kernel<<<1, 32, 0, ctx->stream>>>(r.dev, r.len, qk.p, 2, qi.p); });
        uint64_t h2[2];
        GAMMA_CUDA(cudaMemcpyAsync(h2, qi.p, 16, cudaMemcpyDeviceToHost, ctx->stream));
        ctx->sync();
        ilo = h2[0];
        ihi = hi == ~0ull ? r.len : h2[1];
      };
      std::vector<std::pair<unsigned long long, unsigned long long>> ranges;
      unsigned long long lo = 0;
      for (unsigned long long hi : splits) {
        ranges.push_back({lo, hi});
        lo = hi;
      }
      for (size_t qi_ = 0; qi_ < ranges.size(); qi_++) {
        const unsigned long long rlo = ranges[qi_].first, rhi = ranges[qi_].second;
        std::vector<std::pair<uint64_t, uint64_t>> sl(runs.size());
        uint64_t need = 0;
        for (size_t i = 0; i < runs.size(); i++) {
          matched(runs[i], rlo, rhi, sl[i].first, sl[i].second);
          need += sl[i].second - sl[i].first;
        }
        if (need > M) {   // the sample misjudged this range: split it at its key midpoint
          GAMMA_REQUIRE(rhi - rlo > 1, GAMMA_E_NOMEM, "gamma_fpm: a level-4 merge range exceeds the buffer");
          const unsigned long long mid = rlo + (rhi - rlo) / 2;
          ranges.insert(ranges.begin() + qi_ + 1, {mid, rhi});
          ranges[qi_].second = mid;
          qi_--;
          continue;
        }
        uint64_t at = 0;
        for (size_t i = 0; i < runs.size(); i++) {
          const uint64_t len = sl[i].second - sl[i].first;
          if (!len) continue;
          if (runs[i].dev)
            GAMMA_CUDA(cudaMemcpyAsync(tA.p + at, runs[i].dev + sl[i].first, len * 8, cudaMemcpyDeviceToDevice,
                                       ctx->stream));
          else
            GAMMA_CUDA(cudaMemcpyAsync(tA.p + at, runs[i].host + sl[i].first, len * 8, cudaMemcpyHostToDevice,
                                       ctx->stream));
          at += len;
        }
        cub::DoubleBuffer<unsigned long long> db(tA.p, tB.p);
        const uint64_t u = sort_unique(ctx, db, at, end_bit, tmp, nsel.p);
        if (u)
          ctx->launch(KC_FPM_SUPPORT, [&] {
            count_tuples_kernel<<<g1d((u + 31) / 32), 256, 0, ctx->stream>>>(db.Current(), u, cnt.p);
          });
        ctx->stats.chunks++;
      }
    }
    ctx->launch(KC_FPM_SUPPORT, [&] { support4_kernel<<<g1d(cap4), 256, 0, ctx->stream>>>(key4.p, cap4, cnt.p, sup4.p); });
    std::vector<unsigned long long> hk(cap4), hs(cap4), hi(want_inst ? cap4 : 0);
    GAMMA_CUDA(cudaMemcpyAsync(hk.data(), key4.p, cap4 * 8, cudaMemcpyDeviceToHost, ctx->stream));
    GAMMA_CUDA(cudaMemcpyAsync(hs.data(), sup4.p, cap4 * 8, cudaMemcpyDeviceToHost, ctx->stream));
    if (want_inst) GAMMA_CUDA(cudaMemcpyAsync(hi.data(), inst4.p, cap4 * 8, cudaMemcpyDeviceToHost, ctx->stream));
    ctx->sync();
    for (void *h : pinned) cudaFreeHost(h);
    for (uint64_t s = 0; s < cap4; s++)
      if (hk[s] && hs[s] >= minsup) out.push_back(decode_pattern5(hk[s], hs[s], want_inst ? hi[s] : 0));
    return;
  }
}

// GAMMA_DEBUG: host wall time of the phases of one gamma_fpm call (stream-synchronised)
struct PhaseLog {
  gamma_ctx *ctx;
  bool on;
  std::chrono::steady_clock::time_point t;
  explicit PhaseLog(gamma_ctx *c) : ctx(c), on(getenv("GAMMA_DEBUG") != nullptr), t(std::chrono::steady_clock::now()) {}
  void mark(const char *what) {
    if (!on) return;
    ctx->sync();
    const auto now = std::chrono::steady_clock::now();
    fprintf(stderr, "[gamma_fpm] %-28s %9.2f ms\n", what, std::chrono::duration<double, std::milli>(now - t).count());
    t = now;
  }
};

static void fpm_run(gamma_graph *g, uint32_t max_edges, uint64_t minsup, std::vector<gamma_fpm_pattern> &out) {
  gamma_ctx *ctx = g->ctx;
  PhaseLog plog(ctx);
  const uint32_t n = g->n;
  // ---- label classes: sizes and in-class ranks ----
  uint32_t nlab = 1;
  if (g->labels) {
    GAMMA_CUDA(cudaMemsetAsync(ctx->ctrl + CTRL_AUX1, 0, 8, ctx->stream));
    ctx->launch(KC_FPM, [&] {
      max_label_kernel<<<g1d(n), 256, 0, ctx->stream>>>(g->labels, n, (unsigned long long *)(ctx->ctrl + CTRL_AUX1));
    });
    uint64_t ml = 0;
    GAMMA_CUDA(cudaMemcpyAsync(&ml, ctx->ctrl + CTRL_AUX1, 8, cudaMemcpyDeviceToHost, ctx->stream));
    ctx->sync();
    GAMMA_REQUIRE(ml < 4096, GAMMA_E_UNSUPPORTED, "gamma_fpm: labels must be < 4096");
    GAMMA_REQUIRE(max_edges < 4 || ml < 256, GAMMA_E_UNSUPPORTED, "gamma_fpm: 4-edge patterns need labels < 256");
    nlab = (uint32_t)ml + 1;
  }
  DevBuf<uint32_t> csize(ctx, nlab), lrank(ctx, n);
  GAMMA_CUDA(cudaMemsetAsync(csize.p, 0, nlab * 4, ctx->stream));
  ctx->launch(KC_FPM, [&] { label_hist_kernel<<<g1d(n), 256, 0, ctx->stream>>>(g->labels, n, csize.p, nullptr); });
  {
    DevBuf<uint64_t> k0(ctx, n), k1(ctx, n);
    ctx->launch(KC_FPM, [&] { label_keys_kernel<<<g1d(n), 256, 0, ctx->stream>>>(g->labels, n, k0.p); });
    size_t tmp = 0;
    int endbit = 32;
    while (endbit < 64 && (1ull << (endbit - 32)) <= nlab) endbit++;
    GAMMA_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, tmp, k0.p, k1.p, (uint64_t)n, 0, endbit, ctx->stream));
    DevBuf<uint8_t> t(ctx, tmp);
    ctx->launch(KC_FPM, [&] {
      GAMMA_CUDA(cub::DeviceRadixSort::SortKeys(t.p, tmp, k0.p, k1.p, (uint64_t)n, 0, endbit, ctx->stream));
    });
    ctx->cub_sort_launched(KC_FPM, n, endbit);
    ctx->launch(KC_FPM, [&] { label_rank_kernel<<<g1d(n), 256, 0, ctx->stream>>>(k1.p, n, lrank.p); });
  }
  // ---- pattern table + per-(slot, position) domain bitmaps ----
  size_t fr = 0, tot = 0;
  if (!ctx->desc.dev_alloc) {   // native pool: hand its idle blocks back before sizing from free HBM
    cudaMemPool_t pool;
    GAMMA_CUDA(cudaStreamSynchronize(ctx->stream));
    GAMMA_CUDA(cudaDeviceGetDefaultMemPool(&pool, ctx->device));
    GAMMA_CUDA(cudaMemPoolTrimTo(pool, 0));
  }
  GAMMA_CUDA(cudaMemGetInfo(&fr, &tot));
  const uint64_t budget = ctx->desc.hbm_budget_bytes ? ctx->desc.hbm_budget_bytes : (uint64_t)(fr * 0.85);
  std::vector<uint32_t> hsize(nlab);
  GAMMA_CUDA(cudaMemcpyAsync(hsize.data(), csize.p, nlab * 4, cudaMemcpyDeviceToHost, ctx->stream));
  ctx->sync();
  uint64_t maxw = 1;
  std::vector<uint32_t> hwords(nlab);
  for (uint32_t l = 0; l < nlab; l++) {
    hwords[l] = (hsize[l] + 31) / 32;
    maxw = std::max<uint64_t>(maxw, hwords[l]);
  }
  DevBuf<uint32_t> cwords = to_device(ctx, hwords.data(), nlab);
  std::vector<uint2> htab;
  std::vector<uint32_t> hprm;
  fpm_canon_tables(htab, hprm);
  DevBuf<uint2> canon_tab = to_device(ctx, htab.data(), htab.size());
  DevBuf<uint32_t> perm_tab = to_device(ctx, hprm.data(), hprm.size());
  // Distinct patterns are bounded by the label combinations of each shape (edge,
  // wedge, triangle, 3-star, 3-path); size the table at twice that bound (load <= 1/2,
  // short probe chains) and grow x4 if a chain still gets long.  The domain pool is
  // bounded by the budget and by 4 class bitmaps per slot.
  const double L = nlab;
  double bound = L * (L + 1) / 2;                                  // edges
  if (max_edges >= 2) bound += L * L * (L + 1) / 2;                // wedges
  if (max_edges >= 3) bound += (L + 2) * (L + 1) * L / 6 * (1 + L) + L * L * L * L;   // triangles, 3-stars, 3-paths
  uint64_t cap = 1024;
  while ((double)cap < 2 * bound && cap < (1ull << 24)) cap <<= 1;
  const uint64_t slot_bytes = 8 + 8 + 4 + 8;
  while (cap > 1024 && cap * slot_bytes * 4 > budget) cap >>= 1;
  DevBuf<uint32_t> freq;
  PoolBuf pool;
  DevBuf<unsigned long long> slots, sup, pcur, inst;
  const bool want_inst = (ctx->desc.flags & GAMMA_FLAG_FPM_INSTANCES) != 0;
  FpmArgs a{};
  a.rp = g->row_ptr;
  a.col = g->col;
  a.lab = g->labels;
  a.lrank = lrank.p;
  a.cwords = cwords.p;
  a.canon_tab = canon_tab.p;
  a.perm_tab = perm_tab.p;
  a.n = n;
  a.rank = 0;
  a.world = 1;   // levels < l run on every rank; the last one is split when dist
  a.carve_below = 0xffffffffu;
  a.walk_lo = 0;
  // multi-GPU: the last level is partitioned over the ranks and its domains OR-reduced
  // (fpm_dist_level); without the collectives every rank computes everything
  const bool dist = ctx->desc.world > 1 && ctx->desc.allreduce_sum_u64 && ctx->desc.alltoall_u32;
  std::vector<gamma_fpm_pattern> found_last;
  a.ctrl = (unsigned long long *)ctx->ctrl;
  const int grid_enum = ctx->num_sms * occupancy_blocks((const void *)fpm_enum_kernel, kThreads, 0);
  for (int attempt = 0;; attempt++) {
    GAMMA_REQUIRE(cap * slot_bytes < budget, GAMMA_E_NOMEM, "gamma_fpm: pattern table exceeds the HBM budget");
    const uint64_t pool_words =
        std::max<uint64_t>(64, std::min<uint64_t>((budget - cap * slot_bytes) / 4, cap * 4 * maxw));
    freq.reset(); pool.reset(); slots.reset(); sup.reset(); pcur.reset(); inst.reset();
    slots = DevBuf<unsigned long long>(ctx, 2 * cap);
    sup = DevBuf<unsigned long long>(ctx, cap);
    freq = DevBuf<uint32_t>(ctx, cap);
    plog.mark("setup");
    pool.alloc(pool_words);
    plog.mark("pool cudaMalloc");
    pcur = DevBuf<unsigned long long>(ctx, 1);
    GAMMA_CUDA(cudaMemsetAsync(slots.p, 0, cap * 16, ctx->stream));
    GAMMA_CUDA(cudaMemsetAsync(freq.p, 0, cap * 4, ctx->stream));
    GAMMA_CUDA(cudaMemsetAsync(pool.p, 0, pool_words * 4, ctx->stream));
    GAMMA_CUDA(cudaMemsetAsync(pcur.p, 0, 8, ctx->stream));
    if (want_inst) {
      inst = DevBuf<unsigned long long>(ctx, cap);
      GAMMA_CUDA(cudaMemsetAsync(inst.p, 0, cap * 8, ctx->stream));
    }
    a.T = Table{slots.p, sup.p, freq.p, cap, pool.p, pool_words, pcur.p, want_inst ? inst.p : nullptr};
    plog.mark("table + pool memset");
    bool full = false;
    found_last.clear();
    const uint32_t lmax3 = std::min<uint32_t>(max_edges, 3);   // level 4: fpm_level4 (Opt 3)
    for (uint32_t l = 1; l <= lmax3 && !full; l++) {
      if (dist && l == max_edges) {
        full = !fpm_dist_level(ctx, a, grid_enum, l, minsup, hsize, cap, slots.p, pool.p, pool_words, pcur.p,
                               found_last);
        break;
      }
      a.level = l;
      // first pass of the level: carve domains only for patterns whose smallest label
      // is below T, the largest threshold whose worst-case domains fit the pool (all
      // labels when everything fits); the rest go to label-pruned chunk passes
      a.carve_below = 0xffffffffu;
      if (l >= 2 && nlab <= 64) {
        const std::vector<double> W = fpm_words_by_min_label(l, hwords);
        double acc = 0, total = 0;
        for (double w : W) total += w;
        if (total > (double)pool_words) {
          uint32_t T = 0;
          while (T < nlab && acc + W[T] <= (double)pool_words) acc += W[T++];
          a.carve_below = std::max<uint32_t>(T, 1);
        }
      }
      ctrl_reset(ctx);
      ctx->launch(KC_FPM, [&] { fpm_enum_kernel<<<grid_enum, kThreads, 0, ctx->stream>>>(a); });
      ctx->launch(KC_FPM_SUPPORT, [&] {
        fpm_support_kernel<<<g1d(cap * 32), 256, 0, ctx->stream>>>(a, l, minsup);
      });
      a.carve_below = 0xffffffffu;
      uint64_t carved = 0;
      GAMMA_CUDA(cudaMemcpyAsync(&carved, pcur.p, 8, cudaMemcpyDeviceToHost, ctx->stream));
      ctrl_fetch(ctx);
      count_fpm_bytes(ctx);
      full = ctx->ctrl_host[CTRL_ERR] != 0;
      if (dist) {   // the ranks must agree on growing the table
        uint64_t f = full;
        coll_allreduce(ctx, &f, 1);
        full = f != 0;
      }
      if (full) break;
      plog.mark(l == 1 ? "level 1" : l == 2 ? "level 2" : "level 3");
      ctx->stats.level_entries[l] = ctx->ctrl_host[CTRL_ENTRIES];
      // a level's domains are dead once its supports are known (the next level reads
      // only freq): clear what it used and carve the next level from offset 0
      uint64_t dirty = std::min<uint64_t>(carved, pool_words);
      if (getenv("GAMMA_DEBUG"))
        fprintf(stderr, "[gamma_fpm] level %u: budget %.2f GB, table cap %llu, pool %.2f GB, carved %.2f GB, ovf %llu\n",
                l, budget / 1e9, (unsigned long long)cap, pool_words * 4 / 1e9, carved * 4 / 1e9,
                (unsigned long long)ctx->ctrl_host[CTRL_OVF]);
      const auto clear_pool = [&] {
        if (dirty) GAMMA_CUDA(cudaMemsetAsync(pool.p, 0, dirty * 4, ctx->stream));
        GAMMA_CUDA(cudaMemsetAsync(pcur.p, 0, 8, ctx->stream));
        dirty = 0;
      };
      if (ctx->ctrl_host[CTRL_OVF] == 0) {
        clear_pool();
        continue;
      }
      // The domains of this level did not all fit the pool.  Every pattern of the
      // level is in the table by now (a slot is claimed before its domains are
      // carved), and the slots that got domains have their support: split the rest
      // into chunks that fit the pool and redo the level's enumeration once per
      // chunk, recording only into that chunk's slots (dom = ~0 elsewhere).
      std::vector<unsigned long long> hkey, hdom;
      slots_get(ctx, hkey, slots.p, cap, 0);
      slots_get(ctx, hdom, slots.p, cap, 1);
      ctx->sync();
      std::vector<uint64_t> pending;
      for (uint64_t s = 0; s < cap; s++)
        if (hkey[s] && key_ne(hkey[s]) == l && hdom[s] == ~0ull) pending.push_back(s);
      // by smallest label: a chunk's pass skips every embedding with a smaller label
      std::stable_sort(pending.begin(), pending.end(),
                       [&](uint64_t x, uint64_t y) { return key_label(hkey[x], 0) < key_label(hkey[y], 0); });
      size_t next = 0;
      while (next < pending.size()) {
        std::fill(hdom.begin(), hdom.end(), ~0ull);
        a.walk_lo = key_label(hkey[pending[next]], 0);
        uint64_t used = 0;
        for (; next < pending.size(); next++) {
          const uint64_t k = hkey[pending[next]];
          uint64_t words = 0;
          for (uint32_t p = 0; p < key_nv(k); p++) words += (hsize[key_label(k, p)] + 31) / 32;
          GAMMA_REQUIRE(words <= pool_words, GAMMA_E_NOMEM, "gamma_fpm: one pattern's domains exceed the HBM budget");
          if (used + words > pool_words) break;
          hdom[pending[next]] = 1 + used;
          used += words;
        }
        slots_put(ctx, slots.p, hdom, cap, 1);
        clear_pool();
        dirty = used;
        GAMMA_CUDA(cudaMemcpyAsync(pcur.p, &pool_words, 8, cudaMemcpyHostToDevice, ctx->stream));
        ctrl_reset(ctx);
        ctx->launch(KC_FPM, [&] { fpm_enum_kernel<<<grid_enum, kThreads, 0, ctx->stream>>>(a); });
        ctx->launch(KC_FPM_SUPPORT, [&] {
          fpm_support_kernel<<<g1d(cap * 32), 256, 0, ctx->stream>>>(a, l, minsup);
        });
        ctrl_fetch(ctx);
        count_fpm_bytes(ctx);
        GAMMA_REQUIRE(ctx->ctrl_host[CTRL_ERR] == 0 && ctx->ctrl_host[CTRL_OVF] == 0, GAMMA_E_CUDA,
                      "gamma_fpm: a chunk pass met an unclaimed pattern");
        ctx->stats.chunks++;
      }
      a.walk_lo = 0;
      clear_pool();
    }
    if (!full) break;
    GAMMA_REQUIRE(attempt < 6, GAMMA_E_NOMEM, "gamma_fpm: pattern table keeps overflowing");
    ctx->stats.retries++;   // sizes are only known after the fact: grow and redo
    cap *= 4;
  }
  plog.mark("levels done");
  pool.reset();   // the level <= 3 MNI domains are dead (freq flags stay in the table)
  plog.mark("pool cudaFree");
  // ---- level 4: out-of-core aggregation of (slot, orbit, vertex) tuples ----
  std::vector<gamma_fpm_pattern> found4;
  if (max_edges >= 4) {
    pool.reset();   // the level <= 3 MNI domains are dead (freq flags stay in the table)
    FpmArgs a4 = a;
    a4.level = 4;
    a4.claim_only = 0;
    a4.carve_below = 0xffffffffu;
    a4.walk_lo = 0;
    a4.rank = 0;
    a4.world = 1;   // replicated on every rank (the exchange of level-4 tuples is not implemented)
    a4.T.pool = nullptr;
    const int grid4 = ctx->num_sms * occupancy_blocks((const void *)fpm_enum4_kernel, kThreads, 0);
    ctrl_reset(ctx);
    fpm_level4(g, a4, grid4, minsup, want_inst, found4);
    ctrl_fetch(ctx);
    count_fpm_bytes(ctx);
  }
  plog.mark("level 4 / pool free");
  // ---- collect the frequent patterns: compacted on the device (only frequent slots
  // travel), ordered on the host by one packed key per pattern ----
  uint64_t nf = 0;
  DevBuf<unsigned long long> ck(ctx, cap), cs(ctx, cap), ci(ctx, want_inst ? cap : 1), ccur(ctx, 1);
  GAMMA_CUDA(cudaMemsetAsync(ccur.p, 0, 8, ctx->stream));
  ctx->launch(KC_MISC, [&] {
    collect_kernel<<<g1d(cap), 256, 0, ctx->stream>>>(slots.p, sup.p, freq.p, want_inst ? inst.p : nullptr, cap,
                                                       dist ? max_edges : 0u, ck.p, cs.p, ci.p, ccur.p);
  });
  GAMMA_CUDA(cudaMemcpyAsync(&nf, ccur.p, 8, cudaMemcpyDeviceToHost, ctx->stream));
  ctx->sync();
  std::vector<unsigned long long> hkey(nf), hsup(nf), hinst(want_inst ? nf : 0);
  if (nf) {
    GAMMA_CUDA(cudaMemcpyAsync(hkey.data(), ck.p, nf * 8, cudaMemcpyDeviceToHost, ctx->stream));
    GAMMA_CUDA(cudaMemcpyAsync(hsup.data(), cs.p, nf * 8, cudaMemcpyDeviceToHost, ctx->stream));
    if (want_inst) GAMMA_CUDA(cudaMemcpyAsync(hinst.data(), ci.p, nf * 8, cudaMemcpyDeviceToHost, ctx->stream));
    ctx->sync();
  }
  {   // decode (parallel over host threads: 1.2e6 patterns on C4)
    const size_t base = out.size();
    out.resize(base + nf);
    par_for(nf, [&](size_t i0, size_t i1) {
      for (size_t i = i0; i < i1; i++) out[base + i] = decode_pattern(hkey[i], hsup[i], want_inst ? hinst[i] : 0);
    });
  }
  out.insert(out.end(), found_last.begin(), found_last.end());
  out.insert(out.end(), found4.begin(), found4.end());
  // sort key: (ne, nv, labels in canonical order, edge pairs) packed in 128 bits (unique
  // per pattern, so any sort gives the same order)
  std::vector<std::pair<std::pair<uint64_t, uint64_t>, uint32_t>> order(out.size());
  par_for(out.size(), [&](size_t i0, size_t i1) {
    for (size_t i = i0; i < i1; i++) {
      const gamma_fpm_pattern &x = out[i];
      uint64_t lab60 = 0;   // five 12-bit labels (labels < 4096), canonical order
      for (uint32_t j = 0; j < 5; j++) lab60 = lab60 << 12 | (j < x.nv ? x.labels[j] & 0xfffu : 0u);
      uint64_t ek = 0;      // four edges, 3 + 3 bits each
      for (uint32_t e = 0; e < 4; e++)
        ek = ek << 6 | (e < x.ne ? (uint64_t)(x.edges[e][0] << 3 | x.edges[e][1]) : 0u);
      const uint64_t hi = (uint64_t)x.ne << 61 | (uint64_t)x.nv << 58 | (lab60 >> 2);
      const uint64_t lo = (lab60 & 3u) << 62 | ek;
      order[i] = {{hi, lo}, (uint32_t)i};
    }
  });
  par_sort(order);
  std::vector<gamma_fpm_pattern> sorted(out.size());
  par_for(out.size(), [&](size_t i0, size_t i1) {
    for (size_t i = i0; i < i1; i++) sorted[i] = out[order[i].second];
  });
  out.swap(sorted);
  plog.mark("collect + sort");
  ctx->collect_timings();
}

}  // namespace gamma_impl

using namespace gamma_impl;

extern "C" gamma_status gamma_fpm(gamma_graph *g, uint32_t max_edges, uint64_t minsup, gamma_fpm_result **out) {
  return guarded([&] {
    GAMMA_REQUIRE(g && out, GAMMA_E_INVAL, "gamma_fpm: NULL argument");
    GAMMA_REQUIRE(minsup >= 1, GAMMA_E_INVAL, "gamma_fpm: minsup must be >= 1");
    GAMMA_REQUIRE(max_edges >= 1, GAMMA_E_INVAL, "gamma_fpm: max_edges must be >= 1");
    GAMMA_REQUIRE(max_edges <= 4, GAMMA_E_UNSUPPORTED, "gamma_fpm: max_edges > 4 not supported");
    // the enumeration carries symmetric-CSR offsets (< 2m) as u32
    GAMMA_REQUIRE(2 * g->m < (1ull << 32), GAMMA_E_UNSUPPORTED, "gamma_fpm: graphs with 2m >= 2^32 unsupported");
    gamma_ctx *c = g->ctx;
    GAMMA_CUDA(cudaSetDevice(c->device));
    c->reset_stats();
    c->keep_release();   // FPM sizes its pattern table and domain pool from free HBM
    const auto t0 = std::chrono::steady_clock::now();
    std::vector<gamma_fpm_pattern> pats;
    fpm_run(g, max_edges, minsup, pats);
    c->stats.wall_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    auto *r = new gamma_fpm_result();
    r->n = pats.size();
    r->pats = new gamma_fpm_pattern[pats.size() ? pats.size() : 1];
    std::copy(pats.begin(), pats.end(), r->pats);
    *out = r;
  });
}

extern "C" void gamma_fpm_result_free(gamma_fpm_result *r) {
  if (!r) return;
  delete[] r->pats;
  delete r;
}
