// match.cu -- subgraph matching, Alg. 1 (WOJ, query-vertex-at-a-time vertex
// extension + filtering), labeled, counting distinct
// subgraphs (readings R4-R6, R10); non-induced by default, induced on
// request (the same extension with anti-edge checks, R17).
//
// Host planner:
//  * matching order delta_v (PAPER.md L176 leaves it open; reading R10): the
//    max-degree query vertex first, then repeatedly the vertex with the most
//    already-placed neighbours (ties: higher degree, then lower id);
//  * Aut_L(P) by brute force over nv! permutations;
//  * symmetry breaking by a stabilizer chain along the matching order: for each
//    placed vertex v, phi(v) < phi(u) for every u != v in v's orbit under the
//    stabilizer of the earlier vertices.  Each automorphism class of mappings then
//    has exactly one representative, so constrained count = mappings / |Aut_L|.
//
// Device (per extension depth d -> d+1, one warp per group):
//  * a group = a d-vertex prefix phi_0..phi_{d-1} + a run of valid candidates for
//    position d (the children); the descriptor carries the prefix, so no parent
//    pointers are chased (the prefix tree of PAPER.md L253 is stored per group);
//  * Opt 2: L_m = the intersection of the backward-neighbour lists that do not
//    involve the child (the prefix part) is computed once per group, filtered by
//    label/order/injectivity, and staged in shared memory; every child then probes
//    only its own list against it;
//  * filters ("pruning and label checking at run-time"): label,
//    degree >= pattern degree, injectivity, symmetry order;
//  * children with long runs are sliced into several groups (hub load balance);
//  * last position: counted, not stored.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_select.cuh>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <vector>

#include "device_common.cuh"
#include "internal.cuh"

namespace gamma_impl {

namespace {

constexpr int kMaxV = 8;
constexpr int kWarps = 8;
constexpr int kThreads = kWarps * 32;
constexpr uint32_t kLmCap = 512;     // default staged L_m per warp (u32); longer L_m -> global scratch
constexpr uint32_t kOutCap = 512;    // default staged child run per warp (u32); longer runs go direct
// (both are launch parameters, SmArgs::lm_cap / out_cap: the shared-memory footprint
// sets the CTAs per SM; GAMMA_SM_LMCAP / GAMMA_SM_OUTCAP override them for tuning;
// C3 sweep on B200: 512/512 233 ms, 256/256 243, 1024/512 272, 2048/512 338 per step)
constexpr uint32_t kLongRatio = 1;   // see SmArgs::long_ratio (GAMMA_SM_LONGRATIO overrides; 0 = off)
#ifndef GAMMA_SM_CAP_LOG2   // first entry-table size of an SM level (log2 slots)
#define GAMMA_SM_CAP_LOG2 27
#endif
constexpr uint32_t kBlkV = 4096;
constexpr uint32_t kBlkG = 256;      // descriptors per warp block
constexpr uint32_t kSlice = 64;      // children per group descriptor when the count level consumes them
constexpr uint32_t kSliceExt = 16;   // ... when an extension level does (SmArgs::slice; GAMMA_SM_SLICE /
                                     // GAMMA_SM_SLICE_EXT; C3 sweep in profiles/sm_r01: finer groups
                                     // balance the extension levels, the count level prefers fewer
                                     // L_m rebuilds)
constexpr uint32_t kRootChunk = 16;  // roots per depth-0 group

struct SmPlan {
  uint32_t nv, labeled;
  uint32_t order[kMaxV];
  uint32_t label[kMaxV];    // per position
  uint32_t mindeg[kMaxV];   // per position
  uint32_t bmask[kMaxV];    // backward-neighbour positions
  uint32_t injmask[kMaxV];  // earlier non-neighbour positions (x != phi_j)
  uint32_t ltmask[kMaxV];   // earlier positions j with phi_j < x
  uint32_t gtmask[kMaxV];   // earlier positions j with x < phi_j
  uint32_t antimask[kMaxV]; // induced: earlier non-neighbour positions j with x not in N(phi_j)
  uint64_t aut;
};

struct SmArgs {
  const uint64_t *rp;
  const uint32_t *col;
  const uint32_t *lab;      // nullable (unlabeled graph: all 0)
  const uint32_t *ldeg;     // nullable: label << 24 | min(degree, 2^24 - 1) per vertex (labels < 256):
                            // one 4-byte gather for the label and degree filters
  SmPlan P;
  uint32_t d;               // children are at position d; extend to q = d+1
  const uint32_t *vid_in;
  const uint32_t *desc_in;  // dw_in words per group: beg, len, phi_0..phi_{d-1}
  uint32_t dw_in;
  uint64_t g_begin, g_end;
  uint32_t *vid_out;
  uint32_t *desc_out;
  uint32_t dw_out;
  uint64_t cap_v, cap_g;
  unsigned long long *ctrl;  // this launch's control block (CTRL_* offsets)
  unsigned long long *ovf;   // overflow word (shared by a launch chain: any level's overflow
                             // stops every later level)
  const unsigned long long *gcur_in;   // nullable: groups in = min(*gcur_in, cap_g_in) - g_begin,
  uint64_t cap_g_in;                   // read on the device (chained launch), instead of g_end
  uint32_t batch;
  uint32_t stage;           // 0: never stage L_m (debug)
  uint32_t *lm_scratch;     // per-warp global L_m slices for hub prefixes (nullable)
  uint32_t lm_scratch_cap;  // entries per warp slice
  uint32_t *big_scratch;    // per-warp global slices for child runs above out_cap (nullable)
  uint32_t big_scratch_cap; // entries per warp slice
  uint32_t lm_cap, out_cap; // shared-memory staging per warp (u32 entries)
  uint32_t slice;           // children per group descriptor of the next level
  uint32_t long_ratio;      // last level: child lists > long_ratio * |L_m| are probed from L_m (0: off)
  uint32_t short_lm;        // last level: |L_m| <= short_lm uses the (child, L_m element) pair probes
};

__device__ __forceinline__ uint32_t gdeg(const SmArgs &a, uint32_t v) {
  return (uint32_t)(a.rp[v + 1] - a.rp[v]);
}

struct Bounds {
  int64_t lo;     // x > lo
  uint32_t hi;    // x < hi (0xffffffff: none)
  uint32_t inj;   // positions to check x != phi_j
  uint32_t anti;  // induced: positions to check x not in N(phi_j)
};

// Candidate filter for position q.  `staged`: x comes from (or was found in) a staged
// L_m, whose entries already passed position q's label and degree filters, so only the
// bounds, injectivity and anti-edge checks remain (no label / row-pointer gathers).
__device__ __forceinline__ bool sm_filter(const SmArgs &a, uint32_t q, uint32_t x, const Bounds &b,
                                          const uint32_t *phi, bool last, bool staged = false) {
  if ((int64_t)x <= b.lo || x >= b.hi) return false;
  const bool need_deg = !last && !staged && a.P.mindeg[q] > 1;
  uint32_t ld = 0;
  if (a.ldeg && !staged && (a.P.labeled || need_deg)) {
    ld = __ldg(a.ldeg + x);
    if (a.P.labeled && (ld >> 24) != a.P.label[q]) return false;
  } else if (a.P.labeled && !staged) {
    const uint32_t lx = a.lab ? a.lab[x] : 0u;
    if (lx != a.P.label[q]) return false;
  }
  uint32_t m = b.inj;
  while (m) {
    const int j = __ffs(m) - 1;
    m &= m - 1;
    if (phi[j] == x) return false;
  }
  if (need_deg && (a.ldeg ? (ld & 0xffffffu) : gdeg(a, x)) < a.P.mindeg[q]) return false;
  m = b.anti;   // induced: anti-edge checks, one binary search per non-neighbour
  while (m) {
    const int j = __ffs(m) - 1;
    m &= m - 1;
    const uint64_t s = a.rp[phi[j]];
    const uint32_t l = (uint32_t)(a.rp[phi[j] + 1] - s);
    if (l && sorted_contains(a.col + s, l, x)) return false;
  }
  return true;
}

// `anti_avail`: the placed positions whose anti-edge checks are still to be made
// (a staged L_m has the prefix ones applied already).
__device__ __forceinline__ Bounds bounds_for(const SmArgs &a, uint32_t q, uint32_t avail, const uint32_t *phi,
                                             uint32_t anti_avail) {
  Bounds b{-1, 0xffffffffu, a.P.injmask[q] & avail, a.P.antimask[q] & anti_avail};
  uint32_t m = a.P.ltmask[q] & avail;
  while (m) {
    const int j = __ffs(m) - 1;
    m &= m - 1;
    b.lo = max(b.lo, (int64_t)phi[j]);
  }
  m = a.P.gtmask[q] & avail;
  while (m) {
    const int j = __ffs(m) - 1;
    m &= m - 1;
    b.hi = min(b.hi, phi[j]);
  }
  return b;
}

// bounds_for over a plan (the join kernels have no SmArgs)
__device__ __forceinline__ Bounds bounds_for_join(const SmPlan &P, uint32_t q, uint32_t avail, const uint32_t *phi) {
  Bounds b{-1, 0xffffffffu, 0u, 0u};
  uint32_t m = P.ltmask[q] & avail;
  while (m) {
    const int j = __ffs(m) - 1;
    m &= m - 1;
    b.lo = max(b.lo, (int64_t)phi[j]);
  }
  m = P.gtmask[q] & avail;
  while (m) {
    const int j = __ffs(m) - 1;
    m &= m - 1;
    b.hi = min(b.hi, phi[j]);
  }
  return b;
}

// Intersect the lists N(phi_j), j in `lists`, with filters; results (sorted) go to
// out[] (if WRITE and they fit in cap) or are only counted.  The shortest list
// drives; the others are probed by binary search.  Returns the number of results,
// or UINT32_MAX if WRITE and the results overflow cap.
template <bool WRITE>
__device__ uint32_t sm_intersect(const SmArgs &a, uint32_t q, uint32_t lists, const uint32_t *phi,
                                 const Bounds &bd, bool last, const uint32_t *lm, uint32_t lm_len,
                                 uint32_t *out, uint32_t cap, int lane) {
  // choose the driver: L_m (shared memory) counts as a list when given
  uint32_t best_len = 0xffffffffu, best = 0xffffffffu;
  uint32_t m = lists;
  while (m) {
    const int j = __ffs(m) - 1;
    m &= m - 1;
    const uint32_t dl = gdeg(a, phi[j]);
    if (dl < best_len) { best_len = dl; best = j; }
  }
  const bool drive_lm = lm != nullptr && lm_len <= best_len;
  const uint32_t *drv;
  uint32_t dlen;
  if (drive_lm) {
    drv = lm;
    dlen = lm_len;
  } else {
    drv = a.col + a.rp[phi[best]];
    dlen = best_len;
  }
  const uint32_t probes = drive_lm ? lists : (lists & ~(1u << best));
  // skip driver entries <= lo (sorted)
  uint32_t start = 0;
  if (bd.lo >= 0 && dlen) start = upper_bound_idx(drv, dlen, (uint32_t)bd.lo);
  uint32_t found = 0;
  for (uint32_t j0 = start; j0 < dlen; j0 += 32) {
    const uint32_t jj = j0 + lane;
    const uint32_t x = jj < dlen ? drv[jj] : 0xffffffffu;
    // membership in the staged L_m (shared memory) before the gathers of the full filter
    bool ok = jj < dlen && (int64_t)x > bd.lo && x < bd.hi;
    if (ok && lm && !drive_lm) ok = sorted_contains(lm, lm_len, x);
    ok = ok && sm_filter(a, q, x, bd, phi, last, lm != nullptr);
    uint32_t pm = probes;
    while (ok && pm) {
      const int j = __ffs(pm) - 1;
      pm &= pm - 1;
      const uint64_t s = a.rp[phi[j]];
      const uint32_t l = (uint32_t)(a.rp[phi[j] + 1] - s);
      ok = l > 0 && sorted_contains(a.col + s, l, x);
    }
    const uint32_t bal = __ballot_sync(0xffffffffu, ok);
    if (WRITE && ok) {
      const uint32_t p = found + __popc(bal & lanemask_lt());
      if (p < cap) out[p] = x;
    }
    found += __popc(bal);
    if (__shfl_sync(0xffffffffu, x, 31) >= bd.hi) break;   // driver is sorted
  }
  if (WRITE && found > cap) return 0xffffffffu;
  return found;
}

__global__ void __launch_bounds__(kThreads, 5) sm_kernel(SmArgs a) {
  extern __shared__ uint32_t smem[];
  const int lane = threadIdx.x & 31;
  const int wid = threadIdx.x >> 5;
  uint32_t *slm = smem + wid * (a.lm_cap + a.out_cap);
  uint32_t *sout = slm + a.lm_cap;
  const uint32_t d = a.d, q = d + 1;
  const bool last = q == a.P.nv - 1;
  const BlockPool pv{&a.ctrl[CTRL_VCUR], a.ovf, a.cap_v, kBlkV};
  const BlockPool pg{&a.ctrl[CTRL_GCUR], a.ovf, a.cap_g, kBlkG};
  WarpBlock wv, wg;
  uint64_t acc = 0, in_entries = 0, out_entries = 0;
  uint64_t elems = 0;   // adjacency elements the method fetches (SURVEY §8(d) B_l), lane-partial
  uint64_t g_end = a.g_end;
  if (a.gcur_in) {   // chained launch: the previous level's group cursor, read here
    if (*(volatile unsigned long long *)a.ovf) return;   // an earlier level overflowed
    const uint64_t gc = *(volatile const unsigned long long *)a.gcur_in;
    g_end = gc < a.cap_g_in ? gc : a.cap_g_in;
  }
  const uint64_t ng = g_end > a.g_begin ? g_end - a.g_begin : 0;
  bool stop = false;
  const uint32_t prefix_mask = (1u << d) - 1u;
  const uint32_t bq = a.P.bmask[q];
  const uint32_t bshared = bq & prefix_mask;
  const bool child_in_b = (bq >> d) & 1u;
  const bool anti_d = (a.P.antimask[q] >> d) & 1u;   // induced: x must not be adjacent to the child

  while (!stop) {
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(&a.ctrl[CTRL_WORK], (unsigned long long)a.batch);
    base = __shfl_sync(0xffffffffu, base, 0);
    if (base >= ng) break;
    if (!last && *(volatile unsigned long long *)a.ovf) break;
    const uint64_t bend = min((uint64_t)base + a.batch, ng);
    for (uint64_t gi = a.g_begin + base; gi < a.g_begin + bend && !stop; gi++) {
      const uint32_t *dsc = a.desc_in + gi * a.dw_in;
      const uint32_t w = lane < (int)a.dw_in ? dsc[lane] : 0u;
      const uint32_t beg = __shfl_sync(0xffffffffu, w, 0);
      const uint32_t len = __shfl_sync(0xffffffffu, w, 1);
      if (len == 0) continue;
      uint32_t phi[kMaxV];
#pragma unroll
      for (int j = 0; j < kMaxV; j++) phi[j] = __shfl_sync(0xffffffffu, w, (2 + j) & 31);
      in_entries += (lane == 0) ? len : 0;
      // ---- Opt 2: L_m over the prefix-only backward lists, staged per group ----
      const Bounds bs = bounds_for(a, q, prefix_mask, phi, prefix_mask);
      bool staged = false;
      uint32_t lm_len = 0;
      // L_m lives in shared memory when its bound (the shortest prefix list) fits,
      // else in this warp's slice of a global scratch buffer (hub prefixes)
      uint32_t *lm = slm;
      uint32_t lm_cap = a.lm_cap;
      if (bshared && a.stage) {
        uint32_t bound = 0xffffffffu, mm = bshared;
        while (mm) {
          const int j = __ffs(mm) - 1;
          mm &= mm - 1;
          bound = min(bound, gdeg(a, phi[j]));
        }
        if (bound > a.lm_cap && a.lm_scratch) {
          lm = a.lm_scratch + (uint64_t)(blockIdx.x * kWarps + wid) * a.lm_scratch_cap;
          lm_cap = a.lm_scratch_cap;
        }
        const uint32_t r = sm_intersect<true>(a, q, bshared, phi, bs, last, nullptr, 0, lm, lm_cap, lane);
        __syncwarp();
        if (r != 0xffffffffu) {
          staged = true;
          lm_len = r;
        }
      }
      if (staged && lane == 0) {   // Opt 2: the prefix lists are fetched once per group
        uint32_t m = bshared | (a.P.antimask[q] & prefix_mask);
        while (m) {
          const int j = __ffs(m) - 1;
          m &= m - 1;
          elems += gdeg(a, phi[j]);
        }
      }
      if (staged && lm_len == 0) continue;   // no child can extend
      const uint32_t *run = a.vid_in + beg;
      if (last && staged && !anti_d) {
        // Last level over a staged L_m: count without a per-child warp loop.  The
        // filters that involve the child c = phi_d are an order window (lo_c, hi_c)
        // and possibly x != c; the prefix filters are already applied to L_m.
        const bool lt_d = (a.P.ltmask[q] >> d) & 1u, gt_d = (a.P.gtmask[q] >> d) & 1u;
        const bool inj_d = (a.P.injmask[q] >> d) & 1u;
        uint64_t part = 0;
        if (!child_in_b) {
          // cand(c) = L_m ∩ window minus c: two binary searches per child, lane per child
          for (uint32_t i = lane; i < len; i += 32) {
            const uint32_t c = run[i];
            const int64_t lo = lt_d ? max(bs.lo, (int64_t)c) : bs.lo;
            const uint32_t hi = gt_d ? min(bs.hi, c) : bs.hi;
            const uint32_t a0 = lo < 0 ? 0u : upper_bound_idx(lm, lm_len, (uint32_t)lo);
            const uint32_t a1 = hi == 0 ? 0u : upper_bound_idx(lm, lm_len, hi - 1);
            uint32_t cnt = a1 > a0 ? a1 - a0 : 0u;
            if (inj_d && (int64_t)c > lo && c < hi && cnt && sorted_contains(lm, lm_len, c)) cnt--;
            part += cnt;
          }
        } else if (lm_len > a.short_lm) {
          // cand(c) = L_m ∩ N(c) ∩ window with a long L_m: stream the children's lists
          // N(c) in flattened windows of 32 children (one element per lane per step,
          // child found by an OR-reduction of the window's start offsets) and probe L_m
          // in shared memory
          const uint32_t lmin = lm[0], lmax = lm[lm_len - 1];
          const uint32_t upto = lane == 31 ? 0xffffffffu : ((2u << lane) - 1u);
          const uint64_t long_at = a.long_ratio ? (uint64_t)a.long_ratio * lm_len : ~0ull;
          for (uint32_t w0 = 0; w0 < len; w0 += 32) {
            const uint32_t i = w0 + lane;
            uint32_t c = 0, beg = 0, dl = 0;
            if (i < len) {
              c = run[i];
              const uint64_t s0 = a.rp[c];
              dl = (uint32_t)(a.rp[c + 1] - s0);
              beg = (uint32_t)s0;
            }
            elems += dl;
            // hub children (N(c) much longer than L_m): probe N(c) from L_m's side, one
            // binary search per L_m element inside the child's order window, instead of
            // streaming the whole list (the shorter side drives, as in sm_intersect)
            const uint32_t dl0 = dl;
            uint32_t lmask = __ballot_sync(0xffffffffu, (uint64_t)dl > long_at);
            if (dl > long_at) dl = 0;
            while (lmask) {
              const int src = __ffs(lmask) - 1;
              lmask &= lmask - 1;
              const uint32_t cj = __shfl_sync(0xffffffffu, c, src);
              const uint32_t bj = __shfl_sync(0xffffffffu, beg, src);
              const uint32_t dj = __shfl_sync(0xffffffffu, dl0, src);
              const int64_t lo = lt_d ? max(bs.lo, (int64_t)cj) : bs.lo;
              const uint32_t hi = gt_d ? min(bs.hi, cj) : bs.hi;
              const uint32_t a0 = lo < 0 ? 0u : upper_bound_idx(lm, lm_len, (uint32_t)lo);
              const uint32_t a1 = hi == 0 ? 0u : upper_bound_idx(lm, lm_len, hi - 1);
              for (uint32_t t0 = a0; t0 < a1; t0 += 32) {
                const uint32_t t = t0 + lane;
                bool ok = false;
                if (t < a1) {
                  const uint32_t x = lm[t];
                  ok = !(inj_d && x == cj) && contains_hub(a.col + bj, dj, x);
                }
                part += __popc(__ballot_sync(0xffffffffu, ok)) * (lane == 0);
              }
            }
            const uint32_t nz = __ballot_sync(0xffffffffu, dl > 0);
            const uint32_t nnz = __popc(nz);
            const uint32_t src = lane < (int)nnz ? __fns(nz, 0, lane + 1) : 0;
            const uint32_t cbeg = __shfl_sync(0xffffffffu, beg, src);
            const uint32_t sdl = __shfl_sync(0xffffffffu, dl, src);
            const uint32_t cc = __shfl_sync(0xffffffffu, c, src);
            const uint32_t cdl = lane < (int)nnz ? sdl : 0u;
            uint32_t s = cdl;   // exclusive scan of the compacted lengths
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
              const uint32_t y = __shfl_up_sync(0xffffffffu, s, o);
              if (lane >= o) s += y;
            }
            const uint32_t T = __shfl_sync(0xffffffffu, s, 31);
            const uint32_t ost = s - cdl;
            uint32_t nb = 0;
            for (uint32_t t0 = 0; t0 < T; t0 += 32) {
              const uint32_t t = t0 + lane;
              const uint32_t mine = (lane < (int)nnz && ost >= t0 && ost < t0 + 32) ? (1u << (ost - t0)) : 0u;
              const uint32_t S = __reduce_or_sync(0xffffffffu, mine);
              const int j = (int)(nb + __popc(S & upto)) - 1;
              nb += __popc(S);
              const uint32_t bj = __shfl_sync(0xffffffffu, cbeg, j & 31);
              const uint32_t oj = __shfl_sync(0xffffffffu, ost, j & 31);
              const uint32_t cj = __shfl_sync(0xffffffffu, cc, j & 31);
              bool ok = false;
              if (t < T) {
                const uint32_t x = __ldg(a.col + bj + (t - oj));
                const int64_t lo = lt_d ? max(bs.lo, (int64_t)cj) : bs.lo;
                const uint32_t hi = gt_d ? min(bs.hi, cj) : bs.hi;
                ok = x >= lmin && x <= lmax && (int64_t)x > lo && x < hi && !(inj_d && x == cj) &&
                     sorted_contains(lm, lm_len, x);
              }
              part += __popc(__ballot_sync(0xffffffffu, ok)) * (lane == 0);
            }
          }
        } else {
          // cand(c) = L_m ∩ N(c) ∩ window with a short L_m: flatten (child, L_m element)
          // pairs over the lanes; each pair is one binary search of x in N(c)
          const uint64_t T = (uint64_t)len * lm_len;
          for (uint32_t i = lane; i < len; i += 32) elems += gdeg(a, run[i]);   // each N(c) once
          for (uint64_t t0 = 0; t0 < T; t0 += 32) {
            const uint64_t t = t0 + lane;
            bool ok = false;
            if (t < T) {
              const uint32_t i = (uint32_t)(t / lm_len), j = (uint32_t)(t - (uint64_t)i * lm_len);
              const uint32_t c = run[i], x = lm[j];
              const int64_t lo = lt_d ? max(bs.lo, (int64_t)c) : bs.lo;
              const uint32_t hi = gt_d ? min(bs.hi, c) : bs.hi;
              ok = (int64_t)x > lo && x < hi && !(inj_d && x == c);
              if (ok) {
                const uint64_t s0 = a.rp[c];
                const uint32_t dl = (uint32_t)(a.rp[c + 1] - s0);
                ok = dl > 0 && contains_pair(a.col + s0, dl, x);
              }
            }
            part += __popc(__ballot_sync(0xffffffffu, ok)) * (lane == 0);
          }
        }
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) part += __shfl_down_sync(0xffffffffu, part, off);
        acc += (lane == 0) ? part : 0;   // only lane 0's acc is published
        continue;
      }
      for (uint32_t i = 0; i < len && !stop; i++) {
        const uint32_t c = run[i];
        phi[d] = c;
        if (lane == 0) {   // the lists this child's extension fetches
          uint32_t m = (staged ? (child_in_b ? (1u << d) : 0u) : (bq | (a.P.antimask[q] & prefix_mask))) |
                       (anti_d ? (1u << d) : 0u);
          while (m) {
            const int j = __ffs(m) - 1;
            m &= m - 1;
            elems += gdeg(a, phi[j]);
          }
        }
        const Bounds bc = bounds_for(a, q, prefix_mask | (1u << d), phi,
                                     staged ? (1u << d) : (prefix_mask | (1u << d)));
        uint32_t found;
        uint64_t pos = 0;
        bool big = false, via_scratch = false;
        uint32_t *const bsc =
            a.big_scratch ? a.big_scratch + (uint64_t)(blockIdx.x * kWarps + wid) * a.big_scratch_cap : nullptr;
        if (staged && !child_in_b) {
          // candidates = L_m minus position-d filters (all prefix filters applied); a
          // run longer than the staging buffer goes to the warp's global slice (or,
          // without one, straight to lm_len reserved slots of the level)
          found = 0;
          big = !last && lm_len > a.out_cap;
          via_scratch = big && bsc && lm_len <= a.big_scratch_cap;
          if (big && !via_scratch && !pool_reserve(pv, lm_len, lane, pos)) { stop = true; break; }
          uint32_t *dst = via_scratch ? bsc : big ? a.vid_out + pos : sout;
          const uint64_t cs = a.rp[c];
          const uint32_t cl = anti_d ? (uint32_t)(a.rp[c + 1] - cs) : 0u;
          for (uint32_t j0 = 0; j0 < lm_len; j0 += 32) {
            const uint32_t jj = j0 + lane;
            const uint32_t x = jj < lm_len ? lm[jj] : 0xffffffffu;
            bool ok = jj < lm_len && (int64_t)x > bc.lo && x < bc.hi &&
                      !(((a.P.injmask[q] >> d) & 1u) && x == c);
            if (ok && cl) ok = !sorted_contains(a.col + cs, cl, x);   // induced: x not adjacent to c
            const uint32_t bal = __ballot_sync(0xffffffffu, ok);
            if (!last && ok) dst[found + __popc(bal & lanemask_lt())] = x;
            found += __popc(bal);
          }
        } else {
          const uint32_t lists = child_in_b ? (staged ? (1u << d) : bq) : bq;
          if (!last) {
            // upper bound of the child's run: the shortest list involved
            uint32_t ub = staged ? lm_len : 0xffffffffu;
            uint32_t mm = lists;
            while (mm) {
              const int j = __ffs(mm) - 1;
              mm &= mm - 1;
              ub = min(ub, gdeg(a, phi[j]));
            }
            big = ub > a.out_cap;
            // a run that may not fit the staging buffer goes to the warp's global slice
            // (then exactly `found` pool slots); without one, to ub reserved pool slots
            via_scratch = big && a.big_scratch && ub <= a.big_scratch_cap;
            if (big && !via_scratch && !pool_reserve(pv, ub, lane, pos)) { stop = true; break; }
          }
          if (last)
            found = sm_intersect<false>(a, q, lists, phi, bc, last, staged ? lm : nullptr, lm_len, nullptr, 0, lane);
          else
            found = sm_intersect<true>(a, q, lists, phi, bc, last, staged ? lm : nullptr, lm_len,
                                       via_scratch ? bsc : big ? a.vid_out + pos : sout,
                                       big ? 0xffffffffu : a.out_cap, lane);
        }
        if (last) {
          acc += found;
          continue;
        }
        if (found == 0) continue;
        __syncwarp();
        if (via_scratch) {   // exactly the survivors into the pool (one coalesced copy)
          if (!pool_reserve(pv, found, lane, pos)) { stop = true; break; }
          for (uint32_t t = lane; t < found; t += 32) a.vid_out[pos + t] = bsc[t];
        }
        // descriptors: slices of kSlice children, each carrying the prefix + c
        const uint32_t slice = a.slice;
        // the run may split at a slice boundary: whole slices fill the rest of the warp's
        // block (pos), the others go to a fresh one (pos2) -- abandoning the rest instead
        // wasted up to a run per block (C3: 7x the entries written, GAMMA_DEBUG)
        uint32_t first = found;
        uint64_t pos2 = 0;
        if (!big) {
          const uint64_t rest = wv.e - wv.b;
          first = (uint32_t)(rest / slice * slice < found ? rest / slice * slice : found);
          if (first == found) {
            pos = wv.b;
            wv.b += found;
          } else {
            pos = wv.b;
            wv.b += first;
            if (!wb_reserve(wv, pv, found - first, lane, pos2)) { stop = true; break; }
          }
          for (uint32_t t = lane; t < found; t += 32) a.vid_out[t < first ? pos + t : pos2 + (t - first)] = sout[t];
        }
        const uint32_t ns = (found + slice - 1) / slice;
        uint64_t gpos;
        if (ns <= kBlkG)
          wb_retire_tail(wg, ns, lane, [&](uint64_t s) { a.desc_out[s * a.dw_out + 1] = 0u; });
        bool okg = ns <= kBlkG ? wb_reserve(wg, pg, ns, lane, gpos) : pool_reserve(pg, ns, lane, gpos);
        if (!okg) { stop = true; break; }
        for (uint32_t s = 0; s < ns; s++) {
          uint32_t *o = a.desc_out + (gpos + s) * a.dw_out;
          if (lane < (int)a.dw_out) {
            uint32_t val;
            if (lane == 0) val = (uint32_t)(s * slice < first ? pos + s * slice : pos2 + (s * slice - first));
            else if (lane == 1) val = min(slice, found - s * slice);
            else val = phi[0];
#pragma unroll
            for (int j = 0; j < kMaxV; j++)
              if (lane == 2 + j) val = phi[j];
            o[lane] = val;
          }
        }
        out_entries += (lane == 0) ? found : 0;
        __syncwarp();
      }
      __syncwarp();
    }
  }
  if (!last)   // unused descriptor slots of the last block: empty groups
    for (uint64_t s = wg.b; s < wg.e; s++)
      if (lane == 1) a.desc_out[s * a.dw_out + 1] = 0u;
  if (lane == 0) {
    if (acc) atomicAdd(&a.ctrl[CTRL_COUNT], (unsigned long long)acc);
    atomicAdd(&a.ctrl[CTRL_AUX0], (unsigned long long)in_entries);
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) elems += __shfl_down_sync(0xffffffffu, elems, off);
  if (lane == 0) {
    atomicAdd(&a.ctrl[CTRL_ELEMS], (unsigned long long)elems);
    atomicAdd(&a.ctrl[CTRL_ENTRIES], (unsigned long long)out_entries);
  }
}

// ---- roots: label / degree filter, cost order, rank partition ----
struct RootOk {
  const uint64_t *rp;
  const uint32_t *lab;
  uint32_t labeled, label, mindeg;
  __device__ __forceinline__ bool operator()(const uint32_t &v) const {
    if (labeled && (lab ? lab[v] : 0u) != label) return false;
    return rp[v + 1] - rp[v] >= mindeg;
  }
};

__global__ void sm_max_label(const uint32_t *lab, uint32_t n, unsigned long long *out) {
  unsigned long long mx = 0;
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
    mx = lab[v] > mx ? lab[v] : mx;
  for (int o = 16; o > 0; o >>= 1) {
    const unsigned long long y = __shfl_down_sync(0xffffffffu, mx, o);
    mx = y > mx ? y : mx;
  }
  if ((threadIdx.x & 31) == 0 && mx) atomicMax(out, mx);
}

__global__ void sm_ldeg(const uint64_t *rp, const uint32_t *lab, uint32_t n, uint32_t *ldeg) {
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t d = rp[v + 1] - rp[v];
    ldeg[v] = ((lab ? lab[v] : 0u) << 24) | (uint32_t)(d < 0xffffffull ? d : 0xffffffull);
  }
}

__global__ void sm_iota(uint32_t *p, uint32_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    p[i] = (uint32_t)i;
}

__global__ void sm_root_cost(const uint64_t *rp, const uint32_t *roots, uint64_t nr, uint64_t *cost) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nr; i += (uint64_t)gridDim.x * blockDim.x)
    cost[i] = rp[roots[i] + 1] - rp[roots[i]];
}

__global__ void sm_rank_flag(uint64_t nr, uint32_t rank, uint32_t world, uint8_t *flag) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nr; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t r = i % (2ull * world);
    flag[i] = (r == rank || r == 2ull * world - 1 - rank) ? 1 : 0;
  }
}

// depth-0 groups: chunks of kRootChunk roots, descriptor {beg, len}
__global__ void sm_root_groups(uint64_t nr, uint32_t *desc) {
  const uint64_t ngr = (nr + kRootChunk - 1) / kRootChunk;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < ngr; i += (uint64_t)gridDim.x * blockDim.x) {
    desc[2 * i] = (uint32_t)(i * kRootChunk);
    const uint64_t rest = nr - i * kRootChunk;
    desc[2 * i + 1] = (uint32_t)(rest < kRootChunk ? rest : kRootChunk);
  }
}

inline unsigned g1d(uint64_t n) {
  uint64_t b = (n + 255) / 256;
  return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(b, 148u * 32u));
}

static uint32_t env_u32(const char *name, uint32_t dflt, uint32_t lo, uint32_t hi) {
  const char *v = getenv(name);
  if (!v || !*v) return dflt;
  const unsigned long x = strtoul(v, nullptr, 10);
  return x < lo ? lo : (x > hi ? hi : (uint32_t)x);
}
static uint32_t sm_lm_cap() {
  static const uint32_t v = env_u32("GAMMA_SM_LMCAP", kLmCap, 64, 4096);
  return v;
}
static uint32_t sm_out_cap() {
  static const uint32_t v = env_u32("GAMMA_SM_OUTCAP", kOutCap, 64, 4096);
  return v;
}
static uint32_t sm_long_ratio() {
  static const uint32_t v = env_u32("GAMMA_SM_LONGRATIO", kLongRatio, 0, 1u << 20);
  return v;
}
static uint32_t sm_short_lm() {   // GAMMA_SM_SHORTLM (C3, r02: 32 -> 143 ms/step, 0 -> 145 ms)
  static const uint32_t v = env_u32("GAMMA_SM_SHORTLM", 32, 0, 4096);
  return v;
}
static uint32_t sm_batch() {   // groups per work-queue atomic below the roots
  static const uint32_t v = env_u32("GAMMA_SM_BATCH", 2, 1, 256);   // C3: 1 164, 2 156, 4 171, 8 213 ms
  return v;
}
static uint32_t sm_slice(bool consumer_last) {
  static const uint32_t v = env_u32("GAMMA_SM_SLICE", kSlice, 8, 1024);
  static const uint32_t e = env_u32("GAMMA_SM_SLICE_EXT", kSliceExt, 8, 1024);
  return consumer_last ? v : e;
}
static size_t sm_smem() { return (size_t)kWarps * (sm_lm_cap() + sm_out_cap()) * sizeof(uint32_t); }

}  // namespace

// ------------------------------------------------------------------------------------
// Host planner (also exported for tests through gamma_pattern_plan).
// ------------------------------------------------------------------------------------
static void plan_pattern(const gamma_pattern *p, SmPlan &P) {
  GAMMA_REQUIRE(p->nv >= 1 && p->nv <= (uint32_t)kMaxV, GAMMA_E_INVAL, "pattern: nv must be in [1, 8]");
  GAMMA_REQUIRE(p->induced == 0 || p->induced == 1, GAMMA_E_INVAL, "pattern: induced must be 0 or 1");
  GAMMA_REQUIRE(p->ne == 0 || p->edges, GAMMA_E_INVAL, "pattern: NULL edges");
  const uint32_t nv = p->nv;
  int adj[kMaxV][kMaxV] = {};
  for (uint32_t e = 0; e < p->ne; e++) {
    const uint32_t u = p->edges[2 * e], v = p->edges[2 * e + 1];
    GAMMA_REQUIRE(u < nv && v < nv && u != v, GAMMA_E_INVAL, "pattern: bad edge");
    adj[u][v] = adj[v][u] = 1;
  }
  uint32_t deg[kMaxV] = {};
  for (uint32_t u = 0; u < nv; u++)
    for (uint32_t v = 0; v < nv; v++) deg[u] += adj[u][v];
  uint32_t lab[kMaxV] = {};
  for (uint32_t u = 0; u < nv; u++) lab[u] = p->labels ? p->labels[u] : 0;
  // connectivity
  {
    int seen[kMaxV] = {};
    uint32_t st[kMaxV], sp = 0;
    st[sp++] = 0;
    seen[0] = 1;
    uint32_t cnt = 1;
    while (sp) {
      const uint32_t x = st[--sp];
      for (uint32_t y = 0; y < nv; y++)
        if (adj[x][y] && !seen[y]) { seen[y] = 1; st[sp++] = y; cnt++; }
    }
    GAMMA_REQUIRE(cnt == nv, GAMMA_E_INVAL, "pattern: not connected");
  }
  // matching order (reading R10)
  uint32_t order[kMaxV], pos_of[kMaxV];
  int placed[kMaxV] = {};
  for (uint32_t i = 0; i < nv; i++) {
    int best = -1;
    uint32_t bb = 0, bd = 0;
    for (uint32_t u = 0; u < nv; u++) {
      if (placed[u]) continue;
      uint32_t back = 0;
      for (uint32_t t = 0; t < i; t++) back += adj[u][order[t]];
      if (i > 0 && back == 0) continue;   // keep the order connected
      const bool better = best < 0 || back > bb || (back == bb && deg[u] > bd);
      if (better) { best = (int)u; bb = back; bd = deg[u]; }
    }
    order[i] = (uint32_t)best;
    pos_of[best] = i;
    placed[best] = 1;
  }
  // Aut_L by brute force (Heap's algorithm)
  std::vector<std::vector<uint32_t>> autos;
  {
    uint32_t perm[kMaxV], c[kMaxV] = {};
    for (uint32_t i = 0; i < nv; i++) perm[i] = i;
    for (;;) {
      bool ok = true;
      for (uint32_t i = 0; i < nv && ok; i++) {
        if (lab[perm[i]] != lab[i]) ok = false;
        for (uint32_t j = 0; j < nv && ok; j++)
          if (adj[perm[i]][perm[j]] != adj[i][j]) ok = false;
      }
      if (ok) autos.emplace_back(perm, perm + nv);
      uint32_t i = 1;
      while (i < nv && c[i] >= i) { c[i] = 0; i++; }
      if (i >= nv) break;
      const uint32_t j = (i % 2) ? c[i] : 0;
      std::swap(perm[j], perm[i]);
      c[i]++;
    }
  }
  std::memset(&P, 0, sizeof(P));
  P.nv = nv;
  P.labeled = p->labels != nullptr;
  P.aut = autos.size();
  for (uint32_t i = 0; i < nv; i++) {
    const uint32_t u = order[i];
    P.order[i] = u;
    P.label[i] = lab[u];
    P.mindeg[i] = deg[u];
    for (uint32_t t = 0; t < i; t++) {
      if (adj[u][order[t]]) P.bmask[i] |= 1u << t;
      else P.injmask[i] |= 1u << t;
      if (!adj[u][order[t]] && p->induced) P.antimask[i] |= 1u << t;
    }
  }
  // stabilizer chain along the matching order
  std::vector<std::vector<uint32_t>> G = autos;
  for (uint32_t i = 0; i < nv; i++) {
    const uint32_t v = order[i];
    bool orbit[kMaxV] = {};
    for (auto &g : G) orbit[g[v]] = true;
    for (uint32_t u = 0; u < nv; u++) {
      if (u == v || !orbit[u]) continue;
      // phi(v) < phi(u); u is placed later than v (it is still in v's orbit
      // under the stabilizer of every earlier vertex, so it is not earlier)
      const uint32_t pu = pos_of[u];
      if (pu > i) P.ltmask[pu] |= 1u << i;
      else P.gtmask[i] |= 1u << pu;
    }
    std::vector<std::vector<uint32_t>> H;
    for (auto &g : G)
      if (g[v] == v) H.push_back(g);
    G.swap(H);
  }
}

struct SmLevel {
  DevBuf<uint32_t> vid;
  DevBuf<uint32_t> desc;
  uint64_t cap_v = 0, cap_g = 0;
  uint32_t dw = 0;
};

struct SmRun {
  gamma_graph *g;
  gamma_ctx *ctx;
  SmPlan P;
  std::vector<SmLevel> lv;    // lv[d]: groups at depth d (d = 0: root chunks)
  uint64_t level_share;
  uint64_t total = 0;
  int grid = 0;
  uint32_t stage = 1;
  DevBuf<uint32_t> lm_scratch;       // per-warp global L_m slices (hub prefixes)
  uint32_t lm_scratch_cap = 0;
  DevBuf<uint32_t> big_scratch;      // per-warp global slices for child runs above out_cap
  uint32_t big_scratch_cap = 0;

  // First table size of a level (grow caps it at the level's share of the HBM budget):
  // 2^27 entry slots and 2^23 group descriptors (C3's widest level: 5.1e7 entries, under
  // 2e6 groups).  Round 1's 2^24 overflowed on C3's 4-cycle in every call (the pool cursor
  // ran to 2.8e8 slots while runs reserved upper bounds and abandoned block tails), so
  // the one-read-back chain was thrown away and the query rerun on the careful path.
  uint64_t initial_cap() const {
    return std::max<uint64_t>(1ull << GAMMA_SM_CAP_LOG2, 4ull * kBlkV * kWarps * (uint64_t)grid);
  }

  // Tables of level d for want_v entries and want_g group descriptors (0: cap_v / 8),
  // never smaller than they are, scaled down together to the level's share of the HBM
  // budget.  Returns false when nothing grew.
  bool grow(uint32_t d, uint64_t want_v, uint64_t want_g = 0) {
    SmLevel &L = lv[d];
    const uint32_t dw = 2 + d;
    uint64_t cv = std::max<uint64_t>(std::max<uint64_t>(want_v, 1ull << 16), L.cap_v);
    uint64_t cg = std::max<uint64_t>(std::max<uint64_t>(cv / 8, want_g), L.cap_g);
    const double bytes = 4.0 * cv + 4.0 * dw * cg;
    if (bytes > (double)level_share) {
      const double f = (double)level_share / bytes;
      cv = (uint64_t)(cv * f);
      cg = (uint64_t)(cg * f);
    }
    cv = std::min<uint64_t>(cv, 0xFFFFFFFFull - kBlkV);
    cg = std::max<uint64_t>(cg, 2 * kBlkG);
    if (cv <= L.cap_v && cg <= L.cap_g) return false;
    cv = std::max<uint64_t>(cv, L.cap_v);
    cg = std::max<uint64_t>(cg, L.cap_g);
    // the superseded (smaller) tables are freed, not kept: keeping them would hold
    // ~1/3 more than level_share per level and shrink later budgets
    L.vid.kept = false;
    L.desc.kept = false;
    L.vid.reset();
    L.desc.reset();
    L.vid = DevBuf<uint32_t>(ctx, cv, true);
    L.desc = DevBuf<uint32_t>(ctx, cg * dw, true);
    L.cap_v = cv;
    L.cap_g = cg;
    L.dw = dw;
    return true;
  }

  SmArgs args(uint32_t d, uint64_t g0, uint64_t g1) {
    SmArgs a{};
    a.rp = g->row_ptr;
    a.col = g->col;
    a.lab = g->labels;
    a.ldeg = g->ldeg;
    a.P = P;
    a.d = d;
    a.vid_in = lv[d].vid.p;
    a.desc_in = lv[d].desc.p;
    a.dw_in = 2 + d;
    a.g_begin = g0;
    a.g_end = g1;
    a.ctrl = (unsigned long long *)ctx->ctrl;
    a.ovf = a.ctrl + CTRL_OVF;
    a.gcur_in = nullptr;
    a.batch = d == 0 ? 1 : sm_batch();
    a.stage = stage;
    a.lm_scratch = lm_scratch.p;
    a.lm_scratch_cap = lm_scratch_cap;
    a.big_scratch = big_scratch.p;
    a.big_scratch_cap = big_scratch_cap;
    a.lm_cap = sm_lm_cap();
    a.out_cap = sm_out_cap();
    a.long_ratio = sm_long_ratio();
    a.short_lm = sm_short_lm();
    a.slice = sm_slice(d + 2 >= P.nv - 1);   // the groups written here are consumed at depth d+1
    return a;
  }

  int grid_for(bool last, uint64_t cap_v) const {
    int gr = grid;
    if (!last) {
      const uint64_t warps_ok = std::max<uint64_t>(1, cap_v / (2ull * kBlkV));
      gr = (int)std::max<uint64_t>(1, std::min<uint64_t>(gr, warps_ok / kWarps));
    }
    return gr;
  }

  void run_kernel(const SmArgs &a, bool last, uint64_t cap_v) {
    const int gr = grid_for(last, cap_v);
    ctrl_reset(ctx);
    const int kc = last ? KC_SM_COUNT : KC_SM_EXTEND;
    ctx->launch(kc, [&] { sm_kernel<<<gr, kThreads, sm_smem(), ctx->stream>>>(a); });
    ctrl_fetch(ctx);
    const uint64_t *h = ctx->ctrl_host;
    if (!h[CTRL_OVF]) {   // 12 B per input entry, 4 B per list element, 8 B per output
      ctx->stats.list_elems += h[CTRL_ELEMS];
      ctx->stats.alg_bytes[kc] += 12 * h[CTRL_AUX0] + 4 * h[CTRL_ELEMS] + (last ? 0 : 8 * h[CTRL_ENTRIES]);
    }
  }

  // The whole level chain of a query enqueued back to back with one read-back at the
  // end: level d's launch reads its group count from level d-1's cursor on the device
  // (SmArgs::gcur_in), each level has its own control block (CTRL_LEVELS), and one
  // shared overflow word makes every later level exit at once.  Returns false (nothing
  // recorded) when some level overflowed its table; the caller then runs the careful
  // per-level path (process), which grows tables and halves group ranges.
  // chain_enqueue + chain_collect on the context's own stream and control block
  bool chain(uint64_t ngroups) {
    chain_enqueue(ngroups, ctx->stream, (unsigned long long *)ctx->ctrl, ctx->ctrl_host);
    ctx->sync();
    return chain_collect(ctx->ctrl_host);
  }

  void chain_enqueue(uint64_t ngroups, cudaStream_t st, unsigned long long *ctrl, uint64_t *host) {
    const uint32_t nl = P.nv - 1;   // launches: d = 0 .. nv-2
    for (uint32_t q = 1; q < nl; q++)
      if (lv[q].cap_v == 0) grow(q, initial_cap(), 1ull << 23);
    GAMMA_CUDA(cudaMemsetAsync(ctrl, 0, CTRL_WORDS * sizeof(uint64_t), st));
    for (uint32_t d = 0; d < nl; d++) {
      const uint32_t q = d + 1;
      const bool last = q == P.nv - 1;
      SmArgs a = args(d, 0, ngroups);
      a.ctrl = ctrl + CTRL_LEVELS + CTRL_LSTRIDE * d;
      a.ovf = ctrl + CTRL_OVF;
      if (d > 0) {
        a.gcur_in = ctrl + CTRL_LEVELS + CTRL_LSTRIDE * (d - 1) + CTRL_GCUR;
        a.cap_g_in = lv[d].cap_g;
      }
      if (!last) {
        a.vid_out = lv[q].vid.p;
        a.desc_out = lv[q].desc.p;
        a.dw_out = 2 + q;
        a.cap_v = lv[q].cap_v;
        a.cap_g = lv[q].cap_g;
      }
      const int gr = grid_for(last, last ? 0 : lv[q].cap_v);
      const int kc = last ? KC_SM_COUNT : KC_SM_EXTEND;
      ctx->launch_on(kc, st, [&] { sm_kernel<<<gr, kThreads, sm_smem(), st>>>(a); });
    }
    GAMMA_CUDA(cudaMemcpyAsync(host, ctrl, CTRL_WORDS * sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
  }

  // after the stream of chain_enqueue completed: false (nothing recorded) on an overflow
  bool chain_collect(const uint64_t *h) {
    const uint32_t nl = P.nv - 1;
    if (h[CTRL_OVF]) {
      // hint for the careful path: grow the tables that ran out
      for (uint32_t d = 0; d + 1 < nl; d++) {
        const uint64_t *b = h + CTRL_LEVELS + CTRL_LSTRIDE * d;
        // (a cursor past its capacity: that pool ran out -- entries or group descriptors)
        const bool ov = b[CTRL_VCUR] > lv[d + 1].cap_v, og = b[CTRL_GCUR] > lv[d + 1].cap_g;
        if (getenv("GAMMA_DEBUG"))
          fprintf(stderr, "[gamma sm chain] nv %u level %u: entries %llu / %llu, groups %llu / %llu, share %llu\n",
                  P.nv, d + 1, (unsigned long long)b[CTRL_VCUR], (unsigned long long)lv[d + 1].cap_v,
                  (unsigned long long)b[CTRL_GCUR], (unsigned long long)lv[d + 1].cap_g,
                  (unsigned long long)level_share);
        if (ov || og) grow(d + 1, ov ? 2 * b[CTRL_VCUR] : 0, og ? 2 * b[CTRL_GCUR] : 0);
      }
      return false;
    }
    for (uint32_t d = 0; d < nl; d++) {
      const uint64_t *b = h + CTRL_LEVELS + CTRL_LSTRIDE * d;
      const bool last = d + 2 == P.nv;
      const int kc = last ? KC_SM_COUNT : KC_SM_EXTEND;
      ctx->stats.list_elems += b[CTRL_ELEMS];
      ctx->stats.alg_bytes[kc] += 12 * b[CTRL_AUX0] + 4 * b[CTRL_ELEMS] + (last ? 0 : 8 * b[CTRL_ENTRIES]);
      if (last) {
        total = checked_add(total, b[CTRL_COUNT]);
        ctx->stats.level_entries[P.nv] = checked_add(ctx->stats.level_entries[P.nv], b[CTRL_COUNT]);
      } else {
        ctx->stats.level_entries[d + 2] += b[CTRL_ENTRIES];
        ctx->stats.chunks++;
      }
    }
    return true;
  }

  void process(uint32_t d, uint64_t g0, uint64_t g1) {
    if (g0 >= g1) return;
    const uint32_t q = d + 1;
    const bool last = q == P.nv - 1;
    if (last) {
      SmArgs a = args(d, g0, g1);
      run_kernel(a, true, 0);
      const uint64_t *h = ctx->ctrl_host;
      total = checked_add(total, h[CTRL_COUNT]);
      ctx->stats.level_entries[P.nv] = checked_add(ctx->stats.level_entries[P.nv], h[CTRL_COUNT]);
      return;
    }
    for (;;) {
      SmLevel &L = lv[q];
      if (L.cap_v == 0) grow(q, initial_cap(), 1ull << 23);
      SmArgs a = args(d, g0, g1);
      a.vid_out = L.vid.p;
      a.desc_out = L.desc.p;
      a.dw_out = 2 + q;
      a.cap_v = L.cap_v;
      a.cap_g = L.cap_g;
      run_kernel(a, false, L.cap_v);
      const uint64_t *h = ctx->ctrl_host;
      if (!h[CTRL_OVF]) {
        ctx->stats.level_entries[q + 1] += h[CTRL_ENTRIES];
        ctx->stats.chunks++;
        process(q, 0, std::min<uint64_t>(h[CTRL_GCUR], L.cap_g));
        return;
      }
      ctx->stats.retries++;
      if (grow(q, std::max<uint64_t>(h[CTRL_VCUR], L.cap_v) * 4, std::max<uint64_t>(h[CTRL_GCUR], L.cap_g) * 4))
        continue;
      GAMMA_REQUIRE(g1 - g0 > 1, GAMMA_E_NOMEM, "HBM budget too small for one embedding group (SM)");
      const uint64_t mid = g0 + (g1 - g0) / 2;
      process(d, g0, mid);
      process(d, mid, g1);
      return;
    }
  }
};

static void ensure_ldeg(gamma_graph *g) {
  if (g->ldeg_state >= 0) return;
  gamma_ctx *ctx = g->ctx;
  uint64_t ml = 0;
  if (g->labels) {
    GAMMA_CUDA(cudaMemsetAsync(ctx->ctrl + CTRL_AUX0, 0, 8, ctx->stream));
    ctx->launch(KC_ROOTS, [&] {
      sm_max_label<<<g1d(g->n), 256, 0, ctx->stream>>>(g->labels, g->n, (unsigned long long *)ctx->ctrl + CTRL_AUX0);
    });
    GAMMA_CUDA(cudaMemcpyAsync(&ml, ctx->ctrl + CTRL_AUX0, 8, cudaMemcpyDeviceToHost, ctx->stream));
    ctx->sync();
  }
  g->ldeg_state = 0;
  if (ml >= 256) return;
  DevBuf<uint32_t> ld(ctx, g->n);
  ctx->launch(KC_ROOTS, [&] { sm_ldeg<<<g1d(g->n), 256, 0, ctx->stream>>>(g->row_ptr, g->labels, g->n, ld.p); });
  g->ldeg = ld.release();
  g->device_bytes += (uint64_t)g->n * 4;
  g->ldeg_state = 1;
}

// ---- SM by edge extension ("binary join"):
// the embedding table grows by ONE pattern edge per step instead of one vertex with all
// its backward edges at once (Alg. 1's vertex extension, the path above): a tree edge
// (the position's first backward neighbour b0) expands every row by the candidates in
// N(phi(b0)) (label, degree, injectivity and symmetry-order filters), and every further
// backward edge -- and, induced, every anti-edge -- is a separate pass that keeps the
// rows whose pair is (resp. is not) adjacent.  Same constraints, same count; the
// intermediate tables are what the vertex extension avoids (the ablation's point).
// Rows are phi_0..phi_t (t+1 u32, row-major); root ranges are halved on overflow.
struct JoinArgs {
  const uint64_t *rp;
  const uint32_t *col;
  const uint32_t *ldeg;   // label << 24 | degree (nullable: labels / degrees gathered separately)
  const uint32_t *lab;
  SmPlan P;
  const uint32_t *in;
  uint64_t n_in;
  uint32_t w_in;          // words per input row (= positions placed)
  uint32_t *out;
  uint64_t cap;           // output rows
  unsigned long long *cursor, *ovf, *count;
  uint32_t q;             // expand: the position being placed; check: its later endpoint
  uint32_t b;             // expand: b0; check: the earlier endpoint
  uint32_t anti;          // check: keep rows whose pair is NOT adjacent
  uint32_t count_only;    // last step: count, do not write
};

// one warp per input row: lanes stream N(phi(b0)), survivors are compacted and appended
__global__ void __launch_bounds__(256) sm_join_expand(JoinArgs a) {
  const int lane = threadIdx.x & 31;
  const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  const uint32_t q = a.q, placed = (1u << q) - 1u;
  const bool last = q + 1 == a.P.nv;
  unsigned long long cnt = 0;
  for (uint64_t r = warp; r < a.n_in; r += nw) {
    if (!a.count_only && *(volatile unsigned long long *)a.ovf) break;
    const uint32_t *row = a.in + r * a.w_in;
    uint32_t phi[kMaxV];
#pragma unroll
    for (int j = 0; j < kMaxV; j++) phi[j] = j < (int)a.w_in ? row[j] : 0u;
    const Bounds bd = bounds_for_join(a.P, q, placed, phi);
    const uint64_t s0 = a.rp[phi[a.b]];
    const uint32_t dl = (uint32_t)(a.rp[phi[a.b] + 1] - s0);
    for (uint32_t j0 = 0; j0 < dl; j0 += 32) {
      const uint32_t jj = j0 + lane;
      const uint32_t x = jj < dl ? a.col[s0 + jj] : 0xffffffffu;
      bool ok = jj < dl && (int64_t)x > bd.lo && x < bd.hi;
      if (ok && (a.P.labeled || (!last && a.P.mindeg[q] > 1))) {
        uint32_t lx, dx;
        if (a.ldeg) {
          const uint32_t ld = a.ldeg[x];
          lx = ld >> 24;
          dx = ld & 0xffffffu;
        } else {
          lx = a.lab ? a.lab[x] : 0u;
          dx = (uint32_t)(a.rp[x + 1] - a.rp[x]);
        }
        ok = (!a.P.labeled || lx == a.P.label[q]) && (last || dx >= a.P.mindeg[q]);
      }
#pragma unroll
      for (int j = 0; j < kMaxV; j++)
        if (ok && j < (int)q && phi[j] == x) ok = false;   // injective against every placed position
      const uint32_t bal = __ballot_sync(0xffffffffu, ok);
      if (!bal) continue;
      if (a.count_only) {
        cnt += (lane == 0) ? __popc(bal) : 0;
        continue;
      }
      unsigned long long base = 0;
      if (lane == 0) base = atomicAdd(a.cursor, (unsigned long long)__popc(bal));
      base = __shfl_sync(0xffffffffu, base, 0);
      if (base + __popc(bal) > a.cap) {
        if (lane == 0) atomicExch(a.ovf, 1ull);
        break;
      }
      if (ok) {
        uint32_t *o = a.out + (base + __popc(bal & lanemask_lt())) * (a.w_in + 1);
        for (uint32_t j = 0; j < a.w_in; j++) o[j] = phi[j];
        o[a.w_in] = x;
      }
    }
  }
  if (a.count_only) {
    for (int off = 16; off > 0; off >>= 1) cnt += __shfl_down_sync(0xffffffffu, cnt, off);
    if (lane == 0 && cnt) atomicAdd(a.count, cnt);
  }
}

// one thread per row: keep it iff phi(b) ~ phi(q) (anti: iff not); warp-aggregated append
__global__ void __launch_bounds__(256) sm_join_check(JoinArgs a) {
  const int lane = threadIdx.x & 31;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  unsigned long long cnt = 0;
  for (uint64_t r0 = blockIdx.x * (uint64_t)blockDim.x; r0 < a.n_in; r0 += stride) {
    const uint64_t r = r0 + threadIdx.x;
    bool ok = false;
    if (r < a.n_in) {
      const uint32_t *row = a.in + r * a.w_in;
      const uint32_t u = row[a.b], x = row[a.q];
      const uint64_t s0 = a.rp[u];
      const uint32_t dl = (uint32_t)(a.rp[u + 1] - s0);
      ok = (dl && sorted_contains(a.col + s0, dl, x)) != (a.anti != 0);
    }
    const uint32_t bal = __ballot_sync(0xffffffffu, ok);
    if (a.count_only) {
      cnt += (lane == 0) ? __popc(bal) : 0;
      continue;
    }
    if (!bal) continue;
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(a.cursor, (unsigned long long)__popc(bal));
    base = __shfl_sync(0xffffffffu, base, 0);
    if (base + __popc(bal) > a.cap) {   // cannot happen (a filter shrinks), kept for safety
      if (lane == 0) atomicExch(a.ovf, 1ull);
      break;
    }
    if (ok) {
      const uint32_t *row = a.in + r * a.w_in;
      uint32_t *o = a.out + (base + __popc(bal & lanemask_lt())) * a.w_in;
      for (uint32_t j = 0; j < a.w_in; j++) o[j] = row[j];
    }
  }
  if (a.count_only) {
    for (int off = 16; off > 0; off >>= 1) cnt += __shfl_down_sync(0xffffffffu, cnt, off);
    if (lane == 0 && cnt) atomicAdd(a.count, cnt);
  }
}

struct JoinStep {
  uint32_t kind;   // 0 expand, 1 check, 2 anti-check
  uint32_t q, b;
};

static std::vector<JoinStep> join_steps(const SmPlan &P) {
  std::vector<JoinStep> st;
  for (uint32_t q = 1; q < P.nv; q++) {
    const uint32_t b0 = (uint32_t)__builtin_ctz(P.bmask[q]);
    st.push_back({0, q, b0});
    for (uint32_t m = P.bmask[q] & ~(1u << b0); m; m &= m - 1) st.push_back({1, q, (uint32_t)__builtin_ctz(m)});
    for (uint32_t m = P.antimask[q]; m; m &= m - 1) st.push_back({2, q, (uint32_t)__builtin_ctz(m)});
  }
  return st;
}

// DFS over (step, row range): step i turns its input rows into buffer i; a step whose
// output overflows the buffer halves its input range (any step, not only the roots).
struct JoinRun {
  gamma_graph *g;
  gamma_ctx *ctx;
  SmPlan P;
  std::vector<JoinStep> steps;
  std::vector<DevBuf<uint32_t>> buf;   // one row buffer per step
  uint64_t cap;                        // rows per buffer
  DevBuf<unsigned long long> cur;      // cursor, overflow, count
  uint64_t total = 0;

  void run(size_t i, const uint32_t *in, uint64_t n_in, uint32_t w) {
    if (n_in == 0) return;
    const JoinStep &stp = steps[i];
    JoinArgs a{};
    a.rp = g->row_ptr;
    a.col = g->col;
    a.ldeg = g->ldeg;
    a.lab = g->labels;
    a.P = P;
    a.in = in;
    a.n_in = n_in;
    a.w_in = w;
    a.out = buf[i].p;
    a.cap = cap;
    a.cursor = cur.p;
    a.ovf = cur.p + 1;
    a.count = cur.p + 2;
    a.q = stp.q;
    a.b = stp.b;
    a.anti = stp.kind == 2;
    a.count_only = i + 1 == steps.size();
    GAMMA_CUDA(cudaMemsetAsync(cur.p, 0, 24, ctx->stream));
    const int kc = a.count_only ? KC_SM_COUNT : KC_SM_EXTEND;
    if (stp.kind == 0)
      ctx->launch(kc, [&] { sm_join_expand<<<g1d(n_in * 32), 256, 0, ctx->stream>>>(a); });
    else
      ctx->launch(kc, [&] { sm_join_check<<<g1d(n_in), 256, 0, ctx->stream>>>(a); });
    uint64_t h[3];
    GAMMA_CUDA(cudaMemcpyAsync(h, cur.p, 24, cudaMemcpyDeviceToHost, ctx->stream));
    ctx->sync();
    if (h[1]) {   // overflow: halve this step's input
      ctx->stats.retries++;
      GAMMA_REQUIRE(n_in > 1, GAMMA_E_NOMEM, "edge join: the rows of one embedding exceed the buffer");
      const uint64_t half = n_in / 2;
      run(i, in, half, w);
      run(i, in + half * w, n_in - half, w);
      return;
    }
    if (a.count_only) {
      total = checked_add(total, h[2]);
      ctx->stats.chunks++;
      return;
    }
    const uint32_t w2 = stp.kind == 0 ? w + 1 : w;
    if (stp.kind == 0) ctx->stats.level_entries[w2] += h[0];
    run(i + 1, buf[i].p, h[0], w2);
  }
};

static uint64_t match_join(gamma_graph *g, const SmPlan &P, const uint32_t *roots, uint64_t nr,
                           uint64_t level_share) {
  gamma_ctx *ctx = g->ctx;
  JoinRun J;
  J.g = g;
  J.ctx = ctx;
  J.P = P;
  J.steps = join_steps(P);
  const uint64_t nb = std::max<size_t>(1, J.steps.size() - 1);   // the last step only counts
  J.cap = std::max<uint64_t>(1 << 12, level_share * std::max<uint32_t>(1, P.nv > 2 ? P.nv - 2 : 1) / nb /
                                          (4ull * P.nv));
  for (size_t i = 0; i < J.steps.size(); i++) J.buf.emplace_back(ctx, i + 1 < J.steps.size() ? J.cap * P.nv : 1);
  J.cur = DevBuf<unsigned long long>(ctx, 3);
  for (uint64_t r0 = 0; r0 < nr; r0 += J.cap) J.run(0, roots + r0, std::min<uint64_t>(J.cap, nr - r0), 1);
  ctx->stats.level_entries[P.nv] = J.total;
  ctx->sync();
  ctx->collect_timings();
  return J.total;
}

// Roots, group table and staging scratch of one query (everything before the level
// chain).  Returns true with `count` set when the query is already answered (nv = 1,
// no roots, or the edge-join variant); else ngroups = the depth-0 groups.
static bool match_prepare(gamma_graph *g, const SmPlan &P, SmRun &R, uint64_t &count, uint64_t &ngroups,
                          uint32_t batch = 1) {
  gamma_ctx *ctx = g->ctx;
  ensure_ldeg(g);
  R.g = g;
  R.ctx = ctx;
  R.P = P;
  R.lv.resize(kMaxV + 1);
  R.stage = (ctx->desc.flags & GAMMA_FLAG_DEBUG_NOSTAGE) ? 0u : 1u;
  {
    size_t fr = 0, tot = 0;
    GAMMA_CUDA(cudaMemGetInfo(&fr, &tot));
    // (the context's kept buffers count as free: this call's tables take them back)
    size_t kept = 0;
    for (const auto &b : ctx->kept) kept += b.second;
    const uint64_t budget =
        ctx->desc.hbm_budget_bytes ? ctx->desc.hbm_budget_bytes : (uint64_t)((double)(fr + kept) * 0.8);
    R.level_share = budget / batch / std::max<uint32_t>(1, P.nv > 2 ? P.nv - 2 : 1);
  }
  // ---- roots (position 0) ----
  const uint32_t n = g->n;
  DevBuf<uint32_t> all(ctx, n), sel(ctx, n);
  DevBuf<uint64_t> nsel(ctx, 1);
  ctx->launch(KC_ROOTS, [&] { sm_iota<<<g1d(n), 256, 0, ctx->stream>>>(all.p, n); });
  RootOk op{g->row_ptr, g->labels, P.labeled, P.label[0], P.mindeg[0]};
  size_t tmp = 0;
  GAMMA_CUDA(cub::DeviceSelect::If(nullptr, tmp, all.p, sel.p, nsel.p, (int64_t)n, op, ctx->stream));
  {
    DevBuf<uint8_t> t(ctx, tmp);
    ctx->launch(KC_ROOTS, [&] {
      GAMMA_CUDA(cub::DeviceSelect::If(t.p, tmp, all.p, sel.p, nsel.p, (int64_t)n, op, ctx->stream));
    });
    ctx->cub_select_launched(KC_ROOTS);
  }
  uint64_t nr = 0;
  GAMMA_CUDA(cudaMemcpyAsync(&nr, nsel.p, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
  ctx->sync();
  if (P.nv == 1) {
    if (ctx->desc.world > 1) {   // partition the roots like everything else
      const uint64_t w = ctx->desc.world, r = ctx->desc.rank;
      uint64_t mine = 0;
      for (uint64_t i = 0; i < nr; i++) {
        const uint64_t x = i % (2 * w);
        mine += (x == r || x == 2 * w - 1 - r);
      }
      count = mine;
      return true;
    }
    count = nr;
    return true;
  }
  DevBuf<uint32_t> roots(ctx, nr ? nr : 1);
  if (nr) {
    DevBuf<uint64_t> cost(ctx, nr), cost2(ctx, nr);
    ctx->launch(KC_ROOTS, [&] { sm_root_cost<<<g1d(nr), 256, 0, ctx->stream>>>(g->row_ptr, sel.p, nr, cost.p); });
    int endbit = 1;
    while (endbit < 64 && (1ull << endbit) <= (uint64_t)g->max_degree) endbit++;
    tmp = 0;
    GAMMA_CUDA(cub::DeviceRadixSort::SortPairsDescending(nullptr, tmp, cost.p, cost2.p, sel.p, roots.p, nr, 0,
                                                         endbit, ctx->stream));
    DevBuf<uint8_t> t(ctx, tmp);
    ctx->launch(KC_ROOTS, [&] {
      GAMMA_CUDA(cub::DeviceRadixSort::SortPairsDescending(t.p, tmp, cost.p, cost2.p, sel.p, roots.p, nr, 0,
                                                           endbit, ctx->stream));
    });
    ctx->cub_sort_launched(KC_ROOTS, nr, endbit);
  }
  if (ctx->desc.world > 1 && nr) {
    DevBuf<uint8_t> flag(ctx, nr);
    ctx->launch(KC_ROOTS, [&] {
      sm_rank_flag<<<g1d(nr), 256, 0, ctx->stream>>>(nr, ctx->desc.rank, ctx->desc.world, flag.p);
    });
    DevBuf<uint32_t> mine(ctx, nr);
    tmp = 0;
    GAMMA_CUDA(cub::DeviceSelect::Flagged(nullptr, tmp, roots.p, flag.p, mine.p, nsel.p, (int64_t)nr, ctx->stream));
    {
      DevBuf<uint8_t> t(ctx, tmp);
      ctx->launch(KC_ROOTS, [&] {
        GAMMA_CUDA(cub::DeviceSelect::Flagged(t.p, tmp, roots.p, flag.p, mine.p, nsel.p, (int64_t)nr, ctx->stream));
      });
      ctx->cub_select_launched(KC_ROOTS);
    }
    GAMMA_CUDA(cudaMemcpyAsync(&nr, nsel.p, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
    ctx->sync();
    roots = std::move(mine);
  }
  ctx->stats.level_entries[1] = nr;
  if (nr == 0) {
    count = 0;
    return true;
  }
  if (ctx->desc.flags & GAMMA_FLAG_SM_EDGE_JOIN) {
    count = match_join(g, P, roots.p, nr, R.level_share);
    return true;
  }
  const uint64_t ngr = (nr + kRootChunk - 1) / kRootChunk;
  SmLevel &L0 = R.lv[0];
  L0.desc = DevBuf<uint32_t>(ctx, 2 * ngr);
  L0.dw = 2;
  ctx->launch(KC_ROOTS, [&] { sm_root_groups<<<g1d(ngr), 256, 0, ctx->stream>>>(nr, L0.desc.p); });
  L0.vid = std::move(roots);
  L0.cap_v = nr;
  L0.cap_g = ngr;
  static bool attr = false;
  if (!attr) {
    GAMMA_CUDA(cudaFuncSetAttribute(sm_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm_smem()));
    attr = true;
  }
  R.grid = ctx->num_sms * occupancy_blocks((const void *)sm_kernel, kThreads, sm_smem());
  if (g->max_degree > sm_lm_cap()) {   // room for a hub's L_m (bounded by its degree) per warp
    R.lm_scratch_cap = std::min<uint32_t>(g->max_degree, 1u << 16);
    R.lm_scratch = DevBuf<uint32_t>(ctx, (uint64_t)R.grid * kWarps * R.lm_scratch_cap, true);
  }
  if (P.nv > 2 && g->max_degree > sm_out_cap()) {
    // a child run above the staging buffer is bounded by a list length (<= max degree):
    // kept in the warp's slice, then copied to exactly `found` pool slots (reserving the
    // bound in the pool ran its cursor 5x past the entries written on C3)
    R.big_scratch_cap = std::min<uint32_t>(g->max_degree, 1u << 16);
    R.big_scratch = DevBuf<uint32_t>(ctx, (uint64_t)R.grid * kWarps * R.big_scratch_cap, true);
  }
  ngroups = ngr;
  return false;
}

static bool sm_fast_ok(gamma_ctx *ctx, const SmPlan &P) {
  return (ctx->desc.flags & GAMMA_FLAG_SPILL) == 0 && P.nv >= 2 && P.nv - 1 <= 12 &&
         getenv("GAMMA_SM_NO_CHAIN") == nullptr;
}

static uint64_t match_count(gamma_graph *g, const SmPlan &P) {
  gamma_ctx *ctx = g->ctx;
  SmRun R;
  uint64_t count = 0, ngr = 0;
  if (match_prepare(g, P, R, count, ngr)) return count;
  // fast path: the whole level chain with one read-back; on a table overflow, the
  // careful per-level path (DFS over group ranges with table growth and halving)
  const bool fast = sm_fast_ok(ctx, P);
  if (!fast || !R.chain(ngr)) {
    if (fast) ctx->stats.retries++;
    R.process(0, 0, ngr);
  }
  ctx->sync();
  ctx->collect_timings();
  return R.total;
}

// Several queries at once (gamma_match_batch): roots of every query first, then every
// level chain on its own side stream (a chain's kernels run back to back, the chains
// overlap each other's tails), one wait; an overflowing chain reruns alone on the
// careful path.
static void match_batch(gamma_graph *g, const std::vector<SmPlan> &Ps, std::vector<uint64_t> &counts) {
  gamma_ctx *ctx = g->ctx;
  const size_t nq = Ps.size();
  counts.assign(nq, 0);
  std::vector<std::unique_ptr<SmRun>> runs(nq);
  std::vector<uint64_t> ngr(nq, 0);
  std::vector<bool> done(nq, false);
  const bool dbg = getenv("GAMMA_DEBUG") != nullptr;   // host wall time of the phases
  auto now = [] { return std::chrono::steady_clock::now(); };
  auto ms = [](std::chrono::steady_clock::time_point a, std::chrono::steady_clock::time_point b) {
    return std::chrono::duration<double, std::milli>(b - a).count();
  };
  const auto t0 = now();
  std::vector<double> tprep(nq, 0.0);
  for (size_t i = 0; i < nq; i++) {
    const auto ti = now();
    runs[i].reset(new SmRun());
    uint64_t c = 0;
    done[i] = match_prepare(g, Ps[i], *runs[i], c, ngr[i], (uint32_t)std::min<size_t>(nq, gamma_ctx::kMaxBatch));
    if (done[i]) counts[i] = c;
    tprep[i] = ms(ti, now());
  }
  const auto t1 = now();
  ctx->side_init();
  cudaEvent_t ready;
  GAMMA_CUDA(cudaEventCreateWithFlags(&ready, cudaEventDisableTiming));
  GAMMA_CUDA(cudaEventRecord(ready, ctx->stream));   // roots and tables are on ctx->stream
  std::vector<int> slot(nq, -1);
  int used = 0;
  for (size_t i = 0; i < nq; i++) {
    if (done[i] || !sm_fast_ok(ctx, Ps[i]) || used >= gamma_ctx::kMaxBatch) continue;
    const int sl = used++;
    slot[i] = sl;
    cudaStream_t st = ctx->side_streams[sl];
    GAMMA_CUDA(cudaStreamWaitEvent(st, ready, 0));
    runs[i]->chain_enqueue(ngr[i], st, (unsigned long long *)(ctx->side_ctrl + (size_t)sl * CTRL_WORDS),
                           ctx->side_ctrl_host + (size_t)sl * CTRL_WORDS);
  }
  const auto t2 = now();
  for (int sl = 0; sl < used; sl++) GAMMA_CUDA(cudaStreamSynchronize(ctx->side_streams[sl]));
  const auto t3 = now();
  cudaEventDestroy(ready);
  for (size_t i = 0; i < nq; i++) {
    if (done[i]) continue;
    SmRun &R = *runs[i];
    bool ok = slot[i] >= 0 && R.chain_collect(ctx->side_ctrl_host + (size_t)slot[i] * CTRL_WORDS);
    if (!ok) {
      if (slot[i] >= 0) ctx->stats.retries++;
      R.process(0, 0, ngr[i]);
    }
    counts[i] = R.total;
  }
  ctx->sync();
  ctx->collect_timings();
  if (dbg) {
    fprintf(stderr, "[gamma sm batch] prepare %.2f ms (", ms(t0, t1));
    for (size_t i = 0; i < nq; i++) fprintf(stderr, "%s%.2f", i ? " " : "", tprep[i]);
    fprintf(stderr, "), enqueue %.2f, wait %.2f, collect %.2f ms\n", ms(t1, t2), ms(t2, t3), ms(t3, now()));
  }
}

}  // namespace gamma_impl

using namespace gamma_impl;

extern "C" gamma_status gamma_pattern_plan(const gamma_pattern *p, gamma_plan_info *out) {
  return guarded([&] {
    GAMMA_REQUIRE(p && out, GAMMA_E_INVAL, "gamma_pattern_plan: NULL argument");
    SmPlan P;
    plan_pattern(p, P);
    std::memset(out, 0, sizeof(*out));
    out->nv = P.nv;
    out->aut = P.aut;
    for (uint32_t i = 0; i < P.nv; i++) {
      out->order[i] = P.order[i];
      out->backward_mask[i] = P.bmask[i];
      out->less_mask[i] = P.ltmask[i];
      out->greater_mask[i] = P.gtmask[i];
    }
  });
}

extern "C" gamma_status gamma_match_batch(gamma_graph *g, uint32_t n, const gamma_pattern *ps, uint64_t *counts,
                                          uint64_t *mappings) {
  return guarded([&] {
    GAMMA_REQUIRE(g && (n == 0 || (ps && counts)), GAMMA_E_INVAL, "gamma_match_batch: NULL argument");
    GAMMA_REQUIRE(2 * g->m < (1ull << 32), GAMMA_E_UNSUPPORTED,
                  "gamma_match_batch: graphs with 2m >= 2^32 unsupported");
    std::vector<SmPlan> Ps(n);
    for (uint32_t i = 0; i < n; i++) plan_pattern(ps + i, Ps[i]);
    gamma_ctx *c = g->ctx;
    GAMMA_CUDA(cudaSetDevice(c->device));
    c->reset_stats();
    std::vector<uint64_t> r;
    const auto tb = std::chrono::steady_clock::now();
    match_batch(g, Ps, r);
    if (getenv("GAMMA_DEBUG"))
      fprintf(stderr, "[gamma sm batch] call %.2f ms (incl. table release)\n",
              std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - tb).count());
    if (c->desc.world > 1 && c->desc.allreduce_sum_u64 && n) {
      gamma_status st = c->desc.allreduce_sum_u64(r.data(), n, c->desc.coll_user);
      GAMMA_REQUIRE(st == GAMMA_OK, st, "allreduce_sum_u64 callback failed");
    }
    for (uint32_t i = 0; i < n; i++) {
      counts[i] = r[i];
      if (mappings) {
        uint64_t mp;
        GAMMA_REQUIRE(!__builtin_mul_overflow(r[i], Ps[i].aut, &mp), GAMMA_E_OVERFLOW, "mappings overflow uint64");
        mappings[i] = mp;
      }
    }
  });
}

extern "C" gamma_status gamma_match(gamma_graph *g, const gamma_pattern *p, uint64_t *count,
                                    uint64_t *mappings) {
  return guarded([&] {
    GAMMA_REQUIRE(g && p && count, GAMMA_E_INVAL, "gamma_match: NULL argument");
    // the extension kernels carry symmetric-CSR offsets (< 2m) as u32
    GAMMA_REQUIRE(2 * g->m < (1ull << 32), GAMMA_E_UNSUPPORTED, "gamma_match: graphs with 2m >= 2^32 unsupported");
    SmPlan P;
    plan_pattern(p, P);
    gamma_ctx *c = g->ctx;
    GAMMA_CUDA(cudaSetDevice(c->device));
    c->reset_stats();
    uint64_t r = match_count(g, P);
    if (c->desc.world > 1 && c->desc.allreduce_sum_u64) {
      gamma_status st = c->desc.allreduce_sum_u64(&r, 1, c->desc.coll_user);
      GAMMA_REQUIRE(st == GAMMA_OK, st, "allreduce_sum_u64 callback failed");
    }
    *count = r;
    if (mappings) {
      uint64_t mp;
      GAMMA_REQUIRE(!__builtin_mul_overflow(r, P.aut, &mp), GAMMA_E_OVERFLOW, "mappings overflow uint64");
      *mappings = mp;
    }
  });
}
