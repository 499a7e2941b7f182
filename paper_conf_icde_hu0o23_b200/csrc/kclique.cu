// kclique.cu -- k-clique counting as embedding-table (ET) vertex extension, A2-A8.
//
// Method: vertex extension Ext_v(M) = {M + u | u in N_v(M)} (Def. 3.1,
// L127-139) with early pruning "we only consider the common neighbours" (L146);
// embeddings sharing a prefix are grouped and one warp extends one group against
// the pre-intersected list L_m (Opt 2, L269-278); each warp writes into its own
// memory block taken from a pool and resolves intra-warp slots with a warp prefix
// scan (Opt 1, L263-267); the last extension is counted, not stored (L299).
//
// B200 design:
//  * Degree-ordered DAG.  A group at depth d is the candidate run
//    C(P) = N+(p1) ∩ ... ∩ N+(pd) of a d-vertex prefix P, sorted ascending; every
//    element c of the run is one (d+1)-vertex embedding and its own candidate run
//    is C(P) ∩ N+(c).  So L_m of Opt 2 *is* the parent run: it is staged once per
//    group in shared memory and probed with a branch-free binary search.
//  * Flattened children: a window of up to 32 children is held one per lane (list
//    offset + length in registers, exclusive-scanned with shuffles); the warp then
//    streams the concatenation of their DAG lists 32 elements per step, each lane
//    finding its child by a 5-step shuffle search.  Lanes stay busy even when the
//    lists are short (mean d+ ~ 8), and every step issues one coalesced gather.
//  * Survivors are compacted in order with __ballot_sync/__popc into a per-warp
//    shared staging buffer (child-major, so each child's run is contiguous); per-
//    child hit counts come from ballot & segment masks, in registers.
//  * ET level = column-first vid[] (4 B per embedding) + group table {beg,len}
//    (8 B per kept group).  The parent pointer of the prefix tree is implicit in the
//    group.
//  * Opt 1: per-warp 16 KB vid blocks / 4 KB group blocks, one atomic per block.
//  * Fused tail (DFS hybrid): at depth k-3 the children's runs never leave shared
//    memory -- they are counted in place, so the largest ET level is never written.
//  * A8: DFS over (depth, group range), level buffers grow geometrically up to an
//    equal share of the HBM budget; a range that still overflows is split in halves.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>
#include <cub/device/device_select.cuh>

#include <algorithm>
#include <vector>

#include "device_common.cuh"
#include "internal.cuh"

namespace gamma_impl {

namespace {

constexpr int kWarps = 8;
constexpr int kThreads = kWarps * 32;
constexpr uint32_t kRunCap = 512;    // staged run capacity per warp (u32)
constexpr uint32_t kOutCap = 1024;   // staged output capacity per warp (u32), >= kRunCap
constexpr uint32_t kBlkV = 4096;     // Opt 1 vid block per warp (16 KB)
constexpr uint32_t kBlkG = 512;      // Opt 1 group block per warp (4 KB)

enum { MODE_EXTEND = 0, MODE_COUNT = 1, MODE_FUSED = 2 };

struct KclArgs {
  const uint64_t *dag_ptr;
  const uint32_t *dag_col;
  // input groups: depth 1 (roots) or a level table
  const uint32_t *roots;
  const uint2 *grp_in;        // {beg, len}
  const uint32_t *groot_in;   // per-root mode: root index per group
  const uint32_t *vid_in;
  uint64_t g_begin, g_end;
  uint32_t need_group;        // skip groups with len < need_group
  uint32_t need_child;        // keep children whose own run has >= need_child entries
  // output level (extend; fused: long-run spill)
  uint32_t *vid_out;
  uint2 *grp_out;
  uint32_t *groot_out;
  uint64_t cap_v, cap_g;
  unsigned long long *ctrl;
  unsigned long long *per_root;
  uint32_t batch;
  uint32_t stage_cap;         // kRunCap (0: GAMMA_FLAG_DEBUG_NOSTAGE)
  uint32_t root_len_gt;       // depth 1: only roots with |N+(v)| > this (bitmap path took the rest)
  // Opt 1 ablation (GAMMA_FLAG_TWO_PASS: the count-then-write scheme Opt 1
  // replaces): pass 1 only counts each input group's output vids / groups into gcnt_v /
  // gcnt_g; pass 2 writes them at the exclusive-scanned offsets goff_v / goff_g
  // (indexed by gi - g_begin); 0 = Opt 1's single pass with warp memory blocks
  uint32_t two_pass;
  uint32_t *gcnt_v, *gcnt_g;
  const uint64_t *goff_v, *goff_g;
};

struct Counters {
  uint64_t acc = 0, in_entries = 0, elems = 0, out_entries = 0;
};

__device__ __forceinline__ uint32_t excl_scan(uint32_t x, int lane, uint32_t &total) {
  uint32_t s = x;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(0xffffffffu, s, o);
    if (lane >= o) s += y;
  }
  total = __shfl_sync(0xffffffffu, s, 31);
  return s - x;
}

// Lanes [lo, hi) of a 32-lane tile, clamped.
__device__ __forceinline__ uint32_t seg_mask(int64_t lo, int64_t hi) {
  lo = lo < 0 ? 0 : (lo > 32 ? 32 : lo);
  hi = hi < 0 ? 0 : (hi > 32 ? 32 : hi);
  if (hi <= lo) return 0u;
  uint32_t up = hi >= 32 ? 0xffffffffu : ((1u << hi) - 1u);
  uint32_t dn = lo >= 32 ? 0xffffffffu : ((1u << lo) - 1u);
  return up & ~dn;
}

// The window core: children = one per active lane (list offset `beg`, length `dl`,
// exclusive offsets `o`, total T).  Streams the concatenated lists, probes every
// element against the staged run, and (WRITE) compacts hits into `out` child-major
// and accumulates per-child hit counts in `cnt`.  Returns the number of hits.
template <bool WRITE>
__device__ __forceinline__ uint32_t window_probe(const KclArgs &a, const uint32_t *__restrict__ run,
                                                 uint32_t len, uint32_t rmin, uint32_t rmax, uint32_t beg,
                                                 uint32_t dl, uint32_t o, uint32_t T, int lane,
                                                 uint32_t *out, uint32_t &cnt) {
  uint32_t found = 0;
  for (uint32_t t0 = 0; t0 < T; t0 += 32) {
    const uint32_t t = t0 + lane;
    const bool valid = t < T;
    // j = max{i : o_i <= t} over the window lanes (o is non-decreasing)
    int j = 0;
#pragma unroll
    for (int step = 16; step > 0; step >>= 1) {
      uint32_t oc = __shfl_sync(0xffffffffu, o, (j + step) & 31);
      if (j + step < 32 && oc <= t) j += step;
    }
    const uint32_t bj = __shfl_sync(0xffffffffu, beg, j);
    const uint32_t oj = __shfl_sync(0xffffffffu, o, j);
    const uint32_t y = valid ? __ldg(a.dag_col + bj + (t - oj)) : 0xffffffffu;
    bool hit = false;
    if (valid && y >= rmin && y <= rmax) hit = sorted_contains(run, len, y);
    const uint32_t bal = __ballot_sync(0xffffffffu, hit);
    if (WRITE) {
      if (hit) out[found + __popc(bal & lanemask_lt())] = y;
      cnt += __popc(bal & seg_mask((int64_t)o - t0, (int64_t)o + dl - t0));
    }
    found += __popc(bal);
  }
  return found;
}

// Load the window's children (lane i: child w0+i of the run) and their DAG lists.
__device__ __forceinline__ void load_children(const KclArgs &a, const uint32_t *run, uint32_t len,
                                              uint32_t w0, int lane, uint32_t need, uint32_t &beg,
                                              uint32_t &dl, uint32_t &raw) {
  const uint32_t i = w0 + lane;
  beg = 0;
  dl = 0;
  raw = 0;
  if (i < len) {
    const uint32_t c = run[i];
    const uint64_t b0 = a.dag_ptr[c];
    raw = (uint32_t)(a.dag_ptr[c + 1] - b0);
    beg = (uint32_t)b0;
    dl = raw >= need ? raw : 0;
  }
}

// Count k-cliques under one staged group at the last depth: sum over children c
// of |run ∩ N+(c)|.
__device__ __forceinline__ uint64_t count_staged(const KclArgs &a, const uint32_t *run, uint32_t len,
                                                 int lane, Counters &ct) {
  const uint32_t rmin = run[0], rmax = run[len - 1];
  uint64_t total = 0;
  for (uint32_t w0 = 0; w0 < len; w0 += 32) {
    uint32_t beg, dl, raw, T, dummy = 0;
    load_children(a, run, len, w0, lane, 1, beg, dl, raw);
    ct.elems += raw;
    const uint32_t o = excl_scan(dl, lane, T);
    total += window_probe<false>(a, run, len, rmin, rmax, beg, dl, o, T, lane, nullptr, dummy);
  }
  return total;
}

// Long runs (len > stage capacity): child by child, probing the run in global
// memory; EXTEND/FUSED write each kept child's run with a direct pool reservation.
template <int MODE, bool PER_ROOT>
__device__ bool process_unstaged(const KclArgs &a, const uint32_t *run, uint32_t len, uint32_t root_idx,
                                 int lane, Counters &ct, WarpBlock &wg, uint64_t &gacc, uint64_t gi,
                                 uint32_t &tp_v, uint32_t &tp_g) {
  const BlockPool pv{&a.ctrl[CTRL_VCUR], &a.ctrl[CTRL_OVF], a.cap_v, kBlkV};
  const BlockPool pg{&a.ctrl[CTRL_GCUR], &a.ctrl[CTRL_OVF], a.cap_g, kBlkG};
  const uint32_t rmin = run[0], rmax = run[len - 1];
  const uint32_t need = (MODE == MODE_COUNT) ? 1u : a.need_child;
  for (uint32_t i = 0; i < len; i++) {
    const uint32_t c = run[i];
    const uint64_t lb = a.dag_ptr[c];
    const uint32_t dl = (uint32_t)(a.dag_ptr[c + 1] - lb);
    ct.elems += (lane == 0) ? dl : 0;
    if (dl < need) continue;
    const uint32_t *lst = a.dag_col + lb;
    const uint32_t ub = min(dl, len);
    uint64_t pos = 0;
    const bool tp_write = MODE == MODE_EXTEND && a.two_pass == 2;
    if (tp_write) pos = a.goff_v[gi - a.g_begin] + tp_v;
    else if (MODE != MODE_COUNT && !(MODE == MODE_EXTEND && a.two_pass == 1) && !pool_reserve(pv, ub, lane, pos))
      return false;
    // write pass of the two-pass ablation: a child's run is written only once its size
    // says it is kept (its space was counted for kept children only), i.e. counted again
    const int rounds = tp_write ? 2 : 1;
    uint32_t found = 0;
    for (int rd = 0; rd < rounds; rd++) {
      const bool write = MODE != MODE_COUNT && !(MODE == MODE_EXTEND && a.two_pass == 1) && (!tp_write || rd == 1);
      if (rd == 1 && found < a.need_child) break;
      found = 0;
      for (uint32_t j = 0; j < dl; j += 32) {
        const uint32_t y = (j + lane < dl) ? __ldg(lst + j + lane) : 0xffffffffu;
        bool hit = false;
        if (y >= rmin && y <= rmax) hit = sorted_contains(run, len, y);
        const uint32_t bal = __ballot_sync(0xffffffffu, hit);
        if (write && hit) a.vid_out[pos + found + __popc(bal & lanemask_lt())] = y;
        found += __popc(bal);
        if (__shfl_sync(0xffffffffu, y, 31) > rmax) break;
      }
    }
    if (MODE == MODE_COUNT) {
      gacc += found;
      continue;
    }
    if (found < a.need_child) continue;
    uint64_t gpos;
    if (MODE == MODE_EXTEND && a.two_pass == 1) {
      tp_v += found;
      tp_g += 1;
      ct.out_entries += (lane == 0) ? found : 0;
      continue;
    }
    if (tp_write) {
      gpos = a.goff_g[gi - a.g_begin] + tp_g;
      tp_v += found;
      tp_g += 1;
    } else if (!wb_reserve(wg, pg, 1, lane, gpos)) {
      return false;
    }
    if (lane == 0) {
      a.grp_out[gpos] = make_uint2((uint32_t)pos, found);
      if (PER_ROOT) a.groot_out[gpos] = root_idx;
    }
    ct.out_entries += (lane == 0) ? found : 0;
  }
  return true;
}

template <int MODE, bool ROOT, bool PER_ROOT>
__global__ void __launch_bounds__(kThreads) kcl_kernel(KclArgs a) {
  extern __shared__ uint32_t smem[];
  const int lane = threadIdx.x & 31;
  const int wid = threadIdx.x >> 5;
  uint32_t *srun = smem + wid * kRunCap;
  uint32_t *sout = smem + kWarps * kRunCap + wid * kOutCap;   // unused in MODE_COUNT
  const BlockPool pv{&a.ctrl[CTRL_VCUR], &a.ctrl[CTRL_OVF], a.cap_v, kBlkV};
  const BlockPool pg{&a.ctrl[CTRL_GCUR], &a.ctrl[CTRL_OVF], a.cap_g, kBlkG};
  WarpBlock wv, wg;
  Counters ct;
  const uint64_t ng = a.g_end - a.g_begin;
  bool stop = false;

  while (!stop) {
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(&a.ctrl[CTRL_WORK], (unsigned long long)a.batch);
    base = __shfl_sync(0xffffffffu, base, 0);
    if (base >= ng) break;
    if (MODE != MODE_COUNT && *(volatile unsigned long long *)&a.ctrl[CTRL_OVF]) break;
    const uint64_t bend = min((uint64_t)base + a.batch, ng);
    for (uint64_t gi = a.g_begin + base; gi < a.g_begin + bend && !stop; gi++) {
      // ---- A2/A3: the group's run C(P) ----
      const uint32_t *run;
      uint32_t len;
      uint32_t root_idx = 0;
      if (ROOT) {
        const uint32_t v = a.roots[gi];
        const uint64_t b0 = a.dag_ptr[v];
        len = (uint32_t)(a.dag_ptr[v + 1] - b0);
        run = a.dag_col + b0;
        root_idx = (uint32_t)gi;
      } else {
        const uint2 gd = a.grp_in[gi];
        len = gd.y;
        run = a.vid_in + gd.x;
        if (PER_ROOT) root_idx = a.groot_in[gi];
      }
      if (len < a.need_group || (ROOT && len <= a.root_len_gt)) {
        if (MODE == MODE_EXTEND && a.two_pass == 1 && lane == 0) a.gcnt_v[gi - a.g_begin] = a.gcnt_g[gi - a.g_begin] = 0;
        continue;
      }
      ct.in_entries += (lane == 0) ? len : 0;
      uint64_t gacc = 0;
      uint32_t tp_v = 0, tp_g = 0;   // two-pass ablation: this group's output so far
      if (len > a.stage_cap) {
        if (!process_unstaged<MODE, PER_ROOT>(a, run, len, root_idx, lane, ct, wg, gacc, gi, tp_v, tp_g)) stop = true;
      } else {
        for (uint32_t i = lane; i < len; i += 32) srun[i] = run[i];
        __syncwarp();
        if (MODE == MODE_COUNT) {
          gacc = count_staged(a, srun, len, lane, ct);
        } else {
          // ---- A4-A6: windows of children, outputs staged child-major ----
          const uint32_t rmin = srun[0], rmax = srun[len - 1];
          for (uint32_t w0 = 0; w0 < len && !stop;) {
            uint32_t beg, dl, raw;
            load_children(a, srun, len, w0, lane, a.need_child, beg, dl, raw);
            // window = longest prefix of lanes whose output upper bounds fit kOutCap
            uint32_t ub = min(dl, len), ubt;
            const uint32_t ubx = excl_scan(ub, lane, ubt);
            const bool fits = (w0 + lane < len) && (ubx + ub <= kOutCap);
            const uint32_t nwin = __popc(__ballot_sync(0xffffffffu, fits));   // >= 1
            const bool active = lane < (int)nwin;
            if (!active) dl = 0;
            ct.elems += active ? raw : 0;
            uint32_t T;
            const uint32_t o = excl_scan(dl, lane, T);
            uint32_t cnt = 0;
            const uint32_t found = window_probe<true>(a, srun, len, rmin, rmax, beg, dl, o, T, lane, sout, cnt);
            __syncwarp();
            uint32_t ctot;
            const uint32_t s = excl_scan(cnt, lane, ctot);   // child i's run = sout[s, s+cnt)
            const bool keep = active && cnt >= a.need_child;
            const uint32_t kbal = __ballot_sync(0xffffffffu, keep);
            if (MODE == MODE_EXTEND) {
              if (kbal && a.two_pass == 1) {   // count pass: sizes only
                tp_v += found;
                tp_g += __popc(kbal);
                ct.out_entries += (lane == 0) ? found : 0;
              } else if (kbal) {
                uint64_t pos = 0, gpos = 0;
                if (a.two_pass == 2) {   // write pass: exact offsets from the count pass
                  pos = a.goff_v[gi - a.g_begin] + tp_v;
                  gpos = a.goff_g[gi - a.g_begin] + tp_g;
                  tp_v += found;
                  tp_g += __popc(kbal);
                } else {
                wb_retire_tail(wg, __popc(kbal), lane, [&](uint64_t s) { a.grp_out[s] = make_uint2(0, 0); });
                if (!wb_reserve(wv, pv, found, lane, pos) || !wb_reserve(wg, pg, __popc(kbal), lane, gpos)) {
                  stop = true;
                  break;
                }
                }
                for (uint32_t t = lane; t < found; t += 32) a.vid_out[pos + t] = sout[t];
                if (keep) {
                  const uint64_t gp = gpos + __popc(kbal & lanemask_lt());
                  a.grp_out[gp] = make_uint2((uint32_t)(pos + s), cnt);
                  if (PER_ROOT) a.groot_out[gp] = root_idx;
                }
                ct.out_entries += (lane == 0) ? found : 0;
              }
            } else {   // MODE_FUSED: count each kept child's run in place
              uint32_t rem = kbal;
              while (rem) {
                const int i = __ffs(rem) - 1;
                rem &= rem - 1;
                const uint32_t si = __shfl_sync(0xffffffffu, s, i);
                const uint32_t ci = __shfl_sync(0xffffffffu, cnt, i);
                gacc += count_staged(a, sout + si, ci, lane, ct);
              }
            }
            __syncwarp();
            w0 += nwin;
          }
        }
        __syncwarp();
      }
      ct.acc += gacc;
      if (PER_ROOT && lane == 0 && gacc) atomicAdd(&a.per_root[root_idx], (unsigned long long)gacc);
      if (MODE == MODE_EXTEND && a.two_pass == 1 && lane == 0) {
        a.gcnt_v[gi - a.g_begin] = tp_v;
        a.gcnt_g[gi - a.g_begin] = tp_g;
      }
    }
  }
  // unused group slots of this warp's last block become empty groups
  if (MODE != MODE_COUNT)
    for (uint64_t s = wg.b + lane; s < wg.e; s += 32) a.grp_out[s] = make_uint2(0, 0);
  // counters: lane-partial sums -> one atomic per warp
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    ct.elems += __shfl_down_sync(0xffffffffu, ct.elems, off);
    ct.in_entries += __shfl_down_sync(0xffffffffu, ct.in_entries, off);
    ct.out_entries += __shfl_down_sync(0xffffffffu, ct.out_entries, off);
  }
  if (lane == 0) {
    if (ct.acc) atomicAdd(&a.ctrl[CTRL_COUNT], (unsigned long long)ct.acc);
    atomicAdd(&a.ctrl[CTRL_AUX0], (unsigned long long)ct.in_entries);
    atomicAdd(&a.ctrl[CTRL_ELEMS], (unsigned long long)ct.elems);
    atomicAdd(&a.ctrl[CTRL_ENTRIES], (unsigned long long)ct.out_entries);
  }
}

// ---- A2: roots = vertices with d+(v) >= k-1, heavy first, snake-partitioned ----
struct RootNeed {
  const uint64_t *dag_ptr;
  uint32_t need;
  __device__ __forceinline__ bool operator()(const uint32_t &v) const {
    return dag_ptr[v + 1] - dag_ptr[v] >= need;
  }
};

__global__ void iota_kernel(uint32_t *p, uint32_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x)
    p[i] = (uint32_t)i;
}

__global__ void root_cost_kernel(const uint64_t *dag_ptr, const uint32_t *roots, uint64_t nr,
                                 uint64_t *cost) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nr;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t v = roots[i];
    const uint64_t d = dag_ptr[v + 1] - dag_ptr[v];
    cost[i] = d * d;
  }
}

// Snake (boustrophedon) assignment of cost-sorted roots to ranks: an LPT-style
// balance that needs no coordination.
__global__ void rank_flag_kernel(uint64_t nr, uint32_t rank, uint32_t world, uint8_t *flag) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nr;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t r = i % (2ull * world);
    flag[i] = (r == rank || r == 2ull * world - 1 - rank) ? 1 : 0;
  }
}

__global__ void degree_count_kernel(const uint64_t *dag_ptr, const uint32_t *roots, uint64_t nr,
                                    uint32_t k, unsigned long long *out) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nr;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t v = roots[i];
    out[i] = (k == 1) ? 1ull : (unsigned long long)(dag_ptr[v + 1] - dag_ptr[v]);
  }
}

inline unsigned grid1d(uint64_t n, int threads = 256) {
  uint64_t b = (n + threads - 1) / threads;
  if (b == 0) b = 1;
  return (unsigned)std::min<uint64_t>(b, 148u * 32u);
}

constexpr size_t kcl_smem(int mode) {
  return (size_t)kWarps * (kRunCap + (mode == MODE_COUNT ? 0 : kOutCap)) * sizeof(uint32_t);
}

template <int MODE, bool ROOT, bool PER_ROOT>
void set_smem_attr() {
  GAMMA_CUDA(cudaFuncSetAttribute(kcl_kernel<MODE, ROOT, PER_ROOT>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  (int)kcl_smem(MODE)));
}

template <int MODE>
void set_mode_attrs() {
  set_smem_attr<MODE, false, false>();
  set_smem_attr<MODE, false, true>();
  set_smem_attr<MODE, true, false>();
  set_smem_attr<MODE, true, true>();
}

struct Level {
  DevBuf<uint32_t> vid;
  DevBuf<uint2> grp;
  DevBuf<uint32_t> groot;
  uint64_t cap_v = 0, cap_g = 0;
};

struct KclRun {
  gamma_graph *g;
  gamma_ctx *ctx;
  uint32_t k;
  bool per_root;
  bool fuse;
  const uint32_t *roots;
  uint64_t nroots;
  unsigned long long *per_root_out;
  uint32_t root_len_gt = 0;
  std::vector<Level> levels;   // levels[d] holds groups at depth d (d >= 2)
  uint64_t level_share;        // bytes allowed per level table
  uint64_t total = 0;
  int grid[3] = {0, 0, 0};

  uint64_t bytes_per_slot() const { return 4 + (per_root ? 12 : 8) / 2; }   // vid + cap_g = cap_v/2

  // Grow level d to hold want_v vid slots, within its share of the budget.
  bool grow_level(uint32_t d, uint64_t want_v) {
    Level &L = levels[d];
    uint64_t cv = std::max<uint64_t>(want_v, 1ull << 16);
    cv = std::min<uint64_t>(cv, level_share / bytes_per_slot());
    cv = std::min<uint64_t>(cv, 0xFFFFFFFFull - kBlkV);   // group beg is u32
    if (cv <= L.cap_v) return false;
    const uint64_t cg = cv / 2 + kBlkG;
    L.vid.reset();
    L.grp.reset();
    L.groot.reset();
    L.vid = DevBuf<uint32_t>(ctx, cv);
    L.grp = DevBuf<uint2>(ctx, cg);
    if (per_root) L.groot = DevBuf<uint32_t>(ctx, cg);
    L.cap_v = cv;
    L.cap_g = cg;
    return true;
  }

  KclArgs args_for(uint32_t d, uint64_t g0, uint64_t g1) const {
    KclArgs a{};
    a.dag_ptr = g->dag_ptr;
    a.dag_col = g->dag_col;
    a.ctrl = (unsigned long long *)ctx->ctrl;
    a.per_root = per_root_out;
    a.stage_cap = (ctx->desc.flags & GAMMA_FLAG_DEBUG_NOSTAGE) ? 0u : kRunCap;
    a.root_len_gt = root_len_gt;
    a.g_begin = g0;
    a.g_end = g1;
    if (d == 1) {
      a.roots = roots;
      a.batch = 2;
    } else {
      const Level &L = levels[d];
      a.grp_in = L.grp.p;
      a.groot_in = L.groot.p;
      a.vid_in = L.vid.p;
      a.batch = 16;
    }
    a.need_group = k - d;        // a depth-d group needs k-d more vertices
    a.need_child = k - d - 1;    // a child's run is a depth-(d+1) group
    return a;
  }

  void set_output(KclArgs &a, uint32_t nd) {
    Level &L = levels[nd];
    a.vid_out = L.vid.p;
    a.grp_out = L.grp.p;
    a.groot_out = L.groot.p;
    a.cap_v = L.cap_v;
    a.cap_g = L.cap_g;
  }

  template <int MODE, bool ROOT>
  void launch_t(const KclArgs &a, int grid_) {
    const int kc = MODE == MODE_EXTEND ? KC_EXTEND : (MODE == MODE_COUNT ? KC_COUNT : KC_FUSED);
    const size_t smem = kcl_smem(MODE);
    ctx->launch(kc, [&] {
      if (per_root)
        kcl_kernel<MODE, ROOT, true><<<grid_, kThreads, smem, ctx->stream>>>(a);
      else
        kcl_kernel<MODE, ROOT, false><<<grid_, kThreads, smem, ctx->stream>>>(a);
    });
  }

  template <int MODE>
  void launch(const KclArgs &a, uint32_t d, uint64_t cap_v) {
    int gr = grid[MODE];
    if (MODE == MODE_EXTEND) {   // keep the Opt 1 block waste below half the level
      const uint64_t warps_ok = std::max<uint64_t>(1, cap_v / (2ull * kBlkV));
      gr = (int)std::max<uint64_t>(1, std::min<uint64_t>(gr, warps_ok / kWarps));
    }
    ctrl_reset(ctx);
    if (d == 1) launch_t<MODE, true>(a, gr);
    else launch_t<MODE, false>(a, gr);
    ctrl_fetch(ctx);
  }

  void account(int kc, uint32_t d, const uint64_t *h, bool wrote) {
    if (d == 1) ctx->stats.level_entries[2] += h[CTRL_AUX0];
    ctx->stats.list_elems += h[CTRL_ELEMS];
    ctx->stats.alg_bytes[kc] += 12 * h[CTRL_AUX0] + 4 * h[CTRL_ELEMS] + (wrote ? 8 * h[CTRL_ENTRIES] : 0);
  }

  void add_count(uint64_t c) {
    total = checked_add(total, c);
    ctx->stats.level_entries[k] = checked_add(ctx->stats.level_entries[k], c);
  }

  // DFS over (depth, group range); BFS inside the range.
  void process(uint32_t d, uint64_t g0, uint64_t g1) {
    if (g0 >= g1) return;
    if (d == k - 2) {   // last extension: count, do not store
      KclArgs a = args_for(d, g0, g1);
      a.need_child = 1;
      launch<MODE_COUNT>(a, d, 0);
      const uint64_t *h = ctx->ctrl_host;
      add_count(h[CTRL_COUNT]);
      account(KC_COUNT, d, h, false);
      return;
    }
    const bool fused = fuse && d == k - 3;
    const uint32_t nd = d + 1;
    if (!fused && (ctx->desc.flags & GAMMA_FLAG_TWO_PASS)) {
      process_two_pass(d, g0, g1);
      return;
    }
    for (;;) {
      Level &L = levels[nd];
      if (L.cap_v == 0)
        grow_level(nd, fused ? (1ull << 18)
                             : std::max<uint64_t>(1ull << 24, 4ull * kBlkV * kWarps * (uint64_t)grid[MODE_EXTEND]));
      KclArgs a = args_for(d, g0, g1);
      set_output(a, nd);
      if (fused) launch<MODE_FUSED>(a, d, L.cap_v);
      else launch<MODE_EXTEND>(a, d, L.cap_v);
      const uint64_t *h = ctx->ctrl_host;
      if (!h[CTRL_OVF]) {
        const uint64_t cnt = h[CTRL_COUNT];
        const uint64_t ent = h[CTRL_ENTRIES];
        const uint64_t ng = std::min<uint64_t>(h[CTRL_GCUR], L.cap_g);
        account(fused ? KC_FUSED : KC_EXTEND, d, h, !fused || ent > 0);
        ctx->stats.chunks++;
        if (fused) add_count(cnt);
        else ctx->stats.level_entries[nd + 1] += ent;
        // fused: only long-run (unstaged) children were written; count them now
        process(nd, 0, ng);
        return;
      }
      ctx->stats.retries++;
      if (grow_level(nd, std::max<uint64_t>(h[CTRL_VCUR], L.cap_v) * 4)) continue;
      if (!fused && (ctx->desc.flags & GAMMA_FLAG_SPILL) && ctx->desc.host_spill_bytes) {
        process_spill(d, g0, g1);
        return;
      }
      GAMMA_REQUIRE(g1 - g0 > 1, GAMMA_E_NOMEM,
                    "HBM budget too small for the children of a single embedding group");
      const uint64_t mid = g0 + (g1 - g0) / 2;
      process(d, g0, mid);
      process(d, mid, g1);
      return;
    }
  }

  // Opt 1 ablation (GAMMA_FLAG_TWO_PASS): the count-then-write extension that Opt 1's
  // warp memory blocks replace ("two-pass ... doubles the extension").
  // Pass 1 counts every input group's output, an exclusive scan gives exact offsets,
  // pass 2 recomputes the intersections and writes; no over-allocation, twice the work.
  void process_two_pass(uint32_t d, uint64_t g0, uint64_t g1) {
    const uint32_t nd = d + 1;
    const uint64_t ng_in = g1 - g0;
    Level &L = levels[nd];
    if (L.cap_v == 0) grow_level(nd, std::max<uint64_t>(1ull << 24, 4ull * kBlkV * kWarps * (uint64_t)grid[MODE_EXTEND]));
    DevBuf<uint32_t> cv(ctx, ng_in + 1), cg(ctx, ng_in + 1);
    DevBuf<uint64_t> ov(ctx, ng_in + 1), og(ctx, ng_in + 1);
    GAMMA_CUDA(cudaMemsetAsync(cv.p + ng_in, 0, 4, ctx->stream));
    GAMMA_CUDA(cudaMemsetAsync(cg.p + ng_in, 0, 4, ctx->stream));
    KclArgs a = args_for(d, g0, g1);
    set_output(a, nd);
    a.two_pass = 1;
    a.gcnt_v = cv.p;
    a.gcnt_g = cg.p;
    launch<MODE_EXTEND>(a, d, L.cap_v);
    account(KC_EXTEND, d, ctx->ctrl_host, true);
    size_t tmp = 0;
    GAMMA_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp, cv.p, ov.p, (int64_t)ng_in + 1, ctx->stream));
    {
      DevBuf<uint8_t> t(ctx, tmp);
      ctx->launch(KC_MISC, [&] {
        GAMMA_CUDA(cub::DeviceScan::ExclusiveSum(t.p, tmp, cv.p, ov.p, (int64_t)ng_in + 1, ctx->stream));
      });
      ctx->launch(KC_MISC, [&] {
        GAMMA_CUDA(cub::DeviceScan::ExclusiveSum(t.p, tmp, cg.p, og.p, (int64_t)ng_in + 1, ctx->stream));
      });
    }
    uint64_t tot[2];
    GAMMA_CUDA(cudaMemcpyAsync(&tot[0], ov.p + ng_in, 8, cudaMemcpyDeviceToHost, ctx->stream));
    GAMMA_CUDA(cudaMemcpyAsync(&tot[1], og.p + ng_in, 8, cudaMemcpyDeviceToHost, ctx->stream));
    ctx->sync();
    // exact sizes: grow once, or split the range when even the largest level share cannot hold them
    if (tot[0] > L.cap_v || tot[1] > L.cap_g) grow_level(nd, std::max<uint64_t>(tot[0], 2 * tot[1]));
    if (tot[0] > L.cap_v || tot[1] > L.cap_g) {
      GAMMA_REQUIRE(ng_in > 1, GAMMA_E_NOMEM, "HBM budget too small for the children of a single embedding group");
      ctx->stats.retries++;
      const uint64_t mid = g0 + ng_in / 2;
      process_two_pass(d, g0, mid);
      process_two_pass(d, mid, g1);
      return;
    }
    a.two_pass = 2;
    a.goff_v = ov.p;
    a.goff_g = og.p;
    set_output(a, nd);
    launch<MODE_EXTEND>(a, d, L.cap_v);
    ctx->stats.chunks++;
    ctx->stats.level_entries[nd + 1] += ctx->ctrl_host[CTRL_ENTRIES];
    process(nd, 0, tot[1]);
  }

  // GAMMA_FLAG_SPILL: BFS with a host-resident next level (the ET "should
  // be resident in host memory ... we keep a buffer on the device to write extension
  // results ... and flush them to host memory").  Level d+1 is produced in slabs that
  // fit the device buffer and parked in pinned host memory; the slabs are then streamed
  // back one at a time for the next extension.  Two device buffers alternate (the
  // level's own and a spare of the same size) and every copy runs on the context's copy
  // stream, fenced by events: the D2H of slab i overlaps the extension writing slab
  // i + 1, and the H2D of slab i + 1 overlaps the processing of slab i.
  struct SpillBufs {
    Level spare;
    cudaEvent_t free_ev[2] = {nullptr, nullptr};   // buffer b may be overwritten (copy done / use done)
    cudaEvent_t ready_ev[2] = {nullptr, nullptr};  // buffer b holds its data (produced / copied in)
    ~SpillBufs() {
      for (int i = 0; i < 2; i++) {
        if (free_ev[i]) cudaEventDestroy(free_ev[i]);
        if (ready_ev[i]) cudaEventDestroy(ready_ev[i]);
      }
    }
  };

  void process_spill(uint32_t d, uint64_t g0, uint64_t g1) {
    const uint32_t nd = d + 1;
    struct Slab { size_t off; uint64_t nv, ng; };
    std::vector<Slab> slabs;
    const size_t top0 = ctx->spill_top;
    if (ctx->spill_host == nullptr) {
      ctx->spill_cap = ctx->desc.host_spill_bytes;
      GAMMA_CUDA(cudaMallocHost(&ctx->spill_host, ctx->spill_cap));
    }
    cudaStream_t cs = ctx->copy_stream_get();
    SpillBufs sb;
    for (int i = 0; i < 2; i++) {
      GAMMA_CUDA(cudaEventCreateWithFlags(&sb.free_ev[i], cudaEventDisableTiming));
      GAMMA_CUDA(cudaEventCreateWithFlags(&sb.ready_ev[i], cudaEventDisableTiming));
    }
    Level *buf[2] = {&levels[nd], &sb.spare};
    {   // the spare has the level's capacity
      Level &S = sb.spare;
      S.vid = DevBuf<uint32_t>(ctx, buf[0]->cap_v);
      S.grp = DevBuf<uint2>(ctx, buf[0]->cap_g);
      if (per_root) S.groot = DevBuf<uint32_t>(ctx, buf[0]->cap_g);
      S.cap_v = buf[0]->cap_v;
      S.cap_g = buf[0]->cap_g;
    }
    const auto slab_bytes = [&](const Slab &s) { return s.nv * 4 + s.ng * 8 + (per_root ? s.ng * 4 : 0); };
    // ---- produce: extension into buffer cur, D2H of the previous slab overlapping it ----
    int cur = 0;
    bool pending[2] = {false, false};
    std::vector<std::pair<uint64_t, uint64_t>> todo{{g0, g1}};
    while (!todo.empty()) {
      const auto r = todo.back();
      todo.pop_back();
      Level &L = *buf[cur];
      if (pending[cur]) GAMMA_CUDA(cudaStreamWaitEvent(ctx->stream, sb.free_ev[cur], 0));   // its D2H is done
      if (cur) std::swap(levels[nd], L);   // the kernels write levels[nd]
      KclArgs a = args_for(d, r.first, r.second);
      set_output(a, nd);
      launch<MODE_EXTEND>(a, d, levels[nd].cap_v);
      if (cur) std::swap(levels[nd], L);
      const uint64_t *h = ctx->ctrl_host;
      if (h[CTRL_OVF]) {
        ctx->stats.retries++;
        GAMMA_REQUIRE(r.second - r.first > 1, GAMMA_E_NOMEM,
                      "HBM budget too small for the children of a single embedding group");
        const uint64_t mid = r.first + (r.second - r.first) / 2;
        todo.push_back({mid, r.second});
        todo.push_back({r.first, mid});
        continue;
      }
      account(KC_EXTEND, d, h, true);
      ctx->stats.chunks++;
      ctx->stats.level_entries[nd + 1] += h[CTRL_ENTRIES];
      Slab s{0, std::min<uint64_t>(h[CTRL_VCUR], L.cap_v), std::min<uint64_t>(h[CTRL_GCUR], L.cap_g)};
      const size_t bytes = slab_bytes(s);
      GAMMA_REQUIRE(ctx->spill_top + bytes <= ctx->spill_cap, GAMMA_E_NOMEM,
                    "host spill budget exhausted (raise host_spill_bytes)");
      s.off = ctx->spill_top;
      uint8_t *dst = ctx->spill_host + s.off;
      GAMMA_CUDA(cudaEventRecord(sb.ready_ev[cur], ctx->stream));
      GAMMA_CUDA(cudaStreamWaitEvent(cs, sb.ready_ev[cur], 0));
      GAMMA_CUDA(cudaMemcpyAsync(dst, L.vid.p, s.nv * 4, cudaMemcpyDeviceToHost, cs));
      GAMMA_CUDA(cudaMemcpyAsync(dst + s.nv * 4, L.grp.p, s.ng * 8, cudaMemcpyDeviceToHost, cs));
      if (per_root)
        GAMMA_CUDA(cudaMemcpyAsync(dst + s.nv * 4 + s.ng * 8, L.groot.p, s.ng * 4, cudaMemcpyDeviceToHost, cs));
      GAMMA_CUDA(cudaEventRecord(sb.free_ev[cur], cs));
      pending[cur] = true;
      ctx->spill_top += bytes;
      ctx->stats.spilled_bytes += bytes;
      slabs.push_back(s);
      cur ^= 1;
    }
    GAMMA_CUDA(cudaStreamSynchronize(cs));   // every slab is on the host
    // ---- consume: slab i processed from one buffer while slab i + 1 is copied in ----
    const auto fetch = [&](size_t i, int b) {
      const Slab &s = slabs[i];
      Level &L = *buf[b];
      GAMMA_CUDA(cudaStreamWaitEvent(cs, sb.free_ev[b], 0));   // the previous user is done
      const uint8_t *src = ctx->spill_host + s.off;
      GAMMA_CUDA(cudaMemcpyAsync(L.vid.p, src, s.nv * 4, cudaMemcpyHostToDevice, cs));
      GAMMA_CUDA(cudaMemcpyAsync(L.grp.p, src + s.nv * 4, s.ng * 8, cudaMemcpyHostToDevice, cs));
      if (per_root)
        GAMMA_CUDA(cudaMemcpyAsync(L.groot.p, src + s.nv * 4 + s.ng * 8, s.ng * 4, cudaMemcpyHostToDevice, cs));
      GAMMA_CUDA(cudaEventRecord(sb.ready_ev[b], cs));
      ctx->stats.spilled_bytes += slab_bytes(s);
    };
    for (int b = 0; b < 2; b++) GAMMA_CUDA(cudaEventRecord(sb.free_ev[b], ctx->stream));
    if (!slabs.empty()) fetch(0, 0);
    for (size_t i = 0; i < slabs.size(); i++) {
      const int b = (int)(i & 1);
      if (i + 1 < slabs.size()) fetch(i + 1, b ^ 1);
      GAMMA_CUDA(cudaStreamWaitEvent(ctx->stream, sb.ready_ev[b], 0));
      if (b) std::swap(levels[nd], *buf[b]);   // process() reads levels[nd]
      process(nd, 0, slabs[i].ng);
      if (b) std::swap(levels[nd], *buf[b]);
      GAMMA_CUDA(cudaEventRecord(sb.free_ev[b], ctx->stream));
    }
    ctx->sync();
    GAMMA_CUDA(cudaStreamSynchronize(cs));
    ctx->spill_top = top0;
  }
};

void configure_kernels() {
  static bool done = false;   // function attributes persist for the process
  if (done) return;
  set_mode_attrs<MODE_EXTEND>();
  set_mode_attrs<MODE_COUNT>();
  set_mode_attrs<MODE_FUSED>();
  done = true;
}

}  // namespace

namespace {
__global__ void outdeg_key_kernel(const uint64_t *dag_ptr, uint32_t n, uint32_t *key, uint32_t *val) {
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
    key[v] = (uint32_t)(dag_ptr[v + 1] - dag_ptr[v]);
    val[v] = (uint32_t)v;
  }
}

// d+ histogram of a root list: block-private shared-memory bins (most roots fall in a
// handful of small-degree bins, so global atomics would serialise), flushed once
constexpr uint32_t kHistSmem = 4096;
__global__ void outdeg_hist_kernel(const uint64_t *dag_ptr, const uint32_t *roots, uint64_t nr, uint32_t nb,
                                   uint32_t *hist) {
  __shared__ uint32_t sh[kHistSmem];
  const bool local = nb <= kHistSmem;
  if (local)
    for (uint32_t b = threadIdx.x; b < nb; b += blockDim.x) sh[b] = 0;
  __syncthreads();
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nr; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t v = roots[i];
    const uint32_t d = (uint32_t)(dag_ptr[v + 1] - dag_ptr[v]);
    if (local) atomicAdd(&sh[d], 1u);
    else atomicAdd(&hist[d], 1u);
  }
  __syncthreads();
  if (local)
    for (uint32_t b = threadIdx.x; b < nb; b += blockDim.x)
      if (sh[b]) atomicAdd(&hist[b], sh[b]);
}
}  // namespace

// A2: all vertices sorted by d+ descending (stable: ties by id), this rank's share of
// them (snake over the sorted order), and ge[t] = #roots with
// d+ >= t.  Cached on the graph for the (rank, world) of its context.
void ensure_root_order(gamma_graph *g) {
  gamma_ctx *ctx = g->ctx;
  if (g->root_order && g->root_rank == ctx->desc.rank && g->root_world == ctx->desc.world) return;
  if (g->root_order) {
    ctx->free(g->root_order);
    g->root_order = nullptr;
  }
  const uint32_t n = g->n;
  DevBuf<uint32_t> key(ctx, n), key2(ctx, n), val(ctx, n), order(ctx, n);
  ctx->launch(KC_ROOTS, [&] { outdeg_key_kernel<<<grid1d(n), 256, 0, ctx->stream>>>(g->dag_ptr, n, key.p, val.p); });
  int endbit = 1;
  while (endbit < 32 && (1ull << endbit) <= g->max_out_degree) endbit++;
  size_t tmp = 0;
  GAMMA_CUDA(cub::DeviceRadixSort::SortPairsDescending(nullptr, tmp, key.p, key2.p, val.p, order.p, (uint64_t)n, 0,
                                                       endbit, ctx->stream));
  {
    DevBuf<uint8_t> t(ctx, tmp);
    ctx->launch(KC_ROOTS, [&] {
      GAMMA_CUDA(cub::DeviceRadixSort::SortPairsDescending(t.p, tmp, key.p, key2.p, val.p, order.p, (uint64_t)n, 0,
                                                           endbit, ctx->stream));
    });
    ctx->cub_sort_launched(KC_ROOTS, n, endbit);
  }
  uint64_t nr = n;
  if (ctx->desc.world > 1) {
    DevBuf<uint8_t> flag(ctx, n);
    DevBuf<uint64_t> nsel(ctx, 1);
    ctx->launch(KC_ROOTS, [&] {
      rank_flag_kernel<<<grid1d(n), 256, 0, ctx->stream>>>(n, ctx->desc.rank, ctx->desc.world, flag.p);
    });
    DevBuf<uint32_t> mine(ctx, n);
    tmp = 0;
    GAMMA_CUDA(cub::DeviceSelect::Flagged(nullptr, tmp, order.p, flag.p, mine.p, nsel.p, (int64_t)n, ctx->stream));
    {
      DevBuf<uint8_t> t(ctx, tmp);
      ctx->launch(KC_ROOTS, [&] {
        GAMMA_CUDA(cub::DeviceSelect::Flagged(t.p, tmp, order.p, flag.p, mine.p, nsel.p, (int64_t)n, ctx->stream));
      });
      ctx->cub_select_launched(KC_ROOTS);
    }
    GAMMA_CUDA(cudaMemcpyAsync(&nr, nsel.p, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
    ctx->sync();
    order = std::move(mine);
  }
  const uint32_t nb = g->max_out_degree + 2;
  DevBuf<uint32_t> hist(ctx, nb);
  GAMMA_CUDA(cudaMemsetAsync(hist.p, 0, nb * 4, ctx->stream));
  if (nr)
    ctx->launch(KC_ROOTS, [&] {
      outdeg_hist_kernel<<<std::min<unsigned>(grid1d(nr), 148u * 4u), 256, 0, ctx->stream>>>(g->dag_ptr, order.p,
                                                                                           nr, nb, hist.p);
    });
  std::vector<uint32_t> h(nb);
  GAMMA_CUDA(cudaMemcpyAsync(h.data(), hist.p, nb * 4, cudaMemcpyDeviceToHost, ctx->stream));
  ctx->sync();
  g->root_ge.assign(nb + 1, 0);
  for (int64_t t = (int64_t)nb - 1; t >= 0; t--) g->root_ge[t] = g->root_ge[t + 1] + h[t];
  g->root_order = order.release();
  g->root_rank = ctx->desc.rank;
  g->root_world = ctx->desc.world;
  g->device_bytes += (uint64_t)n * 4;
}

uint64_t kclique_count(gamma_graph *g, uint32_t k, const uint32_t *roots_dev, uint64_t nroots,
                       uint64_t *per_root_dev) {
  gamma_ctx *ctx = g->ctx;
  const bool per_root = per_root_dev != nullptr;
  if (!per_root && ctx->desc.world <= 1 && k <= 2) return k == 1 ? g->n : g->m;
  GAMMA_REQUIRE(g->m < 0xFFFFFFFFull, GAMMA_E_UNSUPPORTED, "DAG with >= 2^32 edges");
  KclRun R;
  if (g->dag_pages)   // host-resident DAG: the bitmap path only (runs <= kWideMaxRun, k <= 12)
    GAMMA_REQUIRE((ctx->desc.flags & GAMMA_FLAG_NO_BITMAP) == 0 && k <= kBitmapMaxK &&
                      g->max_out_degree <= kWideMaxRun, GAMMA_E_UNSUPPORTED,
                  "GAMMA_FLAG_HOST_DAG: only the bitmap kCL path reads the paged DAG");
  R.g = g;
  R.ctx = ctx;
  R.k = k;
  R.per_root = per_root;
  R.fuse = (ctx->desc.flags & GAMMA_FLAG_NO_FUSE) == 0;
  R.per_root_out = (unsigned long long *)per_root_dev;
  R.levels.resize(k + 1);
  // ---- A2: root list ----
  DevBuf<uint32_t> root_buf;
  if (per_root) {
    R.roots = roots_dev;
    R.nroots = nroots;
  } else {
    // heavy-first root order of this rank, computed once per graph (k only decides
    // the prefix: d+(v) >= k-1), so a call needs no select / sort / size round trip
    ensure_root_order(g);
    R.roots = g->root_order;
    R.nroots = (k - 1 < g->root_ge.size()) ? g->root_ge[k - 1] : 0;
  }
  ctx->stats.level_entries[1] = R.nroots;
  if (k <= 2) {   // per-root or partitioned k = 1 / 2: each root contributes 1 / d+(v)
    if (R.nroots == 0) return 0;
    DevBuf<unsigned long long> tmpc(ctx, R.nroots);
    unsigned long long *out = per_root ? (unsigned long long *)per_root_dev : tmpc.p;
    ctx->launch(KC_COUNT, [&] {
      degree_count_kernel<<<grid1d(R.nroots), 256, 0, ctx->stream>>>(g->dag_ptr, R.roots, R.nroots, k, out);
    });
    if (per_root) return 0;
    std::vector<unsigned long long> h(R.nroots);
    GAMMA_CUDA(cudaMemcpyAsync(h.data(), out, R.nroots * 8, cudaMemcpyDeviceToHost, ctx->stream));
    ctx->sync();
    uint64_t s = 0;
    for (auto x : h) s = checked_add(s, x);
    return s;
  }
  configure_kernels();
  R.grid[MODE_EXTEND] = ctx->num_sms * occupancy_blocks((const void *)kcl_kernel<MODE_EXTEND, false, false>,
                                                        kThreads, kcl_smem(MODE_EXTEND));
  R.grid[MODE_COUNT] = ctx->num_sms * occupancy_blocks((const void *)kcl_kernel<MODE_COUNT, false, false>,
                                                       kThreads, kcl_smem(MODE_COUNT));
  R.grid[MODE_FUSED] = ctx->num_sms * occupancy_blocks((const void *)kcl_kernel<MODE_FUSED, false, false>,
                                                       kThreads, kcl_smem(MODE_FUSED));
  const bool bitmap = (ctx->desc.flags & GAMMA_FLAG_NO_BITMAP) == 0 && k >= 3 && k <= kBitmapMaxK;
  if (bitmap && R.nroots) {
    uint64_t n_xl = 0, n_long = 0, n_mid = 0;
    if (!per_root) {
      n_xl = kWideMaxRun + 1 < g->root_ge.size() ? g->root_ge[kWideMaxRun + 1] : 0;
      n_long = kBitmapMaxRun + 1 < g->root_ge.size() ? g->root_ge[kBitmapMaxRun + 1] : 0;
      n_mid = 129 < g->root_ge.size() ? g->root_ge[129] : 0;
    }
    R.add_count(kclique_bitmap(g, k, R.roots, R.nroots, R.per_root_out, !per_root, n_xl, n_long, n_mid));
    R.root_len_gt = kWideMaxRun;
  }
  if (R.nroots && (!bitmap || g->max_out_degree > kWideMaxRun)) {
    size_t fr = 0, tot = 0;
    GAMMA_CUDA(cudaMemGetInfo(&fr, &tot));
    const uint64_t budget = ctx->desc.hbm_budget_bytes ? ctx->desc.hbm_budget_bytes : (uint64_t)(fr * 0.8);
    const uint64_t stored = k >= 4 ? k - 3 : 1;   // level tables at depths 2 .. k-2
    R.level_share = budget / stored;
    R.process(1, 0, R.nroots);
  }
  ctx->sync();
  ctx->collect_timings();
  return R.total;
}

bool kclique_multi(gamma_graph *g, uint32_t kmin, uint32_t kmax, uint64_t *multi_out) {
  gamma_ctx *ctx = g->ctx;
  if ((ctx->desc.flags & GAMMA_FLAG_NO_BITMAP) || kmax < 3 || kmax > kBitmapMaxK ||
      g->max_out_degree > kWideMaxRun)
    return false;
  GAMMA_REQUIRE(g->m < 0xFFFFFFFFull, GAMMA_E_UNSUPPORTED, "DAG with >= 2^32 edges");
  ensure_root_order(g);
  kmin = std::max<uint32_t>(3, std::min(kmin, kmax));
  const uint64_t nroots = kmin - 1 < g->root_ge.size() ? g->root_ge[kmin - 1] : 0;   // d+ >= kmin - 1
  ctx->stats.level_entries[1] = nroots;
  for (uint32_t s = 0; s <= kmax; s++) multi_out[s] = 0;
  if (nroots) {
    const uint64_t n_long = kBitmapMaxRun + 1 < g->root_ge.size() ? g->root_ge[kBitmapMaxRun + 1] : 0;
    const uint64_t n_mid = 129 < g->root_ge.size() ? g->root_ge[129] : 0;
    kclique_bitmap(g, kmax, g->root_order, nroots, nullptr, true, 0, n_long, n_mid, multi_out, kmin);
  }
  ctx->sync();
  ctx->collect_timings();
  return true;
}

}  // namespace gamma_impl
