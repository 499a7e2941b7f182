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
//    group in shared memory and every child's N+(c) is streamed from HBM with
//    coalesced 128 B warp loads and probed against it (branch-free binary search),
//    survivors compacted in order with __ballot_sync/__popc.
//  * ET level = column-first vid[] (4 B per embedding) + group table {beg,len}
//    (8 B per non-empty group).  The parent pointer of the prefix tree is implicit
//    in the group.
//  * Opt 1: per-warp 16 KB vid blocks / 4 KB group blocks reserved with one atomic;
//    a child's run is written contiguously from a shared-memory staging buffer.
//  * A8: DFS over (depth, group range) with level buffers that grow geometrically up
//    to the HBM budget; when a level still overflows, the producing range is split
//    in halves (BFS inside a range, DFS across ranges).
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_select.cuh>

#include <algorithm>
#include <vector>

#include "internal.cuh"

namespace gamma_impl {

namespace {

constexpr int kWarps = 8;
constexpr int kThreads = kWarps * 32;
constexpr uint32_t kRunCap = 1024;   // staged run capacity per warp (u32)
constexpr uint32_t kBlkV = 4096;     // Opt 1 vid block per warp (16 KB)
constexpr uint32_t kBlkG = 512;      // Opt 1 group block per warp (4 KB)

struct KclArgs {
  // graph (DAG)
  const uint64_t *dag_ptr;
  const uint32_t *dag_col;
  // input groups: depth-1 (roots) or a level table
  const uint32_t *roots;      // depth 1
  const uint2 *grp_in;        // depth >= 2: {beg, len}
  const uint32_t *groot_in;   // depth >= 2, per-root mode: root index per group
  const uint32_t *vid_in;
  uint64_t g_begin, g_end;    // group range processed by this launch
  uint32_t need_group;        // skip groups with len < need_group
  uint32_t need_child;        // keep children whose new run has >= need_child entries
  // output level (extend)
  uint32_t *vid_out;
  uint2 *grp_out;
  uint32_t *groot_out;
  uint64_t cap_v, cap_g;
  // control + results
  unsigned long long *ctrl;
  unsigned long long *per_root;  // per-root counts (nullable)
  uint32_t batch;
  uint32_t stage_cap;         // kRunCap (0 under GAMMA_FLAG_DEBUG_NOSTAGE)
};

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

struct WarpBlocks {
  uint64_t vb = 0, ve = 0, gb = 0, ge = 0;
};

// Opt 1: reserve f contiguous vid slots from the warp's current block, taking a
// fresh block from the pool when the block cannot hold them.  Warp-uniform.
__device__ __forceinline__ bool reserve_v(WarpBlocks &w, uint32_t f, const KclArgs &a, int lane,
                                          uint64_t &pos) {
  if (w.vb + f > w.ve) {
    unsigned long long nb = 0;
    if (lane == 0) nb = atomicAdd(&a.ctrl[CTRL_VCUR], (unsigned long long)kBlkV);
    nb = __shfl_sync(0xffffffffu, nb, 0);
    if (nb + kBlkV > a.cap_v) {
      if (lane == 0) atomicExch(&a.ctrl[CTRL_OVF], 1ull);
      return false;
    }
    w.vb = nb;
    w.ve = nb + kBlkV;
  }
  pos = w.vb;
  w.vb += f;
  return true;
}

// Direct reservation of ub slots (children whose run may exceed the staging buffer).
__device__ __forceinline__ bool reserve_big(uint64_t ub, const KclArgs &a, int lane, uint64_t &pos) {
  unsigned long long nb = 0;
  if (lane == 0) nb = atomicAdd(&a.ctrl[CTRL_VCUR], (unsigned long long)ub);
  nb = __shfl_sync(0xffffffffu, nb, 0);
  if (nb + ub > a.cap_v) {
    if (lane == 0) atomicExch(&a.ctrl[CTRL_OVF], 1ull);
    return false;
  }
  pos = nb;
  return true;
}

__device__ __forceinline__ bool reserve_g(WarpBlocks &w, const KclArgs &a, int lane, uint64_t &pos) {
  if (w.gb == w.ge) {
    unsigned long long nb = 0;
    if (lane == 0) nb = atomicAdd(&a.ctrl[CTRL_GCUR], (unsigned long long)kBlkG);
    nb = __shfl_sync(0xffffffffu, nb, 0);
    if (nb + kBlkG > a.cap_g) {
      if (lane == 0) atomicExch(&a.ctrl[CTRL_OVF], 1ull);
      return false;
    }
    w.gb = nb;
    w.ge = nb + kBlkG;
  }
  pos = w.gb++;
  return true;
}

// One kernel body for both the extend step (COUNT=false: write the children's runs
// as the next ET level) and the last step (COUNT=true: sum the run lengths, i.e.
// the k-cliques, without writing).  ROOT: input groups are depth-1 (DAG lists of
// the root vertices) instead of a level table.  PER_ROOT: attribute counts to the
// root of each group (gamma_kclique_roots).
template <bool COUNT, bool ROOT, bool PER_ROOT>
__global__ void __launch_bounds__(kThreads) kcl_step_kernel(KclArgs a) {
  extern __shared__ uint32_t smem[];   // kWarps x kRunCap run (+ kWarps x kRunCap out)
  const int lane = threadIdx.x & 31;
  const int wid = threadIdx.x >> 5;
  uint32_t *srun = smem + wid * kRunCap;
  uint32_t *sout = smem + (kWarps + wid) * kRunCap;
  WarpBlocks wb;
  uint64_t acc = 0, in_entries = 0, elems = 0, out_entries = 0;
  const uint64_t ng = a.g_end - a.g_begin;
  bool stop = false;

  while (!stop) {
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(&a.ctrl[CTRL_WORK], (unsigned long long)a.batch);
    base = __shfl_sync(0xffffffffu, base, 0);
    if (base >= ng) break;
    if (!COUNT && *(volatile unsigned long long *)&a.ctrl[CTRL_OVF]) break;
    const uint64_t bend = min((uint64_t)base + a.batch, ng);
    for (uint64_t gi = a.g_begin + base; gi < a.g_begin + bend && !stop; gi++) {
      // ---- A2/A3: the group's run C(P) ----
      const uint32_t *run;
      uint32_t len;
      uint32_t root_idx = 0;
      if (ROOT) {
        uint32_t v = a.roots[gi];
        uint64_t b0 = a.dag_ptr[v];
        len = (uint32_t)(a.dag_ptr[v + 1] - b0);
        run = a.dag_col + b0;
        root_idx = (uint32_t)gi;
      } else {
        uint2 gd = a.grp_in[gi];
        len = gd.y;
        run = a.vid_in + gd.x;
        if (PER_ROOT) root_idx = a.groot_in[gi];
      }
      if (len < a.need_group) continue;
      in_entries += len;
      const bool staged = len <= a.stage_cap;
      if (staged) {
        for (uint32_t i = lane; i < len; i += 32) srun[i] = run[i];
        __syncwarp();
      }
      const uint32_t *probe = staged ? srun : run;
      const uint32_t rmin = probe[0], rmax = probe[len - 1];
      uint64_t gacc = 0;
      // ---- A4-A6: every child c of the group ----
      for (uint32_t i = 0; i < len; i++) {
        const uint32_t c = probe[i];
        const uint64_t lb = a.dag_ptr[c];
        const uint32_t dl = (uint32_t)(a.dag_ptr[c + 1] - lb);
        elems += dl;
        if (dl < a.need_child) continue;
        const uint32_t *lst = a.dag_col + lb;
        const uint32_t ub = min(dl, len);
        const bool big = !COUNT && ub > a.stage_cap;
        uint64_t bigpos = 0;
        if (big && !reserve_big(ub, a, lane, bigpos)) { stop = true; break; }
        uint32_t found = 0;
        for (uint32_t j = 0; j < dl; j += 32) {
          const uint32_t y = (j + lane < dl) ? __ldg(lst + j + lane) : 0xffffffffu;
          bool hit = false;
          if (y >= rmin && y <= rmax) hit = staged ? sorted_contains(srun, len, y)
                                                   : sorted_contains(run, len, y);
          const uint32_t bal = __ballot_sync(0xffffffffu, hit);
          if (!COUNT && hit) {
            const uint32_t p = found + __popc(bal & lanemask_lt());
            if (big) a.vid_out[bigpos + p] = y;
            else sout[p] = y;
          }
          found += __popc(bal);
          if (__shfl_sync(0xffffffffu, y, 31) > rmax) break;  // rest of N+(c) is > max C(P)
        }
        if (COUNT) {
          gacc += found;
          continue;
        }
        // A6: keep the child's run as a group of the next level
        if (found < a.need_child) continue;
        uint64_t pos;
        if (big) {
          pos = bigpos;
        } else {
          __syncwarp();
          if (!reserve_v(wb, found, a, lane, pos)) { stop = true; break; }
          for (uint32_t t = lane; t < found; t += 32) a.vid_out[pos + t] = sout[t];
        }
        uint64_t gpos;
        if (!reserve_g(wb, a, lane, gpos)) { stop = true; break; }
        if (lane == 0) {
          a.grp_out[gpos] = make_uint2((uint32_t)pos, found);
          if (PER_ROOT) a.groot_out[gpos] = root_idx;
        }
        out_entries += found;
        __syncwarp();
      }
      acc += gacc;
      if (PER_ROOT && COUNT && lane == 0 && gacc) atomicAdd(&a.per_root[root_idx], (unsigned long long)gacc);
      __syncwarp();
    }
  }
  // unused group slots of this warp's last block become empty groups
  if (!COUNT)
    for (uint64_t s = wb.gb + lane; s < wb.ge; s += 32) a.grp_out[s] = make_uint2(0, 0);
  if (lane == 0) {
    if (COUNT && acc) atomicAdd(&a.ctrl[CTRL_COUNT], (unsigned long long)acc);
    atomicAdd(&a.ctrl[CTRL_AUX0], (unsigned long long)in_entries);
    atomicAdd(&a.ctrl[CTRL_ELEMS], (unsigned long long)elems);
    if (!COUNT) atomicAdd(&a.ctrl[CTRL_ENTRIES], (unsigned long long)out_entries);
  }
}

// A2: roots = vertices with d+(v) >= need, cost key for heavy-first ordering.
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
    uint32_t v = roots[i];
    uint64_t d = dag_ptr[v + 1] - dag_ptr[v];
    cost[i] = d * d;
  }
}

// Snake (boustrophedon) assignment of cost-sorted roots to ranks: an LPT-style
// balance that needs no coordination.
__global__ void rank_flag_kernel(uint64_t nr, uint32_t rank, uint32_t world, uint8_t *flag) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nr;
       i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t r = i % (2ull * world);
    flag[i] = (r == rank || r == 2ull * world - 1 - rank) ? 1 : 0;
  }
}

__global__ void degree_count_kernel(const uint64_t *dag_ptr, const uint32_t *roots, uint64_t nr,
                                    uint32_t k, unsigned long long *out) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nr;
       i += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t v = roots[i];
    out[i] = (k == 1) ? 1ull : (unsigned long long)(dag_ptr[v + 1] - dag_ptr[v]);
  }
}

inline unsigned grid1d(uint64_t n, int threads = 256) {
  uint64_t b = (n + threads - 1) / threads;
  if (b == 0) b = 1;
  return (unsigned)std::min<uint64_t>(b, 148u * 32u);
}

constexpr size_t step_smem(bool count) {
  return (count ? 1 : 2) * (size_t)kWarps * kRunCap * sizeof(uint32_t);
}

template <bool COUNT, bool ROOT, bool PER_ROOT>
void set_smem_attr() {
  GAMMA_CUDA(cudaFuncSetAttribute(kcl_step_kernel<COUNT, ROOT, PER_ROOT>,
                                  cudaFuncAttributeMaxDynamicSharedMemorySize, (int)step_smem(COUNT)));
}

void configure_kernels() {
  static bool done = false;   // per process; attributes are per function
  if (done) return;
  set_smem_attr<false, false, false>();
  set_smem_attr<false, false, true>();
  set_smem_attr<false, true, false>();
  set_smem_attr<false, true, true>();
  set_smem_attr<true, false, false>();
  set_smem_attr<true, false, true>();
  set_smem_attr<true, true, false>();
  set_smem_attr<true, true, true>();
  done = true;
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
  const uint32_t *roots;
  uint64_t nroots;
  unsigned long long *per_root_out;
  std::vector<Level> levels;   // levels[d] holds groups at depth d (d >= 2)
  uint64_t budget;             // bytes for all level tables
  uint64_t total = 0;
  int grid_extend = 0, grid_count = 0;

  uint64_t level_bytes(uint64_t cv, uint64_t cg) const {
    return cv * 4 + cg * (per_root ? 12 : 8);
  }
  uint64_t used_bytes() const {
    uint64_t s = 0;
    for (auto &l : levels) s += level_bytes(l.cap_v, l.cap_g);
    return s;
  }

  void ensure_level(uint32_t d, uint64_t want_v) {
    Level &L = levels[d];
    if (L.cap_v >= want_v) return;
    uint64_t cv = std::max<uint64_t>(want_v, 1ull << 20);
    cv = std::min<uint64_t>(cv, 0xFFFFFFFFull - kBlkV);  // beg is u32
    uint64_t cg = cv / 2 + kBlkG * 1024;
    uint64_t others = used_bytes() - level_bytes(L.cap_v, L.cap_g);
    if (others + level_bytes(cv, cg) > budget) {
      // shrink to what the budget allows (at least one block per warp)
      uint64_t avail = budget > others ? budget - others : 0;
      cv = avail / (4 + (per_root ? 12 : 8) / 2);
      cg = cv / 2;
      if (cv <= L.cap_v) return;  // cannot grow
    }
    L.vid.reset(); L.grp.reset(); L.groot.reset();
    L.vid = DevBuf<uint32_t>(ctx, cv);
    L.grp = DevBuf<uint2>(ctx, cg);
    if (per_root) L.groot = DevBuf<uint32_t>(ctx, cg);
    L.cap_v = cv;
    L.cap_g = cg;
  }

  KclArgs base_args() const {
    KclArgs a{};
    a.dag_ptr = g->dag_ptr;
    a.dag_col = g->dag_col;
    a.ctrl = (unsigned long long *)ctx->ctrl;
    a.per_root = per_root_out;
    a.stage_cap = (ctx->desc.flags & GAMMA_FLAG_DEBUG_NOSTAGE) ? 0u : kRunCap;
    return a;
  }

  void fill_input(KclArgs &a, uint32_t d, uint64_t g0, uint64_t g1) const {
    a.g_begin = g0;
    a.g_end = g1;
    if (d == 1) {
      a.roots = roots;
      a.batch = 4;
    } else {
      const Level &L = levels[d];
      a.grp_in = L.grp.p;
      a.groot_in = L.groot.p;
      a.vid_in = L.vid.p;
      a.batch = 32;
    }
    a.need_group = k - d;   // a depth-d group needs k-d more vertices
  }

  template <bool COUNT, bool ROOT>
  void launch_step(const KclArgs &a, int grid) {
    int kc = COUNT ? KC_COUNT : KC_EXTEND;
    const size_t smem = step_smem(COUNT);
    ctx->launch(kc, [&] {
      if (per_root)
        kcl_step_kernel<COUNT, ROOT, true><<<grid, kThreads, smem, ctx->stream>>>(a);
      else
        kcl_step_kernel<COUNT, ROOT, false><<<grid, kThreads, smem, ctx->stream>>>(a);
    });
  }

  // Count the k-cliques under depth-(k-2)... i.e. groups at depth d = k-1 are the
  // k-cliques; the last step reads depth k-2 groups and sums child run lengths.
  void count_range(uint32_t d, uint64_t g0, uint64_t g1) {
    KclArgs a = base_args();
    fill_input(a, d, g0, g1);
    a.need_child = 1;
    ctrl_reset(ctx);
    if (d == 1) launch_step<true, true>(a, grid_count);
    else launch_step<true, false>(a, grid_count);
    ctrl_fetch(ctx);
    const uint64_t *h = ctx->ctrl_host;
    total = checked_add(total, h[CTRL_COUNT]);
    if (d == 1) ctx->stats.level_entries[2] += h[CTRL_AUX0];
    ctx->stats.level_entries[k] = checked_add(ctx->stats.level_entries[k], h[CTRL_COUNT]);
    ctx->stats.list_elems += h[CTRL_ELEMS];
    ctx->stats.alg_bytes[KC_COUNT] += 12 * h[CTRL_AUX0] + 4 * h[CTRL_ELEMS];
  }

  // DFS over (depth, group range); BFS inside the range.
  void process(uint32_t d, uint64_t g0, uint64_t g1) {
    if (g0 >= g1) return;
    if (d == k - 2) {
      count_range(d, g0, g1);
      return;
    }
    const uint32_t nd = d + 1;
    for (int attempt = 0;; attempt++) {
      Level &L = levels[nd];
      if (L.cap_v == 0) ensure_level(nd, 1ull << 24);
      KclArgs a = base_args();
      fill_input(a, d, g0, g1);
      a.need_child = k - d - 1;  // the child's run is a depth-(d+1) group
      a.vid_out = L.vid.p;
      a.grp_out = L.grp.p;
      a.groot_out = L.groot.p;
      a.cap_v = L.cap_v;
      a.cap_g = L.cap_g;
      ctrl_reset(ctx);
      if (d == 1) launch_step<false, true>(a, grid_extend);
      else launch_step<false, false>(a, grid_extend);
      ctrl_fetch(ctx);
      const uint64_t *h = ctx->ctrl_host;
      if (!h[CTRL_OVF]) {
        if (d == 1) ctx->stats.level_entries[2] += h[CTRL_AUX0];
        ctx->stats.level_entries[nd + 1] += h[CTRL_ENTRIES];
        ctx->stats.list_elems += h[CTRL_ELEMS];
        ctx->stats.alg_bytes[KC_EXTEND] += 12 * h[CTRL_AUX0] + 4 * h[CTRL_ELEMS] + 8 * h[CTRL_ENTRIES];
        ctx->stats.chunks++;
        uint64_t ng = std::min<uint64_t>(h[CTRL_GCUR], L.cap_g);
        process(nd, 0, ng);
        return;
      }
      // overflow: grow the level if the budget allows, else split the range
      ctx->stats.retries++;
      uint64_t before = L.cap_v;
      ensure_level(nd, std::max<uint64_t>(h[CTRL_VCUR], L.cap_v) * 4);
      if (levels[nd].cap_v > before) continue;
      GAMMA_REQUIRE(g1 - g0 > 1, GAMMA_E_NOMEM,
                    "HBM budget too small for the children of a single embedding group");
      uint64_t mid = g0 + (g1 - g0) / 2;
      process(d, g0, mid);
      process(d, mid, g1);
      return;
    }
  }
};

}  // namespace

uint64_t kclique_count(gamma_graph *g, uint32_t k, const uint32_t *roots_dev, uint64_t nroots,
                       uint64_t *per_root_dev) {
  gamma_ctx *ctx = g->ctx;
  const bool per_root = per_root_dev != nullptr;
  if (!per_root && ctx->desc.world <= 1 && k <= 2) return k == 1 ? g->n : g->m;
  KclRun R;
  R.g = g;
  R.ctx = ctx;
  R.k = k;
  R.per_root = per_root;
  R.per_root_out = (unsigned long long *)per_root_dev;
  R.levels.resize(k + 1);
  {
    size_t fr = 0, tot = 0;
    GAMMA_CUDA(cudaMemGetInfo(&fr, &tot));
    R.budget = ctx->desc.hbm_budget_bytes ? ctx->desc.hbm_budget_bytes : (uint64_t)(fr * 0.8);
  }
  // ---- A2: root list ----
  DevBuf<uint32_t> root_buf;
  if (per_root) {
    R.roots = roots_dev;
    R.nroots = nroots;
  } else {
    const uint32_t n = g->n;
    DevBuf<uint32_t> all(ctx, n);
    ctx->launch(KC_ROOTS, [&] { iota_kernel<<<grid1d(n), 256, 0, ctx->stream>>>(all.p, n); });
    DevBuf<uint32_t> sel(ctx, n);
    DevBuf<uint64_t> nsel(ctx, 1);
    RootNeed op{g->dag_ptr, k - 1};
    size_t tmp = 0;
    GAMMA_CUDA(cub::DeviceSelect::If(nullptr, tmp, all.p, sel.p, nsel.p, (int64_t)n, op, ctx->stream));
    {
      DevBuf<uint8_t> t(ctx, tmp);
      ctx->launch(KC_ROOTS, [&] {
        GAMMA_CUDA(cub::DeviceSelect::If(t.p, tmp, all.p, sel.p, nsel.p, (int64_t)n, op, ctx->stream));
      });
    }
    uint64_t nr = 0;
    GAMMA_CUDA(cudaMemcpyAsync(&nr, nsel.p, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
    ctx->sync();
    // heavy-first: sort by cost descending
    DevBuf<uint64_t> cost(ctx, nr ? nr : 1), cost2(ctx, nr ? nr : 1);
    root_buf = DevBuf<uint32_t>(ctx, nr ? nr : 1);
    if (nr) {
      ctx->launch(KC_ROOTS, [&] {
        root_cost_kernel<<<grid1d(nr), 256, 0, ctx->stream>>>(g->dag_ptr, sel.p, nr, cost.p);
      });
      int endbit = 1;
      while (endbit < 64 && (1ull << endbit) <= (uint64_t)g->max_out_degree * g->max_out_degree) endbit++;
      tmp = 0;
      GAMMA_CUDA(cub::DeviceRadixSort::SortPairsDescending(nullptr, tmp, cost.p, cost2.p, sel.p, root_buf.p,
                                                           nr, 0, endbit, ctx->stream));
      DevBuf<uint8_t> t(ctx, tmp);
      ctx->launch(KC_ROOTS, [&] {
        GAMMA_CUDA(cub::DeviceRadixSort::SortPairsDescending(t.p, tmp, cost.p, cost2.p, sel.p, root_buf.p,
                                                             nr, 0, endbit, ctx->stream));
      });
    }
    if (ctx->desc.world > 1 && nr) {
      DevBuf<uint8_t> flag(ctx, nr);
      ctx->launch(KC_ROOTS, [&] {
        rank_flag_kernel<<<grid1d(nr), 256, 0, ctx->stream>>>(nr, ctx->desc.rank, ctx->desc.world, flag.p);
      });
      DevBuf<uint32_t> mine(ctx, nr);
      tmp = 0;
      GAMMA_CUDA(cub::DeviceSelect::Flagged(nullptr, tmp, root_buf.p, flag.p, mine.p, nsel.p, (int64_t)nr,
                                            ctx->stream));
      {
        DevBuf<uint8_t> t(ctx, tmp);
        ctx->launch(KC_ROOTS, [&] {
          GAMMA_CUDA(cub::DeviceSelect::Flagged(t.p, tmp, root_buf.p, flag.p, mine.p, nsel.p, (int64_t)nr,
                                                ctx->stream));
        });
      }
      GAMMA_CUDA(cudaMemcpyAsync(&nr, nsel.p, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
      ctx->sync();
      root_buf = std::move(mine);
    }
    R.roots = root_buf.p;
    R.nroots = nr;
  }
  ctx->stats.level_entries[1] = R.nroots;
  if (k <= 2) {
    // per-root (or partitioned) k=1 / k=2: each root contributes 1 / d+(v)
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
  R.grid_extend = ctx->num_sms * occupancy_blocks((const void *)kcl_step_kernel<false, false, false>, kThreads,
                                                  step_smem(false));
  R.grid_count = ctx->num_sms * occupancy_blocks((const void *)kcl_step_kernel<true, false, false>, kThreads,
                                                 step_smem(true));
  if (R.nroots) R.process(1, 0, R.nroots);
  ctx->sync();
  ctx->collect_timings();
  return R.total;
}

}  // namespace gamma_impl
