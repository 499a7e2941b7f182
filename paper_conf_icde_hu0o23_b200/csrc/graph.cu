// graph.cu -- A1: raw edge samples -> symmetric CSR (+ degree-ordered DAG, labels).
//
// PAPER.md L199 (§IV): "We adopt Compressed Sparse Row (CSR) to represent a data
// graph G_d, which is made up of adjacency lists of all vertices"; L204: labels +
// adjacency lists only.  O-0 normalisation (R13): symmetrise, drop
// self-loops and duplicates, sort each list ascending.  DAG (R9, not in
// the paper): keep u->v iff (deg u, u) < (deg v, v).
//
// B200 layout: one packed key per directed edge, (u << b) | v with b = bit width
// of n, radix-sorted over exactly 2b bits (CUB onesweep, one pass per 8 bits);
// duplicates removed by a unique pass; row_ptr / col produced by one fused
// boundary kernel.  Everything stays in HBM; the only host sync is to learn m.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>
#include <cub/device/device_segmented_sort.cuh>
#include <cub/device/device_select.cuh>

#include <algorithm>
#include <vector>

#include "internal.cuh"

namespace gamma_impl {

namespace {

constexpr int kThreads = 256;

inline unsigned grid_for(uint64_t n, int threads = kThreads, unsigned cap = 148u * 64u) {
  uint64_t b = (n + threads - 1) / threads;
  if (b == 0) b = 1;
  return (unsigned)(b < cap ? b : cap);
}

// Two directed keys per raw sample; self-loops and out-of-range ids become the
// invalid key (all 2b bits set), which sorts after every valid key.
__global__ void pack_keys_kernel(const uint32_t *__restrict__ src, const uint32_t *__restrict__ dst,
                                 uint64_t m, uint32_t n, uint32_t b, uint64_t *__restrict__ keys,
                                 unsigned long long *err) {
  const uint64_t invalid = (b >= 32) ? ~0ull : ((1ull << (2 * b)) - 1);
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m;
       i += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t u = src[i], v = dst[i];
    uint64_t k0 = invalid, k1 = invalid;
    if (u >= n || v >= n) {
      atomicOr(err, 1ull);
    } else if (u != v) {
      k0 = ((uint64_t)u << b) | v;
      k1 = ((uint64_t)v << b) | u;
    }
    keys[2 * i] = k0;
    keys[2 * i + 1] = k1;
  }
}

// From M sorted, unique, valid keys (u << b | v): col[i] = v and row_ptr boundaries.
__global__ void csr_from_keys_kernel(const uint64_t *__restrict__ keys, uint64_t M, uint32_t n,
                                     uint32_t b, uint64_t *__restrict__ row_ptr,
                                     uint32_t *__restrict__ col) {
  const uint64_t mask = (b >= 32) ? 0xffffffffull : ((1ull << b) - 1);
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < M;
       i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t key = keys[i];
    uint32_t u = (uint32_t)(key >> b);
    col[i] = (uint32_t)(key & mask);
    // rows (prev_u, u] start at i
    int64_t prev_u = (i == 0) ? -1 : (int64_t)(keys[i - 1] >> b);
    for (int64_t w = prev_u + 1; w <= (int64_t)u; w++) row_ptr[w] = i;
    if (i == M - 1)
      for (uint64_t w = (uint64_t)u + 1; w <= n; w++) row_ptr[w] = M;
  }
}

__global__ void fill_u64_kernel(uint64_t *p, uint64_t n, uint64_t v) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x)
    p[i] = v;
}

// DAG flag: keep directed edge u->v iff (deg u, u) < (deg v, v).
struct DagKeep {
  const uint64_t *row_ptr;
  uint32_t b;
  uint64_t mask;
  __device__ __forceinline__ bool operator()(const uint64_t &key) const {
    uint32_t u = (uint32_t)(key >> b), v = (uint32_t)(key & mask);
    uint64_t du = row_ptr[u + 1] - row_ptr[u], dv = row_ptr[v + 1] - row_ptr[v];
    return du < dv || (du == dv && u < v);
  }
};

__global__ void max_degree_kernel(const uint64_t *__restrict__ rp, uint32_t n,
                                  unsigned long long *out) {
  unsigned long long best = 0;
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n;
       v += (uint64_t)gridDim.x * blockDim.x) {
    unsigned long long d = rp[v + 1] - rp[v];
    best = d > best ? d : best;
  }
  for (int o = 16; o > 0; o >>= 1) {
    unsigned long long x = __shfl_down_sync(0xffffffffu, best, o);
    best = x > best ? x : best;
  }
  if ((threadIdx.x & 31) == 0) atomicMax(out, best);
}

// Expand a CSR into keys (u << b | v) and validate: ids < n, no self-loop, strictly
// ascending lists.  err bit 1: range/self-loop/order violation.
__global__ void csr_to_keys_kernel(const uint64_t *__restrict__ rp, const uint32_t *__restrict__ col,
                                   uint32_t n, uint32_t b, uint64_t *__restrict__ keys,
                                   unsigned long long *err) {
  // one warp per vertex
  const int lane = threadIdx.x & 31;
  for (uint64_t v = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; v < n;
       v += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    uint64_t s = rp[v], e = rp[v + 1];
    if (e < s) {
      if (lane == 0) atomicOr(err, 1ull);
      continue;
    }
    for (uint64_t i = s + lane; i < e; i += 32) {
      uint32_t x = col[i];
      bool bad = x >= n || x == (uint32_t)v || (i > s && col[i - 1] >= x);
      if (bad) atomicOr(err, 1ull);
      keys[i] = ((uint64_t)v << b) | (x < n ? x : 0);
    }
  }
}

// Symmetry: every (v, x) must have v in N(x).  Binary search per element.
__global__ void csr_symmetry_kernel(const uint64_t *__restrict__ rp, const uint32_t *__restrict__ col,
                                    uint32_t n, unsigned long long *err) {
  const int lane = threadIdx.x & 31;
  for (uint64_t v = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; v < n;
       v += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    for (uint64_t i = rp[v] + lane; i < rp[v + 1]; i += 32) {
      uint32_t x = col[i];
      uint64_t lo = rp[x], hi = rp[x + 1];
      while (lo < hi) {
        uint64_t mid = (lo + hi) >> 1;
        if (col[mid] < (uint32_t)v) lo = mid + 1; else hi = mid;
      }
      if (lo >= rp[x + 1] || col[lo] != (uint32_t)v) atomicOr(err, 2ull);
    }
  }
}

__global__ void narrow_u64_kernel(const uint64_t *__restrict__ in, uint64_t n, uint32_t *__restrict__ out) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    out[i] = (uint32_t)in[i];
}

// ---- counting-sort builder (A1 when 2m' < 2^31): degree count -> scan -> scatter ->
// segmented sort of each row -> per-row dedup, all row-local after the scatter ----
__global__ void raw_degree_kernel(const uint32_t *__restrict__ src, const uint32_t *__restrict__ dst, uint64_t m,
                                  uint32_t n, uint32_t *__restrict__ cnt, unsigned long long *err) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t u = src[i], v = dst[i];
    if (u >= n || v >= n) {
      atomicOr(err, 1ull);
      continue;
    }
    if (u == v) continue;   // no self-loops
    atomicAdd(&cnt[u], 1u);
    atomicAdd(&cnt[v], 1u);
  }
}

__global__ void raw_scatter_kernel(const uint32_t *__restrict__ src, const uint32_t *__restrict__ dst, uint64_t m,
                                   uint32_t n, const uint32_t *__restrict__ off, uint32_t *__restrict__ cur,
                                   uint32_t *__restrict__ col) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t u = src[i], v = dst[i];
    if (u >= n || v >= n || u == v) continue;
    col[off[u] + atomicAdd(&cur[u], 1u)] = v;
    col[off[v] + atomicAdd(&cur[v], 1u)] = u;
  }
}

// One warp per row of the sorted raw lists: number of distinct entries.
__global__ void row_unique_count_kernel(const uint32_t *__restrict__ off, const uint32_t *__restrict__ col,
                                        uint32_t n, uint64_t *__restrict__ deg) {
  const int lane = threadIdx.x & 31;
  for (uint64_t v = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; v < n;
       v += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    const uint32_t s = off[v], e = off[v + 1];
    uint32_t c = 0;
    for (uint32_t i0 = s; i0 < e; i0 += 32) {
      const uint32_t i = i0 + lane;
      const bool keep = i < e && (i == s || col[i] != col[i - 1]);
      c += __popc(__ballot_sync(0xffffffffu, keep));
    }
    if (lane == 0) deg[v] = c;
  }
}

// One warp per row: write the distinct entries at row_ptr[v] (ballot compaction) and
// count the DAG out-degree: keep v->x iff (deg v, v) < (deg x, x).
__global__ void row_unique_write_kernel(const uint32_t *__restrict__ off, const uint32_t *__restrict__ col_in,
                                        uint32_t n, const uint64_t *__restrict__ row_ptr,
                                        uint32_t *__restrict__ col, uint64_t *__restrict__ dcnt) {
  const int lane = threadIdx.x & 31;
  const uint32_t below = (1u << lane) - 1u;
  for (uint64_t v = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; v < n;
       v += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    const uint32_t s = off[v], e = off[v + 1];
    const uint64_t dv = row_ptr[v + 1] - row_ptr[v];
    uint64_t w = row_ptr[v];
    uint32_t dc = 0;
    for (uint32_t i0 = s; i0 < e; i0 += 32) {
      const uint32_t i = i0 + lane;
      uint32_t x = 0;
      bool keep = false;
      if (i < e) {
        x = col_in[i];
        keep = i == s || x != col_in[i - 1];
      }
      const uint32_t bal = __ballot_sync(0xffffffffu, keep);
      if (keep) {
        col[w + __popc(bal & below)] = x;
        const uint64_t dx = row_ptr[x + 1] - row_ptr[x];
        dc += (dv < dx || (dv == dx && (uint32_t)v < x)) ? 1u : 0u;
      }
      w += __popc(bal);
    }
    for (int o = 16; o > 0; o >>= 1) dc += __shfl_down_sync(0xffffffffu, dc, o);
    if (lane == 0) dcnt[v] = dc;
  }
}

// One warp per row: the DAG list = the row filtered by the orientation (stays sorted).
__global__ void dag_write_kernel(const uint64_t *__restrict__ row_ptr, const uint32_t *__restrict__ col, uint32_t n,
                                 const uint64_t *__restrict__ dag_ptr, uint32_t *__restrict__ dag_col) {
  const int lane = threadIdx.x & 31;
  const uint32_t below = (1u << lane) - 1u;
  for (uint64_t v = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; v < n;
       v += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    const uint64_t s = row_ptr[v], e = row_ptr[v + 1], dv = e - s;
    uint64_t w = dag_ptr[v];
    for (uint64_t i0 = s; i0 < e; i0 += 32) {
      const uint64_t i = i0 + lane;
      uint32_t x = 0;
      bool keep = false;
      if (i < e) {
        x = col[i];
        const uint64_t dx = row_ptr[x + 1] - row_ptr[x];
        keep = dv < dx || (dv == dx && (uint32_t)v < x);
      }
      const uint32_t bal = __ballot_sync(0xffffffffu, keep);
      if (keep) dag_col[w + __popc(bal & below)] = x;
      w += __popc(bal);
    }
  }
}

// ---- rank-space DAG (kCL): vertices relabelled by their rank in the (degree, id)
// order, so that a DAG list sorted ascending is sorted by rank and every out-neighbour
// has a larger id than its tail; the kCL kernels then trim a child's list at the
// largest rank of the root's run (everything above cannot be in it) ----
__global__ void iota_u32_kernel(uint32_t *p, uint32_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    p[i] = (uint32_t)i;
}

__global__ void rank_keys_kernel(const uint64_t *__restrict__ row_ptr, uint32_t n, uint64_t *__restrict__ keys) {
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x)
    keys[v] = ((row_ptr[v + 1] - row_ptr[v]) << 32) | v;
}

__global__ void rank_scatter_kernel(const uint64_t *__restrict__ sorted, uint32_t n, uint32_t *__restrict__ rank_of) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    rank_of[(uint32_t)sorted[i]] = (uint32_t)i;
}

// one warp per id-space DAG row u: key of every edge u -> x in rank space
__global__ void dag_rank_keys_kernel(const uint64_t *__restrict__ dag_ptr, const uint32_t *__restrict__ dag_col,
                                     const uint32_t *__restrict__ rank_of, uint32_t n, uint32_t b,
                                     uint64_t *__restrict__ keys) {
  const int lane = threadIdx.x & 31;
  for (uint64_t u = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; u < n;
       u += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    const uint64_t ru = (uint64_t)rank_of[u] << b;
    for (uint64_t e = dag_ptr[u] + lane; e < dag_ptr[u + 1]; e += 32) keys[e] = ru | rank_of[dag_col[e]];
  }
}

// id-space DAG (export): d+ of id u, then the sym row of u filtered by rank
__device__ __forceinline__ bool dag_before(const uint64_t *row_ptr, uint32_t v, uint32_t x) {   // (deg, id) order
  const uint64_t dv = row_ptr[v + 1] - row_ptr[v], dx = row_ptr[x + 1] - row_ptr[x];
  return dv < dx || (dv == dx && v < x);
}

__global__ void dag_id_count_kernel(const uint64_t *__restrict__ row_ptr, const uint32_t *__restrict__ col,
                                    uint32_t n, uint64_t *__restrict__ cnt) {
  const int lane = threadIdx.x & 31;
  for (uint64_t v = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; v < n;
       v += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    uint32_t c = 0;
    for (uint64_t i = row_ptr[v] + lane; i < row_ptr[v + 1]; i += 32) c += dag_before(row_ptr, (uint32_t)v, col[i]);
    for (int o = 16; o > 0; o >>= 1) c += __shfl_down_sync(0xffffffffu, c, o);
    if (lane == 0) cnt[v] = c;
  }
}

__global__ void dag_id_write_kernel(const uint64_t *__restrict__ row_ptr, const uint32_t *__restrict__ col,
                                    uint32_t n, const uint64_t *__restrict__ dag_ptr, uint32_t *__restrict__ dag_col) {
  const int lane = threadIdx.x & 31;
  const uint32_t below = (1u << lane) - 1u;
  for (uint64_t v = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; v < n;
       v += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    uint64_t w = dag_ptr[v];
    for (uint64_t i0 = row_ptr[v]; i0 < row_ptr[v + 1]; i0 += 32) {
      const uint64_t i = i0 + lane;
      uint32_t x = 0;
      bool keep = false;
      if (i < row_ptr[v + 1]) {
        x = col[i];
        keep = dag_before(row_ptr, (uint32_t)v, x);
      }
      const uint32_t bal = __ballot_sync(0xffffffffu, keep);
      if (keep) dag_col[w + __popc(bal & below)] = x;
      w += __popc(bal);
    }
  }
}

// ---- host-resident DAG (GAMMA_FLAG_HOST_DAG) ----
__global__ void dag_indeg_kernel(const uint32_t *__restrict__ dag_col, uint64_t m, uint32_t *__restrict__ indeg) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x)
    atomicAdd(&indeg[dag_col[i]], 1u);
}

// page heat: every list is read once as a root's run and once per parent (1 + its DAG
// in-degree); a page's heat = the elements of it those reads fetch
__global__ void dag_heat_kernel(const uint64_t *__restrict__ dag_ptr, const uint32_t *__restrict__ indeg, uint32_t n,
                                unsigned long long *__restrict__ heat) {
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n; v += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t b = dag_ptr[v], e = dag_ptr[v + 1];
    if (b == e) continue;
    const unsigned long long w = 1ull + indeg[v];
    for (uint64_t p = b >> kDagPageShift; p <= (e - 1) >> kDagPageShift; p++) {
      const uint64_t lo = b > (p << kDagPageShift) ? b : (p << kDagPageShift);
      const uint64_t hi = e < ((p + 1) << kDagPageShift) ? e : ((p + 1) << kDagPageShift);
      atomicAdd(&heat[p], w * (hi - lo));
    }
  }
}

uint32_t bit_width(uint32_t n) {  // bits to represent n itself
  uint32_t b = 0;
  while (b < 32 && (uint64_t(1) << b) <= n) b++;
  return b ? b : 1;
}

void sort_keys(gamma_ctx *ctx, const uint64_t *in, uint64_t *out, uint64_t nkeys, int end_bit) {
  size_t tmp = 0;
  GAMMA_CUDA(cub::DeviceRadixSort::SortKeys(nullptr, tmp, in, out, nkeys, 0, end_bit, ctx->stream));
  DevBuf<uint8_t> t(ctx, tmp);
  ctx->launch(KC_BUILD, [&] {
    GAMMA_CUDA(cub::DeviceRadixSort::SortKeys(t.p, tmp, in, out, nkeys, 0, end_bit, ctx->stream));
  });
  ctx->cub_sort_launched(KC_BUILD, nkeys, end_bit);
}

// keys -> (row_ptr, col) on g for M keys.
void keys_to_csr(gamma_ctx *ctx, const uint64_t *keys, uint64_t M, uint32_t n, uint32_t b,
                 uint64_t *row_ptr, uint32_t *col) {
  if (M == 0) {
    ctx->launch(KC_BUILD, [&] {
      fill_u64_kernel<<<grid_for(n + 1), kThreads, 0, ctx->stream>>>(row_ptr, (uint64_t)n + 1, 0);
    });
    return;
  }
  ctx->launch(KC_BUILD, [&] {
    csr_from_keys_kernel<<<grid_for(M), kThreads, 0, ctx->stream>>>(keys, M, n, b, row_ptr, col);
  });
}

uint32_t max_degree(gamma_ctx *ctx, const uint64_t *rp, uint32_t n) {
  GAMMA_CUDA(cudaMemsetAsync(ctx->ctrl + CTRL_AUX0, 0, sizeof(uint64_t), ctx->stream));
  ctx->launch(KC_BUILD, [&] {
    max_degree_kernel<<<grid_for(n), kThreads, 0, ctx->stream>>>(
        rp, n, (unsigned long long *)(ctx->ctrl + CTRL_AUX0));
  });
  uint64_t h = 0;
  GAMMA_CUDA(cudaMemcpyAsync(&h, ctx->ctrl + CTRL_AUX0, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
  ctx->sync();
  return (uint32_t)h;
}

struct BuildTimer {
  gamma_ctx *ctx;
  cudaEvent_t a = nullptr, b = nullptr;
  explicit BuildTimer(gamma_ctx *c) : ctx(c) {
    GAMMA_CUDA(cudaEventCreate(&a));
    GAMMA_CUDA(cudaEventCreate(&b));
    GAMMA_CUDA(cudaEventRecord(a, ctx->stream));
  }
  double stop() {
    GAMMA_CUDA(cudaEventRecord(b, ctx->stream));
    GAMMA_CUDA(cudaEventSynchronize(b));
    float ms = 0;
    GAMMA_CUDA(cudaEventElapsedTime(&ms, a, b));
    return ms;
  }
  ~BuildTimer() {
    if (a) cudaEventDestroy(a);
    if (b) cudaEventDestroy(b);
  }
};

}  // namespace

void build_dag(gamma_graph *g, uint64_t *keys, uint64_t M) {
  gamma_ctx *ctx = g->ctx;
  const uint32_t b = g->bits;
  const uint64_t mask = (b >= 32) ? 0xffffffffull : ((1ull << b) - 1);
  DevBuf<uint64_t> dkeys(ctx, M / 2 + 1);
  DevBuf<uint64_t> nsel(ctx, 1);
  DagKeep op{g->row_ptr, b, mask};
  size_t tmp = 0;
  GAMMA_CUDA(cub::DeviceSelect::If(nullptr, tmp, keys, dkeys.p, nsel.p, (int64_t)M, op, ctx->stream));
  DevBuf<uint8_t> t(ctx, tmp);
  ctx->launch(KC_BUILD, [&] {
    GAMMA_CUDA(cub::DeviceSelect::If(t.p, tmp, keys, dkeys.p, nsel.p, (int64_t)M, op, ctx->stream));
  });
  ctx->cub_select_launched(KC_BUILD);
  uint64_t mdag = 0;
  GAMMA_CUDA(cudaMemcpyAsync(&mdag, nsel.p, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
  ctx->sync();
  GAMMA_REQUIRE(mdag == g->m, GAMMA_E_CUDA, "DAG orientation kept " + std::to_string(mdag) +
                                                " of " + std::to_string(g->m) + " edges");
  DevBuf<uint64_t> dp(ctx, (size_t)g->n + 1);
  DevBuf<uint32_t> dc(ctx, mdag ? mdag : 1);
  keys_to_csr(ctx, dkeys.p, mdag, g->n, b, dp.p, dc.p);
  g->dag_ptr = dp.release();
  g->dag_col = dc.release();
  g->device_bytes += ((uint64_t)g->n + 1) * 8 + mdag * 4;
  g->max_out_degree = max_degree(ctx, g->dag_ptr, g->n);
}

// Relabel the DAG built in id space (g->dag_ptr/dag_col) into rank space (see
// rank_keys_kernel): rank_of by one sort of (degree, id) keys, the edges re-keyed and
// sorted into a rank-space CSR; the id-space DAG is freed.
void rank_dag(gamma_graph *g) {
  gamma_ctx *ctx = g->ctx;
  const uint32_t n = g->n, b = g->bits;
  const uint64_t m = g->m;
  DevBuf<uint32_t> rank_of(ctx, n);
  // Rank-space relabelling is opt-in (GAMMA_RANK_DAG=1): on C2 it cost 11 ms of build and
  // 1 ms of kCL time, on heavy it saved 2 ms (B200 r02, profiles/kcl_ab_r02); by default
  // the DAG keeps vertex ids (rank_of = identity)
  const char *on_env = getenv("GAMMA_RANK_DAG");
  if (!(on_env && *on_env && *on_env != '0')) {
    ctx->launch(KC_BUILD, [&] { iota_u32_kernel<<<grid_for(n), kThreads, 0, ctx->stream>>>(rank_of.p, n); });
    g->rank_of = rank_of.release();
    g->device_bytes += (uint64_t)n * 4;
    return;
  }
  {
    DevBuf<uint64_t> k0(ctx, n), k1(ctx, n);
    ctx->launch(KC_BUILD, [&] { rank_keys_kernel<<<grid_for(n), kThreads, 0, ctx->stream>>>(g->row_ptr, n, k0.p); });
    int endbit = 32;
    while (endbit < 64 && (1ull << (endbit - 32)) <= g->max_degree) endbit++;
    sort_keys(ctx, k0.p, k1.p, n, endbit);
    ctx->launch(KC_BUILD, [&] { rank_scatter_kernel<<<grid_for(n), kThreads, 0, ctx->stream>>>(k1.p, n, rank_of.p); });
  }
  if (m) {
    DevBuf<uint64_t> k0(ctx, m), k1(ctx, m);
    ctx->launch(KC_BUILD, [&] {
      dag_rank_keys_kernel<<<grid_for((uint64_t)n * 32), kThreads, 0, ctx->stream>>>(g->dag_ptr, g->dag_col,
                                                                                     rank_of.p, n, b, k0.p);
    });
    sort_keys(ctx, k0.p, k1.p, m, 2 * b);
    ctx->launch(KC_BUILD, [&] {
      csr_from_keys_kernel<<<grid_for(m), kThreads, 0, ctx->stream>>>(k1.p, m, n, b, g->dag_ptr, g->dag_col);
    });
  }
  g->rank_of = rank_of.release();
  g->rank_space = true;
  g->device_bytes += (uint64_t)n * 4;
}

namespace {
__global__ void to_rank_kernel(uint32_t *v, uint64_t nv, const uint32_t *rank_of, uint32_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nv; i += (uint64_t)gridDim.x * blockDim.x)
    if (v[i] < n) v[i] = rank_of[v[i]];   // ids >= n stay invalid
}
}  // namespace

void to_rank_space(gamma_graph *g, uint32_t *ids, uint64_t nids) {
  if (!nids) return;
  gamma_ctx *ctx = g->ctx;
  ctx->launch(KC_ROOTS, [&] {
    to_rank_kernel<<<grid_for(nids), kThreads, 0, ctx->stream>>>(ids, nids, g->rank_of, g->n);
  });
}

// Move the kCL DAG columns to pinned, mapped host memory and keep the hottest pages in
// an HBM cache of cache_bytes (0: half of the DAG); the page table replaces dag_col.
void host_dag(gamma_graph *g, uint64_t cache_bytes) {
  gamma_ctx *ctx = g->ctx;
  const uint64_t m = g->m;
  if (m == 0) return;
  const uint64_t page = 1ull << kDagPageShift;
  const uint64_t np = (m + page - 1) / page;
  std::vector<unsigned long long> heat(np);
  {
    DevBuf<uint32_t> indeg(ctx, g->n);
    DevBuf<unsigned long long> dh(ctx, np);
    GAMMA_CUDA(cudaMemsetAsync(indeg.p, 0, (size_t)g->n * 4, ctx->stream));
    GAMMA_CUDA(cudaMemsetAsync(dh.p, 0, np * 8, ctx->stream));
    ctx->launch(KC_BUILD, [&] { dag_indeg_kernel<<<grid_for(m), kThreads, 0, ctx->stream>>>(g->dag_col, m, indeg.p); });
    ctx->launch(KC_BUILD, [&] {
      dag_heat_kernel<<<grid_for(g->n), kThreads, 0, ctx->stream>>>(g->dag_ptr, indeg.p, g->n, dh.p);
    });
    GAMMA_CUDA(cudaMemcpyAsync(heat.data(), dh.p, np * 8, cudaMemcpyDeviceToHost, ctx->stream));
    ctx->sync();
  }
  GAMMA_CUDA(cudaHostAlloc((void **)&g->dag_host, m * 4, cudaHostAllocMapped));
  GAMMA_CUDA(cudaMemcpyAsync(g->dag_host, g->dag_col, m * 4, cudaMemcpyDeviceToHost, ctx->stream));
  uint32_t *host_dev = nullptr;
  GAMMA_CUDA(cudaHostGetDevicePointer((void **)&host_dev, g->dag_host, 0));
  const uint64_t want = cache_bytes ? cache_bytes : m * 2;
  const uint64_t k = std::min<uint64_t>(np, want / (page * 4));
  std::vector<uint64_t> order(np);
  for (uint64_t p = 0; p < np; p++) order[p] = p;
  std::stable_sort(order.begin(), order.end(), [&](uint64_t x, uint64_t y) { return heat[x] > heat[y]; });
  std::vector<uint64_t> table(np);
  for (uint64_t p = 0; p < np; p++) table[p] = (uint64_t)(uintptr_t)(host_dev + p * page);
  if (k) {
    DevBuf<uint32_t> cache(ctx, k * page);
    for (uint64_t i = 0; i < k; i++) {
      const uint64_t p = order[i];
      const uint64_t len = std::min<uint64_t>(page, m - p * page);
      GAMMA_CUDA(cudaMemcpyAsync(cache.p + i * page, g->dag_col + p * page, len * 4, cudaMemcpyDeviceToDevice,
                                 ctx->stream));
      table[p] = (uint64_t)(uintptr_t)(cache.p + i * page);
    }
    g->dag_cache = cache.release();
  }
  DevBuf<uint64_t> pt = to_device(ctx, table.data(), np);
  ctx->sync();
  g->dag_pages = pt.release();
  g->dag_npages = np;
  g->dag_cached = k;
  ctx->free(g->dag_col);
  g->dag_col = nullptr;
  g->device_bytes += np * 8 + k * page * 4;
  g->device_bytes -= m * 4;
}

// The id-space DAG (gamma_graph_copy_csr(which = 1)): out-lists of every vertex id,
// ascending by id, oriented by the (degree, id) order.
void export_dag_ids(gamma_graph *g, uint64_t *dag_ptr_out, uint32_t *dag_col_out) {
  gamma_ctx *ctx = g->ctx;
  const uint32_t n = g->n;
  DevBuf<uint64_t> cnt(ctx, (size_t)n + 1), dp(ctx, (size_t)n + 1);
  DevBuf<uint32_t> dc(ctx, g->m ? g->m : 1);
  GAMMA_CUDA(cudaMemsetAsync(cnt.p + n, 0, 8, ctx->stream));
  ctx->launch(KC_MISC, [&] {
    dag_id_count_kernel<<<grid_for((uint64_t)n * 32), kThreads, 0, ctx->stream>>>(g->row_ptr, g->col, n, cnt.p);
  });
  size_t tmp = 0;
  GAMMA_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp, cnt.p, dp.p, (int64_t)n + 1, ctx->stream));
  {
    DevBuf<uint8_t> t(ctx, tmp);
    ctx->launch(KC_MISC, [&] {
      GAMMA_CUDA(cub::DeviceScan::ExclusiveSum(t.p, tmp, cnt.p, dp.p, (int64_t)n + 1, ctx->stream));
    });
  }
  ctx->launch(KC_MISC, [&] {
    dag_id_write_kernel<<<grid_for((uint64_t)n * 32), kThreads, 0, ctx->stream>>>(g->row_ptr, g->col, n, dp.p,
                                                                                  dc.p);
  });
  GAMMA_CUDA(cudaMemcpyAsync(dag_ptr_out, dp.p, ((size_t)n + 1) * 8, cudaMemcpyDefault, ctx->stream));
  if (g->m) GAMMA_CUDA(cudaMemcpyAsync(dag_col_out, dc.p, g->m * 4, cudaMemcpyDefault, ctx->stream));
  ctx->sync();
}

namespace {

template <class T>
void exclusive_sum(gamma_ctx *ctx, const T *in, uint64_t *out, uint64_t n) {
  size_t tmp = 0;
  GAMMA_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp, in, out, (int64_t)n, ctx->stream));
  DevBuf<uint8_t> t(ctx, tmp);
  ctx->launch(KC_BUILD, [&] { GAMMA_CUDA(cub::DeviceScan::ExclusiveSum(t.p, tmp, in, out, (int64_t)n, ctx->stream)); });
  ctx->extra_launches(KC_BUILD, 1);   // init + scan
}

uint64_t read_u64(gamma_ctx *ctx, const uint64_t *p) {
  uint64_t h = 0;
  GAMMA_CUDA(cudaMemcpyAsync(&h, p, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
  ctx->sync();
  return h;
}

// A1 without a global key sort (GAMMA_FLAG_COUNT_SORT_BUILD, inputs with 2m' < 2^31;
// measured slower than the key sort on C2, 6.2 vs 3.1 ms, because CUB's large-segment
// kernel sorts each hub row with one CTA): count each vertex's raw
// degree, scatter every sample into its two rows, sort each row (CUB segmented sort),
// then one warp per row drops duplicates, writes the symmetric list and counts the
// DAG out-degree; a last warp-per-row pass writes the DAG lists (filtered rows stay
// sorted).  Same result as the key-sort builder: symmetric, self-loop free,
// duplicate free, ascending lists (O-0).
void build_counting(gamma_graph *g, const uint32_t *src, const uint32_t *dst, uint64_t m) {
  gamma_ctx *ctx = g->ctx;
  const uint32_t n = g->n;
  DevBuf<uint32_t> cnt(ctx, (size_t)n + 1);
  GAMMA_CUDA(cudaMemsetAsync(cnt.p, 0, ((size_t)n + 1) * 4, ctx->stream));
  GAMMA_CUDA(cudaMemsetAsync(ctx->ctrl + CTRL_ERR, 0, sizeof(uint64_t), ctx->stream));
  ctx->launch(KC_BUILD, [&] {
    raw_degree_kernel<<<grid_for(m), kThreads, 0, ctx->stream>>>(src, dst, m, n, cnt.p,
                                                                  (unsigned long long *)(ctx->ctrl + CTRL_ERR));
  });
  DevBuf<uint64_t> off64(ctx, (size_t)n + 1);
  exclusive_sum(ctx, cnt.p, off64.p, (uint64_t)n + 1);
  uint64_t h[2] = {0, 0};
  GAMMA_CUDA(cudaMemcpyAsync(&h[0], off64.p + n, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
  GAMMA_CUDA(cudaMemcpyAsync(&h[1], ctx->ctrl + CTRL_ERR, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
  ctx->sync();
  GAMMA_REQUIRE(h[1] == 0, GAMMA_E_INVAL, "gamma_load_edges: vertex id >= n");
  const uint64_t total = h[0];   // 2 x (samples without self-loops) < 2^31
  // 32-bit row offsets for the segmented sort (total < 2^31)
  DevBuf<uint32_t> off(ctx, (size_t)n + 1);
  ctx->launch(KC_BUILD, [&] {
    narrow_u64_kernel<<<grid_for((uint64_t)n + 1), kThreads, 0, ctx->stream>>>(off64.p, (uint64_t)n + 1, off.p);
  });
  off64.reset();
  GAMMA_CUDA(cudaMemsetAsync(cnt.p, 0, ((size_t)n + 1) * 4, ctx->stream));
  DevBuf<uint32_t> raw(ctx, total ? total : 1), sorted(ctx, total ? total : 1);
  ctx->launch(KC_BUILD, [&] {
    raw_scatter_kernel<<<grid_for(m), kThreads, 0, ctx->stream>>>(src, dst, m, n, off.p, cnt.p, raw.p);
  });
  cnt.reset();
  if (total) {
    size_t tmp = 0;
    GAMMA_CUDA(cub::DeviceSegmentedSort::SortKeys(nullptr, tmp, raw.p, sorted.p, (int)total, (int)n, off.p,
                                                  off.p + 1, ctx->stream));
    DevBuf<uint8_t> t(ctx, tmp);
    ctx->launch(KC_BUILD, [&] {
      GAMMA_CUDA(cub::DeviceSegmentedSort::SortKeys(t.p, tmp, raw.p, sorted.p, (int)total, (int)n, off.p, off.p + 1,
                                                    ctx->stream));
    });
    ctx->extra_launches(KC_BUILD, 2);   // partition + small/medium + large segment kernels
  }
  raw.reset();
  const unsigned wgrid = grid_for((uint64_t)n * 32);
  DevBuf<uint64_t> deg(ctx, (size_t)n + 1);
  GAMMA_CUDA(cudaMemsetAsync(deg.p + n, 0, sizeof(uint64_t), ctx->stream));
  ctx->launch(KC_BUILD, [&] { row_unique_count_kernel<<<wgrid, kThreads, 0, ctx->stream>>>(off.p, sorted.p, n, deg.p); });
  DevBuf<uint64_t> rp(ctx, (size_t)n + 1);
  exclusive_sum(ctx, deg.p, rp.p, (uint64_t)n + 1);
  const uint64_t M = read_u64(ctx, rp.p + n);
  GAMMA_REQUIRE(M % 2 == 0, GAMMA_E_CUDA, "asymmetric rows after dedup");
  DevBuf<uint32_t> col(ctx, M ? M : 1);
  GAMMA_CUDA(cudaMemsetAsync(deg.p + n, 0, sizeof(uint64_t), ctx->stream));   // deg reused as DAG counts
  ctx->launch(KC_BUILD, [&] {
    row_unique_write_kernel<<<wgrid, kThreads, 0, ctx->stream>>>(off.p, sorted.p, n, rp.p, col.p, deg.p);
  });
  sorted.reset();
  off.reset();
  DevBuf<uint64_t> dp(ctx, (size_t)n + 1);
  exclusive_sum(ctx, deg.p, dp.p, (uint64_t)n + 1);
  const uint64_t mdag = read_u64(ctx, dp.p + n);
  GAMMA_REQUIRE(mdag == M / 2, GAMMA_E_CUDA, "DAG orientation kept " + std::to_string(mdag) + " of " +
                                                 std::to_string(M / 2) + " edges");
  DevBuf<uint32_t> dc(ctx, mdag ? mdag : 1);
  ctx->launch(KC_BUILD, [&] { dag_write_kernel<<<wgrid, kThreads, 0, ctx->stream>>>(rp.p, col.p, n, dp.p, dc.p); });
  g->m = M / 2;
  g->row_ptr = rp.release();
  g->col = col.release();
  g->dag_ptr = dp.release();
  g->dag_col = dc.release();
  g->device_bytes += 2 * (((uint64_t)n + 1) * 8) + M * 4 + mdag * 4;
  g->max_degree = max_degree(ctx, g->row_ptr, n);
  g->max_out_degree = max_degree(ctx, g->dag_ptr, n);
}

}  // namespace

void build_from_edges(gamma_graph *g, const uint32_t *src, const uint32_t *dst, uint64_t m,
                      bool on_device) {
  gamma_ctx *ctx = g->ctx;
  BuildTimer timer(ctx);
  const uint32_t n = g->n;
  const uint32_t b = bit_width(n);
  g->bits = b;
  DevBuf<uint32_t> s_copy, d_copy;
  if (!on_device && m) {
    s_copy = to_device(ctx, src, m);
    d_copy = to_device(ctx, dst, m);
    src = s_copy.p;
    dst = d_copy.p;
  }
  if (m && 2 * m < (1ull << 31) && (ctx->desc.flags & GAMMA_FLAG_COUNT_SORT_BUILD) != 0) {
    build_counting(g, src, dst, m);
    rank_dag(g);
    if (ctx->desc.flags & GAMMA_FLAG_HOST_DAG) host_dag(g, ctx->desc.dag_cache_bytes);
    g->build_ms = timer.stop();
    return;
  }
  const uint64_t nkeys = 2 * m;
  uint64_t M = 0;
  DevBuf<uint64_t> uniq;
  if (nkeys) {
    DevBuf<uint64_t> keys(ctx, nkeys);
    GAMMA_CUDA(cudaMemsetAsync(ctx->ctrl + CTRL_ERR, 0, sizeof(uint64_t), ctx->stream));
    ctx->launch(KC_BUILD, [&] {
      pack_keys_kernel<<<grid_for(m), kThreads, 0, ctx->stream>>>(
          src, dst, m, n, b, keys.p, (unsigned long long *)(ctx->ctrl + CTRL_ERR));
    });
    s_copy.reset();
    d_copy.reset();
    DevBuf<uint64_t> sorted(ctx, nkeys);
    sort_keys(ctx, keys.p, sorted.p, nkeys, (int)(2 * b));
    keys.reset();
    uniq = DevBuf<uint64_t>(ctx, nkeys);
    DevBuf<uint64_t> nsel(ctx, 2);
    size_t tmp = 0;
    GAMMA_CUDA(cub::DeviceSelect::Unique(nullptr, tmp, sorted.p, uniq.p, nsel.p, (int64_t)nkeys, ctx->stream));
    {
      DevBuf<uint8_t> t(ctx, tmp);
      ctx->launch(KC_BUILD, [&] {
        GAMMA_CUDA(cub::DeviceSelect::Unique(t.p, tmp, sorted.p, uniq.p, nsel.p, (int64_t)nkeys, ctx->stream));
      });
      ctx->cub_select_launched(KC_BUILD);
    }
    uint64_t h[2] = {0, 0};
    GAMMA_CUDA(cudaMemcpyAsync(&h[0], nsel.p, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
    GAMMA_CUDA(cudaMemcpyAsync(&h[1], ctx->ctrl + CTRL_ERR, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
    ctx->sync();
    GAMMA_REQUIRE(h[1] == 0, GAMMA_E_INVAL, "gamma_load_edges: vertex id >= n");
    M = h[0];
    if (M) {  // drop the (single, last) invalid key if present
      uint64_t last = 0;
      GAMMA_CUDA(cudaMemcpyAsync(&last, uniq.p + M - 1, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
      ctx->sync();
      const uint64_t invalid = (b >= 32) ? ~0ull : ((1ull << (2 * b)) - 1);
      if (last == invalid) M--;
    }
  }
  GAMMA_REQUIRE(M % 2 == 0, GAMMA_E_CUDA, "asymmetric key set after unique");
  g->m = M / 2;
  DevBuf<uint64_t> rp(ctx, (size_t)n + 1);
  DevBuf<uint32_t> col(ctx, M ? M : 1);
  keys_to_csr(ctx, uniq.p, M, n, b, rp.p, col.p);
  g->row_ptr = rp.release();
  g->col = col.release();
  g->device_bytes += ((uint64_t)n + 1) * 8 + M * 4;
  g->max_degree = max_degree(ctx, g->row_ptr, n);
  build_dag(g, uniq.p, M);
  rank_dag(g);
  if (ctx->desc.flags & GAMMA_FLAG_HOST_DAG) host_dag(g, ctx->desc.dag_cache_bytes);
  g->build_ms = timer.stop();
}

void build_from_csr(gamma_graph *g, const uint64_t *row_ptr, const uint32_t *col) {
  gamma_ctx *ctx = g->ctx;
  BuildTimer timer(ctx);
  const uint32_t n = g->n;
  g->bits = bit_width(n);
  DevBuf<uint64_t> rp = to_device(ctx, row_ptr, (size_t)n + 1);
  uint64_t M = 0, first = 0;
  GAMMA_CUDA(cudaMemcpyAsync(&first, rp.p, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
  GAMMA_CUDA(cudaMemcpyAsync(&M, rp.p + n, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
  ctx->sync();
  GAMMA_REQUIRE(first == 0, GAMMA_E_INVAL, "gamma_load_csr: row_ptr[0] != 0");
  GAMMA_REQUIRE(M % 2 == 0, GAMMA_E_INVAL, "gamma_load_csr: odd number of directed edges");
  GAMMA_REQUIRE(M == 0 || col, GAMMA_E_INVAL, "gamma_load_csr: NULL col");
  DevBuf<uint32_t> cl = to_device(ctx, col, M ? M : 0);
  if (!M) cl = DevBuf<uint32_t>(ctx, 1);
  DevBuf<uint64_t> keys(ctx, M ? M : 1);
  GAMMA_CUDA(cudaMemsetAsync(ctx->ctrl + CTRL_ERR, 0, sizeof(uint64_t), ctx->stream));
  unsigned grid = grid_for((uint64_t)n * 32);
  if (M) {
    ctx->launch(KC_BUILD, [&] {
      csr_to_keys_kernel<<<grid, kThreads, 0, ctx->stream>>>(rp.p, cl.p, n, g->bits, keys.p,
                                                             (unsigned long long *)(ctx->ctrl + CTRL_ERR));
    });
    uint64_t err = 0;
    GAMMA_CUDA(cudaMemcpyAsync(&err, ctx->ctrl + CTRL_ERR, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
    ctx->sync();
    GAMMA_REQUIRE(err == 0, GAMMA_E_INVAL, "gamma_load_csr: list not strictly ascending, self-loop, or id >= n");
    ctx->launch(KC_BUILD, [&] {
      csr_symmetry_kernel<<<grid, kThreads, 0, ctx->stream>>>(rp.p, cl.p, n,
                                                              (unsigned long long *)(ctx->ctrl + CTRL_ERR));
    });
    GAMMA_CUDA(cudaMemcpyAsync(&err, ctx->ctrl + CTRL_ERR, sizeof(uint64_t), cudaMemcpyDeviceToHost, ctx->stream));
    ctx->sync();
    GAMMA_REQUIRE(err == 0, GAMMA_E_INVAL, "gamma_load_csr: adjacency is not symmetric");
  }
  g->m = M / 2;
  g->row_ptr = rp.release();
  g->col = cl.release();
  g->device_bytes += ((uint64_t)n + 1) * 8 + M * 4;
  g->max_degree = max_degree(ctx, g->row_ptr, n);
  build_dag(g, keys.p, M);
  rank_dag(g);
  if (ctx->desc.flags & GAMMA_FLAG_HOST_DAG) host_dag(g, ctx->desc.dag_cache_bytes);
  g->build_ms = timer.stop();
}

}  // namespace gamma_impl
