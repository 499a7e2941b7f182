// internal.cuh -- shared internals of libgamma (CUDA side only; never included by
// oracle/).  Context, graph, error plumbing, device allocation, launch timing.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "gamma.h"

namespace gamma_impl {

// ---- thread-local error message -------------------------------------------------
void set_error(const std::string &msg);
void clear_error();

struct Fail {
  gamma_status st;
  std::string msg;
};

#define GAMMA_CUDA(expr)                                                              \
  do {                                                                                \
    cudaError_t e_ = (expr);                                                          \
    if (e_ != cudaSuccess)                                                            \
      throw ::gamma_impl::Fail{GAMMA_E_CUDA, std::string(#expr) + ": " +              \
                                                 cudaGetErrorString(e_)};             \
  } while (0)

#define GAMMA_REQUIRE(cond, status, msg)                                              \
  do {                                                                                \
    if (!(cond)) throw ::gamma_impl::Fail{(status), (msg)};                           \
  } while (0)

// Runs f(), converting Fail / std exceptions into a status + thread-local message.
template <class F>
gamma_status guarded(F &&f) {
  try {
    clear_error();
    f();
    return GAMMA_OK;
  } catch (const Fail &e) {
    set_error(e.msg);
    return e.st;
  } catch (const std::bad_alloc &) {
    set_error("host allocation failed");
    return GAMMA_E_NOMEM;
  } catch (const std::exception &e) {
    set_error(e.what());
    return GAMMA_E_INVAL;
  } catch (...) {
    set_error("unknown error");
    return GAMMA_E_INVAL;
  }
}

// ---- per-kernel-class statistics -------------------------------------------------
enum KernelClass {
  KC_BUILD = 0,      // A1 CSR/DAG build kernels (incl. CUB sort)
  KC_ROOTS,          // A2 root list / cost / partition
  KC_EXTEND,         // A3-A6 extend (stage + intersect + filter + compact + write)
  KC_COUNT,          // A4+A7 last-level intersect-and-count
  KC_FUSED,          // A3-A7 fused last two levels (DFS tail)
  KC_SM_EXTEND,      // SM extend
  KC_SM_COUNT,       // SM last level
  KC_FPM,            // FPM edge extension / canonical code / domain bits
  KC_FPM_SUPPORT,    // FPM popc / min over orbits
  KC_MISC,           // memsets, small helpers
  KC_BITMAP,         // kCL local-bitmap path (depth-2 list intersection + bitmap DFS)
  KC_NUM
};
extern const char *kKernelClassName[KC_NUM];

struct Ctrl;  // device control block (counters), defined in ctx.cu

struct gamma_ctx_impl;
}  // namespace gamma_impl

struct gamma_ctx {
  gamma_ctx_desc desc;
  int device = 0;
  int num_sms = 148;
  size_t mem_total = 0;   // device memory (bytes), read once at creation
  size_t smem_optin = 0;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  // device control block: counters reset per launch
  uint64_t *ctrl = nullptr;  // CTRL_WORDS u64 on device
  uint64_t *ctrl_host = nullptr;  // pinned mirror
  // pinned host arena for spilled ET levels (GAMMA_FLAG_SPILL), used as a stack
  uint8_t *spill_host = nullptr;
  size_t spill_cap = 0, spill_top = 0;
  // second stream for the spill copies (created on first use, non-blocking)
  cudaStream_t copy_stream = nullptr;
  cudaStream_t copy_stream_get() {
    if (!copy_stream) GAMMA_CUDA(cudaStreamCreateWithFlags(&copy_stream, cudaStreamNonBlocking));
    return copy_stream;
  }
  // stats of the last call
  gamma_run_stats stats;
  // event pool for kernel timing
  std::vector<cudaEvent_t> ev_pool;
  std::vector<std::pair<int, std::pair<cudaEvent_t, cudaEvent_t>>> pending;
  size_t ev_next = 0;

  void *alloc(size_t bytes);
  void free(void *p);
  // Idle device buffers kept across calls (SM level tables and L_m scratch): sizing them
  // from free HBM per call made consecutive calls ask the allocator for different sizes.
  std::vector<std::pair<void *, size_t>> kept;
  void *keep_take(size_t bytes, size_t &got);   // smallest kept buffer >= bytes, else alloc
  void keep_give(void *p, size_t bytes);
  void keep_release();                          // free every kept buffer
  void keep_release_if_tight();                 // ... when less than half the HBM is free
  void reset_stats();
  // Launch helper: brackets the launch with events when timing is on.
  template <class F>
  void launch(int kc, F &&f) {
    launch_on(kc, stream, f);
  }
  // the same on another stream of this context (batched SM queries)
  template <class F>
  void launch_on(int kc, cudaStream_t s, F &&f) {
    cudaEvent_t a = nullptr, b = nullptr;
    bool timing = (desc.flags & GAMMA_FLAG_TIME_KERNELS) != 0;
    if (timing) {
      a = next_event();
      b = next_event();
      cudaEventRecord(a, s);
    }
    f();
    GAMMA_CUDA(cudaGetLastError());
    if (timing) {
      cudaEventRecord(b, s);
      pending.push_back({kc, {a, b}});
    }
    stats.launches[kc]++;
    stats.total_launches++;
  }
  // side streams and pinned control mirrors for batched queries (created on first use)
  std::vector<cudaStream_t> side_streams;
  uint64_t *side_ctrl = nullptr, *side_ctrl_host = nullptr;   // kMaxBatch x CTRL_WORDS
  static constexpr int kMaxBatch = 16;
  void side_init();
  // Library calls (CUB) that launch several kernels inside one ctx->launch(): add the
  // kernels beyond the first so total_launches matches the launch list.
  void extra_launches(int kc, uint64_t n) {
    stats.launches[kc] += n;
    stats.total_launches += n;
  }
  // CUB onesweep radix sort: histogram + exclusive-sum + one pass per 8 key bits
  // (a single-tile kernel for tiny inputs); DeviceSelect: init + sweep.
  void cub_sort_launched(int kc, uint64_t items, int bits) {
    extra_launches(kc, items <= 4096 ? 0 : 1 + (uint64_t)((bits + 7) / 8));
  }
  void cub_select_launched(int kc) { extra_launches(kc, 1); }
  cudaEvent_t next_event();
  void collect_timings();  // after a stream sync
  void sync() { GAMMA_CUDA(cudaStreamSynchronize(stream)); }
};

// control block layout (u64 words)
enum {
  CTRL_WORK = 0,      // dynamic work counter
  CTRL_VCUR = 1,      // vid cursor of the level being written
  CTRL_GCUR = 2,      // group cursor of the level being written
  CTRL_OVF = 3,       // overflow flag
  CTRL_COUNT = 4,     // result accumulator
  CTRL_ELEMS = 5,     // adjacency elements fetched (algorithmic)
  CTRL_ENTRIES = 6,   // entries produced (kept)
  CTRL_ERR = 7,       // validation error flag
  CTRL_AUX0 = 8,
  CTRL_AUX1 = 9,
  CTRL_AUX2 = 10,
  CTRL_WORK2 = 11,    // a second work counter (a launch running concurrently with another)
  CTRL_MULTI = 16,    // CTRL_MULTI + s: number of s-cliques (gamma_kclique_multi), s <= 32
  CTRL_LEVELS = 64,   // CTRL_LEVELS + CTRL_LSTRIDE * d: a per-level control block (same word
  CTRL_LSTRIDE = 16,  // offsets as above) for launch chains read back once (match.cu)
  CTRL_WORDS = 64 + 16 * 12
};

struct gamma_graph {
  gamma_ctx *ctx = nullptr;
  uint32_t n = 0;
  uint64_t m = 0;
  uint32_t bits = 1;             // bits needed for a vertex id (ids < 2^bits)
  uint64_t *row_ptr = nullptr;   // n+1
  uint32_t *col = nullptr;       // 2m
  // kCL DAG in RANK space (graph.cu rank_dag): vertex r = the r-th vertex in the
  // (degree, id) order; lists ascending (= by rank); rank_of maps an id to its rank
  uint64_t *dag_ptr = nullptr;   // n+1
  uint32_t *dag_col = nullptr;   // m
  uint32_t *rank_of = nullptr;   // n
  bool rank_space = false;       // the DAG ids are ranks (GAMMA_RANK_DAG=1), else ids (rank_of = identity)
  // SM filters: label << 24 | min(degree, 2^24 - 1) per vertex, built on the first
  // gamma_match when every label is < 256 (ldeg_state: -1 not yet, 0 unusable, 1 built)
  uint32_t *ldeg = nullptr;
  int32_t ldeg_state = -1;
  // GAMMA_FLAG_HOST_DAG (graph.cu host_dag): dag_col is freed; its 2^kDagPageShift-entry
  // pages live in pinned host memory (dag_host, mapped) or in the HBM cache
  // (dag_cache); dag_pages[p] = the device address of page p's first entry
  uint64_t *dag_pages = nullptr;
  uint32_t *dag_host = nullptr, *dag_cache = nullptr;
  uint64_t dag_npages = 0, dag_cached = 0;
  uint32_t *labels = nullptr;    // n (nullptr: unlabeled, all 0)
  uint32_t max_degree = 0, max_out_degree = 0;
  uint64_t device_bytes = 0;
  double build_ms = 0;
  // kCL root order cache (kclique.cu ensure_root_order): this rank's vertices sorted by
  // d+ descending, and root_ge[t] = how many of them have d+ >= t
  uint32_t *root_order = nullptr;
  std::vector<uint64_t> root_ge;
  int32_t root_rank = -1, root_world = -1;
};

// RAII device buffer through the ctx allocator.
template <class T>
struct DevBuf {
  gamma_ctx *ctx = nullptr;
  T *p = nullptr;
  size_t n = 0;
  size_t bytes = 0;   // kept buffers: the size actually held
  bool kept = false;  // taken from / returned to the context's kept-buffer list
  DevBuf() = default;
  DevBuf(gamma_ctx *c, size_t count) : ctx(c), n(count) {
    p = static_cast<T *>(c->alloc(count * sizeof(T) ? count * sizeof(T) : 16));
  }
  // kept = true: reuse an idle buffer of >= count elements kept by the context from an
  // earlier call (no allocator round trip), and keep this one when it is released
  DevBuf(gamma_ctx *c, size_t count, bool keep) : ctx(c), n(count), kept(keep) {
    const size_t want = count * sizeof(T) ? count * sizeof(T) : 16;
    p = static_cast<T *>(keep ? c->keep_take(want, bytes) : c->alloc(want));
  }
  DevBuf(const DevBuf &) = delete;
  DevBuf &operator=(const DevBuf &) = delete;
  DevBuf(DevBuf &&o) noexcept : ctx(o.ctx), p(o.p), n(o.n), bytes(o.bytes), kept(o.kept) { o.p = nullptr; }
  DevBuf &operator=(DevBuf &&o) noexcept {
    reset();
    ctx = o.ctx; p = o.p; n = o.n; bytes = o.bytes; kept = o.kept; o.p = nullptr;
    return *this;
  }
  ~DevBuf() { reset(); }
  void reset() {
    if (p && ctx) {
      if (kept) ctx->keep_give(p, bytes);
      else ctx->free(p);
    }
    p = nullptr;
  }
  T *release() { T *q = p; p = nullptr; return q; }
};

namespace gamma_impl {
// Is ptr a device (or managed) pointer usable by kernels?
bool is_device_ptr(const void *ptr);
// Copy n elements of an input array (host or device) into a fresh device buffer.
template <class T>
DevBuf<T> to_device(gamma_ctx *ctx, const T *src, size_t n) {
  DevBuf<T> d(ctx, n);
  if (n) GAMMA_CUDA(cudaMemcpyAsync(d.p, src, n * sizeof(T), cudaMemcpyDefault, ctx->stream));
  return d;
}
void ctrl_reset(gamma_ctx *ctx);                 // zero all control words (async)
void ctrl_fetch(gamma_ctx *ctx);                 // async D2H into ctrl_host + sync
int occupancy_blocks(const void *kernel, int threads, size_t smem);
uint64_t checked_add(uint64_t a, uint64_t b);    // throws E_OVERFLOW

// A1: builders (graph.cu)
void build_from_edges(gamma_graph *g, const uint32_t *src, const uint32_t *dst, uint64_t m,
                      bool src_on_device);
void build_from_csr(gamma_graph *g, const uint64_t *row_ptr, const uint32_t *col);
void build_dag(gamma_graph *g, uint64_t *sorted_keys_dev, uint64_t nkeys);
void rank_dag(gamma_graph *g);                       // id-space DAG -> rank space (+ rank_of)
void export_dag_ids(gamma_graph *g, uint64_t *dag_ptr_out, uint32_t *dag_col_out);
void to_rank_space(gamma_graph *g, uint32_t *ids_dev, uint64_t nids);   // in place, on the stream
constexpr uint32_t kDagPageShift = 14;   // 64 KiB pages of the host-resident DAG
void host_dag(gamma_graph *g, uint64_t cache_bytes);   // GAMMA_FLAG_HOST_DAG (graph.cu)

// kCL (kclique.cu)
uint64_t kclique_count(gamma_graph *g, uint32_t k, const uint32_t *roots_dev, uint64_t nroots,
                       uint64_t *per_root_dev);
// kCL local-bitmap path for roots with |N+(v)| <= kBitmapMaxRun (kclique_bitmap.cu)
constexpr uint32_t kBitmapMaxRun = 512;     // shared-memory rows up to here
constexpr uint32_t kWideMaxRun = 8192;      // global-scratch rows ("wide") up to here
constexpr uint32_t kBitmapMaxK = 12;
uint64_t kclique_bitmap(gamma_graph *g, uint32_t k, const uint32_t *roots, uint64_t nroots,
                        unsigned long long *per_root, bool sorted, uint64_t n_xl, uint64_t n_long, uint64_t n_mid,
                        uint64_t *multi_out = nullptr, uint32_t kmin = 3);
// One bitmap pass counting every clique size kmin..kmax (multi_out[s], kmin <= s <= kmax;
// kmin >= 3: roots with d+ < kmin - 1 hold no such clique and are skipped); false
// when the graph needs the ET path (max out-degree > kWideMaxRun or kmax too big).
bool kclique_multi(gamma_graph *g, uint32_t kmin, uint32_t kmax, uint64_t *multi_out);
void ensure_root_order(gamma_graph *g);
}  // namespace gamma_impl
