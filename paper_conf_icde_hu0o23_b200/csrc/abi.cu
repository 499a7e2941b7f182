// abi.cu -- the extern "C" entry points of include/gamma.h, the context (stream,
// allocator, control block, launch timing) and argument validation.  Compute lives
// in graph.cu (A1), kclique.cu (A2-A8 kCL), match.cu (SM) and fpm.cu (FPM).
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstring>
#include <new>
#include <string>

#include "internal.cuh"

namespace gamma_impl {

static thread_local std::string g_err;
void set_error(const std::string &msg) { g_err = msg; }
void clear_error() { g_err.clear(); }

const char *kKernelClassName[KC_NUM] = {"build",  "roots",     "extend", "count",
                                        "fused",  "sm_extend", "sm_count", "fpm",
                                        "fpm_support", "misc", "bitmap"};

bool is_device_ptr(const void *ptr) {
  if (!ptr) return false;
  cudaPointerAttributes a;
  cudaError_t e = cudaPointerGetAttributes(&a, ptr);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

void ctrl_reset(gamma_ctx *ctx) {
  GAMMA_CUDA(cudaMemsetAsync(ctx->ctrl, 0, CTRL_WORDS * sizeof(uint64_t), ctx->stream));
}

void ctrl_fetch(gamma_ctx *ctx) {
  GAMMA_CUDA(cudaMemcpyAsync(ctx->ctrl_host, ctx->ctrl, CTRL_WORDS * sizeof(uint64_t),
                             cudaMemcpyDeviceToHost, ctx->stream));
  ctx->sync();
}

int occupancy_blocks(const void *kernel, int threads, size_t smem) {
  int b = 0;
  GAMMA_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kernel, threads, smem));
  return b > 0 ? b : 1;
}

uint64_t checked_add(uint64_t a, uint64_t b) {
  uint64_t r;
  if (__builtin_add_overflow(a, b, &r)) throw Fail{GAMMA_E_OVERFLOW, "uint64 count overflow"};
  return r;
}

}  // namespace gamma_impl

using namespace gamma_impl;

void *gamma_ctx::alloc(size_t bytes) {
  void *p = nullptr;
  if (desc.dev_alloc) {
    p = desc.dev_alloc(bytes, (void *)stream, desc.alloc_user);
    if (!p) throw Fail{GAMMA_E_NOMEM, "device allocation of " + std::to_string(bytes) + " bytes failed"};
    return p;
  }
  cudaError_t e = cudaMallocAsync(&p, bytes, stream);
  if (e != cudaSuccess) {
    cudaGetLastError();
    throw Fail{GAMMA_E_NOMEM, "cudaMallocAsync(" + std::to_string(bytes) + "): " + cudaGetErrorString(e)};
  }
  return p;
}

void *gamma_ctx::keep_take(size_t bytes, size_t &got) {
  size_t best = kept.size();
  for (size_t i = 0; i < kept.size(); i++)
    if (kept[i].second >= bytes && (best == kept.size() || kept[i].second < kept[best].second)) best = i;
  if (best < kept.size()) {
    void *p = kept[best].first;
    got = kept[best].second;
    kept.erase(kept.begin() + best);
    return p;
  }
  got = bytes;
  return alloc(bytes);
}

// Kept bytes are capped at an eighth of the device memory: beyond it a returned buffer
// is freed instead (an idle context must not starve other processes on the GPU).  (Round 1's 8 GiB held a fraction of a batched SM call's tables --
// eight level chains of up to three levels -- so every C3 step re-allocated most of
// them through the caching allocator.)
void gamma_ctx::keep_give(void *p, size_t bytes) {
  if (!p) return;
  size_t held = 0;
  for (auto &b : kept) held += b.second;
  if (held + bytes > mem_total / 8) {
    free(p);
    return;
  }
  kept.emplace_back(p, bytes);
}

void gamma_ctx::keep_release() {
  for (auto &b : kept) free(b.first);
  kept.clear();
}

// Before a graph build: release the kept buffers only when less than half of the
// device memory is free (the build's scratch scales with the input).
void gamma_ctx::keep_release_if_tight() {
  if (kept.empty()) return;
  size_t fr = 0, tot = 0;
  if (cudaMemGetInfo(&fr, &tot) != cudaSuccess || fr < tot / 2) keep_release();
}

void gamma_ctx::free(void *p) {
  if (!p) return;
  if (desc.dev_free) desc.dev_free(p, desc.alloc_user);
  else cudaFreeAsync(p, stream);
}

void gamma_ctx::side_init() {
  if (!side_ctrl) {
    GAMMA_CUDA(cudaMalloc(&side_ctrl, kMaxBatch * CTRL_WORDS * sizeof(uint64_t)));
    GAMMA_CUDA(cudaMallocHost(&side_ctrl_host, kMaxBatch * CTRL_WORDS * sizeof(uint64_t)));
  }
  while (side_streams.size() < (size_t)kMaxBatch) {
    cudaStream_t st;
    GAMMA_CUDA(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
    side_streams.push_back(st);
  }
}

void gamma_ctx::reset_stats() {
  pending.clear();
  ev_next = 0;
  std::memset(&stats, 0, sizeof(stats));
  stats.n_classes = KC_NUM;
  for (int i = 0; i < KC_NUM; i++) std::strncpy(stats.name[i], kKernelClassName[i], 31);
}

cudaEvent_t gamma_ctx::next_event() {
  if (ev_next == ev_pool.size()) {
    cudaEvent_t e;
    GAMMA_CUDA(cudaEventCreate(&e));
    ev_pool.push_back(e);
  }
  return ev_pool[ev_next++];
}

void gamma_ctx::collect_timings() {
  for (auto &p : pending) {
    float ms = 0;
    if (cudaEventElapsedTime(&ms, p.second.first, p.second.second) == cudaSuccess)
      stats.ms[p.first] += ms;
    else
      cudaGetLastError();
  }
  pending.clear();
  ev_next = 0;
}

// ------------------------------------------------------------------------------------
extern "C" {

int32_t gamma_abi_version(void) { return GAMMA_ABI_VERSION; }

const char *gamma_last_error(void) { return g_err.c_str(); }

gamma_status gamma_ctx_create(const gamma_ctx_desc *desc, gamma_ctx **out) {
  return guarded([&] {
    GAMMA_REQUIRE(desc && out, GAMMA_E_INVAL, "gamma_ctx_create: NULL argument");
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess || ndev == 0) {
      cudaGetLastError();
      throw Fail{GAMMA_E_CUDA, "no CUDA device available (there is no CPU fallback)"};
    }
    GAMMA_REQUIRE(desc->device >= 0 && desc->device < ndev, GAMMA_E_INVAL, "bad device ordinal");
    GAMMA_REQUIRE((desc->dev_alloc == nullptr) == (desc->dev_free == nullptr), GAMMA_E_INVAL,
                  "dev_alloc and dev_free must be given together");
    auto *c = new gamma_ctx();
    c->desc = *desc;
    if (c->desc.world < 1) c->desc.world = 1;
    if (c->desc.rank < 0 || c->desc.rank >= c->desc.world) {
      delete c;
      throw Fail{GAMMA_E_INVAL, "rank must be in [0, world)"};
    }
    c->device = desc->device;
    try {
      GAMMA_CUDA(cudaSetDevice(c->device));
      cudaDeviceProp prop;
      GAMMA_CUDA(cudaGetDeviceProperties(&prop, c->device));
      c->num_sms = prop.multiProcessorCount;
      c->mem_total = prop.totalGlobalMem;
      c->smem_optin = prop.sharedMemPerBlockOptin;
      if (desc->stream) {
        c->stream = (cudaStream_t)desc->stream;
      } else {
        GAMMA_CUDA(cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking));
        c->own_stream = true;
      }
      if (!desc->dev_alloc) {   // native allocation: keep freed blocks in the stream-ordered
        cudaMemPool_t pool;     // pool across synchronisations (default threshold 0 trims them)
        GAMMA_CUDA(cudaDeviceGetDefaultMemPool(&pool, c->device));
        uint64_t keep = ~0ull;
        GAMMA_CUDA(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep));
      }
      GAMMA_CUDA(cudaMalloc(&c->ctrl, CTRL_WORDS * sizeof(uint64_t)));
      GAMMA_CUDA(cudaMallocHost(&c->ctrl_host, CTRL_WORDS * sizeof(uint64_t)));
      c->reset_stats();
    } catch (...) {
      gamma_ctx_destroy(c);
      throw;
    }
    *out = c;
  });
}

void gamma_ctx_destroy(gamma_ctx *ctx) {
  if (!ctx) return;
  cudaSetDevice(ctx->device);
  if (ctx->stream) cudaStreamSynchronize(ctx->stream);
  try {
    ctx->keep_release();
  } catch (...) {
  }
  if (ctx->ctrl) cudaFree(ctx->ctrl);
  if (ctx->ctrl_host) cudaFreeHost(ctx->ctrl_host);
  if (ctx->spill_host) cudaFreeHost(ctx->spill_host);
  if (ctx->copy_stream) cudaStreamDestroy(ctx->copy_stream);
  for (auto st : ctx->side_streams) cudaStreamDestroy(st);
  if (ctx->side_ctrl) cudaFree(ctx->side_ctrl);
  if (ctx->side_ctrl_host) cudaFreeHost(ctx->side_ctrl_host);
  for (auto e : ctx->ev_pool) cudaEventDestroy(e);
  if (ctx->own_stream && ctx->stream) cudaStreamDestroy(ctx->stream);
  cudaGetLastError();
  delete ctx;
}

gamma_status gamma_ctx_trim(gamma_ctx *ctx) {
  return guarded([&] {
    GAMMA_REQUIRE(ctx, GAMMA_E_INVAL, "gamma_ctx_trim: NULL argument");
    GAMMA_CUDA(cudaSetDevice(ctx->device));
    ctx->keep_release();
    GAMMA_CUDA(cudaStreamSynchronize(ctx->stream));
  });
}

gamma_status gamma_get_stats(const gamma_ctx *ctx, gamma_run_stats *out) {
  return guarded([&] {
    GAMMA_REQUIRE(ctx && out, GAMMA_E_INVAL, "gamma_get_stats: NULL argument");
    *out = ctx->stats;
  });
}

gamma_status gamma_load_edges(gamma_ctx *ctx, uint32_t n, const uint32_t *src, const uint32_t *dst,
                              uint64_t m, const uint32_t *labels, gamma_graph **out) {
  return guarded([&] {
    GAMMA_REQUIRE(ctx && out, GAMMA_E_INVAL, "gamma_load_edges: NULL argument");
    GAMMA_REQUIRE(n > 0, GAMMA_E_INVAL, "gamma_load_edges: n must be > 0");
    GAMMA_REQUIRE(m == 0 || (src && dst), GAMMA_E_INVAL, "gamma_load_edges: NULL src/dst");
    GAMMA_REQUIRE(n < 0xFFFFFFFFu, GAMMA_E_INVAL, "gamma_load_edges: n too large");
    GAMMA_CUDA(cudaSetDevice(ctx->device));
    ctx->reset_stats();
    ctx->keep_release_if_tight();   // the build needs room; kept SM tables only when it is there
    auto *g = new gamma_graph();
    g->ctx = ctx;
    g->n = n;
    try {
      if (labels) {
        DevBuf<uint32_t> l = to_device(ctx, labels, n);
        g->labels = l.release();
        g->device_bytes += sizeof(uint32_t) * (uint64_t)n;
      }
      build_from_edges(g, src, dst, m, is_device_ptr(src) && is_device_ptr(dst));
    } catch (...) {
      gamma_graph_free(g);
      throw;
    }
    *out = g;
  });
}

gamma_status gamma_load_csr(gamma_ctx *ctx, uint32_t n, const uint64_t *row_ptr, const uint32_t *col,
                            const uint32_t *labels, gamma_graph **out) {
  return guarded([&] {
    GAMMA_REQUIRE(ctx && out && row_ptr, GAMMA_E_INVAL, "gamma_load_csr: NULL argument");
    GAMMA_REQUIRE(n > 0 && n < 0xFFFFFFFFu, GAMMA_E_INVAL, "gamma_load_csr: bad n");
    GAMMA_CUDA(cudaSetDevice(ctx->device));
    ctx->reset_stats();
    ctx->keep_release_if_tight();
    auto *g = new gamma_graph();
    g->ctx = ctx;
    g->n = n;
    try {
      if (labels) {
        DevBuf<uint32_t> l = to_device(ctx, labels, n);
        g->labels = l.release();
        g->device_bytes += sizeof(uint32_t) * (uint64_t)n;
      }
      build_from_csr(g, row_ptr, col);
    } catch (...) {
      gamma_graph_free(g);
      throw;
    }
    *out = g;
  });
}

void gamma_graph_free(gamma_graph *g) {
  if (!g) return;
  gamma_ctx *c = g->ctx;
  if (c) {
    cudaSetDevice(c->device);
    c->free(g->row_ptr);
    c->free(g->col);
    c->free(g->dag_ptr);
    c->free(g->dag_col);
    c->free(g->labels);
    c->free(g->root_order);
    c->free(g->rank_of);
    c->free(g->ldeg);
    c->free(g->dag_pages);
    c->free(g->dag_cache);
    // (kept SM tables stay with the context: their sizes come from the budget and the
    // level caps, not from this graph, and the next graph's SM calls take them back
    // without an allocator round trip)
    cudaStreamSynchronize(c->stream);
  }
  if (g->dag_host) cudaFreeHost(g->dag_host);
  cudaGetLastError();
  delete g;
}

gamma_status gamma_graph_get_info(const gamma_graph *g, gamma_graph_info *info) {
  return guarded([&] {
    GAMMA_REQUIRE(g && info, GAMMA_E_INVAL, "gamma_graph_get_info: NULL argument");
    info->n = g->n;
    info->m = g->m;
    info->max_degree = g->max_degree;
    info->max_out_degree = g->max_out_degree;
    info->device_bytes = g->device_bytes;
    info->build_ms = g->build_ms;
  });
}

gamma_status gamma_graph_copy_csr(const gamma_graph *g, int which, uint64_t *row_ptr, uint32_t *col) {
  return guarded([&] {
    GAMMA_REQUIRE(g && row_ptr && (col || g->m == 0), GAMMA_E_INVAL, "gamma_graph_copy_csr: NULL argument");
    GAMMA_REQUIRE(which == 0 || which == 1, GAMMA_E_INVAL, "which must be 0 (symmetric) or 1 (DAG)");
    gamma_ctx *c = g->ctx;
    GAMMA_CUDA(cudaSetDevice(c->device));
    if (which == 1) {   // the kCL DAG lives in rank space: export it in id space
      export_dag_ids(const_cast<gamma_graph *>(g), row_ptr, col);
      return;
    }
    const uint64_t ne = 2 * g->m;
    GAMMA_CUDA(cudaMemcpyAsync(row_ptr, g->row_ptr, ((size_t)g->n + 1) * sizeof(uint64_t), cudaMemcpyDefault,
                               c->stream));
    if (ne) GAMMA_CUDA(cudaMemcpyAsync(col, g->col, ne * sizeof(uint32_t), cudaMemcpyDefault, c->stream));
    c->sync();
  });
}

gamma_status gamma_kclique(gamma_graph *g, uint32_t k, uint64_t *count) {
  return guarded([&] {
    GAMMA_REQUIRE(g && count, GAMMA_E_INVAL, "gamma_kclique: NULL argument");
    GAMMA_REQUIRE(k >= 1, GAMMA_E_INVAL, "gamma_kclique: k must be >= 1");
    GAMMA_REQUIRE(k <= 32, GAMMA_E_UNSUPPORTED, "gamma_kclique: k > 32 unsupported");
    gamma_ctx *c = g->ctx;
    GAMMA_CUDA(cudaSetDevice(c->device));
    c->reset_stats();
    c->keep_release();   // kCL sizes its levels from free HBM
    auto t0 = std::chrono::steady_clock::now();
    uint64_t r = kclique_count(g, k, nullptr, 0, nullptr);
    if (c->desc.world > 1 && c->desc.allreduce_sum_u64) {
      gamma_status st = c->desc.allreduce_sum_u64(&r, 1, c->desc.coll_user);
      GAMMA_REQUIRE(st == GAMMA_OK, st, "allreduce_sum_u64 callback failed");
    }
    c->stats.wall_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    *count = r;
  });
}

gamma_status gamma_kclique_multi(gamma_graph *g, uint32_t nk, const uint32_t *ks, uint64_t *counts) {
  return guarded([&] {
    GAMMA_REQUIRE(g && (nk == 0 || (ks && counts)), GAMMA_E_INVAL, "gamma_kclique_multi: NULL argument");
    uint32_t kmax = 0, kmin = 0xffffffffu;
    for (uint32_t i = 0; i < nk; i++) {
      GAMMA_REQUIRE(ks[i] >= 1, GAMMA_E_INVAL, "gamma_kclique_multi: k must be >= 1");
      GAMMA_REQUIRE(ks[i] <= 32, GAMMA_E_UNSUPPORTED, "gamma_kclique_multi: k > 32 unsupported");
      kmax = std::max(kmax, ks[i]);
      if (ks[i] >= 3) kmin = std::min(kmin, ks[i]);
    }
    gamma_ctx *c = g->ctx;
    GAMMA_CUDA(cudaSetDevice(c->device));
    c->reset_stats();
    c->keep_release();   // kCL sizes its levels from free HBM
    if (nk == 0) return;
    auto t0 = std::chrono::steady_clock::now();
    uint64_t bysize[33] = {};
    const bool one_pass = kmax >= 3 && kclique_multi(g, kmin, kmax, bysize);
    std::vector<uint64_t> r(nk);
    for (uint32_t i = 0; i < nk; i++)
      r[i] = (one_pass && ks[i] >= 3) ? bysize[ks[i]] : kclique_count(g, ks[i], nullptr, 0, nullptr);
    if (c->desc.world > 1 && c->desc.allreduce_sum_u64) {
      gamma_status st = c->desc.allreduce_sum_u64(r.data(), nk, c->desc.coll_user);
      GAMMA_REQUIRE(st == GAMMA_OK, st, "allreduce_sum_u64 callback failed");
    }
    c->stats.wall_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    for (uint32_t i = 0; i < nk; i++) counts[i] = r[i];
  });
}

gamma_status gamma_kclique_roots(gamma_graph *g, uint32_t k, uint64_t nroots, const uint32_t *roots,
                                 uint64_t *counts) {
  return guarded([&] {
    GAMMA_REQUIRE(g && (nroots == 0 || (roots && counts)), GAMMA_E_INVAL, "gamma_kclique_roots: NULL argument");
    GAMMA_REQUIRE(k >= 1, GAMMA_E_INVAL, "gamma_kclique_roots: k must be >= 1");
    GAMMA_REQUIRE(k <= 32, GAMMA_E_UNSUPPORTED, "gamma_kclique_roots: k > 32 unsupported");
    gamma_ctx *c = g->ctx;
    GAMMA_CUDA(cudaSetDevice(c->device));
    c->reset_stats();
    c->keep_release();   // kCL sizes its levels from free HBM
    if (nroots == 0) return;
    DevBuf<uint32_t> r = to_device(c, roots, nroots);
    to_rank_space(g, r.p, nroots);   // the kCL DAG is in rank space (graph.cu rank_dag)
    DevBuf<uint64_t> out(c, nroots);
    GAMMA_CUDA(cudaMemsetAsync(out.p, 0, nroots * sizeof(uint64_t), c->stream));
    kclique_count(g, k, r.p, nroots, out.p);
    GAMMA_CUDA(cudaMemcpyAsync(counts, out.p, nroots * sizeof(uint64_t), cudaMemcpyDefault, c->stream));
    c->sync();
  });
}

}  // extern "C"
