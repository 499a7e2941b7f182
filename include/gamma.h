/*
 * gamma.h -- C ABI of the B200-native GAMMA hot path (embedding-table extension).
 *
 * What the calls compute (PAPER.md = /root/reference/PAPER.md, line numbers):
 *   gamma_kclique  k-clique counting, the kCL task of PAPER.md L15, L269, L449, run
 *                  as vertex extension (Def. 3.1) with early pruning to
 *                  common neighbours (L146) over a degree-ordered DAG.
 *   gamma_match    subgraph matching, "all subgraphs of G_d isomorphic to a pattern
 *                  P" (L112), by worst-case-optimal-join vertex extension + filtering
 *                  (Alg. 1).  Labeled, counted as distinct subgraphs
 *                  (readings R4-R6); non-induced, or induced with
 *                  anti-edge checks (R17).
 *   gamma_fpm      frequent pattern mining, "all patterns P whose support is at least a
 *                  given threshold" (L113, L144), by edge extension + aggregation +
 *                  filtering (Alg. 2), edge-induced, MNI support (R1-R3).
 *   gamma_load_*   the CSR graph_data G_d of Fig. 3 (L158) / §IV (L199): adjacency
 *                  lists and vertex labels, built on the GPU from raw edge samples.
 *
 * Conventions (all entry points):
 *   - Return GAMMA_OK (0) or a negative gamma_status; outputs are written only on
 *     GAMMA_OK.  gamma_last_error() gives a thread-local message for the last
 *     failure on the calling thread (valid until the next call on that thread).
 *   - Input arrays are BORROWED for the duration of the call and may be host or
 *     device pointers (classified with cudaPointerGetAttributes); they are copied.
 *   - Handles and result objects are OWNED by the library and released with the
 *     matching *_free / *_destroy call.  No C++ exception crosses this ABI.
 *   - One gamma_ctx per thread / process.  All device work runs on ctx's stream.
 *   - There is no CPU fallback: with no usable CUDA device every call that computes
 *     returns GAMMA_E_CUDA.
 *   - Vertex ids are uint32 in [0, n); counts are uint64.  A count that would wrap
 *     uint64 returns GAMMA_E_OVERFLOW.
 */
#ifndef GAMMA_H_
#define GAMMA_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GAMMA_ABI_VERSION 3

typedef int32_t gamma_status;
enum {
  GAMMA_OK = 0,
  GAMMA_E_INVAL = -1,        /* bad argument, malformed graph or pattern            */
  GAMMA_E_NOMEM = -2,        /* device allocation failed or HBM/spill budget too small */
  GAMMA_E_CUDA = -3,         /* CUDA runtime / kernel error (incl. no device)        */
  GAMMA_E_OVERFLOW = -4,     /* uint64 count overflow                                */
  GAMMA_E_UNSUPPORTED = -5   /* valid request outside this version (k>32, max_edges>3) */
};

typedef struct gamma_ctx gamma_ctx;
typedef struct gamma_graph gamma_graph;

/* Context descriptor.  Zero-initialise, then set what you need. */
typedef struct {
  int32_t device;            /* CUDA device ordinal                                  */
  int32_t rank, world;       /* root-chunk partition: this process handles share
                                `rank` of `world` (world <= 1: everything)          */
  void *stream;              /* cudaStream_t to run on; NULL: the ctx creates one    */
  /* Optional device allocator (e.g. PyTorch's caching allocator).  NULL: the
     library uses cudaMallocAsync / cudaFreeAsync on ctx's stream.                   */
  void *(*dev_alloc)(size_t bytes, void *stream, void *user);
  void (*dev_free)(void *ptr, void *user);
  void *alloc_user;
  /* Optional collective: in-place SUM of n uint64 values held in HOST memory across
     all `world` ranks (e.g. torch.distributed all_reduce over NCCL).  NULL: results
     of gamma_kclique / gamma_match are this rank's partial counts.                   */
  gamma_status (*allreduce_sum_u64)(uint64_t *host_buf, size_t n, void *user);
  void *coll_user;
  uint64_t hbm_budget_bytes; /* cap on embedding-table bytes; 0: 80% of free HBM     */
  uint64_t host_spill_bytes; /* pinned-host spill capacity for ET levels; 0: none    */
  uint32_t flags;            /* GAMMA_FLAG_* below                                   */
  /* Optional collective used by gamma_fpm when world > 1 (together with
     allreduce_sum_u64): all-to-all of DEVICE buffers.  Rank r's
     send[g*n_per_rank .. (g+1)*n_per_rank) arrives in rank g's
     recv[r*n_per_rank .. (r+1)*n_per_rank).  The library has synchronised its stream
     before the call; the callback returns once recv is complete.  NULL: gamma_fpm
     computes the whole result on every rank (replicas).                             */
  gamma_status (*alltoall_u32)(const uint32_t *send, uint32_t *recv, uint64_t n_per_rank, void *user);
  /* GAMMA_FLAG_HOST_DAG: HBM bytes for the cache of the hottest DAG pages (the rest
     stay in pinned host memory, read over the host link); 0: half of the DAG       */
  uint64_t dag_cache_bytes;
} gamma_ctx_desc;

#define GAMMA_FLAG_TIME_KERNELS 0x1u   /* record per-launch CUDA-event times (stats) */
#define GAMMA_FLAG_NO_FUSE      0x2u   /* materialise every ET level (no fused tail) */
#define GAMMA_FLAG_SPILL        0x4u   /* BFS with host-resident levels
                                          instead of the DFS-over-chunks policy      */
#define GAMMA_FLAG_DEBUG_NOSTAGE 0x8u  /* test hook: never stage runs in shared memory
                                          (exercises the hub / long-run code path)   */
#define GAMMA_FLAG_NO_BITMAP    0x10u  /* kCL: use the ET-level path for every root
                                          (no local-bitmap DFS; ablation / testing)  */
#define GAMMA_FLAG_NO_SPLIT     0x20u  /* kCL bitmap path: never split heavy roots    */
#define GAMMA_FLAG_DEBUG_SPLIT_ALL 0x40u /* test hook: split every root (k >= 6)      */
#define GAMMA_FLAG_COUNT_SORT_BUILD 0x80u /* gamma_load_edges: counting sort + segmented row
                                          sort instead of the global key sort (2m' < 2^31
                                          only; same CSR; slower on hub-heavy graphs, where
                                          the hub rows fall to CUB's large-segment kernel) */
#define GAMMA_FLAG_TWO_PASS     0x200u /* kCL ET path, ablation of Opt 1: each
                                          extension counts its output, scans, then writes at
                                          exact offsets (twice the intersections, no blocks)  */
#define GAMMA_FLAG_SM_EDGE_JOIN 0x400u /* gamma_match by edge extension ("binary join",
                                          PAPER.md L141, L170): one pattern edge per ET step,
                                          non-tree edges as separate filter passes; same
                                          count, larger intermediate tables (ablation)   */
#define GAMMA_FLAG_HOST_DAG      0x800u /* host-resident kCL DAG (the B200
                                          analogue of the paper's host-memory graph):
                                          the DAG columns live in pinned host memory, mapped into
                                          the device address space, with an HBM cache of the
                                          64 KiB pages ranked by heat (reads x elements, reads of
                                          a list = 1 + its in-degree); bitmap kCL path only    */
#define GAMMA_FLAG_FPM_INSTANCES 0x100u /* gamma_fpm: also count each pattern's instances
                                          (connected edge sets mapped to it; one atomic
                                          per embedding -- a parity check, not for timing) */

/* Create / destroy a context.  Errors: E_INVAL (NULL args), E_CUDA (no device). */
gamma_status gamma_ctx_create(const gamma_ctx_desc *desc, gamma_ctx **out);
void gamma_ctx_destroy(gamma_ctx *ctx);
const char *gamma_last_error(void);
int32_t gamma_abi_version(void);
/* Give every idle device buffer the context keeps across calls (SM level tables and
 * L_m scratch, capped at 8 GiB) back to the allocator, then synchronise the stream.
 * Call before trimming an external caching allocator (the Python binding does so
 * before gamma_fpm, which sizes its pattern table and MNI domain pool from free HBM).
 * Errors: E_INVAL (NULL), E_CUDA. */
gamma_status gamma_ctx_trim(gamma_ctx *ctx);

/* ---- Graph data G_d (A1) ------------------------------------------------------
 * gamma_load_edges: build the graph from m raw samples (src[i], dst[i]) over n
 * vertices: symmetrise, drop self-loops and duplicates, sort every adjacency list
 * ascending (O-0), then orient each edge u->v iff
 * (deg u, u) < (deg v, v) (the degree-ordered DAG used by kCL; R9).
 * labels: n uint32 vertex labels or NULL (all 0).  src/dst/labels host or device.
 * Errors: E_INVAL (vertex id >= n, n == 0), E_NOMEM, E_CUDA.                      */
gamma_status gamma_load_edges(gamma_ctx *ctx, uint32_t n, const uint32_t *src,
                              const uint32_t *dst, uint64_t m, const uint32_t *labels,
                              gamma_graph **out);

/* gamma_load_csr: adopt a symmetric CSR (row_ptr: n+1 uint64, col: row_ptr[n]
 * uint32).  Validated on the device: every list strictly ascending, no self-loop,
 * ids < n, and symmetric; else E_INVAL.  The DAG is derived as above.            */
gamma_status gamma_load_csr(gamma_ctx *ctx, uint32_t n, const uint64_t *row_ptr,
                            const uint32_t *col, const uint32_t *labels, gamma_graph **out);

void gamma_graph_free(gamma_graph *g);

typedef struct {
  uint32_t n;
  uint64_t m;                /* undirected edges                                     */
  uint32_t max_degree, max_out_degree;
  uint64_t device_bytes;     /* HBM held by the graph                                */
  double build_ms;           /* device time of the last gamma_load_* (CUDA events)   */
} gamma_graph_info;
gamma_status gamma_graph_get_info(const gamma_graph *g, gamma_graph_info *info);

/* Copy the symmetric CSR (row_ptr n+1, col 2m) or the DAG CSR (row_ptr n+1, col m)
 * into caller buffers (host or device).  which: 0 symmetric, 1 DAG.               */
gamma_status gamma_graph_copy_csr(const gamma_graph *g, int which, uint64_t *row_ptr,
                                  uint32_t *col);

/* ---- k-clique counting (A2-A8) ------------------------------------------------
 * *count = number of vertex sets S, |S| = k, every pair adjacent.  k = 1 gives n,
 * k = 2 gives m.  k > 32: E_UNSUPPORTED; k == 0: E_INVAL.  With world > 1 only
 * this rank's roots are processed and the count is all-reduced if the ctx has a
 * collective (else partial).                                                       */
gamma_status gamma_kclique(gamma_graph *g, uint32_t k, uint64_t *count);

/* Several clique sizes in one call: counts[i] = number of ks[i]-cliques (host
 * arrays, nk entries, each 1 <= ks[i] <= 32).  When every ks[i] <= 12 and the DAG's
 * max out-degree is <= 512, all sizes 3..max(ks) come from ONE bitmap DFS pass over
 * the roots (each visited node with t chosen vertices adds popc(candidates) to the
 * (t+1)-clique count), so the cost is that of the largest k alone; otherwise each
 * size runs as gamma_kclique.  Same rank/world and all-reduce rules as
 * gamma_kclique (one collective for all nk counts).                               */
gamma_status gamma_kclique_multi(gamma_graph *g, uint32_t nk, const uint32_t *ks, uint64_t *counts);

/* Per-root counts: counts[i] = number of k-cliques whose lowest vertex under
 * (deg, id) order is roots[i] (roots/counts host or device, nroots entries).  Used
 * for sampled parity at full size; ignores rank/world.                            */
gamma_status gamma_kclique_roots(gamma_graph *g, uint32_t k, uint64_t nroots,
                                 const uint32_t *roots, uint64_t *counts);

/* ---- Subgraph matching (Alg. 1) ----------------------------------------------- */
typedef struct {
  uint32_t nv, ne;           /* 1 <= nv <= 8, connected                              */
  const uint32_t *edges;     /* 2*ne vertex ids (host memory)                        */
  const uint32_t *labels;    /* nv labels or NULL (unlabeled: any vertex matches)    */
  int32_t induced;           /* 0: non-induced (edges of P -> edges of G); 1: induced
                                (also non-edges of P -> non-edges of G); else E_INVAL  */
} gamma_pattern;

/* Host-only planning of a pattern (no device needed): the matching order delta_v
 * (Alg. 1 line 1; R10), |Aut_L(P)| and the symmetry-breaking
 * order constraints gamma_match applies.  Masks are over matching-order positions.
 * Errors: E_INVAL (nv out of [1,8], bad edge, disconnected, induced not 0/1).     */
typedef struct {
  uint32_t nv;
  uint32_t order[8];         /* position -> pattern vertex                           */
  uint32_t backward_mask[8]; /* earlier positions adjacent to this one               */
  uint32_t less_mask[8];     /* earlier positions j with phi_j < phi_i required      */
  uint32_t greater_mask[8];  /* earlier positions j with phi_i < phi_j required      */
  uint64_t aut;              /* |Aut_L(P)|                                           */
} gamma_plan_info;
gamma_status gamma_pattern_plan(const gamma_pattern *p, gamma_plan_info *out);

/* *count = number of distinct subgraphs of G isomorphic to P (labels respected);
 * mappings (nullable) = *count * |Aut_L(P)|.  Partitioned / reduced like kclique. */
gamma_status gamma_match(gamma_graph *g, const gamma_pattern *p, uint64_t *count,
                         uint64_t *mappings);

/* n queries at once (the same results as n gamma_match calls, in order): every query's
 * roots first, then the level chains on separate streams of the context, so the tails of
 * one query's launches overlap the others' (C3's eight (query, labeling) runs).
 * counts[n] (and mappings[n], nullable) are written on GAMMA_OK; n <= 16 run
 * concurrently, the rest sequentially.  Errors as gamma_match.                     */
gamma_status gamma_match_batch(gamma_graph *g, uint32_t n, const gamma_pattern *patterns, uint64_t *counts,
                               uint64_t *mappings);

/* ---- Frequent pattern mining (Alg. 2) ------------------------------------------ */
typedef struct {
  uint32_t nv, ne;
  uint32_t labels[8];        /* labels in canonical vertex order                     */
  uint8_t edges[8][2];       /* sorted (a<b) pairs in canonical positions            */
  uint64_t support;          /* MNI support                                          */
  uint64_t instances;        /* edge sets mapped to the pattern (GAMMA_FLAG_FPM_INSTANCES;
                                0 otherwise)                                         */
} gamma_fpm_pattern;

typedef struct {
  uint64_t n;
  gamma_fpm_pattern *pats;   /* sorted by (ne, nv, labels, edges)                    */
} gamma_fpm_result;

/* All connected edge-induced patterns with 1..max_edges edges and MNI support >=
 * minsup (max_edges in [1,3] in v1; minsup >= 1; vertex labels < 4096, else
 * E_UNSUPPORTED).  Result owned by the library (free with gamma_fpm_result_free).
 * With world > 1 and both collectives (allreduce_sum_u64, alltoall_u32) levels
 * 1..max_edges-1 run on every rank and the last level is split over the ranks by
 * root-edge batch; its MNI domain bitmaps are OR-reduced by an all-to-all of word
 * shards plus a SUM all-reduce of per-shard popcounts, and every rank
 * returns the same full result.  Without the collectives every rank computes the
 * full result alone (replicas).                                                  */
gamma_status gamma_fpm(gamma_graph *g, uint32_t max_edges, uint64_t minsup,
                       gamma_fpm_result **out);
void gamma_fpm_result_free(gamma_fpm_result *r);

/* ---- Run statistics of the last gamma_kclique / gamma_match / gamma_fpm --------
 * Per kernel class: launches, summed CUDA-event time (only with
 * GAMMA_FLAG_TIME_KERNELS), algorithmic bytes (SURVEY.md §8(d) B_l; DESIGN.md
 * "Algorithmic bytes"), and per-level embedding counts.                            */
#define GAMMA_MAX_KERNEL_CLASSES 16
#define GAMMA_MAX_LEVELS 34
typedef struct {
  uint32_t n_classes;
  char name[GAMMA_MAX_KERNEL_CLASSES][32];
  uint64_t launches[GAMMA_MAX_KERNEL_CLASSES];
  double ms[GAMMA_MAX_KERNEL_CLASSES];
  uint64_t alg_bytes[GAMMA_MAX_KERNEL_CLASSES];
  uint64_t level_entries[GAMMA_MAX_LEVELS];  /* embeddings kept at each level       */
  uint64_t list_elems;       /* adjacency elements the method fetches (sum |list|)   */
  uint64_t chunks;           /* root chunks processed (after overflow splits)        */
  uint64_t retries;          /* chunk splits caused by the HBM budget                */
  uint64_t spilled_bytes;    /* bytes staged through pinned host memory              */
  uint64_t total_launches;   /* every kernel this library launched in the call      */
  double wall_ms;            /* host wall time of the call                           */
} gamma_run_stats;
gamma_status gamma_get_stats(const gamma_ctx *ctx, gamma_run_stats *out);

#ifdef __cplusplus
}
#endif
#endif /* GAMMA_H_ */
