/*
 * oracle/oracle.c -- the CPU ORACLE for the GAMMA hot path.
 *
 * TEST INFRASTRUCTURE, NOT PRODUCT CODE.  Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or helper with the CUDA path
 * (paper_conf_icde_hu0o23_b200/csrc); the only shared inputs are the raw arrays
 * drawn by gamma_gen/.
 *
 * Every function is the plain definition, written slowly and checkably:
 *   og_build       O-0  undirected simple graph from raw samples
 *                       (§IV "CSR ... made up of adjacency lists";
 *                        L119, L204: one label per vertex, no edge labels)
 *   og_kclique     O-1  |{S subset of V : |S|=k, S a clique}|
 *   og_kclique_levels  O-1b  #t-cliques and sum of d+(last vertex) per ET level t, for
 *                       SURVEY.md §8(d)'s algorithmic bytes
 *   og_match       O-2  #injective label-preserving edge-preserving maps / |Aut_L(P)|
 *                       ("all subgraphs isomorphic to a pattern P";
 *                        Alg. 1); induced=1 also maps non-edges of P to
 *                        non-edges of G
 *   og_fpm_*       O-3  edge-induced patterns with <= l edges and MNI support >= minsup
 *                       (Alg. 2; MNI per
 *                        DESIGN.md reading R1)
 *
 * Readings of the paper that these functions take are listed in DESIGN.md
 * ("Readings").  Parity-pinning tests: tests/test_oracle_*.py.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <omp.h>

#define OG_OK 0
#define OG_EINVAL -1
#define OG_ENOMEM -2
#define OG_ENOTDIV -3

typedef struct {
  uint32_t n;
  uint64_t m;        /* undirected edges after O-0 */
  uint64_t *off;     /* n+1 offsets into adj */
  uint32_t *adj;     /* 2m entries, every list ascending by vertex id */
  uint32_t *lab;     /* n labels (all 0 when none given) */
} og_graph;

static int cmp_u64(const void *a, const void *b) {
  uint64_t x = *(const uint64_t *)a, y = *(const uint64_t *)b;
  return (x > y) - (x < y);
}
static int cmp_u32(const void *a, const void *b) {
  uint32_t x = *(const uint32_t *)a, y = *(const uint32_t *)b;
  return (x > y) - (x < y);
}

static void set_threads(int threads) {
  if (threads > 0) omp_set_num_threads(threads);
}

/* ---------------------------------------------------------------------------
 * O-0: symmetrise, drop self-loops, drop duplicates, sort every list.
 * ------------------------------------------------------------------------- */
og_graph *og_build(uint32_t n, uint64_t m_raw, const uint32_t *src, const uint32_t *dst,
                   const uint32_t *labels) {
  /* The same steps as the plain definition -- one key (min, max) per sample without
   * self-loops, sort, drop duplicates, count degrees, fill and sort the lists -- with
   * the sort done per bucket of the smaller endpoint's high bits so that threads can
   * share it (a key's duplicates all fall in its own bucket).  Needed for C5 (~2e9
   * samples); the result does not depend on the bucketing. */
  og_graph *g = (og_graph *)calloc(1, sizeof(og_graph));
  if (!g) return NULL;
  g->n = n;
  int bad = 0;
#pragma omp parallel for reduction(| : bad)
  for (int64_t i = 0; i < (int64_t)m_raw; i++) bad |= (src[i] >= n || dst[i] >= n);
  if (bad) { free(g); return NULL; }
  int sh = 0;
  while (((uint64_t)n >> sh) > 65536) sh++;
  const uint64_t nb = ((uint64_t)n >> sh) + 1;
  const int T = omp_get_max_threads();
  uint64_t *hist = (uint64_t *)calloc((size_t)T * nb + 1, sizeof(uint64_t));
  uint64_t *key = (uint64_t *)malloc((m_raw ? m_raw : 1) * sizeof(uint64_t));
  uint64_t *bstart = (uint64_t *)calloc(nb + 1, sizeof(uint64_t));
  uint64_t *bkeep = (uint64_t *)calloc(nb + 1, sizeof(uint64_t));
  /* pass 1: per-thread bucket histograms (static schedule: same ranges in pass 2) */
#pragma omp parallel num_threads(T)
  {
    uint64_t *h = hist + (size_t)omp_get_thread_num() * nb;
#pragma omp for schedule(static)
    for (int64_t i = 0; i < (int64_t)m_raw; i++) {
      uint32_t u = src[i], v = dst[i];
      if (u == v) continue;                     /* no self-loops */
      h[(u < v ? u : v) >> sh]++;
    }
  }
  /* bucket-major, thread-minor offsets */
  uint64_t run = 0;
  for (uint64_t b = 0; b < nb; b++) {
    bstart[b] = run;
    for (int t = 0; t < T; t++) {
      uint64_t c = hist[(size_t)t * nb + b];
      hist[(size_t)t * nb + b] = run;
      run += c;
    }
  }
  bstart[nb] = run;
  /* pass 2: scatter one key per undirected edge sample into its bucket */
#pragma omp parallel num_threads(T)
  {
    uint64_t *h = hist + (size_t)omp_get_thread_num() * nb;
#pragma omp for schedule(static)
    for (int64_t i = 0; i < (int64_t)m_raw; i++) {
      uint32_t u = src[i], v = dst[i];
      if (u == v) continue;
      uint32_t a = u < v ? u : v, b = u < v ? v : u;
      key[h[a >> sh]++] = ((uint64_t)a << 32) | b;
    }
  }
  free(hist);
  /* sort each bucket and drop duplicates in place */
#pragma omp parallel for schedule(dynamic, 16)
  for (int64_t b = 0; b < (int64_t)nb; b++) {
    uint64_t *kb = key + bstart[b];
    uint64_t len = bstart[b + 1] - bstart[b], w = 0;
    qsort(kb, len, sizeof(uint64_t), cmp_u64);
    for (uint64_t i = 0; i < len; i++)
      if (i == 0 || kb[i] != kb[i - 1]) kb[w++] = kb[i];
    bkeep[b] = w;
  }
  uint64_t m = 0;
  for (uint64_t b = 0; b < nb; b++) m += bkeep[b];
  g->m = m;
  /* degrees */
  uint64_t *deg = (uint64_t *)calloc((size_t)n + 1, sizeof(uint64_t));
#pragma omp parallel for schedule(dynamic, 16)
  for (int64_t b = 0; b < (int64_t)nb; b++)
    for (uint64_t i = bstart[b]; i < bstart[b] + bkeep[b]; i++) {
      __atomic_fetch_add(&deg[key[i] >> 32], 1, __ATOMIC_RELAXED);
      __atomic_fetch_add(&deg[key[i] & 0xffffffffu], 1, __ATOMIC_RELAXED);
    }
  g->off = (uint64_t *)malloc(((size_t)n + 1) * sizeof(uint64_t));
  g->off[0] = 0;
  for (uint32_t v = 0; v < n; v++) g->off[v + 1] = g->off[v] + deg[v];
  g->adj = (uint32_t *)malloc((m > 0 ? 2 * m : 1) * sizeof(uint32_t));
  for (uint32_t v = 0; v < n; v++) deg[v] = g->off[v];   /* reuse as fill cursor */
#pragma omp parallel for schedule(dynamic, 16)
  for (int64_t b = 0; b < (int64_t)nb; b++)
    for (uint64_t i = bstart[b]; i < bstart[b] + bkeep[b]; i++) {
      uint32_t a = (uint32_t)(key[i] >> 32), c = (uint32_t)(key[i] & 0xffffffffu);
      g->adj[__atomic_fetch_add(&deg[a], 1, __ATOMIC_RELAXED)] = c;
      g->adj[__atomic_fetch_add(&deg[c], 1, __ATOMIC_RELAXED)] = a;
    }
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t v = 0; v < (int64_t)n; v++)
    qsort(g->adj + g->off[v], g->off[v + 1] - g->off[v], sizeof(uint32_t), cmp_u32);
  g->lab = (uint32_t *)malloc(((size_t)n ? n : 1) * sizeof(uint32_t));
  for (uint32_t v = 0; v < n; v++) g->lab[v] = labels ? labels[v] : 0;
  free(deg);
  free(key);
  free(bstart);
  free(bkeep);
  return g;
}

void og_free(og_graph *g) {
  if (!g) return;
  free(g->off); free(g->adj); free(g->lab); free(g);
}

uint32_t og_n(const og_graph *g) { return g->n; }
uint64_t og_m(const og_graph *g) { return g->m; }
/* Copy out the symmetric CSR (off: n+1, adj: 2m). */
void og_csr(const og_graph *g, uint64_t *off, uint32_t *adj) {
  memcpy(off, g->off, ((size_t)g->n + 1) * sizeof(uint64_t));
  memcpy(adj, g->adj, 2 * g->m * sizeof(uint32_t));
}

static uint64_t deg_of(const og_graph *g, uint32_t v) { return g->off[v + 1] - g->off[v]; }

/* Is x in N(v)?  Plain binary search on the sorted list. */
static int adjacent(const og_graph *g, uint32_t v, uint32_t x) {
  uint64_t lo = g->off[v], hi = g->off[v + 1];
  while (lo < hi) {
    uint64_t mid = lo + (hi - lo) / 2;
    uint32_t y = g->adj[mid];
    if (y == x) return 1;
    if (y < x) lo = mid + 1; else hi = mid;
  }
  return 0;
}

/* ---------------------------------------------------------------------------
 * O-1: k-clique counting.  Each k-clique is counted once, at its lowest vertex
 * under the order r(v) = (deg v, v) (order_mode 0) or r(v) = v (order_mode 1).
 * Candidates are filtered by explicit adjacency checks (not list intersection).
 * ------------------------------------------------------------------------- */
static int r_less(const og_graph *g, int mode, uint32_t a, uint32_t b) {
  if (mode == 1) return a < b;
  uint64_t da = deg_of(g, a), db = deg_of(g, b);
  return da < db || (da == db && a < b);
}

static uint64_t kcl_rec(const og_graph *g, int mode, uint32_t k, uint32_t size,
                        const uint32_t *cand, uint64_t nc, uint32_t **buf) {
  if (size == k - 1) return nc;   /* every remaining candidate completes a k-clique */
  uint64_t total = 0;
  uint32_t *next = buf[size];
  for (uint64_t i = 0; i < nc; i++) {
    uint32_t w = cand[i];
    uint64_t nn = 0;
    for (uint64_t j = 0; j < nc; j++) {
      uint32_t x = cand[j];
      if (r_less(g, mode, w, x) && adjacent(g, w, x)) next[nn++] = x;
    }
    total += kcl_rec(g, mode, k, size + 1, next, nn, buf);
  }
  return total;
}

static uint64_t max_degree(const og_graph *g) {
  uint64_t md = 0;
  for (uint32_t v = 0; v < g->n; v++) if (deg_of(g, v) > md) md = deg_of(g, v);
  return md;
}

/* Count k-cliques whose lowest-ranked vertex is v (k >= 2). */
static uint64_t kcl_root(const og_graph *g, int mode, uint32_t k, uint32_t v, uint32_t **buf) {
  uint32_t *cand = buf[0];
  uint64_t nc = 0;
  for (uint64_t e = g->off[v]; e < g->off[v + 1]; e++)
    if (r_less(g, mode, v, g->adj[e])) cand[nc++] = g->adj[e];
  return kcl_rec(g, mode, k, 1, cand, nc, buf);
}

static uint32_t **alloc_bufs(uint32_t levels, uint64_t width) {
  uint32_t **buf = (uint32_t **)malloc(levels * sizeof(uint32_t *));
  for (uint32_t i = 0; i < levels; i++) buf[i] = (uint32_t *)malloc((width ? width : 1) * sizeof(uint32_t));
  return buf;
}
static void free_bufs(uint32_t **buf, uint32_t levels) {
  for (uint32_t i = 0; i < levels; i++) free(buf[i]);
  free(buf);
}

uint64_t og_kclique(const og_graph *g, uint32_t k, int order_mode, int threads) {
  if (k == 0) return 0;
  if (k == 1) return g->n;
  set_threads(threads);
  uint64_t md = max_degree(g), total = 0;
#pragma omp parallel reduction(+ : total)
  {
    uint32_t **buf = alloc_bufs(k + 1, md);
#pragma omp for schedule(dynamic, 64)
    for (int64_t v = 0; v < (int64_t)g->n; v++) total += kcl_root(g, order_mode, k, (uint32_t)v, buf);
    free_bufs(buf, k + 1);
  }
  return total;
}

/* Per-root counts (order_mode 0 ranks) for sampled parity at full size. */
void og_kclique_roots(const og_graph *g, uint32_t k, uint64_t nroots, const uint32_t *roots,
                      uint64_t *counts, int threads) {
  set_threads(threads);
  uint64_t md = max_degree(g);
#pragma omp parallel
  {
    uint32_t **buf = alloc_bufs(k + 1, md);
#pragma omp for schedule(dynamic, 1)
    for (int64_t i = 0; i < (int64_t)nroots; i++)
      counts[i] = (k == 1) ? 1 : kcl_root(g, 0, k, roots[i], buf);
    free_bufs(buf, k + 1);
  }
}

/* ---------------------------------------------------------------------------
 * O-1b: level statistics of the k-clique embedding table, for SURVEY.md §8(d)'s
 * algorithmic bytes (not a parity quantity).  The ET level t (PAPER.md L253-257,
 * §V-A) holds one entry per t-clique; extending an entry whose last-matched vertex
 * is w fetches w's out-list N+(w) = {x in N(w) : r(x) > r(w)} (the "intersect"
 * step).  For t = 1..k:
 *   N[t] = #t-cliques,   S[t] = sum over t-cliques C of d+(max_r C).
 * Same enumeration as og_kclique (order_mode 0): each clique is visited once,
 * with its vertices chosen in increasing r.
 * ------------------------------------------------------------------------- */
static uint64_t out_degree(const og_graph *g, uint32_t w) {
  uint64_t c = 0;
  for (uint64_t e = g->off[w]; e < g->off[w + 1]; e++)
    if (r_less(g, 0, w, g->adj[e])) c++;
  return c;
}

static void kcl_levels_rec(const og_graph *g, const uint64_t *dplus, uint32_t k, uint32_t size, uint32_t last,
                           const uint32_t *cand, uint64_t nc, uint32_t **buf, uint64_t *N, uint64_t *S) {
  N[size] += 1;
  S[size] += dplus[last];
  if (size == k) return;
  if (size + 1 == k) {   /* every candidate ends one k-clique: no need to descend */
    N[k] += nc;
    for (uint64_t i = 0; i < nc; i++) S[k] += dplus[cand[i]];
    return;
  }
  uint32_t *next = buf[size];
  for (uint64_t i = 0; i < nc; i++) {
    uint32_t w = cand[i];
    uint64_t nn = 0;
    for (uint64_t j = 0; j < nc; j++) {
      uint32_t x = cand[j];
      if (r_less(g, 0, w, x) && adjacent(g, w, x)) next[nn++] = x;
    }
    kcl_levels_rec(g, dplus, k, size + 1, w, next, nn, buf, N, S);
  }
}

/* N, S: arrays of k+1 entries (index 0 unused, set to 0). */
void og_kclique_levels(const og_graph *g, uint32_t k, uint64_t *N, uint64_t *S, int threads) {
  for (uint32_t t = 0; t <= k; t++) N[t] = S[t] = 0;
  if (k == 0) return;
  set_threads(threads);
  uint64_t md = max_degree(g);
  uint64_t *dplus = (uint64_t *)malloc(((size_t)g->n + 1) * sizeof(uint64_t));
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t v = 0; v < (int64_t)g->n; v++) dplus[v] = out_degree(g, (uint32_t)v);
#pragma omp parallel
  {
    uint64_t *n_loc = (uint64_t *)calloc(k + 1, sizeof(uint64_t));
    uint64_t *s_loc = (uint64_t *)calloc(k + 1, sizeof(uint64_t));
    uint32_t **buf = alloc_bufs(k + 1, md);
#pragma omp for schedule(dynamic, 64)
    for (int64_t v = 0; v < (int64_t)g->n; v++) {
      uint32_t *cand = buf[0];
      uint64_t nc = 0;
      for (uint64_t e = g->off[v]; e < g->off[v + 1]; e++)
        if (r_less(g, 0, (uint32_t)v, g->adj[e])) cand[nc++] = g->adj[e];
      kcl_levels_rec(g, dplus, k, 1, (uint32_t)v, cand, nc, buf, n_loc, s_loc);
    }
#pragma omp critical
    for (uint32_t t = 0; t <= k; t++) {
      N[t] += n_loc[t];
      S[t] += s_loc[t];
    }
    free_bufs(buf, k + 1);
    free(n_loc);
    free(s_loc);
  }
  free(dplus);
}

/* ---------------------------------------------------------------------------
 * O-2: labeled subgraph matching.  count = mappings / |Aut_L(P)|.
 * Non-induced (reading R4): edges of P map to edges of G.  Induced
 * ("anti-edge checks"): in addition, every
 * non-edge of P maps to a non-edge of G.  Aut_L(P) is the same group for both
 * (a permutation preserving E_P preserves its complement).
 * Matching order: BFS from pattern vertex 0 (deliberately not the GPU planner's
 * order).  Candidates of pattern vertex q = N(phi(bfs parent of q)); every other
 * backward edge checked by binary search; injectivity by linear scan.
 * ------------------------------------------------------------------------- */
#define OG_MAXV 8

typedef struct {
  uint32_t nv;
  int adjm[OG_MAXV][OG_MAXV];
  int labeled;
  int induced;                 /* 1: also require non-edges of P to map to non-edges of G */
  uint32_t plab[OG_MAXV];
  uint32_t order[OG_MAXV];     /* BFS order */
  uint32_t parent[OG_MAXV];    /* BFS parent of order[i] (i>0) */
} og_pat;

static int pat_init(og_pat *p, uint32_t nv, uint32_t ne, const uint32_t *edges, const uint32_t *plabels) {
  if (nv < 1 || nv > OG_MAXV) return OG_EINVAL;
  memset(p, 0, sizeof(*p));
  p->nv = nv;
  for (uint32_t e = 0; e < ne; e++) {
    uint32_t a = edges[2 * e], b = edges[2 * e + 1];
    if (a >= nv || b >= nv || a == b) return OG_EINVAL;
    p->adjm[a][b] = p->adjm[b][a] = 1;
  }
  p->labeled = plabels != NULL;
  for (uint32_t i = 0; i < nv; i++) p->plab[i] = plabels ? plabels[i] : 0;
  /* BFS from vertex 0 */
  int seen[OG_MAXV] = {0};
  uint32_t head = 0, tail = 0;
  p->order[tail++] = 0; seen[0] = 1;
  while (head < tail) {
    uint32_t x = p->order[head++];
    for (uint32_t y = 0; y < nv; y++)
      if (p->adjm[x][y] && !seen[y]) { seen[y] = 1; p->parent[tail] = x; p->order[tail++] = y; }
  }
  if (tail != nv) return OG_EINVAL;   /* disconnected */
  return OG_OK;
}

/* |Aut_L(P)| by brute force over all nv! permutations (Heap's algorithm). */
static uint64_t pat_aut(const og_pat *p) {
  uint32_t nv = p->nv, perm[OG_MAXV], c[OG_MAXV];
  for (uint32_t i = 0; i < nv; i++) { perm[i] = i; c[i] = 0; }
  uint64_t count = 0;
  for (;;) {
    int ok = 1;
    for (uint32_t i = 0; i < nv && ok; i++) {
      if (p->plab[perm[i]] != p->plab[i]) ok = 0;
      for (uint32_t j = 0; j < nv && ok; j++)
        if (p->adjm[perm[i]][perm[j]] != p->adjm[i][j]) ok = 0;
    }
    count += ok;
    /* next permutation (Heap) */
    uint32_t i = 1;
    while (i < nv && c[i] >= i) { c[i] = 0; i++; }
    if (i >= nv) break;
    uint32_t j = (i % 2) ? c[i] : 0;
    uint32_t t = perm[j]; perm[j] = perm[i]; perm[i] = t;
    c[i]++;
  }
  return count;
}

static uint64_t match_rec(const og_graph *g, const og_pat *p, uint32_t pos, uint32_t *phi) {
  if (pos == p->nv) return 1;
  uint32_t q = p->order[pos], par = p->parent[pos];
  uint32_t base = phi[par];
  uint64_t total = 0;
  for (uint64_t e = g->off[base]; e < g->off[base + 1]; e++) {
    uint32_t x = g->adj[e];
    if (p->labeled && g->lab[x] != p->plab[q]) continue;
    int ok = 1;
    for (uint32_t i = 0; i < pos && ok; i++) if (phi[p->order[i]] == x) ok = 0;   /* injective */
    for (uint32_t i = 0; i < pos && ok; i++) {
      uint32_t b = p->order[i];
      if (b != par && p->adjm[q][b] && !adjacent(g, phi[b], x)) ok = 0;           /* backward edges */
      if (p->induced && !p->adjm[q][b] && adjacent(g, phi[b], x)) ok = 0;          /* backward non-edges */
    }
    if (!ok) continue;
    phi[q] = x;
    total += match_rec(g, p, pos + 1, phi);
  }
  return total;
}

int og_match(const og_graph *g, uint32_t nv, uint32_t ne, const uint32_t *edges,
             const uint32_t *plabels, int induced, int threads, uint64_t *count, uint64_t *mappings,
             uint64_t *aut) {
  og_pat p;
  int st = pat_init(&p, nv, ne, edges, plabels);
  if (st) return st;
  p.induced = induced != 0;
  set_threads(threads);
  uint64_t total = 0;
  uint32_t r = p.order[0];
#pragma omp parallel for schedule(dynamic, 64) reduction(+ : total)
  for (int64_t v = 0; v < (int64_t)g->n; v++) {
    if (p.labeled && g->lab[v] != p.plab[r]) continue;
    uint32_t phi[OG_MAXV];
    phi[r] = (uint32_t)v;
    total += match_rec(g, &p, 1, phi);
  }
  uint64_t a = pat_aut(&p);
  if (aut) *aut = a;
  if (mappings) *mappings = total;
  if (total % a) return OG_ENOTDIV;
  if (count) *count = total / a;
  return OG_OK;
}

/* Mappings whose image of BFS-order vertex 0 (pattern vertex 0) is roots[i]; the sum
 * over all vertices is the `mappings` of og_match.  For sampled timing / parity. */
int og_match_roots(const og_graph *g, uint32_t nv, uint32_t ne, const uint32_t *edges,
                   const uint32_t *plabels, int induced, uint64_t nroots, const uint32_t *roots,
                   uint64_t *out, int threads) {
  og_pat p;
  int st = pat_init(&p, nv, ne, edges, plabels);
  if (st) return st;
  p.induced = induced != 0;
  set_threads(threads);
  uint32_t r = p.order[0];
#pragma omp parallel for schedule(dynamic, 16)
  for (int64_t i = 0; i < (int64_t)nroots; i++) {
    uint32_t v = roots[i];
    out[i] = 0;
    if (v >= g->n || (p.labeled && g->lab[v] != p.plab[r])) continue;
    uint32_t phi[OG_MAXV];
    phi[r] = v;
    out[i] = match_rec(g, &p, 1, phi);
  }
  return OG_OK;
}

/* ---------------------------------------------------------------------------
 * O-2b: per-level statistics of SM in a GIVEN matching order with GIVEN order
 * constraints (SURVEY.md §8(d) algorithmic bytes of the SM path; the order and the
 * constraints are the method's choices -- DESIGN.md readings R10 and R16 -- computed
 * by this oracle's own planner, oracle/__init__.py plan_r10_r16).  Position t holds
 * pattern vertex order[t]; a partial match of t positions is an injective map of
 * order[0..t-1] that respects labels, the pattern edges among them, the constraints
 * phi(t) > phi(j) for j in lt[t] and phi(t) < phi(j) for j in gt[t], and (positions
 * t < nv-1 only: a pruning that never removes a full match) deg(phi(t)) >=
 * deg_P(order[t]) ("pruning ... at run-time").
 *   N[t]  = number of partial matches with t positions (N[nv] = the match count);
 *   G[t]  = sum over partial matches with t-1 positions of the degrees of the images
 *           of the backward neighbours of position t that lie in positions < t-1
 *           (Opt 2: the group's prefix lists, fetched once per group);
 *   C[t]  = sum over partial matches with t positions of deg(phi(t-1)) if position
 *           t-1 is a backward neighbour of position t (each child's own list).
 * Step t -> t+1 of the ET then reads 12 N[t] + 4 (G[t] + C[t]) + 8 N[t+1] [t+1 < nv]
 * bytes.  Candidates are enumerated by a check-based scan of N(phi(first backward
 * neighbour)), as in og_match.
 * ------------------------------------------------------------------------- */
typedef struct {
  uint32_t nv, order[OG_MAXV], lab[OG_MAXV], pdeg[OG_MAXV], labeled;
  uint32_t back[OG_MAXV], lt[OG_MAXV], gt[OG_MAXV];   /* position bitmasks */
} og_lplan;

static uint64_t gdegree(const og_graph *g, uint32_t v) { return g->off[v + 1] - g->off[v]; }

static void levels_rec(const og_graph *g, const og_lplan *P, uint32_t t, uint32_t *phi, uint64_t *N, uint64_t *G,
                       uint64_t *C) {
  /* a partial match of t positions */
  N[t] += 1;
  if (t >= 1 && t < P->nv && ((P->back[t] >> (t - 1)) & 1u)) C[t] += gdegree(g, phi[t - 1]);
  if (t + 1 < P->nv) {   /* as the group (prefix) of the children at position t */
    uint32_t m = P->back[t + 1] & ((1u << t) - 1u);
    for (uint32_t j = 0; j < t; j++) if ((m >> j) & 1u) G[t + 1] += gdegree(g, phi[j]);
  }
  if (t == P->nv) return;
  uint32_t b0 = (uint32_t)__builtin_ctz(P->back[t]);   /* first backward neighbour */
  uint32_t base = phi[b0];
  for (uint64_t e = g->off[base]; e < g->off[base + 1]; e++) {
    uint32_t x = g->adj[e];
    if (P->labeled && g->lab[x] != P->lab[t]) continue;
    if (t + 1 < P->nv && gdegree(g, x) < P->pdeg[t]) continue;
    int ok = 1;
    for (uint32_t j = 0; j < t && ok; j++) {
      if (phi[j] == x) ok = 0;
      else if (((P->lt[t] >> j) & 1u) && !(x > phi[j])) ok = 0;
      else if (((P->gt[t] >> j) & 1u) && !(x < phi[j])) ok = 0;
      else if (j != b0 && ((P->back[t] >> j) & 1u) && !adjacent(g, phi[j], x)) ok = 0;
    }
    if (!ok) continue;
    phi[t] = x;
    levels_rec(g, P, t + 1, phi, N, G, C);
  }
}

int og_match_levels(const og_graph *g, uint32_t nv, uint32_t ne, const uint32_t *edges, const uint32_t *plabels,
                    const uint32_t *order, const uint32_t *lt, const uint32_t *gt, int threads, uint64_t *N,
                    uint64_t *G, uint64_t *C) {
  if (nv < 1 || nv > OG_MAXV) return OG_EINVAL;
  og_lplan P;
  memset(&P, 0, sizeof(P));
  P.nv = nv;
  P.labeled = plabels != NULL;
  uint32_t adjm[OG_MAXV][OG_MAXV];
  memset(adjm, 0, sizeof(adjm));
  for (uint32_t e = 0; e < ne; e++) {
    uint32_t a = edges[2 * e], b = edges[2 * e + 1];
    if (a >= nv || b >= nv || a == b) return OG_EINVAL;
    adjm[a][b] = adjm[b][a] = 1;
  }
  uint32_t pos_of[OG_MAXV], seen = 0;
  for (uint32_t t = 0; t < nv; t++) {
    if (order[t] >= nv || ((seen >> order[t]) & 1u)) return OG_EINVAL;
    seen |= 1u << order[t];
    pos_of[order[t]] = t;
  }
  for (uint32_t t = 0; t < nv; t++) {
    uint32_t v = order[t];
    P.order[t] = v;
    P.lab[t] = plabels ? plabels[v] : 0;
    P.lt[t] = lt[t] & ((1u << t) - 1u);
    P.gt[t] = gt[t] & ((1u << t) - 1u);
    for (uint32_t u = 0; u < nv; u++) {
      if (!adjm[v][u]) continue;
      P.pdeg[t]++;
      if (pos_of[u] < t) P.back[t] |= 1u << pos_of[u];
    }
    if (t > 0 && P.back[t] == 0) return OG_EINVAL;   /* the order must stay connected */
  }
  for (uint32_t t = 0; t <= nv; t++) N[t] = G[t] = C[t] = 0;
  set_threads(threads);
#pragma omp parallel
  {
    uint64_t n_loc[OG_MAXV + 1] = {0}, g_loc[OG_MAXV + 1] = {0}, c_loc[OG_MAXV + 1] = {0};
#pragma omp for schedule(dynamic, 64)
    for (int64_t v = 0; v < (int64_t)g->n; v++) {
      if (P.labeled && g->lab[v] != P.lab[0]) continue;
      if (nv > 1 && gdegree(g, (uint32_t)v) < P.pdeg[0]) continue;
      uint32_t phi[OG_MAXV];
      phi[0] = (uint32_t)v;
      levels_rec(g, &P, 1, phi, n_loc, g_loc, c_loc);
    }
#pragma omp critical
    for (uint32_t t = 0; t <= nv; t++) { N[t] += n_loc[t]; G[t] += g_loc[t]; C[t] += c_loc[t]; }
  }
  return OG_OK;
}

/* ---------------------------------------------------------------------------
 * O-3: frequent pattern mining, edge-induced patterns of 1..l edges (l <= 4),
 * MNI support.
 *
 * Canonical code of a connected edge set S with vertex set W (|W| = nv <= 5):
 *   min over bijections pi : {0..nv-1} -> W  of
 *     ( lab(pi(0)), ..., lab(pi(nv-1)),  sorted list of pairs (i<j) with {pi(i),pi(j)} in S )
 *   compared lexicographically (labels first, then the sorted edge-pair list).
 * Domain of canonical position i: union over every minimizing pi of {pi(i)}.
 * sup(P) = min_i |domain(P, i)|  (MNI).  Output: every P with sup >= minsup.
 * ------------------------------------------------------------------------- */
#define FPM_MAXNV 5
#define FPM_MAXE 4
#define FPM_NPERM 120   /* 5! */

typedef struct {
  uint32_t nv, ne;
  uint32_t lab[FPM_MAXNV];
  uint32_t e[FPM_MAXE][2];
} og_code;

static int code_cmp(const og_code *x, const og_code *y) {
  if (x->nv != y->nv) return x->nv < y->nv ? -1 : 1;
  for (uint32_t i = 0; i < x->nv; i++)
    if (x->lab[i] != y->lab[i]) return x->lab[i] < y->lab[i] ? -1 : 1;
  if (x->ne != y->ne) return x->ne < y->ne ? -1 : 1;
  for (uint32_t i = 0; i < x->ne; i++) {
    if (x->e[i][0] != y->e[i][0]) return x->e[i][0] < y->e[i][0] ? -1 : 1;
    if (x->e[i][1] != y->e[i][1]) return x->e[i][1] < y->e[i][1] ? -1 : 1;
  }
  return 0;
}

/* Hash table of patterns -> domain bitsets (nv * ceil(n/64) words each). */
typedef struct {
  uint64_t cap;          /* slots, power of two */
  og_code *key;
  int *used;             /* 0 empty, 1 being written, 2 ready */
  uint64_t **dom;        /* dom[slot] = FPM_MAXNV bitsets of `words` words */
  uint64_t *inst;        /* inst[slot] = number of edge sets mapped to the pattern */
  uint64_t words;
  omp_lock_t lock;
  int overflow;
} og_ptab;

static uint64_t code_hash(const og_code *c) {
  uint64_t h = 1469598103934665603ull;
  const uint32_t *w = (const uint32_t *)c;
  for (size_t i = 0; i < sizeof(og_code) / 4; i++) { h ^= w[i]; h *= 1099511628211ull; }
  return h;
}

static int64_t ptab_get(og_ptab *t, const og_code *c) {
  uint64_t h = code_hash(c) & (t->cap - 1);
  for (uint64_t probe = 0; probe < t->cap; probe++, h = (h + 1) & (t->cap - 1)) {
    int u = __atomic_load_n(&t->used[h], __ATOMIC_ACQUIRE);
    if (u == 2) { if (code_cmp(&t->key[h], c) == 0) return (int64_t)h; continue; }
    /* empty or in flight: take the lock and re-check */
    omp_set_lock(&t->lock);
    u = t->used[h];
    if (u == 2) {
      omp_unset_lock(&t->lock);
      if (code_cmp(&t->key[h], c) == 0) return (int64_t)h;
      continue;
    }
    t->key[h] = *c;
    t->dom[h] = (uint64_t *)calloc(FPM_MAXNV * t->words, sizeof(uint64_t));
    __atomic_store_n(&t->used[h], 2, __ATOMIC_RELEASE);
    omp_unset_lock(&t->lock);
    return (int64_t)h;
  }
  t->overflow = 1;
  return -1;
}

/* Canonicalise the edge set {ed[0..ne-1]} on vertex set W (nv vertices) and
 * OR every minimizing assignment into the pattern's domains. */
/* All 120 orders of 5 symbols, lexicographic (filled once). */
static uint8_t g_perms5[FPM_NPERM][FPM_MAXNV];
static int g_perms5_ready = 0;
static void perms5_init(void) {
  if (__atomic_load_n(&g_perms5_ready, __ATOMIC_ACQUIRE)) return;
#pragma omp critical(og_perms5)
  if (!g_perms5_ready) {
    uint8_t p[FPM_MAXNV] = {0, 1, 2, 3, 4};
    for (int r = 0; r < FPM_NPERM; r++) {
      memcpy(g_perms5[r], p, FPM_MAXNV);
      /* next permutation */
      int i = FPM_MAXNV - 2;
      while (i >= 0 && p[i] > p[i + 1]) i--;
      if (i < 0) break;
      int j = FPM_MAXNV - 1;
      while (p[j] < p[i]) j--;
      uint8_t x = p[i]; p[i] = p[j]; p[j] = x;
      for (int a = i + 1, b = FPM_MAXNV - 1; a < b; a++, b--) { x = p[a]; p[a] = p[b]; p[b] = x; }
    }
    __atomic_store_n(&g_perms5_ready, 1, __ATOMIC_RELEASE);
  }
}

static void fpm_record(const og_graph *g, og_ptab *t, uint32_t nv, const uint32_t *W, uint32_t ne,
                       const uint32_t (*ed)[2]) {
  perms5_init();
  og_code best; int have = 0;
  uint32_t bestpi[FPM_NPERM][FPM_MAXNV]; int nbest = 0;
  for (int pi = 0; pi < FPM_NPERM; pi++) {
    const uint8_t *P = g_perms5[pi];
    int valid = 1;   /* permutation of the first nv symbols only (the rest fixed) */
    for (uint32_t i = 0; i < nv; i++) if (P[i] >= nv) valid = 0;
    for (uint32_t i = nv; i < FPM_MAXNV; i++) if (P[i] != i) valid = 0;
    if (!valid) continue;
    /* position i holds data vertex W[P[i]] */
    og_code c; memset(&c, 0, sizeof(c));
    c.nv = nv; c.ne = ne;
    uint32_t pos_of[FPM_MAXNV];
    for (uint32_t i = 0; i < nv; i++) { c.lab[i] = g->lab[W[P[i]]]; pos_of[P[i]] = i; }
    for (uint32_t e = 0; e < ne; e++) {
      uint32_t a = 0, b = 0;
      for (uint32_t w = 0; w < nv; w++) { if (W[w] == ed[e][0]) a = pos_of[w]; if (W[w] == ed[e][1]) b = pos_of[w]; }
      c.e[e][0] = a < b ? a : b; c.e[e][1] = a < b ? b : a;
    }
    /* sort the edge pairs (insertion sort, ne <= 4) */
    for (uint32_t i = 1; i < ne; i++)
      for (uint32_t j = i; j > 0; j--) {
        uint32_t *x = c.e[j - 1], *y = c.e[j];
        if (x[0] > y[0] || (x[0] == y[0] && x[1] > y[1])) {
          uint32_t t0 = x[0], t1 = x[1]; x[0] = y[0]; x[1] = y[1]; y[0] = t0; y[1] = t1;
        }
      }
    int cmp = have ? code_cmp(&c, &best) : -1;
    if (cmp < 0) { best = c; have = 1; nbest = 0; }
    if (cmp <= 0) {
      for (uint32_t i = 0; i < nv; i++) bestpi[nbest][i] = W[P[i]];
      nbest++;
    }
  }
  int64_t slot = ptab_get(t, &best);
  if (slot < 0) return;
  uint64_t *dom = t->dom[slot];
  __atomic_fetch_add(&t->inst[slot], 1, __ATOMIC_RELAXED);
  for (int b = 0; b < nbest; b++)
    for (uint32_t i = 0; i < nv; i++) {
      uint32_t v = bestpi[b][i];
      __atomic_fetch_or(&dom[i * t->words + v / 64], 1ull << (v % 64), __ATOMIC_RELAXED);
    }
}

/* Shape-by-shape enumeration of every connected edge set with 1..l edges, each
 * exactly once:
 *   1 edge:   {u,v}, u<v
 *   2 edges:  wedge, centre c with an unordered neighbour pair {a,b}
 *   3 edges:  triangle u<v<w; 3-star, centre c with a neighbour triple a<b<d;
 *             3-path a-b-c-d keyed by its middle edge {b,c} (b<c), a in N(b)-{c},
 *             d in N(c)-{b}, a != d.
 *   4 edges:  4-star, centre c with a neighbour quadruple;
 *             4-cycle a-b-c-d-a keyed by its smallest vertex a and a's two cycle
 *             neighbours b < d, c in N(b) & N(d), c != a (c > a);
 *             paw (triangle + pendant edge): each triangle u<v<w once, the pendant at
 *             x in {u,v,w} to y in N(x) outside the triangle;
 *             4-path a-b-c-d-e keyed by its middle vertex c and its two legs c-b-a,
 *             c-d-e taken unordered ((b,a) < (d,e)), five distinct vertices;
 *             fork (spider with legs 2,1,1): centre c of degree 3, long leg c-x-w,
 *             short legs y < z, all in N(c) (x, y, z distinct), w in N(x) - {c,y,z}. */
static void fpm_enum_shapes(const og_graph *g, og_ptab *t, uint32_t l) {
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t vv = 0; vv < (int64_t)g->n; vv++) {
    uint32_t v = (uint32_t)vv;
    uint64_t s = g->off[v], e = g->off[v + 1];
    for (uint64_t i = s; i < e; i++) {
      uint32_t u = g->adj[i];
      if (u > v) {   /* edge {v,u} */
        uint32_t W[2] = {v, u}; uint32_t ed[1][2] = {{v, u}};
        fpm_record(g, t, 2, W, 1, ed);
      }
    }
    if (l >= 2)
      for (uint64_t i = s; i < e; i++)
        for (uint64_t j = i + 1; j < e; j++) {   /* wedge a-v-b */
          uint32_t a = g->adj[i], b = g->adj[j];
          uint32_t W[3] = {v, a, b}; uint32_t ed[2][2] = {{v, a}, {v, b}};
          fpm_record(g, t, 3, W, 2, ed);
        }
    if (l >= 3) {
      for (uint64_t i = s; i < e; i++)
        for (uint64_t j = i + 1; j < e; j++)
          for (uint64_t q = j + 1; q < e; q++) {   /* 3-star */
            uint32_t a = g->adj[i], b = g->adj[j], d = g->adj[q];
            uint32_t W[4] = {v, a, b, d}; uint32_t ed[3][2] = {{v, a}, {v, b}, {v, d}};
            fpm_record(g, t, 4, W, 3, ed);
          }
      for (uint64_t i = s; i < e; i++) {
        uint32_t u = g->adj[i];
        if (u <= v) continue;
        for (uint64_t j = i + 1; j < e; j++) {   /* triangle v<u<w */
          uint32_t w = g->adj[j];
          if (adjacent(g, u, w)) {
            uint32_t W[3] = {v, u, w}; uint32_t ed[3][2] = {{v, u}, {v, w}, {u, w}};
            fpm_record(g, t, 3, W, 3, ed);
          }
        }
        /* 3-paths with middle edge {v,u}, v<u: a-v-u-d */
        for (uint64_t x = s; x < e; x++) {
          uint32_t a = g->adj[x];
          if (a == u) continue;
          for (uint64_t y = g->off[u]; y < g->off[u + 1]; y++) {
            uint32_t d = g->adj[y];
            if (d == v || d == a) continue;
            uint32_t W[4] = {a, v, u, d}; uint32_t ed[3][2] = {{a, v}, {v, u}, {u, d}};
            fpm_record(g, t, 4, W, 3, ed);
          }
        }
      }
    }
    if (l >= 4) {
      /* 4-star */
      for (uint64_t i = s; i < e; i++)
        for (uint64_t j = i + 1; j < e; j++)
          for (uint64_t q = j + 1; q < e; q++)
            for (uint64_t r = q + 1; r < e; r++) {
              uint32_t a = g->adj[i], b = g->adj[j], c = g->adj[q], d = g->adj[r];
              uint32_t W[5] = {v, a, b, c, d}; uint32_t ed[4][2] = {{v, a}, {v, b}, {v, c}, {v, d}};
              fpm_record(g, t, 5, W, 4, ed);
            }
      /* 4-cycle v-b-c-d-v with v the smallest vertex, b < d */
      for (uint64_t i = s; i < e; i++) {
        uint32_t b = g->adj[i];
        if (b <= v) continue;
        for (uint64_t j = i + 1; j < e; j++) {
          uint32_t d = g->adj[j];
          for (uint64_t x = g->off[b]; x < g->off[b + 1]; x++) {
            uint32_t c = g->adj[x];
            if (c <= v || c == d || !adjacent(g, d, c)) continue;
            uint32_t W[4] = {v, b, c, d}; uint32_t ed[4][2] = {{v, b}, {b, c}, {c, d}, {d, v}};
            fpm_record(g, t, 4, W, 4, ed);
          }
        }
      }
      /* paw: triangle v<u<w + pendant */
      for (uint64_t i = s; i < e; i++) {
        uint32_t u = g->adj[i];
        if (u <= v) continue;
        for (uint64_t j = i + 1; j < e; j++) {
          uint32_t w = g->adj[j];
          if (!adjacent(g, u, w)) continue;
          uint32_t tri[3] = {v, u, w};
          for (int xi = 0; xi < 3; xi++) {
            uint32_t x = tri[xi];
            for (uint64_t y = g->off[x]; y < g->off[x + 1]; y++) {
              uint32_t z = g->adj[y];
              if (z == v || z == u || z == w) continue;
              uint32_t W[4] = {v, u, w, z}; uint32_t ed[4][2] = {{v, u}, {v, w}, {u, w}, {x, z}};
              fpm_record(g, t, 4, W, 4, ed);
            }
          }
        }
      }
      /* 4-path a-b-v-d-c2 with middle vertex v, legs (b,a) < (d,c2) */
      for (uint64_t i = s; i < e; i++) {
        uint32_t b = g->adj[i];
        for (uint64_t j = s; j < e; j++) {
          uint32_t d = g->adj[j];
          if (d == b) continue;
          for (uint64_t x = g->off[b]; x < g->off[b + 1]; x++) {
            uint32_t a = g->adj[x];
            if (a == v || a == d) continue;
            for (uint64_t y = g->off[d]; y < g->off[d + 1]; y++) {
              uint32_t c2 = g->adj[y];
              if (c2 == v || c2 == b || c2 == a) continue;
              if (!(b < d || (b == d && a < c2))) continue;   /* unordered legs, once */
              uint32_t W[5] = {a, b, v, d, c2}; uint32_t ed[4][2] = {{a, b}, {b, v}, {v, d}, {d, c2}};
              fpm_record(g, t, 5, W, 4, ed);
            }
          }
        }
      }
      /* fork: centre v, long leg v-x-w, short legs y < z */
      for (uint64_t i = s; i < e; i++) {
        uint32_t x = g->adj[i];
        for (uint64_t q = g->off[x]; q < g->off[x + 1]; q++) {
          uint32_t w = g->adj[q];
          if (w == v) continue;
          for (uint64_t j = s; j < e; j++) {
            uint32_t y = g->adj[j];
            if (y == x || y == w) continue;
            for (uint64_t r = j + 1; r < e; r++) {
              uint32_t z = g->adj[r];
              if (z == x || z == w) continue;
              uint32_t W[5] = {v, x, w, y, z}; uint32_t ed[4][2] = {{v, x}, {x, w}, {v, y}, {v, z}};
              fpm_record(g, t, 5, W, 4, ed);
            }
          }
        }
      }
    }
  }
}

/* Brute-force enumeration (tiny graphs only): every set of 1..l distinct edges
 * whose edge set is connected, taken by its minimum edge id e1 < e2 < e3.  Edges
 * are ids into the list of undirected edges (u<v) in CSR order. */
static int edges_connected(uint32_t ne, const uint32_t (*ed)[2]) {
  uint32_t comp[FPM_MAXE]; for (uint32_t i = 0; i < ne; i++) comp[i] = i;
  for (int it = 0; it < FPM_MAXE; it++)
    for (uint32_t i = 0; i < ne; i++)
      for (uint32_t j = 0; j < ne; j++)
        if (ed[i][0] == ed[j][0] || ed[i][0] == ed[j][1] || ed[i][1] == ed[j][0] || ed[i][1] == ed[j][1]) {
          uint32_t c = comp[i] < comp[j] ? comp[i] : comp[j]; comp[i] = comp[j] = c;
        }
  for (uint32_t i = 0; i < ne; i++) if (comp[i] != 0) return 0;
  return 1;
}

static void fpm_enum_brute(const og_graph *g, og_ptab *t, uint32_t l) {
  uint64_t m = g->m, k = 0;
  uint32_t (*E)[2] = (uint32_t (*)[2])malloc((m ? m : 1) * sizeof(*E));
  for (uint32_t v = 0; v < g->n; v++)
    for (uint64_t i = g->off[v]; i < g->off[v + 1]; i++)
      if (g->adj[i] > v) { E[k][0] = v; E[k][1] = g->adj[i]; k++; }
  /* every set of ne = 1..l distinct edge ids i0 < i1 < ... (lexicographic odometer
   * over the first edge in parallel) */
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t a = 0; a < (int64_t)m; a++) {
    for (uint32_t ne = 1; ne <= l; ne++) {
      uint64_t ids[FPM_MAXE];
      ids[0] = (uint64_t)a;
      for (uint32_t i = 1; i < ne; i++) ids[i] = ids[i - 1] + 1;
      if (ne > 1 && ids[ne - 1] >= m) continue;
      for (;;) {
        uint32_t ed[FPM_MAXE][2];
        for (uint32_t i = 0; i < ne; i++) { ed[i][0] = E[ids[i]][0]; ed[i][1] = E[ids[i]][1]; }
        if (edges_connected(ne, (const uint32_t (*)[2])ed)) {
          uint32_t W[2 * FPM_MAXE], nv = 0;
          for (uint32_t e = 0; e < ne; e++)
            for (int s2 = 0; s2 < 2; s2++) {
              uint32_t x = ed[e][s2]; int f = 0;
              for (uint32_t w = 0; w < nv; w++) if (W[w] == x) f = 1;
              if (!f) W[nv++] = x;
            }
          if (nv <= FPM_MAXNV) fpm_record(g, t, nv, W, ne, (const uint32_t (*)[2])ed);
        }
        /* next combination with ids[0] fixed */
        int i = (int)ne - 1;
        while (i >= 1 && ids[i] == m - ne + (uint64_t)i) i--;
        if (i < 1) break;
        ids[i]++;
        for (uint32_t j = (uint32_t)i + 1; j < ne; j++) ids[j] = ids[j - 1] + 1;
      }
    }
  }
  free(E);
}

/* Result record layout (uint64 x 17):
 *   [0]=ne [1]=nv [2..6]=labels [7..14]=edge pairs (a0,b0,...,a3,b3) [15]=support
 *   [16]=number of edge sets (instances) mapped to the pattern. */
#define OG_REC 17

typedef struct { og_code c; uint64_t sup; uint64_t inst; } og_fres;

static int fres_cmp(const void *a, const void *b) {
  const og_fres *x = (const og_fres *)a, *y = (const og_fres *)b;
  if (x->c.ne != y->c.ne) return x->c.ne < y->c.ne ? -1 : 1;
  return code_cmp(&x->c, &y->c);
}

/* Run FPM.  method 0: shape enumeration, 1: brute-force edge subsets.
 * Writes up to max_out records into out; returns the number of frequent patterns
 * (which may exceed max_out), or <0 on error. */
int64_t og_fpm(const og_graph *g, uint32_t l, uint64_t minsup, int method, int threads,
               uint64_t max_out, uint64_t *out, uint64_t pattern_cap) {
  if (l < 1 || l > FPM_MAXE || minsup < 1) return OG_EINVAL;
  set_threads(threads);
  og_ptab t; memset(&t, 0, sizeof(t));
  t.cap = 1; while (t.cap < (pattern_cap ? pattern_cap : (1u << 16))) t.cap <<= 1;
  t.key = (og_code *)calloc(t.cap, sizeof(og_code));
  t.used = (int *)calloc(t.cap, sizeof(int));
  t.dom = (uint64_t **)calloc(t.cap, sizeof(uint64_t *));
  t.inst = (uint64_t *)calloc(t.cap, sizeof(uint64_t));
  t.words = ((uint64_t)g->n + 63) / 64;
  omp_init_lock(&t.lock);
  if (method == 0) fpm_enum_shapes(g, &t, l); else fpm_enum_brute(g, &t, l);
  int64_t nres = 0;
  og_fres *res = (og_fres *)malloc(t.cap * sizeof(og_fres));
  for (uint64_t h = 0; h < t.cap; h++) {
    if (t.used[h] != 2) continue;
    og_fres r; memset(&r, 0, sizeof(r)); r.c = t.key[h];
    uint64_t sup = UINT64_MAX;
    for (uint32_t i = 0; i < r.c.nv; i++) {
      uint64_t cnt = 0;
      for (uint64_t w = 0; w < t.words; w++) cnt += (uint64_t)__builtin_popcountll(t.dom[h][i * t.words + w]);
      if (cnt < sup) sup = cnt;
    }
    r.sup = sup;
    r.inst = t.inst[h];
    if (sup >= minsup) res[nres++] = r;
    free(t.dom[h]);
  }
  qsort(res, (size_t)nres, sizeof(og_fres), fres_cmp);
  for (int64_t i = 0; i < nres && (uint64_t)i < max_out; i++) {
    uint64_t *o = out + i * OG_REC;
    memset(o, 0, OG_REC * sizeof(uint64_t));
    o[0] = res[i].c.ne; o[1] = res[i].c.nv;
    for (int j = 0; j < FPM_MAXNV; j++) o[2 + j] = j < (int)res[i].c.nv ? res[i].c.lab[j] : 0;
    for (uint32_t e = 0; e < res[i].c.ne; e++) { o[7 + 2 * e] = res[i].c.e[e][0]; o[8 + 2 * e] = res[i].c.e[e][1]; }
    o[15] = res[i].sup;
    o[16] = res[i].inst;
  }
  int ovf = t.overflow;
  free(res); free(t.key); free(t.used); free(t.dom); free(t.inst);
  omp_destroy_lock(&t.lock);
  return ovf ? OG_ENOMEM : nres;
}

/* MNI support of ONE labeled pattern, by subgraph-matching enumeration (O-2's
 * enumerator, without symmetry breaking): domain(i) = {phi(i)} over all mappings.
 * Used for sampled FPM parity at full size and as an independent pin of og_fpm. */
int og_pattern_mni(const og_graph *g, uint32_t nv, uint32_t ne, const uint32_t *edges,
                   const uint32_t *plabels, int threads, uint64_t *support) {
  og_pat p;
  int st = pat_init(&p, nv, ne, edges, plabels);
  if (st) return st;
  set_threads(threads);
  uint64_t words = ((uint64_t)g->n + 63) / 64;
  uint64_t *dom = (uint64_t *)calloc(nv * words, sizeof(uint64_t));
  uint32_t r = p.order[0];
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t v = 0; v < (int64_t)g->n; v++) {
    if (p.labeled && g->lab[v] != p.plab[r]) continue;
    /* explicit DFS stack over match_rec's recursion so every mapping is visited */
    uint32_t phi[OG_MAXV]; uint64_t it[OG_MAXV];
    phi[r] = (uint32_t)v;
    uint32_t pos = 1;
    if (p.nv == 1) { __atomic_fetch_or(&dom[r * words + v / 64], 1ull << (v % 64), __ATOMIC_RELAXED); continue; }
    it[1] = g->off[phi[p.parent[1]]];
    while (pos >= 1) {
      uint32_t q = p.order[pos], par = p.parent[pos], base = phi[par];
      int advanced = 0;
      while (it[pos] < g->off[base + 1]) {
        uint32_t x = g->adj[it[pos]++];
        if (p.labeled && g->lab[x] != p.plab[q]) continue;
        int ok = 1;
        for (uint32_t i = 0; i < pos && ok; i++) if (phi[p.order[i]] == x) ok = 0;
        for (uint32_t i = 0; i < pos && ok; i++) {
          uint32_t b = p.order[i];
          if (b != par && p.adjm[q][b] && !adjacent(g, phi[b], x)) ok = 0;
        }
        if (!ok) continue;
        phi[q] = x;
        if (pos + 1 == p.nv) {
          for (uint32_t i = 0; i < p.nv; i++)
            __atomic_fetch_or(&dom[i * words + phi[i] / 64], 1ull << (phi[i] % 64), __ATOMIC_RELAXED);
          continue;
        }
        advanced = 1;
        break;
      }
      if (advanced) { pos++; it[pos] = g->off[phi[p.parent[pos]]]; }
      else pos--;
    }
  }
  uint64_t sup = UINT64_MAX;
  for (uint32_t i = 0; i < nv; i++) {
    uint64_t c = 0;
    for (uint64_t w = 0; w < words; w++) c += (uint64_t)__builtin_popcountll(dom[i * words + w]);
    if (c < sup) sup = c;
  }
  free(dom);
  *support = sup;
  return OG_OK;
}
