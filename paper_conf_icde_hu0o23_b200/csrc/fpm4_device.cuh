// fpm4_device.cuh -- FPM level 4 (4-edge patterns, <= 5 vertices),
// device side.  Included by fpm.cu inside its anonymous namespace (uses FpmArgs, Table,
// canonical(), table_slot(), ekey(), shares(), labof()).
//
// Level 4 is aggregated out of core (Opt 3): the number of distinct
// 4-edge patterns times one MNI bitmap per position does not fit any memory, so each
// embedding emits one 64-bit tuple per vertex,
//     (pattern slot << 35) | (orbit representative << 32) | vertex,
// into an HBM buffer; a pass of root-edge batches ends in a segment sort + unique of its
// tuples (a sorted "run"), and the runs are multi-merged by key range with matched
// indices (Def. 5.1, Alg. 3) so that |domain(pattern, orbit)| = the number of distinct
// tuples of that (slot, orbit) (fpm.cu, fpm_level4).
//
// Generation rule (reading R11 extended): a connected edge set S is produced once, from
// its canonical growth sequence s1 = min(S), s_{i+1} = the smallest edge of S adjacent to
// V(s1..s_i).  The level-3 prefixes (e1, e2, e3) the enumeration produces are such
// sequences; a 4th edge e extends one iff e > s1, e is adjacent to V(P), e is not in P,
// not (e ~ V(s1) and e < s2) and not (e ~ V(s1, s2) and e < s3).
#pragma once

constexpr int kCanon5Entries = 1 << 14;   // (10-bit sorted-position edge mask) x (4-bit tie mask)
constexpr uint32_t kL4Pad = 0x3ffu;       // padding label: sorts after every label < 256
constexpr int kQ4 = 64;                    // level-3 prefixes queued per warp
constexpr int kQ4Words = 10;

// pair index of positions p < q of a <= 5-vertex pattern, in lexicographic (p, q) order:
// (0,1)0 (0,2)1 (0,3)2 (0,4)3 (1,2)4 (1,3)5 (1,4)6 (2,3)7 (2,4)8 (3,4)9
__host__ __device__ __forceinline__ uint32_t pid5(uint32_t p, uint32_t q) {
  return p * (9 - p) / 2 + (q - p - 1);
}
__host__ __device__ __forceinline__ uint32_t pid5u(uint32_t a, uint32_t b) { return a < b ? pid5(a, b) : pid5(b, a); }
// endpoints of pair i (3 bits each)
constexpr uint32_t kA5 = 0u | 0u << 3 | 0u << 6 | 0u << 9 | 1u << 12 | 1u << 15 | 1u << 18 | 2u << 21 | 2u << 24 | 3u << 27;
constexpr uint32_t kB5 = 1u | 2u << 3 | 3u << 6 | 4u << 9 | 2u << 12 | 3u << 15 | 4u << 18 | 3u << 21 | 4u << 24 | 4u << 27;

// 5-element sorting network (9 comparators), also checked exhaustively on the host
__host__ __device__ __forceinline__ void sort5(uint32_t &c0, uint32_t &c1, uint32_t &c2, uint32_t &c3, uint32_t &c4) {
#define GAMMA_CX5(x, y)                 \
  {                                     \
    const uint32_t t_ = x < y ? x : y;  \
    y = x < y ? y : x;                  \
    x = t_;                             \
  }
  GAMMA_CX5(c0, c1);
  GAMMA_CX5(c3, c4);
  GAMMA_CX5(c2, c4);
  GAMMA_CX5(c2, c3);
  GAMMA_CX5(c1, c4);
  GAMMA_CX5(c0, c3);
  GAMMA_CX5(c0, c2);
  GAMMA_CX5(c1, c3);
  GAMMA_CX5(c1, c2);
#undef GAMMA_CX5
}

// Key of a <= 5-vertex pattern: bits 0..39 five 8-bit labels (canonical order), 40..55
// the sorted pair indices of its <= 4 edges (4 bits each, first edge most significant,
// unused 0xf), 56..58 nv, 59..61 ne, 63 set.
__host__ __device__ __forceinline__ uint32_t key5_nv(uint64_t k) { return (uint32_t)((k >> 56) & 7); }
__host__ __device__ __forceinline__ uint32_t key5_ne(uint64_t k) { return (uint32_t)((k >> 59) & 7); }
__host__ __device__ __forceinline__ uint32_t key5_edges(uint64_t k) { return (uint32_t)((k >> 40) & 0xffff); }
__host__ __device__ __forceinline__ uint32_t key5_label(uint64_t k, uint32_t p) { return (uint32_t)((k >> (8 * p)) & 0xff); }

struct Fpm4Args {
  const uint2 *tab5;            // kCanon5Entries: {edge key, sg0 (3 bits / canonical position) | orbit reps << 15}
  unsigned long long *key4;     // level-4 pattern table (0 = empty), cap4 slots (power of two)
  unsigned long long *inst4;    // nullable: per-slot instances of this pass
  uint64_t cap4;
  unsigned long long *tup;      // tuple buffer of this pass
  uint64_t tup_cap;
  unsigned long long *flags;    // [0] tuple cursor, [1] tuple buffer full, [2] pattern table full, [3] embeddings
  uint64_t b_begin, b_end;      // root-edge batch range of this pass
};

__device__ __forceinline__ int64_t slot4(const Fpm4Args &b, uint64_t key) {
  uint64_t h = mix64(key) & (b.cap4 - 1);
  const uint64_t max_probe = b.cap4 < 4096 ? b.cap4 : 4096;
  for (uint64_t probe = 0; probe < max_probe; probe++, h = (h + 1) & (b.cap4 - 1)) {
    const unsigned long long k = __ldcg(b.key4 + h);
    if (k == key) return (int64_t)h;
    if (k == 0) {
      const unsigned long long prev = atomicCAS(b.key4 + h, 0ull, (unsigned long long)key);
      if (prev == 0 || prev == key) return (int64_t)h;
    }
  }
  atomicExch(b.flags + 2, 1ull);
  return -1;
}

// Canonical code of a connected 4-edge set on nv <= 5 local vertices (labels l[i] < 256,
// local pair mask em over pid5), and for each canonical position c its vertex (under the
// first minimizing order) and orbit representative.
struct Canon5 {
  uint64_t key;
  uint32_t vtx[5];
  uint32_t rep[5];
};

__device__ __forceinline__ Canon5 canonical5(const uint2 *tab, const uint32_t (&l)[5], const uint32_t (&v)[5],
                                            uint32_t nv, uint32_t em) {
  uint32_t c0 = (l[0] << 3) | 0u, c1 = ((nv > 1 ? l[1] : kL4Pad) << 3) | 1u, c2 = ((nv > 2 ? l[2] : kL4Pad) << 3) | 2u;
  uint32_t c3 = ((nv > 3 ? l[3] : kL4Pad) << 3) | 3u, c4 = ((nv > 4 ? l[4] : kL4Pad) << 3) | 4u;
  sort5(c0, c1, c2, c3, c4);
  const uint32_t cs[5] = {c0, c1, c2, c3, c4};
  uint32_t pos = 0;   // sorted position of local i in bits 3i
#pragma unroll
  for (uint32_t s = 0; s < 5; s++) pos |= s << (3 * (cs[s] & 7u));
  uint32_t M = 0;
#pragma unroll
  for (uint32_t i = 0; i < 10; i++)
    if ((em >> i) & 1u) {
      const uint32_t pa = (pos >> (3 * ((kA5 >> (3 * i)) & 7u))) & 7u;
      const uint32_t pb = (pos >> (3 * ((kB5 >> (3 * i)) & 7u))) & 7u;
      M |= 1u << pid5u(pa, pb);
    }
  uint32_t tie = 0;
#pragma unroll
  for (uint32_t s = 0; s < 4; s++)
    if (s + 1 < nv && (cs[s] >> 3) == (cs[s + 1] >> 3)) tie |= 1u << s;
  const uint2 e = tab[(M << 4) | tie];
  Canon5 r;
  r.key = (1ull << 63) | ((uint64_t)__popc(M) << 59) | ((uint64_t)nv << 56) | ((uint64_t)(e.x & 0xffffu) << 40);
#pragma unroll
  for (uint32_t s = 0; s < 5; s++)
    if (s < nv) r.key |= (uint64_t)((cs[s] >> 3) & 0xffu) << (8 * s);
#pragma unroll
  for (uint32_t c = 0; c < 5; c++) {
    const uint32_t sp = (e.y >> (3 * c)) & 7u;        // sorted position placed at canonical c
    const uint32_t loc = cs[sp < 5 ? sp : 0] & 7u;   // its local index
    uint32_t x = v[0];
#pragma unroll
    for (uint32_t q = 1; q < 5; q++)
      if (loc == q) x = v[q];
    r.vtx[c] = x;
    r.rep[c] = (e.y >> (15 + 3 * c)) & 7u;
  }
  return r;
}

// Is the pattern of a 3-edge prefix on nv <= 4 vertices (local mask em over pid) frequent?
__device__ __forceinline__ bool frequent4(const FpmArgs &a, const uint2 *tab, uint32_t l0, uint32_t l1, uint32_t l2,
                                          uint32_t l3, uint32_t nv, uint32_t em) {
  const Canon cn = canonical(tab, l0, l1, l2, l3, nv, em);
  unsigned long long d;
  const int64_t s = table_slot(a, cn.key, false, d);
  return s >= 0 && a.T.freq[s];
}

// pid (4-vertex pair index) mask -> pid5 mask
__device__ __forceinline__ uint32_t em4_to_em5(uint32_t em) {
  uint32_t r = 0;
#pragma unroll
  for (uint32_t i = 0; i < 6; i++)
    if ((em >> i) & 1u) r |= 1u << pid5((kPairA >> (2 * i)) & 3u, (kPairB >> (2 * i)) & 3u);
  return r;
}

// Level-4 extension of up to 32 queued 3-edge prefixes (lane k <-> queue entry k): their
// candidate 4th edges N(u) ++ N(v) ++ N(y) (++ N(z)) are streamed in flattened windows
// by all 32 lanes; every valid extension gets its canonical code, pattern slot and nv
// tuples (deduplicated across the warp by __match_any_sync before the write).
__device__ void level4_flush(const FpmArgs &a, const Fpm4Args &b, const uint2 *tab5, const uint32_t *q, uint32_t cnt,
                             int lane, uint64_t &emb, uint64_t &elems, bool &stop) {
  // entry words: 0 u, 1 v, 2 y, 3 z, 4 labels (4 x 8 bits), 5 em5 | nv3 << 16, 6/7 e2, 8/9 e3
  uint32_t u = 0, v = 0, y = 0, z = 0, lb = 0, meta = 0, du = 0, dv = 0, dy = 0, dz = 0;
  uint64_t su = 0, sv = 0, sy = 0, sz = 0, e2 = 0, e3 = 0;
  if (lane < (int)cnt) {
    const uint32_t *w = q + lane * kQ4Words;
    u = w[0]; v = w[1]; y = w[2]; z = w[3]; lb = w[4]; meta = w[5];
    e2 = ((uint64_t)w[7] << 32) | w[6];
    e3 = ((uint64_t)w[9] << 32) | w[8];
    su = a.rp[u]; du = (uint32_t)(a.rp[u + 1] - su);
    sv = a.rp[v]; dv = (uint32_t)(a.rp[v + 1] - sv);
    sy = a.rp[y]; dy = (uint32_t)(a.rp[y + 1] - sy);
    if ((meta >> 16) == 4) { sz = a.rp[z]; dz = (uint32_t)(a.rp[z + 1] - sz); }
  }
  const uint32_t tl = du + dv + dy + dz;
  uint32_t sc = tl;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t t = __shfl_up_sync(0xffffffffu, sc, o);
    if (lane >= o) sc += t;
  }
  const uint32_t T = __shfl_sync(0xffffffffu, sc, 31);
  if (lane == 0) elems += T;
  const uint32_t ost = sc - tl;
  const uint32_t upto = lane == 31 ? 0xffffffffu : ((2u << lane) - 1u);
  uint32_t nb = 0;
  for (uint32_t t0 = 0; t0 < T; t0 += 32) {
    if (*(volatile unsigned long long *)(b.flags + 1)) {
      stop = true;
      return;
    }
    const uint32_t t = t0 + lane;
    // the entry owning element t: the last one starting at or before t (every queued
    // prefix has tl > 0 -- its vertices have degree >= 1 -- so starts strictly increase)
    const uint32_t mine = (lane < (int)cnt && ost >= t0 && ost < t0 + 32) ? (1u << (ost - t0)) : 0u;
    const uint32_t S = __reduce_or_sync(0xffffffffu, mine);
    const int j = ((int)(nb + __popc(S & upto)) - 1) & 31;
    nb += __popc(S);
    const uint32_t ju = __shfl_sync(0xffffffffu, u, j), jv = __shfl_sync(0xffffffffu, v, j);
    const uint32_t jy = __shfl_sync(0xffffffffu, y, j), jz = __shfl_sync(0xffffffffu, z, j);
    const uint32_t jlb = __shfl_sync(0xffffffffu, lb, j), jmeta = __shfl_sync(0xffffffffu, meta, j);
    const uint32_t jdu = __shfl_sync(0xffffffffu, du, j), jdv = __shfl_sync(0xffffffffu, dv, j);
    const uint32_t jdy = __shfl_sync(0xffffffffu, dy, j), jost = __shfl_sync(0xffffffffu, ost, j);
    const uint64_t jsu = __shfl_sync(0xffffffffu, su, j), jsv = __shfl_sync(0xffffffffu, sv, j);
    const uint64_t jsy = __shfl_sync(0xffffffffu, sy, j), jsz = __shfl_sync(0xffffffffu, sz, j);
    const uint64_t je2 = __shfl_sync(0xffffffffu, e2, j), je3 = __shfl_sync(0xffffffffu, e3, j);
    bool ok = t < T;
    uint32_t w = 0, lw = 0, zp = 0;
    if (ok) {
      const uint32_t r = t - jost;
      uint64_t zi;
      if (r < jdu) { w = ju; lw = 0; zi = jsu + r; }
      else if (r < jdu + jdv) { w = jv; lw = 1; zi = jsv + (r - jdu); }
      else if (r < jdu + jdv + jdy) { w = jy; lw = 2; zi = jsy + (r - jdu - jdv); }
      else { w = jz; lw = 3; zi = jsz + (r - jdu - jdv - jdy); }
      zp = a.col[zi];
    }
    const uint32_t nv3 = jmeta >> 16;
    uint32_t lz = zp == ju ? 0u : zp == jv ? 1u : zp == jy ? 2u : (nv3 == 4 && zp == jz) ? 3u : nv3;
    const bool closes = lz < nv3;
    if (ok && closes && zp < w) ok = false;   // seen from both ends: keep the smaller
    const uint64_t e1 = ekey(ju, jv), e4 = ekey(w, zp);
    if (ok && (e4 == e1 || e4 == je2 || e4 == je3)) ok = false;
    if (ok) {
      const bool touch12 = w == ju || w == jv || w == jy || zp == ju || zp == jv || zp == jy;
      ok = e4 > e1 && !(shares(e4, e1) && e4 < je2) && !(touch12 && e4 < je3);
    }
    uint32_t lz_lab = 0;
    if (ok && !closes) {
      lz_lab = labof(a, zp);
      ok = lz_lab < 256u;   // (the host rejects graphs with labels >= 256 for l = 4)
    }
    Canon5 cn;
    uint32_t nv4 = 0;
    int64_t sl = -1;
    if (ok) {
      uint32_t l[5] = {jlb & 0xffu, (jlb >> 8) & 0xffu, (jlb >> 16) & 0xffu, (jlb >> 24) & 0xffu, 0u};
      if (!closes) {
        if (nv3 == 3) l[3] = lz_lab;
        else l[4] = lz_lab;
      }
      const uint32_t vv[5] = {ju, jv, jy, nv3 == 4 ? jz : zp, zp};
      nv4 = closes ? nv3 : nv3 + 1;
      const uint32_t em = (jmeta & 0xffffu) | (1u << pid5u(lw, lz));
      cn = canonical5(tab5, l, vv, nv4, em);
      sl = slot4(b, cn.key);
      ok = sl >= 0;
    }
    if (ok) {
      emb++;
      if (b.inst4) atomicAdd(b.inst4 + sl, 1ull);
    }
    // tuples, deduplicated across the warp (the prefix vertices repeat across lanes)
    uint32_t wbits = 0;
    unsigned long long tv[5];
#pragma unroll
    for (uint32_t c = 0; c < 5; c++) {
      tv[c] = (ok && c < nv4) ? (((unsigned long long)sl << 35) | ((unsigned long long)cn.rep[c] << 32) | cn.vtx[c])
                              : 0ull;
      const uint32_t mm = __match_any_sync(0xffffffffu, tv[c]);
      if (tv[c] && (__ffs(mm) - 1) == lane) wbits |= 1u << c;
    }
    const uint32_t nw = __popc(wbits);
    uint32_t ex = nw;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t x = __shfl_up_sync(0xffffffffu, ex, o);
      if (lane >= o) ex += x;
    }
    const uint32_t tot = __shfl_sync(0xffffffffu, ex, 31);
    ex -= nw;
    unsigned long long base = 0;
    if (lane == 0 && tot) base = atomicAdd(b.flags + 0, (unsigned long long)tot);
    base = __shfl_sync(0xffffffffu, base, 0);
    if (tot && base + tot > b.tup_cap) {
      if (lane == 0) atomicExch(b.flags + 1, 1ull);
      stop = true;
      return;
    }
    uint32_t k = 0;
#pragma unroll
    for (uint32_t c = 0; c < 5; c++)
      if ((wbits >> c) & 1u) b.tup[base + ex + k++] = tv[c];
  }
}

// One warp per batch of root edges of this pass; levels 1-3 regenerated with Alg. 2's
// pruning (frequent edge, wedge and 3-edge patterns, looked up in the level <= 3 table),
// frequent 3-edge prefixes queued in shared memory and extended by level4_flush.
__global__ void __launch_bounds__(kThreads) fpm_enum4_kernel(FpmArgs a, Fpm4Args b) {
  __shared__ uint2 s_tab[kCanonEntries];
  __shared__ uint32_t s_q[kThreads / 32][kQ4 * kQ4Words];
  for (int i = threadIdx.x; i < kCanonEntries; i += blockDim.x) s_tab[i] = a.canon_tab[i];
  __syncthreads();
  const int lane = threadIdx.x & 31;
  uint32_t *Q = s_q[threadIdx.x >> 5];
  uint32_t qn = 0;
  uint64_t emb = 0, elems = 0;
  bool stop = false;
  const uint64_t ndir = a.rp[a.n];
  constexpr uint64_t kBatch = 8;
  for (;;) {
    if (stop) break;
    unsigned long long bi = 0;
    if (lane == 0) bi = atomicAdd(&a.ctrl[CTRL_WORK], 1ull);
    bi = __shfl_sync(0xffffffffu, bi, 0) + b.b_begin;
    if (bi >= b.b_end) break;
    if (*(volatile unsigned long long *)(b.flags + 1)) break;
    const uint64_t i0 = (bi * a.world + a.rank) * kBatch;
    if (i0 >= ndir) break;
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
    for (uint64_t i1 = i0; i1 < iend && !stop; i1++) {
      while (a.rp[u + 1] <= i1) u++;
      const uint32_t v = a.col[i1];
      if (v < u) continue;
      const uint64_t us = a.rp[u], ue = a.rp[u + 1];
      const uint64_t e1 = ekey(u, v);
      const uint32_t lu = labof(a, u), lv = labof(a, v);
      if (!frequent(a, s_tab, lu, lv, 0u, 2, 1u << pid(0, 1))) continue;
      const uint64_t vs = a.rp[v], ve = a.rp[v + 1];
      const uint64_t nu = ue - us, ncand = nu + (ve - vs);
      if (lane == 0) elems += ncand;
      for (uint64_t c0 = 0; c0 < ncand && !stop; c0 += 32) {
        const uint64_t ci = c0 + lane;
        bool valid = ci < ncand;
        uint64_t e2 = 0;
        uint32_t y = 0, ly = 0, em2 = 0;
        if (valid) {
          const bool at_u = ci < nu;
          y = at_u ? a.col[us + ci] : a.col[vs + (ci - nu)];
          e2 = ekey(at_u ? u : v, y);
          valid = e2 > e1;
          em2 = (1u << pid(0, 1)) | (1u << pid(at_u ? 0 : 1, 2));
        }
        if (valid) {
          ly = labof(a, y);
          valid = frequent(a, s_tab, lu, lv, ly, 3, em2);
        }
        const uint32_t du = (uint32_t)nu, dv = (uint32_t)(ve - vs);
        uint32_t by = 0, dy = 0;
        if (valid) {
          by = (uint32_t)a.rp[y];
          dy = (uint32_t)(a.rp[y + 1] - by);
        }
        const uint32_t tl = valid ? du + dv + dy : 0u;
        const uint32_t nz = __ballot_sync(0xffffffffu, tl > 0);
        const uint32_t nnz = __popc(nz);
        const uint32_t src = lane < (int)nnz ? __fns(nz, 0, lane + 1) : 0;
        const uint32_t cy = __shfl_sync(0xffffffffu, y, src);
        const uint32_t cl = __shfl_sync(0xffffffffu, ly | (em2 << 16), src);
        const uint32_t cby = __shfl_sync(0xffffffffu, by, src);
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
        for (uint32_t t0 = 0; t0 < T && !stop; t0 += 32) {
          const uint32_t t = t0 + lane;
          const uint32_t mine = (lane < (int)nnz && ost >= t0 && ost < t0 + 32) ? (1u << (ost - t0)) : 0u;
          const uint32_t S = __reduce_or_sync(0xffffffffu, mine);
          const int j = ((int)(nb + __popc(S & upto)) - 1) & 31;
          nb += __popc(S);
          const uint32_t py = __shfl_sync(0xffffffffu, cy, j);
          const uint32_t pl = __shfl_sync(0xffffffffu, cl, j);
          const uint32_t pby = __shfl_sync(0xffffffffu, cby, j);
          const uint32_t oj = __shfl_sync(0xffffffffu, ost, j);
          bool ok = t < T;
          uint32_t w = 0, z = 0, lw = 0, lz = 3, em3 = 0, l3 = 0;
          uint64_t pe2 = 0, e3 = 0;
          if (ok) {
            const uint32_t r = t - oj;
            uint32_t zi;
            if (r < du) { w = u; zi = (uint32_t)us + r; lw = 0; }
            else if (r < du + dv) { w = v; zi = (uint32_t)vs + (r - du); lw = 1; }
            else { w = py; zi = pby + (r - du - dv); lw = 2; }
            z = a.col[zi];
            lz = z == u ? 0u : z == v ? 1u : z == py ? 2u : 3u;
            if (lz < 3 && z < w) ok = false;
            pe2 = ekey((pl >> 16) & (1u << pid(1, 2)) ? v : u, py);
            e3 = ekey(w, z);
            if (ok && (e3 == e1 || e3 == pe2)) ok = false;
            if (ok) ok = (e3 > pe2) || (e3 > e1 && shares(e3, pe2) && !shares(e3, e1));
            if (ok) {
              em3 = (pl >> 16) | (1u << pid(lw, lz));
              l3 = lz == 3 ? labof(a, z) : 0u;
              ok = frequent4(a, s_tab, lu, lv, pl & 0xffffu, l3, lz == 3 ? 4 : 3, em3);
            }
          }
          // queue the frequent prefixes (ballot compaction into shared memory)
          const uint32_t bal = __ballot_sync(0xffffffffu, ok);
          if (ok) {
            uint32_t *e = Q + (qn + __popc(bal & lanemask_lt())) * kQ4Words;
            e[0] = u; e[1] = v; e[2] = py; e[3] = z;
            e[4] = (lu & 0xffu) | (lv & 0xffu) << 8 | (pl & 0xffu) << 16 | (l3 & 0xffu) << 24;
            e[5] = em4_to_em5(em3) | ((lz == 3 ? 4u : 3u) << 16);
            e[6] = (uint32_t)pe2; e[7] = (uint32_t)(pe2 >> 32);
            e[8] = (uint32_t)e3; e[9] = (uint32_t)(e3 >> 32);
          }
          qn += __popc(bal);
          __syncwarp();
          if (qn >= 32) {
            level4_flush(a, b, b.tab5, Q, 32, lane, emb, elems, stop);
            __syncwarp();
            // move the rest (< 32 entries) to the front
            for (uint32_t i = lane; i < (qn - 32) * kQ4Words; i += 32) Q[i] = Q[32 * kQ4Words + i];
            qn -= 32;
            __syncwarp();
          }
        }
      }
    }
    if (qn && !stop) {   // drain the queue at the end of the batch
      level4_flush(a, b, b.tab5, Q, qn, lane, emb, elems, stop);
      qn = 0;
      __syncwarp();
    }
  }
  for (int off = 16; off > 0; off >>= 1) {
    emb += __shfl_down_sync(0xffffffffu, emb, off);
    elems += __shfl_down_sync(0xffffffffu, elems, off);
  }
  if (lane == 0 && emb) atomicAdd(b.flags + 3, (unsigned long long)emb);
  if (lane == 0 && elems) atomicAdd(&a.ctrl[CTRL_ELEMS], (unsigned long long)elems);
}

// sorted unique tuples -> |domain| per (slot, orbit representative): each thread a
// contiguous chunk, one atomic per run of equal (slot, orbit)
__global__ void count_tuples_kernel(const unsigned long long *keys, uint64_t n, uint32_t *cnt) {
  constexpr uint64_t kChunk = 32;
  for (uint64_t c = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; c * kChunk < n;
       c += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t b0 = c * kChunk, b1 = b0 + kChunk < n ? b0 + kChunk : n;
    uint64_t cur = keys[b0] >> 32;
    uint32_t run = 0;
    for (uint64_t i = b0; i < b1; i++) {
      const uint64_t g = keys[i] >> 32;
      if (g != cur) {
        atomicAdd(cnt + cur, run);
        cur = g;
        run = 0;
      }
      run++;
    }
    atomicAdd(cnt + cur, run);
  }
}

// support of every level-4 slot: min over its orbit representatives' counts (only
// representatives carry tuples, and every one of an occurring pattern has >= 1)
__global__ void support4_kernel(const unsigned long long *key4, uint64_t cap4, const uint32_t *cnt,
                                unsigned long long *sup) {
  for (uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; s < cap4; s += (uint64_t)gridDim.x * blockDim.x) {
    if (key4[s] == 0) {
      sup[s] = 0;
      continue;
    }
    uint32_t m = 0xffffffffu;
    for (uint32_t c = 0; c < 8; c++) {
      const uint32_t x = cnt[s * 8 + c];
      if (x && x < m) m = x;
    }
    sup[s] = m == 0xffffffffu ? 0 : m;
  }
}

// lower bound of `key` in each sorted run (matched index, Def. 5.1) for device runs
__global__ void lower_bound_kernel(const unsigned long long *run, uint64_t len, const unsigned long long *keys,
                                   uint32_t nkeys, uint64_t *out) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= nkeys) return;
  const unsigned long long k = keys[i];
  uint64_t lo = 0, hi = len;
  while (lo < hi) {
    const uint64_t mid = (lo + hi) >> 1;
    if (run[mid] < k) lo = mid + 1; else hi = mid;
  }
  out[i] = lo;
}

__global__ void add_u64_kernel(unsigned long long *dst, const unsigned long long *src, uint64_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    dst[i] += src[i];
}
