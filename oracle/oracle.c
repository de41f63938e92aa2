/*
 * oracle.c -- CPU ORACLE (test infrastructure only; see oracle.h header).
 *
 * Plain sequential C written from PAPER.md and the readings in DESIGN.md.
 * No blocking, no fusion, no parallelism: a reader should be able to check
 * each loop against the cited passage by eye.
 */
#include "oracle.h"

#include <stdlib.h>
#include <string.h>

/* ---------------------------------------------------------------------------
 * RNG.  Philox4x32-10 exactly as Random123 defines it (multipliers
 * 0xD2511F53 / 0xCD9E8D57, Weyl key bumps 0x9E3779B9 / 0xBB67AE85).  The
 * paper does not name its RNG (reading Q4); a counter-based generator makes
 * each draw a pure function of (seed, vertex, slot, batch, epoch, hop), so a
 * sample is one well-defined value and any parallel schedule can reproduce it.
 * ------------------------------------------------------------------------- */
void orc_philox(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
  uint32_t x0 = ctr[0], x1 = ctr[1], x2 = ctr[2], x3 = ctr[3];
  uint32_t k0 = key[0], k1 = key[1];
  for (int round = 0; round < 10; ++round) {
    if (round > 0) {
      k0 += 0x9E3779B9u;
      k1 += 0xBB67AE85u;
    }
    uint64_t prod0 = (uint64_t)0xD2511F53u * (uint64_t)x0;
    uint64_t prod1 = (uint64_t)0xCD9E8D57u * (uint64_t)x2;
    uint32_t hi0 = (uint32_t)(prod0 >> 32), lo0 = (uint32_t)prod0;
    uint32_t hi1 = (uint32_t)(prod1 >> 32), lo1 = (uint32_t)prod1;
    uint32_t y0 = hi1 ^ x1 ^ k0;
    uint32_t y1 = lo1;
    uint32_t y2 = hi0 ^ x3 ^ k1;
    uint32_t y3 = lo0;
    x0 = y0; x1 = y1; x2 = y2; x3 = y3;
  }
  out[0] = x0; out[1] = x1; out[2] = x2; out[3] = x3;
}

uint32_t orc_c3(uint32_t epoch, uint32_t hop, uint32_t domain) {
  return ((epoch & 0xFFFFu) << 16) | ((hop & 0xFFu) << 8) | (domain & 0xFFu);
}

uint64_t orc_draw64(uint64_t seed, uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3, int half) {
  uint32_t ctr[4] = {c0, c1, c2, c3};
  uint32_t key[2] = {(uint32_t)(seed & 0xFFFFFFFFu), (uint32_t)(seed >> 32)};
  uint32_t w[4];
  orc_philox(ctr, key, w);
  if (half == 0) return ((uint64_t)w[1] << 32) | (uint64_t)w[0];
  return ((uint64_t)w[3] << 32) | (uint64_t)w[2];
}

uint32_t orc_bounded(uint64_t r, uint32_t n) {
  unsigned __int128 p = (unsigned __int128)r * (unsigned __int128)n;
  return (uint32_t)(p >> 64);
}

/* ---------------------------------------------------------------------------
 * a1: epoch shuffle (§6.2).  A permutation defined as a sort
 * of per-index random keys, ties broken by index.
 * ------------------------------------------------------------------------- */
typedef struct { uint64_t key; uint64_t idx; } orc_keyed;

static int orc_cmp_keyed(const void* a, const void* b) {
  const orc_keyed* x = (const orc_keyed*)a;
  const orc_keyed* y = (const orc_keyed*)b;
  if (x->key != y->key) return x->key < y->key ? -1 : 1;
  if (x->idx != y->idx) return x->idx < y->idx ? -1 : 1;
  return 0;
}

int orc_shuffle(const uint32_t* T, uint64_t n, uint64_t seed, uint32_t epoch, uint32_t* out) {
  if (epoch > 0xFFFFu) return ORC_ERANGE;
  if (n > 0xFFFFFFFFull) return ORC_ERANGE;
  orc_keyed* a = (orc_keyed*)malloc(sizeof(orc_keyed) * (n ? n : 1));
  if (!a) return ORC_ENOMEM;
  uint32_t c3 = orc_c3(epoch, 0, ORC_SHUFFLE);
  for (uint64_t i = 0; i < n; ++i) {
    a[i].key = orc_draw64(seed, (uint32_t)i, 0, 0, c3, 0);
    a[i].idx = i;
  }
  qsort(a, n, sizeof(orc_keyed), orc_cmp_keyed);
  for (uint64_t j = 0; j < n; ++j) out[j] = T[a[j].idx];
  free(a);
  return ORC_OK;
}

/* ---------------------------------------------------------------------------
 * Relabel helper state ("the sampled vertices may be
 * deduplicated and reassigned with consecutive IDs (starting from 0)";
 * reading Q5: seeds get 0..n0-1 in the given order, every later vertex gets
 * the next id at its first occurrence in (frontier vertex, slot) order).
 * ------------------------------------------------------------------------- */
typedef struct {
  int32_t* lid;      /* lid[gid] or -1 */
  uint32_t* uniq;    /* gid by lid */
  uint64_t n;        /* |uniq| */
  uint64_t cap;
} orc_relabel;

/* returns lid of u, inserting it if unseen; -1 when uniq is full */
static int64_t orc_lid_of(orc_relabel* r, uint32_t u) {
  if (r->lid[u] < 0) {
    if (r->n >= r->cap) return -1;
    r->lid[u] = (int32_t)r->n;
    r->uniq[r->n] = u;
    r->n += 1;
  }
  return r->lid[u];
}

static void orc_relabel_reset(orc_relabel* r) {
  for (uint64_t i = 0; i < r->n; ++i) r->lid[r->uniq[i]] = -1;
}

static int orc_insert_seeds(orc_relabel* r, const uint32_t* seeds, uint64_t n0, uint64_t V) {
  for (uint64_t i = 0; i < n0; ++i) {
    if (seeds[i] >= V) return ORC_EINVAL;              /* id out of range */
    if (r->lid[seeds[i]] >= 0) return ORC_EINVAL;      /* duplicate seed (reading Q6) */
    if (orc_lid_of(r, seeds[i]) < 0) return ORC_ENOMEM;
  }
  return ORC_OK;
}

/* ---------------------------------------------------------------------------
 * a2 + a3: k-hop uniform neighbourhood sampling (Fig 7: per hop
 * i, nbrs = uniform_select(nbrs, sizes[i])) with dedup/remap (Fig 9).
 *
 * uniform_select for one vertex v with n = deg(v) CSR positions and fanout
 * k (reading Q2):
 *   n <= k : all positions 0..n-1 in CSR order, no draws;
 *   n  > k : Floyd's algorithm -- for s = 0..k-1, j = n-k+s,
 *            t = bounded(draw64(v, s>>1, batch, c3(epoch,l,KHOP), s&1), j+1),
 *            choose t if t is not chosen yet, else j.
 * The frontier of hop l is every vertex discovered so far (reading Q3,
 * DGL block semantics): block l has dst = lids 0..n_l-1, src = 0..n_{l+1}-1.
 * ------------------------------------------------------------------------- */
int orc_sample_khop(const uint64_t* indptr, const uint32_t* indices, uint64_t V,
                    const uint32_t* seeds, uint64_t n0, const uint32_t* fanouts, uint32_t L,
                    uint64_t seed, uint32_t epoch, uint32_t batch, int32_t* lid_scratch,
                    uint32_t* uniq, uint64_t uniq_cap, uint64_t* sizes,
                    uint32_t* blk_indptr, uint64_t indptr_cap,
                    uint32_t* blk_indices, uint64_t indices_cap, uint64_t* nnz,
                    uint32_t* picks, uint64_t picks_cap) {
  if (epoch > 0xFFFFu || L > 0xFFu) return ORC_ERANGE;
  for (uint32_t l = 0; l < L; ++l)
    if (fanouts[l] == 0 || fanouts[l] > 1024) return ORC_EINVAL;
  orc_relabel r = {lid_scratch, uniq, 0, uniq_cap};
  int rc = orc_insert_seeds(&r, seeds, n0, V);
  if (rc != ORC_OK) { orc_relabel_reset(&r); return rc; }
  sizes[0] = r.n;

  uint64_t ip_off = 0, ix_off = 0, pk_off = 0;
  uint32_t chosen[1024];
  for (uint32_t l = 0; l < L; ++l) {
    uint32_t k = fanouts[l];
    uint64_t n_l = r.n;                     /* frontier = everything so far */
    uint32_t c3 = orc_c3(epoch, l, ORC_KHOP);
    if (ip_off + n_l + 1 > indptr_cap) { orc_relabel_reset(&r); return ORC_ENOMEM; }
    uint32_t* bptr = blk_indptr + ip_off;
    uint64_t e = 0;
    for (uint64_t d = 0; d < n_l; ++d) {
      uint32_t v = r.uniq[d];
      uint64_t lo = indptr[v];
      uint64_t deg = indptr[v + 1] - indptr[v];
      if (deg > 0xFFFFFFFFull) { orc_relabel_reset(&r); return ORC_ERANGE; }
      uint32_t n = (uint32_t)deg;
      uint32_t m;                           /* number chosen */
      if (n <= k) {
        for (uint32_t p = 0; p < n; ++p) chosen[p] = p;
        m = n;
      } else {
        for (uint32_t s = 0; s < k; ++s) {
          uint32_t j = n - k + s;
          uint64_t rr = orc_draw64(seed, v, s >> 1, batch, c3, (int)(s & 1u));
          uint32_t t = orc_bounded(rr, j + 1);
          int taken = 0;
          for (uint32_t q = 0; q < s; ++q)
            if (chosen[q] == t) taken = 1;
          chosen[s] = taken ? j : t;
        }
        m = k;
      }
      if (picks) {
        if (pk_off + (d + 1) * (uint64_t)k > picks_cap) { orc_relabel_reset(&r); return ORC_ENOMEM; }
        for (uint32_t s = 0; s < k; ++s)
          picks[pk_off + d * k + s] = s < m ? chosen[s] : 0xFFFFFFFFu;
      }
      bptr[d] = (uint32_t)e;
      for (uint32_t s = 0; s < m; ++s) {
        uint32_t u = indices[lo + chosen[s]];
        int64_t lu = orc_lid_of(&r, u);
        if (lu < 0 || ix_off + e >= indices_cap) { orc_relabel_reset(&r); return ORC_ENOMEM; }
        blk_indices[ix_off + e] = (uint32_t)lu;
        e += 1;
      }
    }
    bptr[n_l] = (uint32_t)e;
    nnz[l] = e;
    sizes[l + 1] = r.n;
    ip_off += n_l + 1;
    ix_off += e;
    pk_off += n_l * (uint64_t)k;
  }
  orc_relabel_reset(&r);
  return ORC_OK;
}

/* ---------------------------------------------------------------------------
 * NEXT-1: k-hop WEIGHTED neighbourhood sampling (L81 fn1 "non-uniform (e.g., in
 * proportion to the edge weight)", L148 fn5, L136, L434 Fig 12 "GCN (W.)";
 * reading Q19): for a frontier vertex v whose row carries weights w_0..w_{n-1}
 * (W = their sum), slot s = 0..k-1 draws WITH replacement:
 *   x = floor(draw64(v, s>>1, batch, c3(epoch,l,WEIGHTED=8), s&1) * W / 2^64),
 *   pick = the first position p with w_0 + ... + w_p > x   (inverse CDF).
 * A row with W = 0 yields no picks.  Relabel exactly as in k-hop.
 * ------------------------------------------------------------------------- */
int orc_sample_khop_weighted(const uint64_t* indptr, const uint32_t* indices,
                             const uint32_t* weights, uint64_t V, const uint32_t* seeds,
                             uint64_t n0, const uint32_t* fanouts, uint32_t L, uint64_t seed,
                             uint32_t epoch, uint32_t batch, int32_t* lid_scratch,
                             uint32_t* uniq, uint64_t uniq_cap, uint64_t* sizes,
                             uint32_t* blk_indptr, uint64_t indptr_cap,
                             uint32_t* blk_indices, uint64_t indices_cap, uint64_t* nnz) {
  if (epoch > 0xFFFFu || L > 0xFFu) return ORC_ERANGE;
  for (uint32_t l = 0; l < L; ++l)
    if (fanouts[l] == 0 || fanouts[l] > 1024) return ORC_EINVAL;
  orc_relabel r = {lid_scratch, uniq, 0, uniq_cap};
  int rc = orc_insert_seeds(&r, seeds, n0, V);
  if (rc != ORC_OK) { orc_relabel_reset(&r); return rc; }
  sizes[0] = r.n;
  uint64_t ip_off = 0, ix_off = 0;
  for (uint32_t l = 0; l < L; ++l) {
    uint32_t k = fanouts[l];
    uint64_t n_l = r.n;
    uint32_t c3 = orc_c3(epoch, l, 8);
    if (ip_off + n_l + 1 > indptr_cap) { orc_relabel_reset(&r); return ORC_ENOMEM; }
    uint32_t* bptr = blk_indptr + ip_off;
    uint64_t e = 0;
    for (uint64_t d = 0; d < n_l; ++d) {
      uint32_t v = r.uniq[d];
      uint64_t lo = indptr[v], hi = indptr[v + 1];
      unsigned __int128 W = 0;
      for (uint64_t q = lo; q < hi; ++q) W += weights[q];
      bptr[d] = (uint32_t)e;
      if (W == 0) continue;
      for (uint32_t s = 0; s < k; ++s) {
        uint64_t rr = orc_draw64(seed, v, s >> 1, batch, c3, (int)(s & 1u));
        unsigned __int128 x = ((unsigned __int128)rr * W) >> 64;
        uint64_t p = lo;
        unsigned __int128 cum = weights[p];
        while (cum <= x) { ++p; cum += weights[p]; }
        int64_t lu = orc_lid_of(&r, indices[p]);
        if (lu < 0 || ix_off + e >= indices_cap) { orc_relabel_reset(&r); return ORC_ENOMEM; }
        blk_indices[ix_off + e] = (uint32_t)lu;
        e += 1;
      }
    }
    bptr[n_l] = (uint32_t)e;
    nnz[l] = e;
    sizes[l + 1] = r.n;
    ip_off += n_l + 1;
    ix_off += e;
  }
  orc_relabel_reset(&r);
  return ORC_OK;
}

/* ---------------------------------------------------------------------------
 * a2': PinSAGE random-walk selection (L209, L353; reading Q13).  For each
 * frontier vertex v: `walks` walks of `walk_len` steps from v; step t of
 * walk w at vertex cur picks CSR position
 *   bounded(draw64(v, (w<<8)|(t>>1), batch, c3(epoch,l,RWALK), t&1), deg(cur));
 * a walk stops at a vertex with no out-edges; every visit to a vertex other
 * than v counts once.  The `topk` vertices with the largest counts (ties:
 * smaller gid first) are v's neighbours, in that order, weight = count.
 * ------------------------------------------------------------------------- */
int orc_sample_rwalk(const uint64_t* indptr, const uint32_t* indices, uint64_t V,
                     const uint32_t* seeds, uint64_t n0, uint32_t L, uint32_t walks,
                     uint32_t walk_len, uint32_t topk, uint64_t seed, uint32_t epoch,
                     uint32_t batch, int32_t* lid_scratch, uint32_t* uniq, uint64_t uniq_cap,
                     uint64_t* sizes, uint32_t* blk_indptr, uint64_t indptr_cap,
                     uint32_t* blk_indices, uint32_t* blk_weights, uint64_t indices_cap,
                     uint64_t* nnz) {
  if (epoch > 0xFFFFu || L > 0xFFu) return ORC_ERANGE;
  if (walks == 0 || walks > 256 || walk_len == 0 || walk_len > 512 || topk == 0) return ORC_EINVAL;
  if ((uint64_t)walks * walk_len > 4096) return ORC_EINVAL;
  orc_relabel r = {lid_scratch, uniq, 0, uniq_cap};
  int rc = orc_insert_seeds(&r, seeds, n0, V);
  if (rc != ORC_OK) { orc_relabel_reset(&r); return rc; }
  sizes[0] = r.n;

  uint32_t vis[4096];       /* distinct visited vertices */
  uint32_t cnt[4096];       /* their visit counts */
  uint64_t ip_off = 0, ix_off = 0;
  for (uint32_t l = 0; l < L; ++l) {
    uint64_t n_l = r.n;
    uint32_t c3 = orc_c3(epoch, l, ORC_RWALK);
    if (ip_off + n_l + 1 > indptr_cap) { orc_relabel_reset(&r); return ORC_ENOMEM; }
    uint32_t* bptr = blk_indptr + ip_off;
    uint64_t e = 0;
    for (uint64_t d = 0; d < n_l; ++d) {
      uint32_t v = r.uniq[d];
      uint32_t nv = 0;
      for (uint32_t w = 0; w < walks; ++w) {
        uint32_t cur = v;
        for (uint32_t t = 0; t < walk_len; ++t) {
          uint64_t deg = indptr[cur + 1] - indptr[cur];
          if (deg == 0) break;
          if (deg > 0xFFFFFFFFull) { orc_relabel_reset(&r); return ORC_ERANGE; }
          uint64_t rr = orc_draw64(seed, v, (w << 8) | (t >> 1), batch, c3, (int)(t & 1u));
          cur = indices[indptr[cur] + orc_bounded(rr, (uint32_t)deg)];
          if (cur != v) {
            uint32_t q = 0;
            while (q < nv && vis[q] != cur) ++q;
            if (q == nv) { vis[nv] = cur; cnt[nv] = 0; ++nv; }
            cnt[q] += 1;
          }
        }
      }
      /* selection of the top-k by (count desc, gid asc): repeated arg-max */
      bptr[d] = (uint32_t)e;
      uint32_t take = nv < topk ? nv : topk;
      for (uint32_t s = 0; s < take; ++s) {
        uint32_t best = 0;
        for (uint32_t q = 1; q < nv; ++q)
          if (cnt[q] > cnt[best] || (cnt[q] == cnt[best] && vis[q] < vis[best])) best = q;
        int64_t lu = orc_lid_of(&r, vis[best]);
        if (lu < 0 || ix_off + e >= indices_cap) { orc_relabel_reset(&r); return ORC_ENOMEM; }
        blk_indices[ix_off + e] = (uint32_t)lu;
        blk_weights[ix_off + e] = cnt[best];
        e += 1;
        /* remove it from further selection: a removed entry has count 0 and
           every live entry has count >= 1, and take <= nv, so a removed entry
           is never chosen again. */
        cnt[best] = 0;
        vis[best] = 0xFFFFFFFFu;
      }
    }
    bptr[n_l] = (uint32_t)e;
    nnz[l] = e;
    sizes[l + 1] = r.n;
    ip_off += n_l + 1;
    ix_off += e;
  }
  orc_relabel_reset(&r);
  return ORC_OK;
}

/* ---------------------------------------------------------------------------
 * Random caching policy (L442 §7.4 "Random"): each vertex's hotness is the high
 * word of its own draw, domain POLICY = 7 -- a uniformly random order.
 * ------------------------------------------------------------------------- */
void orc_policy_random(uint64_t seed, uint64_t V, uint32_t* out) {
  uint32_t c3 = orc_c3(0, 0, 7);
  for (uint64_t v = 0; v < V; ++v) out[v] = (uint32_t)(orc_draw64(seed, (uint32_t)v, 0, 0, c3, 0) >> 32);
}

/* ---------------------------------------------------------------------------
 * a7: extract (L79, L241, L252).  A byte copy of each requested row; whether
 * a row comes from the GPU cache or from host memory does not change its
 * bytes, so the oracle reads every row from the feature matrix.
 * ------------------------------------------------------------------------- */
int orc_extract(const float* features, uint64_t V, uint32_t D, const uint32_t* vertices,
                uint64_t n, float* out) {
  for (uint64_t i = 0; i < n; ++i) {
    if (vertices[i] >= V) return ORC_EINVAL;
    memcpy(out + i * (uint64_t)D, features + (uint64_t)vertices[i] * D, sizeof(float) * D);
  }
  return ORC_OK;
}
