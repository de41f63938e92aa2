/*
 * synth.c -- seeded synthetic INPUT generator (graph topology, features,
 * training set).  Shared by the oracle and the CUDA path as *data only*: it
 * holds none of the method's arithmetic (no sampling, relabel, ranking or
 * gather).  Its random numbers are its own (Philox4x32-10 for edge draws and
 * features, a splitmix64 Feistel network for permutations); the method's
 * draws are implemented separately by oracle/ and by the CUDA library.
 *
 * Recipe (SURVEY.md §8(d) "Generator"):
 *   - Chung-Lu style power law.  Out-weights w_r = (r+1)^(-1/(g_out-1)) by
 *     rank r; rank r is vertex perm_out(r) (Feistel bijection, hubs scattered).
 *   - Out-degrees: ranks 0..m-1 are capped at `cap`, the remaining E' edges
 *     are apportioned by cumulative flooring F(r)=floor(E' P_r / P), so
 *     sum(deg) == E exactly.
 *   - Targets: Vose alias table over in-weights (q+1)^(-1/(g_in-1)), in-rank q
 *     is vertex perm(q) -- the same permutation as the out-ranks (correlated
 *     in/out degrees).  Edge (u, j) uses Philox counter
 *     (u, j, 0, c3(0,0,GEN_GRAPH)).  Rows unsorted; multi-edges and
 *     self-loops allowed (PAPER.md L67 does not exclude them).
 *   - Features f(v,d) = ((draw64(v,d,0,c3(0,0,FEATURES),0) >> 40) * 2^-23) - 1,
 *     exactly representable in f32 (float32 features: Table 3).
 *   - Training set: first |T| of a Feistel permutation (tag TRAINSET), sorted
 *     ("randomly selects a small portion of vertices").
 * Output is independent of the thread count: every value is a pure function
 * of (seed, index).
 */
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <unistd.h>

#define SY_GEN_GRAPH 4u
#define SY_TRAINSET 5u
#define SY_FEATURES 6u
/* One rank permutation for both directions: a vertex's out-degree rank equals its
 * in-weight rank, so in- and out-degree are correlated as in real graphs (for the
 * undirected ogbn-products they are equal) -- the premise of the Degree policy. */
#define SY_PERM_OUT 7u
#define SY_PERM_IN SY_PERM_OUT

static inline void sy_philox(uint32_t c[4], uint32_t k0, uint32_t k1) {
  for (int r = 0; r < 10; ++r) {
    if (r) { k0 += 0x9E3779B9u; k1 += 0xBB67AE85u; }
    uint64_t p0 = (uint64_t)0xD2511F53u * c[0];
    uint64_t p1 = (uint64_t)0xCD9E8D57u * c[2];
    uint32_t n0 = (uint32_t)(p1 >> 32) ^ c[1] ^ k0;
    uint32_t n2 = (uint32_t)(p0 >> 32) ^ c[3] ^ k1;
    c[0] = n0; c[1] = (uint32_t)p1; c[2] = n2; c[3] = (uint32_t)p0;
  }
}

static inline uint32_t sy_c3(uint32_t epoch, uint32_t hop, uint32_t dom) {
  return ((epoch & 0xFFFFu) << 16) | ((hop & 0xFFu) << 8) | (dom & 0xFFu);
}

static inline uint64_t sy_splitmix(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

/* ---- Feistel bijection on [0, n) with cycle walking ---- */
typedef struct { uint64_t n; uint32_t half; uint64_t mask; uint64_t rk[4]; } sy_perm;

static void sy_perm_init(sy_perm* p, uint64_t n, uint64_t seed, uint32_t tag) {
  uint32_t b = 2;
  while (b < 64 && (1ull << b) < n) ++b;
  if (b & 1) ++b;
  p->n = n; p->half = b / 2; p->mask = (1ull << p->half) - 1;
  for (int r = 0; r < 4; ++r) p->rk[r] = sy_splitmix(seed * 0x100000001B3ull + tag * 16u + r);
}
static inline uint64_t sy_perm_apply(const sy_perm* p, uint64_t x) {
  if (p->n <= 1) return 0;
  do {
    uint64_t L = x >> p->half, R = x & p->mask;
    for (int r = 0; r < 4; ++r) {
      uint64_t F = sy_splitmix(R ^ p->rk[r]) & p->mask;
      uint64_t nL = R, nR = L ^ F;
      L = nL; R = nR;
    }
    x = (L << p->half) | R;
  } while (x >= p->n);
  return x;
}

uint64_t synth_perm(uint64_t n, uint64_t seed, uint32_t tag, uint64_t x) {
  sy_perm p; sy_perm_init(&p, n, seed, tag); return sy_perm_apply(&p, x);
}

/* out[r] = perm(r) for r < n (the rank -> vertex map of the generator; tools only) */
void synth_perm_fill(uint64_t n, uint64_t seed, uint32_t tag, uint32_t* out) {
  sy_perm p; sy_perm_init(&p, n, seed, tag);
  for (uint64_t r = 0; r < n; ++r) out[r] = (uint32_t)sy_perm_apply(&p, r);
}

/* ---- tiny parallel-for ---- */
typedef void (*sy_body)(void* ctx, uint64_t lo, uint64_t hi);
typedef struct { sy_body f; void* ctx; uint64_t n, chunk; uint64_t* next; pthread_mutex_t* mu; } sy_job;
static void* sy_worker(void* a) {
  sy_job* j = (sy_job*)a;
  for (;;) {
    pthread_mutex_lock(j->mu);
    uint64_t lo = *j->next; *j->next += j->chunk;
    pthread_mutex_unlock(j->mu);
    if (lo >= j->n) break;
    uint64_t hi = lo + j->chunk < j->n ? lo + j->chunk : j->n;
    j->f(j->ctx, lo, hi);
  }
  return NULL;
}
static void sy_parallel(sy_body f, void* ctx, uint64_t n, uint64_t chunk, int threads) {
  if (threads <= 0) threads = (int)sysconf(_SC_NPROCESSORS_ONLN);
  if (threads < 1) threads = 1;
  if (threads > 256) threads = 256;
  uint64_t next = 0; pthread_mutex_t mu; pthread_mutex_init(&mu, NULL);
  sy_job j = {f, ctx, n, chunk ? chunk : 1, &next, &mu};
  pthread_t th[256];
  for (int t = 1; t < threads; ++t) pthread_create(&th[t], NULL, sy_worker, &j);
  sy_worker(&j);
  for (int t = 1; t < threads; ++t) pthread_join(th[t], NULL);
  pthread_mutex_destroy(&mu);
}

/* ---- degrees ---- */
int synth_degrees(uint64_t V, uint64_t E, double gamma_out, uint64_t cap, uint64_t seed,
                  uint64_t* indptr /* V+1 */) {
  if (V == 0 || gamma_out <= 1.0) return -1;
  if (cap == 0) cap = E;
  if ((long double)cap * V < (long double)E) return -2;
  double ex = -1.0 / (gamma_out - 1.0);
  double* suffix = (double*)malloc(sizeof(double) * (V + 1));
  uint64_t* deg_rank = (uint64_t*)malloc(sizeof(uint64_t) * V);
  if (!suffix || !deg_rank) { free(suffix); free(deg_rank); return -3; }
  suffix[V] = 0.0;
  for (uint64_t r = V; r-- > 0;) suffix[r] = suffix[r + 1] + pow((double)(r + 1), ex);
  uint64_t m = 0;
  while (m < V && (double)(E - m * cap) * pow((double)(m + 1), ex) / suffix[m] > (double)cap) ++m;
  for (uint64_t r = 0; r < m; ++r) deg_rank[r] = cap;
  uint64_t Erest = E - m * cap;
  double Ptot = suffix[m];
  uint64_t Fprev = 0;
  for (uint64_t r = m; r < V; ++r) {
    uint64_t F;
    if (r + 1 == V) F = Erest;
    else {
      double P = Ptot - suffix[r + 1];
      long double q = (long double)Erest * (long double)P / (long double)Ptot;
      F = (uint64_t)floorl(q);
      if (F > Erest) F = Erest;
      if (F < Fprev) F = Fprev;
    }
    deg_rank[r] = F - Fprev;
    Fprev = F;
  }
  free(suffix);
  sy_perm p; sy_perm_init(&p, V, seed, SY_PERM_OUT);
  /* indptr[u+1] temporarily holds deg(u) */
  memset(indptr, 0, sizeof(uint64_t) * (V + 1));
  for (uint64_t r = 0; r < V; ++r) indptr[sy_perm_apply(&p, r) + 1] = deg_rank[r];
  free(deg_rank);
  for (uint64_t u = 0; u < V; ++u) indptr[u + 1] += indptr[u];
  return indptr[V] == E ? 0 : -4;
}

/* ---- edges ---- */
typedef struct {
  uint64_t V; const uint64_t* indptr; uint32_t* indices;
  const double* prob; const uint32_t* alias; sy_perm pin; uint32_t k0, k1;
} sy_edge_ctx;

static void sy_edge_body(void* vc, uint64_t lo, uint64_t hi) {
  sy_edge_ctx* c = (sy_edge_ctx*)vc;
  for (uint64_t u = lo; u < hi; ++u) {
    uint64_t b = c->indptr[u], e = c->indptr[u + 1];
    for (uint64_t j = 0; j < e - b; ++j) {
      uint32_t w[4] = {(uint32_t)u, (uint32_t)j, (uint32_t)(j >> 32), sy_c3(0, 0, SY_GEN_GRAPH)};
      sy_philox(w, c->k0, c->k1);
      uint64_t r1 = ((uint64_t)w[1] << 32) | w[0];
      uint64_t r2 = ((uint64_t)w[3] << 32) | w[2];
      uint64_t col = (uint64_t)(((unsigned __int128)r1 * c->V) >> 64);
      double coin = (double)(r2 >> 11) * (1.0 / 9007199254740992.0);
      uint64_t q = coin < c->prob[col] ? col : c->alias[col];
      c->indices[b + j] = (uint32_t)sy_perm_apply(&c->pin, q);
    }
  }
}

int synth_edges(uint64_t V, const uint64_t* indptr, double gamma_in, uint64_t seed,
                uint32_t* indices, int threads) {
  if (V == 0 || V > 0xFFFFFFFFull || gamma_in <= 1.0) return -1;
  double ex = -1.0 / (gamma_in - 1.0);
  double* prob = (double*)malloc(sizeof(double) * V);
  uint32_t* alias = (uint32_t*)malloc(sizeof(uint32_t) * V);
  uint32_t* small = (uint32_t*)malloc(sizeof(uint32_t) * V);
  uint32_t* large = (uint32_t*)malloc(sizeof(uint32_t) * V);
  if (!prob || !alias || !small || !large) { free(prob); free(alias); free(small); free(large); return -3; }
  double W = 0.0;
  for (uint64_t q = V; q-- > 0;) W += pow((double)(q + 1), ex);
  uint64_t ns = 0, nl = 0;
  for (uint64_t q = 0; q < V; ++q) {
    prob[q] = pow((double)(q + 1), ex) * (double)V / W;
    alias[q] = (uint32_t)q;
    if (prob[q] < 1.0) small[ns++] = (uint32_t)q; else large[nl++] = (uint32_t)q;
  }
  while (ns && nl) {
    uint32_t s = small[--ns], l = large[nl - 1];
    alias[s] = l;
    prob[l] = (prob[l] + prob[s]) - 1.0;
    if (prob[l] < 1.0) { --nl; small[ns++] = l; }
  }
  while (nl) prob[large[--nl]] = 1.0;
  while (ns) prob[small[--ns]] = 1.0;
  free(small); free(large);
  sy_edge_ctx c; c.V = V; c.indptr = indptr; c.indices = indices; c.prob = prob; c.alias = alias;
  sy_perm_init(&c.pin, V, seed, SY_PERM_IN);
  c.k0 = (uint32_t)seed; c.k1 = (uint32_t)(seed >> 32);
  sy_parallel(sy_edge_body, &c, V, 4096, threads);
  free(prob); free(alias);
  return 0;
}

/* ---- features ---- */
typedef struct { uint32_t D; float* out; uint32_t k0, k1; } sy_feat_ctx;
static void sy_feat_body(void* vc, uint64_t lo, uint64_t hi) {
  sy_feat_ctx* c = (sy_feat_ctx*)vc;
  for (uint64_t v = lo; v < hi; ++v)
    for (uint32_t d = 0; d < c->D; ++d) {
      uint32_t w[4] = {(uint32_t)v, d, 0u, sy_c3(0, 0, SY_FEATURES)};
      sy_philox(w, c->k0, c->k1);
      uint64_t r = ((uint64_t)w[1] << 32) | w[0];
      c->out[v * c->D + d] = (float)(r >> 40) * (1.0f / 8388608.0f) - 1.0f;
    }
}
int synth_features(uint64_t V, uint32_t D, uint64_t seed, float* out, int threads) {
  sy_feat_ctx c = {D, out, (uint32_t)seed, (uint32_t)(seed >> 32)};
  sy_parallel(sy_feat_body, &c, V, 2048, threads);
  return 0;
}

/* ---- training set ---- */
static int sy_cmp_u32(const void* a, const void* b) {
  uint32_t x = *(const uint32_t*)a, y = *(const uint32_t*)b;
  return (x > y) - (x < y);
}
int synth_trainset(uint64_t V, uint64_t n, uint64_t seed, uint32_t* out) {
  if (n > V) return -1;
  sy_perm p; sy_perm_init(&p, V, seed, SY_TRAINSET);
  for (uint64_t i = 0; i < n; ++i) out[i] = (uint32_t)sy_perm_apply(&p, i);
  qsort(out, n, sizeof(uint32_t), sy_cmp_u32);
  return 0;
}

/* ---- edge weights (weighted sampling input: "The weight of a vertex
 * represents the year registered, and the sampling algorithm prefers to select the
 * newer neighbors"): w(u->t) = year(t), year(t) in 1..levels drawn per vertex. ---- */
typedef struct { const uint32_t* indices; uint32_t* w; uint32_t levels; uint32_t k0, k1; } sy_w_ctx;
static void sy_w_body(void* vc, uint64_t lo, uint64_t hi) {
  sy_w_ctx* c = (sy_w_ctx*)vc;
  for (uint64_t e = lo; e < hi; ++e) {
    uint32_t w[4] = {c->indices[e], 0u, 0u, sy_c3(0, 0, 9u)};
    sy_philox(w, c->k0, c->k1);
    c->w[e] = 1u + (uint32_t)(((uint64_t)w[0] * c->levels) >> 32);
  }
}
int synth_edge_weights(uint64_t E, const uint32_t* indices, uint32_t levels, uint64_t seed,
                       uint32_t* out, int threads) {
  sy_w_ctx c = {indices, out, levels ? levels : 1u, (uint32_t)seed, (uint32_t)(seed >> 32)};
  sy_parallel(sy_w_body, &c, E, 1 << 16, threads);
  return 0;
}
