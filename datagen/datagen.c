/*
 * datagen.c -- seeded synthetic INPUTS shared by the oracle-side tests and the
 * CUDA path's tests / bench.  It holds none of the sampling method's
 * arithmetic (no Philox, no Floyd, no relabel): only the graph, the
 * renumbering, the feature table and the train-id set that both sides read.
 *
 * Recipe (shapes from PAPER.md Table 3):
 *   * R-MAT (Chakrabarti et al. 2004) with quadrant probabilities (a,b,c,d)
 *     over S = ceil(log2 N) levels.  Undirected edge e in [0, M) takes its
 *     endpoints from a counter-based hash of (graph_seed, e, attempt, level);
 *     it is redrawn (attempt + 1) while an endpoint is >= N or u == v.
 *     Both directions are stored (symmetric graph: in-neighbours ==
 *     out-neighbours), rows sorted ascending, duplicates removed.
 *   * Renumbering ("consecutive global ids"): every id goes through a
 *     Feistel bijection pi on [0, N) (cycle walking), keyed by graph_seed and
 *     independent of the GPU count.  Rank r then owns [bounds[r], bounds[r+1])
 *     with bounds[r] = floor(r N / P).
 *   * Features: feat(g, c) = bits(0x3F800000 | (splitmix64(feat_seed ^
 *     (g * dim + c)) >> 41)), an fp32 value in [1, 2) (Table 3: fp32 rows).
 *   * Train ids: sigma(0 .. count-1) for a second Feistel bijection sigma.
 *
 * OpenMP-parallel but deterministic: every random value is a pure function of
 * its counter, and every row is sorted before use.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <omp.h>

static inline uint64_t splitmix64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

static inline uint64_t hash4(uint64_t seed, uint64_t a, uint64_t b, uint64_t c) {
  uint64_t h = splitmix64(seed ^ 0x6A09E667F3BCC909ull);
  h = splitmix64(h ^ a);
  h = splitmix64(h ^ (b * 0x100000001B3ull));
  return splitmix64(h ^ (c + 0x3C6EF372FE94F82Bull));
}

/* ------------------------------------------------------------ Feistel */

typedef struct {
  int half;        /* bits per half */
  uint64_t mask;   /* (1 << half) - 1 */
  uint64_t n;      /* domain [0, n) */
  uint64_t key;
} feistel_t;

static feistel_t feistel_make(uint64_t n, uint64_t key) {
  feistel_t f;
  int bits = 1;
  while (bits < 62 && ((uint64_t)1 << bits) < n) ++bits;
  f.half = (bits + 1) / 2;
  f.mask = ((uint64_t)1 << f.half) - 1;
  f.n = n;
  f.key = key;
  return f;
}

static inline uint64_t feistel_once(const feistel_t *f, uint64_t x) {
  uint64_t L = x >> f->half, R = x & f->mask;
  for (int round = 0; round < 4; ++round) {
    uint64_t nl = R;
    uint64_t nr = L ^ (hash4(f->key, (uint64_t)round, R, 0x5151) & f->mask);
    L = nl;
    R = nr;
  }
  return (L << f->half) | R;
}

/* bijection on [0, n) by cycle walking the bijection on [0, 2^(2 half)) */
static inline uint64_t feistel_apply(const feistel_t *f, uint64_t x) {
  do {
    x = feistel_once(f, x);
  } while (x >= f->n);
  return x;
}

int64_t datagen_permute(int64_t n, uint64_t key, int64_t x) {
  feistel_t f = feistel_make((uint64_t)n, key);
  return (int64_t)feistel_apply(&f, (uint64_t)x);
}

void datagen_permute_many(int64_t n, uint64_t key, const int64_t *x, int64_t cnt, int64_t *out) {
  feistel_t f = feistel_make((uint64_t)n, key);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < cnt; ++i) out[i] = (int64_t)feistel_apply(&f, (uint64_t)x[i]);
}

/* -------------------------------------------------------------- R-MAT */

typedef struct {
  int64_t n;
  int scale;
  uint32_t ta, tab, tabc; /* cumulative thresholds in 2^32 units */
  uint64_t seed;
} rmat_t;

static inline void rmat_edge(const rmat_t *g, int64_t e, int64_t *uo, int64_t *vo) {
  for (uint64_t attempt = 0;; ++attempt) {
    uint64_t u = 0, v = 0;
    uint64_t h = 0;
    for (int level = 0; level < g->scale; ++level) {
      if ((level & 1) == 0) h = hash4(g->seed, (uint64_t)e, attempt, (uint64_t)level);
      uint32_t r = (level & 1) ? (uint32_t)(h >> 32) : (uint32_t)h;
      uint64_t bu, bv;
      if (r < g->ta) { bu = 0; bv = 0; }
      else if (r < g->tab) { bu = 0; bv = 1; }
      else if (r < g->tabc) { bu = 1; bv = 0; }
      else { bu = 1; bv = 1; }
      u = (u << 1) | bu;
      v = (v << 1) | bv;
    }
    if ((int64_t)u < g->n && (int64_t)v < g->n && u != v) {
      *uo = (int64_t)u;
      *vo = (int64_t)v;
      return;
    }
  }
}

static int cmp_i32(const void *a, const void *b) {
  int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
  return (x > y) - (x < y);
}

/* Builds the renumbered symmetric CSR.  indptr: int64[N+1] (caller-owned).
 * *indices_out: malloc'ed int32[nnz] (free with datagen_free).  Returns nnz
 * or -1 on allocation failure. */
int64_t datagen_rmat_csr(int64_t N, int64_t M, double a, double b, double c, uint64_t graph_seed,
                         int threads, int64_t *indptr, int32_t **indices_out) {
  if (threads > 0) omp_set_num_threads(threads);
  rmat_t g;
  g.n = N;
  g.scale = 1;
  while (((int64_t)1 << g.scale) < N) ++g.scale;
  g.ta = (uint32_t)(a * 4294967296.0);
  g.tab = (uint32_t)((a + b) * 4294967296.0);
  g.tabc = (uint32_t)((a + b + c) * 4294967296.0);
  g.seed = graph_seed;
  feistel_t pi = feistel_make((uint64_t)N, graph_seed * 0x9E3779B97F4A7C15ull + 1);

  int64_t *deg = (int64_t *)calloc((size_t)N + 1, sizeof(int64_t));
  if (!deg) return -1;
  /* pass 1: degrees (both directions) */
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < M; ++e) {
    int64_t u, v;
    rmat_edge(&g, e, &u, &v);
    u = (int64_t)feistel_apply(&pi, (uint64_t)u);
    v = (int64_t)feistel_apply(&pi, (uint64_t)v);
#pragma omp atomic
    deg[u]++;
#pragma omp atomic
    deg[v]++;
  }
  int64_t *cur = (int64_t *)malloc(sizeof(int64_t) * ((size_t)N + 1));
  if (!cur) { free(deg); return -1; }
  cur[0] = 0;
  for (int64_t x = 0; x < N; ++x) cur[x + 1] = cur[x] + deg[x];
  int64_t total = cur[N];
  int32_t *tmp = (int32_t *)malloc(sizeof(int32_t) * (size_t)(total > 0 ? total : 1));
  if (!tmp) { free(deg); free(cur); return -1; }
  memcpy(deg, cur, sizeof(int64_t) * ((size_t)N + 1)); /* deg := row starts */
  /* pass 2: fill (order within a row is fixed by the sort below) */
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < M; ++e) {
    int64_t u, v, pu, pv;
    rmat_edge(&g, e, &u, &v);
    u = (int64_t)feistel_apply(&pi, (uint64_t)u);
    v = (int64_t)feistel_apply(&pi, (uint64_t)v);
#pragma omp atomic capture
    pu = cur[u]++;
#pragma omp atomic capture
    pv = cur[v]++;
    tmp[pu] = (int32_t)v;
    tmp[pv] = (int32_t)u;
  }
  /* sort + dedup each row; new degree in cur[x] */
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t x = 0; x < N; ++x) {
    int32_t *row = tmp + deg[x];
    int64_t d = deg[x + 1] - deg[x];
    qsort(row, (size_t)d, sizeof(int32_t), cmp_i32);
    int64_t w = 0;
    for (int64_t i = 0; i < d; ++i)
      if (w == 0 || row[i] != row[w - 1]) row[w++] = row[i];
    cur[x] = w;
  }
  indptr[0] = 0;
  for (int64_t x = 0; x < N; ++x) indptr[x + 1] = indptr[x] + cur[x];
  int64_t nnz = indptr[N];
  int32_t *out = (int32_t *)malloc(sizeof(int32_t) * (size_t)(nnz > 0 ? nnz : 1));
  if (!out) { free(deg); free(cur); free(tmp); return -1; }
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t x = 0; x < N; ++x)
    memcpy(out + indptr[x], tmp + deg[x], sizeof(int32_t) * (size_t)(indptr[x + 1] - indptr[x]));
  free(tmp);
  free(deg);
  free(cur);
  *indices_out = out;
  return nnz;
}

void datagen_free(void *p) { free(p); }

/* ----------------------------------------------------------- features */

static inline float feat_value(uint64_t g, uint64_t col, uint64_t dim, uint64_t feat_seed) {
  uint32_t bits = 0x3F800000u | (uint32_t)(splitmix64(feat_seed ^ (g * dim + col)) >> 41);
  float f;
  memcpy(&f, &bits, sizeof(f));
  return f;
}

/* out[(g - lo) * dim + col] = feat(g, col) for g in [lo, hi) */
void datagen_features(int64_t lo, int64_t hi, int32_t dim, uint64_t feat_seed, int threads,
                      float *out) {
  if (threads > 0) omp_set_num_threads(threads);
#pragma omp parallel for schedule(static)
  for (int64_t g = lo; g < hi; ++g)
    for (int32_t col = 0; col < dim; ++col)
      out[(g - lo) * dim + col] = feat_value((uint64_t)g, (uint64_t)col, (uint64_t)dim, feat_seed);
}

/* features of arbitrary ids (for checking samples of huge tables) */
void datagen_features_of(const int32_t *ids, int64_t n, int32_t dim, uint64_t feat_seed, float *out) {
#pragma omp parallel for schedule(static)
  for (int64_t r = 0; r < n; ++r)
    for (int32_t col = 0; col < dim; ++col)
      out[r * dim + col] = feat_value((uint64_t)ids[r], (uint64_t)col, (uint64_t)dim, feat_seed);
}
