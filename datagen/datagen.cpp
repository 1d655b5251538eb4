// datagen.cpp -- seeded synthetic INPUTS shared by the oracle-side tests and
// the CUDA path's tests / bench.  It holds none of the sampling method's
// arithmetic (no Philox, no Floyd, no relabel): only the graph, the
// renumbering, the feature table and the train-id set that both sides read.
//
// Recipe (shapes from PAPER.md Table 3):
//   * R-MAT (Chakrabarti et al. 2004) with quadrant probabilities (a,b,c,d)
//     over S = ceil(log2 N) levels.  Undirected edge e in [0, M) takes its
//     endpoints from counter-based random words of (graph_seed, e, attempt)
//     (16-bit quadrant draws, four levels per 64-bit word); it is redrawn
//     (attempt + 1) while an endpoint is >= N or u == v.  Both directions are
//     stored (symmetric graph: in-neighbours == out-neighbours), rows
//     sorted ascending, duplicates removed.
//   * Renumbering ("consecutive global ids"): every id goes through a
//     Feistel bijection pi on [0, N) (cycle walking), keyed by graph_seed and
//     independent of the GPU count.  Rank r then owns [bounds[r], bounds[r+1])
//     with bounds[r] = floor(r N / P).
//   * Features: feat(g, c) = bits(0x3F800000 | (splitmix64(feat_seed ^
//     (g * dim + c)) >> 41)), an fp32 value in [1, 2) (Table 3: fp32 rows).
//   * Train ids: sigma(0 .. count-1) for a second Feistel bijection sigma.
//
// OpenMP-parallel but deterministic: every random value is a pure function of
// its counter, and every row is sorted before use.
#include <omp.h>

#include <algorithm>
#include <atomic>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <vector>
#include <chrono>
#include <cstdio>

namespace {

inline uint64_t splitmix64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

// ------------------------------------------------------------------ Feistel
struct Feistel {
  int half;
  uint64_t mask, n, key[4];
};

Feistel feistel_make(uint64_t n, uint64_t key) {
  Feistel f;
  int bits = 1;
  while (bits < 62 && ((uint64_t)1 << bits) < n) ++bits;
  f.half = (bits + 1) / 2;
  f.mask = ((uint64_t)1 << f.half) - 1;
  f.n = n;
  for (int r = 0; r < 4; ++r) f.key[r] = splitmix64(key + 0x1234567ull * (r + 1));
  return f;
}

inline uint64_t feistel_once(const Feistel &f, uint64_t x) {
  uint64_t L = x >> f.half, R = x & f.mask;
  for (int r = 0; r < 4; ++r) {
    uint64_t h = (R ^ f.key[r]) * 0x9E3779B97F4A7C15ull;
    h ^= h >> 29;
    h *= 0xBF58476D1CE4E5B9ull;
    const uint64_t nr = L ^ ((h >> 17) & f.mask);
    L = R;
    R = nr;
  }
  return (L << f.half) | R;
}

// bijection on [0, n) by cycle walking the bijection on [0, 2^(2 half))
inline uint64_t feistel_apply(const Feistel &f, uint64_t x) {
  do {
    x = feistel_once(f, x);
  } while (x >= f.n);
  return x;
}

// -------------------------------------------------------------------- R-MAT
struct Rmat {
  int64_t n;
  int scale;
  uint32_t ta, tab, tabc;  // cumulative thresholds in 2^16 units
  uint64_t seed;
};

inline void rmat_edge(const Rmat &g, int64_t e, int64_t *uo, int64_t *vo) {
  const uint64_t base = splitmix64(g.seed ^ ((uint64_t)e * 0xD1B54A32D192ED03ull));
  for (uint64_t attempt = 0;; ++attempt) {
    uint64_t u = 0, v = 0, w = 0;
    for (int level = 0; level < g.scale; ++level) {
      if ((level & 3) == 0) w = splitmix64(base + attempt * 0x632BE59BD9B4E019ull + (uint64_t)level);
      const uint32_t r = (uint32_t)(w >> (16 * (level & 3))) & 0xffffu;
      const uint64_t bu = r >= g.tab, bv = (r >= g.ta && r < g.tab) || r >= g.tabc;
      u = (u << 1) | bu;
      v = (v << 1) | bv;
    }
    if ((int64_t)u < g.n && (int64_t)v < g.n && u != v) {
      *uo = (int64_t)u;
      *vo = (int64_t)v;
      return;
    }
  }
}

inline float feat_value(uint64_t g, uint64_t col, uint64_t dim, uint64_t feat_seed) {
  const uint32_t bits = 0x3F800000u | (uint32_t)(splitmix64(feat_seed ^ (g * dim + col)) >> 41);
  float f;
  memcpy(&f, &bits, sizeof(f));
  return f;
}

}  // namespace

extern "C" {

int64_t datagen_permute(int64_t n, uint64_t key, int64_t x) {
  const Feistel f = feistel_make((uint64_t)n, key);
  return (int64_t)feistel_apply(f, (uint64_t)x);
}

void datagen_permute_many(int64_t n, uint64_t key, const int64_t *x, int64_t cnt, int64_t *out) {
  const Feistel f = feistel_make((uint64_t)n, key);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < cnt; ++i) out[i] = (int64_t)feistel_apply(f, (uint64_t)x[i]);
}

// Builds the renumbered symmetric CSR.  indptr: int64[N+1] (caller-owned).
// *indices_out: malloc'ed int32[nnz] (free with datagen_free).  Returns nnz
// or -1 on allocation failure.
int64_t datagen_rmat_csr(int64_t N, int64_t M, double a, double b, double c, uint64_t graph_seed, int threads,
                         int64_t *indptr, int32_t **indices_out) {
  if (threads > 0) omp_set_num_threads(threads);
  Rmat g;
  g.n = N;
  g.scale = 1;
  while (((int64_t)1 << g.scale) < N) ++g.scale;
  g.ta = (uint32_t)(a * 65536.0);
  g.tab = (uint32_t)((a + b) * 65536.0);
  g.tabc = (uint32_t)((a + b + c) * 65536.0);
  g.seed = graph_seed;
  const Feistel pi = feistel_make((uint64_t)N, graph_seed * 0x9E3779B97F4A7C15ull + 1);

  const bool verbose = getenv("DATAGEN_VERBOSE") != nullptr;
  auto t0 = std::chrono::steady_clock::now();
  auto lap = [&](const char *what) {
    if (!verbose) return;
    auto t1 = std::chrono::steady_clock::now();
    fprintf(stderr, "datagen %-10s %.2f s\n", what, std::chrono::duration<double>(t1 - t0).count());
    t0 = t1;
  };
  // pass 1: renumbered undirected edges
  uint64_t *edges = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(M > 0 ? M : 1));
  int64_t *cur = (int64_t *)calloc((size_t)N + 1, sizeof(int64_t));
  if (!edges || !cur) {
    free(edges);
    free(cur);
    return -1;
  }
  std::atomic<int64_t> *deg = reinterpret_cast<std::atomic<int64_t> *>(cur);
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < M; ++e) {
    int64_t u, v;
    rmat_edge(g, e, &u, &v);
    u = (int64_t)feistel_apply(pi, (uint64_t)u);
    v = (int64_t)feistel_apply(pi, (uint64_t)v);
    edges[e] = ((uint64_t)u << 32) | (uint64_t)v;
    deg[u].fetch_add(1, std::memory_order_relaxed);
    deg[v].fetch_add(1, std::memory_order_relaxed);
  }
  lap("edges");
  // row starts (exclusive scan) into indptr
  indptr[0] = 0;
  for (int64_t x = 0; x < N; ++x) indptr[x + 1] = indptr[x] + cur[x];
  const int64_t total = indptr[N];
  int32_t *col = (int32_t *)malloc(sizeof(int32_t) * (size_t)(total > 0 ? total : 1));
  if (!col) {
    free(edges);
    free(cur);
    return -1;
  }
  for (int64_t x = 0; x < N; ++x) cur[x] = indptr[x];
  std::atomic<int64_t> *pos = reinterpret_cast<std::atomic<int64_t> *>(cur);
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < M; ++e) {
    const int64_t u = (int64_t)(edges[e] >> 32), v = (int64_t)(uint32_t)edges[e];
    col[pos[u].fetch_add(1, std::memory_order_relaxed)] = (int32_t)v;
    col[pos[v].fetch_add(1, std::memory_order_relaxed)] = (int32_t)u;
  }
  free(edges);
  lap("fill");
  // sort + dedup each row in place; new degree in cur[x]
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t x = 0; x < N; ++x) {
    int32_t *row = col + indptr[x];
    const int64_t d = indptr[x + 1] - indptr[x];
    std::sort(row, row + d);
    cur[x] = std::unique(row, row + d) - row;
  }
  lap("sort");
  // compact in place (rows only move left)
  int64_t w = 0;
  for (int64_t x = 0; x < N; ++x) {
    const int64_t s = indptr[x], d = cur[x];
    if (w != s) memmove(col + w, col + s, sizeof(int32_t) * (size_t)d);
    indptr[x] = w;
    w += d;
  }
  indptr[N] = w;
  free(cur);
  lap("compact");
  int32_t *shrunk = (int32_t *)realloc(col, sizeof(int32_t) * (size_t)(w > 0 ? w : 1));
  *indices_out = shrunk ? shrunk : col;
  return w;
}

void datagen_free(void *p) { free(p); }

// out[(g - lo) * dim + col] = feat(g, col) for g in [lo, hi)
void datagen_features(int64_t lo, int64_t hi, int32_t dim, uint64_t feat_seed, int threads, float *out) {
  if (threads > 0) omp_set_num_threads(threads);
#pragma omp parallel for schedule(static)
  for (int64_t g = lo; g < hi; ++g)
    for (int32_t col = 0; col < dim; ++col)
      out[(g - lo) * dim + col] = feat_value((uint64_t)g, (uint64_t)col, (uint64_t)dim, feat_seed);
}

// Node weights for biased sampling: about 1/32 of the nodes get
// weight 0, the others a multiple of 1/16 in (0, 256] (exact in fp32 and in
// the 16.16 fixed point the method uses).
void datagen_node_weights(int64_t n, uint64_t seed, float *out) {
#pragma omp parallel for schedule(static)
  for (int64_t u = 0; u < n; ++u) {
    const uint64_t h = splitmix64(seed ^ ((uint64_t)u * 0x9E3779B97F4A7C15ull));
    out[u] = (h & 31u) == 0 ? 0.0f : (float)((h >> 40) % 4096u + 1u) / 16.0f;
  }
}

// edge weight = weight of the edge's neighbour: out[e] = w[indices[e]]
void datagen_edge_weights(const int32_t *indices, int64_t nnz, const float *w, float *out) {
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < nnz; ++e) out[e] = w[indices[e]];
}

// features of arbitrary ids (for checking samples of huge tables)
void datagen_features_of(const int32_t *ids, int64_t n, int32_t dim, uint64_t feat_seed, float *out) {
#pragma omp parallel for schedule(static)
  for (int64_t r = 0; r < n; ++r)
    for (int32_t col = 0; col < dim; ++col)
      out[r * dim + col] = feat_value((uint64_t)ids[r], (uint64_t)col, (uint64_t)dim, feat_seed);
}

}  // extern "C"
