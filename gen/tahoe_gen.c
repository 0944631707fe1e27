/*
 * gen/tahoe_gen.c — seeded synthetic forests and sample matrices (SURVEY §8(d) "The synthetic
 * inputs").  This module is INPUT GENERATION ONLY: it is shared by the CPU oracle (oracle/) and
 * the CUDA path (paper_conf_eurosys_xiedlll21_b200/), and holds none of the method's arithmetic
 * (no prediction, no combination, no layout).  Growing a random tree on calibration rows uses the
 * same "x < b" split test a tree is defined by, because that is how a tree partitions its
 * training rows; the generated node arrays are then consumed as plain data by both sides.
 *
 * Every random number is counter-based: element (row i, column j) of a sample matrix is a pure
 * function of (seed, i, j), and tree t is grown from its own xoshiro256** stream seeded by
 * (seed, t).  Outputs therefore do not depend on the thread count or on which rows are asked for.
 *
 * Forest recipe ("random, post-pruned, unbalanced"):
 *   split iff depth < D_max, |rows| >= 2*min_leaf and (root or U < p_split);
 *   feature ~ U[0,d); threshold = that feature's value in a uniformly random row of the node
 *   (quantile mode: the q-quantile of the node's values, q ~ Beta(0.35,0.35));
 *   retry <= 8 times when a side would get < min_leaf rows, else make a leaf;
 *   one bottom-up post-prune sweep collapses an internal node whose two children are leaves
 *   with probability prune_p;  leaf values k/leaf_k (k ~ U{-leaf_k..leaf_k}, "dyadic") or N(0,0.1).
 *   Nodes of each tree are emitted in breadth-first order; trees are concatenated.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define GEN_API __attribute__((visibility("default")))

/* ---------------- counter-based RNG ---------------- */
static inline uint64_t sm64(uint64_t x) {
  x += 0x9e3779b97f4a7c15ULL;
  x = (x ^ (x >> 30)) * 0xbf58476d1ce4e5b9ULL;
  x = (x ^ (x >> 27)) * 0x94d049bb133111ebULL;
  return x ^ (x >> 31);
}
static inline uint64_t key3(uint64_t seed, uint64_t a, uint64_t b) {
  return sm64(sm64(sm64(seed) ^ a) ^ (b * 0xd1b54a32d192ed03ULL));
}
static inline double u01_53(uint64_t u) { return (double)(u >> 11) * (1.0 / 9007199254740992.0); }
/* uniform in [0,1) with a 24-bit mantissa fill */
static inline float u01_24(uint64_t u) { return (float)(u >> 40) * (1.0f / 16777216.0f); }
static inline double normal_of(uint64_t k) {
  double u1 = ((double)((sm64(k ^ 0x1111) >> 11) + 1)) * (1.0 / 9007199254740992.0); /* (0,1] */
  double u2 = u01_53(sm64(k ^ 0x2222));
  return sqrt(-2.0 * log(u1)) * cos(6.283185307179586 * u2);
}

typedef struct { uint64_t s[4]; } xo256;
static inline uint64_t rotl(uint64_t x, int k) { return (x << k) | (x >> (64 - k)); }
static inline uint64_t xo_next(xo256* r) {
  uint64_t* s = r->s;
  uint64_t res = rotl(s[1] * 5, 7) * 9, t = s[1] << 17;
  s[2] ^= s[0]; s[3] ^= s[1]; s[1] ^= s[2]; s[0] ^= s[3]; s[2] ^= t; s[3] = rotl(s[3], 45);
  return res;
}
static void xo_seed(xo256* r, uint64_t k) {
  for (int i = 0; i < 4; i++) { k = sm64(k + (uint64_t)i * 0x632be59bd9b4e019ULL); r->s[i] = k | 1; }
}
static inline double xo_u01(xo256* r) { return u01_53(xo_next(r)); }
static inline uint64_t xo_below(xo256* r, uint64_t n) { return xo_next(r) % n; }
static double xo_normal(xo256* r) {
  double u1 = ((double)((xo_next(r) >> 11) + 1)) * (1.0 / 9007199254740992.0);
  double u2 = xo_u01(r);
  return sqrt(-2.0 * log(u1)) * cos(6.283185307179586 * u2);
}
/* Gamma(a,1) by Marsaglia-Tsang (a < 1 boosted by U^(1/a)) */
static double xo_gamma(xo256* r, double a) {
  if (a < 1.0) {
    double u = xo_u01(r);
    if (u <= 0) u = 1e-300;
    return xo_gamma(r, a + 1.0) * pow(u, 1.0 / a);
  }
  double d = a - 1.0 / 3.0, c = 1.0 / sqrt(9.0 * d);
  for (;;) {
    double x, v;
    do { x = xo_normal(r); v = 1.0 + c * x; } while (v <= 0);
    v = v * v * v;
    double u = xo_u01(r);
    if (u < 1.0 - 0.0331 * x * x * x * x) return d * v;
    if (log(u) < 0.5 * x * x + d * (1.0 - v + log(v))) return d * v;
  }
}
static double xo_beta(xo256* r, double a, double b) {
  double x = xo_gamma(r, a), y = xo_gamma(r, b);
  return x / (x + y);
}

/* ---------------- column distributions (per config "shape") ---------------- */
/* shape: 1 = N(0,1); 2 = Higgs-like (28); 3 = covtype-like (54); 4 = epsilon-like N(0,1)/sqrt(d);
 *        5 = 90 x N(0,1) + 10 five-level discrete.  Any d is accepted; columns past the shape's
 *        natural width repeat its pattern. */
static const double kPi = 3.14159265358979323846;
static const int kCovLo[10] = {1859, 0, 0, 0, -173, 0, 0, 0, 0, 0};
static const int kCovHi[10] = {3858, 360, 66, 1397, 601, 7117, 254, 254, 254, 7173};

static float gen_value(int shape, uint64_t seed, int64_t i, int32_t j, int32_t d) {
  uint64_t k = key3(seed, (uint64_t)i, (uint64_t)j);
  switch (shape) {
    case 2: {
      int jj = j % 28;
      if (jj < 15) {
        int kind = jj % 3;
        if (kind == 0) return (float)exp(0.5 * normal_of(k));
        if (kind == 1) return (float)normal_of(k);
        return (float)(-kPi + 2.0 * kPi * u01_53(sm64(k)));
      }
      if (jj == 15) return (float)exp(0.5 * normal_of(k));
      if (jj == 16) return (float)(-kPi + 2.0 * kPi * u01_53(sm64(k)));
      if (jj < 21) {
        static const float lv[3] = {0.0f, 1.0866f, 2.1731f};
        return lv[sm64(k) % 3];
      }
      return (float)exp(0.3 * normal_of(k));
    }
    case 3: {
      int jj = j % 54;
      if (jj < 10) {
        int lo = kCovLo[jj], hi = kCovHi[jj];
        return (float)(lo + (int)(sm64(k) % (uint64_t)(hi - lo + 1)));
      }
      /* one-hot groups: the hot category is a function of (row, group) only */
      if (jj < 14) {
        uint64_t g = key3(seed ^ 0xabcdefULL, (uint64_t)i, (uint64_t)(j / 54) * 2 + 0);
        return (jj - 10) == (int)(sm64(g) % 4) ? 1.0f : 0.0f;
      } else {
        uint64_t g = key3(seed ^ 0xabcdefULL, (uint64_t)i, (uint64_t)(j / 54) * 2 + 1);
        return (jj - 14) == (int)(sm64(g) % 40) ? 1.0f : 0.0f;
      }
    }
    case 4:
      return (float)(normal_of(k) / sqrt((double)d));
    case 5: {
      int jj = j % 100;
      if (jj < 90) return (float)normal_of(k);
      return (float)(sm64(k) % 5);
    }
    default:
      return (float)normal_of(k);
  }
}

/* X[r*d + j] for rows row0 .. row0+nrows-1 */
GEN_API void gen_rows(int32_t shape, uint64_t seed, int64_t row0, int64_t nrows, int32_t d,
                      float* out, int32_t nthreads) {
#ifdef _OPENMP
  if (nthreads <= 0) nthreads = omp_get_max_threads();
#pragma omp parallel for schedule(static) num_threads(nthreads)
#endif
  for (int64_t r = 0; r < nrows; r++)
    for (int32_t j = 0; j < d; j++) out[r * (int64_t)d + j] = gen_value(shape, seed, row0 + r, j, d);
}

/* rows by explicit index (seeded subsamples of a large workload) */
GEN_API void gen_rows_idx(int32_t shape, uint64_t seed, const int64_t* idx, int64_t nrows,
                          int32_t d, float* out, int32_t nthreads) {
#ifdef _OPENMP
  if (nthreads <= 0) nthreads = omp_get_max_threads();
#pragma omp parallel for schedule(static) num_threads(nthreads)
#endif
  for (int64_t r = 0; r < nrows; r++)
    for (int32_t j = 0; j < d; j++) out[r * (int64_t)d + j] = gen_value(shape, seed, idx[r], j, d);
}

/* ---------------- forest growth ---------------- */
typedef struct {
  int32_t n_trees, max_depth, n_features, n_classes, shape;
  int32_t min_leaf, quantile_thresholds, leaf_mode, leaf_k, _pad;
  double p_split, prune_p;
  int64_t n_cal;
  uint64_t seed_forest, seed_cal;
} gen_forest_params;

typedef struct {
  int32_t n;           /* nodes */
  int32_t* feature;    /* -1 leaf */
  float* threshold;
  int32_t* left;
  int32_t* right;
  float* value;
  uint8_t* dleft;
} gtree;

typedef struct {
  int32_t cap, n;
  int32_t *feature, *left, *right, *depth;
  float* threshold;
} tmp_tree;

static int32_t tt_new(tmp_tree* t, int depth) {
  if (t->n == t->cap) {
    t->cap = t->cap ? t->cap * 2 : 64;
    t->feature = realloc(t->feature, sizeof(int32_t) * t->cap);
    t->left = realloc(t->left, sizeof(int32_t) * t->cap);
    t->right = realloc(t->right, sizeof(int32_t) * t->cap);
    t->depth = realloc(t->depth, sizeof(int32_t) * t->cap);
    t->threshold = realloc(t->threshold, sizeof(float) * t->cap);
  }
  int32_t id = t->n++;
  t->feature[id] = -1; t->left[id] = t->right[id] = -1; t->depth[id] = depth; t->threshold[id] = 0;
  return id;
}

static int cmp_float(const void* a, const void* b) {
  float x = *(const float*)a, y = *(const float*)b;
  return (x > y) - (x < y);
}

/* quickselect k-th smallest of v[0..m) (destroys order) */
static float kth_smallest(float* v, int64_t m, int64_t k) {
  int64_t lo = 0, hi = m - 1;
  while (hi - lo > 16) {
    float p = v[lo + (hi - lo) / 2];
    int64_t i = lo, j = hi;
    while (i <= j) {
      while (v[i] < p) i++;
      while (v[j] > p) j--;
      if (i <= j) { float t = v[i]; v[i] = v[j]; v[j] = t; i++; j--; }
    }
    if (k <= j) hi = j; else if (k >= i) lo = i; else return v[k];
  }
  qsort(v + lo, (size_t)(hi - lo + 1), sizeof(float), cmp_float);
  return v[k];
}

typedef struct {
  const gen_forest_params* p;
  const float* X;  /* n_cal x d */
  int32_t* idx;    /* row index workspace */
  int32_t* tmp;
  float* vals;
  xo256 rng;
  tmp_tree tree;
} grow_ctx;

static void grow(grow_ctx* c, int32_t node, int64_t lo, int64_t hi, int depth) {
  const gen_forest_params* p = c->p;
  int64_t m = hi - lo;
  int d = p->n_features;
  int split = depth < p->max_depth && m >= 2 * (int64_t)p->min_leaf &&
              (depth == 0 || xo_u01(&c->rng) < p->p_split);
  if (!split) return;
  for (int attempt = 0; attempt < 8; attempt++) {
    int32_t f = (int32_t)xo_below(&c->rng, (uint64_t)d);
    float thr;
    if (p->quantile_thresholds) {
      double q = xo_beta(&c->rng, 0.35, 0.35);
      for (int64_t r = 0; r < m; r++) c->vals[r] = c->X[(int64_t)c->idx[lo + r] * d + f];
      int64_t kq = (int64_t)(q * (double)(m - 1) + 0.5);
      if (kq < 0) kq = 0;
      if (kq > m - 1) kq = m - 1;
      thr = kth_smallest(c->vals, m, kq);
    } else {
      int64_t r = lo + (int64_t)xo_below(&c->rng, (uint64_t)m);
      thr = c->X[(int64_t)c->idx[r] * d + f];
    }
    int64_t nl = 0;
    for (int64_t r = lo; r < hi; r++) nl += (c->X[(int64_t)c->idx[r] * d + f] < thr);
    if (nl < p->min_leaf || m - nl < p->min_leaf) continue;
    /* stable partition: left rows first */
    int64_t a = lo, b = 0;
    for (int64_t r = lo; r < hi; r++) {
      int32_t row = c->idx[r];
      if (c->X[(int64_t)row * d + f] < thr) c->idx[a++] = row; else c->tmp[b++] = row;
    }
    memcpy(c->idx + a, c->tmp, sizeof(int32_t) * (size_t)b);
    int32_t L = tt_new(&c->tree, depth + 1);
    int32_t R = tt_new(&c->tree, depth + 1);
    c->tree.feature[node] = f;
    c->tree.threshold[node] = thr;
    c->tree.left[node] = L;
    c->tree.right[node] = R;
    grow(c, L, lo, lo + nl, depth + 1);
    grow(c, R, lo + nl, hi, depth + 1);
    return;
  }
}

typedef struct {
  const gen_forest_params* p;
  float* Xcal;
  gtree* trees;
} forest_handle;

static void build_tree(const gen_forest_params* p, const float* Xcal, int32_t t, gtree* out) {
  grow_ctx c;
  memset(&c, 0, sizeof(c));
  c.p = p;
  c.X = Xcal;
  c.idx = malloc(sizeof(int32_t) * (size_t)p->n_cal);
  c.tmp = malloc(sizeof(int32_t) * (size_t)p->n_cal);
  c.vals = p->quantile_thresholds ? malloc(sizeof(float) * (size_t)p->n_cal) : NULL;
  for (int64_t r = 0; r < p->n_cal; r++) c.idx[r] = (int32_t)r;
  xo_seed(&c.rng, key3(p->seed_forest, (uint64_t)t, 0x7ee5ULL));
  int32_t root = tt_new(&c.tree, 0);
  grow(&c, root, 0, p->n_cal, 0);
  tmp_tree* T = &c.tree;

  /* breadth-first order of the grown tree (root first) */
  int32_t* bfs = malloc(sizeof(int32_t) * (size_t)T->n);
  int32_t nb = 0, head = 0;
  bfs[nb++] = root;
  while (head < nb) {
    int32_t v = bfs[head++];
    if (T->feature[v] >= 0) { bfs[nb++] = T->left[v]; bfs[nb++] = T->right[v]; }
  }
  /* one bottom-up post-prune sweep (reverse BFS: children before parents, so collapses cascade) */
  uint8_t* dead = calloc((size_t)T->n, 1);
  for (int32_t q = nb - 1; q >= 0; q--) {
    int32_t v = bfs[q];
    if (T->feature[v] < 0) continue;
    int32_t L = T->left[v], R = T->right[v];
    if (T->feature[L] < 0 && T->feature[R] < 0 && xo_u01(&c.rng) < p->prune_p) {
      T->feature[v] = -1;
      dead[L] = dead[R] = 1;
    }
  }
  /* re-emit in BFS order over the surviving nodes */
  int32_t* newid = malloc(sizeof(int32_t) * (size_t)T->n);
  nb = 0; head = 0;
  bfs[nb++] = root;
  while (head < nb) {
    int32_t v = bfs[head++];
    if (T->feature[v] >= 0) { bfs[nb++] = T->left[v]; bfs[nb++] = T->right[v]; }
  }
  for (int32_t q = 0; q < nb; q++) newid[bfs[q]] = q;
  out->n = nb;
  out->feature = malloc(sizeof(int32_t) * (size_t)nb);
  out->threshold = malloc(sizeof(float) * (size_t)nb);
  out->left = malloc(sizeof(int32_t) * (size_t)nb);
  out->right = malloc(sizeof(int32_t) * (size_t)nb);
  out->value = malloc(sizeof(float) * (size_t)nb);
  out->dleft = malloc((size_t)nb);
  xo256 lr;
  xo_seed(&lr, key3(p->seed_forest, (uint64_t)t, 0x1eafULL));
  for (int32_t q = 0; q < nb; q++) {
    int32_t v = bfs[q];
    int leaf = T->feature[v] < 0;
    out->feature[q] = leaf ? -1 : T->feature[v];
    out->threshold[q] = leaf ? 0.0f : T->threshold[v];
    out->left[q] = leaf ? -1 : newid[T->left[v]];
    out->right[q] = leaf ? -1 : newid[T->right[v]];
    uint64_t u = xo_next(&lr);
    out->dleft[q] = leaf ? 0 : (uint8_t)(u & 1);
    if (leaf) {
      if (p->leaf_mode == 0) {
        int64_t K = p->leaf_k;
        int64_t k = (int64_t)((u >> 1) % (uint64_t)(2 * K + 1)) - K;
        out->value[q] = (float)((double)k / 256.0);
      } else {
        out->value[q] = (float)(0.1 * xo_normal(&lr));
      }
    } else {
      out->value[q] = 0.0f;
    }
  }
  (void)dead;
  free(dead); free(newid); free(bfs);
  free(T->feature); free(T->left); free(T->right); free(T->depth); free(T->threshold);
  free(c.idx); free(c.tmp); free(c.vals);
}

GEN_API void* gen_forest_grow(const gen_forest_params* p, int32_t nthreads) {
  forest_handle* h = calloc(1, sizeof(forest_handle));
  h->p = p;
  h->Xcal = malloc(sizeof(float) * (size_t)(p->n_cal * p->n_features));
  gen_rows(p->shape, p->seed_cal, 0, p->n_cal, p->n_features, h->Xcal, nthreads);
  h->trees = calloc((size_t)p->n_trees, sizeof(gtree));
#ifdef _OPENMP
  if (nthreads <= 0) nthreads = omp_get_max_threads();
#pragma omp parallel for schedule(dynamic, 1) num_threads(nthreads)
#endif
  for (int32_t t = 0; t < p->n_trees; t++) build_tree(p, h->Xcal, t, &h->trees[t]);
  free(h->Xcal);
  h->Xcal = NULL;
  return h;
}

GEN_API int64_t gen_forest_n_nodes(void* hp) {
  forest_handle* h = hp;
  int64_t s = 0;
  for (int32_t t = 0; t < h->p->n_trees; t++) s += h->trees[t].n;
  return s;
}

/* global node arrays; trees concatenated, root[t] = first node of tree t */
GEN_API void gen_forest_export(void* hp, int32_t* root, int32_t* feature, float* threshold,
                               int32_t* left, int32_t* right, float* leaf_value,
                               uint8_t* default_left, int32_t* tree_class) {
  forest_handle* h = hp;
  int64_t base = 0;
  for (int32_t t = 0; t < h->p->n_trees; t++) {
    gtree* g = &h->trees[t];
    root[t] = (int32_t)base;
    tree_class[t] = t % h->p->n_classes;
    for (int32_t q = 0; q < g->n; q++) {
      int64_t o = base + q;
      feature[o] = g->feature[q];
      threshold[o] = g->threshold[q];
      left[o] = g->left[q] < 0 ? -1 : (int32_t)(base + g->left[q]);
      right[o] = g->right[q] < 0 ? -1 : (int32_t)(base + g->right[q]);
      leaf_value[o] = g->value[q];
      default_left[o] = g->dleft[q];
    }
    base += g->n;
  }
}

GEN_API void gen_forest_free(void* hp) {
  forest_handle* h = hp;
  if (!h) return;
  for (int32_t t = 0; t < h->p->n_trees; t++) {
    gtree* g = &h->trees[t];
    free(g->feature); free(g->threshold); free(g->left); free(g->right); free(g->value);
    free(g->dleft);
  }
  free(h->trees);
  free(h);
}

/* seeded sorted subsample of k distinct row indices from [0, n) (Floyd's algorithm + sort) */
static int cmp_i64(const void* a, const void* b) {
  int64_t x = *(const int64_t*)a, y = *(const int64_t*)b;
  return (x > y) - (x < y);
}
GEN_API void gen_subsample(uint64_t seed, int64_t n, int64_t k, int64_t* out) {
  if (k >= n) { for (int64_t i = 0; i < n; i++) out[i] = i; return; }
  /* open-addressing set */
  int64_t cap = 1;
  while (cap < 2 * k) cap <<= 1;
  int64_t* set = malloc(sizeof(int64_t) * (size_t)cap);
  for (int64_t i = 0; i < cap; i++) set[i] = -1;
  int64_t m = 0;
  for (int64_t j = n - k; j < n; j++) {
    int64_t t = (int64_t)(sm64(key3(seed, (uint64_t)j, 0x5a3ULL)) % (uint64_t)(j + 1));
    int64_t pick = t;
    for (int pass = 0; pass < 2; pass++) {
      int64_t hsh = (int64_t)(sm64((uint64_t)pick) & (uint64_t)(cap - 1)), found = 0;
      while (set[hsh] >= 0) { if (set[hsh] == pick) { found = 1; break; } hsh = (hsh + 1) & (cap - 1); }
      if (!found) { set[hsh] = pick; out[m++] = pick; break; }
      pick = j;
    }
  }
  free(set);
  qsort(out, (size_t)m, sizeof(int64_t), cmp_i64);
}
