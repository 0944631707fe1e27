/*
 * oracle/tahoe_oracle.c — the CPU ORACLE for batched decision-tree-ensemble prediction.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference leg may load or call this file.  It shares no code, header, table or helper with
 * the CUDA path (paper_conf_eurosys_xiedlll21_b200/); it reads the same user-level node arrays that
 * are passed to tahoe_forest_build, plus X.
 *
 * What it computes is the plain definition of the result; Tahoe's techniques change
 * memory layout and scheduling only, so no layout appears here.
 *
 *   for each sample i, for each tree t in input order:
 *       k = root[t]
 *       while feature[k] >= 0:                      node = {attribute index, threshold}
 *           x = X[i*d + feature[k]]
 *           go_left = isnan(x) ? default_left[k]    default path D for a missing value (
 *                                                   reading Z3: NaN only; no array => comparison,
 *                                                   which is false => right)
 *                              : (x < threshold[k]) the choice "x_j < b_i"; true => left
 *                                                   (reading Z1), IEEE fp32 '<', equal => right (Z2)
 *           k = go_left ? left[k] : right[k]; visits++
 *       leaf[i][t] = k                              original global node id (Z21)
 *       fp += mix64(((u64)t << 32) | (u32)k)        order-independent fingerprint
 *       combine: acc[class(t)] += (double)value[k]  "predictions ... combined together" (P:51-53,
 *                (VOTE: votes[(int)value[k]]++)       P:435-437); class(t) = tree_class or t % C (Z15)
 *   finalize (reading Z14/Z17; fp64 throughout, then one round-to-nearest to fp32):
 *       SUM       out = acc + base
 *       AVERAGE   out = acc / T + base
 *       BINARY    out = acc + base;  class = out > 0 (fp64 margin; tie at 0 => 0)
 *       CLASS_SUM out[c] = acc[c] + base; class = argmax_c (lowest c on ties)
 *       VOTE      out[c] = votes[c];  class = argmax_c (lowest c on ties)
 *
 * The OpenMP driver only splits the sample loop; the per-sample code is unchanged.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define OR_API __attribute__((visibility("default")))

enum { OR_SUM = 0, OR_AVERAGE = 1, OR_BINARY = 2, OR_CLASS_SUM = 3, OR_VOTE = 4 };

/* splitmix64 finaliser (the fingerprint mixing function named in SURVEY §8(b)) */
static inline uint64_t or_mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
  return z ^ (z >> 31);
}

OR_API int oracle_n_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

/*
 * rows == NULL: samples 0..n-1 of X.  rows != NULL: sample r is row rows[r] of X (n entries).
 * Outputs (any may be NULL):
 *   out       float  [n * n_out]   n_out = 1 for SUM/AVERAGE/BINARY, n_classes otherwise
 *   out_raw   double [n * n_out]   the fp64 combined value before rounding
 *   out_class int32  [n]           BINARY / CLASS_SUM / VOTE
 *   out_leaf  int32  [n * T]       reached leaf (original node id), tree order
 *   out_fp    uint64 [n]
 *   out_visits uint64 [n]          internal nodes visited, summed over trees
 */
OR_API int oracle_predict(int32_t n_trees, const int32_t* root, int32_t n_nodes,
                          const int32_t* feature, const float* threshold, const int32_t* left,
                          const int32_t* right, const float* leaf_value,
                          const uint8_t* default_left, const int32_t* tree_class,
                          int32_t n_classes, int32_t agg, float base_score, const float* X,
                          int64_t n, int32_t d, const int64_t* rows, float* out, double* out_raw,
                          int32_t* out_class, int32_t* out_leaf, uint64_t* out_fp,
                          uint64_t* out_visits, int32_t nthreads) {
  (void)n_nodes;
  const int n_out = (agg == OR_CLASS_SUM || agg == OR_VOTE) ? n_classes : 1;
#ifdef _OPENMP
  if (nthreads <= 0) nthreads = omp_get_max_threads();
#pragma omp parallel num_threads(nthreads)
#endif
  {
    double* acc = malloc(sizeof(double) * (size_t)n_classes);
    int64_t* votes = malloc(sizeof(int64_t) * (size_t)n_classes);
#ifdef _OPENMP
#pragma omp for schedule(dynamic, 64)
#endif
    for (int64_t i = 0; i < n; i++) {
      const float* x = X + (rows ? rows[i] : i) * (int64_t)d;
      for (int c = 0; c < n_classes; c++) { acc[c] = 0.0; votes[c] = 0; }
      uint64_t fp = 0, visits = 0;
      for (int32_t t = 0; t < n_trees; t++) {
        int32_t k = root[t];
        while (feature[k] >= 0) {
          float v = x[feature[k]];
          int go_left;
          if (isnan(v)) go_left = default_left ? (default_left[k] != 0) : 0;
          else go_left = v < threshold[k];
          k = go_left ? left[k] : right[k];
          visits++;
        }
        if (out_leaf) out_leaf[i * (int64_t)n_trees + t] = k;
        fp += or_mix64(((uint64_t)(uint32_t)t << 32) | (uint64_t)(uint32_t)k);
        if (agg == OR_VOTE) {
          votes[(int)leaf_value[k]]++;
        } else {
          int c = tree_class ? tree_class[t] : (t % n_classes);
          acc[c] += (double)leaf_value[k];
        }
      }
      double s0;
      switch (agg) {
        case OR_SUM:
          s0 = acc[0] + (double)base_score;
          if (out) out[i] = (float)s0;
          if (out_raw) out_raw[i] = s0;
          break;
        case OR_AVERAGE:
          s0 = acc[0] / (double)n_trees + (double)base_score;
          if (out) out[i] = (float)s0;
          if (out_raw) out_raw[i] = s0;
          break;
        case OR_BINARY:
          s0 = acc[0] + (double)base_score;
          if (out) out[i] = (float)s0;
          if (out_raw) out_raw[i] = s0;
          if (out_class) out_class[i] = s0 > 0.0 ? 1 : 0;
          break;
        case OR_CLASS_SUM: {
          int best = 0;
          double bv = 0;
          for (int c = 0; c < n_classes; c++) {
            double s = acc[c] + (double)base_score;
            if (out) out[i * n_out + c] = (float)s;
            if (out_raw) out_raw[i * n_out + c] = s;
            if (c == 0 || s > bv) { best = c; bv = s; }
          }
          if (out_class) out_class[i] = best;
          break;
        }
        case OR_VOTE: {
          int best = 0;
          int64_t bv = -1;
          for (int c = 0; c < n_classes; c++) {
            if (out) out[i * n_out + c] = (float)votes[c];
            if (out_raw) out_raw[i * n_out + c] = (double)votes[c];
            if (votes[c] > bv) { best = c; bv = votes[c]; }
          }
          if (out_class) out_class[i] = best;
          break;
        }
      }
      if (out_fp) out_fp[i] = fp;
      if (out_visits) out_visits[i] = visits;
    }
    free(acc);
    free(votes);
  }
  return 0;
}

/*
 * Layout-side helper (never used for result parity): per-node visit counts of a calibration set,
 * count[k] = number of calibration rows whose path passes through node k.  Edge probability of
 * (parent -> child) = count[child] / count[parent]; node probability = count[k] / n = product of
 * edge probabilities on the root path.
 */
OR_API int oracle_node_counts(int32_t n_trees, const int32_t* root, const int32_t* feature,
                              const float* threshold, const int32_t* left, const int32_t* right,
                              const uint8_t* default_left, const float* X, int64_t n, int32_t d,
                              uint64_t* count) {
  for (int64_t i = 0; i < n; i++) {
    const float* x = X + i * (int64_t)d;
    for (int32_t t = 0; t < n_trees; t++) {
      int32_t k = root[t];
      count[k]++;
      while (feature[k] >= 0) {
        float v = x[feature[k]];
        int go_left = isnan(v) ? (default_left ? default_left[k] != 0 : 0) : (v < threshold[k]);
        k = go_left ? left[k] : right[k];
        count[k]++;
      }
    }
  }
  return 0;
}
