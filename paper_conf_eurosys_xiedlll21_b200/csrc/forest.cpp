// forest.cpp — tahoe_forest_build's validation and the compact host model.
// A forest is a set of binary trees; a node holds an attribute index, a threshold and a default
// path; leaves hold the tree's prediction.
#include <cmath>
#include <cstring>
#include <algorithm>
#include <numeric>

#include "internal.hpp"

namespace tahoe {

int32_t feature_bits(int32_t n_features) {
  int32_t b = 1;
  while (b < 31 && (1 << b) < n_features) b++;
  return b;
}

tahoe_status build_forest(Forest& F, int32_t n_trees, const int32_t* root, int32_t n_nodes,
                          const int32_t* feature, const float* threshold, const int32_t* left,
                          const int32_t* right, const float* leaf_value,
                          const uint8_t* default_left, const int32_t* tree_class,
                          int32_t n_features, int32_t n_classes, int32_t agg, float base) {
  if (n_trees < 1) return fail(TAHOE_E_INVAL, "n_trees must be >= 1");
  if (n_classes < 1) return fail(TAHOE_E_INVAL, "n_classes must be >= 1");
  if (n_nodes < 1) return fail(TAHOE_E_INVAL, "n_nodes must be >= 1");
  if (n_features < 1) return fail(TAHOE_E_INVAL, "n_features must be >= 1");
  if (agg < TAHOE_AGG_SUM || agg > TAHOE_AGG_VOTE) return fail(TAHOE_E_INVAL, "unknown aggregation");
  if (!root || !feature || !threshold || !left || !right || !leaf_value)
    return fail(TAHOE_E_INVAL, "NULL node array");
  if (std::isnan(base)) return fail(TAHOE_E_INVAL, "NaN base_score");

  F = Forest();
  F.n_trees = n_trees;
  F.n_trees_full = n_trees;
  F.n_nodes_user = n_nodes;
  F.n_features = n_features;
  F.n_classes = n_classes;
  F.agg = agg;
  F.base = base;
  F.node_base.assign(1, 0);
  std::vector<uint8_t> seen((size_t)n_nodes, 0);
  std::vector<int32_t> stack;
  std::vector<int32_t> local;       // caller id -> compact id for the current tree
  std::vector<std::pair<int32_t, int32_t>> kids;  // pending child wiring (compact parent, caller child)
  for (int32_t t = 0; t < n_trees; t++) {
    int32_t r = root[t];
    if (r < 0 || r >= n_nodes) return fail(TAHOE_E_INVAL, "root of tree " + std::to_string(t) + " out of range");
    int32_t c = tree_class ? tree_class[t] : t % n_classes;
    if (c < 0 || c >= n_classes) return fail(TAHOE_E_INVAL, "tree_class out of range for tree " + std::to_string(t));
    F.tclass.push_back(c);
    F.tree_orig.push_back(t);
    // depth-first, left child first; compact ids in visit order
    const int32_t base_id = (int32_t)F.feat.size();
    stack.assign(1, r);
    std::vector<int32_t> dstack(1, 0);
    std::vector<int32_t> parent_slot(1, -1);   // compact parent, and which side (encoded)
    while (!stack.empty()) {
      int32_t k = stack.back(); stack.pop_back();
      int32_t dep = dstack.back(); dstack.pop_back();
      int32_t ps = parent_slot.back(); parent_slot.pop_back();
      if (k < 0 || k >= n_nodes) return fail(TAHOE_E_INVAL, "child index out of range in tree " + std::to_string(t));
      if (seen[k]) return fail(TAHOE_E_INVAL, "node " + std::to_string(k) + " reachable twice (shared or cyclic)");
      seen[k] = 1;
      int32_t id = (int32_t)F.feat.size();
      if (ps >= 0) {
        int32_t p = ps >> 1;
        if (ps & 1) F.rc[p] = id; else F.lc[p] = id;
      }
      int32_t f = feature[k];
      F.orig.push_back(k);
      F.depth.push_back(dep);
      F.dl.push_back(default_left ? (default_left[k] ? 1 : 0) : 0);
      F.lc.push_back(-1);
      F.rc.push_back(-1);
      if (f < 0) {
        float v = leaf_value[k];
        if (agg == TAHOE_AGG_VOTE) {
          if (!(v >= 0.0f && v < (float)n_classes && v == std::floor(v)))
            return fail(TAHOE_E_INVAL, "VOTE leaf " + std::to_string(k) + " is not a class id");
        } else if (!std::isfinite(v)) {
          return fail(TAHOE_E_INVAL, "non-finite leaf value at node " + std::to_string(k));
        }
        F.feat.push_back(-1);
        F.thr.push_back(0.0f);
        F.val.push_back(v);
      } else {
        if (f >= n_features) return fail(TAHOE_E_INVAL, "feature " + std::to_string(f) + " >= n_features at node " + std::to_string(k));
        if (std::isnan(threshold[k])) return fail(TAHOE_E_INVAL, "NaN threshold at node " + std::to_string(k));
        F.feat.push_back(f);
        F.thr.push_back(threshold[k]);
        F.val.push_back(0.0f);
        F.max_feature = std::max(F.max_feature, f);
        // push right first so left is visited first (preorder, left first)
        stack.push_back(right[k]); dstack.push_back(dep + 1); parent_slot.push_back((id << 1) | 1);
        stack.push_back(left[k]);  dstack.push_back(dep + 1); parent_slot.push_back((id << 1) | 0);
      }
    }
    (void)base_id;
    F.node_base.push_back((int32_t)F.feat.size());
  }
  default_layout(F);
  return TAHOE_OK;
}

// Layout before any calibration: left child first everywhere, input tree order (class-major),
// expected reads under 50/50 branch probabilities.
void default_layout(Forest& F) {
  const size_t N = F.feat.size();
  F.hot_left.assign(N, 1);
  F.count.assign(N, 0);
  F.calibrated = false;
  F.n_cal = 0;
  F.exp_reads.assign(F.n_trees, 0.0);
  for (int32_t t = 0; t < F.n_trees; t++) {
    double s = 0;
    for (int32_t k = F.node_base[t]; k < F.node_base[t + 1]; k++) s += std::ldexp(1.0, -F.depth[k]);
    F.exp_reads[t] = s;
  }
  F.order.clear();
  for (int32_t c = 0; c < F.n_classes; c++)
    for (int32_t t = 0; t < F.n_trees; t++)
      if (F.tclass[t] == c) F.order.push_back(t);
}

// Trees of `rank` out of `world`: LPT on expected reads (deterministic), kept in the parent's
// class-major similarity order.  Layout decisions (hot children, counts) are inherited.
Forest make_shard(const Forest& F, int32_t rank, int32_t world) {
  std::vector<int32_t> byw(F.n_trees);
  std::iota(byw.begin(), byw.end(), 0);
  std::stable_sort(byw.begin(), byw.end(), [&](int32_t a, int32_t b) {
    if (F.exp_reads[a] != F.exp_reads[b]) return F.exp_reads[a] > F.exp_reads[b];
    return a < b;
  });
  std::vector<double> load((size_t)world, 0.0);
  std::vector<int32_t> owner((size_t)F.n_trees, 0);
  for (int32_t t : byw) {
    int32_t best = 0;
    for (int32_t r = 1; r < world; r++) if (load[r] < load[best]) best = r;
    owner[t] = best;
    load[best] += F.exp_reads[t];
  }
  Forest S;
  S.n_trees_full = F.n_trees_full;
  S.n_nodes_user = F.n_nodes_user;
  S.n_features = F.n_features;
  S.n_classes = F.n_classes;
  S.agg = F.agg;
  S.base = F.base;
  S.max_feature = F.max_feature;
  S.calibrated = F.calibrated;
  S.n_cal = F.n_cal;
  S.opts = F.opts;
  S.Xsim = F.Xsim;
  S.dsim = F.dsim;
  S.node_base.assign(1, 0);
  std::vector<int32_t> newidx((size_t)F.n_trees, -1);
  for (int32_t t = 0; t < F.n_trees; t++) {
    if (owner[t] != rank) continue;
    newidx[t] = S.n_trees++;
    const int32_t b = F.node_base[t], e = F.node_base[t + 1];
    const int32_t nb = (int32_t)S.feat.size();
    for (int32_t k = b; k < e; k++) {
      S.feat.push_back(F.feat[k]);
      S.thr.push_back(F.thr[k]);
      S.lc.push_back(F.lc[k] < 0 ? -1 : F.lc[k] - b + nb);
      S.rc.push_back(F.rc[k] < 0 ? -1 : F.rc[k] - b + nb);
      S.val.push_back(F.val[k]);
      S.dl.push_back(F.dl[k]);
      S.orig.push_back(F.orig[k]);
      S.depth.push_back(F.depth[k]);
      S.count.push_back(F.count[k]);
      S.hot_left.push_back(F.hot_left[k]);
    }
    S.node_base.push_back((int32_t)S.feat.size());
    S.tclass.push_back(F.tclass[t]);
    S.tree_orig.push_back(F.tree_orig[t]);
    S.exp_reads.push_back(F.exp_reads[t]);
  }
  for (int32_t t : F.order)
    if (newidx[t] >= 0) S.order.push_back(newidx[t]);
  return S;
}

}  // namespace tahoe
