// internal.hpp — host-side model of a forest, its layout state and its encoded images.
// Everything here is product code (libtahoe.so); nothing is shared with oracle/.
#pragma once
#include <cstdint>
#include <mutex>
#include <cuda_runtime.h>
#include <string>
#include <vector>

#include "tahoe.h"
#include "kernels.hpp"

namespace tahoe {

// Set the thread-local error message and return the status.
tahoe_status fail(tahoe_status st, const std::string& msg);

// Forest in compact form: every tree's reachable nodes, tree-local DFS order (left first),
// concatenated.  Child indices are compact (global within this struct).  P:181-192.
struct Forest {
  int32_t n_trees = 0;
  int32_t n_trees_full = 0;     // tree count of the full forest (AVERAGE divides by it; shards)
  int32_t n_nodes_user = 0;     // length of the caller's arrays
  int32_t n_features = 0;
  int32_t n_classes = 1;
  int32_t agg = 0;
  float base = 0.0f;
  int32_t max_feature = -1;     // largest attribute index used by an internal node

  std::vector<int32_t> node_base;   // [T+1]
  std::vector<int32_t> feat;        // -1 = leaf
  std::vector<float> thr;
  std::vector<int32_t> lc, rc;      // compact children
  std::vector<float> val;
  std::vector<uint8_t> dl;          // default_left (NaN goes left)
  std::vector<int32_t> orig;        // caller node id
  std::vector<int32_t> depth;       // node depth (root 0)
  std::vector<int32_t> tclass;      // per tree
  std::vector<int32_t> tree_orig;   // caller tree index

  // ---- layout state (tahoe_forest_layout) ----
  bool calibrated = false;
  int64_t n_cal = 0;
  std::vector<uint64_t> count;      // calibration visits per compact node
  std::vector<uint8_t> hot_left;    // 1 = left child is the hot child
  std::vector<double> exp_reads;    // per tree: expected nodes read per sample (incl. leaf)
  std::vector<int32_t> order;       // tree order (class-major, similarity order within class)
  std::vector<float> Xsim;          // <= 1024 calibration rows kept to simulate and balance lockstep work
  int32_t dsim = 0;
  tahoe_layout_opts opts{};

  int32_t n_out() const { return (agg == TAHOE_AGG_CLASS_SUM || agg == TAHOE_AGG_VOTE) ? n_classes : 1; }
  int32_t tree_size(int32_t t) const { return node_base[t + 1] - node_base[t]; }
};

// Build + validate from the caller's arrays (tahoe_forest_build's checks).
tahoe_status build_forest(Forest& F, int32_t n_trees, const int32_t* root, int32_t n_nodes,
                          const int32_t* feature, const float* threshold, const int32_t* left,
                          const int32_t* right, const float* leaf_value,
                          const uint8_t* default_left, const int32_t* tree_class,
                          int32_t n_features, int32_t n_classes, int32_t agg, float base);
void default_layout(Forest& F);
Forest make_shard(const Forest& F, int32_t rank, int32_t world);

// ---- layout steps (layout.cpp) ----
void calibrate(Forest& F, const float* X, int64_t n, int32_t d);
void set_counts(Forest& F, const uint64_t* counts_by_caller_id, int64_t n_calib);
void reorder_nodes(Forest& F, bool enable);
std::vector<int32_t> hot_preorder(const Forest& F, int32_t t);   // compact ids, hot child first
void tree_tokens(const Forest& F, int32_t t, int32_t t_nodes, std::vector<int32_t>& tok_nodes,
                 std::vector<double>& weights);
void tree_simhash(const Forest& F, int32_t t, int32_t t_nodes, int32_t l_hash,
                  std::vector<double>& checksum, std::vector<uint8_t>& bits);
void sha1(const uint8_t* msg, size_t len, uint8_t out[20]);
void simhash(const int8_t* strings, const double* w, int32_t n, int32_t l, double* cs, uint8_t* bits);
std::vector<int32_t> lsh_order(const std::vector<uint8_t>& bits, int32_t n_trees, int32_t l_hash,
                               int32_t m_chunks, std::vector<uint16_t>* collisions);
void order_trees(Forest& F);

// ---- encoded images (encode.cpp) ----
struct SlicedImage {
  bool valid = false;
  std::string why_invalid;
  int32_t n_slices = 0, slots_max = 0, fbits = 0;
  std::vector<int32_t> slots, cls, ntrees;       // per slice
  std::vector<int32_t> col_len;                  // [ns*16]
  std::vector<int32_t> col_mid;                  // [ns*16] slot of the first tree of the column's
                                                 // second half by expected work (== col_len: none)
  std::vector<uint32_t> nodes;                   // [ns*slots_max*32*2]
  std::vector<int32_t> leaf_meta;                // [ns*slots_max*32*2] {tree, node}
  std::vector<int32_t> class_ptr, class_parts;   // class -> slices (CSR)
  double eff = 0.0;                              // est. lockstep efficiency (mean/max column)
  double eff_sim = 0.0;                          // simulated 2-chain lockstep efficiency
  double trees_per_lane = 0.0;
  std::vector<double> slice_work;                // issued lane-steps per row, per slice
  // Rank-coded twin of `nodes` (reading R7): same slots and packing, internal x = threshold rank
  // t = j + 1 (j = index of the threshold in its attribute's sorted distinct thresholds), attribute
  // field a byte offset into rows of u16 codes; thr_tab/thr_off hold the sorted thresholds.
  bool code_valid = false;
  std::string code_why;
  std::vector<uint32_t> cnodes;                  // [ns*slots_max*16*2]
  std::vector<float> thr_tab;                    // concatenated sorted distinct thresholds
  std::vector<int32_t> thr_off;                  // [n_features + 1]
  std::vector<int32_t> code_slot;                // [n_features] u16 slot of each attribute in a code row (R10)
  std::vector<int32_t> slot_attr;                // [2^fbits] its inverse (-1 = pad slot)
  // bank-private threshold tables for the row-coding pre-pass (encode.cpp build_code_banks);
  // empty when they do not fit shared memory (the pre-pass then bisects thr_tab through L2)
  std::vector<float> cb_img;                     // [cb_rows][32] words: the shared-memory image
  std::vector<int32_t> cb_desc;                  // [passes][32 lanes] {slot, attribute, word0, sh<<16|K}
  int32_t cb_passes = 0, cb_rows = 0;
  // Wide rank codes (reading R8): rows of more than 127 attributes become u8 codes over VIRTUAL
  // attributes (an attribute with K distinct thresholds is split into ceil(K / 127) pieces, each
  // coding its own <= 127 thresholds), so that a 16-row tile of code rows can be staged in shared
  // memory next to a (smaller) slice.  When code8 is set, cnodes hold the u8 node words
  // (kernels.hpp "wide codes"), thr_tab/thr_off are per virtual attribute and v_src maps a
  // virtual attribute to its source column.
  bool code8 = false;
  int32_t vfbits = 0;                            // code row = 2^vfbits bytes
  int32_t n_virtual = 0;
  std::vector<int32_t> v_src;                    // [2^vfbits] source column, -1 = pad byte
  std::vector<float> c8_img;                     // pre-pass tables, bank-private, band after band
  std::vector<int32_t> c8_grp;                   // [2^vfbits / 32] {word offset in band, probes, band, 0}
  std::vector<int32_t> c8_band;                  // [bands] {byte offset, bytes, first group, end group}
  int32_t c8_bands = 0;
  int64_t bytes() const { return (int64_t)nodes.size() * 4; }
};

struct DirectImage {
  int32_t fbits = 0;
  std::vector<uint32_t> nodes;        // [N*2]
  std::vector<int32_t> root, cls, tree_orig;
  std::vector<int32_t> slot_orig;     // caller node id per node slot
  std::vector<int32_t> cls_seg;       // [n_classes + 1]: tree slots of class c are [cls_seg[c], cls_seg[c+1])
  int64_t bytes() const { return (int64_t)nodes.size() * 4; }
};

int32_t feature_bits(int32_t n_features);
tahoe_status encode_direct(const Forest& F, DirectImage& D);
// max_smem > 0 enables the wide rank codes (reading R8) for forests over more than 127 attributes:
// the slices are then packed for the smaller budget that leaves room for the u8 code-tile ring.
tahoe_status encode_sliced(const Forest& F, int32_t slot_budget, SlicedImage& S, int32_t max_smem = 0);

// Cost model (costmodel.cpp) — Algorithm 1 lines 8-13 re-targeted.
struct PlanStats {
  double V = 0;            // expected nodes read per sample (sum over trees)
  double sliced_eff = 0;   // simulated lockstep efficiency of the sliced packing
  int32_t n_slices = 0;
  int32_t num_sms = 148;
  bool sliced_ok = false;
  bool rows_global = false;  // sliced rows too wide to stage in shared memory
  bool wide_rows = false;    // d > 256: direct reads attributes from rows far apart in memory
  bool coded_ok = false;     // rank-coded twin available and enabled (reading R7)
  int32_t code_passes = 1;   // row-coding passes of 32 attributes
  bool code8 = false;        // the coded twin is the wide-code one (reading R8)
  bool rows_ok = false;      // the ROWS strategy fits shared memory (row + per-tree values)
  int32_t rows_per_sm = 1;   // resident ROWS CTAs per SM
  int32_t n_trees = 1;
  int32_t d = 0;             // attributes per row of the batch
  int32_t n_out = 1;         // output groups (classes)
  bool scalar = true;        // one output, not VOTE (the direct large-batch kernel applies)
};
// Fitted per-platform constants (costmodel_b200.json, scripts/fit_costmodel.py), microseconds.
struct CostParams {
  double a_s = 22.3, b_s = 9.5e-5;           // sliced: launch + slice staging; per work unit
  double g_s = 4.0;                          // sliced: slowdown when rows stay in global memory
  double a_d = 11.8, l_d = 0.34, b_d = 6.3e-4; // direct: launch; per-visit latency; per unit
  double b_t = 2.0e-4;                         // direct, >= 32K rows, scalar: staged rows, 8 threads per row
  double g_d = 4.0;                            // direct: slowdown for wide rows (d > 256)
  double a_c = 30.0, b_c = 6.6e-5, e_c = 1.6e-5; // coded: launches; per unit; per row-pass per SM
  double a_w = 40.0, b_w = 1.5e-4, e_w = 1.6e-5; // wide codes (reading R8): the same three terms
  // rows (f1): launch; per dependent node read (latency); per row and SM (throughput): per node
  // read, per output class (the block reduction), per attribute (row staging)
  double a_r = 2.0, b_r = 0.9, c_r = 3.3e-4, k_r = 0.2, w_r = 2.4e-4;
  bool fitted = false;
};
const CostParams& cost_params();
double predict_us(const PlanStats& st, int32_t strategy, int64_t n);
int32_t select_strategy(const PlanStats& st, int64_t n, int32_t d, int32_t agg);
PlanStats plan_stats_for(const struct ::tahoe_forest* f, int32_t d);

}  // namespace tahoe

// The opaque handle.
struct tahoe_forest {
  tahoe::Forest host;
  tahoe::DirectImage di;
  tahoe::SlicedImage sl;
  int32_t device = -1;
  int32_t slot_budget = 0;       // slot rows of 32 nodes that fit the per-CTA forest smem budget
  int32_t num_sms = 0;
  // direct strategy: tree-slot boundaries of L2-sized chunks (one launch per chunk when the direct
  // image exceeds the L2 budget, so each chunk's nodes stay L2-resident while every row walks it)
  std::vector<int32_t> direct_chunks;   // [0, s1, s2, ..., n_slots]
  int32_t max_smem = 0;
  // device copies
  tahoe::DevDirect dd{};
  tahoe::DevSliced ds{};
  int32_t* d_class_ptr = nullptr;   // sliced class CSR
  // CTAs of a full-GPU sliced launch per slice, proportional to slice_work (prefix, ns + 1):
  // the slices' CTAs then grab tiles dynamically, so every slice finishes at about the same time
  std::vector<int32_t> cta_start;
  int32_t* d_cta_start = nullptr;
  int32_t* d_class_parts = nullptr;
  // tahoe_predict_host's copy / compute / copy-back streams and their events, created on first use
  // and kept for the handle's lifetime (not per call); host_mu serialises concurrent host calls on
  // one handle (they share these streams)
  struct HostPipe {
    bool ready = false;
    cudaStream_t s_in = nullptr, s_cmp = nullptr, s_cmp2 = nullptr, s_out = nullptr;
    cudaEvent_t ev_start = nullptr, ev_in[3] = {}, ev_cmp[3] = {}, ev_out[3] = {};
  } hp;
  std::mutex host_mu;
};
