// encode.cpp — the adaptive forest format re-targeted to B200.
//
// Work units: the trees of one class, in similarity order, are cut into SLICES whose
// nodes fit one CTA's shared memory; inside a slice each tree is dealt to one of 16 LANE COLUMNS
// ("assigned to threads in a round-robin way, such that loads are roughly balanced"),
// with a longest-processing-time alternative when it balances expected work better (reading Z12).
// A lane column holds its trees back to back, each in left-first preorder (reading R1), so the
// left child of every node is the next slot.  Slot s of column c lives at word pair (16*s + c):
// the two half-warps each walk all 16 columns (for different samples), and an 8-byte load of a
// half-warp whose lanes sit at 16 different slots hits 16 different bank pairs.
#include <algorithm>
#include <cmath>
#include <cstring>
#include <limits>
#include <cstdlib>
#include <numeric>
#include <string>

#include "internal.hpp"

namespace tahoe {

static uint32_t f2u(float f) { uint32_t u; std::memcpy(&u, &f, 4); return u; }

int64_t code8_chunk_mb() {
  static const int64_t mb = [] {
    const char* e = std::getenv("TAHOE_CODE8_CHUNK_MB");
    return e && *e ? (int64_t)std::atoll(e) : (int64_t)0;
  }();
  return mb;
}

// ------------------------------------------------------------------ direct image
tahoe_status encode_direct(const Forest& F, DirectImage& D) {
  D = DirectImage();
  D.fbits = feature_bits(F.n_features);
  const uint32_t off_lim = 1u << (kOffsetTop - D.fbits);
  D.nodes.assign(F.feat.size() * 2, 0);
  D.slot_orig.assign(F.feat.size(), -1);
  int64_t base = 0;
  std::vector<int64_t> slot(F.feat.size());
  for (int32_t t : F.order) {
    std::vector<int32_t> pre = hot_preorder(F, t);
    for (size_t i = 0; i < pre.size(); i++) slot[pre[i]] = base + (int64_t)i;
    D.root.push_back((int32_t)base);
    D.cls.push_back(F.tclass[t]);
    D.tree_orig.push_back(F.tree_orig[t]);
    for (size_t i = 0; i < pre.size(); i++) {
      const int32_t k = pre[i];
      const int64_t s = base + (int64_t)i;
      D.slot_orig[s] = F.orig[k];
      uint32_t y;
      if (F.feat[k] < 0) {
        y = kLeafBit | (uint32_t)F.orig[k];
        D.nodes[2 * s] = f2u(F.val[k]);
      } else {
        const int32_t hot = F.hot_left[k] ? F.lc[k] : F.rc[k];
        const int32_t cold = F.hot_left[k] ? F.rc[k] : F.lc[k];
        if (slot[hot] != s + 1) return fail(TAHOE_E_INVAL, "internal: hot child not adjacent");
        const int64_t delta = slot[cold] - s;
        if (delta <= 0 || (uint64_t)delta >= off_lim)
          return fail(TAHOE_E_UNSUPPORTED, "tree too large for the node encoding (cold offset " +
                                                std::to_string(delta) + ")");
        y = (F.dl[k] ? kDefaultLeftBit : 0u) | (F.hot_left[k] ? kHotLeftBit : 0u) |
            ((uint32_t)delta << D.fbits) | (uint32_t)F.feat[k];
        D.nodes[2 * s] = f2u(F.thr[k]);
      }
      D.nodes[2 * s + 1] = y;
    }
    base += (int64_t)pre.size();
  }
  // trees are class-major (F.order), so each class's tree slots are one contiguous range
  D.cls_seg.assign(F.n_classes + 1, 0);
  for (int32_t c : D.cls) D.cls_seg[c + 1]++;
  for (int32_t c = 0; c < F.n_classes; c++) D.cls_seg[c + 1] += D.cls_seg[c];
  return TAHOE_OK;
}

// ------------------------------------------------------------------ sliced image
struct Pack {
  std::vector<std::vector<int32_t>> lanes = std::vector<std::vector<int32_t>>(kSlicedCols);
  int32_t max_len = 0;
  double max_work = 0, sum_work = 0;
};

// Slots a tree occupies in a lane column: a single-leaf tree is encoded as a 3-node stump (an
// internal root whose two children are copies of the leaf) so that every tree starts with an
// internal node — two consecutive steps of a lane then never both meet a nonzero leaf.
static int32_t enc_size(const Forest& F, int32_t t) {
  return F.tree_size(t) == 1 ? 3 : F.tree_size(t);
}

static void pack_stats(const Forest& F, Pack& P) {
  P.max_len = 0; P.max_work = 0; P.sum_work = 0;
  for (auto& L : P.lanes) {
    int32_t len = 0; double w = 0;
    for (int32_t t : L) { len += enc_size(F, t); w += F.exp_reads[t]; }
    P.max_len = std::max(P.max_len, len);
    P.max_work = std::max(P.max_work, w);
    P.sum_work += w;
  }
}

static bool pack_round_robin(const Forest& F, const std::vector<int32_t>& trees, int32_t cap, Pack& P) {
  P = Pack();
  for (size_t j = 0; j < trees.size(); j++) P.lanes[j % kSlicedCols].push_back(trees[j]);
  pack_stats(F, P);
  return P.max_len <= cap;
}

static bool pack_lpt(const Forest& F, const std::vector<int32_t>& trees, int32_t cap, Pack& P) {
  P = Pack();
  std::vector<int32_t> ts(trees);
  std::stable_sort(ts.begin(), ts.end(), [&](int32_t a, int32_t b) {
    if (F.exp_reads[a] != F.exp_reads[b]) return F.exp_reads[a] > F.exp_reads[b];
    return enc_size(F, a) > enc_size(F, b);
  });
  std::vector<double> w(kSlicedCols, 0.0);
  std::vector<int32_t> len(kSlicedCols, 0);
  for (int32_t t : ts) {
    int32_t best = -1;
    for (int32_t l = 0; l < kSlicedCols; l++) {
      if (len[l] + enc_size(F, t) > cap) continue;
      if (best < 0 || w[l] < w[best] || (w[l] == w[best] && len[l] < len[best])) best = l;
    }
    if (best < 0) return false;
    P.lanes[best].push_back(t);
    w[best] += F.exp_reads[t];
    len[best] += enc_size(F, t);
  }
  pack_stats(F, P);
  return true;
}

// Rounds: the similarity-ordered trees are dealt 16 at a time, one per lane (similar trees walk in
// different lanes at the same time, the paper's grouping + round-robin dealing), and
// inside each round the heaviest remaining tree goes to the lane with the least work so far
// (keeps the columns balanced like LPT).
static bool pack_rounds(const Forest& F, const std::vector<int32_t>& trees, int32_t cap, Pack& P) {
  P = Pack();
  const size_t C = kSlicedCols;
  std::vector<double> w(C, 0.0);
  std::vector<int32_t> len(C, 0);
  for (size_t r0 = 0; r0 < trees.size(); r0 += C) {
    std::vector<int32_t> round(trees.begin() + r0, trees.begin() + std::min(trees.size(), r0 + C));
    std::stable_sort(round.begin(), round.end(), [&](int32_t a, int32_t b) {
      if (F.exp_reads[a] != F.exp_reads[b]) return F.exp_reads[a] > F.exp_reads[b];
      return enc_size(F, a) > enc_size(F, b);
    });
    std::vector<int32_t> lanes(C);
    std::iota(lanes.begin(), lanes.end(), 0);
    std::stable_sort(lanes.begin(), lanes.end(), [&](int32_t a, int32_t b) {
      if (w[a] != w[b]) return w[a] < w[b];
      return len[a] < len[b];
    });
    std::vector<uint8_t> used(C, 0);
    for (int32_t t : round) {
      int32_t pick = -1;
      for (int32_t l : lanes)
        if (!used[l] && len[l] + enc_size(F, t) <= cap) { pick = l; break; }
      if (pick < 0) return false;
      used[pick] = 1;
      P.lanes[pick].push_back(t);
      w[pick] += F.exp_reads[t];
      len[pick] += enc_size(F, t);
    }
  }
  pack_stats(F, P);
  return true;
}

static bool pack_best(const Forest& F, const std::vector<int32_t>& trees, int32_t cap, Pack& P) {
  Pack a, b;
  static const char* mode = std::getenv("TAHOE_PACK");   // experiments: "rr" or "lpt"
  if (mode && std::string(mode) == "rr") return pack_round_robin(F, trees, cap, P);
  if (mode && std::string(mode) == "lpt") return pack_lpt(F, trees, cap, P);
  if (mode && std::string(mode) == "rounds") return pack_rounds(F, trees, cap, P);
  bool ra = pack_round_robin(F, trees, cap, a);
  bool rb = pack_lpt(F, trees, cap, b);
  if (!ra && !rb) return false;
  if (ra && (!rb || a.max_work <= b.max_work * 1.000001)) P = a; else P = b;
  return true;
}

// Nodes read per (calibration row, tree) — the kernel's step count for that walk (a single-leaf
// tree is a 3-node stump: 2 steps).  Empty when no rows were kept.
static std::vector<int32_t> sim_reads(const Forest& F, int64_t& m) {
  m = F.Xsim.empty() ? 0 : (int64_t)F.Xsim.size() / F.dsim;
  std::vector<int32_t> reads((size_t)m * F.n_trees);
  for (int64_t r = 0; r < m; r++) {
    const float* x = &F.Xsim[(size_t)r * F.dsim];
    for (int32_t t = 0; t < F.n_trees; t++) {
      int32_t k = F.node_base[t], c = 1;
      while (F.feat[k] >= 0) {
        const float v = x[F.feat[k]];
        const bool left = std::isnan(v) ? F.dl[k] != 0 : v < F.thr[k];
        k = left ? F.lc[k] : F.rc[k];
        c++;
      }
      reads[(size_t)r * F.n_trees + t] = (F.tree_size(t) == 1) ? 2 : c;
    }
  }
  return reads;
}

// Work units balanced on measured paths ("loads are roughly balanced", reading R6): a
// warp walks 4 rows x 16 lane columns in lockstep and waits for the longest of the 64 walks, so
// the cost of a packing on the kept calibration rows is sum over 4-row units of the maximum
// column work.  Greedy local search from the expected-work packing: tree swaps / moves between a
// unit's bottleneck column and another column, accepted when the cost drops and the slot cap
// holds.  Deterministic (fixed-seed generator).
static int kRefineIters = std::getenv("TAHOE_REFINE_ITERS") ? std::atoi(std::getenv("TAHOE_REFINE_ITERS")) : 200;
static void pack_refine(const Forest& F, const std::vector<int32_t>& reads, int64_t m, int32_t cap,
                        Pack& P) {
  const int32_t C = kSlicedCols;
  const int64_t U = m / 4;
  if (U < 4) return;
  const int32_t T = F.n_trees;
  std::vector<double> W((size_t)m * C, 0.0);         // W[r][c]
  std::vector<int32_t> len(C, 0);
  for (int32_t c = 0; c < C; c++)
    for (int32_t t : P.lanes[c]) {
      len[c] += enc_size(F, t);
      for (int64_t r = 0; r < m; r++) W[(size_t)r * C + c] += reads[(size_t)r * T + t];
    }
  auto colmax = [&](int64_t u, int32_t c, const double* wa) {   // max over the unit's rows
    double mx = 0;
    for (int64_t q = 4 * u; q < 4 * u + 4; q++) mx = std::max(mx, wa ? wa[q] : W[(size_t)q * C + c]);
    return mx;
  };
  std::vector<double> M((size_t)U * C), umax(U);
  for (int64_t u = 0; u < U; u++) {
    umax[u] = 0;
    for (int32_t c = 0; c < C; c++) { M[(size_t)u * C + c] = colmax(u, c, nullptr); umax[u] = std::max(umax[u], M[(size_t)u * C + c]); }
  }
  uint64_t st = 0x9E3779B97F4A7C15ull;
  auto rnd = [&](uint64_t lim) {
    st += 0x9E3779B97F4A7C15ull;
    uint64_t z = st;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return (z ^ (z >> 31)) % lim;
  };
  std::vector<double> na(m), nb(m), Ma(U), Mb(U);
  const int iters = kRefineIters * (int)std::max<size_t>(1, [&] { size_t k = 0; for (auto& L : P.lanes) k += L.size(); return k; }());
  for (int it = 0; it < iters; it++) {
    const int64_t u0 = (int64_t)rnd((uint64_t)U);
    int32_t a = 0;
    for (int32_t c = 1; c < C; c++) if (M[(size_t)u0 * C + c] > M[(size_t)u0 * C + a]) a = c;
    if (P.lanes[a].empty()) continue;
    const int32_t b = (a + 1 + (int32_t)rnd(C - 1)) % C;
    const size_t ia = rnd(P.lanes[a].size());
    const bool move = P.lanes[b].empty() || rnd(4) == 0;
    const size_t ib = move ? 0 : rnd(P.lanes[b].size());
    const int32_t ta = P.lanes[a][ia], tb = move ? -1 : P.lanes[b][ib];
    const int32_t sa = enc_size(F, ta), sb = move ? 0 : enc_size(F, tb);
    if (len[a] - sa + sb > cap || len[b] - sb + sa > cap) continue;
    for (int64_t r = 0; r < m; r++) {
      const double ra = reads[(size_t)r * T + ta], rb = move ? 0.0 : reads[(size_t)r * T + tb];
      na[r] = W[(size_t)r * C + a] - ra + rb;
      nb[r] = W[(size_t)r * C + b] - rb + ra;
    }
    double delta = 0;
    for (int64_t u = 0; u < U; u++) {
      Ma[u] = colmax(u, a, na.data());
      Mb[u] = colmax(u, b, nb.data());
      double mx = std::max(Ma[u], Mb[u]);
      for (int32_t c = 0; c < C; c++) if (c != a && c != b) mx = std::max(mx, M[(size_t)u * C + c]);
      delta += mx - umax[u];
    }
    if (delta >= 0) continue;
    // accept
    if (move) {
      P.lanes[a].erase(P.lanes[a].begin() + (long)ia);
      P.lanes[b].push_back(ta);
    } else {
      std::swap(P.lanes[a][ia], P.lanes[b][ib]);
    }
    len[a] += sb - sa;
    len[b] += sa - sb;
    for (int64_t r = 0; r < m; r++) { W[(size_t)r * C + a] = na[r]; W[(size_t)r * C + b] = nb[r]; }
    for (int64_t u = 0; u < U; u++) {
      M[(size_t)u * C + a] = Ma[u];
      M[(size_t)u * C + b] = Mb[u];
      double mx = 0;
      for (int32_t c = 0; c < C; c++) mx = std::max(mx, M[(size_t)u * C + c]);
      umax[u] = mx;
    }
  }
  // keep each column's trees in similarity order
  std::vector<int32_t> rank((size_t)T, 0);
  for (size_t q = 0; q < F.order.size(); q++) rank[(size_t)F.order[q]] = (int32_t)q;
  for (auto& L : P.lanes)
    std::sort(L.begin(), L.end(), [&](int32_t x, int32_t y) { return rank[x] < rank[y]; });
  pack_stats(F, P);
}

// Code-row slot of every attribute (reading R7; R10).  The two half-warps of a coded
// walk read u16 codes from two different rows; rows of >= 128 bytes keep attribute slot j of the
// second half's row at slot j ^ 32 (code_slot_swz), so logical words w and w ^ 16 of the two rows
// share a bank and collide (two wavefronts) whenever one half reads word w while the other reads
// word w ^ 16 (rows of 256 bytes: also words w and w + 32 of one row).  Which attribute sits in
// which slot does not change a single decision, so the slots are chosen to make collisions rare:
// every lane reads the word holding its node's attribute (probability of attribute a = its share
// of the calibrated internal visits, or of 2^-depth without calibration) or, at a leaf, the pad
// word of slot 2^F - 1 (probability T / (visits + T)); a deterministic local search (swaps and
// moves to free slots) minimises the estimated probability that some bank sees two addresses
// (16 active lanes per half, independent lanes).  Slot 2^F - 1 stays the leaves' pad.  Rows of
// 64 bytes (F <= 5) put the two rows in the two halves of one bank line: identity.
static std::vector<int32_t> code_slots(const Forest& F, int32_t fbits) {
  const int32_t nf = F.n_features;
  std::vector<int32_t> slot(nf);
  std::iota(slot.begin(), slot.end(), 0);
  const int32_t NS = 1 << fbits;
  if (fbits < 6 || nf <= 0 || nf >= NS) return slot;
  std::vector<double> wa(nf, 0.0);
  double visits = 0.0;
  const bool cal = !F.count.empty() && F.n_cal > 0;
  for (int32_t t = 0; t < F.n_trees; t++)
    for (int32_t k = F.node_base[t]; k < F.node_base[t + 1]; k++) {
      if (F.feat[k] < 0) continue;
      const double pk = cal ? (double)F.count[k] / (double)F.n_cal : std::ldexp(1.0, -std::min(F.depth[k], 60));
      wa[F.feat[k]] += pk;
      visits += pk;
    }
  if (!(visits > 0.0)) return slot;
  const double pl = (double)F.n_trees / (visits + (double)F.n_trees);
  for (auto& v : wa) v = v / visits * (1.0 - pl);
  const int32_t NW = NS / 2, leafw = (NS - 1) / 2;
  constexpr int kLanes = 16;
  auto cost = [&](const std::vector<int32_t>& sl) {
    std::vector<double> M(NW, 0.0);
    for (int32_t a = 0; a < nf; a++) M[sl[a] / 2] += wa[a];
    M[leafw] += pl;
    // physical word pw of half h holds logical word pw ^ (16 h); bank = pw % 32
    double ok = 1.0;
    for (int32_t b = 0; b < 32; b++) {
      double none = 1.0, one = 0.0;
      for (int32_t h = 0; h < 2; h++)
        for (int32_t pw = b; pw < NW; pw += 32) {
          const double u = 1.0 - std::pow(1.0 - M[pw ^ (16 * h)], kLanes);   // address used
          one = one * (1.0 - u) + none * u;
          none *= 1.0 - u;
        }
      ok *= none + one;   // at most one address in bank b
    }
    return 1.0 - ok;
  };
  std::vector<int32_t> best = slot;
  double bc = cost(best);
  std::vector<int32_t> free_slots;
  {
    std::vector<uint8_t> used(NS, 0);
    for (int32_t a = 0; a < nf; a++) used[slot[a]] = 1;
    for (int32_t j = 0; j < NS - 1; j++)
      if (!used[j]) free_slots.push_back(j);
  }
  uint64_t rs = 0x9E3779B97F4A7C15ull;
  auto rnd = [&](uint64_t m) {   // xorshift64*, deterministic
    rs ^= rs >> 12; rs ^= rs << 25; rs ^= rs >> 27;
    return (rs * 0x2545F4914F6CDD1Dull >> 33) % m;
  };
  for (int it = 0; it < 20000; it++) {
    if (free_slots.empty() || rnd(2) == 0) {
      const int32_t i = (int32_t)rnd(nf), j = (int32_t)rnd(nf);
      if (i == j) continue;
      std::swap(best[i], best[j]);
      const double c = cost(best);
      if (c < bc) bc = c;
      else std::swap(best[i], best[j]);
    } else {
      const int32_t i = (int32_t)rnd(nf);
      const size_t k = (size_t)rnd(free_slots.size());
      std::swap(best[i], free_slots[k]);
      const double c = cost(best);
      if (c < bc) bc = c;
      else std::swap(best[i], free_slots[k]);
    }
  }
  return best;
}

// Bank-private threshold tables for k_encode_rows_banks (reading R7).  A warp codes one row per
// pass: lane l of pass p bisects the sorted thresholds of one attribute, and every attribute of a
// pass owns its own set of m = 2^sh shared-memory banks {b, b + 32/m, b + 2*32/m, ...}: element i
// sits at word (region * 32 + b + i * 32/m), so the probe address is one multiply-add and the 32
// probes of a warp never collide, whatever the row values are.  Bank sets are handed out largest
// first (aligned blocks of the bit-reversed bank index, so they never fragment).  Passes = 2^F / 32
// code slots (at least 1); lanes without an attribute write a pad slot.  Spare banks go to the
// attributes with the most thresholds (halving their depth); the attributes are split over passes
// in decreasing order of threshold count, trying every size of the first pass.  The image is used
// when it fits kCodeBankBudget bytes of shared memory.
static void build_code_banks(const std::vector<std::vector<float>>& tabs, int32_t fbits,
                             const std::vector<int32_t>& code_slot, SlicedImage& S) {
  S.cb_img.clear();
  S.cb_desc.clear();
  S.cb_passes = 0;
  S.cb_rows = 0;
  const int32_t nf = (int32_t)tabs.size();
  const int32_t slots = 1 << fbits;
  const int32_t P = std::max(1, slots / 32);
  std::vector<int32_t> ord(nf);
  std::iota(ord.begin(), ord.end(), 0);
  std::stable_sort(ord.begin(), ord.end(), [&](int32_t a, int32_t b) { return tabs[a].size() > tabs[b].size(); });
  // one pass: spare-bank doubling, returns depth (rows) and per-feature shift
  auto plan_pass = [&](const std::vector<int32_t>& fs, std::vector<int32_t>& sh) -> int64_t {
    sh.assign(fs.size(), 0);
    int32_t spare = 32 - (int32_t)fs.size();
    for (;;) {
      int64_t best = -1;
      size_t bi = 0;
      for (size_t q = 0; q < fs.size(); q++) {
        const int64_t m = 1 << sh[q];
        const int64_t depth = ((int64_t)tabs[fs[q]].size() + m - 1) / m;
        if (m <= spare && sh[q] < 5 && depth > best) { best = depth; bi = q; }
      }
      if (best <= 1) break;
      spare -= 1 << sh[bi];
      sh[bi]++;
    }
    int64_t D = 0;
    for (size_t q = 0; q < fs.size(); q++)
      D = std::max<int64_t>(D, ((int64_t)tabs[fs[q]].size() + (1 << sh[q]) - 1) >> sh[q]);
    return D;
  };
  std::vector<std::vector<int32_t>> best_fs;
  int64_t best_rows = INT64_MAX;
  const int32_t lo0 = std::max(1, nf - 32 * (P - 1)), hi0 = std::min(32, nf);
  for (int32_t n0 = (nf == 0 ? 0 : lo0); n0 <= (nf == 0 ? 0 : hi0); n0++) {
    std::vector<std::vector<int32_t>> fs(P);
    fs[0].assign(ord.begin(), ord.begin() + n0);
    const int32_t rest = nf - n0;
    for (int32_t q = 0; q < rest; q++) fs[1 + (q * (P - 1)) / std::max(1, rest)].push_back(ord[n0 + q]);
    bool ok = true;
    int64_t rows = 0;
    for (auto& g : fs) {
      if ((int32_t)g.size() > 32) { ok = false; break; }
      std::vector<int32_t> sh;
      rows += plan_pass(g, sh);
    }
    if (ok && rows < best_rows) { best_rows = rows; best_fs = fs; }
  }
  if (best_fs.empty() || best_rows * 128 > kCodeBankBudget) return;
  S.cb_passes = P;
  S.cb_rows = (int32_t)best_rows;
  S.cb_img.assign((size_t)best_rows * 32, 0.0f);
  S.cb_desc.assign((size_t)P * 32 * 4, -1);
  // pad slots: every code slot that no attribute writes
  std::vector<int32_t> pads;
  {
    std::vector<uint8_t> used((size_t)std::max(slots, 32), 0);
    for (int32_t a = 0; a < nf; a++) used[code_slot[a]] = 1;
    for (int32_t j = 0; j < std::max(slots, 32); j++)
      if (!used[j]) pads.push_back(j);
  }
  size_t pad_i = 0;
  int64_t region = 0;
  for (int32_t p = 0; p < P; p++) {
    std::vector<int32_t> sh;
    const int64_t D = plan_pass(best_fs[p], sh);
    // bank sets, largest first: m banks {b + k * 32/m}, b the smallest base whose set is free
    std::vector<size_t> by_m(best_fs[p].size());
    std::iota(by_m.begin(), by_m.end(), 0);
    std::stable_sort(by_m.begin(), by_m.end(), [&](size_t a, size_t b) { return sh[a] > sh[b]; });
    uint32_t used = 0;
    int32_t lane = 0;
    for (size_t q : by_m) {
      const int32_t m = 1 << sh[q], stride = 32 / m;
      int32_t b = 0;
      for (; b < stride; b++) {
        uint32_t set = 0;
        for (int32_t k = 0; k < m; k++) set |= 1u << (b + k * stride);
        if (!(used & set)) { used |= set; break; }
      }
      const int32_t a = best_fs[p][q];
      const auto& v = tabs[a];
      for (size_t i = 0; i < v.size(); i++) S.cb_img[(size_t)region * 32 + b + i * stride] = v[i];
      int32_t* d = &S.cb_desc[((size_t)p * 32 + lane++) * 4];
      d[0] = code_slot[a];                                 // code slot written
      d[1] = a;                                            // attribute read
      d[2] = (int32_t)((region * 32 + b) * 4);             // byte offset of element 0
      d[3] = ((stride * 4) << 16) | (int32_t)v.size();     // element stride (bytes) | K
    }
    for (; lane < 32; lane++) {
      int32_t* d = &S.cb_desc[((size_t)p * 32 + lane) * 4];
      if (pad_i < pads.size()) d[0] = pads[pad_i++];
      d[1] = -1;
      d[2] = 0;
      d[3] = 0;
    }
    region += D;
  }
}

// Pre-pass tables of the wide codes (reading R8): groups of 32 consecutive virtual attributes, lane
// a of group g bisecting the sorted thresholds of virtual attribute 32g + a.  Element i of lane a
// sits at word (row0_g + i) * 32 + a (lane a owns bank a: the 32 probes of a warp never collide);
// every lane of a group is padded with NaN to 2^k - 1 elements, k = the group's probe count, so
// the bisection has a uniform trip count ("tab[i] <= x" stays true on a prefix: NaN <= x is
// false).  Groups are dealt to bands of balanced size <= kCode8BandBudget bytes and at most
// kCode8BandGroups groups (the TMA-staged pre-pass reads a band's attributes as one tensor box
// per row); a pre-pass CTA stages one band.
static void build_code8_banks(const std::vector<std::vector<float>>& vt, int32_t vfbits,
                              SlicedImage& S) {
  const int32_t G = (1 << vfbits) / 32;
  std::vector<int32_t> probes(G, 0);
  int64_t total = 0;
  for (int32_t g = 0; g < G; g++) {
    size_t mk = 0;
    for (int32_t a = 0; a < 32; a++) {
      const size_t v = (size_t)g * 32 + a;
      if (v < vt.size()) mk = std::max(mk, vt[v].size());
    }
    (void)mk;
    probes[g] = 7;   // every lane padded to 127 elements: one uniform 7-probe bisection
    total += (((int64_t)1 << probes[g]) - 1) * 128;
  }
  auto gbytes = [&](int32_t g) { return (((int64_t)1 << probes[g]) - 1) * 128; };
  std::vector<int32_t> cut;
  for (int32_t nb = (int32_t)std::max<int64_t>({(int64_t)1, (total + kCode8BandBudget - 1) / kCode8BandBudget,
                                                 ((int64_t)G + kCode8BandGroups - 1) / kCode8BandGroups});; nb++) {
    const int64_t target = (total + nb - 1) / nb;
    cut.assign(1, 0);
    int32_t g = 0;
    for (int32_t b = 0; b < nb; b++) {
      int64_t acc = 0;
      while (g < G && acc + gbytes(g) <= kCode8BandBudget && g - cut.back() < kCode8BandGroups &&
             (acc < target || b == nb - 1))
        acc += gbytes(g++);
      cut.push_back(g);
    }
    if (g == G) break;
  }
  cut.erase(std::unique(cut.begin(), cut.end()), cut.end());   // no empty bands
  S.c8_bands = (int32_t)cut.size() - 1;
  S.c8_grp.assign((size_t)G * 4, 0);
  S.c8_band.assign((size_t)S.c8_bands * 4, 0);
  S.c8_img.clear();
  const float qnan = std::numeric_limits<float>::quiet_NaN();
  for (int32_t b = 0; b < S.c8_bands; b++) {
    const int64_t off_words = (int64_t)S.c8_img.size();
    int64_t row = 0;
    for (int32_t g = cut[b]; g < cut[b + 1]; g++) {
      const int32_t D = (1 << probes[g]) - 1;
      S.c8_grp[(size_t)g * 4 + 0] = (int32_t)(row * 32);
      S.c8_grp[(size_t)g * 4 + 1] = probes[g];
      S.c8_grp[(size_t)g * 4 + 2] = b;
      S.c8_img.resize((size_t)(off_words + (row + D) * 32), qnan);
      for (int32_t a = 0; a < 32; a++) {
        const size_t v = (size_t)g * 32 + a;
        if (v >= vt.size()) continue;
        for (size_t i = 0; i < vt[v].size(); i++)
          S.c8_img[(size_t)(off_words + (row + (int64_t)i) * 32 + a)] = vt[v][i];
      }
      row += D;
    }
    S.c8_band[(size_t)b * 4 + 0] = (int32_t)(off_words * 4);
    S.c8_band[(size_t)b * 4 + 1] = (int32_t)(row * 128);
    S.c8_band[(size_t)b * 4 + 2] = cut[b];
    S.c8_band[(size_t)b * 4 + 3] = cut[b + 1];
  }
}

tahoe_status encode_sliced(const Forest& F, int32_t cap, SlicedImage& S, int32_t max_smem) {
  S = SlicedImage();
  S.fbits = feature_bits(F.n_features + 1);   // all-ones attribute field marks a leaf
  // per attribute the sorted distinct thresholds (IEEE equality: -0.0 and +0.0 are one value),
  // for the rank codes of readings R7 / R8
  std::vector<std::vector<float>> tabs(F.n_features);
  bool sub_leaf = false;
  for (size_t k = 0; k < F.feat.size(); k++) {
    if (F.feat[k] >= 0) tabs[F.feat[k]].push_back(F.thr[k]);
    else if (std::fpclassify(F.val[k]) == FP_SUBNORMAL) sub_leaf = true;
  }
  for (auto& v : tabs) {
    std::sort(v.begin(), v.end(), [](float p, float q) { return p < q; });
    v.erase(std::unique(v.begin(), v.end(), [](float p, float q) { return p == q; }), v.end());
  }
  // Wide codes (reading R8): rows of more than 127 attributes, coded as u8 over virtual attributes
  // and staged in shared memory next to slices packed for the room the code-tile ring leaves.
  std::vector<int32_t> vbase(F.n_features + 1, 0);
  if (max_smem > 0 && S.fbits > kCodeMaxFbits && F.agg != TAHOE_AGG_VOTE && !sub_leaf) {
    for (int32_t a = 0; a < F.n_features; a++)
      vbase[a + 1] = vbase[a] + ((int32_t)tabs[a].size() + kCode8MaxRank - 1) / kCode8MaxRank;
    const int32_t nv = vbase[F.n_features];
    const int32_t vfb = std::max(5, feature_bits(nv + 1));   // byte 2^V - 1 is the pad a leaf reads
    if (vfb <= kCode8MaxFbits) {
      const int64_t room = (int64_t)max_smem - code8_ring_smem(vfb);
      const int32_t cap8 = (int32_t)std::max<int64_t>(0, (room & ~1023LL) / kSlotBytes);
      bool fits = cap8 >= 16;
      // offsets within a tree (right child, next root) stay below the tree's size; the code word
      // keeps 32 - (V + 1) bits of byte offset (slots of 128 bytes)
      const int32_t off8 = 1 << std::min(30, 32 - (vfb + 1) - 7);
      for (int32_t t = 0; t < F.n_trees && fits; t++) fits = enc_size(F, t) <= cap8 - 1 && enc_size(F, t) < off8;
      if (fits) {
        S.code8 = true;
        S.vfbits = vfb;
        S.n_virtual = nv;
        cap = std::min(cap, cap8);
      }
    }
  }
  cap -= 1;                                    // one terminal slot per lane column
  if (F.agg == TAHOE_AGG_VOTE) { S.why_invalid = "VOTE runs on the direct strategy"; return TAHOE_OK; }
  if (cap < 1) { S.why_invalid = "no shared memory budget"; return TAHOE_OK; }
  // a node word keeps 32 - (F + 3) bits of byte offset (slots of 128 bytes); offsets within a tree
  // (right child, next tree root) stay below the tree's size
  const int64_t off_slots = (int64_t)1 << std::max(0, 32 - (S.fbits + 3) - 7);
  for (int32_t t = 0; t < F.n_trees; t++) {
    if (enc_size(F, t) > cap) { S.why_invalid = "a tree exceeds one lane column of shared memory"; return TAHOE_OK; }
    if (enc_size(F, t) >= off_slots) { S.why_invalid = "a tree is too large for the node word's offset field"; return TAHOE_OK; }
  }

  int64_t m = 0;
  const std::vector<int32_t> reads = sim_reads(F, m);
  static const char* pack_mode = std::getenv("TAHOE_PACK");          // experiments: fixed packer
  const bool refine = m >= 16 && F.opts.tree_group != 0 && !pack_mode &&
                      !(std::getenv("TAHOE_PACK_REFINE") && std::string(std::getenv("TAHOE_PACK_REFINE")) == "0");
  std::vector<std::vector<int32_t>> groups(F.n_classes);
  for (int32_t t : F.order) groups[F.tclass[t]].push_back(t);
  std::vector<Pack> packs;
  for (int32_t c = 0; c < F.n_classes; c++) {
    const auto& G = groups[c];
    if (G.empty()) continue;
    int64_t total = 0;
    for (int32_t t : G) total += enc_size(F, t);
    int32_t k = (int32_t)std::max<int64_t>(1, (int64_t)std::ceil((double)total / ((double)kSlicedCols * cap * 0.97)));
    // experiment ($TAHOE_SLICES_TARGET, single-class forests): at least this many slices, cut by
    // expected work, so an SM count divisible by the slice count gives every slice the same CTAs
    static const int32_t k_target = std::getenv("TAHOE_SLICES_TARGET") ? std::atoi(std::getenv("TAHOE_SLICES_TARGET")) : 0;
    const bool by_work = F.n_classes == 1 && k_target > k && !F.exp_reads.empty();
    if (by_work) k = k_target;
    auto weight = [&](int32_t t) -> double { return by_work ? F.exp_reads[t] : (double)enc_size(F, t); };
    double wtotal = 0;
    for (int32_t t : G) wtotal += weight(t);
    for (;; k++) {
      if (k > (int32_t)G.size()) { S.why_invalid = "cannot pack trees into slices"; return TAHOE_OK; }
      // k contiguous chunks of balanced node counts (each non-empty)
      std::vector<size_t> cut((size_t)k + 1, 0);
      cut[k] = G.size();
      {
        size_t pos = 0;
        double acc = 0;
        for (int32_t j = 1; j < k; j++) {
          const double target = wtotal * j / k;
          while (pos < G.size() && acc < target) acc += weight(G[pos++]);
          cut[j] = std::min(std::max(pos, cut[j - 1] + 1), G.size() - (size_t)(k - j));
          pos = cut[j];
          acc = 0;
          for (size_t q = 0; q < pos; q++) acc += weight(G[q]);
        }
      }
      std::vector<Pack> ps;
      bool ok = true;
      // chunks left to right; a chunk that does not pack hands up to kRecut of its last trees to the
      // next chunk before k is raised (a similarity order can cluster large trees at a cut): C4
      // (the bench's calibration) 33 -> 30 slices, simulated lockstep 0.638 -> 0.681, walk
      // 5.18 -> 5.09 ms
      constexpr size_t kRecut = 64;
      // one left-to-right pass over `order`; refinement only once a whole pass packs
      auto pass = [&](const std::vector<int32_t>& order, std::vector<Pack>& out,
                      std::vector<int32_t>& nt) -> bool {
        out.clear();
        nt.clear();
        size_t start = 0;
        for (int32_t j = 0; j < k; j++) {
          // this chunk's share of what is left (re-balanced after a chunk handed trees on)
          size_t end0 = order.size();
          if (j < k - 1) {
            double rest = 0.0;
            for (size_t q = start; q < order.size(); q++) rest += weight(order[q]);
            const double target = rest / (double)(k - j);
            double acc = 0.0;
            end0 = start;
            while (end0 < order.size() && acc < target) acc += weight(order[end0++]);
            end0 = std::max(end0, start + 1);
          }
          if (end0 > order.size() || order.size() - end0 < (size_t)(k - 1 - j)) return false;
          Pack P;
          bool packed = false;
          size_t end = end0;
          for (; end > start; end--) {
            std::vector<int32_t> chunk(order.begin() + start, order.begin() + end);
            if (pack_best(F, chunk, cap, P)) { packed = true; break; }
            if (j == k - 1 || end0 - end >= kRecut) break;   // the last chunk cannot hand trees on
          }
          if (!packed) return false;
          out.push_back(P);
          nt.push_back((int32_t)(end - start));
          start = end;
        }
        return true;
      };
      // left to right, then (a failing cut may sit at the other end) right to left
      std::vector<int32_t> nt;
      ok = pass(G, ps, nt);
      if (!ok) {
        std::vector<int32_t> R(G.rbegin(), G.rend());
        ok = pass(R, ps, nt);
      }
      if (ok) {
        for (size_t q = 0; q < ps.size(); q++) {
          if (refine) pack_refine(F, reads, m, cap, ps[q]);
          S.cls.push_back(c);
          S.ntrees.push_back(nt[q]);
        }
      }
      if (ok) { packs.insert(packs.end(), ps.begin(), ps.end()); break; }
      S.cls.resize(packs.size());
      S.ntrees.resize(packs.size());
    }
  }
  S.n_slices = (int32_t)packs.size();
  S.slots_max = 0;
  double work = 0, padded = 0;
  for (auto& P : packs) {
    P.max_len += 1;  // terminal slot
    S.slots_max = std::max(S.slots_max, P.max_len);
    work += P.sum_work;
    padded += (double)kSlicedCols * P.max_work;
  }
  S.eff = padded > 0 ? work / padded : 0;
  // Simulated lockstep efficiency of k_sliced (two rows per warp, two steps per exit test) on the
  // kept calibration rows: useful node reads / lane-steps issued.  Falls back to 0.75 x expected.
  S.eff_sim = S.eff * 0.75;
  // per-slice work (issued lane-steps per row): shares the GPU's CTAs out among the slices
  S.slice_work.assign(packs.size(), 0.0);
  for (size_t s = 0; s < packs.size(); s++) S.slice_work[s] = std::max(1e-9, packs[s].max_work * (double)kSlicedCols);
  if (m > 0) {
    // a warp walks 4 rows at once (2 per half-warp x 2 chains); its loop runs until the slowest
    // of the 64 (row, column) walks ends, two steps per exit test
    double useful = 0, issued = 0;
    for (size_t s = 0; s < packs.size(); s++) {
      auto& P = packs[s];
      double issued_s = 0;
      for (int64_t r = 0; r + 3 < m; r += 4) {
        double mx = 0;
        for (int64_t q = r; q < r + 4; q++)
          for (int32_t l = 0; l < kSlicedCols; l++) {
            double w = 0;
            for (int32_t t : P.lanes[l]) w += reads[(size_t)q * F.n_trees + t];
            useful += w;
            mx = std::max(mx, w);
          }
        issued_s += 64.0 * 2.0 * std::ceil(mx / 2.0);
      }
      issued += issued_s;
      if (issued_s > 0) S.slice_work[s] = issued_s / (double)(m / 4 * 4);
    }
    if (issued > 0) S.eff_sim = useful / issued;
  }
  S.trees_per_lane = (double)F.n_trees / ((double)kSlicedCols * std::max(1, S.n_slices));
  // Sliced node words (kernels.hpp "sliced encoding"): left child first, right child at +off,
  // leaves carry the all-ones attribute field and the delta to the lane's next tree root; one
  // self-looping terminal leaf (value 0.0, delta 0) closes every lane column.
  const uint32_t fmask = (1u << S.fbits) - 1u;
  const int32_t C = kSlicedCols;
  const int32_t sb = 7;                                  // log2(kSlotBytes): offsets stored in bytes
  static_assert(kSlotBytes == 128, "slot row is 128 bytes");
  const uint32_t off_lim = 1u << (32 - (S.fbits + 3) - sb);
  const size_t per_slice = (size_t)S.slots_max * C;
  // Rank codes (reading R7): per attribute the sorted distinct thresholds (IEEE equality, so -0.0
  // and +0.0 are one value); a node's threshold b = tab[j] is stored as t = j + 1, and
  // x < b  <=>  #{k : tab[k] <= x} < j + 1, exactly.  Requires F <= 7 (rows of <= 128 u16 codes),
  // at most kCodeMaxRank distinct thresholds per attribute, and no subnormal leaf value (the
  // kernel adds internal words, which are subnormal as floats, with flush-to-zero).
  S.code_valid = true;
  S.code_why.clear();
  if (sub_leaf) { S.code_valid = false; S.code_why = "subnormal leaf value"; }
  else if (S.code8) {
    // reading R8: virtual attribute vbase[a] + k codes thresholds tab_a[127k .. 127k + 126]
    std::vector<std::vector<float>> vt((size_t)S.n_virtual);
    S.v_src.assign((size_t)1 << S.vfbits, -1);
    S.thr_off.assign(S.n_virtual + 1, 0);
    for (int32_t a = 0; a < F.n_features; a++)
      for (int32_t v = vbase[a]; v < vbase[a + 1]; v++) {
        const size_t i0 = (size_t)(v - vbase[a]) * kCode8MaxRank;
        const size_t i1 = std::min(tabs[a].size(), i0 + kCode8MaxRank);
        vt[v].assign(tabs[a].begin() + i0, tabs[a].begin() + i1);
        S.v_src[v] = a;
      }
    for (int32_t v = 0; v < S.n_virtual; v++) S.thr_off[v + 1] = S.thr_off[v] + (int32_t)vt[v].size();
    for (auto& v : vt) S.thr_tab.insert(S.thr_tab.end(), v.begin(), v.end());
    build_code8_banks(vt, S.vfbits, S);
  } else if (S.fbits > kCodeMaxFbits) {
    S.code_valid = false;
    S.code_why = "too many attributes for u16 code rows (and no room for wide code tiles)";
  } else {
    S.thr_off.assign(F.n_features + 1, 0);
    for (int32_t a = 0; a < F.n_features && S.code_valid; a++) {
      if ((int32_t)tabs[a].size() > kCodeMaxRank) { S.code_valid = false; S.code_why = "too many distinct thresholds for one attribute"; }
      S.thr_off[a + 1] = S.thr_off[a] + (int32_t)tabs[a].size();
    }
    if (S.code_valid) {
      S.thr_tab.reserve(S.thr_off[F.n_features]);
      for (auto& v : tabs) S.thr_tab.insert(S.thr_tab.end(), v.begin(), v.end());
      S.code_slot = code_slots(F, S.fbits);
      build_code_banks(tabs, S.fbits, S.code_slot, S);
      // the fallback pre-pass (k_encode_rows) writes attribute j at slot j
      if (S.cb_passes == 0) std::iota(S.code_slot.begin(), S.code_slot.end(), 0);
      S.slot_attr.assign((size_t)1 << S.fbits, -1);
      for (int32_t a = 0; a < F.n_features; a++) S.slot_attr[S.code_slot[a]] = a;
    }
  }
  auto index_of = [&](int32_t a, float b) -> uint32_t {   // j: b == tab_a[j]
    const auto& v = tabs[a];
    return (uint32_t)(std::lower_bound(v.begin(), v.end(), b, [](float p, float q) { return p < q; }) - v.begin());
  };
  auto rank_of = [&](int32_t a, float b) -> uint32_t {   // t = j + 1 (R8: within the piece)
    const uint32_t j = index_of(a, b);
    return S.code8 ? j % (uint32_t)kCode8MaxRank + 1u : j + 1u;
  };
  auto code_attr = [&](int32_t a, float b) -> uint32_t {   // attribute field of a code word
    return S.code8 ? (uint32_t)vbase[a] + index_of(a, b) / (uint32_t)kCode8MaxRank : (uint32_t)S.code_slot[a] << 1;
  };
  // code words: R7 off_bytes << (F+2) | dl << (F+1) | attribute << 1;
  //             R8 off_bytes << (V+1) | dl << V | virtual attribute
  const int32_t csh = S.code8 ? S.vfbits + 1 : S.fbits + 2;
  const uint32_t cdl = S.code8 ? 1u << S.vfbits : 1u << (S.fbits + 1);
  const uint32_t cleaf = S.code8 ? (1u << S.vfbits) - 1u : fmask << 1;

  S.nodes.assign((size_t)S.n_slices * per_slice * 2, 0);
  if (S.code_valid) S.cnodes.assign((size_t)S.n_slices * per_slice * 2, 0);
  S.leaf_meta.assign((size_t)S.n_slices * per_slice * 2, -1);
  S.col_len.assign((size_t)S.n_slices * C, 0);
  S.col_mid.assign((size_t)S.n_slices * C, 0);
  S.slots.assign(S.n_slices, 0);
  std::vector<int32_t> slot(F.feat.size(), -1);
  std::vector<int32_t> pre, st;
  for (int32_t s = 0; s < S.n_slices; s++) {
    const Pack& P = packs[s];
    S.slots[s] = P.max_len;
    for (int32_t l = 0; l < C; l++) {
      int32_t pos = 0;
      const auto& L = P.lanes[l];
      std::vector<int32_t> root_pos;   // slot of each tree's root in this column
      for (size_t ti = 0; ti < L.size(); ti++) {
        const int32_t t = L[ti];
        root_pos.push_back(pos);
        if (F.tree_size(t) == 1) {  // 3-node stump: root (attribute 0, +2 slots right) + 2 leaves
          const int32_t k = F.node_base[t];
          const uint32_t ynode = (2u << sb) << (S.fbits + 3);
          const uint32_t yleaf1 = (2u << sb) << (S.fbits + 3) | (fmask << 2);
          const uint32_t yleaf2 = (1u << sb) << (S.fbits + 3) | (fmask << 2);
          const uint32_t ys[3] = {ynode, yleaf1, yleaf2};
          const uint32_t cys[3] = {(2u << sb) << csh, (2u << sb) << csh | cleaf,
                                   (1u << sb) << csh | cleaf};
          for (int32_t q = 0; q < 3; q++) {
            const size_t w = ((size_t)s * per_slice + (size_t)(pos + q) * C + l);
            S.nodes[2 * w] = q == 0 ? 0u : f2u(F.val[k]);
            S.nodes[2 * w + 1] = ys[q];
            if (S.code_valid) {   // stump root: both children hold the same leaf, any rank will do
              S.cnodes[2 * w] = q == 0 ? 1u : f2u(F.val[k]);
              S.cnodes[2 * w + 1] = cys[q];
            }
            if (q > 0) { S.leaf_meta[2 * w] = F.tree_orig[t]; S.leaf_meta[2 * w + 1] = F.orig[k]; }
          }
          pos += 3;
          continue;
        }
        pre.clear();
        st.assign(1, F.node_base[t]);
        while (!st.empty()) {  // preorder, left child first
          int32_t k = st.back(); st.pop_back();
          pre.push_back(k);
          if (F.feat[k] >= 0) { st.push_back(F.rc[k]); st.push_back(F.lc[k]); }
        }
        for (size_t i = 0; i < pre.size(); i++) slot[pre[i]] = pos + (int32_t)i;
        const int32_t next_root = pos + (int32_t)pre.size();
        for (size_t i = 0; i < pre.size(); i++) {
          const int32_t k = pre[i];
          const int32_t sl = pos + (int32_t)i;
          const size_t w = ((size_t)s * per_slice + (size_t)sl * C + l);
          uint32_t y, cy;
          if (F.feat[k] < 0) {
            if ((uint32_t)(next_root - sl) >= off_lim) return fail(TAHOE_E_UNSUPPORTED, "leaf offset overflow");
            y = ((uint32_t)(next_root - sl) << (S.fbits + 3 + sb)) | (fmask << 2);
            cy = ((uint32_t)(next_root - sl) << (csh + sb)) | cleaf;
            S.nodes[2 * w] = f2u(F.val[k]);
            if (S.code_valid) S.cnodes[2 * w] = f2u(F.val[k]);
            S.leaf_meta[2 * w] = F.tree_orig[t];
            S.leaf_meta[2 * w + 1] = F.orig[k];
          } else {
            if (slot[F.lc[k]] != sl + 1) return fail(TAHOE_E_INVAL, "internal: left child not adjacent");
            const int32_t delta = slot[F.rc[k]] - sl;   // in slots; stored as bytes
            if (delta <= 0 || (uint32_t)delta >= off_lim) return fail(TAHOE_E_UNSUPPORTED, "right offset overflow");
            y = ((uint32_t)delta << (S.fbits + 3 + sb)) | ((F.dl[k] ? 1u : 0u) << (S.fbits + 2)) |
                ((uint32_t)F.feat[k] << 2);
            cy = ((uint32_t)delta << (csh + sb)) | (F.dl[k] ? cdl : 0u) |
                 (S.code_valid ? code_attr(F.feat[k], F.thr[k]) : 0u);
            S.nodes[2 * w] = f2u(F.thr[k]);
            if (S.code_valid) S.cnodes[2 * w] = rank_of(F.feat[k], F.thr[k]);
          }
          S.nodes[2 * w + 1] = y;
          if (S.code_valid) S.cnodes[2 * w + 1] = cy;
        }
        pos = next_root;
      }
      // terminal self-loop
      const size_t w = ((size_t)s * per_slice + (size_t)pos * C + l);
      S.nodes[2 * w] = 0u;
      S.nodes[2 * w + 1] = fmask << 2;
      if (S.code_valid) { S.cnodes[2 * w] = 0u; S.cnodes[2 * w + 1] = cleaf; }
      S.col_len[(size_t)s * C + l] = pos;
      // the column's split point for two chains per row (wide codes): the tree root that best
      // halves the column's expected work (no split: the terminal slot, the second chain idles)
      {
        double total = 0.0, pre = 0.0, best = 1e300;
        for (int32_t t : L) total += F.exp_reads[t];
        int32_t mid = pos;
        for (size_t ti = 0; ti < L.size(); ti++) {
          if (ti > 0 && std::max(pre, total - pre) < best) { best = std::max(pre, total - pre); mid = root_pos[ti]; }
          pre += F.exp_reads[L[ti]];
        }
        S.col_mid[(size_t)s * C + l] = mid;
      }
    }
  }
  // class -> slices (in slice order: the fixed fp64 summation order of the finalize step)
  S.class_ptr.assign(F.n_classes + 1, 0);
  for (int32_t s = 0; s < S.n_slices; s++) S.class_ptr[S.cls[s] + 1]++;
  for (int32_t c = 0; c < F.n_classes; c++) S.class_ptr[c + 1] += S.class_ptr[c];
  S.class_parts.assign(S.n_slices, 0);
  std::vector<int32_t> fillp(S.class_ptr.begin(), S.class_ptr.end() - 1);
  for (int32_t s = 0; s < S.n_slices; s++) S.class_parts[fillp[S.cls[s]]++] = s;
  S.valid = true;
  return TAHOE_OK;
}

}  // namespace tahoe
