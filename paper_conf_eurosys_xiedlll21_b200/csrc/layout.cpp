// layout.cpp — tahoe_forest_layout's host steps (Algorithm 1 lines 5-6):
//   calibrate      edge / node probability from visit counts on calibration rows
//   reorder_nodes  probability-based node rearrangement: hot child next to its parent
//   tree_tokens    tokenization of root->leaf paths into T_nodes windows
//   tree_simhash   SHA1 strings weighted by node probability, summed, normalised
//   lsh_order      M chunks, Rabin-Karp keys, collision counts, greedy placement
// Readings Z5-Z11 of DESIGN.md fix the details the paper leaves open.
#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstring>
#include <numeric>
#include <thread>
#include <unordered_map>

#include "internal.hpp"

namespace tahoe {

static int host_threads() {
  unsigned h = std::thread::hardware_concurrency();
  return (int)std::max(1u, std::min(h, 64u));
}

template <class Fn>
static void parallel_for(int64_t n, Fn fn) {
  int nt = (int)std::min<int64_t>(host_threads(), std::max<int64_t>(1, n));
  if (nt <= 1) { for (int64_t i = 0; i < n; i++) fn(i); return; }
  std::vector<std::thread> th;
  std::atomic<int64_t> next{0};
  for (int w = 0; w < nt; w++)
    th.emplace_back([&] {
      for (;;) {
        int64_t i = next.fetch_add(1);
        if (i >= n) break;
        fn(i);
      }
    });
  for (auto& x : th) x.join();
}

// ---------------------------------------------------------------- calibration
void calibrate(Forest& F, const float* X, int64_t n, int32_t d) {
  F.count.assign(F.feat.size(), 0);
  parallel_for(F.n_trees, [&](int64_t t) {
    const int32_t r = F.node_base[t];
    for (int64_t i = 0; i < n; i++) {
      const float* x = X + i * d;
      int32_t k = r;
      F.count[k]++;
      while (F.feat[k] >= 0) {
        float v = x[F.feat[k]];
        bool left = std::isnan(v) ? (F.dl[k] != 0) : (v < F.thr[k]);
        k = left ? F.lc[k] : F.rc[k];
        F.count[k]++;
      }
    }
  });
  F.n_cal = n;
  F.calibrated = true;
  F.exp_reads.assign(F.n_trees, 0.0);
  for (int32_t t = 0; t < F.n_trees; t++) {
    uint64_t s = 0;
    for (int32_t k = F.node_base[t]; k < F.node_base[t + 1]; k++) s += F.count[k];
    F.exp_reads[t] = n ? (double)s / (double)n : 0.0;
  }
}

// Counts measured elsewhere (the GPU visit counter, Algorithm 1 line 16), indexed by caller node id.
void set_counts(Forest& F, const uint64_t* counts, int64_t n) {
  F.count.assign(F.feat.size(), 0);
  for (size_t k = 0; k < F.feat.size(); k++) F.count[k] = counts[F.orig[k]];
  F.n_cal = n;
  F.calibrated = true;
  F.exp_reads.assign(F.n_trees, 0.0);
  for (int32_t t = 0; t < F.n_trees; t++) {
    uint64_t s = 0;
    for (int32_t k = F.node_base[t]; k < F.node_base[t + 1]; k++) s += F.count[k];
    F.exp_reads[t] = n ? (double)s / (double)n : 0.0;
  }
}

// ------------------------------------------------------ node rearrangement (Z5)
void reorder_nodes(Forest& F, bool enable) {
  F.hot_left.assign(F.feat.size(), 1);
  if (!enable || !F.calibrated) return;
  for (size_t k = 0; k < F.feat.size(); k++)
    if (F.feat[k] >= 0 && F.count[F.rc[k]] > F.count[F.lc[k]]) F.hot_left[k] = 0;
}

std::vector<int32_t> hot_preorder(const Forest& F, int32_t t) {
  std::vector<int32_t> out, st(1, F.node_base[t]);
  out.reserve(F.tree_size(t));
  while (!st.empty()) {
    int32_t k = st.back(); st.pop_back();
    out.push_back(k);
    if (F.feat[k] >= 0) {
      int32_t hot = F.hot_left[k] ? F.lc[k] : F.rc[k];
      int32_t cold = F.hot_left[k] ? F.rc[k] : F.lc[k];
      st.push_back(cold);
      st.push_back(hot);
    }
  }
  return out;
}

// ------------------------------------------------------------------ SHA1 (FIPS 180-4)
static inline uint32_t rol(uint32_t x, int k) { return (x << k) | (x >> (32 - k)); }
void sha1(const uint8_t* msg, size_t len, uint8_t out[20]) {
  uint32_t h[5] = {0x67452301u, 0xEFCDAB89u, 0x98BADCFEu, 0x10325476u, 0xC3D2E1F0u};
  const uint64_t bitlen = (uint64_t)len * 8;
  size_t total = ((len + 9 + 63) / 64) * 64;
  std::vector<uint8_t> buf(total, 0);
  if (len) std::memcpy(buf.data(), msg, len);
  buf[len] = 0x80;
  for (int i = 0; i < 8; i++) buf[total - 1 - i] = (uint8_t)(bitlen >> (8 * i));
  uint32_t w[80];
  for (size_t off = 0; off < total; off += 64) {
    for (int i = 0; i < 16; i++)
      w[i] = ((uint32_t)buf[off + 4 * i] << 24) | ((uint32_t)buf[off + 4 * i + 1] << 16) |
             ((uint32_t)buf[off + 4 * i + 2] << 8) | (uint32_t)buf[off + 4 * i + 3];
    for (int i = 16; i < 80; i++) w[i] = rol(w[i - 3] ^ w[i - 8] ^ w[i - 14] ^ w[i - 16], 1);
    uint32_t a = h[0], b = h[1], c = h[2], d = h[3], e = h[4];
    for (int i = 0; i < 80; i++) {
      uint32_t f, k;
      if (i < 20) { f = (b & c) | (~b & d); k = 0x5A827999u; }
      else if (i < 40) { f = b ^ c ^ d; k = 0x6ED9EBA1u; }
      else if (i < 60) { f = (b & c) | (b & d) | (c & d); k = 0x8F1BBCDCu; }
      else { f = b ^ c ^ d; k = 0xCA62C1D6u; }
      uint32_t tmp = rol(a, 5) + f + e + k + w[i];
      e = d; d = c; c = rol(b, 30); b = a; a = tmp;
    }
    h[0] += a; h[1] += b; h[2] += c; h[3] += d; h[4] += e;
  }
  for (int i = 0; i < 5; i++)
    for (int j = 0; j < 4; j++) out[4 * i + j] = (uint8_t)(h[i] >> (24 - 8 * j));
}

// ------------------------------------------------------------ tokenization (Z6)
// A window of T_nodes consecutive nodes on a root->leaf path is determined by its last node, so
// the distinct windows are: one per node of depth >= T_nodes-1, plus every whole path shorter
// than T_nodes.  Tokens are ordered by their last node in hot-first preorder.
void tree_tokens(const Forest& F, int32_t t, int32_t t_nodes, std::vector<int32_t>& tok_nodes,
                 std::vector<double>& weights) {
  tok_nodes.clear();
  weights.clear();
  std::vector<int32_t> parent(F.tree_size(t), -1);
  const int32_t b = F.node_base[t];
  for (int32_t k = b; k < F.node_base[t + 1]; k++)
    if (F.feat[k] >= 0) { parent[F.lc[k] - b] = k; parent[F.rc[k] - b] = k; }
  const double ncal = F.n_cal ? (double)F.n_cal : 0.0;
  std::vector<int32_t> win;
  for (int32_t k : hot_preorder(F, t)) {
    const bool full = F.depth[k] >= t_nodes - 1;
    const bool short_path = F.feat[k] < 0 && F.depth[k] < t_nodes - 1;
    if (!full && !short_path) continue;
    win.clear();
    for (int32_t v = k; v >= 0 && (int32_t)win.size() < t_nodes; v = parent[v - b]) win.push_back(v);
    std::reverse(win.begin(), win.end());
    for (int32_t i = 0; i < t_nodes; i++) tok_nodes.push_back(i < (int32_t)win.size() ? win[i] : -1);
    // weight: node probability of the token's last node; before calibration use the
    // 50/50 prior 2^-depth
    weights.push_back(ncal > 0 ? (double)F.count[k] / ncal : std::ldexp(1.0, -F.depth[k]));
  }
}

// token bytes (Z6): per node u16 LE attribute index (0xFFFF leaf) + step byte to the next node of
// the token (0 original left child, 1 original right child, 0xFF last node)
static void token_bytes(const Forest& F, const int32_t* tok, int32_t t_nodes, std::vector<uint8_t>& out) {
  out.clear();
  int32_t len = 0;
  while (len < t_nodes && tok[len] >= 0) len++;
  for (int32_t i = 0; i < len; i++) {
    int32_t k = tok[i];
    uint32_t f = F.feat[k] < 0 ? 0xFFFFu : (uint32_t)F.feat[k];
    out.push_back((uint8_t)(f & 0xFF));
    out.push_back((uint8_t)((f >> 8) & 0xFF));
    if (i + 1 < len) out.push_back(F.lc[k] == tok[i + 1] ? 0 : 1);
    else out.push_back(0xFF);
  }
}

// bits of SHA1 (Z7): first l_hash bits MSB-first; beyond 160 bits SHA1(data || u8(k)) blocks
static void token_bits(const std::vector<uint8_t>& data, int32_t l_hash, std::vector<uint8_t>& bits) {
  bits.assign(l_hash, 0);
  uint8_t dig[20];
  if (l_hash <= 160) {
    sha1(data.data(), data.size(), dig);
    for (int32_t i = 0; i < l_hash; i++) bits[i] = (dig[i >> 3] >> (7 - (i & 7))) & 1;
    return;
  }
  std::vector<uint8_t> m(data);
  m.push_back(0);
  for (int32_t blk = 0; blk * 160 < l_hash; blk++) {
    m.back() = (uint8_t)blk;
    sha1(m.data(), m.size(), dig);
    for (int32_t i = 0; i < 160 && blk * 160 + i < l_hash; i++)
      bits[blk * 160 + i] = (dig[i >> 3] >> (7 - (i & 7))) & 1;
  }
}

void simhash(const int8_t* strings, const double* w, int32_t n, int32_t l, double* cs, uint8_t* bits) {
  for (int32_t j = 0; j < l; j++) cs[j] = 0.0;
  for (int32_t i = 0; i < n; i++)
    for (int32_t j = 0; j < l; j++) cs[j] += w[i] * (double)strings[(int64_t)i * l + j];
  for (int32_t j = 0; j < l; j++) bits[j] = cs[j] >= 0.0 ? 1 : 0;   // P:788-791, Z9
}

void tree_simhash(const Forest& F, int32_t t, int32_t t_nodes, int32_t l_hash,
                  std::vector<double>& checksum, std::vector<uint8_t>& bits) {
  std::vector<int32_t> toks;
  std::vector<double> w;
  tree_tokens(F, t, t_nodes, toks, w);
  checksum.assign(l_hash, 0.0);
  std::vector<uint8_t> data, tb;
  const int32_t nt = (int32_t)w.size();
  for (int32_t i = 0; i < nt; i++) {
    token_bytes(F, &toks[(size_t)i * t_nodes], t_nodes, data);
    token_bits(data, l_hash, tb);
    for (int32_t j = 0; j < l_hash; j++) checksum[j] += w[i] * (tb[j] ? 1.0 : -1.0);
  }
  bits.assign(l_hash, 0);
  for (int32_t j = 0; j < l_hash; j++) bits[j] = checksum[j] >= 0.0 ? 1 : 0;
}

// ----------------------------------------------------------------- LSH (Z10-Z11)
static uint64_t rabin_karp(const uint8_t* b, int32_t len) {
  const uint64_t mod = (1ull << 61) - 1, base = 257;
  uint64_t h = 0;
  for (int32_t i = 0; i < len; i++) h = (uint64_t)(((unsigned __int128)h * base + b[i] + 1) % mod);
  return h;
}

std::vector<int32_t> lsh_order(const std::vector<uint8_t>& bits, int32_t T, int32_t l_hash,
                               int32_t m_chunks, std::vector<uint16_t>* collisions) {
  const int32_t w = std::max(1, l_hash / m_chunks);
  std::vector<uint16_t> col((size_t)T * T, 0);
  std::vector<std::pair<uint64_t, int32_t>> keys(T);
  for (int32_t c = 0; c < m_chunks; c++) {
    for (int32_t t = 0; t < T; t++) keys[t] = {rabin_karp(&bits[(size_t)t * l_hash + c * w], w), t};
    std::sort(keys.begin(), keys.end());
    for (int32_t i = 0; i < T;) {
      int32_t j = i;
      while (j < T && keys[j].first == keys[i].first) j++;
      for (int32_t a = i; a < j; a++)
        for (int32_t b2 = a + 1; b2 < j; b2++) {
          int32_t x = keys[a].second, y = keys[b2].second;
          col[(size_t)x * T + y]++;
          col[(size_t)y * T + x]++;
        }
      i = j;
    }
  }
  // pairs by (count desc, a, b): bucket by count, each bucket filled in (a, b) order
  std::vector<std::vector<std::pair<int32_t, int32_t>>> bucket(m_chunks + 1);
  for (int32_t a = 0; a < T; a++)
    for (int32_t b2 = a + 1; b2 < T; b2++) {
      uint16_t c = col[(size_t)a * T + b2];
      if (c > 0) bucket[std::min<int32_t>(c, m_chunks)].push_back({a, b2});
    }
  // chains as paths: neighbour lists + (head, tail) per chain root; union-find for chain ids
  std::vector<int32_t> uf(T), head(T), tail(T), nb0(T, -1), nb1(T, -1);
  std::vector<int64_t> first_link(T, -1);
  std::iota(uf.begin(), uf.end(), 0);
  std::iota(head.begin(), head.end(), 0);
  std::iota(tail.begin(), tail.end(), 0);
  auto find = [&](int32_t x) { while (uf[x] != x) { uf[x] = uf[uf[x]]; x = uf[x]; } return x; };
  auto endpoint = [&](int32_t x) { return nb1[x] < 0; };
  auto link = [&](int32_t x, int32_t y) {
    (nb0[x] < 0 ? nb0[x] : nb1[x]) = y;
    (nb0[y] < 0 ? nb0[y] : nb1[y]) = x;
  };
  int64_t idx = 0;
  for (int32_t c = m_chunks; c >= 1; c--) {
    for (auto [a, b2] : bucket[c]) {
      int64_t my = idx++;
      int32_t ca = find(a), cb = find(b2);
      if (ca == cb || !endpoint(a) || !endpoint(b2)) continue;
      int32_t keep, other, x, y;
      int64_t la = first_link[ca], lb = first_link[cb];
      if (la >= 0 && (lb < 0 || la < lb)) { keep = ca; other = cb; x = a; y = b2; }
      else if (lb >= 0) { keep = cb; other = ca; x = b2; y = a; }
      else { keep = ca; other = cb; x = a; y = b2; }  // a < b2: the smaller id's chain is kept
      int32_t nh, ntl;
      if (tail[keep] == x) { nh = head[keep]; ntl = (head[other] == y) ? tail[other] : head[other]; }
      else { nh = (tail[other] == y) ? head[other] : tail[other]; ntl = tail[keep]; }
      link(x, y);
      uf[other] = keep;
      head[keep] = nh;
      tail[keep] = ntl;
      int64_t fl = my;
      if (la >= 0) fl = std::min(fl, la);
      if (lb >= 0) fl = std::min(fl, lb);
      first_link[keep] = fl;
    }
  }
  std::vector<std::pair<int64_t, int32_t>> chains;
  for (int32_t t = 0; t < T; t++)
    if (find(t) == t && first_link[t] >= 0) chains.push_back({first_link[t], t});
  std::sort(chains.begin(), chains.end());
  std::vector<int32_t> order;
  order.reserve(T);
  for (auto [fl, r] : chains) {
    (void)fl;
    int32_t prev = -1, cur = head[r];
    while (cur >= 0) {
      order.push_back(cur);
      int32_t nx = (nb0[cur] != prev) ? nb0[cur] : nb1[cur];
      if (nx == prev) nx = -1;
      prev = cur;
      cur = nx;
    }
  }
  for (int32_t t = 0; t < T; t++)
    if (find(t) == t && first_link[t] < 0) order.push_back(t);
  if (collisions) collisions->swap(col);
  return order;
}

// Similarity order of the trees of each class (trees of different classes never share a work
// unit), class-major.
void order_trees(Forest& F) {
  const tahoe_layout_opts& o = F.opts;
  std::vector<std::vector<int32_t>> by_class(F.n_classes);
  for (int32_t t = 0; t < F.n_trees; t++) by_class[F.tclass[t]].push_back(t);
  F.order.clear();
  if (!o.tree_group) {
    for (auto& v : by_class) F.order.insert(F.order.end(), v.begin(), v.end());
    return;
  }
  std::vector<std::vector<uint8_t>> tb(F.n_trees);
  parallel_for(F.n_trees, [&](int64_t t) {
    std::vector<double> cs;
    tree_simhash(F, (int32_t)t, o.t_nodes, o.l_hash, cs, tb[t]);
  });
  for (auto& v : by_class) {
    const int32_t T = (int32_t)v.size();
    if (T == 0) continue;
    std::vector<uint8_t> bits((size_t)T * o.l_hash);
    for (int32_t i = 0; i < T; i++) std::copy(tb[v[i]].begin(), tb[v[i]].end(), bits.begin() + (size_t)i * o.l_hash);
    std::vector<int32_t> ord = lsh_order(bits, T, o.l_hash, o.m_chunks, nullptr);
    for (int32_t i : ord) F.order.push_back(v[i]);
  }
}

}  // namespace tahoe
