// costmodel.cpp — per-batch strategy choice (Algorithm 1 lines 8-13; Eq. 1-7
// reconstructed in SURVEY Appendix A), re-targeted to the B200 strategies.
//
// Eq. 1 (T = T_SMEM + T_GMEM + T_B_REDU + T_G_REDU) becomes, per batch of n rows:
//   sliced : T = a_s + b_s * U_s * (rows in global memory ? g_s : 1),
//            U_s = ceil(tiles / cps) * 64 * V / (slices * eff)
//            the node reads of the busiest CTA (T_SMEM at the simulated lockstep efficiency eff);
//            a_s absorbs launch, slice staging and the fixed-order slice reduction (T_G_REDU);
//   direct : T = a_d + (d > 256 ? g_d : 1) * max(l_d * V, (tlp ? b_t : b_d) * V * n / SMs)
//            one thread per sample: latency-bound below a full GPU of threads (l_d per visit),
//            L1/L2-throughput-bound above it (T_GMEM); tlp = the staged-row kernel with eight
//            threads per row that launch_direct takes for >= 32K rows of scalar outputs;
//   coded  : T = a_c + b_c * U_s + e_c * ceil(n / 64) * 64 * passes / SMs
//            the rank-coded slices (reading R7): the same busiest-CTA node reads at a cheaper
//            per-read cost b_c, plus the row-coding pre-pass (passes of 32 attributes per row);
//   rows   : T = a_r + max(b_r * ceil(T_trees / 512) * V / T_trees, n * (c_r V + k_r C + w_r d) / SMs)
//            one CTA per sample (small batches): the chain of dependent node reads of one thread
//            (L2 latency per read) while the GPU is not full, the per-row throughput beyond (node
//            reads, the block reduction per output class, the row staging per attribute).
// V = expected node reads per sample (calibrated E[path] + 1 leaf read, summed over trees,
// reading Z16).  The constants are fitted on the chip by scripts/fit_costmodel.py and read from
// costmodel_b200.json next to libtahoe.so (or $TAHOE_COSTMODEL); defaults are round-1 B200
// measurements.
#include <dlfcn.h>

#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>

#include "internal.hpp"

namespace tahoe {

static bool read_key(const std::string& js, const char* key, double* v) {
  const std::string k = std::string("\"") + key + "\"";
  size_t p = js.find(k);
  if (p == std::string::npos) return false;
  p = js.find(':', p);
  if (p == std::string::npos) return false;
  return std::sscanf(js.c_str() + p + 1, "%lf", v) == 1;
}

static std::string lib_dir() {
  Dl_info info;
  if (dladdr(reinterpret_cast<void*>(&cost_params), &info) && info.dli_fname) {
    std::string s(info.dli_fname);
    size_t k = s.rfind('/');
    if (k != std::string::npos) return s.substr(0, k);
  }
  return ".";
}

const CostParams& cost_params() {
  static CostParams P = [] {
    CostParams c;
    const char* env = std::getenv("TAHOE_COSTMODEL");
    std::string path = env && *env ? std::string(env) : lib_dir() + "/costmodel_b200.json";
    FILE* fp = std::fopen(path.c_str(), "rb");
    if (!fp) return c;
    std::string js;
    char buf[4096];
    size_t k;
    while ((k = std::fread(buf, 1, sizeof(buf), fp)) > 0) js.append(buf, k);
    std::fclose(fp);
    double v;
    bool all = true;
    all &= read_key(js, "a_s", &v); if (all) c.a_s = v;
    all &= read_key(js, "b_s", &v); if (all) c.b_s = v;
    all &= read_key(js, "a_d", &v); if (all) c.a_d = v;
    all &= read_key(js, "l_d", &v); if (all) c.l_d = v;
    all &= read_key(js, "b_d", &v); if (all) c.b_d = v;
    if (read_key(js, "g_s", &v)) c.g_s = v;
    if (read_key(js, "g_d", &v)) c.g_d = v;
    if (read_key(js, "a_c", &v)) c.a_c = v;
    if (read_key(js, "b_c", &v)) c.b_c = v;
    if (read_key(js, "e_c", &v)) c.e_c = v;
    if (read_key(js, "a_w", &v)) c.a_w = v;
    if (read_key(js, "b_w", &v)) c.b_w = v;
    if (read_key(js, "e_w", &v)) c.e_w = v;
    if (read_key(js, "a_r", &v)) c.a_r = v;
    if (read_key(js, "b_r", &v)) c.b_r = v;
    if (read_key(js, "c_r", &v)) c.c_r = v;
    if (read_key(js, "k_r", &v)) c.k_r = v;
    if (read_key(js, "b_t", &v)) c.b_t = v;
    if (read_key(js, "w_r", &v)) c.w_r = v;
    c.fitted = all;
    return c;
  }();
  return P;
}

double predict_us(const PlanStats& st, int32_t strategy, int64_t n) {
  const CostParams& c = cost_params();
  if (strategy == TAHOE_STRATEGY_SLICED || strategy == TAHOE_STRATEGY_SLICED_CODED) {
    if (!st.sliced_ok || st.n_slices < 1) return INFINITY;
    if (strategy == TAHOE_STRATEGY_SLICED_CODED && !st.coded_ok) return INFINITY;
    const int64_t tiles = (n + 63) / 64;
    const int64_t cps = st.n_slices <= st.num_sms
                            ? std::max<int64_t>(1, std::min<int64_t>(st.num_sms / st.n_slices, tiles))
                            : 1;
    const double passes = st.n_slices <= st.num_sms ? 1.0 : std::ceil((double)st.n_slices / st.num_sms);
    const double eff = st.sliced_eff > 0.05 ? st.sliced_eff : 0.05;
    const double U = (double)((tiles + cps - 1) / cps) * 64.0 * st.V / (st.n_slices * eff) * passes;
    if (strategy == TAHOE_STRATEGY_SLICED_CODED && st.code8)
      return c.a_w + c.b_w * U + c.e_w * (double)(tiles * 64) * st.code_passes / std::max(1, st.num_sms);
    if (strategy == TAHOE_STRATEGY_SLICED_CODED)
      return c.a_c + c.b_c * U + c.e_c * (double)(tiles * 64) * st.code_passes / std::max(1, st.num_sms);
    return c.a_s + c.b_s * U * (st.rows_global ? c.g_s : 1.0);
  }
  const double sms = st.num_sms > 0 ? st.num_sms : 148;
  if (strategy == TAHOE_STRATEGY_ROWS) {
    // rows: latency-bound while the batch leaves the GPU idle (a thread's chain of ceil(T / 512)
    // trees of mean path V / T dependent node reads, b_r per read), throughput-bound beyond
    // (c_r per node read per SM)
    if (!st.rows_ok) return INFINITY;
    const double chain = std::ceil((double)st.n_trees / kRowsThreads) * st.V / std::max(1, st.n_trees);
    const double per_row = c.c_r * st.V + c.k_r * st.n_out + c.w_r * st.d;
    return c.a_r + std::max(c.b_r * chain, (double)n * per_row / sms);
  }
  const double g = st.wide_rows ? c.g_d : 1.0;
  // >= 32K rows with one output and rows of <= 256 attributes: the staged-row kernel with eight
  // threads per row (launch_direct's default), a cheaper per-read throughput b_t
  const bool tlp = n >= 32768 && st.scalar && !st.wide_rows;
  return c.a_d + g * std::max(c.l_d * st.V, (tlp ? c.b_t : c.b_d) * st.V * (double)n / sms);
}

int32_t select_strategy(const PlanStats& st, int64_t n, int32_t d, int32_t agg) {
  (void)d;
  int32_t best = TAHOE_STRATEGY_DIRECT;
  double tb = predict_us(st, TAHOE_STRATEGY_DIRECT, n);
  {
    const double t = predict_us(st, TAHOE_STRATEGY_ROWS, n);
    if (t < tb) { tb = t; best = TAHOE_STRATEGY_ROWS; }
  }
  if (agg == TAHOE_AGG_VOTE || !st.sliced_ok) return best;
  for (int32_t s : {TAHOE_STRATEGY_SLICED, TAHOE_STRATEGY_SLICED_CODED}) {
    const double t = predict_us(st, s, n);
    if (t < tb) { tb = t; best = s; }
  }
  return best;
}

}  // namespace tahoe
