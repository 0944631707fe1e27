// costmodel.cpp — per-batch strategy choice (Algorithm 1 lines 8-13; Eq. 1-7
// reconstructed in SURVEY Appendix A), re-targeted to the two B200 strategies.
//
// Per-sample time (Eq. 1: T = T_SMEM + T_GMEM + T_B_REDU + T_G_REDU) becomes
//   direct : V * c_gmem_visit                                   (T_GMEM: nodes + attributes from
//                                                                 L1/L2, no reduction)
//   sliced : V * c_smem_visit / eff  + P * (c_reduce + 4 d / BW) (T_SMEM of a lockstep warp at
//                                                                 packing efficiency eff, plus one
//                                                                 warp reduction and one row read
//                                                                 per slice P: T_B_REDU + T_G_REDU)
// V = expected node reads per sample (calibrated E[path]+1 summed over trees, reading Z16).
// Constants are in units of one conflict-free shared-memory node visit; they can be overridden by
// TAHOE_COST_GMEM / TAHOE_COST_REDUCE / TAHOE_COST_ROWBYTE (fitted on the chip).
#include <cstdlib>

#include "internal.hpp"

namespace tahoe {

static double env_or(const char* name, double dflt) {
  const char* v = std::getenv(name);
  return (v && *v) ? std::atof(v) : dflt;
}

int32_t select_strategy(const PlanStats& st, int64_t n, int32_t d, int32_t agg) {
  if (agg == TAHOE_AGG_VOTE || !st.sliced_ok) return TAHOE_STRATEGY_DIRECT;
  const double c_gmem = env_or("TAHOE_COST_GMEM", 4.0);
  const double c_reduce = env_or("TAHOE_COST_REDUCE", 24.0);
  const double c_rowbyte = env_or("TAHOE_COST_ROWBYTE", 0.02);
  const double eff = st.sliced_eff > 0.05 ? st.sliced_eff : 0.05;
  const double t_direct = st.V * c_gmem;
  const double t_sliced = st.V / eff + st.n_slices * (c_reduce + c_rowbyte * 4.0 * d);
  (void)n;
  return t_sliced <= t_direct ? TAHOE_STRATEGY_SLICED : TAHOE_STRATEGY_DIRECT;
}

}  // namespace tahoe
