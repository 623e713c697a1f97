// planner.hpp — tile-size search and cost models of libtc.
//
// Structure follows Section IV of the paper: enumerate mapping / tile-size choices per side
// (Alg. 2), take the Cartesian product of the partial configs,
// prune by hardware and performance constraints, rank by a cost model
// (P:L296-324).  Two cost models:
//   * TC_COST_PAPER — Alg. 3 verbatim (128-B transactions) with the paper's V100
//     value sets {4,8,16} / {2,4,6,8}; the chosen tiles then run on the B200 kernel.
//   * TC_COST_B200  — re-derived for B200: per-SM FP64-pipe and shared-memory
//     cycles of the PADDED work (bank conflicts simulated on the real slot tables), wave
//     quantisation over 148 SMs, 32-B sector traffic at L2 and HBM, L2 reuse.
#pragma once
#include <map>
#include <string>
#include <vector>

#include "contraction.hpp"
#include "tiles.hpp"

namespace tc {

struct PlanStats {
  int64_t raw = 0;       // configurations enumerated
  int64_t pruned = 0;    // removed by the constraints
  int64_t ranked = 0;    // cost-model evaluations
  double plan_ms = 0;
  int cost_mode = 0;
  // best predicted time per kernel variant (variant id, seconds), ascending: the candidate
  // set of measured tuning (tc_plan_tuned; the paper's "auto-tuned across a selected set",
  // P:L346-348)
  std::vector<std::pair<int, double>> per_variant;
};

struct ForcedTiles {
  bool on = false;
  std::map<std::string, int> tile;  // by index name
  int morder = -1;                  // >= 0: only this m digit order (tests of both epilogues)
};

// Choose a configuration.  forced_variant < 0: planner's choice.
Status choose(const Contraction &c, int kind, int cost_mode, int forced_variant, const ForcedTiles &ft,
              Config &out, PlanStats &stats, std::string &err);

// B200 model (seconds); fills cfg's model outputs.
using WfCache = std::map<std::vector<int64_t>, std::pair<double, double>>;
// Does the configuration fit the kernel variant (tile extents, grid limits)?
bool config_fits(const Config &cfg, const Variant &v);
double model_time(const Contraction &c, Config &cfg, const Variant &v, WfCache *cache = nullptr,
                  bool lower_bound = false);   // lower_bound: ideal smem / sector terms, no simulation
double paper_alg3_cost(const Contraction &c, const Config &cfg, const std::vector<int> &tbx,
                       const std::vector<int> &regx, const std::vector<int> &tby,
                       const std::vector<int> &regy);
// Contiguous run (elements) of tensor t's tile along its memory order (cal_Cont).
int64_t contiguous_run(const Contraction &c, int t, const std::vector<int> &T);

}  // namespace tc
