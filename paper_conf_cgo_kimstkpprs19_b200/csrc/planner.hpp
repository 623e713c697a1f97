// planner.hpp — tile-size search and cost models of libtc.
//
// Structure follows Section IV of the paper: enumerate mapping / tile-size choices per side
// (Alg. 2), take the Cartesian product of the partial configs,
// prune by hardware and performance constraints, rank by a cost model
// (P:L296-324).  Two cost models:
//   * TC_COST_PAPER — Alg. 3 verbatim (128-B transactions) with the paper's V100
//     value sets {4,8,16} / {2,4,6,8}; the chosen tiles then run on the B200 kernel.
//   * TC_COST_B200  — re-derived for B200: FP64-pipe time of the PADDED
//     work with wave quantisation over 148 SMs, 32-B-sector traffic at L2 and HBM, L2 reuse,
//     exposed epilogue stores.  Constants measured in profiles/r01_peaks.json.
#pragma once
#include <map>
#include <string>
#include <vector>

#include "contraction.hpp"

namespace tc {

// Compiled kernel shapes (kernel_f64.cuh template instances).
struct Variant {
  int BM, BN, BK, WM, WN, stages, threads, occ;
};
const std::vector<Variant> &variants();

struct Config {
  int variant = -1;
  int X = 1, Y = 2;                 // tensor ids (1 = A, 2 = B) on the M / N side
  std::vector<int> mdig, ndig, kdig;  // index ids, compute order
  std::vector<int> T;               // tile per index id (size = nidx)
  // model outputs
  double t_pred = 0, t_comp = 0, t_mem = 0, t_l2 = 0, dram_bytes = 0, flops_pad = 0;
  double paper_cost = 0;            // Alg. 3 transactions (paper mode)
  int64_t nctas = 0, nsteps = 0;
  int64_t Mt = 1, Nt = 1, Kt = 1;
  // paper-mode mapping (Table II): which indices went to TB_x / REG_x / TB_y / REG_y / TB_k
  std::string paper_mapping;
};

struct PlanStats {
  int64_t raw = 0;       // configurations enumerated
  int64_t pruned = 0;    // removed by the constraints
  int64_t ranked = 0;    // cost-model evaluations
  double plan_ms = 0;
  int cost_mode = 0;
};

struct ForcedTiles {
  bool on = false;
  std::map<std::string, int> tile;  // by index name (pre-fusion names only)
};

// Choose a configuration.  forced_variant < 0: planner's choice.
Status choose(const Contraction &c, int cost_mode, int forced_variant, const ForcedTiles &ft,
              Config &out, PlanStats &stats, std::string &err);

// Helpers exposed for plan metadata / info.
int x_tensor(const Contraction &c);  // 1 or 2
double model_time(const Contraction &c, const Config &cfg, const Variant &v, double *comp,
                  double *mem, double *l2, double *dram);
double paper_alg3_cost(const Contraction &c, const Config &cfg, const std::vector<int> &tbx,
                       const std::vector<int> &regx, const std::vector<int> &tby,
                       const std::vector<int> &regy);
// Contiguous run (elements) of tensor t's tile along its memory order (cal_Cont).
int64_t contiguous_run(const Contraction &c, int t, const std::vector<int> &T);

}  // namespace tc
