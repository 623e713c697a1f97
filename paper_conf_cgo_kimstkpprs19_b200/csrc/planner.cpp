// planner.cpp — enumeration (Alg. 2 generalised), pruning and the two cost
// models (Alg. 3 verbatim, and the B200 re-derivation) of libtc.  See planner.hpp.
#include "planner.hpp"

#include <algorithm>
#include <chrono>
#include <cmath>
#include <map>
#include <set>

namespace tc {

// ---------------------------------------------------------------- hardware constants
// B200, measured (profiles/r01_peaks.json): DMMA 37.1 TFLOP/s = 148 SMs x 64 FMA/clk x 2 x
// 1.965 GHz; HBM read 7.36 TB/s, f64 write 6.7 TB/s, copy 6.55 TB/s (MEASURED_PEAKS.json).
static constexpr double kSMs = 148, kFmaPerClk = 64, kClk = 1.965e9;
// kL2Bw: effective L2->SM bandwidth of the cp.async gathers, fitted to the variant sweeps
// (tools/variant_sweep.py; profiles/r01_*): ~7 TB/s.
static constexpr double kHbm = 6.5e12, kL2Bw = 7.0e12, kL2Bytes = 126.0e6;
static constexpr double kLaunch = 3.0e-6;
static constexpr double kStepOverhead = 40;   // cycles per k-step: mbarrier hand-off

static int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }
// multiply-adds per clock per SM of the kernel family's MMA pipe: DMMA 64 (measured), BF16
// tcgen05 4096 (2.25 PFLOP/s dense nominal at 1.86 GHz; MEASURED_PEAKS.json has cuBLAS's
// sustained figure)
// TF32 half the BF16 rate; F32X3 issues three TF32 MMAs per k-step
static double fma_per_clk(int kind) {
  return kind == KIND_BF16_UMMA ? 4096.0 : kind == KIND_TF32_UMMA ? 2048.0 : kind == KIND_F32X3_UMMA ? 2048.0 / 3 : kFmaPerClk;
}

int64_t contiguous_run(const Contraction &c, int t, const std::vector<int> &T) {
  // cal_Cont: elements contiguous in memory within the tile hyper-rectangle
  int64_t run = 1, expect = 1;
  const auto &v = c.t[t];
  for (size_t k = 0; k < v.idx.size(); k++) {
    if (v.stride[k] != expect) break;       // a gap in memory (restricted views)
    int id = v.idx[k];
    run *= T[id];
    if (T[id] < c.ix[id].n) break;
    expect = v.stride[k] * c.ix[id].n;
  }
  return run;
}

// Fraction of 32-B sector bytes that are useful for a run of `run` doubles.
static double sector_eff(int64_t run, double es = 8.0) {
  double b = es * run;
  return b / (std::ceil(b / 32.0) * 32.0);
}

// Simulated cp.async smem wavefronts and global sectors of one stage of operand t, memoised
// on everything the slot table depends on (tiles, digit orders, layout, vector, shape).
static std::pair<double, double> operand_sim(const Contraction &c, const Config &cfg, int t, int vec,
                                             bool kmaj, int BMN, int BK, WfCache *cache) {
  std::vector<int64_t> key{t, vec, kmaj, BMN, BK, cfg.morder, cfg.korder, cfg.kind};
  for (int id : c.t[t].idx) key.push_back(cfg.T[id]);
  for (int id : cfg.kdig) key.push_back(cfg.T[id]);
  if (cache) {
    auto it = cache->find(key);
    if (it != cache->end()) return it->second;
  }
  const SlotTable st = build_slots(c, cfg, t, vec, kmaj, BMN, BK);
  const int es = kind_esize(cfg.kind);
  const std::pair<double, double> r{slot_wavefronts(st, vec, es, cfg.kind), slot_sectors(st, vec, es)};
  if (cache) (*cache)[key] = r;
  return r;
}

// ---------------------------------------------------------------- B200 cost model
double model_time(const Contraction &c, Config &cfg, const Variant &v, WfCache *cache, bool lower_bound) {
  finish_counts(c, cfg);
  const double nctas = (double)cfg.nctas * (double)c.nbatch(), steps = (double)cfg.nsteps;
  // per CTA-step pipe cycles on one SM: FP64 (DMMA) and shared memory
  double dmma = (double)v.BM * v.BN * v.BK / fma_per_clk(v.kind);
  if (is_umma(v.kind)) {   // the kernel trims N and the K instructions to the tile
    int nm, km;
    umma_trim(cfg, v, &nm, &km);
    dmma = (double)v.BM * nm * km * (32 / v.esize()) / fma_per_clk(v.kind);
  }
  const bool umma = is_umma(v.kind);
  const int maxv = 16 / kind_esize(cfg.kind);   // 16 B per cp.async
  cfg.vecX = vec_width(c, cfg, cfg.X, maxv);
  cfg.vecY = vec_width(c, cfg, cfg.Y, maxv);
  // lower_bound: the conflict-free ideal of the simulated terms (every smem wavefront and every
  // global sector fully used) — a cheap bound that prunes configurations before simulating
  const double es0 = kind_esize(cfg.kind);
  const auto ideal = [&](int64_t rows) {
    const double b = (double)rows * cfg.Kt * es0;
    return std::pair<double, double>{std::ceil(b / 128.0), std::ceil(b / 32.0)};
  };
  // tcgen05 with TMA operand boxes: one thread issues a few boxes per stage, the TMA unit writes
  // the swizzled planes at full smem bandwidth and fetches whole rows (no cp.async slots)
  TmaOperand ox, oy;
  const bool tma = umma && umma_tma_spec(c, cfg, v, cfg.X, nullptr, &ox) && umma_tma_spec(c, cfg, v, cfg.Y, nullptr, &oy);
  // (TMA: the boxes' own bytes — a K-major box spans BK of k whatever Kt is)
  const auto boxes = [](const TmaOperand &o) {
    const double b = (double)o.tx * o.nsub;
    return std::pair<double, double>{std::ceil(b / 128.0), std::ceil(b / 32.0)};
  };
  // CTA pairs: each CTA loads one X and one Y box per k-step for two tiles of work
  bool pair = tma && cta_pair_default(cfg);
  if (pair) {   // (as api.cu: the pair epilogue needs C's FVI leading m when it stores runs)
    int s0 = 1, t0 = 1;
    pair = c_run_rows(c, cfg, 8, &s0, &t0) != 8 || s0 == 1;
  }
  const auto sx = tma ? boxes(ox) : lower_bound ? ideal(cfg.Mt) : operand_sim(c, cfg, cfg.X, cfg.vecX, cfg.xKmajor, v.BM, v.BK, cache);
  const auto sy = tma ? boxes(oy) : lower_bound ? ideal(cfg.Nt) : operand_sim(c, cfg, cfg.Y, cfg.vecY, cfg.yKmajor, v.BN, v.BK, cache);
  cfg.wfX = sx.first;
  cfg.wfY = sy.first;
  cfg.secX = sx.second;
  cfg.secY = sy.second;
  const int MI = v.WM / 8, NJ = v.WN / 8, warps = v.cwarps();
  // FP64: consumer-warp fragment loads; UMMA reads its operands from smem descriptors
  const double lds = umma ? 0.0 : (double)warps * (v.BK / 4) * (MI + NJ) * 2;
  // producer warps: one LDGSTS warp-instruction per 32 slots, ~8 LSU cycles each
  const double nslots = (double)cfg.Mt * cfg.Kt / cfg.vecX + (double)cfg.Kt * cfg.Nt / cfg.vecY;
  const double ldgsts = tma ? 16.0 * (ox.nsub + oy.nsub) : std::ceil(nslots / 32.0) * 8.0;
  const double step = std::max({dmma, cfg.wfX + cfg.wfY + lds, ldgsts}) + kStepOverhead;
  // store issue per tile; UMMA: 4 warps x BN column stores, overlapped with the next
  // tile's MMAs by the double-buffered TMEM accumulator
  const double epi = umma ? 0.0 : (double)warps * MI * NJ * 2 * 6 / 4;
  const double epi_umma = umma ? (double)v.BN * 4 * 4 : 0.0;
  // memory: sector efficiencies of each tensor's tile along its own memory order
  const double es = v.esize();
  const double eX = sector_eff(contiguous_run(c, cfg.X, cfg.T), es);
  const double eY = sector_eff(contiguous_run(c, cfg.Y, cfg.T), es);
  const double eC = sector_eff(contiguous_run(c, 0, cfg.T), es);
  // the C tile leaves at the SM's share of the HBM write bandwidth (profiles/r01_*: the 6D
  // CCSD(T) cases); FP64: not overlapped with the same CTA's mainloop (the consumer warps
  // store), only with the other resident CTAs'; UMMA: overlapped through the TMEM buffers
  const double c_tile = (double)cfg.Mt * cfg.Nt * es / eC / (kHbm / kSMs / kClk);
  const double t_main = steps * step;
  double t_tile;
  if (umma) {
    t_tile = std::max({t_main, epi_umma, c_tile});
  } else if (v.stg) {
    // staged epilogue: the consumers only write the raw tile to smem (2 wavefronts per
    // fragment store); the producers drain it between their cp.async issues, so the C write
    // overlaps the next tile's mainloop; the producers' LSU issue carries loads + drain
    const double sts = (double)warps * MI * NJ * 2 * 2;
    const double drain = (double)v.BM * v.BN * es / 128.0 + std::ceil((double)cfg.Mt * cfg.Nt / 32.0) * 4.0;
    t_tile = std::max({t_main + sts, c_tile, steps * ldgsts + drain});
  } else {
    const double t_epi = std::max(epi, c_tile);
    t_tile = std::max(t_main, t_epi) + std::min(t_main, t_epi) / v.occ;
  }
  // persistent CTAs: grid = 148 * occ, tiles round-robin; t_tile is per tile per SM
  const double slots = kSMs * v.occ;
  const double tiles_per_sm = pair ? 2.0 * std::ceil((double)((cfg.mtiles + 1) / 2) * ((cfg.ntiles + 1) / 2) / (kSMs / 2))
                                   : std::ceil(nctas / slots) * v.occ;
  const double cyc_sm = tiles_per_sm * t_tile;
  cfg.t_comp = cyc_sm / kClk;
  // store-instruction efficiency: 8 consecutive rows of a DMMA fragment are contiguous in C
  // iff m's first digit is C's FVI
  // (UMMA: a warp stores 32 rows of one column)
  const int64_t srun = umma ? 32 : 8;
  double eS = es / 32.0;
  if (c.t[0].idx.empty()) eS = 1;
  else if (!cfg.mdig.empty() && cfg.mdig[0] == c.t[0].idx[0])
    eS = sector_eff(std::min<int64_t>(srun, cfg.T[cfg.mdig[0]]), es);
  else if (umma) {
    // staged epilogue: C's FVI anywhere in m, runs of 8 C-contiguous elements per store
    int s0, t0;
    if (c_run_rows(c, cfg, 8, &s0, &t0) == 8) eS = sector_eff(std::min<int64_t>(32, t0), es);
  }
  const double bx = es * c.numel(cfg.X), by = es * c.numel(cfg.Y), bc = es * c.numel(0);
  double rx = 1, ry = 1;
  if (bx + by > 0.5 * kL2Bytes) {
    const double f = (bx + by) / kL2Bytes;
    rx = std::min((double)cfg.ntiles, 1.0 + f);
    ry = std::min((double)cfg.mtiles, 1.0 + f);
  }
  cfg.dram_bytes = bx * rx / eX + by * ry / eY + bc / eC;
  cfg.t_mem = cfg.dram_bytes / kHbm;
  // L2 -> SM: the simulated sectors of every stage of every tile, plus the C stores
  const double l2b = nctas * steps * 32.0 * (cfg.secX + cfg.secY) * (pair ? 0.5 : 1.0) + bc / eS;
  cfg.t_l2 = l2b / kL2Bw;
  cfg.flops_pad = 2.0 * nctas * steps * v.BM * v.BN * v.BK;
  cfg.t_pred = std::max({cfg.t_comp, cfg.t_mem, cfg.t_l2}) * v.cal + kLaunch;
  return cfg.t_pred;
}

// ---------------------------------------------------------------- Alg. 3 (paper mode)
double paper_alg3_cost(const Contraction &c, const Config &cfg, const std::vector<int> &tbx,
                       const std::vector<int> &regx, const std::vector<int> &tby,
                       const std::vector<int> &regy) {
  const auto &T = cfg.T;
  auto prod = [&](const std::vector<int> &l) {
    double p = 1;
    for (int id : l) p *= T[id];
    return p;
  };
  double TBx = prod(tbx), REGx = prod(regx), TBy = prod(tby), REGy = prod(regy), TBk = 1;
  for (int id : cfg.kdig) TBk *= T[id];
  double steps = 1, tbs = 1;
  for (int id : cfg.kdig) steps *= (double)cdiv(c.ix[id].n, T[id]);
  for (int id : cfg.mdig) tbs *= (double)cdiv(c.ix[id].n, T[id]);
  for (int id : cfg.ndig) tbs *= (double)cdiv(c.ix[id].n, T[id]);
  // Alg. 3 lines 2-12: a row of TB_x threads walks the tensor's FVI; 128-B transactions
  auto trans_row = [&](int t) {
    double cont = (double)contiguous_run(c, t, T);
    return TBx / std::min(cont, TBx);
  };
  const double a = trans_row(cfg.X) * TBk * REGx * steps * tbs;               // Alg. 3 verbatim
  const double b = trans_row(cfg.Y) * (TBy * REGy * TBk / TBx) * steps * tbs;  // "similarly"
  const double cc = trans_row(0) * (TBy * REGx * REGy) * tbs;                  // C stored once
  return a + b + cc;
}

// ---------------------------------------------------------------- enumeration helpers
namespace {

using Tiling = std::vector<std::pair<int, int>>;  // (index id, tile) in mapping order

int64_t largest_divisor_le(int64_t n, int64_t cap) {
  for (int64_t d = std::min(n, cap); d >= 1; d--)
    if (n % d == 0) return d;
  return 1;
}
int64_t pow2_le(int64_t x) {
  int64_t p = 1;
  while (p * 2 <= x) p *= 2;
  return p;
}

// Crossing-tile candidates when an index of extent n overshoots the target: P:L218 uses
// floor(target/prev) (R12); the B200 mode adds the largest divisor of n and the largest
// power of two not above it (no partial tiles / vector alignment).
std::vector<int64_t> crossing(int64_t n, int64_t cap, bool paper) {
  std::vector<int64_t> v{std::max<int64_t>(1, cap)};
  if (!paper) {
    v.push_back(largest_divisor_le(n, cap));
    v.push_back(pow2_le(std::max<int64_t>(1, cap)));
  }
  std::sort(v.begin(), v.end());
  v.erase(std::unique(v.begin(), v.end()), v.end());
  return v;
}

// Alg. 2 greedy: map `seq` in order onto a dimension of target size S starting from a
// partial product `prev`; full extents while below the target, the crossing index gets a
// candidate tile and closes the dimension.  "Not mapped" (all fit) is kept (R13).
void greedy(const Contraction &c, const std::vector<int> &seq, size_t at, int64_t prev, int64_t S,
            Tiling cur, bool paper, std::vector<Tiling> &out) {
  for (size_t i = at; i < seq.size(); i++) {
    const int id = seq[i];
    const int64_t n = c.ix[id].n;
    if (prev * n >= S) {
      if (prev * n == S) {
        cur.push_back({id, (int)n});
        out.push_back(cur);
      } else {
        for (int64_t t : crossing(n, S / prev, paper)) {
          Tiling x = cur;
          x.push_back({id, (int)t});
          out.push_back(x);
        }
      }
      return;
    }
    cur.push_back({id, (int)n});
    prev *= n;
  }
  out.push_back(cur);
}

// Rotations of `lst` starting at s_idx (from s_idx to the SVI, then 0..s_idx-1).
std::vector<std::vector<int>> rotations(const std::vector<int> &lst) {
  std::vector<std::vector<int>> r;
  for (size_t s = 0; s < lst.size(); s++) {
    std::vector<int> v(lst.begin() + s, lst.end());
    v.insert(v.end(), lst.begin(), lst.begin() + s);
    r.push_back(v);
  }
  if (r.empty()) r.push_back(std::vector<int>());
  return r;
}

// Two-level enumeration (TB then REG) for one side of the B200 kernel: the
// first index of each rotation gets a first-level tile from the power-of-two targets, the
// rest are filled greedily up to the side's total target S.
std::vector<Tiling> enum_side(const Contraction &c, const std::vector<int> &order, int fixed_first,
                              int64_t S) {
  std::vector<Tiling> uniq;   // (sorted and deduplicated at the end)
  std::vector<std::vector<int>> rots;
  if (fixed_first >= 0) {
    std::vector<int> rest;
    for (int id : order) if (id != fixed_first) rest.push_back(id);
    for (auto &r : rotations(rest)) {
      std::vector<int> v{fixed_first};
      v.insert(v.end(), r.begin(), r.end());
      rots.push_back(v);
    }
  } else {
    rots = rotations(order);
  }
  for (auto &seq : rots) {
    if (seq.empty()) { uniq.push_back(Tiling()); continue; }
    const int first = seq[0];
    const int64_t n0 = c.ix[first].n;
    std::set<int64_t> t0s;
    for (int64_t s1 = 1; s1 <= S; s1 *= 2)
      for (int64_t t : crossing(n0, s1, false)) t0s.insert(std::min(t, n0));
    t0s.insert(std::min(n0, S));
    for (int64_t t0 : t0s) {
      Tiling cur{{first, (int)t0}};
      std::vector<Tiling> res;
      if (t0 < n0) res.push_back(cur);  // first index alone (the others on the grid)
      greedy(c, seq, 1, t0, S, cur, false, res);
      uniq.insert(uniq.end(), res.begin(), res.end());
    }
  }
  std::sort(uniq.begin(), uniq.end());
  uniq.erase(std::unique(uniq.begin(), uniq.end()), uniq.end());
  return uniq;
}

int64_t tprod(const Tiling &t) {
  int64_t p = 1;
  for (auto &x : t) p *= x.second;
  return p;
}

void apply_tiling(const Tiling &t, std::vector<int> &T) {
  for (auto &x : t) T[x.first] = x.second;
}

std::string tiling_str(const Contraction &c, const Tiling &t) {
  std::string s;
  for (auto &x : t) s += (s.empty() ? "" : ",") + c.ix[x.first].name + ":" + std::to_string(x.second);
  return "[" + s + "]";
}

bool better(const Config &a, const Config &b) {
  // deterministic: cost, then more CTAs, then larger tile, then variant / order ids
  if (a.t_pred != b.t_pred) return a.t_pred < b.t_pred;
  // the same bounding term: the one with less pressure on the others (e.g. an L2-bound tie
  // between a scalar and a vectorised load order goes to the vectorised one)
  const double sa = a.t_comp + a.t_mem + a.t_l2, sb = b.t_comp + b.t_mem + b.t_l2;
  if (sa != sb) return sa < sb;
  if (a.nctas != b.nctas) return a.nctas > b.nctas;
  if (a.Mt * a.Nt != b.Mt * b.Nt) return a.Mt * a.Nt > b.Mt * b.Nt;
  if (a.variant != b.variant) return a.variant < b.variant;
  if (a.morder != b.morder) return a.morder < b.morder;
  return a.korder < b.korder;
}

bool fits(const Config &cfg, const Variant &v) {
  return cfg.Mt <= v.BM && cfg.Nt <= v.BN && cfg.Kt <= v.BK && cfg.nctas < (1LL << 31) &&
         cfg.mtiles < (1LL << 26) && cfg.ntiles < (1LL << 26) && cfg.nsteps < (1LL << 24);   // (tile tables: 56 B per tile)
}

// The distinct (morder, korder) digit-order options of a contraction.
std::vector<Config> order_options(const Contraction &c, int kind, int only_morder = -1) {
  std::vector<Config> out;
  for (int mo = 0; mo < 2; mo++)
    if (only_morder < 0 || mo == only_morder)
    for (int ko = 0; ko < 2; ko++) {
      Config cfg;
      cfg.morder = mo;
      cfg.korder = ko;
      cfg.kind = kind;
      digit_orders(c, cfg);
      bool dup = false;
      for (auto &o : out) dup |= o.mdig == cfg.mdig && o.kdig == cfg.kdig;
      if (!dup) out.push_back(cfg);
    }
  return out;
}

}  // namespace

// (exported for representative-size plans: api.cu tc_plan_resize / tc_plan_select)
bool config_fits(const Config &cfg, const Variant &v) { return fits(cfg, v); }

// ---------------------------------------------------------------- B200 mode
static Status choose_b200(const Contraction &c, int kind, int forced_variant, int only_morder, Config &best,
                          PlanStats &st) {
  WfCache cache;
  Config base;
  base.kind = kind;
  digit_orders(c, base);
  base.T.assign(c.ix.size(), 1);
  // Alg. 2 walks each input's index list; C's FVI is mapped first on the X side
  std::vector<int> mx, ny, kx;
  for (int id : c.t[base.X].idx) if (is_ext(c.ix[id].cls)) mx.push_back(id);
  for (int id : c.t[base.Y].idx) if (is_ext(c.ix[id].cls)) ny.push_back(id);
  for (int id : c.t[base.X].idx) if (c.ix[id].cls == INTL) kx.push_back(id);
  const int c0 = c.c_fvi();
  int kfirst = -1;
  if (!c.t[base.X].idx.empty() && c.ix[c.t[base.X].idx[0]].cls == INTL) kfirst = c.t[base.X].idx[0];
  else if (!c.t[base.Y].idx.empty() && c.ix[c.t[base.Y].idx[0]].cls == INTL) kfirst = c.t[base.Y].idx[0];
  const auto orders = order_options(c, kind, only_morder);
  bool found = false;
  // the side enumerations depend only on the side's target size: shared by the variants
  std::map<int64_t, std::vector<Tiling>> msC, nsC, ksC;
  auto side_of = [&](std::map<int64_t, std::vector<Tiling>> &m, const std::vector<int> &ids, int first, int64_t S)
      -> const std::vector<Tiling> & {
    auto it = m.find(S);
    if (it == m.end()) it = m.emplace(S, enum_side(c, ids, first, S)).first;
    return it->second;
  };
  // variants in order of their DMMA-pipe lower bound at their fullest tiles, so that a good
  // configuration is known early and bounds the others (planning time)
  std::vector<int> vorder;
  for (int vi = 0; vi < (int)variants().size(); vi++)
    if ((forced_variant < 0 || vi == forced_variant) && variants()[vi].kind == kind) vorder.push_back(vi);
  for (int vi : vorder) {
    const auto &v = variants()[vi];
    bool vfound = false;
    Config vbest;
    const auto &ms0 = side_of(msC, mx, c0, v.BM);
    const auto &ns0 = side_of(nsC, ny, -1, v.BN);
    const auto &ks = side_of(ksC, kx, kfirst, v.BK);
    // keep the k tilings with the least padding, top 4 (sorted by index: no tiling copies)
    std::vector<std::pair<double, int>> kscore;
    for (size_t q = 0; q < ks.size(); q++) {
      const Tiling &k = ks[q];
      if (tprod(k) > v.BK) continue;
      std::vector<int> T(c.ix.size(), 1);
      apply_tiling(k, T);
      double steps = 1, need = 1;
      for (int id : kx) { steps *= (double)cdiv(c.ix[id].n, T[id]); need *= (double)c.ix[id].n; }
      // padding first; among equals, longer runs along the inputs' internal FVIs
      double run = 1;
      for (int t = 1; t <= 2; t++)
        if (!c.t[t].idx.empty() && c.ix[c.t[t].idx[0]].cls == INTL)
          run *= std::min(32 / v.esize(), T[c.t[t].idx[0]]);   // one 32-B sector
      kscore.push_back({steps * v.BK / need / run, (int)q});
    }
    std::stable_sort(kscore.begin(), kscore.end(), [](auto &a, auto &b) { return a.first < b.first; });
    std::vector<std::pair<double, Tiling>> kr;
    for (size_t q = 0; q < kscore.size() && q < 4; q++) kr.push_back({kscore[q].first, ks[kscore[q].second]});
    // drop m / n tilings that fill less than half of what the fullest one fills
    auto fill = [](const std::vector<Tiling> &v, int64_t S) {
      int64_t mx = 0;
      for (auto &t : v) if (tprod(t) <= S) mx = std::max(mx, tprod(t));
      std::vector<const Tiling *> o;
      for (auto &t : v) if (tprod(t) <= S && 2 * tprod(t) >= mx) o.push_back(&t);
      return o;
    };
    const size_t raw_m = ms0.size(), raw_n = ns0.size();
    const auto ms = fill(ms0, v.BM);
    const auto ns = fill(ns0, v.BN);
    st.raw += (int64_t)raw_m * raw_n * ks.size() * orders.size();
    st.pruned += (int64_t)(raw_m * raw_n * ks.size() - ms.size() * ns.size() * kr.size()) * orders.size();
    // one scratch configuration per digit order: no Config copies in the loop
    std::vector<Config> scratch(orders.begin(), orders.end());
    for (const Tiling *m : ms)
      for (const Tiling *n : ns)
        for (auto &k : kr)
          for (Config &cfg : scratch) {
            cfg.T.assign(c.ix.size(), 1);
            apply_tiling(*m, cfg.T);
            apply_tiling(*n, cfg.T);
            apply_tiling(k.second, cfg.T);
            finish_counts(c, cfg);
            if (!fits(cfg, v)) { st.pruned++; continue; }
            cfg.variant = vi;
            // bound: the MMA-pipe time of the padded work alone (no smem / memory terms),
            // against this variant's best so far and 1.5x the best of every variant (a variant
            // that far behind is no tuning candidate: its per-variant figure stays an upper one)
            {
              const double tiles = std::ceil((double)cfg.nctas * (double)c.nbatch() / (kSMs * v.occ));
              const double lb = tiles * v.occ * (double)cfg.nsteps * v.BM * v.BN * v.BK /
                                fma_per_clk(v.kind) / kClk + kLaunch;
              if ((vfound && lb > vbest.t_pred) || (found && lb > 1.5 * best.t_pred)) { st.pruned++; continue; }
            }
            if (vfound || found) {   // the conflict-free ideal of this configuration
              const double lb = model_time(c, cfg, v, &cache, true);
              if ((vfound && lb > vbest.t_pred) || (found && lb > 1.5 * best.t_pred)) { st.pruned++; continue; }
            }
            model_time(c, cfg, v, &cache);
            st.ranked++;
            if (!vfound || better(cfg, vbest)) { vbest = cfg; vfound = true; }
          }
    if (!vfound) continue;
    st.per_variant.push_back({vi, vbest.t_pred});
    if (!found || better(vbest, best)) { best = vbest; found = true; }
  }
  std::stable_sort(st.per_variant.begin(), st.per_variant.end(),
                   [](const auto &a, const auto &b) { return a.second < b.second; });
  return found ? ST_OK : ST_NO_CONFIG;
}

// ---------------------------------------------------------------- paper mode
// enum_X_TB / enum_X_REG / Y / TB_k with the V100 value sets of P:L176 and Alg. 2's
// greedy (floor crossing tile, R12); product; prune by P:L172 (smem, registers) and
// P:L174 (FVI on a thread dimension, #TBs above one wave); rank by Alg. 3.
static Status choose_paper(const Contraction &c, int kind, int forced_variant, Config &best, PlanStats &st) {
  WfCache cache;
  Config base;
  base.kind = kind;
  digit_orders(c, base);
  base.T.assign(c.ix.size(), 1);
  const int X = base.X, Y = base.Y;
  const int c0 = c.c_fvi();
  std::vector<int> xe, ye, ki;
  for (int id : c.t[X].idx) if (is_ext(c.ix[id].cls)) xe.push_back(id);
  for (int id : c.t[Y].idx) if (is_ext(c.ix[id].cls)) ye.push_back(id);
  for (int id : c.t[X].idx) if (c.ix[id].cls == INTL) ki.push_back(id);
  const int64_t TBS[3] = {4, 8, 16}, REGS[4] = {2, 4, 6, 8};

  struct Part { Tiling tb, reg; };
  auto enum_tb_reg = [&](const std::vector<int> &ext, int first, int fvi_rule) {
    std::set<std::pair<Tiling, Tiling>> uniq;
    for (int64_t S : TBS) {
      std::vector<std::vector<int>> seqs;
      if (first >= 0) {
        std::vector<int> rest;
        for (int id : ext) if (id != first) rest.push_back(id);
        for (auto &r : rotations(rest)) {
          std::vector<int> v{first};
          v.insert(v.end(), r.begin(), r.end());
          seqs.push_back(v);
        }
      } else {
        seqs = rotations(ext);
      }
      for (auto &seq : seqs) {
        std::vector<Tiling> tbs;
        greedy(c, seq, 0, 1, S, Tiling(), true, tbs);
        for (auto &tb : tbs) {
          if (fvi_rule >= 0) {
            bool has = false;
            for (auto &x : tb) has |= x.first == fvi_rule;
            if (!has) continue;  // the input's FVI is always on a thread dimension
          }
          std::vector<int> left;
          for (int id : ext) {
            bool used = false;
            for (auto &x : tb) used |= x.first == id;
            if (!used) left.push_back(id);
          }
          bool any = false;
          for (int64_t R : REGS)
            for (auto &rs : rotations(left)) {
              std::vector<Tiling> regs;
              greedy(c, rs, 0, 1, R, Tiling(), true, regs);
              for (auto &rg : regs) { uniq.insert({tb, rg}); any = true; }
            }
          if (!any) uniq.insert({tb, Tiling()});
        }
      }
    }
    std::vector<Part> out;
    for (auto &u : uniq) out.push_back({u.first, u.second});
    return out;
  };
  const int yfvi = (!c.t[Y].idx.empty() && is_ext(c.ix[c.t[Y].idx[0]].cls)) ? c.t[Y].idx[0] : -1;
  auto px = enum_tb_reg(xe, c0, -1);
  auto py = enum_tb_reg(ye, -1, yfvi);
  std::set<Tiling> kset;
  const int kfvi = (!c.t[X].idx.empty() && c.ix[c.t[X].idx[0]].cls == INTL) ? c.t[X].idx[0] : -1;
  const int kfvi2 = (!c.t[Y].idx.empty() && c.ix[c.t[Y].idx[0]].cls == INTL) ? c.t[Y].idx[0] : -1;
  for (int64_t S : TBS)
    for (auto &seq : rotations(ki)) {
      std::vector<Tiling> r;
      greedy(c, seq, 0, 1, S, Tiling(), true, r);
      for (auto &t : r) {
        bool ok = true;
        for (int f : {kfvi, kfvi2}) {
          if (f < 0) continue;
          bool has = false;
          for (auto &x : t) has |= x.first == f;
          ok &= has;
        }
        if (ok) kset.insert(t);
      }
    }
  if (kset.empty()) kset.insert(Tiling());
  st.raw = (int64_t)px.size() * py.size() * kset.size();
  bool found = false;
  // best B200-model time per variant over the configs the paper's rules keep: the candidate
  // list of measured tuning (tc_plan_tuned) in paper mode too
  std::map<int, double> vbest;
  for (auto &x : px)
    for (auto &y : py)
      for (auto &k : kset) {
        Config cfg = base;
        apply_tiling(x.tb, cfg.T); apply_tiling(x.reg, cfg.T);
        apply_tiling(y.tb, cfg.T); apply_tiling(y.reg, cfg.T);
        apply_tiling(k, cfg.T);
        finish_counts(c, cfg);
        const double TBx = (double)tprod(x.tb), REGx = (double)tprod(x.reg);
        const double TBy = (double)tprod(y.tb), REGy = (double)tprod(y.reg);
        const double TBk = (double)tprod(k);
        // P:L172 hardware constraints (V100: 48 KB smem per block, 255 registers/thread)
        const double smem = (double)kind_esize(kind) * (TBx * TBk * REGx + TBy * TBk * REGy);
        bool ok = smem <= 48 * 1024 && REGx * REGy <= 64 && TBx * TBy <= 1024;
        // enough thread blocks (R16: at least one wave of the running GPU)
        ok &= (double)cfg.nctas >= kSMs;
        // it must also map onto one of the compiled B200 kernels
        int vi_best = -1;
        Config fit;
        if (ok) {
          for (int vi = 0; vi < (int)variants().size(); vi++) {
            if (forced_variant >= 0 && vi != forced_variant) continue;
            if (variants()[vi].kind != kind) continue;
            if (!fits(cfg, variants()[vi])) continue;
            Config t = cfg;
            t.variant = vi;
            model_time(c, t, variants()[vi], &cache);
            auto vb = vbest.find(vi);
            if (vb == vbest.end() || t.t_pred < vb->second) vbest[vi] = t.t_pred;
            if (vi_best < 0 || better(t, fit)) { fit = t; vi_best = vi; }
          }
        }
        if (!ok || vi_best < 0) { st.pruned++; continue; }
        auto ids = [](const Tiling &t) { std::vector<int> v; for (auto &q : t) v.push_back(q.first); return v; };
        fit.paper_cost = paper_alg3_cost(c, fit, ids(x.tb), ids(x.reg), ids(y.tb), ids(y.reg));
        fit.paper_mapping = "TB_x=" + tiling_str(c, x.tb) + " REG_x=" + tiling_str(c, x.reg) +
                            " TB_y=" + tiling_str(c, y.tb) + " REG_y=" + tiling_str(c, y.reg) +
                            " TB_k=" + tiling_str(c, k);
        st.ranked++;
        const bool win = !found || fit.paper_cost < best.paper_cost ||
                         (fit.paper_cost == best.paper_cost && better(fit, best));
        if (win) { best = fit; found = true; }
      }
  for (auto &kv : vbest) st.per_variant.push_back(kv);
  std::stable_sort(st.per_variant.begin(), st.per_variant.end(),
                   [](const auto &a, const auto &b) { return a.second < b.second; });
  return found ? ST_OK : ST_NO_CONFIG;
}

// ---------------------------------------------------------------- forced tiles
static Status choose_forced(const Contraction &c, int kind, const ForcedTiles &ft, int forced_variant,
                            Config &best, std::string &err) {
  WfCache cache;
  bool found = false;
  for (const auto &o : order_options(c, kind, ft.morder)) {
    Config cfg = o;
    cfg.T.assign(c.ix.size(), 1);
    for (size_t id = 0; id < c.ix.size(); id++) {
      auto it = ft.tile.find(c.ix[id].name);
      if (it != ft.tile.end())
        cfg.T[id] = (int)std::max<int64_t>(1, std::min<int64_t>(it->second, c.ix[id].n));
    }
    finish_counts(c, cfg);
    for (int vi = 0; vi < (int)variants().size(); vi++) {
      if (forced_variant >= 0 && vi != forced_variant) continue;
      if (variants()[vi].kind != kind) continue;
      if (!fits(cfg, variants()[vi])) continue;
      Config t = cfg;
      t.variant = vi;
      model_time(c, t, variants()[vi], &cache);
      if (!found || better(t, best)) { best = t; found = true; }
    }
  }
  if (!found) { err = "forced tiles fit no compiled kernel variant"; return ST_NO_CONFIG; }
  return ST_OK;
}

Status choose(const Contraction &c, int kind, int cost_mode, int forced_variant, const ForcedTiles &ft,
              Config &out, PlanStats &stats, std::string &err) {
  auto t0 = std::chrono::steady_clock::now();
  stats = PlanStats();
  stats.cost_mode = cost_mode;
  Status s;
  if (ft.on) s = choose_forced(c, kind, ft, forced_variant, out, err);
  else if (cost_mode == 1) s = choose_paper(c, kind, forced_variant, out, stats);
  else s = choose_b200(c, kind, forced_variant, ft.morder, out, stats);
  if (s == ST_NO_CONFIG && !ft.on && cost_mode == 1) {
    // the paper's value sets can leave nothing after pruning (tiny problems): fall back to
    // the B200 enumeration so that every legal contraction gets a plan (R13)
    PlanStats st2;
    s = choose_b200(c, kind, forced_variant, ft.morder, out, st2);
    stats.ranked += st2.ranked;
    stats.per_variant = st2.per_variant;
  }
  if (s != ST_OK && err.empty()) err = "no legal configuration";
  stats.plan_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return s;
}

}  // namespace tc
