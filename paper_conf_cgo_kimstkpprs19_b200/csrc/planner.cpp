// planner.cpp — enumeration (Alg. 2 generalised), pruning and the two cost
// models (Alg. 3 verbatim, and the B200 re-derivation) of libtc.  See planner.hpp.
#include "planner.hpp"

#include <algorithm>
#include <chrono>
#include <cmath>
#include <set>
#include <sstream>

namespace tc {

// ---------------------------------------------------------------- hardware constants
// B200, measured in profiles/r01_peaks.json (DMMA 37.1 TFLOP/s = 148 SM x 64 FMA/clk x
// 2 x 1.965 GHz; HBM read 7.36 TB/s, write 6.7 TB/s, copy 6.55 TB/s MEASURED_PEAKS).
static constexpr double kSMs = 148, kFmaPerClk = 64, kClk = 1.965e9;
static constexpr double kHbm = 6.5e12, kL2Bw = 10.0e12, kL2Bytes = 126.0e6;
static constexpr double kLaunch = 3.0e-6;

const std::vector<Variant> &variants() {
  // BM, BN, BK, WM, WN, stages, threads, CTAs/SM (from ptxas registers and smem)
  static const std::vector<Variant> v = {
      {128, 128, 16, 64, 32, 4, 256, 1},
      {128, 64, 16, 64, 32, 3, 128, 2},
      {64, 128, 16, 32, 64, 3, 128, 2},
      {64, 64, 16, 32, 32, 4, 128, 2},
      {128, 128, 8, 64, 32, 4, 256, 1},
      {64, 64, 8, 32, 32, 4, 128, 3},
  };
  return v;
}

int x_tensor(const Contraction &c) {
  if (c.t[0].idx.empty()) return 1;
  return c.pos_in(1, c.t[0].idx[0]) >= 0 ? 1 : 2;
}

static int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

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
static double sector_eff(int64_t run) {
  double b = 8.0 * run;
  return b / (std::ceil(b / 32.0) * 32.0);
}

// ---------------------------------------------------------------- B200 cost model
double model_time(const Contraction &c, const Config &cfg, const Variant &v, double *comp,
                  double *mem, double *l2, double *dram) {
  const auto &T = cfg.T;
  int64_t mt = 1, nt = 1, steps = 1;
  for (int id : cfg.mdig) mt *= cdiv(c.ix[id].n, T[id]);
  for (int id : cfg.ndig) nt *= cdiv(c.ix[id].n, T[id]);
  for (int id : cfg.kdig) steps *= cdiv(c.ix[id].n, T[id]);
  const double nctas = (double)mt * nt;
  // FP64 pipe time of the PADDED work, quantised to waves of 148 * occ CTAs
  const double slots = kSMs * v.occ;
  const double waves = std::ceil(nctas / slots);
  const double fma_cta = (double)steps * v.BM * v.BN * v.BK;
  const double t_comp = waves * v.occ * fma_cta / (kFmaPerClk * kClk);
  // sector efficiencies of each tensor's tile along its own memory order
  const double eX = sector_eff(contiguous_run(c, cfg.X, T));
  const double eY = sector_eff(contiguous_run(c, cfg.Y, T));
  const double eC = sector_eff(contiguous_run(c, 0, T));
  // L2 -> SM traffic: every CTA streams its X and Y slabs
  const double Mt = (double)cfg.Mt, Nt = (double)cfg.Nt, Kt = (double)cfg.Kt;
  const double l2b = nctas * steps * 8.0 * (Mt * Kt / eX + Kt * Nt / eY);
  const double t_l2 = l2b / kL2Bw;
  // DRAM: inputs once if they stay in L2, otherwise re-read per tile row / column
  const double bx = 8.0 * c.numel(cfg.X), by = 8.0 * c.numel(cfg.Y), bc = 8.0 * c.numel(0);
  double rx = 1, ry = 1;
  if (bx + by > 0.5 * kL2Bytes) {
    const double f = (bx + by) / kL2Bytes;
    rx = std::min((double)nt, 1.0 + f);
    ry = std::min((double)mt, 1.0 + f);
  }
  const double d = bx * rx / eX + by * ry / eY + bc / eC;
  const double t_mem = d / kHbm;
  // with one CTA per SM the C store of a tile is not overlapped by MMA work
  const double t_store = (bc / eC) / kHbm / std::max(1, v.occ);
  double t = std::max({t_comp + t_store, t_mem, t_l2}) + kLaunch;
  if (comp) *comp = t_comp;
  if (mem) *mem = t_mem;
  if (l2) *l2 = t_l2;
  if (dram) *dram = d;
  return t;
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

// Crossing-tile candidates when index of extent n overshoots the target: P:L218 uses
// floor(target/prev) (R12); we add the largest divisor of n and the largest power of two
// not above it, which avoid partial tiles / keep vector alignment.
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
  if (r.empty()) r.push_back({});
  return r;
}

// Two-level enumeration (TB then REG) for one side of the B200 kernel:
// the first index of each rotation gets a first-level tile from the power-of-two targets,
// the rest are filled greedily up to the side's total target S.
std::vector<Tiling> enum_side(const Contraction &c, const std::vector<int> &order, int fixed_first,
                              int64_t S) {
  std::set<Tiling> uniq;
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
    if (seq.empty()) { uniq.insert(Tiling{}); continue; }
    const int first = seq[0];
    const int64_t n0 = c.ix[first].n;
    std::set<int64_t> t0s;
    for (int64_t s1 = 1; s1 <= S; s1 *= 2) {
      for (int64_t t : crossing(n0, s1, false)) t0s.insert(std::min(t, n0));
    }
    t0s.insert(std::min(n0, S));
    for (int64_t t0 : t0s) {
      Tiling cur{{first, (int)t0}};
      std::vector<Tiling> res;
      if (t0 < n0) {
        res.push_back(cur);  // first index alone (others tile 1)
        // plus filling the rest on top (TB then REG)
        greedy(c, seq, 1, t0, S, cur, false, res);
      } else {
        greedy(c, seq, 1, t0, S, cur, false, res);
      }
      for (auto &x : res) uniq.insert(x);
    }
  }
  return std::vector<Tiling>(uniq.begin(), uniq.end());
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

}  // namespace

// Compute-order digit lists (kparams.hpp): m = C's indices in X, n = C's indices in Y (both
// in C order, so C's FVI leads m); k = internals with an input's FVI first.
static void digit_orders(const Contraction &c, Config &cfg) {
  cfg.X = x_tensor(c);
  cfg.Y = 3 - cfg.X;
  cfg.mdig.clear(); cfg.ndig.clear(); cfg.kdig.clear();
  for (int id : c.t[0].idx) (c.pos_in(cfg.X, id) >= 0 ? cfg.mdig : cfg.ndig).push_back(id);
  int first = -1;
  const auto &xv = c.t[cfg.X].idx, &yv = c.t[cfg.Y].idx;
  if (!xv.empty() && c.ix[xv[0]].cls == INTL) first = xv[0];
  else if (!yv.empty() && c.ix[yv[0]].cls == INTL) first = yv[0];
  if (first >= 0) cfg.kdig.push_back(first);
  for (int id : xv)
    if (c.ix[id].cls == INTL && id != first) cfg.kdig.push_back(id);
}

static void finish(const Contraction &c, Config &cfg) {
  cfg.Mt = cfg.Nt = cfg.Kt = 1;
  cfg.nctas = 1;
  cfg.nsteps = 1;
  for (int id : cfg.mdig) { cfg.Mt *= cfg.T[id]; cfg.nctas *= cdiv(c.ix[id].n, cfg.T[id]); }
  for (int id : cfg.ndig) { cfg.Nt *= cfg.T[id]; cfg.nctas *= cdiv(c.ix[id].n, cfg.T[id]); }
  for (int id : cfg.kdig) { cfg.Kt *= cfg.T[id]; cfg.nsteps *= cdiv(c.ix[id].n, cfg.T[id]); }
}

static bool better(const Config &a, const Config &b) {
  // deterministic: cost, then more CTAs, then larger tile, then variant id
  if (a.t_pred != b.t_pred) return a.t_pred < b.t_pred;
  if (a.nctas != b.nctas) return a.nctas > b.nctas;
  if (a.Mt * a.Nt != b.Mt * b.Nt) return a.Mt * a.Nt > b.Mt * b.Nt;
  return a.variant < b.variant;
}

static void evaluate(const Contraction &c, Config &cfg, int vi) {
  cfg.variant = vi;
  finish(c, cfg);
  cfg.t_pred = model_time(c, cfg, variants()[vi], &cfg.t_comp, &cfg.t_mem, &cfg.t_l2, &cfg.dram_bytes);
  const auto &v = variants()[vi];
  cfg.flops_pad = 2.0 * (double)cfg.nctas * cfg.nsteps * v.BM * v.BN * v.BK;
}

static bool fits(const Config &cfg, const Variant &v) {
  return cfg.Mt <= v.BM && cfg.Nt <= v.BN && cfg.Kt <= v.BK && cfg.nctas < (1LL << 31);
}

// ---------------------------------------------------------------- B200 mode
static Status choose_b200(const Contraction &c, int forced_variant, Config &best, PlanStats &st) {
  Config base;
  digit_orders(c, base);
  base.T.assign(c.ix.size(), 1);
  // the X side's externals in X's order (Alg. 2 walks the input's index list)
  std::vector<int> mx, ny, kx;
  for (int id : c.t[base.X].idx) if (c.ix[id].cls != INTL) mx.push_back(id);
  for (int id : c.t[base.Y].idx) if (c.ix[id].cls != INTL) ny.push_back(id);
  kx = base.kdig;
  const int c0 = base.mdig.empty() ? -1 : base.mdig[0];
  const int kfirst = base.kdig.empty() ? -1 : base.kdig[0];
  bool found = false;
  for (int vi = 0; vi < (int)variants().size(); vi++) {
    if (forced_variant >= 0 && vi != forced_variant) continue;
    const auto &v = variants()[vi];
    auto ms = enum_side(c, mx, c0, v.BM);
    auto ns = enum_side(c, ny, -1, v.BN);
    auto ks = enum_side(c, kx, kfirst, v.BK);
    // keep the k tilings with the least padding (ties: longer runs), top 4
    std::vector<std::pair<double, Tiling>> kr;
    for (auto &k : ks) {
      if (tprod(k) > v.BK) continue;
      std::vector<int> T(c.ix.size(), 1);
      apply_tiling(k, T);
      double steps = 1, need = 1;
      for (int id : base.kdig) { steps *= (double)cdiv(c.ix[id].n, T[id]); need *= (double)c.ix[id].n; }
      double pad = steps * v.BK / need;
      kr.push_back({pad, k});
    }
    std::sort(kr.begin(), kr.end(), [](auto &a, auto &b) { return a.first < b.first; });
    if (kr.size() > 4) kr.resize(4);
    st.raw += (int64_t)ms.size() * ns.size() * ks.size();
    for (auto &m : ms) {
      if (tprod(m) > v.BM) { st.pruned += (int64_t)ns.size() * ks.size(); continue; }
      for (auto &n : ns) {
        if (tprod(n) > v.BN) { st.pruned += (int64_t)ks.size(); continue; }
        for (auto &k : kr) {
          Config cfg = base;
          apply_tiling(m, cfg.T);
          apply_tiling(n, cfg.T);
          apply_tiling(k.second, cfg.T);
          finish(c, cfg);
          if (!fits(cfg, v)) { st.pruned++; continue; }
          evaluate(c, cfg, vi);
          st.ranked++;
          if (!found || better(cfg, best)) { best = cfg; found = true; }
        }
      }
    }
  }
  return found ? ST_OK : ST_NO_CONFIG;
}

// ---------------------------------------------------------------- paper mode
// enum_X_TB / enum_X_REG / Y / TB_k with the V100 value sets of P:L176 and Alg. 2's
// greedy (floor crossing tile, R12); product; prune by P:L172 (smem, registers) and
// P:L174 (FVI on a thread dimension, #TBs above one wave); rank by Alg. 3.
static Status choose_paper(const Contraction &c, int forced_variant, Config &best, PlanStats &st) {
  Config base;
  digit_orders(c, base);
  base.T.assign(c.ix.size(), 1);
  const int X = base.X, Y = base.Y;
  const int c0 = base.mdig.empty() ? -1 : base.mdig[0];
  std::vector<int> xe, ye, ki;
  for (int id : c.t[X].idx) if (c.ix[id].cls != INTL) xe.push_back(id);
  for (int id : c.t[Y].idx) if (c.ix[id].cls != INTL) ye.push_back(id);
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
        greedy(c, seq, 0, 1, S, {}, true, tbs);
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
          for (int64_t R : REGS) {
            for (auto &rs : rotations(left)) {
              std::vector<Tiling> regs;
              greedy(c, rs, 0, 1, R, {}, true, regs);
              for (auto &rg : regs) { uniq.insert({tb, rg}); any = true; }
            }
          }
          if (!any) uniq.insert({tb, {}});
        }
      }
    }
    std::vector<Part> out;
    for (auto &u : uniq) out.push_back({u.first, u.second});
    return out;
  };
  const int yfvi = (!c.t[Y].idx.empty() && c.ix[c.t[Y].idx[0]].cls != INTL) ? c.t[Y].idx[0] : -1;
  auto px = enum_tb_reg(xe, c0, -1);
  auto py = enum_tb_reg(ye, -1, yfvi);
  std::set<Tiling> kset;
  int kfvi = -1;
  if (!c.t[X].idx.empty() && c.ix[c.t[X].idx[0]].cls == INTL) kfvi = c.t[X].idx[0];
  int kfvi2 = (!c.t[Y].idx.empty() && c.ix[c.t[Y].idx[0]].cls == INTL) ? c.t[Y].idx[0] : -1;
  for (int64_t S : TBS)
    for (auto &seq : rotations(ki)) {
      std::vector<Tiling> r;
      greedy(c, seq, 0, 1, S, {}, true, r);
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
  if (kset.empty()) kset.insert(Tiling{});
  st.raw = (int64_t)px.size() * py.size() * kset.size();
  bool found = false;
  for (auto &x : px)
    for (auto &y : py)
      for (auto &k : kset) {
        Config cfg = base;
        apply_tiling(x.tb, cfg.T); apply_tiling(x.reg, cfg.T);
        apply_tiling(y.tb, cfg.T); apply_tiling(y.reg, cfg.T);
        apply_tiling(k, cfg.T);
        finish(c, cfg);
        const double TBx = (double)tprod(x.tb), REGx = (double)tprod(x.reg);
        const double TBy = (double)tprod(y.tb), REGy = (double)tprod(y.reg);
        const double TBk = (double)tprod(k);
        // P:L172 hardware constraints (V100: 48 KB smem per block, 255 registers/thread)
        const double smem = 8.0 * (TBx * TBk * REGx + TBy * TBk * REGy);
        bool ok = smem <= 48 * 1024 && REGx * REGy <= 64 && TBx * TBy <= 1024;
        // enough thread blocks (R16: at least one wave of the running GPU)
        ok &= (double)cfg.nctas >= kSMs;
        // it must also map onto one of the compiled B200 kernels
        int vi_best = -1;
        Config fit;
        if (ok) {
          for (int vi = 0; vi < (int)variants().size(); vi++) {
            if (forced_variant >= 0 && vi != forced_variant) continue;
            if (!fits(cfg, variants()[vi])) continue;
            Config t = cfg;
            evaluate(c, t, vi);
            if (vi_best < 0 || better(t, fit)) { fit = t; vi_best = vi; }
          }
        }
        if (!ok || vi_best < 0) { st.pruned++; continue; }
        fit.paper_cost = paper_alg3_cost(c, fit, [&] { std::vector<int> v; for (auto &q : x.tb) v.push_back(q.first); return v; }(),
                                         [&] { std::vector<int> v; for (auto &q : x.reg) v.push_back(q.first); return v; }(),
                                         [&] { std::vector<int> v; for (auto &q : y.tb) v.push_back(q.first); return v; }(),
                                         [&] { std::vector<int> v; for (auto &q : y.reg) v.push_back(q.first); return v; }());
        fit.paper_mapping = "TB_x=" + tiling_str(c, x.tb) + " REG_x=" + tiling_str(c, x.reg) +
                            " TB_y=" + tiling_str(c, y.tb) + " REG_y=" + tiling_str(c, y.reg) +
                            " TB_k=" + tiling_str(c, k);
        st.ranked++;
        bool win = !found || fit.paper_cost < best.paper_cost ||
                   (fit.paper_cost == best.paper_cost && better(fit, best));
        if (win) { best = fit; found = true; }
      }
  return found ? ST_OK : ST_NO_CONFIG;
}

// ---------------------------------------------------------------- forced tiles
static Status choose_forced(const Contraction &c, const ForcedTiles &ft, int forced_variant,
                            Config &best, std::string &err) {
  Config cfg;
  digit_orders(c, cfg);
  cfg.T.assign(c.ix.size(), 1);
  for (size_t id = 0; id < c.ix.size(); id++) {
    auto it = ft.tile.find(c.ix[id].name);
    if (it != ft.tile.end()) cfg.T[id] = (int)std::max<int64_t>(1, std::min<int64_t>(it->second, c.ix[id].n));
  }
  finish(c, cfg);
  bool found = false;
  for (int vi = 0; vi < (int)variants().size(); vi++) {
    if (forced_variant >= 0 && vi != forced_variant) continue;
    if (!fits(cfg, variants()[vi])) continue;
    Config t = cfg;
    evaluate(c, t, vi);
    if (!found || better(t, best)) { best = t; found = true; }
  }
  if (!found) { err = "forced tiles fit no compiled kernel variant"; return ST_NO_CONFIG; }
  return ST_OK;
}

Status choose(const Contraction &c, int cost_mode, int forced_variant, const ForcedTiles &ft,
              Config &out, PlanStats &stats, std::string &err) {
  auto t0 = std::chrono::steady_clock::now();
  stats = PlanStats();
  stats.cost_mode = cost_mode;
  Status s;
  if (ft.on) s = choose_forced(c, ft, forced_variant, out, err);
  else if (cost_mode == 1) s = choose_paper(c, forced_variant, out, stats);
  else s = choose_b200(c, forced_variant, out, stats);
  if (s == ST_NO_CONFIG && !ft.on && cost_mode == 1) {
    // the paper's value sets can leave nothing after pruning (tiny problems): fall back to
    // the B200 enumeration so that every legal contraction gets a plan (R13)
    PlanStats st2;
    s = choose_b200(c, forced_variant, out, st2);
    stats.ranked += st2.ranked;
  }
  if (s != ST_OK && err.empty()) err = "no legal configuration";
  stats.plan_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return s;
}

}  // namespace tc
