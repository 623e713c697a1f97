// tiles.cpp — see tiles.hpp.
#include "tiles.hpp"

#include <algorithm>
#include <set>

namespace tc {

const std::vector<Variant> &variants() {
  // FP64 shapes from variants.def (must match the kernel instances of kernel_table.cuh);
  // BF16 x BF16 -> FP32 on tcgen05 (kernel_bf16.cuh): BM = 128 (UMMA M), BK = 64.
  static const std::vector<Variant> v = [] {
    std::vector<Variant> t(kNumVariants);
#define TC_F64_VARIANT(id, BM, BN, BK, WM, WN, ST, PW, OCC, STG) \
  t[id] = Variant{BM, BN, BK, WM, WN, ST, PW, OCC, KIND_F64_DMMA, STG};
#include "variants.def"
#undef TC_F64_VARIANT
    t[11] = Variant{128, 64, 64, 32, 32, 6, 4, 1, KIND_BF16_UMMA};
    t[12] = Variant{128, 128, 64, 32, 32, 5, 4, 1, KIND_BF16_UMMA};
    // TF32 (FP32 storage): same 128-B rows, BK = 32 elements
    t[21] = Variant{128, 64, 32, 32, 32, 6, 4, 1, KIND_TF32_UMMA};
    t[22] = Variant{128, 128, 32, 32, 32, 5, 4, 1, KIND_TF32_UMMA};
    // FP32 as split TF32 (hi + lo planes per stage: twice the smem per stage)
    t[23] = Variant{128, 64, 32, 32, 32, 3, 4, 1, KIND_F32X3_UMMA};
    t[24] = Variant{128, 128, 32, 32, 32, 2, 4, 1, KIND_F32X3_UMMA};
    // Calibration of the B200 model per FP64 variant: the median over the TCCG-48 cases of
    // measured / predicted time of the variant's best configuration (tools/model_calib.py on
    // one B200, profiles/r02_model_calib.jsonl; 10 ranked variants x 48 cases).  The model
    // counts pipes and bytes; what it misses (issue, latency, epilogue drains) is per kernel
    // shape.  With it the model's first choice is within 10 % of the fastest ranked variant on
    // 46 / 48 cases (leave-one-case-out fits: the same 46), against 3 / 48 without.
    const double cal[][2] = {{0, 1.094}, {1, 1.114}, {2, 1.284}, {3, 1.307}, {4, 1.132}, {5, 1.131},
                             {6, 1.383}, {7, 1.405}, {8, 1.557}, {9, 1.539}, {10, 1.220}, {13, 1.840},
                             {14, 1.802}, {15, 1.842}, {16, 2.766}, {17, 1.924}, {18, 1.351},
                             {19, 2.392}, {20, 2.108}, {25, 1.374}, {26, 2.862}};
    for (auto &c : cal) t[(int)c[0]].cal = c[1];
    return t;
  }();
  return v;
}

static int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

void digit_orders(const Contraction &c, Config &cfg) {
  // X = the input holding C's FVI — the first non-batch index of C
  int cf = -1;
  for (int id : c.t[0].idx)
    if (c.ix[id].cls != BATCH) { cf = id; break; }
  cfg.X = cf < 0 ? 1 : (c.pos_in(1, cf) >= 0 ? 1 : 2);
  cfg.Y = 3 - cfg.X;
  cfg.mdig.clear();
  cfg.ndig.clear();
  cfg.kdig.clear();
  const auto &xv = c.t[cfg.X].idx, &yv = c.t[cfg.Y].idx;
  // m: C order puts C's FVI first (coalesced C rows); X order follows X's memory
  // (coalesced, vectorisable X loads)
  if (cfg.morder == 0) {
    for (int id : c.t[0].idx) if (c.pos_in(cfg.X, id) >= 0 && is_ext(c.ix[id].cls)) cfg.mdig.push_back(id);
  } else {
    for (int id : xv) if (is_ext(c.ix[id].cls)) cfg.mdig.push_back(id);
  }
  // n: Y's memory order (C's FVI is never on the n side)
  for (int id : yv) if (is_ext(c.ix[id].cls)) cfg.ndig.push_back(id);
  // k: X's or Y's order of the internal indices
  for (int id : (cfg.korder == 0 ? xv : yv)) if (c.ix[id].cls == INTL) cfg.kdig.push_back(id);
  // smem layout: k-contiguous iff the operand's FVI is internal
  cfg.xKmajor = !xv.empty() && c.ix[xv[0]].cls == INTL;
  cfg.yKmajor = !yv.empty() && c.ix[yv[0]].cls == INTL;
}

void finish_counts(const Contraction &c, Config &cfg) {
  cfg.Mt = cfg.Nt = cfg.Kt = 1;
  cfg.mtiles = cfg.ntiles = cfg.nsteps = 1;
  for (int id : cfg.mdig) { cfg.Mt *= cfg.T[id]; cfg.mtiles *= cdiv(c.ix[id].n, cfg.T[id]); }
  for (int id : cfg.ndig) { cfg.Nt *= cfg.T[id]; cfg.ntiles *= cdiv(c.ix[id].n, cfg.T[id]); }
  for (int id : cfg.kdig) { cfg.Kt *= cfg.T[id]; cfg.nsteps *= cdiv(c.ix[id].n, cfg.T[id]); }
  cfg.nctas = cfg.mtiles * cfg.ntiles;
}

int vec_width(const Contraction &c, const Config &cfg, int t, int maxv) {
  // the operand's FVI leads its smem-contiguous dimension; tile, extent, every other stride
  // and the base divisible by the width (every vector aligned to its size)
  const auto &v = c.t[t];
  if (v.idx.empty() || v.stride[0] != 1) return 1;
  const int f = v.idx[0];
  const bool isk = c.ix[f].cls == INTL;
  const bool kmaj = t == cfg.X ? cfg.xKmajor : cfg.yKmajor;
  if (isk != kmaj) return 1;
  const auto &lst = isk ? cfg.kdig : (t == cfg.X ? cfg.mdig : cfg.ndig);
  if (lst.empty() || lst[0] != f) return 1;
  for (int w = maxv; w >= 2; w /= 2) {
    bool ok = cfg.T[f] % w == 0 && c.ix[f].n % w == 0 && v.base % w == 0;
    for (size_t p = 1; p < v.stride.size(); p++) ok &= v.stride[p] % w == 0;
    if (ok) return w;
  }
  return 1;
}

int c_vec_width(const Contraction &c, const Config &cfg, int maxv) {
  const auto &v = c.t[0];
  if (v.idx.empty() || v.stride[0] != 1 || cfg.mdig.empty() || cfg.mdig[0] != v.idx[0]) return 1;
  const int f = v.idx[0];
  for (int w = maxv; w >= 2; w /= 2) {
    bool ok = cfg.T[f] % w == 0 && c.ix[f].n % w == 0 && v.base % w == 0;
    for (size_t p = 1; p < v.stride.size(); p++) ok &= v.stride[p] % w == 0;
    if (ok) return w;
  }
  return 1;
}

int c_run_rows(const Contraction &c, const Config &cfg, int w, int *s0, int *t0) {
  const auto &v = c.t[0];
  *s0 = 1;
  *t0 = 1;
  if (v.idx.empty() || v.stride[0] != 1) return 1;
  const int f = v.idx[0];
  int stride = 1;
  bool found = false;
  for (int id : cfg.mdig) {
    if (id == f) { found = true; break; }
    stride *= cfg.T[id];
  }
  if (!found) return 1;
  bool ok = cfg.T[f] % w == 0 && c.ix[f].n % w == 0 && v.base % w == 0;
  for (size_t p = 1; p < v.stride.size(); p++) ok &= v.stride[p] % w == 0;
  // the CTA-wide staged path gives every one of its 256 threads one run: Mt / w runs must
  // divide 256
  if (stride > 1) {
    const int64_t nr = cfg.Mt / w;
    ok &= cfg.Mt % w == 0 && nr > 0 && nr <= 256 && (nr & (nr - 1)) == 0;
  }
  if (!ok) return 1;
  *s0 = stride;
  *t0 = cfg.T[f];
  return w;
}

bool vec_possible(const Contraction &c, const Config &cfg, int t) { return vec_width(c, cfg, t, 2) == 2; }

SlotTable build_slots(const Contraction &c, const Config &cfg, int t, int vec, bool kmajor,
                      int BMN, int BK) {
  SlotTable out;
  const auto &v = c.t[t];
  const auto &side = t == cfg.X ? cfg.mdig : cfg.ndig;
  const int r = (int)v.idx.size();
  std::vector<int> T(r), mul(r), isk(r);
  std::vector<int64_t> st(r);
  for (int p = 0; p < r; p++) {
    const int id = v.idx[p];
    T[p] = cfg.T[id];
    isk[p] = c.ix[id].cls == INTL;
    st[p] = v.stride[p];
    const auto &lst = isk[p] ? cfg.kdig : side;
    int m = 1;
    for (int q : lst) {
      if (q == id) break;
      m *= cfg.T[q];
    }
    mul[p] = m;
  }
  // packed slot: smem offset (elements) | k | row; FP64: 13 | 6 | 13 bits, UMMA: 14 | 6 | 12
  const int kshift = is_umma(cfg.kind) ? 14 : 13, mshift = is_umma(cfg.kind) ? 20 : 19;
  int64_t nslot = 1;
  for (int p = 0; p < r; p++) nslot *= p == 0 ? (T[p] + vec - 1) / vec : T[p];
  out.rel.reserve(nslot);
  out.pack.reserve(nslot);
  std::vector<int> d(r, 0);
  for (;;) {
    int mn = 0, k = 0;
    int64_t rel = 0;
    for (int p = 0; p < r; p++) {
      (isk[p] ? k : mn) += d[p] * mul[p];
      rel += d[p] * st[p];
    }
    out.rel.push_back(rel);
    out.pack.push_back((uint32_t)smem_off(cfg.kind, kmajor, mn, k, BMN, BK) | ((uint32_t)k << kshift) |
                       ((uint32_t)mn << mshift));
    int p = 0;
    for (; p < r; p++) {
      d[p] += (p == 0 ? vec : 1);
      if (d[p] < T[p]) break;
      d[p] = 0;
    }
    if (p == r) break;
  }
  return out;
}

double slot_sectors(const SlotTable &s, int vec, int esize) {
  const size_t n = s.rel.size();
  double total = 0;
  int64_t sec[64];
  for (size_t b = 0; b < n; b += 32) {
    const size_t e = std::min(n, b + 32);
    int k = 0;
    for (size_t i = b; i < e; i++) {
      sec[k++] = (s.rel[i] * esize) >> 5;
      sec[k++] = (s.rel[i] * esize + esize * vec - 1) >> 5;
    }
    std::sort(sec, sec + k);
    total += (double)(std::unique(sec, sec + k) - sec);
  }
  return total;
}

double slot_wavefronts(const SlotTable &s, int vec, int esize, int kind) {
  // per warp instruction (32 slots): the words each of the 32 banks serves.  The slots of a
  // table are distinct tile elements (build_slots: no padding slots), so their words are
  // distinct: a histogram per bank, no sort (the planner simulates every table it ranks).
  const size_t n = s.pack.size();
  double total = 0;
  for (size_t b = 0; b < n; b += 32) {
    const size_t e = std::min(n, b + 32);
    int cnt[32] = {0};
    for (size_t i = b; i < e; i++) {
      const uint32_t byte0 = slot_off(s.pack[i], kind) * (uint32_t)esize;
      for (uint32_t w = byte0 / 4; w < (byte0 + (uint32_t)(esize * vec) + 3) / 4; w++) cnt[w & 31]++;
    }
    int wf = 0;
    for (int k = 0; k < 32; k++) wf = std::max(wf, cnt[k]);
    const int minwf = (int)(((e - b) * esize * vec + 127) / 128);
    total += std::max(wf, minwf);
  }
  return total;
}

TileTables build_tile_tables(const Contraction &c, const Config &cfg, const Variant &v) {
  TileTables tt;
  const int X = cfg.X, Y = cfg.Y;
  // TMA epilogue: C as a tensor of its own dims (C order), the tile as the box
  const auto &cv = c.t[0];
  const int crank = (int)cv.idx.size();
  tt.tma_ok = crank >= 1 && crank <= kMaxTmaDims && cv.stride[0] == 1 && cfg.T[cv.idx[0]] % 2 == 0;
  for (int p = 1; p < crank && tt.tma_ok; p++)
    tt.tma_ok = (cv.stride[p] * 8) % 16 == 0 && cv.stride[p] * 8 < (1ll << 40);
  for (int p = 0; p < crank && tt.tma_ok; p++) tt.tma_ok = c.ix[cv.idx[p]].n < (1ll << 31);
  std::vector<int64_t> boxst(crank, 1);              // box strides (elements)
  for (int p = 1; p < crank; p++) boxst[p] = boxst[p - 1] * cfg.T[cv.idx[p - 1]];
  auto side = [&](const std::vector<int> &dig, int op, int64_t opbase, int64_t cbase,
                  std::vector<TileInfo> &tiles, std::vector<int64_t> &relC,
                  std::vector<int32_t> &box, int BMN) {
    const int nd = (int)dig.size();
    std::vector<int64_t> nt(nd);
    int64_t ntot = 1;
    for (int i = 0; i < nd; i++) {
      nt[i] = cdiv(c.ix[dig[i]].n, cfg.T[dig[i]]);
      ntot *= nt[i];
    }
    // tile-local digits, C offsets and smem-box offsets of every row (column) of the tile
    int64_t tot = 1;
    for (int id : dig) tot *= cfg.T[id];
    relC.assign(BMN, 0);
    box.assign(BMN, 0);
    std::vector<std::vector<int>> rd(std::min<int64_t>(tot, BMN), std::vector<int>(nd));
    for (int64_t r = 0; r < tot && r < BMN; r++) {
      int64_t q = r, off = 0, bo = 0;
      for (int i = 0; i < nd; i++) {
        rd[r][i] = (int)(q % cfg.T[dig[i]]);
        q /= cfg.T[dig[i]];
        off += rd[r][i] * c.stride_of(0, dig[i]);
        bo += rd[r][i] * boxst[c.pos_in(0, dig[i])];
      }
      relC[r] = off;
      box[r] = (int32_t)bo;
    }
    tiles.resize(ntot);
    std::vector<int64_t> cd(nd, 0);
    std::vector<int64_t> lim(nd);
    for (int64_t t = 0; t < ntot; t++) {
      TileInfo ti{opbase, cbase, {0, 0}, {0, 0, 0, 0, 0}, 0};
      for (int i = 0; i < nd; i++) {
        const int id = dig[i];
        const int64_t o = cd[i] * cfg.T[id];
        ti.op += o * c.stride_of(op, id);
        ti.c += o * c.stride_of(0, id);
        lim[i] = std::min<int64_t>(cfg.T[id], c.ix[id].n - o);
        const int p = c.pos_in(0, id);
        if (p >= 0 && p < kMaxTmaDims) ti.coord[p] = (int32_t)o;
      }
      bool full = true;
      for (int i = 0; i < nd; i++) full &= lim[i] == cfg.T[dig[i]];
      if (full && t > 0) {
        // interior tile: same rows as tile 0 (the origin tile is always interior, T <= N)
        ti.mask[0] = tiles[0].mask[0];
        ti.mask[1] = tiles[0].mask[1];
      } else {
        for (size_t r = 0; r < rd.size(); r++) {
          bool ok = true;
          for (int i = 0; i < nd; i++) ok &= rd[r][i] < lim[i];
          if (ok) ti.mask[r >> 6] |= 1ull << (r & 63);
        }
      }
      tiles[t] = ti;
      for (int i = 0; i < nd; i++) {
        if (++cd[i] < nt[i]) break;
        cd[i] = 0;
      }
    }
  };
  side(cfg.mdig, X, c.t[X].base, c.t[0].base, tt.tileM, tt.relCm, tt.boxM, v.BM);
  side(cfg.ndig, Y, c.t[Y].base, 0, tt.tileN, tt.relCn, tt.boxN, v.BN);
  // k steps
  const int nk = (int)cfg.kdig.size();
  std::vector<int64_t> kt(nk), kn(nk);
  for (int i = 0; i < nk; i++) {
    kn[i] = c.ix[cfg.kdig[i]].n;
    kt[i] = cfg.T[cfg.kdig[i]];
  }
  const int Kt = (int)cfg.Kt;
  const uint64_t full = Kt >= 64 ? ~0ull : ((1ull << Kt) - 1);
  // per digit: tile count, offset per tile step and the k-mask factor at its last tile
  std::vector<int64_t> cnt(nk), dx(nk), dy(nk);
  std::vector<uint64_t> tail(nk);
  int64_t inner = 1;                      // product of the tiles of the faster k digits
  for (int i = 0; i < nk; i++) {
    cnt[i] = cdiv(kn[i], kt[i]);
    const int64_t rem = kn[i] - (cnt[i] - 1) * kt[i];
    dx[i] = kt[i] * c.stride_of(X, cfg.kdig[i]);
    dy[i] = kt[i] * c.stride_of(Y, cfg.kdig[i]);
    uint64_t m = 0;
    for (int k = 0; k < Kt; k++)
      if ((k / inner) % kt[i] < rem) m |= 1ull << k;
    tail[i] = m & full;
    inner *= kt[i];
  }
  tt.kbase = full;
  std::vector<int> moving;
  for (int i = 0; i < nk; i++) {
    if (cnt[i] == 1) tt.kbase &= tail[i];   // fixed digit: its (partial) range always applies
    else moving.push_back(i);
  }
  tt.kcnt0 = 1;
  tt.ktail0 = tt.kbase;
  size_t first_outer = 0;
  if (!moving.empty()) {
    const int i = moving[0];
    tt.kcnt0 = (int)cnt[i];
    tt.kdX0 = dx[i];
    tt.kdY0 = dy[i];
    tt.ktail0 = tt.kbase & tail[i];
    first_outer = 1;
  }
  // outer moving digits: every combination, first outer digit fastest
  std::vector<int64_t> od(moving.size(), 0);
  for (;;) {
    KOuter e{0, 0, ~0ull};
    for (size_t q = first_outer; q < moving.size(); q++) {
      const int i = moving[q];
      e.x += od[q] * dx[i];
      e.y += od[q] * dy[i];
      if (od[q] == cnt[i] - 1) e.mask &= tail[i];
    }
    tt.kouter.push_back(e);
    size_t q = first_outer;
    for (; q < moving.size(); q++) {
      if (++od[q] < cnt[moving[q]]) break;
      od[q] = 0;
    }
    if (q == moving.size()) break;
  }
  return tt;
}

// tcgen05 operand t loaded by TMA boxes straight into its 128-B swizzled UMMA plane
// (kernel_umma.cuh, TMA producer).  The map's dimension 0 is the operand's FVI (stride 1);
// the others may come in any order, so they follow the plane's row order:
//   K-major  (FVI = the k index): [k | side digits in compute order], box (BK, T...)  —
//            (a k tile below BK loads the next step's k too; the MMAs never read them)
//            tile-local row r = mixed radix over the side digits = box row r (128 B each);
//   MN-major (FVI = side[0]):     [side[0] | k | side[1..]], box (E, Kt, T...) — one 128-B
//            atom column per E elements of side[0]; wider tiles of side[0] (the other side
//            digits then untiled) take ceil(T0/E) boxes, each BK * 128 B further on.
// Conditions: one k digit whose tile is a multiple of the MMA K or its whole extent (TMA
// zero-fills past the end, as the cp.async producers do), no batch index, rank <= 5, side digits among
// C's first 5 positions (the tile origin coordinates), 16-B multiple strides.  The split
// FP32 kind converts in smem and keeps its cp.async producers.
bool umma_tma_spec(const Contraction &c, const Config &cfg, const Variant &v, int t, OperandMap *mp,
                   TmaOperand *op) {
  const bool kmaj = t == cfg.X ? cfg.xKmajor : cfg.yKmajor;
  const std::vector<int> &side = t == cfg.X ? cfg.mdig : cfg.ndig;
  OperandMap mloc;
  TmaOperand oloc;
  OperandMap &m = mp ? *mp : mloc;
  TmaOperand &o = op ? *op : oloc;
  if (cfg.kind != KIND_BF16_UMMA && cfg.kind != KIND_TF32_UMMA) return false;
  if (cfg.kdig.size() != 1 || c.nbatch() != 1 || side.empty()) return false;
  const int es = kind_esize(cfg.kind), E = 128 / es, kid = cfg.kdig[0];
  const TensorView &tv = c.t[t];
  const int r = (int)tv.idx.size();
  if (r > kMaxTmaDims || tv.stride[0] != 1) return false;
  // the MMAs consume ceil(Kt / KI) * KI k of a stage: k past Kt must be absent (zero-filled
  // past the extent) or never read (Kt a multiple of KI)
  const int Kt = cfg.T[kid], KI = 32 / es;
  if (Kt > v.BK || (Kt % KI != 0 && Kt != c.ix[kid].n)) return false;
  std::vector<int> dims;
  if (kmaj) {
    dims.push_back(kid);
    dims.insert(dims.end(), side.begin(), side.end());
  } else {
    dims.push_back(side[0]);
    dims.push_back(kid);
    dims.insert(dims.end(), side.begin() + 1, side.end());
  }
  if ((int)dims.size() != r || dims[0] != tv.idx[0]) return false;
  // a box's start along map dim 0 must sit on a 16-B boundary: the tile (MN-major) or k-step
  // (K-major) origins along it move in multiples of 16 B
  const int a16 = 16 / es;
  if (kmaj ? (Kt % a16 != 0 && Kt < c.ix[kid].n) : (cfg.T[side[0]] % a16 != 0 && cfg.T[side[0]] < c.ix[side[0]].n))
    return false;
  const int T0 = cfg.T[side[0]];
  int nsub = 1;
  bool rest1 = true;
  for (size_t q = 1; q < side.size(); q++) rest1 &= cfg.T[side[q]] == 1;
  // k extent of the box: an MN-major box of one atom column may stop at Kt (its k rows are
  // the stage's first Kt rows); otherwise the box spans BK so that a multi-digit box lands its
  // atom columns BK rows apart, as the plane expects (the extra k are never read)
  const uint32_t kbox = !kmaj && rest1 && Kt % KI == 0 ? (uint32_t)Kt : (uint32_t)v.BK;
  if (!kmaj) {
    if (rest1) {
      nsub = (T0 + E - 1) / E;          // (atom columns past T0: rows / columns never stored)
    } else if (T0 != E) {
      return false;                     // other atom widths would interleave the digits
    }
  }
  uint32_t pack = 0, tx = (uint32_t)es;
  for (int j = 0; j < r; j++) {
    const int id = dims[j];
    const int sp = c.pos_in(t, id);
    if (sp < 0) return false;
    m.dims[j] = c.ix[id].n;
    if (j > 0) {
      const int64_t sb = tv.stride[sp] * es;
      if (sb % 16 != 0 || sb >= (int64_t(1) << 40)) return false;
      m.strides[j - 1] = sb;
    }
    uint32_t src;
    if (id == kid) {
      src = 7;
      m.box[j] = kbox;
    } else {
      const int cp = c.pos_in(0, id);
      if (cp < 0 || cp >= kMaxTmaDims) return false;
      src = (uint32_t)cp;
      m.box[j] = (uint32_t)(j == 0 ? E : cfg.T[id]);
    }
    if (m.box[j] > 256) return false;
    pack |= src << (3 * j);
    tx *= m.box[j];
  }
  m.rank = r;
  m.base = tv.base;
  m.swz32 = !kmaj && es == 4;
  o.pack = pack | ((uint32_t)r << 16);
  o.nsub = nsub;
  o.sub_bytes = E * v.BK * es;
  o.sub_crd = E;
  o.tx = (int)tx;
  return true;
}

}  // namespace tc
