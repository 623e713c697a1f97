// group.cpp — planner of the fused grouped contraction (see group.hpp).
//
// Enumerate -> prune -> cost, as for one contraction, but over the tile of the
// SHARED output: one tile T_p per C position, such that every member's Mt_i (product over
// the C positions of its operand X_i) and Nt_i fit the 64 x 64 DMMA register tiles; ranked
// by the number of C tiles (each tile costs every member's k-steps once) and padding.  Per
// member and per load mode (TMA boxes / cp.async gathers), the digit order of rows and
// columns is chosen by simulating the shared-memory wavefronts of the stage writes (cp.async),
// of the DMMA fragment loads (TMA: swizzled boxes in the operand's own order) and of the
// member's read-modify-write of the swizzled C box.
#include "group.hpp"

#include <algorithm>
#include <chrono>
#include <cmath>
#include <functional>
#include <map>
#include <set>

namespace tc {

namespace {

int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Shared-memory wavefronts of a sequence of warp instructions: entries (byte offset, bytes)
// in lane order, 32 per instruction; a bank (4-byte words, 32 banks) serves one word per
// wavefront.  The entries of one instruction are distinct elements (their words differ):
// a histogram per bank.
double smem_wavefronts(const std::vector<std::pair<int64_t, int>> &acc) {
  double total = 0;
  for (size_t b = 0; b < acc.size(); b += 32) {
    const size_t e = std::min(acc.size(), b + 32);
    int cnt[32] = {0};
    int64_t bytes = 0;
    for (size_t i = b; i < e; i++) {
      for (int64_t w = acc[i].first / 4; w < (acc[i].first + acc[i].second + 3) / 4; w++) cnt[w & 31]++;
      bytes += acc[i].second;
    }
    int wf = 0;
    for (int k = 0; k < 32; k++) wf = std::max(wf, cnt[k]);
    total += (double)std::max<int64_t>(wf, (bytes + 127) / 128);
  }
  return total;
}

struct Member {
  const Contraction *c = nullptr;
  int X = 1, Y = 2;               // tensor ids (1 = A, 2 = B)
  std::vector<int> mpos, npos;    // C positions held by X / Y
  std::vector<int> kid;           // internal index ids, in k-digit order
  std::vector<int> Tk;            // k tile per kid
  int64_t nsteps = 1;
};

// Operand description: dims in the operand's memory order.
struct OpDim {
  int id;          // member-local index id
  int cpos;        // C position, or -1 (internal)
  int64_t tile, n, gstride, sstride;
};

// cp.async planes: smem element offset of (row, k) — k-major rows of pitch BK + 4, or
// mn-major k rows of pitch BMN + 4 (4 mod 16 doubles: conflict-free DMMA fragment loads, as
// in the single-contraction kernel).
int64_t plane_off(bool kmajor, int64_t row, int64_t k, int BMN, int BK) {
  return kmajor ? row * (BK + 4) + k : k * (BMN + 4) + row;
}

// row multiplier of C position p in a digit order (product of the tiles before it)
int64_t row_mul(const std::vector<int> &ord, const int32_t *T, int p) {
  int64_t mul = 1;
  for (int q : ord) {
    if (q == p) break;
    mul *= T[q];
  }
  return mul;
}

// The dims of operand t of member M (cp.async planes: sstride = smem element stride).
std::vector<OpDim> op_dims(const Member &M, int t, const std::vector<int> &roword, const int32_t *T,
                           bool kmajor, int BMN, int BK) {
  const Contraction &c = *M.c;
  std::vector<OpDim> d;
  for (size_t j = 0; j < c.t[t].idx.size(); j++) {
    const int id = c.t[t].idx[j];
    OpDim o{id, c.pos_in(0, id), 1, c.ix[id].n, c.t[t].stride[j], 0};
    if (o.cpos >= 0) {
      o.tile = T[o.cpos];
      o.sstride = plane_off(kmajor, row_mul(roword, T, o.cpos), 0, BMN, BK);
    } else {
      int64_t mul = 1;
      for (size_t q = 0; q < M.kid.size(); q++) {
        if (M.kid[q] == id) { o.tile = M.Tk[q]; break; }
        mul *= M.Tk[q];
      }
      o.sstride = plane_off(kmajor, 0, mul, BMN, BK);
    }
    d.push_back(o);
  }
  return d;
}

struct Runs {
  std::vector<int32_t> rel;
  std::vector<uint32_t> soff;
  std::vector<uint64_t> dig;
  int runlen = 1, vec = 1;
};

// cp.async runs along dim 0 (when it is smem-contiguous), enumerated over dims 1.. (first
// fastest).
Runs build_runs(const std::vector<OpDim> &d, int64_t base, std::string &err, bool &ok) {
  Runs r;
  ok = true;
  if (d.empty()) {
    r.rel.push_back(0);
    r.soff.push_back(0);
    r.dig.push_back(0);
    return r;
  }
  const bool contiguous = d[0].sstride == 1;
  r.runlen = contiguous ? (int)d[0].tile : 1;
  const size_t first = contiguous ? 1 : 0;
  bool ev = contiguous && d[0].tile % 2 == 0 && d[0].n % 2 == 0 && base % 2 == 0;
  for (size_t j = 1; j < d.size(); j++) ev &= d[j].gstride % 2 == 0;
  r.vec = ev ? 2 : 1;
  std::vector<int64_t> dg(d.size(), 0);
  for (;;) {
    int64_t rel = 0, so = 0;
    uint64_t pk = 0;
    for (size_t j = first; j < d.size(); j++) {
      rel += dg[j] * d[j].gstride;
      so += dg[j] * d[j].sstride;
      pk |= (uint64_t)dg[j] << (8 * j);
    }
    if (rel > INT32_MAX || rel < INT32_MIN) { err = "operand tile spans more than 2^31 elements"; ok = false; return r; }
    r.rel.push_back((int32_t)rel);
    r.soff.push_back((uint32_t)so);
    r.dig.push_back(pk);
    size_t j = first;
    for (; j < d.size(); j++) {
      if (++dg[j] < d[j].tile) break;
      dg[j] = 0;
    }
    if (j == d.size()) break;
  }
  return r;
}

// cp.async stage-write wavefronts of one operand: vectors w in order, warp = 32 consecutive w.
double runs_wavefronts(const Runs &r, int64_t plane_byte0) {
  std::vector<std::pair<int64_t, int>> acc;
  const int vpr = r.runlen / r.vec;
  for (size_t q = 0; q < r.rel.size(); q++)
    for (int v = 0; v < vpr; v++) acc.push_back({plane_byte0 + 8 * ((int64_t)r.soff[q] + v * r.vec), 8 * r.vec});
  return smem_wavefronts(acc);
}

// digit values of row r in a digit order
std::vector<int64_t> row_digits(int64_t r, const std::vector<int> &order, const int32_t *T) {
  std::vector<int64_t> d(kGMaxCdims, 0);
  for (int p : order) {
    d[p] = r % T[p];
    r /= T[p];
  }
  return d;
}

// box offset of every row (column) of a member tile, from the digit order and the tiles
std::vector<int32_t> row_box(const std::vector<int> &order, const int32_t *T, const int64_t *bst, int BMN) {
  std::vector<int32_t> out(BMN, -1);
  int64_t tot = 1;
  for (int p : order) tot *= T[p];
  for (int64_t r = 0; r < tot && r < BMN; r++) {
    const auto d = row_digits(r, order, T);
    int64_t o = 0;
    for (int p : order) o += d[p] * bst[p];
    out[r] = (int32_t)o;
  }
  return out;
}

// member RMW of the box: 4 consumer warps (2 x 2 of 32 x 32), each the DMMA m8n8k4
// accumulator layout (lane g = row i*8 + g, t = column pair 2t + h); load + store
double flush_wavefronts(const std::vector<int32_t> &R, const std::vector<int32_t> &Q) {
  double total = 0;
  for (int wm = 0; wm < 2; wm++)
    for (int wn = 0; wn < 2; wn++)
      for (int i = 0; i < 4; i++)
        for (int jj = 0; jj < 4; jj++)
          for (int h = 0; h < 2; h++) {
            std::vector<std::pair<int64_t, int>> acc;
            for (int lane = 0; lane < 32; lane++) {
              const int g = lane >> 2, t = lane & 3;
              const int r = R[wm * 32 + i * 8 + g], c = Q[wn * 32 + jj * 8 + 2 * t + h];
              if (r >= 0 && c >= 0) acc.push_back({8 * (int64_t)gbox_sw(r + c), 8});
            }
            if (!acc.empty()) total += 2 * smem_wavefronts(acc);
          }
  return total;
}

// TMA box layout of one operand: the tensor map lists the operand's dims in the order perm
// (perm[0] = 0, the FVI; dims 1.. permuted — the map's strides need not grow), the box is the
// tile (a k-FVI box padded to a pitch of 4 mod 8 doubles), dense in smem in the map's order,
// no swizzle: the order is chosen so that the DMMA fragment loads are conflict-free.
struct TmaLayout {
  bool ok = false;
  std::vector<int> perm;        // map dim j -> operand dim perm[j]
  std::vector<int64_t> box;     // box extent per map dim
  std::vector<int64_t> bs;      // element stride inside the box of each OPERAND dim
  int64_t bytes = 0;
  int64_t byte(const std::vector<int64_t> &d) const {
    int64_t o = 0;
    for (size_t j = 0; j < d.size(); j++) o += d[j] * bs[j];
    return 8 * o;
  }
};

int64_t kpitch(int64_t t) {   // smallest p >= t with p = 4 (mod 8): conflict-free k-major rows
  int64_t p = t;
  while (p % 8 != 4) p++;
  return p;
}

bool tma_eligible(const std::vector<OpDim> &d, int64_t base) {
  if (d.empty() || d.size() > (size_t)kGMaxTmaDims || d[0].gstride != 1 || base % 2 != 0) return false;
  if (d[0].cpos >= 0 && d[0].tile % 2 != 0) return false;          // box dim 0: 16-B multiple
  for (size_t j = 1; j < d.size(); j++)
    if (d[j].gstride % 2 != 0 || d[j].gstride * 8 >= (1ll << 40)) return false;
  for (auto &x : d)
    if (x.n >= (1ll << 32) || x.tile > 256 || kpitch(x.tile) > 256) return false;
  return true;
}

TmaLayout tma_make(const std::vector<OpDim> &d, const std::vector<int> &perm) {
  TmaLayout L;
  L.perm = perm;
  L.box.assign(d.size(), 1);
  L.bs.assign(d.size(), 0);
  int64_t m = 1;
  for (size_t j = 0; j < perm.size(); j++) {
    const OpDim &x = d[perm[j]];
    L.box[j] = (j == 0 && x.cpos < 0) ? kpitch(x.tile) : x.tile;
    L.bs[perm[j]] = m;
    m *= L.box[j];
  }
  L.bytes = 8 * m;
  L.ok = true;
  return L;
}

// DMMA fragment-load wavefronts of one operand tile in smem: per row group i (8 rows) and k4
// step, thread (g, t) loads element (row 8i + g, k 4kk + t); rowe / ke are element offsets;
// 32 doubles need >= 2 wavefronts, and each bank pair serves one distinct double per wavefront
double frag_wavefronts(const std::vector<int64_t> &rowe, const std::vector<int64_t> &ke, int kq) {
  double total = 0;
  for (int i = 0; i < 8; i++)
    for (int kk = 0; kk < kq; kk++) {
      int64_t seen[16][32];
      int cnt[16] = {0};
      int wf = 2;
      for (int lane = 0; lane < 32; lane++) {
        const int g = lane >> 2, t = lane & 3;
        const int64_t a = rowe[i * 8 + g] + ke[kk * 4 + t];
        const int b = (int)(a & 15);
        bool dup = false;
        for (int q = 0; q < cnt[b]; q++) dup |= seen[b][q] == a;
        if (!dup) {
          seen[b][cnt[b]++] = a;
          wf = std::max(wf, cnt[b]);
        }
      }
      total += wf;
    }
  return total;
}

std::vector<std::vector<int>> orders_with_first(const std::vector<int> &pos, int first, size_t cap) {
  std::vector<int> rest;
  for (int p : pos) if (p != first) rest.push_back(p);
  std::sort(rest.begin(), rest.end());
  std::vector<std::vector<int>> out;
  do {
    std::vector<int> o;
    if (first >= 0) o.push_back(first);
    o.insert(o.end(), rest.begin(), rest.end());
    out.push_back(o);
    if (out.size() >= cap) break;
  } while (std::next_permutation(rest.begin(), rest.end()));
  return out;
}

}  // namespace

Status plan_group(const std::vector<const Contraction *> &members, GroupTables &g, std::string &err) {
  const auto t0 = std::chrono::steady_clock::now();
  g = GroupTables();
  const int n = (int)members.size();
  if (n < 1 || n > kGMaxMembers) { err = "fused group: 1 to 32 members"; return ST_UNSUPPORTED; }
  const Contraction &c0 = *members[0];
  const int rank = (int)c0.t[0].idx.size();
  if (rank < 1 || rank > kGMaxCdims) { err = "fused group: C rank must be 1..8"; return ST_UNSUPPORTED; }
  g.rank = rank;
  for (int p = 0; p < rank; p++) {
    g.N[p] = c0.ix[c0.t[0].idx[p]].n;
    g.cstride[p] = c0.t[0].stride[p];
  }
  g.cbase = c0.t[0].base;

  // ---- members: X = the operand holding C position 0, rows / columns = the C
  //      positions of X / Y
  std::vector<Member> M(n);
  for (int i = 0; i < n; i++) {
    const Contraction &c = *members[i];
    M[i].c = &c;
    for (auto &ix : c.ix)
      if (ix.cls == BATCH) { err = "fused group: batch indices are not supported"; return ST_UNSUPPORTED; }
    if ((int)c.t[0].idx.size() != rank) { err = "fused group: C rank differs"; return ST_UNSUPPORTED; }
    if ((int)c.t[1].idx.size() > kGMaxOpDims || (int)c.t[2].idx.size() > kGMaxOpDims) {
      err = "fused group: operand rank > 8"; return ST_UNSUPPORTED;
    }
    const int id0 = c.t[0].idx[0];
    M[i].X = c.pos_in(1, id0) >= 0 ? 1 : 2;
    M[i].Y = 3 - M[i].X;
    for (int p = 0; p < rank; p++) {
      const int id = c.t[0].idx[p];
      (c.pos_in(M[i].X, id) >= 0 ? M[i].mpos : M[i].npos).push_back(p);
    }
    // k digits: the operand whose FVI is internal leads (its loads run along k)
    const auto &xv = c.t[M[i].X].idx, &yv = c.t[M[i].Y].idx;
    const bool xk = !xv.empty() && c.ix[xv[0]].cls == INTL, yk = !yv.empty() && c.ix[yv[0]].cls == INTL;
    const auto &ko = (!xk && yk) ? yv : xv;
    for (int id : ko) if (c.ix[id].cls == INTL) M[i].kid.push_back(id);
    g.flops += c.flops();
  }

  // ---- enumerate the C tile: T_p in {powers of two <= 64} u {N_p if <= 64}; prune by the
  //      member bounds Mt_i, Nt_i <= 64; rank by tiles, then padding, then a longer C run
  std::vector<std::vector<int32_t>> cand(rank);
  for (int p = 0; p < rank; p++) {
    std::set<int32_t> s;
    for (int t = 1; t <= 64 && t <= g.N[p]; t *= 2) s.insert(t);
    if (g.N[p] <= 64) s.insert((int32_t)g.N[p]);
    cand[p].assign(s.begin(), s.end());
  }
  std::vector<std::vector<char>> inX(n, std::vector<char>(rank, 0));
  for (int i = 0; i < n; i++)
    for (int p : M[i].mpos) inX[i][p] = 1;
  int32_t best[kGMaxCdims] = {}, cur[kGMaxCdims] = {};
  double bestTiles = 0, bestPad = 0;
  int64_t bestRun = 0;
  bool found = false;
  std::vector<int64_t> mprod(n, 1), nprod(n, 1);
  std::function<void(int)> dfs = [&](int p) {
    if (p == rank) {
      double tiles = 1, pad = 0;
      for (int q = 0; q < rank; q++) {
        tiles *= (double)cdiv(g.N[q], cur[q]);
        pad += (double)(cdiv(g.N[q], cur[q]) * cur[q] - g.N[q]) / (double)g.N[q];
      }
      const bool win = !found || tiles < bestTiles || (tiles == bestTiles && pad < bestPad) ||
                       (tiles == bestTiles && pad == bestPad && cur[0] > bestRun);
      if (win) {
        std::copy(cur, cur + rank, best);
        bestTiles = tiles;
        bestPad = pad;
        bestRun = cur[0];
        found = true;
      }
      return;
    }
    for (int32_t t : cand[p]) {
      bool ok = true;
      for (int i = 0; i < n && ok; i++) ok = (inX[i][p] ? mprod[i] : nprod[i]) * t <= (inX[i][p] ? kGBM : kGBN);
      if (!ok) continue;
      for (int i = 0; i < n; i++) (inX[i][p] ? mprod[i] : nprod[i]) *= t;
      cur[p] = t;
      dfs(p + 1);
      for (int i = 0; i < n; i++) (inX[i][p] ? mprod[i] : nprod[i]) /= t;
    }
  };
  dfs(0);
  if (!found) { err = "fused group: no common C tile fits"; return ST_UNSUPPORTED; }
  int64_t bst[kGMaxCdims];
  g.ntiles = 1;
  g.box = 1;
  for (int p = 0; p < rank; p++) {
    g.T[p] = best[p];
    g.ntl[p] = (int32_t)cdiv(g.N[p], best[p]);
    g.ntiles *= g.ntl[p];
    bst[p] = g.box;
    g.box *= best[p];
  }
  if (g.ntiles >= (1ll << 31)) { err = "fused group: more than 2^31 C tiles"; return ST_UNSUPPORTED; }

  // ---- BK (compiled: 16 and 24): fewest padded k-steps; per member the first k digit takes
  //      the tile with the fewest steps (the smallest such), the others fill up to BK
  auto ktiles = [&](const Member &m, int BK, std::vector<int> &Tk) {
    int64_t prod = 1, steps = 1;
    Tk.clear();
    for (size_t q = 0; q < m.kid.size(); q++) {
      const int64_t nk = m.c->ix[m.kid[q]].n;
      int64_t t;
      if (q == 0) {
        t = std::min<int64_t>(nk, BK);
        t = cdiv(nk, cdiv(nk, t));      // same steps, smallest tile: the padding goes
      } else {
        t = std::min<int64_t>(nk, std::max<int64_t>(1, BK / prod));
      }
      Tk.push_back((int)t);
      prod *= t;
      steps *= cdiv(nk, t);
    }
    return steps;
  };
  double bestK = 0;
  for (int BK : {24, 16}) {
    double cost = 0;
    std::vector<int> Tk;
    for (auto &m : M) {
      const int64_t steps = ktiles(m, BK, Tk);
      cost += (double)steps * BK + 4.0 * steps;   // (+ per-step hand-off)
    }
    if (bestK == 0 || cost < bestK) { bestK = cost; g.BK = BK; }
  }
  g.variant = g.BK == 16 ? 0 : 1;
  const int BK = g.BK;
  for (auto &m : M) m.nsteps = ktiles(m, BK, m.Tk);

  // ---- per member: digit orders (simulated smem wavefronts), runs, TMA boxes, steps, tables
  const int XS = gplane_doubles(kGBM, BK);
  g.tma = true;
  std::vector<TmaLayout> tlx(n), tly(n);
  std::vector<std::vector<int>> tord_m(n), tord_n(n), cord_m(n), cord_n(n);
  for (int i = 0; i < n; i++) {
    Member &m = M[i];
    const Contraction &c = *m.c;
    const auto &xv = c.t[m.X].idx, &yv = c.t[m.Y].idx;
    const bool xkm = !xv.empty() && c.ix[xv[0]].cls == INTL;
    const bool ykm = !yv.empty() && c.ix[yv[0]].cls == INTL;
    int64_t Kt = 1;
    for (int t : m.Tk) Kt *= t;
    const int kq = (int)cdiv(Kt, 4);
    // (a) cp.async planes: rows led by the operand's FVI (runs are smem-contiguous)
    const int xf = (!xv.empty() && !xkm) ? c.pos_in(0, xv[0]) : -1;
    const int yf = (!yv.empty() && !ykm) ? c.pos_in(0, yv[0]) : -1;
    double bestc = 0, bestFl = 0, bestLd = 0;
    for (auto &ro : orders_with_first(m.mpos, xf, 120))
      for (auto &co : orders_with_first(m.npos, yf, 120)) {
        const auto R = row_box(ro, g.T, bst, kGBM), Q = row_box(co, g.T, bst, kGBN);
        const double fl = flush_wavefronts(R, Q);
        bool ok1 = true, ok2 = true;
        const Runs rx = build_runs(op_dims(m, m.X, ro, g.T, xkm, kGBM, BK), c.t[m.X].base, err, ok1);
        const Runs ry = build_runs(op_dims(m, m.Y, co, g.T, ykm, kGBN, BK), c.t[m.Y].base, err, ok2);
        if (!ok1 || !ok2) return ST_UNSUPPORTED;
        const double ld = runs_wavefronts(rx, 0) + runs_wavefronts(ry, 8ll * XS);
        const double cost = fl + ld * (double)m.nsteps;
        if (cord_m[i].empty() || cost < bestc) { bestc = cost; cord_m[i] = ro; cord_n[i] = co; bestFl = fl; bestLd = ld; }
      }
    g.flushWf.push_back(bestFl);
    g.loadWf.push_back(bestLd);
    // (b) TMA boxes (one internal index, Kt a multiple of 4): per operand the map's dim order
    //     and the row order with the fewest fragment-load wavefronts, then among those the
    //     pair with the cheapest box read-modify-write
    const auto dx = op_dims(m, m.X, m.mpos, g.T, false, kGBM, BK), dy = op_dims(m, m.Y, m.npos, g.T, false, kGBN, BK);
    const bool tok = m.kid.size() <= 1 && Kt % 4 == 0 && tma_eligible(dx, c.t[m.X].base) &&
                     tma_eligible(dy, c.t[m.Y].base);
    g.tma = g.tma && tok;
    double bestT = -1;
    if (tok) {
      const int kidx = m.kid.empty() ? -1 : m.kid[0];
      struct Cand { TmaLayout L; std::vector<int> ord; double wf; };
      auto search = [&](int t, const std::vector<OpDim> &d, const std::vector<int> &pos, int BMN) {
        std::vector<int> rest;
        for (size_t q = 1; q < d.size(); q++) rest.push_back((int)q);
        std::vector<Cand> all;
        double bestwf = -1;
        do {
          std::vector<int> perm{0};
          perm.insert(perm.end(), rest.begin(), rest.end());
          const TmaLayout L = tma_make(d, perm);
          const int jk = kidx >= 0 ? c.pos_in(t, kidx) : -1;
          std::vector<int64_t> ke(32, 0);
          for (int k = 0; k < 32; k++) ke[k] = jk >= 0 ? (k < Kt ? k : 0) * L.bs[jk] : 0;
          for (auto &ord : orders_with_first(pos, -1, 120)) {
            std::vector<int64_t> rowe(BMN, 0);
            int64_t tot = 1;
            for (int p : ord) tot *= g.T[p];
            for (int64_t r = 0; r < tot && r < BMN; r++) {
              const auto dg = row_digits(r, ord, g.T);
              for (size_t q = 0; q < d.size(); q++)
                if (d[q].cpos >= 0) rowe[r] += dg[d[q].cpos] * L.bs[q];
            }
            const double wf = frag_wavefronts(rowe, ke, (int)cdiv(Kt, 4));
            if (bestwf < 0 || wf < bestwf) { bestwf = wf; all.clear(); }
            if (wf == bestwf && all.size() < 16) all.push_back({L, ord, wf});
          }
        } while (std::next_permutation(rest.begin(), rest.end()));
        return all;
      };
      const auto cx = search(m.X, dx, m.mpos, kGBM), cy = search(m.Y, dy, m.npos, kGBN);
      for (auto &a : cx)
        for (auto &b : cy) {
          const double cost = flush_wavefronts(row_box(a.ord, g.T, bst, kGBM), row_box(b.ord, g.T, bst, kGBN)) +
                              (double)m.nsteps * (a.wf + b.wf) * 4;
          if (bestT < 0 || cost < bestT) {
            bestT = cost;
            tlx[i] = a.L;
            tly[i] = b.L;
            tord_m[i] = a.ord;
            tord_n[i] = b.ord;
          }
        }
      g.tma_stage_bytes = (int)std::max<int64_t>(g.tma_stage_bytes, (tlx[i].bytes + 127) / 128 * 128 + tly[i].bytes);
    }
    g.fragWf.push_back(bestT);
  }

  for (int i = 0; i < n; i++) {
    Member &m = M[i];
    const Contraction &c = *m.c;
    const auto &xv = c.t[m.X].idx, &yv = c.t[m.Y].idx;
    const bool xkm = !xv.empty() && c.ix[xv[0]].cls == INTL;
    const bool ykm = !yv.empty() && c.ix[yv[0]].cls == INTL;
    int64_t Kt = 1;
    for (int t : m.Tk) Kt *= t;
    GMemberDev D{};
    D.xIsA = m.X == 1;
    D.kq = (int32_t)cdiv(Kt, 4);
    // cp.async side: runs in the cp.async digit order
    auto fill_op = [&](GOperandDev &o, int t, const std::vector<int> &ord, bool km, int BMN) -> bool {
      const auto dims = op_dims(m, t, ord, g.T, km, BMN, BK);
      bool ok = true;
      Runs r = build_runs(dims, c.t[t].base, err, ok);
      if (!ok) return false;
      for (int p = 0; p < rank; p++) o.tstep[p] = (int64_t)g.T[p] * c.stride_of(t, c.t[0].idx[p]);
      o.run0 = (int32_t)g.runRel.size();
      o.nrun = (int32_t)r.rel.size();
      o.runlen = r.runlen;
      o.vec = r.vec;
      o.ndim = (int32_t)dims.size();
      for (int j = 0; j < kGMaxOpDims; j++) o.cpos[j] = j < (int)dims.size() ? dims[j].cpos : -1;
      g.runRel.insert(g.runRel.end(), r.rel.begin(), r.rel.end());
      g.runSoff.insert(g.runSoff.end(), r.soff.begin(), r.soff.end());
      g.runDig.insert(g.runDig.end(), r.dig.begin(), r.dig.end());
      // consumer k addressing, cp.async planes: k is linear in the plane (k-major: 1 element
      // per k, mn-major: a pitch per k); no chunks, no swizzle
      o.kch_log2[0] = 30;
      o.kchunk[0] = 0;
      o.kmul[0] = 8 * (km ? 1 : BMN + 4);
      o.swz[0] = 0;
      return true;
    };
    if (!fill_op(D.x, m.X, cord_m[i], xkm, kGBM) || !fill_op(D.y, m.Y, cord_n[i], ykm, kGBN)) return ST_UNSUPPORTED;
    // TMA side
    auto fill_tma = [&](GOperandDev &o, int t, const TmaLayout &L, std::vector<GroupTables::TmaSpec> &spec) {
      GroupTables::TmaSpec s;
      for (int j = 0; j < kGMaxTmaDims; j++) o.tma_cpos[j] = -1;
      o.tma_kdim = -1;
      if (g.tma) {
        const auto dims = op_dims(m, t, m.X == t ? tord_m[i] : tord_n[i], g.T, false, kGBM, BK);
        s.rank = (int)dims.size();
        for (int j = 0; j < s.rank; j++) {   // map dim j = operand dim perm[j]
          const OpDim &x = dims[L.perm[j]];
          s.dims[j] = (uint64_t)x.n;
          if (j > 0) s.strides[j - 1] = (uint64_t)(8 * x.gstride);
          s.box[j] = (uint32_t)L.box[j];
          o.tma_cpos[j] = x.cpos;
          if (x.cpos < 0) o.tma_kdim = j;
        }
        s.base = c.t[t].base;
        o.tma_tx = (int32_t)L.bytes;
        o.tma_pack = (uint32_t)s.rank << 20 | (uint32_t)(o.tma_kdim < 0 ? 15 : o.tma_kdim) << 24;
        for (int j = 0; j < kGMaxTmaDims; j++) o.tma_pack |= (uint32_t)(o.tma_cpos[j] < 0 ? 15 : o.tma_cpos[j]) << (4 * j);
        const int kidx = m.kid.empty() ? -1 : m.kid[0];
        const int jk = kidx >= 0 ? c.pos_in(t, kidx) : -1;
        o.kch_log2[1] = 30;                 // one box: k is linear in it
        o.kchunk[1] = 0;
        o.kmul[1] = jk >= 0 ? (int32_t)(8 * L.bs[jk]) : 0;
        o.swz[1] = 0;
      }
      spec.push_back(s);
    };
    fill_tma(D.x, m.X, tlx[i], g.tmaX);
    fill_tma(D.y, m.Y, tly[i], g.tmaY);
    D.tma_yoff = g.tma ? (int32_t)((tlx[i].bytes + 127) / 128 * 128) : 0;
    // k steps: the k-tile grid, first k digit fastest
    D.step0 = (int32_t)g.steps.size();
    D.nsteps = (int32_t)m.nsteps;
    {
      const size_t nk = m.kid.size();
      std::vector<int64_t> od(nk, 0);
      for (;;) {
        GStepDev s{};
        s.full = 1;
        for (size_t q = 0; q < nk; q++) {
          const int id = m.kid[q];
          const int64_t o = od[q] * m.Tk[q], lim = std::min<int64_t>(m.Tk[q], c.ix[id].n - o);
          s.kx += o * c.stride_of(m.X, id);
          s.ky += o * c.stride_of(m.Y, id);
          if (lim != m.Tk[q]) s.full = 0;
          const int jx = c.pos_in(m.X, id), jy = c.pos_in(m.Y, id);
          s.klimX |= (uint64_t)lim << (8 * jx);
          s.klimY |= (uint64_t)lim << (8 * jy);
          if (q == 0) s.kc = (int32_t)o;   // (TMA groups have one internal index)
        }
        g.steps.push_back(s);
        size_t q = 0;
        for (; q < nk; q++) {
          if (++od[q] < cdiv(c.ix[m.kid[q]].n, m.Tk[q])) break;
          od[q] = 0;
        }
        if (q == nk) break;
      }
    }
    // cp.async k padding (Kt < BK): zero the k rows / columns [Kt, BK) of both planes
    D.pad0 = (int32_t)g.pad.size();
    if (Kt < BK) {
      for (int plane = 0; plane < 2; plane++) {
        const bool km = plane == 0 ? xkm : ykm;
        const int BMN = plane == 0 ? kGBM : kGBN;
        for (int64_t row = 0; row < BMN; row++)
          for (int64_t k = Kt; k < BK; k++)
            g.pad.push_back((uint32_t)(8 * (plane_off(km, row, k, BMN, BK) + (plane ? XS : 0))));
      }
    }
    D.npad = (int32_t)g.pad.size() - D.pad0;
    // consumer tables per mode: row bytes of X / Y in the plane, box offsets of rows / columns
    for (int mode = 0; mode < 2; mode++) {
      const auto &om = mode ? tord_m[i] : cord_m[i];
      const auto &on = mode ? tord_n[i] : cord_n[i];
      // rows outside the member's tile load from a valid plane address (0) and are never
      // written back (box offset -1)
      std::vector<int32_t> tab(kGCtab, -1);
      std::fill(tab.begin(), tab.begin() + 128, 0);
      if (mode == 0 || g.tma) {
        const auto R = row_box(om, g.T, bst, kGBM), Q = row_box(on, g.T, bst, kGBN);
        for (int r = 0; r < 64; r++) {
          tab[128 + r] = R[r];
          tab[192 + r] = Q[r];
        }
        for (int side = 0; side < 2; side++) {
          const int t = side ? m.Y : m.X;
          const auto &ord = side ? on : om;
          int64_t tot = 1;
          for (int p : ord) tot *= g.T[p];
          for (int64_t r = 0; r < tot && r < 64; r++) {
            int64_t b;
            if (mode == 0) {
              const bool km = side ? ykm : xkm;
              int64_t row = 0;
              const auto dg = row_digits(r, ord, g.T);
              for (int p : ord) row += dg[p] * row_mul(ord, g.T, p);
              b = 8 * plane_off(km, row, 0, side ? kGBN : kGBM, BK);
            } else {
              const TmaLayout &L = side ? tly[i] : tlx[i];
              const auto dg = row_digits(r, ord, g.T);
              std::vector<int64_t> d(c.t[t].idx.size(), 0);
              for (size_t j = 0; j < d.size(); j++) {
                const int cp = c.pos_in(0, c.t[t].idx[j]);
                if (cp >= 0) d[j] = dg[cp];
              }
              b = L.byte(d);
            }
            tab[side * 64 + r] = (int32_t)b;
          }
        }
      }
      g.ctab[mode].insert(g.ctab[mode].end(), tab.begin(), tab.end());
    }
    g.mem.push_back(D);
    int64_t Mt = 1, Nt = 1;
    for (int p : m.mpos) Mt *= g.T[p];
    for (int p : m.npos) Nt *= g.T[p];
    g.Mt.push_back(Mt);
    g.Nt.push_back(Nt);
    g.Kt.push_back(Kt);
    g.padded_flops += 2.0 * (double)g.ntiles * (double)m.nsteps * kGBM * kGBN * 4 * cdiv(Kt, 4);
  }

  // ---- execution order: members whose register tile maps onto the box the same way (in the
  //      mode that runs: TMA when every operand allows it) become neighbours, and chain — the
  //      tile stays in registers from one to the next (the sum's order changes; any order is
  //      a correct result, DESIGN R22)
  {
    const int run_mode = g.tma ? 1 : 0;
    auto boxmap = [&](int mo, int i) {
      return std::vector<int32_t>(g.ctab[mo].begin() + (size_t)i * kGCtab + 128,
                                  g.ctab[mo].begin() + (size_t)(i + 1) * kGCtab);
    };
    std::vector<int> ord;
    std::vector<char> used(n, 0);
    for (int i = 0; i < n; i++) {
      if (used[i]) continue;
      used[i] = 1;
      ord.push_back(i);
      const auto bi = boxmap(run_mode, i);
      for (int k = i + 1; k < n; k++)
        if (!used[k] && boxmap(run_mode, k) == bi) {
          used[k] = 1;
          ord.push_back(k);
        }
    }
    auto permute = [&](auto &v) {
      auto w = v;
      for (int k = 0; k < n; k++) w[k] = v[ord[k]];
      v = w;
    };
    permute(g.mem);
    permute(g.tmaX);
    permute(g.tmaY);
    permute(g.Mt);
    permute(g.Nt);
    permute(g.Kt);
    permute(g.flushWf);
    permute(g.loadWf);
    permute(g.fragWf);
    for (int mo = 0; mo < 2; mo++) {
      std::vector<int32_t> t(g.ctab[mo].size());
      for (int k = 0; k < n; k++)
        std::copy(g.ctab[mo].begin() + (size_t)ord[k] * kGCtab, g.ctab[mo].begin() + (size_t)(ord[k] + 1) * kGCtab,
                  t.begin() + (size_t)k * kGCtab);
      g.ctab[mo] = t;
    }
    g.order = ord;
    for (int k = 0; k < n; k++)
      for (int mo = 0; mo < 2; mo++)
        g.mem[k].chain[mo] = (k + 1 < n && (mo == 0 || g.tma) && boxmap(mo, k) == boxmap(mo, k + 1)) ? 1 : 0;
  }

  // ---- copy-out units: the box in C order, 2 elements per unit when 16-B stores are legal
  bool u2 = g.T[0] % 2 == 0 && g.N[0] % 2 == 0 && g.cstride[0] == 1 && g.cbase % 2 == 0;
  for (int p = 1; p < rank; p++) u2 &= g.cstride[p] % 2 == 0;
  g.uvec = u2 ? 2 : 1;
  for (int64_t o = 0; o < g.box; o += g.uvec) {
    int64_t q = o, rel = 0;
    uint64_t dg = 0;
    for (int p = 0; p < rank; p++) {
      const int64_t d = q % g.T[p];
      q /= g.T[p];
      rel += d * g.cstride[p];
      dg |= (uint64_t)d << (8 * p);
    }
    g.unitRel.push_back(rel);
    g.unitDig.push_back(dg);
  }
  g.plan_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  return ST_OK;
}

}  // namespace tc
