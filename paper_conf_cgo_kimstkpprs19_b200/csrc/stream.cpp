// stream.cpp — eligibility, tile choice and tables of the streaming path (stream.hpp).
//
// The tile is a box of X's externals (a CTA owns a hyper-rectangle prod T_i of C); the
// internal index k is walked in steps of KB (one TMA box per step), Y stays whole in shared
// memory.  A tile is cut into warp units: AR consecutive values of C's FVI a times 16 rows
// (SM_T: two octets of 8 consecutive values of X's FVI; SM_K: 16 rows of the other m dims).
// Tiles are chosen for the DRAM runs they produce: the X box is read as runs along X's memory
// order and C written as runs along C's FVI (coalescing along each tensor's FVI is
// what the paper's cost model counts, Alg. 3, here in 32-B sectors).
#include "stream.hpp"

#include <algorithm>
#include <climits>
#include <cmath>
#include <cstdio>
#include <cstdlib>

#include "tiles.hpp"

namespace tc {
namespace {

// the kernel instances (kernels_stream.cu): n8 blocks NB = 1..4, runs AR = 4 (two CTAs per SM)
// or 8 (one CTA per SM; not with NB = 4: 128 accumulator registers)
bool instance_exists(int NB, int AR) { return NB >= 1 && NB <= 4 && (AR == 4 || (AR == 8 && NB <= 3)); }
// FP64 (DMMA m8n8k4: 8-row units, accumulators 2 doubles per n8 block and a value)
bool instance_exists_f64(int NB, int AR) {
  // (NB = 9 with AR = 4 spills at ptxas' 168-register choice)
  return (NB >= 1 && NB <= 4 && (AR == 4 || (AR == 8 && NB <= 3))) || (NB == 9 && AR == 2);
}

int round_up(int64_t x, int m) { return (int)((x + m - 1) / m * m); }

// contiguous bytes of one box row run: dims from 0 while the box covers the whole (dense) dim
double run_bytes(const int64_t *dims, const int64_t *str, const uint32_t *box, int rank, int es) {
  double run = es;
  int64_t dense = 1;
  for (int j = 0; j < rank; j++) {
    if (str[j] != dense) break;
    run *= std::min<int64_t>(box[j], dims[j]);
    if ((int64_t)box[j] < dims[j]) break;
    dense *= dims[j];
  }
  return run;
}

// DRAM efficiency of runs of r bytes (32-B sectors; whole 64/128-B lines when r allows); writes
// pay more for short runs than reads (BF16 tile sweeps on TCCG #1, profiles/r02_stream_sweep_*)
double run_eff(double r) { return r >= 128 ? 1.0 : r >= 64 ? 0.9 : r >= 32 ? 0.75 : 0.4; }
double run_eff_w(double r) { return r >= 128 ? 1.0 : r >= 64 ? 0.85 : r >= 32 ? 0.6 : 0.3; }

}  // namespace

bool stream_plan(const Contraction &c, int kind, int sms, StreamCfg &s, int rank) {
  s = StreamCfg();
  auto no = [&](const char *why) { s.why = why; return false; };
  const bool f64 = kind == KIND_F64_DMMA;
  const int es = kind_esize(kind);   // 8 FP64, 2 BF16, 4 TF32 / FP32 split
  const int ru = f64 ? 8 : kSRows;   // rows of one MMA block: m8 (DMMA) / m16 (mma.sync)
  const int kq = es == 2 ? 16 : 8;   // k granule: one HMMA k16 / one TF32 k8 / two DMMA k4 steps
  for (auto &ix : c.ix) if (ix.cls == BATCH) return no("batch index");
  const int a = c.c_fvi();
  if (a < 0 || c.t[0].stride.empty() || c.t[0].stride[0] != 1 || c.t[0].idx[0] != a) return no("C's FVI");
  const int X = c.ix[a].cls == EXT_A ? 1 : 2, Yt = 3 - X;
  const int xcls = X == 1 ? EXT_A : EXT_B, ycls = X == 1 ? EXT_B : EXT_A;
  int kid = -1, nid = -1, nk = 0, nn = 0;
  std::vector<int> mids;
  for (int id = 0; id < (int)c.ix.size(); id++) {
    if (c.ix[id].cls == INTL) { kid = id; nk++; }
    else if (c.ix[id].cls == ycls) { nid = id; nn++; }
    else if (c.ix[id].cls == xcls) mids.push_back(id);
  }
  if (nk != 1 || nn != 1) return no("needs one internal and one Y-side external index");
  if ((int)mids.size() > kSMaxMdims) return no("more than 4 X externals");
  const TensorView &xv = c.t[X], &cv = c.t[0], &yv = c.t[Yt];
  const int xr = (int)xv.idx.size();
  if (xr > kMaxTmaDims) return no("rank > 5");
  if (xv.stride[0] != 1) return no("X not unit-stride along its FVI");
  for (int j = 1; j < xr; j++)
    if ((xv.stride[j] * es) % 16 || xv.stride[j] >= ((int64_t)1 << 39)) return no("X strides (TMA)");
  const int64_t N = c.ix[nid].n, K = c.ix[kid].n;
  if (N > (f64 ? 72 : 32)) return no("Y-side extent above the kernels' n blocks (32; FP64 72)");
  const int NB = N > 32 ? 9 : (int)((N + 7) / 8), N8 = 8 * NB;
  const int KP = round_up(K, kq);
  // conflict-free B-fragment rows (8 rows n at consecutive 8 / 4 threads' k)
  const int YP = es == 8 ? round_up(KP, 16) + 4 : es == 4 ? round_up(KP, 32) + 4 : KP + 8;
  const size_t ybytes = (size_t)N8 * YP * es;
  if (ybytes > (f64 ? 64 : 48) * 1024) return no("Y does not fit shared memory");
  const int x0 = xv.idx[0];
  if (x0 == a && !f64) return no("X's FVI is C's FVI (the tcgen05 path stores those runs directly)");
  const int mode = x0 == kid ? SM_K : x0 == a ? SM_M : SM_T;
  // the octet dim (8 consecutive values per 8 fragment rows) and the run dim (AR consecutive
  // values per warp, one MMA block each): SM_T octets of X's FVI, runs of C's FVI a; SM_K rows
  // of the other dims, runs of a; SM_M (FP64) octets of a (= X's FVI), runs of the next X dim
  int adim = a;
  if (mode == SM_M) {
    adim = -1;
    for (int j = 1; j < xr && adim < 0; j++)
      if (xv.idx[j] != kid) adim = xv.idx[j];
    if (adim < 0) return no("X has no second external for the runs");
  }
  const int E = mode == SM_T ? x0 : mode == SM_M ? a : -1;
  std::vector<int> rest;   // the other m dims, X order
  for (int j = 0; j < xr; j++) {
    const int id = xv.idx[j];
    if (id != adim && id != E && id != kid) rest.push_back(id);
  }
  auto mult = [](int64_t n, int step, int cap) {
    std::vector<int> v;
    const int top = std::min(cap, round_up(n, step));
    for (int t = step; t <= top; t += step) v.push_back(t);
    return v;
  };
  std::vector<int> Te = E >= 0 ? mult(c.ix[E].n, 8, 256) : std::vector<int>{1};
  std::vector<int> p2 = {1, 2, 4, 8, 16};
  std::vector<int> kbs;
  for (int kb = kq; kb <= std::min(f64 ? 64 : es == 4 ? 128 : 256, KP); kb += kq) kbs.push_back(kb);
  const double hbm = 6.5e12;
  double best = 1e30;
  std::vector<StreamCfg> top;   // the kStreamRanks best configurations, model order
  std::vector<std::vector<int>> restopts;
  for (int id : rest) {
    std::vector<int> o;
    for (int t : p2) if (t == 1 || t <= round_up(c.ix[id].n, 2)) o.push_back(t);
    restopts.push_back(o);
  }
  // pass 0: tiles that divide every extent (an edge tile costs its MMAs, ring space and the
  // checked store path: 2-5x on TCCG #1 measured); pass 1: any tile
  for (int pass = 0; pass < 2 && best >= 1e29; pass++) {
  std::vector<size_t> rix(rest.size(), 0);
  for (;;) {
    int rprod = 1;
    std::vector<int> rt(rest.size());
    for (size_t q = 0; q < rest.size(); q++) { rt[q] = restopts[q][rix[q]]; rprod *= rt[q]; }
    for (int AR : {2, 4, 8}) {
      if (!(f64 ? instance_exists_f64(NB, AR) : instance_exists(NB, AR))) continue;
      // the C box leaves in 16-B chunks: every C stride (and C's origin) a multiple of 16 B
      bool cal = (cv.base * es) % 16 == 0;
      for (size_t j = 1; j < cv.stride.size(); j++) cal &= (cv.stride[j] * es) % 16 == 0;
      if (!cal) continue;
      for (int ta : mult(c.ix[adim].n, mode == SM_M ? AR : 8, mode == SM_M ? 64 : 128))
        for (int te : Te) {
          // row sets of 16: SM_T octet pairs (E octets x rest), SM_K 16 rows of the rest dims
          // (an odd octet count / a rest product off 16 pads the last set with rows that are
          //  computed but never stored)
          int64_t rowsets = 0;
          if (mode != SM_K) {
            rowsets = ((int64_t)(te / 8) * rprod + (ru / 8 - 1)) / (ru / 8);
          } else {
            rowsets = rprod < 8 ? 0 : (rprod + ru - 1) / ru;
          }
          if (!rowsets) continue;
          const int64_t units = rowsets * (ta / AR);
          if (units > kSWarps) continue;
          for (int kb : kbs) {
            const int nks = (KP + kb - 1) / kb;
            StreamCfg q;
            q.NB = NB;
            q.AR = AR;
            q.X = X;
            q.mode = mode;
            int T[kMaxIdx];
            for (int id = 0; id < (int)c.ix.size(); id++) T[id] = 1;
            T[adim] = ta;
            if (E >= 0) T[E] = te;
            for (size_t r = 0; r < rest.size(); r++) T[rest[r]] = rt[r];
            T[kid] = kb;
            T[nid] = N8;
            q.xrank = xr;
            bool boxok = true;
            int64_t boxel = 1;
            for (int j = 0; j < xr; j++) {
              q.xdims[j] = c.ix[xv.idx[j]].n;
              q.xstr[j] = xv.stride[j];
              q.xbox[j] = (uint32_t)T[xv.idx[j]];
              boxok &= q.xbox[j] <= 256;
              boxel *= q.xbox[j];
            }
            if (!boxok) continue;
            // the box's first dim as one TMA swizzle span (16 B chunks XOR the row): ldmatrix
            // rows (k rows in SM_T, m rows in SM_K) land in distinct bank groups
            const int inner = (int)q.xbox[0] * es;
            const int swz = inner == 32 ? 1 : inner == 64 ? 2 : inner == 128 ? 3 : 0;
            const int stage = (int)(boxel * es);
            const int64_t rows = (int64_t)units * ru * AR;   // tile rows (m)
            const size_t stg = (size_t)round_up(rows * N8 * es, 128);
            const size_t tabb = (size_t)units * 2 * ru * 4 + (size_t)rows * N8 * es / 16 * 4;
            const int occ = stream_occ(NB, AR);
            const size_t cap = occ == 2 ? 115712 : 232448;
            // two C boxes when they leave >= 3 ring stages (one block-wide barrier per tile
            // instead of two), else one
            int stages = 0, nstg = 0;
            for (int nb2 = 2; nb2 >= 1 && !stages; nb2--) {
              const size_t fixed = 1024 + round_up((int64_t)ybytes, 128) + nb2 * stg + round_up((int64_t)tabb, 64) + 16 * 8;
              for (int st = 6; st >= (nb2 == 2 ? 3 : 2); st--)
                if (fixed + (size_t)st * round_up(stage, 1024) <= cap) { stages = st; nstg = nb2; break; }
            }
            if (!stages) continue;
            int64_t tiles = 1;
            for (int id : mids) tiles *= (c.ix[id].n + T[id] - 1) / T[id];
            if (tiles > (int64_t)1 << 30) continue;
            // DRAM: X box runs; C runs along its FVI (the tile's extent of a, longer when the
            // tile covers a and C's next dim)
            const double rx = run_bytes(q.xdims, q.xstr, q.xbox, xr, es);
            double rc = es * (double)std::min<int64_t>(T[a], c.ix[a].n);
            if (T[a] >= c.ix[a].n && cv.idx.size() > 1 && T[cv.idx[1]] > 1 && cv.stride[1] == c.ix[a].n)
              rc *= std::min<int64_t>(T[cv.idx[1]], c.ix[cv.idx[1]].n);
            const double bx = (double)c.numel(X) * es, bc = (double)c.numel(0) * es;
            double t = (bx / run_eff(rx) + bc / run_eff_w(rc)) / hbm;
            // the TMA engine moves a box row (its first dim) every ~3 SM clocks (measured on
            // B200 with 64-B rows, tools/stream_ablation.py): short rows bound the X stream
            const double trows = (double)tiles * nks * ((double)boxel / q.xbox[0]) * 3.0 / ((double)sms * 1.9e9);
            t = std::max(t, trows);
            if (f64) {
              // DMMA work (padded tiles, padded k): the FP64 pipe at the measured 37.16 TFLOP/s
              // needs ~8 issuing warps per SM (fragment loads and DMMA latency per warp)
              const double fl = 2.0 * tiles * rows * N8 * (double)nks * kb;
              const double weff = std::min(1.0, (double)units * occ / 8.0);
              t = std::max(t, fl / (37.16e12 * weff));
            }
            const int64_t slots = (int64_t)sms * occ;
            const double waves = std::ceil((double)tiles / slots);
            t /= std::min(1.0, (double)tiles / (waves * slots)) + 1e-12;
            // pipeline fill and drain: the first tile's loads and the last tile's stores of each
            // CTA do not overlap other work (~one tile time per CTA)
            t *= (waves + 1.0) / waves;
            // bytes in flight per SM (the X ring): under ~64 KB HBM latency is exposed
            const double inflight = (double)stages * stage * occ;
            if (inflight < 64e3) t *= 64e3 / inflight;
            // compute warps per SM: fewer than 8 leave the ldmatrix / MMA latency exposed
            if (units * occ < 8) t *= 1.0 + 0.5 * (8.0 - units * occ) / 8.0;
            // ragged tiles (box past the extent) waste MMA and ring space, not DRAM: tie-break
            double fill = 1.0;
            for (int id : mids) fill *= (double)c.ix[id].n / (((c.ix[id].n + T[id] - 1) / T[id]) * T[id]);
            if (pass == 0 && fill < 1.0) continue;
            t *= 1.0 + 0.6 * (1.0 - fill) + 0.02 * ((double)nks * kb - K) / K;
            if (!swz) t *= 1.3;   // bank conflicts on the fragment loads
#ifdef TC_STREAM_DEV
            // (tools/stream_sweep.py side builds only: TC_STREAM_FORCE="<ta>,<te>,<AR>,<kb>,<rprod>")
            if (const char *fz = std::getenv("TC_STREAM_FORCE")) {
              int fta = 0, fte = 0, far = 0, fkb = 0, frp = 0;
              if (std::sscanf(fz, "%d,%d,%d,%d,%d", &fta, &fte, &far, &fkb, &frp) == 5 &&
                  (ta != fta || (E >= 0 && te != fte) || AR != far || kb != fkb || rprod != frp))
                continue;
            }
#endif
            {   // keep the best few configurations (rank: tc_plan_tuned times the first ones)
              best = std::min(best, t);
              // measured / modelled time of the streaming kernels on TCCG #1-8 (one B200, median
              // per kind, profiles/r02_stream_check_*.jsonl): the reported prediction only — the
              // factor is common to every candidate of a kind, so it leaves the ranking alone
              const double cal = kind == KIND_F64_DMMA ? 1.43 : kind == KIND_BF16_UMMA ? 1.09
                               : kind == KIND_TF32_UMMA ? 1.54 : 1.92;
              q.t_pred = t * cal + 4e-6;
              q.occ = occ;
              q.xswz = swz;
              q.kp.KB = kb;
              q.kp.nks = nks;
              q.kp.stages = stages;
              q.kp.nstg = nstg;
              q.kp.stage_bytes = stage;
              q.kp.ntiles = (int)tiles;
              q.kp.nunits = (int)units;
              for (int id = 0; id < (int)c.ix.size(); id++) q.T[id] = T[id];
              top.push_back(q);
              std::sort(top.begin(), top.end(), [](const StreamCfg &x, const StreamCfg &y) { return x.t_pred < y.t_pred; });
              if ((int)top.size() > kStreamRanks) top.pop_back();
            }
          }
        }
    }
    size_t q = 0;
    while (q < rest.size() && ++rix[q] == restopts[q].size()) rix[q++] = 0;
    if (q == rest.size()) break;
  }
  }
  if (best >= 1e29 || top.empty()) return no("no tile fits");
  s = top[std::min<int>(rank, (int)top.size() - 1)];
  s.rank = std::min<int>(rank, (int)top.size() - 1);
  s.nranks = (int)top.size();
  SParams &k = s.kp;
  const int *T = s.T;
  k.K = (int)K;
  k.N = (int)N;
  k.KP = KP;
  k.YP = YP;
  k.xrank = xr;
  k.ysk = c.stride_of(Yt, kid);
  k.ysn = c.stride_of(Yt, nid);
  k.csn = c.stride_of(0, nid);
  s.xbase = xv.base;
  s.cbase = cv.base;
  s.ybase = yv.base;
  auto bsx = [&](int id) {   // element stride of index id in the X box
    int64_t st = 1;
    for (int j = 0; j < xr; j++) {
      if (xv.idx[j] == id) return st;
      st *= T[xv.idx[j]];
    }
    return (int64_t)0;
  };
  // m dims in raster order: C's FVI first, then the other X externals in X order
  std::vector<int> md = {a};
  for (int j = 0; j < xr; j++) {
    const int id = xv.idx[j];
    if (id != a && id != kid) md.push_back(id);
  }
  k.nmd = (int)md.size();
  for (int d = 0; d < k.nmd; d++) {
    const int id = md[d];
    k.mT[d] = T[id];
    k.mNt[d] = (int)((c.ix[id].n + T[id] - 1) / T[id]);
    k.mX[d] = c.pos_in(X, id);
    k.mN[d] = (int)c.ix[id].n;
    k.mCs[d] = c.stride_of(0, id);
  }
  k.kX = c.pos_in(X, kid);
  k.xpitchk = (int)(bsx(kid) * es);
  k.xpitcha = (int)(bsx(adim) * es);
  k.xswz = s.xswz == 1 ? 1 : s.xswz == 2 ? 3 : s.xswz == 3 ? 7 : 0;
  // the C box: C's dims in C order, m dims at their tiles, n at 8 NB (element strides cbs)
  const int cr = (int)cv.idx.size();
  if (cr > kMaxTmaDims) return no("C rank > 5");
  std::vector<int64_t> cbs(cr);
  k.crank = cr;
  {
    int64_t st = 1;
    for (int j = 0; j < cr; j++) {
      const int id = cv.idx[j];
      cbs[j] = st;
      k.cbox[j] = T[id];
      k.cmd[j] = -1;
      for (int d = 0; d < k.nmd; d++)
        if (md[d] == id) k.cmd[j] = d;
      if (id == nid) k.cbsn = (int)st;
      st *= T[id];
    }
  }
  auto bsc = [&](int id) {
    for (int j = 0; j < cr; j++)
      if (cv.idx[j] == id) return cbs[j];
    return (int64_t)0;
  };
  // units: u -> (row set p = u / agroups, a group g = u % agroups); 16 rows each
  const int agroups = T[adim] / s.AR;
  k.cbsj = (int)bsc(adim);
  k.ru = ru;
  std::vector<uint32_t> xo, bo;
  for (int u = 0; u < k.nunits; u++) {
    const int p = u / agroups, a0 = (u % agroups) * s.AR;
    for (int i = 0; i < ru; i++) {
      // the row's coordinates in the tile per raster dim (md order)
      int crd[kSMaxMdims] = {0, 0, 0, 0};
      int64_t ri;   // index into the rest enumeration (rest dims in X order, first fastest)
      for (int d = 0; d < k.nmd; d++)
        if (md[d] == adim) crd[d] = a0;
      int64_t nrest = 1;
      for (int id : rest) nrest *= T[id];
      const int oct = (ru / 8) * p + (i >> 3);   // SM_T: the row's octet
      const bool dummy = s.mode != SM_K ? oct >= (T[E] / 8) * nrest : (int64_t)ru * p + i >= nrest;
      if (dummy) {   // padding row: reads row 0 of the box, never stored
        xo.push_back(0);
        bo.push_back(0xFFFFFFFFu);
        continue;
      }
      if (s.mode != SM_K) {
        const int eo = oct % (T[E] / 8);
        ri = oct / (T[E] / 8);
        for (int d = 0; d < k.nmd; d++)
          if (md[d] == E) crd[d] = 8 * eo + (i & 7);
      } else {
        ri = (int64_t)ru * p + i;
      }
      for (int id : rest) {
        const int v = (int)(ri % T[id]);
        ri /= T[id];
        for (int d = 0; d < k.nmd; d++)
          if (md[d] == id) crd[d] = v;
      }
      int64_t xoff = 0, boff = 0;
      for (int d = 0; d < k.nmd; d++) {
        xoff += crd[d] * bsx(md[d]);
        boff += crd[d] * bsc(md[d]);
      }
      xo.push_back((uint32_t)(xoff * es));
      bo.push_back((uint32_t)boff);
    }
  }
  for (int u = 0; u < k.nunits; u++) {
    s.tab.insert(s.tab.end(), xo.begin() + ru * u, xo.begin() + ru * (u + 1));
    s.tab.insert(s.tab.end(), bo.begin() + ru * u, bo.begin() + ru * (u + 1));
  }
  // per 16-B chunk of the C box (box order): its element offset in C from the tile origin
  int64_t cel = 1;
  for (int j = 0; j < cr; j++) cel *= k.cbox[j];
  const int epc = 16 / es;   // elements per 16-B chunk
  k.nchunk = (int)(cel / epc);
  {
    std::vector<int> bc(cr, 0);
    for (int ch = 0; ch < k.nchunk; ch++) {
      int64_t off = 0;
      for (int j = 0; j < cr; j++) off += (int64_t)bc[j] * cv.stride[j];
      if (off > INT32_MAX) return no("tile spans more than 2^31 elements of C");
      s.tab.push_back((uint32_t)off);
      int j = 0;
      bc[0] += epc;
      while (j < cr && bc[j] >= k.cbox[j]) { bc[j] = 0; if (++j < cr) bc[j]++; }
    }
  }
  // staging swizzle: simulate the epilogue's writes (one warp instruction = its 32 lanes' runs
  // of AR elements at fixed (row half h, n8 block, c2); per 16-B chunk) and keep the fold with
  // the fewest bank wavefronts
  {
    const int sh[][2] = {{3, 6}, {2, 5}, {3, 5}, {1, 4}, {4, 8}, {2, 4}};
    long bestw = -1;
    const int halves = ru / 8;
    const int cpr = std::max(1, s.AR * es / 16);   // chunks per run
    for (auto &f : sh) {
      long wf = 0;
      for (int u = 0; u < k.nunits; u++)
        for (int h = 0; h < halves; h++)
          for (int nb = 0; nb < NB; nb++)
            for (int c2 = 0; c2 < 2; c2++)
              for (int cc = 0; cc < cpr; cc++) {
                int cnt[8] = {0};
                for (int lane = 0; lane < 32; lane++) {
                  const int g = lane >> 2, t4 = lane & 3;
                  if (bo[ru * u + 8 * h + g] == 0xFFFFFFFFu) continue;
                  const int64_t el = bo[ru * u + 8 * h + g] + (int64_t)(8 * nb + 2 * t4 + c2) * k.cbsn;
                  const int64_t ch = el * es / 16 + cc;
                  const int64_t x = ch >> 3;
                  cnt[(int)((ch ^ ((x ^ (x >> f[0]) ^ (x >> f[1])) & 7)) & 7)]++;
                }
                int mx = 0;
                for (int b = 0; b < 8; b++) mx = std::max(mx, cnt[b]);
                wf += mx;
              }
      if (bestw < 0 || wf < bestw) {
        bestw = wf;
        k.cs1 = f[0];
        k.cs2 = f[1];
      }
    }
  }
  // shared memory map (from the 1 KB aligned base): X ring, C box, Y, tables, barriers
  k.stage_pitch = round_up(k.stage_bytes, 1024);
  int off = k.stages * k.stage_pitch;
  k.off_stg = off;
  k.stg_pitch = round_up(cel * es, 128);
  off += k.nstg * k.stg_pitch;
  k.off_y = off;
  off += round_up((int64_t)ybytes, 128);
  k.off_tab = off;
  off += round_up((int64_t)s.tab.size() * 4, 64);
  k.off_bar = off;
  off += 16 * k.stages;
  s.smem = (size_t)off + 1024;
  s.bytes = (double)(c.numel(1) + c.numel(2) + c.numel(0)) * es;
  s.on = s.smem <= (s.occ == 2 ? 115712u : 232448u);
  // arithmetic intensity of the streamed contraction: 2 N K flops per X row of es (K + N) bytes;
  // the FP64 ridge is 37.16 TFLOP/s / 6.55 TB/s = 5.7 (measured B200 peaks)
  const double inten = 2.0 * N * K / (es * (double)(K + N));
  // 32-bit operands in SM_K: the plain k-contiguous fragment loads lose to the tcgen05 path
  // (TCCG #7 / #8 in TF32 and split FP32, measured): tuning still times both
  s.preferred = f64 ? inten <= 0.8 * 5.67 : (es == 2 || s.mode == SM_T);
  if (!s.on) s.why = "shared memory";
  return s.on;
}

}  // namespace tc
