// api.cu — the C ABI of libtc (include/libtc.h): plan construction (rows a1-a4), launch
// metadata (row a4), kernel dispatch (rows a5-a7), restriction (row e) and introspection.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <map>
#include <memory>
#include <new>
#include <sstream>
#include <string>
#include <vector>

#include "../../include/libtc.h"
#include "contraction.hpp"
#include "kernel_f64.cuh"
#include "kparams.hpp"
#include "planner.hpp"

using namespace tc;

namespace {
thread_local std::string g_err;

tc_status_t fail(Status s, const std::string &msg) {
  g_err = msg;
  return (tc_status_t)s;
}

// ---------------------------------------------------------------- kernel table
struct KernelEntry {
  const void *fn;
  int threads;
  size_t smem;
};

template <int BM, int BN, int BK, int WM, int WN, int ST>
KernelEntry entry() {
  using K = F64Kernel<BM, BN, BK, WM, WN, ST>;
  return {(const void *)&tc_f64_dmma_kernel<BM, BN, BK, WM, WN, ST>, K::THREADS, K::smem_bytes()};
}

const std::vector<KernelEntry> &kernels() {
  // must match planner.cpp variants() one-to-one
  static const std::vector<KernelEntry> k = {
      entry<128, 128, 16, 64, 32, 4>(),
      entry<128, 64, 16, 64, 32, 3>(),
      entry<64, 128, 16, 32, 64, 3>(),
      entry<64, 64, 16, 32, 32, 4>(),
      entry<128, 128, 8, 64, 32, 4>(),
      entry<64, 64, 8, 32, 32, 4>(),
  };
  return k;
}

struct DevTables {
  void *buf = nullptr;
  size_t bytes = 0;
};

}  // namespace

struct tc_plan_s {
  Contraction parsed;      // as parsed (before normalisation) — restriction starts here
  Contraction c;           // normalised (dropped extent-1 indices, fused runs)
  int dtype = 0;
  int device = -1;
  bool host_only = false;
  Config cfg;
  PlanStats stats;
  tc_plan_opts opts{};
  std::string force_tiles;
  // host copies of the tables
  std::vector<int64_t> stepX, stepY;
  std::vector<uint64_t> kmask;
  std::vector<uint32_t> slotX1, slotY1, slotX2, slotY2;
  bool vecX_ok = false, vecY_ok = false;
  KParams kp{};            // device pointers filled in; X/Y/C/alpha/beta set per call
  DevTables dev;
  // device pointers into dev.buf
  const uint32_t *d_slotX1 = nullptr, *d_slotY1 = nullptr, *d_slotX2 = nullptr, *d_slotY2 = nullptr;
  ~tc_plan_s() {
    if (dev.buf) {
      int cur = -1;
      cudaGetDevice(&cur);
      if (cur != device) cudaSetDevice(device);
      cudaFree(dev.buf);
      if (cur != device && cur >= 0) cudaSetDevice(cur);
    }
  }
};

namespace {

int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Load slots of operand t (X or Y) in the operand's OWN memory order, packed
// (mn << 8) | k.  vec = 2: the operand's FVI is stepped by 2 (16-B cp.async).
std::vector<uint32_t> build_slots(const Contraction &c, const Config &cfg, int t, int vec,
                                  const std::vector<int> &side) {
  std::vector<uint32_t> out;
  const auto &v = c.t[t];
  const int r = (int)v.idx.size();
  std::vector<int> T(r), mul(r), isk(r);
  // multipliers of each index in the compute-order multi-index (side digits / k digits)
  for (int p = 0; p < r; p++) {
    const int id = v.idx[p];
    T[p] = cfg.T[id];
    isk[p] = c.ix[id].cls == INTL;
    const auto &lst = isk[p] ? cfg.kdig : side;
    int m = 1;
    for (int q : lst) {
      if (q == id) break;
      m *= cfg.T[q];
    }
    mul[p] = m;
  }
  std::vector<int> d(r, 0);
  for (;;) {
    int mn = 0, k = 0;
    for (int p = 0; p < r; p++) (isk[p] ? k : mn) += d[p] * mul[p];
    out.push_back(((uint32_t)mn << 8) | (uint32_t)k);
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

// Can operand t use 16-B vectors?  Its FVI must be the leading digit of its smem-contiguous
// dimension, with even tile and extent, stride 1, and every other stride / base even.
bool vec_ok(const Contraction &c, const Config &cfg, int t, const std::vector<int> &side) {
  const auto &v = c.t[t];
  if (v.idx.empty() || v.stride[0] != 1) return false;
  const int f = v.idx[0];
  const bool isk = c.ix[f].cls == INTL;
  const auto &lst = isk ? cfg.kdig : side;
  if (lst.empty() || lst[0] != f) return false;
  if (cfg.T[f] % 2 || c.ix[f].n % 2) return false;
  for (size_t p = 1; p < v.stride.size(); p++) if (v.stride[p] % 2) return false;
  return v.base % 2 == 0;
}

Status build_tables(tc_plan_s *P, std::string &err) {
  const Contraction &c = P->c;
  const Config &cfg = P->cfg;
  const Variant &var = variants()[cfg.variant];
  KParams &kp = P->kp;
  std::memset(&kp, 0, sizeof(kp));
  const int X = cfg.X, Y = cfg.Y;
  kp.baseX = c.t[X].base;
  kp.baseY = c.t[Y].base;
  kp.baseC = c.t[0].base;
  auto side = [&](SideDesc &sd, const std::vector<int> &dig, int op) {
    sd.nd = (int)dig.size();
    sd.tiles = 1;
    for (int i = 0; i < sd.nd; i++) {
      const int id = dig[i];
      sd.T[i] = cfg.T[id];
      sd.N[i] = c.ix[id].n;
      sd.ntile[i] = cdiv(c.ix[id].n, cfg.T[id]);
      sd.sOp[i] = c.stride_of(op, id);
      sd.sC[i] = c.stride_of(0, id);
      sd.tiles *= sd.ntile[i];
    }
  };
  if ((int)cfg.mdig.size() > kMaxDigits || (int)cfg.ndig.size() > kMaxDigits) {
    err = "too many digits";
    return ST_UNSUPPORTED;
  }
  side(kp.m, cfg.mdig, X);
  side(kp.n, cfg.ndig, Y);
  kp.nctas = kp.m.tiles * kp.n.tiles;
  kp.group_m = 8;
  // k side
  const int nk = (int)cfg.kdig.size();
  std::vector<int64_t> kt(nk), kn(nk);
  int64_t steps = 1;
  for (int i = 0; i < nk; i++) {
    kn[i] = c.ix[cfg.kdig[i]].n;
    kt[i] = cfg.T[cfg.kdig[i]];
    steps *= cdiv(kn[i], kt[i]);
  }
  if (steps > (1LL << 30)) { err = "too many k steps"; return ST_UNSUPPORTED; }
  kp.nsteps = (int)steps;
  for (int k = 0; k < 64; k++) { kp.relKX[k] = 0; kp.relKY[k] = 0; }
  const int Kt = (int)cfg.Kt;
  for (int k = 0; k < Kt && k < 64; k++) {
    int q = k;
    for (int i = 0; i < nk; i++) {
      const int d = q % (int)kt[i];
      q /= (int)kt[i];
      kp.relKX[k] += d * c.stride_of(X, cfg.kdig[i]);
      kp.relKY[k] += d * c.stride_of(Y, cfg.kdig[i]);
    }
  }
  P->stepX.resize(steps);
  P->stepY.resize(steps);
  P->kmask.resize(steps);
  std::vector<int64_t> cd(nk, 0);
  for (int64_t s = 0; s < steps; s++) {
    int64_t bx = 0, by = 0;
    for (int i = 0; i < nk; i++) {
      bx += cd[i] * kt[i] * c.stride_of(X, cfg.kdig[i]);
      by += cd[i] * kt[i] * c.stride_of(Y, cfg.kdig[i]);
    }
    uint64_t mask = 0;
    for (int k = 0; k < Kt; k++) {
      int q = k;
      bool ok = true;
      for (int i = 0; i < nk; i++) {
        const int d = q % (int)kt[i];
        q /= (int)kt[i];
        ok &= cd[i] * kt[i] + d < kn[i];
      }
      if (ok) mask |= 1ull << k;
    }
    P->stepX[s] = bx;
    P->stepY[s] = by;
    P->kmask[s] = mask;
    for (int i = 0; i < nk; i++) {
      if (++cd[i] < cdiv(kn[i], kt[i])) break;
      cd[i] = 0;
    }
  }
  // smem layouts: k-contiguous iff the operand's FVI is internal
  kp.xKmajor = !c.t[X].idx.empty() && c.ix[c.t[X].idx[0]].cls == INTL;
  kp.yKmajor = !c.t[Y].idx.empty() && c.ix[c.t[Y].idx[0]].cls == INTL;
  P->slotX1 = build_slots(c, cfg, X, 1, cfg.mdig);
  P->slotY1 = build_slots(c, cfg, Y, 1, cfg.ndig);
  P->vecX_ok = vec_ok(c, cfg, X, cfg.mdig);
  P->vecY_ok = vec_ok(c, cfg, Y, cfg.ndig);
  if (P->vecX_ok) P->slotX2 = build_slots(c, cfg, X, 2, cfg.mdig);
  if (P->vecY_ok) P->slotY2 = build_slots(c, cfg, Y, 2, cfg.ndig);
  (void)var;
  return ST_OK;
}

Status upload(tc_plan_s *P, std::string &err) {
  // one device buffer: stepX | stepY | kmask | slotX1 | slotY1 | slotX2 | slotY2
  size_t off[8];
  size_t o = 0;
  auto al = [](size_t x) { return (x + 255) & ~(size_t)255; };
  off[0] = o; o = al(o + 8 * P->stepX.size());
  off[1] = o; o = al(o + 8 * P->stepY.size());
  off[2] = o; o = al(o + 8 * P->kmask.size());
  off[3] = o; o = al(o + 4 * P->slotX1.size());
  off[4] = o; o = al(o + 4 * P->slotY1.size());
  off[5] = o; o = al(o + 4 * P->slotX2.size());
  off[6] = o; o = al(o + 4 * P->slotY2.size());
  off[7] = o;
  std::vector<char> h(o, 0);
  std::memcpy(h.data() + off[0], P->stepX.data(), 8 * P->stepX.size());
  std::memcpy(h.data() + off[1], P->stepY.data(), 8 * P->stepY.size());
  std::memcpy(h.data() + off[2], P->kmask.data(), 8 * P->kmask.size());
  std::memcpy(h.data() + off[3], P->slotX1.data(), 4 * P->slotX1.size());
  std::memcpy(h.data() + off[4], P->slotY1.data(), 4 * P->slotY1.size());
  if (!P->slotX2.empty()) std::memcpy(h.data() + off[5], P->slotX2.data(), 4 * P->slotX2.size());
  if (!P->slotY2.empty()) std::memcpy(h.data() + off[6], P->slotY2.data(), 4 * P->slotY2.size());
  cudaError_t e = cudaMalloc(&P->dev.buf, o);
  if (e != cudaSuccess) { err = std::string("cudaMalloc: ") + cudaGetErrorString(e); return ST_ALLOC; }
  P->dev.bytes = o;
  e = cudaMemcpy(P->dev.buf, h.data(), o, cudaMemcpyHostToDevice);
  if (e != cudaSuccess) { err = std::string("cudaMemcpy: ") + cudaGetErrorString(e); return ST_CUDA; }
  char *b = (char *)P->dev.buf;
  P->kp.stepX = (const int64_t *)(b + off[0]);
  P->kp.stepY = (const int64_t *)(b + off[1]);
  P->kp.kmask = (const uint64_t *)(b + off[2]);
  P->d_slotX1 = (const uint32_t *)(b + off[3]);
  P->d_slotY1 = (const uint32_t *)(b + off[4]);
  P->d_slotX2 = (const uint32_t *)(b + off[5]);
  P->d_slotY2 = (const uint32_t *)(b + off[6]);
  const KernelEntry &ke = kernels()[P->cfg.variant];
  e = cudaFuncSetAttribute(ke.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ke.smem);
  if (e != cudaSuccess) { err = std::string("cudaFuncSetAttribute: ") + cudaGetErrorString(e); return ST_CUDA; }
  return ST_OK;
}

bool parse_force(const char *s, ForcedTiles &ft) {
  ft.on = s != nullptr;
  if (!s) return true;
  std::string str(s);
  std::stringstream ss(str);
  std::string item;
  while (std::getline(ss, item, ';')) {
    auto p = item.find(':');
    if (item.find_first_not_of(" \t") == std::string::npos) continue;
    if (p == std::string::npos) return false;
    std::string k = item.substr(0, p);
    k.erase(0, k.find_first_not_of(" \t"));
    k.erase(k.find_last_not_of(" \t") + 1);
    try {
      ft.tile[k] = std::stoi(item.substr(p + 1));
    } catch (...) {
      return false;
    }
  }
  return true;
}

tc_status_t finish_plan(tc_plan_s *P, tc_plan_t *out) {
  std::string err;
  P->c = P->parsed;
  normalize(P->c, !P->opts.no_fusion);
  ForcedTiles ft;
  if (!parse_force(P->opts.force_tiles, ft)) { delete P; return fail(ST_INVALID_ARG, "malformed force_tiles"); }
  if (ft.on && !P->opts.no_fusion) {
    // forced tiles name the original indices: plan without fusion so names survive
    P->c = P->parsed;
    normalize(P->c, false);
  }
  int fv = P->opts.variant > 0 ? P->opts.variant - 1 : -1;
  if (fv >= (int)variants().size()) { delete P; return fail(ST_INVALID_ARG, "variant out of range"); }
  Status s = choose(P->c, P->opts.cost_mode, fv, ft, P->cfg, P->stats, err);
  if (s != ST_OK) { delete P; return fail(s, err); }
  s = build_tables(P, err);
  if (s != ST_OK) { delete P; return fail(s, err); }
  if (!P->host_only) {
    if (cudaGetDevice(&P->device) != cudaSuccess) {
      cudaGetLastError();
      delete P;
      return fail(ST_CUDA, "no CUDA device (use opts.host_only to plan without one)");
    }
    s = upload(P, err);
    if (s != ST_OK) { delete P; return fail(s, err); }
  }
  *out = P;
  return TC_SUCCESS;
}

bool overlaps(const void *a, size_t na, const void *b, size_t nb) {
  const char *x = (const char *)a, *y = (const char *)b;
  return x < y + nb && y < x + na;
}

}  // namespace

extern "C" {

const char *tc_version(void) { return "libtc 0.1 (sm_100a, FP64 DMMA)"; }

const char *tc_status_string(tc_status_t s) {
  switch (s) {
    case TC_SUCCESS: return "TC_SUCCESS";
    case TC_ERR_INVALID_ARG: return "TC_ERR_INVALID_ARG";
    case TC_ERR_PARSE: return "TC_ERR_PARSE";
    case TC_ERR_INDEX: return "TC_ERR_INDEX";
    case TC_ERR_EXTENT: return "TC_ERR_EXTENT";
    case TC_ERR_UNSUPPORTED: return "TC_ERR_UNSUPPORTED";
    case TC_ERR_NO_CONFIG: return "TC_ERR_NO_CONFIG";
    case TC_ERR_CUDA: return "TC_ERR_CUDA";
    case TC_ERR_ALLOC: return "TC_ERR_ALLOC";
  }
  return "TC_ERR_UNKNOWN";
}

const char *tc_last_error(void) { return g_err.c_str(); }

tc_status_t tc_check(const char *expr, const char *extents) {
  try {
    Contraction c;
    std::string err;
    Status s = parse(expr, extents, c, err);
    if (s != ST_OK) return fail(s, err);
    return TC_SUCCESS;
  } catch (...) {
    return fail(ST_ALLOC, "exception in tc_check");
  }
}

tc_status_t tc_plan_ex(tc_plan_t *plan, const char *expr, const char *extents, tc_dtype_t dtype,
                       const tc_plan_opts *opts) {
  if (!plan) return fail(ST_INVALID_ARG, "plan is NULL");
  *plan = nullptr;
  try {
    tc_plan_s *P = new tc_plan_s();
    if (opts) P->opts = *opts;
    if (opts && opts->force_tiles) {
      P->force_tiles = opts->force_tiles;
      P->opts.force_tiles = P->force_tiles.c_str();
    }
    P->host_only = opts && opts->host_only;
    std::string err;
    Status s = parse(expr, extents, P->parsed, err);
    if (s != ST_OK) { delete P; return fail(s, err); }
    if (dtype != TC_F64) { delete P; return fail(ST_UNSUPPORTED, "only TC_F64 is built in this version"); }
    if (opts && (opts->cost_mode < 0 || opts->cost_mode > 1)) { delete P; return fail(ST_INVALID_ARG, "cost_mode"); }
    P->dtype = dtype;
    return finish_plan(P, plan);
  } catch (std::bad_alloc &) {
    return fail(ST_ALLOC, "out of host memory");
  } catch (...) {
    return fail(ST_ALLOC, "exception in tc_plan");
  }
}

tc_status_t tc_plan(tc_plan_t *plan, const char *expr, const char *extents, tc_dtype_t dtype) {
  return tc_plan_ex(plan, expr, extents, dtype, nullptr);
}

void tc_plan_destroy(tc_plan_t plan) { delete plan; }

double tc_plan_flops(const tc_plan_t plan) { return plan ? plan->parsed.flops() : 0.0; }

int64_t tc_plan_numel(const tc_plan_t plan, int t) {
  if (!plan || t < 0 || t > 2) return -1;
  return plan->parsed.numel(t);
}

tc_status_t tc_plan_restrict(tc_plan_t *sub, const tc_plan_t parent, const char *index,
                             int64_t begin, int64_t len, unsigned flags) {
  if (!sub || !parent || !index) return fail(ST_INVALID_ARG, "NULL argument");
  *sub = nullptr;
  try {
    const Contraction &pc = parent->parsed;
    int id = -1;
    for (size_t i = 0; i < pc.ix.size(); i++) if (pc.ix[i].name == index) id = (int)i;
    if (id < 0) return fail(ST_INDEX, std::string("unknown index '") + index + "'");
    if (begin < 0 || len < 1 || begin + len > pc.ix[id].n) return fail(ST_EXTENT, "slab out of range");
    tc_plan_s *P = new tc_plan_s();
    P->opts = parent->opts;
    P->force_tiles = parent->force_tiles;
    P->opts.force_tiles = parent->opts.force_tiles ? P->force_tiles.c_str() : nullptr;
    P->host_only = parent->host_only;
    P->dtype = parent->dtype;
    Contraction c = pc;
    c.ix[id].n = len;
    const unsigned slab[3] = {TC_SLAB_C, TC_SLAB_A, TC_SLAB_B};
    for (int t = 0; t < 3; t++) {
      int p = c.pos_in(t, id);
      if (p < 0) continue;
      if (flags & slab[t]) {
        // compact slab: a dense tensor of its own
        int64_t st = 1;
        for (size_t k = 0; k < c.t[t].idx.size(); k++) {
          c.t[t].stride[k] = st;
          st *= c.ix[c.t[t].idx[k]].n;
        }
        c.t[t].base = 0;
        c.parent_numel[t] = st;
      } else {
        c.t[t].base += begin * c.t[t].stride[p];
      }
    }
    P->parsed = c;
    return finish_plan(P, sub);
  } catch (...) {
    return fail(ST_ALLOC, "exception in tc_plan_restrict");
  }
}

tc_status_t tc_execute(const tc_plan_t plan, const void *A, const void *B, void *C, double alpha,
                       double beta, tc_stream_t stream) {
  if (!plan || !A || !B || !C) return fail(ST_INVALID_ARG, "NULL plan or tensor pointer");
  if (plan->host_only || !plan->dev.buf) return fail(ST_CUDA, "plan was made host_only");
  const Contraction &c = plan->c;
  const size_t es = 8;
  const size_t nA = (size_t)plan->parsed.span(1) * es, nB = (size_t)plan->parsed.span(2) * es,
               nC = (size_t)plan->parsed.span(0) * es;
  if (overlaps(C, nC, A, nA) || overlaps(C, nC, B, nB)) return fail(ST_INVALID_ARG, "C overlaps A or B");
  int cur = -1;
  if (cudaGetDevice(&cur) != cudaSuccess || cur != plan->device)
    return fail(ST_INVALID_ARG, "current device differs from the plan's device");
  KParams kp = plan->kp;
  const int X = plan->cfg.X;
  kp.X = X == 1 ? A : B;
  kp.Y = X == 1 ? B : A;
  kp.C = C;
  kp.alpha = alpha;
  kp.beta = beta;
  const bool ax = ((uintptr_t)kp.X % 16) == 0, ay = ((uintptr_t)kp.Y % 16) == 0;
  const bool vx = plan->vecX_ok && ax, vy = plan->vecY_ok && ay;
  kp.slotX = vx ? plan->d_slotX2 : plan->d_slotX1;
  kp.nslotX = (int)(vx ? plan->slotX2.size() : plan->slotX1.size());
  kp.vecX = vx ? 2 : 1;
  kp.slotY = vy ? plan->d_slotY2 : plan->d_slotY1;
  kp.nslotY = (int)(vy ? plan->slotY2.size() : plan->slotY1.size());
  kp.vecY = vy ? 2 : 1;
  (void)c;
  const KernelEntry &ke = kernels()[plan->cfg.variant];
  void *args[] = {&kp};
  cudaError_t e = cudaLaunchKernel(ke.fn, dim3((unsigned)kp.nctas), dim3(ke.threads), args, ke.smem,
                                   (cudaStream_t)stream);
  if (e != cudaSuccess) return fail(ST_CUDA, std::string("launch: ") + cudaGetErrorString(e));
  return TC_SUCCESS;
}

size_t tc_plan_workspace_bytes(const tc_plan_t plan) {
  if (!plan) return 0;
  auto al = [](size_t x) { return (x + 255) & ~(size_t)255; };
  const Contraction &c = plan->parsed;
  return al(8 * c.parent_numel[1]) + al(8 * c.parent_numel[2]) + al(8 * c.parent_numel[0]);
}

tc_status_t tc_execute_host(const tc_plan_t plan, const void *A_host, const void *B_host, void *C_host,
                            double alpha, double beta, void *workspace, size_t workspace_bytes,
                            tc_stream_t stream) {
  if (!plan || !A_host || !B_host || !C_host || !workspace) return fail(ST_INVALID_ARG, "NULL argument");
  if (workspace_bytes < tc_plan_workspace_bytes(plan)) return fail(ST_INVALID_ARG, "workspace too small");
  auto al = [](size_t x) { return (x + 255) & ~(size_t)255; };
  const Contraction &c = plan->parsed;
  const size_t bA = 8 * c.parent_numel[1], bB = 8 * c.parent_numel[2], bC = 8 * c.parent_numel[0];
  char *w = (char *)workspace;
  void *dA = w, *dB = w + al(bA), *dC = w + al(bA) + al(bB);
  cudaStream_t s = (cudaStream_t)stream;
  cudaError_t e = cudaMemcpyAsync(dA, A_host, bA, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = cudaMemcpyAsync(dB, B_host, bB, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess && beta != 0.0) e = cudaMemcpyAsync(dC, C_host, bC, cudaMemcpyHostToDevice, s);
  if (e != cudaSuccess) return fail(ST_CUDA, std::string("H2D: ") + cudaGetErrorString(e));
  tc_status_t st = tc_execute(plan, dA, dB, dC, alpha, beta, stream);
  if (st != TC_SUCCESS) return st;
  e = cudaMemcpyAsync(C_host, dC, bC, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return fail(ST_CUDA, std::string("D2H/sync: ") + cudaGetErrorString(e));
  return TC_SUCCESS;
}

tc_status_t tc_plan_info(const tc_plan_t plan, char *json, size_t cap, size_t *needed) {
  if (!plan) return fail(ST_INVALID_ARG, "plan is NULL");
  try {
    const Contraction &c = plan->c;
    const Config &g = plan->cfg;
    const Variant &v = variants()[g.variant];
    std::ostringstream o;
    auto names = [&](const std::vector<int> &l) {
      std::string s = "[";
      for (size_t i = 0; i < l.size(); i++) s += (i ? ",\"" : "\"") + c.ix[l[i]].name + "\"";
      return s + "]";
    };
    o << "{\"dtype\":\"f64\",\"X\":\"" << (g.X == 1 ? "A" : "B") << "\"";
    o << ",\"indices\":[";
    for (size_t i = 0; i < c.ix.size(); i++) {
      const char *cls = c.ix[i].cls == EXT_A ? "extA" : c.ix[i].cls == EXT_B ? "extB" : "int";
      o << (i ? "," : "") << "{\"name\":\"" << c.ix[i].name << "\",\"n\":" << c.ix[i].n
        << ",\"cls\":\"" << cls << "\",\"tile\":" << g.T[i] << "}";
    }
    o << "],\"tensors\":{";
    const char *tn[3] = {"C", "A", "B"};
    for (int t = 0; t < 3; t++) {
      o << (t ? "," : "") << "\"" << tn[t] << "\":{\"idx\":" << names(c.t[t].idx) << ",\"stride\":[";
      for (size_t k = 0; k < c.t[t].stride.size(); k++) o << (k ? "," : "") << c.t[t].stride[k];
      o << "],\"base\":" << c.t[t].base << "}";
    }
    o << "},\"m\":" << names(g.mdig) << ",\"n\":" << names(g.ndig) << ",\"k\":" << names(g.kdig);
    o << ",\"variant\":" << g.variant << ",\"BM\":" << v.BM << ",\"BN\":" << v.BN << ",\"BK\":" << v.BK
      << ",\"threads\":" << v.threads << ",\"stages\":" << v.stages << ",\"occ\":" << v.occ;
    o << ",\"Mt\":" << g.Mt << ",\"Nt\":" << g.Nt << ",\"Kt\":" << g.Kt << ",\"nctas\":" << g.nctas
      << ",\"nsteps\":" << g.nsteps;
    o << ",\"vecX\":" << (plan->vecX_ok ? 2 : 1) << ",\"vecY\":" << (plan->vecY_ok ? 2 : 1)
      << ",\"xKmajor\":" << plan->kp.xKmajor << ",\"yKmajor\":" << plan->kp.yKmajor;
    char buf[512];
    std::snprintf(buf, sizeof buf,
                  ",\"t_pred_ms\":%.6g,\"t_comp_ms\":%.6g,\"t_mem_ms\":%.6g,\"t_l2_ms\":%.6g,"
                  "\"dram_bytes\":%.6g,\"flops\":%.6g,\"flops_padded\":%.6g,\"paper_cost\":%.6g",
                  g.t_pred * 1e3, g.t_comp * 1e3, g.t_mem * 1e3, g.t_l2 * 1e3, g.dram_bytes,
                  plan->parsed.flops(), g.flops_pad, g.paper_cost);
    o << buf;
    o << ",\"paper_mapping\":\"" << g.paper_mapping << "\"";
    o << ",\"stats\":{\"cost_mode\":\"" << (plan->stats.cost_mode ? "paper" : "b200")
      << "\",\"raw\":" << plan->stats.raw << ",\"pruned\":" << plan->stats.pruned
      << ",\"ranked\":" << plan->stats.ranked << ",\"plan_ms\":" << plan->stats.plan_ms << "}";
    o << ",\"host_only\":" << (plan->host_only ? "true" : "false") << "}";
    std::string s = o.str();
    if (needed) *needed = s.size() + 1;
    if (json && cap) {
      size_t n = std::min(cap - 1, s.size());
      std::memcpy(json, s.data(), n);
      json[n] = 0;
    }
    return TC_SUCCESS;
  } catch (...) {
    return fail(ST_ALLOC, "exception in tc_plan_info");
  }
}

}  // extern "C"
