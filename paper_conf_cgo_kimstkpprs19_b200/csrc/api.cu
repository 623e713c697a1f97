// api.cu — the C ABI of libtc (include/libtc.h): plan construction (rows a1-a4), launch
// metadata (row a4), kernel dispatch (rows a5-a7), restriction (row e) and introspection.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cmath>
#include <map>
#include <mutex>
#include <cstdio>
#include <cstring>
#include <new>
#include <sstream>
#include <string>
#include <vector>

#include "../../include/libtc.h"
#include "contraction.hpp"
#include "kernel_table.cuh"
#include "kparams.hpp"
#include "planner.hpp"
#include "tiles.hpp"
#include "plan_internal.hpp"

using namespace tc;

namespace {
thread_local std::string g_err;

tc_status_t fail(Status s, const std::string &msg) {
  g_err = msg;
  return (tc_status_t)s;
}
}  // namespace

namespace tc {
tc_status_t set_error(Status s, const std::string &msg) { return fail(s, msg); }
std::string &last_error_string() { return g_err; }
}  // namespace tc

namespace {

// ---------------------------------------------------------------- kernel table
struct KernelEntry {
  const void *fn;
  int threads;
  size_t smem;       // without the TMA staging box
  size_t smem_tma;   // with it
};

// Kernel family of a dtype: FP64 -> DMMA; BF16 / TF32 / FP32 (split TF32) -> tcgen05.
int kind_of(int dtype) {
  return dtype == TC_BF16 ? KIND_BF16_UMMA : dtype == TC_TF32 ? KIND_TF32_UMMA
       : dtype == TC_F32 ? KIND_F32X3_UMMA : KIND_F64_DMMA;
}

// The instance for the plan's variant and smem layouts (kernel_table.cuh).
KernelEntry kernel_for(const Config &cfg, bool tma_operands = false) {
  const Variant &v = variants()[cfg.variant];
  if (is_umma(v.kind)) {
    size_t smem = 0;
    int threads = 0;
    const void *fn = kernel_ptr_umma(cfg.variant, cfg.xKmajor, cfg.yKmajor, tma_operands, &smem, &threads);
    return {fn, threads, smem, smem};
  }
  const F64Instance k = cfg.xKmajor ? (cfg.yKmajor ? f64_instance_11(cfg.variant) : f64_instance_10(cfg.variant))
                                    : (cfg.yKmajor ? f64_instance_01(cfg.variant) : f64_instance_00(cfg.variant));
  return {k.fn, k.threads, k.smem, k.smem_tma};
}

}  // namespace


namespace {

void build_host_tables(tc_plan_s *P) {
  const Contraction &c = P->c;
  const Config &cfg = P->cfg;
  const Variant &v = variants()[cfg.variant];
  P->tt = build_tile_tables(c, cfg, v);
  if (is_umma(cfg.kind)) {
    // padding entry past each tile list: the CTA-pair kernel's blocks that overhang the tile
    // grid read it (coordinates outside every tensor -> TMA zero fill; masks 0 -> no stores)
    TileInfo pad{};
    for (int q = 0; q < kMaxTmaDims; q++) pad.coord[q] = 1 << 30;
    P->tt.tileM.push_back(pad);
    P->tt.tileN.push_back(pad);
  }
  P->slotX1 = build_slots(c, cfg, cfg.X, 1, cfg.xKmajor, v.BM, v.BK);
  P->slotY1 = build_slots(c, cfg, cfg.Y, 1, cfg.yKmajor, v.BN, v.BK);
  if (cfg.vecX > 1) P->slotX2 = build_slots(c, cfg, cfg.X, cfg.vecX, cfg.xKmajor, v.BM, v.BK);
  if (cfg.vecY > 1) P->slotY2 = build_slots(c, cfg, cfg.Y, cfg.vecY, cfg.yKmajor, v.BN, v.BK);
  int cs0 = 1, ct0 = 1;
  P->cvec = is_umma(cfg.kind) ? c_run_rows(c, cfg, 8, &cs0, &ct0) : (v.stg ? c_vec_width(c, cfg, 2) : 1);
  KParams &kp = P->kp;
  std::memset(&kp, 0, sizeof(kp));
  kp.mtiles = (int)cfg.mtiles;
  kp.ntiles = (int)cfg.ntiles;
  kp.ntotal = (int)cfg.nctas;
  kp.group_m = 8;
  kp.nsteps = (int)cfg.nsteps;
  for (int w = 0; w < kMaskWords; w++) {
    kp.fullM[w] = P->tt.tileM[0].mask[w];   // the origin tile is always interior (T <= N)
    kp.fullN[w] = P->tt.tileN[0].mask[w];
  }
  kp.fullK = cfg.Kt >= 64 ? ~0ull : ((1ull << cfg.Kt) - 1);
  kp.kcnt0 = P->tt.kcnt0;
  kp.kdX0 = P->tt.kdX0;
  kp.kdY0 = P->tt.kdY0;
  kp.ktail0 = P->tt.ktail0;
  kp.kbase = P->tt.kbase;
  kp.nouter = (int)P->tt.kouter.size();
  kp.Mt = (int)cfg.Mt;
  P->batch.clear();
  for (size_t id = 0; id < c.ix.size(); id++)
    if (c.ix[id].cls == BATCH)
      P->batch.push_back({c.ix[id].n, c.stride_of(cfg.X, (int)id), c.stride_of(cfg.Y, (int)id),
                          c.stride_of(0, (int)id)});
  kp.cs0 = cs0;
  kp.nmma = v.BN;
  kp.kmma = v.BK;
  if (is_umma(cfg.kind)) umma_trim(cfg, v, &kp.nmma, &kp.kmma);
  kp.ct0 = ct0;
  kp.Nt = (int)cfg.Nt;
  kp.c_rank = (int)c.t[0].idx.size();
  // old-C prefetch (beta != 0): C's FVI leads the m digits, so runs of its tile are C-contiguous
  // rows: one address per 128-B line (16 doubles)
  P->umma_tma = !P->opts.no_tma_operands && !P->out_f32 &&
                umma_tma_spec(c, cfg, v, cfg.X, &P->mapX, &kp.xt) &&
                umma_tma_spec(c, cfg, v, cfg.Y, &P->mapY, &kp.yt);
  kp.kt = cfg.kdig.empty() ? 0 : (int)cfg.T[cfg.kdig[0]];
  // CTA pairs: BN = 128 BF16 / TF32 instances with TMA operands, when asked for (cta_pair 2)
  // or (planner's choice) when the grid holds at least two waves of pair blocks
  {
    // (the pair epilogue stores from TMEM rows: C's FVI must lead m when the plan stores runs)
    const bool can = P->umma_tma && (cfg.variant == 12 || cfg.variant == 22) && (P->cvec != 8 || cs0 == 1);
    P->pair = can && (P->opts.cta_pair == 2 || (P->opts.cta_pair == 0 && cta_pair_default(cfg)));
  }
  P->pf_step = 0;
  if (cfg.kind == KIND_F64_DMMA && !cfg.mdig.empty() && !c.t[0].idx.empty() && cfg.mdig[0] == c.t[0].idx[0] &&
      c.t[0].stride[0] == 1)
    P->pf_step = std::min<int>(16, cfg.T[cfg.mdig[0]]);
}

Status upload(tc_plan_s *P, std::string &err) {
  struct Part { const void *src; size_t bytes; size_t off; };
  std::vector<Part> parts;
  size_t o = 0;
  auto add = [&](const void *src, size_t bytes) {
    parts.push_back({src, bytes, o});
    o = (o + bytes + 255) & ~(size_t)255;
    return parts.size() - 1;
  };
  const TileTables &tt = P->tt;
  size_t iM = add(tt.tileM.data(), sizeof(TileInfo) * tt.tileM.size());
  size_t iN = add(tt.tileN.data(), sizeof(TileInfo) * tt.tileN.size());
  size_t iRm = add(tt.relCm.data(), 8 * tt.relCm.size());
  size_t iRn = add(tt.relCn.data(), 8 * tt.relCn.size());
  size_t iBm = add(tt.boxM.data(), 4 * tt.boxM.size());
  size_t iBn = add(tt.boxN.data(), 4 * tt.boxN.size());
  size_t iKo = add(tt.kouter.data(), sizeof(KOuter) * tt.kouter.size());
  // slot offsets inside a (tile, step) are 32-bit in the kernel (registers are scarce)
  std::vector<int32_t> r32[4];
  const SlotTable *sts[4] = {&P->slotX1, &P->slotY1, &P->slotX2, &P->slotY2};
  for (int q = 0; q < 4; q++)
    for (int64_t v : sts[q]->rel) {
      if (v > INT32_MAX || v < INT32_MIN) { err = "tile spans more than 2^31 elements of an operand"; return ST_UNSUPPORTED; }
      r32[q].push_back((int32_t)v);
    }
  size_t iX1 = add(r32[0].data(), 4 * r32[0].size());
  size_t iX1p = add(P->slotX1.pack.data(), 4 * P->slotX1.pack.size());
  size_t iY1 = add(r32[1].data(), 4 * r32[1].size());
  size_t iY1p = add(P->slotY1.pack.data(), 4 * P->slotY1.pack.size());
  size_t iX2 = add(r32[2].data(), 4 * r32[2].size());
  size_t iX2p = add(P->slotX2.pack.data(), 4 * P->slotX2.pack.size());
  size_t iY2 = add(r32[3].data(), 4 * r32[3].size());
  size_t iY2p = add(P->slotY2.pack.data(), 4 * P->slotY2.pack.size());
  size_t iS = add(P->stream.tab.data(), 4 * P->stream.tab.size());
  std::vector<char> h(o + 256, 0);
  for (auto &p : parts) if (p.bytes) std::memcpy(h.data() + p.off, p.src, p.bytes);
  cudaError_t e = cudaMalloc(&P->dev, h.size());
  if (e != cudaSuccess) { err = std::string("cudaMalloc: ") + cudaGetErrorString(e); return ST_ALLOC; }
  P->dev_bytes = h.size();
  e = cudaMemcpy(P->dev, h.data(), h.size(), cudaMemcpyHostToDevice);
  if (e != cudaSuccess) { err = std::string("cudaMemcpy: ") + cudaGetErrorString(e); return ST_CUDA; }
  char *b = (char *)P->dev;
  KParams &kp = P->kp;
  kp.tileM = (const TileInfo *)(b + parts[iM].off);
  kp.tileN = (const TileInfo *)(b + parts[iN].off);
  kp.relCm = (const int64_t *)(b + parts[iRm].off);
  kp.relCn = (const int64_t *)(b + parts[iRn].off);
  kp.boxM = (const int32_t *)(b + parts[iBm].off);
  kp.boxN = (const int32_t *)(b + parts[iBn].off);
  kp.kouter = (const KOuter *)(b + parts[iKo].off);
  P->d_relX1 = (const int32_t *)(b + parts[iX1].off);
  P->d_packX1 = (const uint32_t *)(b + parts[iX1p].off);
  P->d_relY1 = (const int32_t *)(b + parts[iY1].off);
  P->d_packY1 = (const uint32_t *)(b + parts[iY1p].off);
  P->d_relX2 = (const int32_t *)(b + parts[iX2].off);
  P->d_packX2 = (const uint32_t *)(b + parts[iX2p].off);
  P->d_relY2 = (const int32_t *)(b + parts[iY2].off);
  P->d_packY2 = (const uint32_t *)(b + parts[iY2p].off);
  if (P->stream.on) {
    P->stream.kp.tab = (const uint32_t *)(b + parts[iS].off);
    const void *fn = stream_kernel_ptr(P->cfg.kind, P->stream.NB, P->stream.AR, P->stream.mode != SM_K, false);
    if (!fn) { err = "no streaming kernel instance for the plan"; return ST_UNSUPPORTED; }
    // (the instances are shared by plans of different sizes: always the opt-in maximum)
    e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, 232448);
    if (e != cudaSuccess) { err = std::string("cudaFuncSetAttribute: ") + cudaGetErrorString(e); return ST_CUDA; }
    if (const void *fb = stream_kernel_ptr(P->cfg.kind, P->stream.NB, P->stream.AR, P->stream.mode != SM_K, true)) {
      e = cudaFuncSetAttribute(fb, cudaFuncAttributeMaxDynamicSharedMemorySize, 232448);
      if (e != cudaSuccess) { err = std::string("cudaFuncSetAttribute: ") + cudaGetErrorString(e); return ST_CUDA; }
    }
    int socc = 0, nsm = 148;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&socc, fn, kSThreads, P->stream.smem);
    if (e != cudaSuccess || socc < 1) { err = "streaming kernel cannot be resident"; return ST_CUDA; }
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, P->device);
    P->stream_grid = nsm * std::min(socc, P->stream.occ);
  }
  if (P->umma_tma) {   // the TMA-operand instance: same smem, its own attribute
    const KernelEntry kt = kernel_for(P->cfg, true);
    e = cudaFuncSetAttribute(kt.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kt.smem);
    if (e != cudaSuccess) { err = std::string("cudaFuncSetAttribute: ") + cudaGetErrorString(e); return ST_CUDA; }
  }
  if (P->out_f32) {
    size_t sm = 0;
    int th = 0;
    const void *fn = kernel_ptr_umma_f32out(P->cfg.variant, P->cfg.xKmajor, P->cfg.yKmajor, &sm, &th);
    if (!fn) { err = "no FP32-output instance for the variant"; return ST_UNSUPPORTED; }
    e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) { err = std::string("cudaFuncSetAttribute: ") + cudaGetErrorString(e); return ST_CUDA; }
  }
  if (P->pair) {
    size_t sm = 0;
    int th = 0;
    const void *fn = kernel_ptr_umma_pair(P->cfg.variant, P->cfg.xKmajor, P->cfg.yKmajor, &sm, &th);
    if (!fn) { err = "no CTA-pair instance for the variant"; return ST_UNSUPPORTED; }
    e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) { err = std::string("cudaFuncSetAttribute: ") + cudaGetErrorString(e); return ST_CUDA; }
  }
  const KernelEntry ke = kernel_for(P->cfg);
  const bool tma = P->tt.tma_ok && P->opts.tma_epilogue && P->cfg.kind == KIND_F64_DMMA &&
                   !variants()[P->cfg.variant].stg;
  // The attribute belongs to the kernel instance, which many plans share: always set the
  // largest size any plan of the instance may launch with (the TMA staging box when it fits),
  // so a later plan without the TMA epilogue cannot shrink it under an earlier plan's launch.
  const size_t kMaxSmem = 227 * 1024;
  const size_t smem_max = ke.smem_tma <= kMaxSmem ? std::max(ke.smem, ke.smem_tma) : ke.smem;
  if (tma && ke.smem_tma > smem_max) { err = "TMA epilogue staging exceeds shared memory"; return ST_UNSUPPORTED; }
  e = cudaFuncSetAttribute(ke.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_max);
  if (e != cudaSuccess) { err = std::string("cudaFuncSetAttribute: ") + cudaGetErrorString(e); return ST_CUDA; }
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ke.fn, ke.threads, tma ? ke.smem_tma : ke.smem);
  if (e != cudaSuccess || occ < 1) { err = "kernel variant cannot be resident"; return ST_CUDA; }
  cudaDeviceGetAttribute(&P->sms, cudaDevAttrMultiProcessorCount, P->device);
  P->sms *= std::min(occ, variants()[P->cfg.variant].occ);
  return ST_OK;
}

bool parse_force(const char *s, ForcedTiles &ft) {
  ft.on = s != nullptr;
  if (!s) return true;
  std::stringstream ss{std::string(s)};
  std::string item;
  while (std::getline(ss, item, ';')) {
    if (item.find_first_not_of(" \t") == std::string::npos) continue;
    auto p = item.find(':');
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

// Same normalised index structure (names, classes, tensor index lists): a configuration made
// for one contraction's extents is then a legal configuration of the other's (tiles clamped).
bool same_structure(const Contraction &a, const Contraction &b) {
  if (a.ix.size() != b.ix.size()) return false;
  for (size_t i = 0; i < a.ix.size(); i++)
    if (a.ix[i].name != b.ix[i].name || a.ix[i].cls != b.ix[i].cls) return false;
  for (int t = 0; t < 3; t++)
    if (a.t[t].idx != b.t[t].idx) return false;
  return true;
}

// rep (optional): a plan whose configuration (variant, digit orders, tiles) is reused when the
// structures match — tiles clamped to the new extents, tables rebuilt, no search (NEXT-1,
// P:L77, L300); otherwise the planner runs as usual.
tc_status_t finish_plan(tc_plan_s *P, tc_plan_t *out, const tc_plan_s *rep = nullptr) {
  std::string err;
  ForcedTiles ft;
  if (!parse_force(P->opts.force_tiles, ft)) { delete P; return fail(ST_INVALID_ARG, "malformed force_tiles"); }
  if (P->opts.morder < 0 || P->opts.morder > 2) { delete P; return fail(ST_INVALID_ARG, "morder must be 0, 1 or 2"); }
  if (P->opts.cta_pair < 0 || P->opts.cta_pair > 2) { delete P; return fail(ST_INVALID_ARG, "cta_pair must be 0, 1 or 2"); }
  if (P->opts.out_f32 != 0 && (P->opts.out_f32 != 1 || P->dtype != TC_BF16))
    { delete P; return fail(ST_INVALID_ARG, "out_f32 is a TC_BF16 option (0 or 1)"); }
  P->out_f32 = P->opts.out_f32 == 1;
  if (P->opts.stream < 0 || P->opts.stream > 2) { delete P; return fail(ST_INVALID_ARG, "stream must be 0, 1 or 2"); }
  if (P->opts.stream_rank < 0 || P->opts.stream_rank >= kStreamRanks)
    { delete P; return fail(ST_INVALID_ARG, "stream_rank out of range"); }
  for (int r : P->opts.reserved)
    if (r != 0) { delete P; return fail(ST_INVALID_ARG, "tc_plan_opts.reserved[] must be zero"); }
  ft.morder = P->opts.morder - 1;
  // forced tiles name the original indices: plan without fusion so the names survive
  P->c = P->parsed;
  normalize(P->c, !P->opts.no_fusion && !ft.on);
  if (!split_large(P->c, err)) { delete P; return fail(ST_UNSUPPORTED, err); }
  const int fv = P->opts.variant > 0 ? P->opts.variant - 1 : -1;
  if (fv >= (int)variants().size()) { delete P; return fail(ST_INVALID_ARG, "variant out of range"); }
  const int kind = kind_of(P->dtype);
  if (fv >= 0 && variants()[fv].kind != kind) { delete P; return fail(ST_INVALID_ARG, "variant is not built for this dtype"); }
  {
    int nb = 0;
    for (auto &ix : P->c.ix) nb += ix.cls == BATCH;
    if (nb > 4 || P->c.nbatch() > 65535) {
      delete P;
      return fail(ST_UNSUPPORTED, "more than 4 batch indices or more than 65535 batch values");
    }
  }
  Status s = ST_NO_CONFIG;
  if (rep && !ft.on && same_structure(rep->c, P->c)) {
    Config cfg = rep->cfg;
    for (size_t id = 0; id < P->c.ix.size(); id++)
      cfg.T[id] = (int)std::min<int64_t>(cfg.T[id], P->c.ix[id].n);
    finish_counts(P->c, cfg);
    if (config_fits(cfg, variants()[cfg.variant])) {
      model_time(P->c, cfg, variants()[cfg.variant]);   // vector widths, predicted time
      P->cfg = cfg;
      P->stats = PlanStats();
      P->stats.cost_mode = P->opts.cost_mode;
      P->resized = true;
      s = ST_OK;
    }
  }
  if (s != ST_OK) s = choose(P->c, kind, P->opts.cost_mode, fv, ft, P->cfg, P->stats, err);
  if (s != ST_OK) { delete P; return fail(s, err); }
  build_host_tables(P);
  // the streaming path (stream.hpp) beside the configuration: on when eligible, unless the
  // caller forced a variant (tests, tuning candidates) or opts.stream says otherwise
  P->stream = StreamCfg();
  P->stream_active = false;
  if (P->opts.stream != 1 && !P->out_f32 && (fv < 0 || P->opts.stream == 2) && !ft.on) {
    StreamCfg sc;
    if (stream_plan(P->c, kind, 148, sc, P->opts.stream_rank)) {
      P->stream = sc;
      P->stream_active = sc.preferred || P->opts.stream == 2;
    } else {
      P->stream.why = sc.why;
    }
  } else {
    P->stream.why = "off (options)";
  }
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

size_t elem_bytes(const tc_plan_s *P) { return (size_t)kind_esize(kind_of(P->dtype)); }
size_t elem_bytes_c(const tc_plan_s *P) { return P->out_f32 ? 4 : elem_bytes(P); }

bool overlaps(const void *a, size_t na, const void *b, size_t nb) {
  const char *x = (const char *)a, *y = (const char *)b;
  return x < y + nb && y < x + na;
}

// cuTensorMapEncodeTiled through the runtime's driver entry point (no -lcuda needed).
PFN_cuTensorMapEncodeTiled_v12000 tma_encoder() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = [] {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess) {
      cudaGetLastError();
      return (PFN_cuTensorMapEncodeTiled_v12000) nullptr;
    }
    return (PFN_cuTensorMapEncodeTiled_v12000)p;
  }();
  return fn;
}

// TMA descriptor of a tcgen05 operand (umma_tma_spec) at this call's pointer.
bool encode_operand_map(const tc_plan_s *P, const OperandMap &m, const void *ptr, TmaDesc &out) {
  auto enc = tma_encoder();
  if (!enc) return false;
  const int es = kind_esize(P->cfg.kind);
  const char *base = (const char *)ptr + (int64_t)es * m.base;
  if ((uintptr_t)base % 16) return false;
  cuuint64_t dims[kMaxTmaDims], strides[kMaxTmaDims];
  cuuint32_t box[kMaxTmaDims], el[kMaxTmaDims];
  for (int j = 0; j < m.rank; j++) {
    dims[j] = (cuuint64_t)m.dims[j];
    box[j] = m.box[j];
    el[j] = 1;
    if (j > 0) strides[j - 1] = (cuuint64_t)m.strides[j - 1];
  }
  CUresult e = enc(reinterpret_cast<CUtensorMap *>(&out),
                   es == 2 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                   (cuuint32_t)m.rank, (void *)base, dims, strides, box, el, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   m.swz32 ? CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B : CU_TENSOR_MAP_SWIZZLE_128B,
#ifdef TC_UMMA_TMA_PROMO
                   (CUtensorMapL2promotion)TC_UMMA_TMA_PROMO,
#else
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
#endif
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return e == CUDA_SUCCESS;
}

// TMA descriptor of the plan's C view: dims in C order, the C tile as the box.
bool encode_c_map(const tc_plan_s *P, void *C, TmaDesc &out) {
  auto enc = tma_encoder();
  if (!enc) return false;
  const Contraction &c = P->c;
  const auto &cv = c.t[0];
  const int r = (int)cv.idx.size();
  const char *base = (const char *)C + 8 * cv.base;
  if ((uintptr_t)base % 16) return false;
  cuuint64_t dims[kMaxTmaDims], strides[kMaxTmaDims];
  cuuint32_t box[kMaxTmaDims], es[kMaxTmaDims];
  for (int p = 0; p < r; p++) {
    const int id = cv.idx[p];
    dims[p] = (cuuint64_t)c.ix[id].n;
    box[p] = (cuuint32_t)P->cfg.T[id];
    es[p] = 1;
    if (p > 0) strides[p - 1] = (cuuint64_t)(cv.stride[p] * 8);
  }
  static_assert(sizeof(TmaDesc) == sizeof(CUtensorMap), "descriptor size");
  CUresult e = enc(reinterpret_cast<CUtensorMap *>(&out), CU_TENSOR_MAP_DATA_TYPE_FLOAT64, (cuuint32_t)r,
                   (void *)base, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return e == CUDA_SUCCESS;
}

// The streaming path's X tensor map at this call's pointer (stream.hpp): X boxes in X's order,
// zero fill outside the tensor.  C must be aligned for the AR-element run stores.
bool encode_stream_maps(const tc_plan_s *P, const void *Xp, void *C, SParams &sp) {
  auto enc = tma_encoder();
  if (!enc) return false;
  const StreamCfg &s = P->stream;
  const int es = kind_esize(P->cfg.kind);
  const char *xb = (const char *)Xp + es * s.xbase;
  const char *cb = (const char *)C + es * s.cbase;
  if ((uintptr_t)xb % 16 || (uintptr_t)cb % 16) return false;
  cuuint64_t dims[kMaxTmaDims], strides[kMaxTmaDims];
  cuuint32_t box[kMaxTmaDims], el[kMaxTmaDims];
  for (int j = 0; j < s.xrank; j++) {
    dims[j] = (cuuint64_t)s.xdims[j];
    box[j] = s.xbox[j];
    el[j] = 1;
    if (j > 0) strides[j - 1] = (cuuint64_t)(s.xstr[j] * es);
  }
  return enc(reinterpret_cast<CUtensorMap *>(&sp.xmap),
             es == 8 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT64 : es == 4 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, (cuuint32_t)s.xrank,
             (void *)xb, dims, strides, box, el, CU_TENSOR_MAP_INTERLEAVE_NONE, (CUtensorMapSwizzle)s.xswz,
#ifdef TC_STREAM_PROMO
             (CUtensorMapL2promotion)TC_STREAM_PROMO,
#else
             CU_TENSOR_MAP_L2_PROMOTION_NONE,
#endif
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

}  // namespace

extern "C" {

const char *tc_version(void) { return "libtc 0.4 (sm_100a, FP64 DMMA + BF16/TF32/FP32-split tcgen05, persistent)"; }

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
    if (dtype != TC_F64 && dtype != TC_BF16 && dtype != TC_TF32 && dtype != TC_F32)
      { delete P; return fail(ST_UNSUPPORTED, "dtype must be TC_F64, TC_F32, TC_TF32 or TC_BF16"); }
    if (opts && (opts->cost_mode < 0 || opts->cost_mode > 1)) { delete P; return fail(ST_INVALID_ARG, "cost_mode"); }
    P->dtype = dtype;
    P->expr = expr;
    return finish_plan(P, plan);
  } catch (std::bad_alloc &) {
    return fail(ST_ALLOC, "out of host memory");
  } catch (...) {
    return fail(ST_ALLOC, "exception in tc_plan");
  }
}

tc_status_t tc_plan_strided(tc_plan_t *plan, const char *expr, const char *extents, tc_dtype_t dtype,
                            const int64_t *strideC, const int64_t *strideA, const int64_t *strideB,
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
    if (dtype != TC_F64 && dtype != TC_BF16 && dtype != TC_TF32 && dtype != TC_F32)
      { delete P; return fail(ST_UNSUPPORTED, "dtype must be TC_F64, TC_F32, TC_TF32 or TC_BF16"); }
    if (opts && (opts->cost_mode < 0 || opts->cost_mode > 1)) { delete P; return fail(ST_INVALID_ARG, "cost_mode"); }
    P->dtype = dtype;
    Contraction &c = P->parsed;
    const int64_t *st[3] = {strideC, strideA, strideB};
    for (int t = 0; t < 3; t++) {
      if (!st[t]) continue;
      TensorView &v = c.t[t];
      long double span = 1;
      for (size_t k = 0; k < v.idx.size(); k++) {
        if (st[t][k] < (t == 0 ? 1 : 0)) { delete P; return fail(ST_INVALID_ARG, "negative stride (or a zero stride of C)"); }
        v.stride[k] = st[t][k];
        span += (long double)(c.ix[v.idx[k]].n - 1) * (long double)st[t][k];
      }
      if (span > (long double)(int64_t(1) << 62)) { delete P; return fail(ST_INVALID_ARG, "strided span overflows"); }
      if (t == 0) {   // C must not alias itself: sorted by stride, each dim clears the previous
        std::vector<std::pair<int64_t, int64_t>> d;
        for (size_t k = 0; k < v.idx.size(); k++)
          if (c.ix[v.idx[k]].n > 1) d.push_back({v.stride[k], c.ix[v.idx[k]].n});
        std::sort(d.begin(), d.end());
        for (size_t k = 1; k < d.size(); k++)
          if (d[k].first < d[k - 1].first * d[k - 1].second) { delete P; return fail(ST_INVALID_ARG, "C strides overlap"); }
      }
      c.parent_numel[t] = c.span(t);
    }
    return finish_plan(P, plan);
  } catch (std::bad_alloc &) {
    return fail(ST_ALLOC, "out of host memory");
  } catch (...) {
    return fail(ST_ALLOC, "exception in tc_plan_strided");
  }
}

tc_status_t tc_plan_resize(tc_plan_t *sized, const tc_plan_t rep, const char *extents) {
  if (!sized || !rep || !extents) return fail(ST_INVALID_ARG, "NULL argument");
  *sized = nullptr;
  if (rep->expr.empty()) return fail(ST_INVALID_ARG, "only plans made by tc_plan / tc_plan_ex / tc_plan_cached resize");
  try {
    tc_plan_s *P = new tc_plan_s();
    P->opts = rep->opts;
    P->force_tiles = rep->force_tiles;
    P->opts.force_tiles = rep->opts.force_tiles ? P->force_tiles.c_str() : nullptr;
    P->host_only = rep->host_only;
    P->dtype = rep->dtype;
    P->expr = rep->expr;
    std::string err;
    Status s = parse(P->expr.c_str(), extents, P->parsed, err);
    if (s != ST_OK) { delete P; return fail(s, err); }
    if (!rep->host_only) {
      int dev = -1;
      if (cudaGetDevice(&dev) != cudaSuccess || dev != rep->device) {
        cudaGetLastError();
        delete P;
        return fail(ST_INVALID_ARG, "current device differs from the plan's device");
      }
    }
    return finish_plan(P, sized, rep);
  } catch (std::bad_alloc &) {
    return fail(ST_ALLOC, "out of host memory");
  } catch (...) {
    return fail(ST_ALLOC, "exception in tc_plan_resize");
  }
}

tc_status_t tc_plan_select(tc_plan_t *sized, const tc_plan_t *versions, int n, const char *extents, int *chosen) {
  if (!sized || !versions || n < 1 || !extents) return fail(ST_INVALID_ARG, "NULL argument or n < 1");
  *sized = nullptr;
  try {
    // the cost model at the actual extents ranks the versions' configurations ("the
    // kernel is selected at runtime based on the closest representative for the performance")
    int best = -1;
    double bt = 0;
    for (int i = 0; i < n; i++) {
      const tc_plan_s *R = versions[i];
      if (!R || R->expr.empty()) return fail(ST_INVALID_ARG, "version is NULL or not resizable");
      if (R->expr != versions[0]->expr || R->dtype != versions[0]->dtype)
        return fail(ST_INVALID_ARG, "versions differ in expression or dtype");
      Contraction c;
      std::string err;
      Status s = parse(R->expr.c_str(), extents, c, err);
      if (s != ST_OK) return fail(s, err);
      normalize(c, !R->opts.no_fusion && !R->opts.force_tiles);
      if (!split_large(c, err)) continue;
      if (!same_structure(R->c, c)) continue;
      Config cfg = R->cfg;
      for (size_t id = 0; id < c.ix.size(); id++) cfg.T[id] = (int)std::min<int64_t>(cfg.T[id], c.ix[id].n);
      finish_counts(c, cfg);
      if (!config_fits(cfg, variants()[cfg.variant])) continue;
      const double t = model_time(c, cfg, variants()[cfg.variant]);
      if (best < 0 || t < bt) { best = i; bt = t; }
    }
    if (chosen) *chosen = best < 0 ? 0 : best;
    return tc_plan_resize(sized, versions[best < 0 ? 0 : best], extents);
  } catch (...) {
    return fail(ST_ALLOC, "exception in tc_plan_select");
  }
}

}  // extern "C"

namespace {
__global__ void round_bf16_kernel(__nv_bfloat16 *__restrict__ d, const float *__restrict__ s, int64_t n) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    d[i] = __float2bfloat16_rn(s[i]);
}
}  // namespace

extern "C" {

tc_status_t tc_round_bf16(void *dst, const void *src, int64_t n, tc_stream_t stream) {
  if (!dst || !src || n < 0) return fail(ST_INVALID_ARG, "NULL pointer or n < 0");
  if (n == 0) return TC_SUCCESS;
  if (overlaps(dst, 2 * (size_t)n, src, 4 * (size_t)n)) return fail(ST_INVALID_ARG, "dst overlaps src");
  const int blocks = (int)std::min<int64_t>((n + 255) / 256, 148 * 8);
  round_bf16_kernel<<<blocks, 256, 0, (cudaStream_t)stream>>>(static_cast<__nv_bfloat16 *>(dst),
                                                             static_cast<const float *>(src), n);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(ST_CUDA, std::string("launch: ") + cudaGetErrorString(e));
  return TC_SUCCESS;
}

int64_t tc_plan_span(const tc_plan_t plan, int t) {
  if (!plan || t < 0 || t > 2) return -1;
  return plan->parsed.span(t);
}

tc_status_t tc_plan(tc_plan_t *plan, const char *expr, const char *extents, tc_dtype_t dtype) {
  return tc_plan_ex(plan, expr, extents, dtype, nullptr);
}

void tc_plan_destroy(tc_plan_t plan) {
  if (plan && plan->refs.fetch_sub(1) == 1) delete plan;
}

// ---------------------------------------------------------------- plan cache (NEXT-1)
namespace {
std::mutex g_cache_mu;
std::map<std::string, tc_plan_t> &plan_cache() {
  static std::map<std::string, tc_plan_t> m;
  return m;
}
std::string cache_key(const char *expr, const char *extents, tc_dtype_t dtype, const tc_plan_opts *o,
                      int dev) {
  std::ostringstream k;
  k << expr << '\x1f' << extents << '\x1f' << (int)dtype << '\x1f' << dev;
  if (o)
    k << '\x1f' << o->cost_mode << ',' << o->host_only << ',' << o->variant << ',' << o->no_fusion << ','
      << o->tma_epilogue << ',' << o->morder << ',' << o->no_tma_operands << ',' << o->cta_pair << ','
      << o->out_f32 << ',' << o->stream << ',' << o->stream_rank << ',' << (o->force_tiles ? o->force_tiles : "");
  return k.str();
}
}  // namespace

tc_status_t tc_plan_cached(tc_plan_t *plan, const char *expr, const char *extents, tc_dtype_t dtype,
                           const tc_plan_opts *opts) {
  if (!plan || !expr || !extents) return fail(ST_INVALID_ARG, "NULL argument");
  *plan = nullptr;
  try {
    int dev = -1;
    if (!(opts && opts->host_only) && cudaGetDevice(&dev) != cudaSuccess) {
      cudaGetLastError();
      dev = -1;
    }
    const std::string key = cache_key(expr, extents, dtype, opts, dev);
    std::lock_guard<std::mutex> lock(g_cache_mu);
    auto &m = plan_cache();
    auto it = m.find(key);
    if (it != m.end()) {
      it->second->refs.fetch_add(1);
      *plan = it->second;
      return TC_SUCCESS;
    }
    tc_plan_t p = nullptr;
    tc_status_t st = tc_plan_ex(&p, expr, extents, dtype, opts);
    if (st != TC_SUCCESS) return st;
    p->refs.fetch_add(1);   // the cache's reference
    m[key] = p;
    *plan = p;
    return TC_SUCCESS;
  } catch (...) {
    return fail(ST_ALLOC, "exception in tc_plan_cached");
  }
}

size_t tc_plan_cache_size(void) {
  std::lock_guard<std::mutex> lock(g_cache_mu);
  return plan_cache().size();
}

void tc_plan_cache_clear(void) {
  std::lock_guard<std::mutex> lock(g_cache_mu);
  for (auto &kv : plan_cache()) tc_plan_destroy(kv.second);
  plan_cache().clear();
}

double tc_plan_flops(const tc_plan_t plan) { return plan ? plan->parsed.flops() : 0.0; }

int64_t tc_plan_numel(const tc_plan_t plan, int t) {
  if (!plan || t < 0 || t > 2) return -1;
  return plan->parsed.numel(t);
}

tc_status_t tc_plan_tuned(tc_plan_t *tuned, const tc_plan_t plan, const void *A, const void *B, void *C,
                          int topk, int reps, tc_stream_t stream) {
  return tc_plan_tuned_beta(tuned, plan, A, B, C, topk, reps, 0.0, stream);
}

constexpr int kTunedStream = 99;   // tc_plan_tuned's log entry of the streaming path
constexpr size_t kFlushBytes = (size_t)256 << 20;   // tc_plan_tuned: L2 flush between launches

tc_status_t tc_plan_tuned_beta(tc_plan_t *tuned, const tc_plan_t plan, const void *A, const void *B, void *C,
                               int topk, int reps, double beta, tc_stream_t stream) {
  if (!tuned || !plan || !A || !B || !C) return fail(ST_INVALID_ARG, "NULL argument");
  *tuned = nullptr;
  if (plan->host_only || !plan->dev) return fail(ST_CUDA, "plan was made host_only");
  if (topk < 1 || reps < 1) return fail(ST_INVALID_ARG, "topk and reps must be >= 1");
  {
    int cur = -1;
    if (cudaGetDevice(&cur) != cudaSuccess || cur != plan->device)
      return fail(ST_INVALID_ARG, "current device differs from the plan's device");
  }
  try {
    // candidates: the best configuration of each of the top-k variants by predicted time
    std::vector<int> cand;
    for (auto &pv : plan->stats.per_variant)
      if ((int)cand.size() < topk) cand.push_back(pv.first);
    if (cand.empty()) cand.push_back(plan->cfg.variant);
    cudaEvent_t e0, e1;
    if (cudaEventCreate(&e0) != cudaSuccess || cudaEventCreate(&e1) != cudaSuccess)
      return fail(ST_CUDA, "cudaEventCreate");
    // an L2-sized scratch buffer (twice the 126 MB L2) written before every timed launch;
    // without memory for it the tuning runs warm
    void *flush = nullptr;
    if (cudaMalloc(&flush, kFlushBytes) != cudaSuccess) {
      cudaGetLastError();
      flush = nullptr;
    }
    tc_plan_t best = nullptr;
    float best_ms = 0;
    std::vector<std::pair<int, double>> log;
    tc_status_t rc = TC_SUCCESS;
    // the streaming path (stream.hpp) competes when the plan has it and beta == 0: its model's
    // best configurations as candidates 99, 98, 97 (rank 0, 1, 2)
    if (plan->stream.on && (beta == 0.0 || plan->cfg.kind != KIND_BF16_UMMA))
      for (int r = 0; r < plan->stream.nranks; r++) cand.push_back(kTunedStream - r);
    for (int v : cand) {
      tc_plan_s *P = new tc_plan_s();
      P->opts = plan->opts;
      P->force_tiles = plan->force_tiles;
      P->opts.force_tiles = plan->opts.force_tiles ? P->force_tiles.c_str() : nullptr;
      const bool sv = v > kTunedStream - kStreamRanks && v <= kTunedStream;
      P->opts.variant = (sv ? plan->cfg.variant : v) + 1;
      P->opts.stream = sv ? 2 : 1;
      P->opts.stream_rank = sv ? kTunedStream - v : 0;
      P->dtype = plan->dtype;
      P->parsed = plan->parsed;
      tc_plan_t cp = nullptr;
      rc = finish_plan(P, &cp);
      if (rc != TC_SUCCESS) break;
      cp->stats.per_variant = plan->stats.per_variant;
      // one warm-up, then the median of reps single launches, each after an L2 flush (the
      // conditions a stream of different contractions sees; C is overwritten)
      rc = tc_execute(cp, A, B, C, 1.0, beta, stream);
      std::vector<float> ts;
      for (int r = 0; r < reps && rc == TC_SUCCESS; r++) {
        if (flush) cudaMemsetAsync(flush, r & 0xFF, kFlushBytes, (cudaStream_t)stream);
        cudaEventRecord(e0, (cudaStream_t)stream);
        rc = tc_execute(cp, A, B, C, 1.0, beta, stream);
        cudaEventRecord(e1, (cudaStream_t)stream);
        if (cudaEventSynchronize(e1) != cudaSuccess) { rc = fail(ST_CUDA, "tuning launch failed"); break; }
        float t = 0;
        cudaEventElapsedTime(&t, e0, e1);
        ts.push_back(t);
      }
      std::sort(ts.begin(), ts.end());
      const float ms = ts.empty() ? 1e30f : ts[ts.size() / 2];
      if (rc != TC_SUCCESS) { tc_plan_destroy(cp); break; }
      log.push_back({v, ms});
      if (!best || ms < best_ms) {
        tc_plan_destroy(best);
        best = cp;
        best_ms = ms;
      } else {
        tc_plan_destroy(cp);
      }
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    if (flush) {
      cudaStreamSynchronize((cudaStream_t)stream);
      cudaFree(flush);
    }
    if (rc != TC_SUCCESS) { tc_plan_destroy(best); return rc; }
    best->tuned = log;
    *tuned = best;
    return TC_SUCCESS;
  } catch (...) {
    return fail(ST_ALLOC, "exception in tc_plan_tuned_beta");
  }
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
    if (begin < 0 || len < 1 || len > pc.ix[id].n || begin > pc.ix[id].n - len)   // (no int64 overflow)
      return fail(ST_EXTENT, "slab out of range");
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

namespace {
// Everything tc_execute checks before it launches (also run for every member of a group
// before the group's first launch, so a bad member leaves C untouched).
tc_status_t check_execute(const tc_plan_t plan, const void *A, const void *B, const void *C) {
  if (!plan || !A || !B || !C) return fail(ST_INVALID_ARG, "NULL plan or tensor pointer");
  if (plan->host_only || !plan->dev) return fail(ST_CUDA, "plan was made host_only");
  const size_t es = elem_bytes(plan);
  const size_t nA = (size_t)plan->parsed.span(1) * es, nB = (size_t)plan->parsed.span(2) * es,
               nC = (size_t)plan->parsed.span(0) * elem_bytes_c(plan);
  if (overlaps(C, nC, A, nA) || overlaps(C, nC, B, nB)) return fail(ST_INVALID_ARG, "C overlaps A or B");
  int cur = -1;
  if (cudaGetDevice(&cur) != cudaSuccess || cur != plan->device)
    return fail(ST_INVALID_ARG, "current device differs from the plan's device");
  return TC_SUCCESS;
}
}  // namespace

tc_status_t tc_execute(const tc_plan_t plan, const void *A, const void *B, void *C, double alpha,
                       double beta, tc_stream_t stream) {
  const tc_status_t chk = check_execute(plan, A, B, C);
  if (chk != TC_SUCCESS) return chk;
  const size_t es = elem_bytes(plan);
  if (plan->stream.on && plan->stream_active && (beta == 0.0 || plan->cfg.kind != KIND_BF16_UMMA) &&
      plan->batch.empty()) {
    // the streaming path (BF16 with beta != 0 runs the tile configuration below: its epilogue
    // rounds alpha * sum + beta * C once)
    SParams sp = plan->stream.kp;
    const void *Xp = plan->stream.X == 1 ? A : B, *Yp = plan->stream.X == 1 ? B : A;
    if (encode_stream_maps(plan, Xp, C, sp)) {
      sp.Y = static_cast<const char *>(Yp) + es * plan->stream.ybase;
      sp.C = static_cast<char *>(C) + es * plan->stream.cbase;
      sp.alpha = (float)alpha;
      sp.alpha64 = alpha;
      sp.beta = beta;
      const void *fn = stream_kernel_ptr(plan->cfg.kind, plan->stream.NB, plan->stream.AR, plan->stream.mode != SM_K,
                                         beta != 0.0);
      const int grid = std::min(sp.ntiles, plan->stream_grid);
      void *sargs[] = {&sp};
      cudaError_t e = cudaLaunchKernel(fn, dim3(grid), dim3(kSThreads), sargs, plan->stream.smem, (cudaStream_t)stream);
      if (e != cudaSuccess) return fail(ST_CUDA, std::string("launch (stream): ") + cudaGetErrorString(e));
      return TC_SUCCESS;
    }
  }
  KParams kp = plan->kp;
  const Config &cfg = plan->cfg;
  kp.X = cfg.X == 1 ? A : B;
  kp.Y = cfg.X == 1 ? B : A;
  kp.C = C;
  kp.alpha = alpha;
  kp.beta = beta;
  // TMA epilogue when the C view is a legal tensor map and C is only written
  kp.use_tma = plan->tt.tma_ok && plan->opts.tma_epilogue && cfg.kind == KIND_F64_DMMA && beta == 0.0 &&
               plan->batch.empty() &&
               !variants()[cfg.variant].stg &&
               encode_c_map(plan, C, kp.cmap);
  // vector slots need operands aligned to the vector; otherwise the scalar slot tables run
  const bool vx = cfg.vecX > 1 && ((uintptr_t)kp.X % (es * cfg.vecX)) == 0;
  const bool vy = cfg.vecY > 1 && ((uintptr_t)kp.Y % (es * cfg.vecY)) == 0;
  kp.relX = vx ? plan->d_relX2 : plan->d_relX1;
  kp.packX = vx ? plan->d_packX2 : plan->d_packX1;
  kp.nslotX = (int)(vx ? plan->slotX2.pack.size() : plan->slotX1.pack.size());
  kp.vecX = vx ? cfg.vecX : 1;
  kp.relY = vy ? plan->d_relY2 : plan->d_relY1;
  kp.packY = vy ? plan->d_packY2 : plan->d_packY1;
  kp.nslotY = (int)(vy ? plan->slotY2.pack.size() : plan->slotY1.pack.size());
  kp.vecY = vy ? cfg.vecY : 1;
  // C stores in 16-B vectors: 8 elements (staged UMMA epilogue: one 16-B BF16 or two 16-B FP32
  // stores) / 2 FP64 (STG drain)
  kp.vecC = plan->cvec > 1 && ((uintptr_t)C % 16) == 0 ? plan->cvec : 1;
  kp.pf_mstep = beta != 0.0 ? plan->pf_step : 0;
  // tcgen05: operands by TMA when the plan allows and both views encode at these pointers
  const bool tma_ops = plan->umma_tma && encode_operand_map(plan, plan->mapX, kp.X, kp.xmap) &&
                       encode_operand_map(plan, plan->mapY, kp.Y, kp.ymap);
  KernelEntry ke = kernel_for(cfg, tma_ops);
  if (plan->out_f32) {   // BF16 operands, FP32 C
    ke.fn = kernel_ptr_umma_f32out(cfg.variant, cfg.xKmajor, cfg.yKmajor, &ke.smem, &ke.threads);
    ke.smem_tma = ke.smem;
    if (!ke.fn) return fail(ST_UNSUPPORTED, "no FP32-output instance for the variant");
  }
  const int grid = (int)std::min<int64_t>(cfg.nctas, plan->sms);
  if (tma_ops && plan->pair) {   // clusters of two CTAs over 2 x 2 tile blocks (persistent)
    size_t sm = 0;
    int th = 0;
    const void *fn = kernel_ptr_umma_pair(cfg.variant, cfg.xKmajor, cfg.yKmajor, &sm, &th);
    const int64_t units = ((cfg.mtiles + 1) / 2) * ((cfg.ntiles + 1) / 2);
    const int ncl = (int)std::min<int64_t>(units, plan->sms / 2);
    cudaLaunchConfig_t lc = {};
    lc.gridDim = dim3(2 * ncl);
    lc.blockDim = dim3(th);
    lc.dynamicSmemBytes = sm;
    lc.stream = (cudaStream_t)stream;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    lc.attrs = at;
    lc.numAttrs = 1;
    void *pargs[] = {&kp};
    cudaError_t e = cudaLaunchKernelExC(&lc, fn, pargs);
    if (e != cudaSuccess) return fail(ST_CUDA, std::string("launch (CTA pair): ") + cudaGetErrorString(e));
    return TC_SUCCESS;
  }
  void *args[] = {&kp};
  const int64_t nb = plan->c.nbatch();
  const char *X0 = static_cast<const char *>(kp.X), *Y0 = static_cast<const char *>(kp.Y);
  char *C0 = static_cast<char *>(kp.C);
  for (int64_t b = 0; b < nb; b++) {
    if (!plan->batch.empty()) {   // batch slab b (mixed radix, first batch index fastest)
      int64_t r = b, ox = 0, oy = 0, oc = 0;
      for (const auto &d : plan->batch) {
        const int64_t i = r % d.n;
        r /= d.n;
        ox += i * d.sX;
        oy += i * d.sY;
        oc += i * d.sC;
      }
      kp.X = X0 + es * ox;
      kp.Y = Y0 + es * oy;
      kp.C = C0 + elem_bytes_c(plan) * oc;
    }
    cudaError_t e = cudaLaunchKernel(ke.fn, dim3(grid), dim3(ke.threads), args,
                                     kp.use_tma ? ke.smem_tma : ke.smem, (cudaStream_t)stream);
    if (e != cudaSuccess) return fail(ST_CUDA, std::string("launch: ") + cudaGetErrorString(e));
  }
  return TC_SUCCESS;
}

tc_status_t tc_execute_group(const tc_plan_t *plans, const void *const *A, const void *const *B,
                             int n, void *C, double alpha, double beta, tc_stream_t stream) {
  if (!plans || !A || !B || !C || n < 1) return fail(ST_INVALID_ARG, "NULL array or n < 1");
  for (int i = 0; i < n; i++)
    if (!plans[i] || !A[i] || !B[i]) return fail(ST_INVALID_ARG, "NULL plan or tensor pointer in group");
  // every member must see the same C: extents and strides per position, origin, dtype, device
  const Contraction &c0 = plans[0]->parsed;
  for (int i = 1; i < n; i++) {
    const Contraction &ci = plans[i]->parsed;
    bool same = plans[i]->dtype == plans[0]->dtype && plans[i]->device == plans[0]->device &&
                ci.t[0].idx.size() == c0.t[0].idx.size() && ci.t[0].base == c0.t[0].base &&
                ci.parent_numel[0] == c0.parent_numel[0];
    for (size_t k = 0; same && k < c0.t[0].idx.size(); k++)
      same = ci.ix[ci.t[0].idx[k]].n == c0.ix[c0.t[0].idx[k]].n && ci.t[0].stride[k] == c0.t[0].stride[k];
    if (!same) return fail(ST_INVALID_ARG, "group member " + std::to_string(i) + " gives C another layout");
  }
  for (int i = 0; i < n; i++) {
    const tc_status_t chk = check_execute(plans[i], A[i], B[i], C);
    if (chk != TC_SUCCESS) {
      g_err = "group member " + std::to_string(i) + ": " + g_err;
      return chk;
    }
  }
  for (int i = 0; i < n; i++) {
    tc_status_t st = tc_execute(plans[i], A[i], B[i], C, alpha, i == 0 ? beta : 1.0, stream);
    if (st != TC_SUCCESS) return st;
  }
  return TC_SUCCESS;
}

size_t tc_plan_workspace_bytes(const tc_plan_t plan) {
  if (!plan) return 0;
  auto al = [](size_t x) { return (x + 255) & ~(size_t)255; };
  const Contraction &c = plan->parsed;
  const size_t es = elem_bytes(plan);
  return al(es * c.parent_numel[1]) + al(es * c.parent_numel[2]) + al(elem_bytes_c(plan) * c.parent_numel[0]);
}

tc_status_t tc_execute_host(const tc_plan_t plan, const void *A_host, const void *B_host, void *C_host,
                            double alpha, double beta, void *workspace, size_t workspace_bytes,
                            tc_stream_t stream) {
  if (!plan || !A_host || !B_host || !C_host || !workspace) return fail(ST_INVALID_ARG, "NULL argument");
  if (workspace_bytes < tc_plan_workspace_bytes(plan)) return fail(ST_INVALID_ARG, "workspace too small");
  auto al = [](size_t x) { return (x + 255) & ~(size_t)255; };
  const Contraction &c = plan->parsed;
  const size_t es = elem_bytes(plan);
  const size_t bA = es * c.parent_numel[1], bB = es * c.parent_numel[2], bC = elem_bytes_c(plan) * c.parent_numel[0];
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
    static const char *dn[4] = {"f64", "bf16", "tf32", "f32"};
    o << "{\"dtype\":\"" << dn[g.kind] << "\",\"X\":\"" << (g.X == 1 ? "A" : "B") << "\"";
    o << ",\"indices\":[";
    for (size_t i = 0; i < c.ix.size(); i++) {
      const char *cls = c.ix[i].cls == EXT_A ? "extA" : c.ix[i].cls == EXT_B ? "extB"
                      : c.ix[i].cls == BATCH ? "batch" : "int";
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
    o << ",\"morder\":" << g.morder << ",\"korder\":" << g.korder;
    o << ",\"variant\":" << g.variant << ",\"BM\":" << v.BM << ",\"BN\":" << v.BN << ",\"BK\":" << v.BK
      << ",\"WM\":" << v.WM << ",\"WN\":" << v.WN << ",\"stg\":" << v.stg
      << ",\"threads\":" << v.threads() << ",\"stages\":" << v.stages << ",\"occ\":" << v.occ;
    o << ",\"Mt\":" << g.Mt << ",\"Nt\":" << g.Nt << ",\"Kt\":" << g.Kt << ",\"nctas\":" << g.nctas
      << ",\"mtiles\":" << g.mtiles << ",\"ntiles\":" << g.ntiles << ",\"nsteps\":" << g.nsteps
      << ",\"grid\":" << std::min<int64_t>(g.nctas, plan->sms)
      << ",\"nbatch\":" << c.nbatch();
    o << ",\"vecX\":" << g.vecX << ",\"vecY\":" << g.vecY << ",\"vecC\":" << plan->cvec << ",\"cs0\":" << plan->kp.cs0 << ",\"xKmajor\":" << g.xKmajor
      << ",\"yKmajor\":" << g.yKmajor << ",\"tma_operands\":" << (plan->umma_tma ? 1 : 0)
      << ",\"cta_pair\":" << (plan->pair ? 1 : 0) << ",\"resized\":" << (plan->resized ? 1 : 0)
      << ",\"out_f32\":" << (plan->out_f32 ? 1 : 0)
      << ",\"wfX\":" << g.wfX << ",\"wfY\":" << g.wfY;
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
      << ",\"ranked\":" << plan->stats.ranked << ",\"plan_ms\":" << plan->stats.plan_ms
      << ",\"per_variant\":[";
    for (size_t q = 0; q < plan->stats.per_variant.size(); q++)
      o << (q ? "," : "") << "[" << plan->stats.per_variant[q].first << "," << plan->stats.per_variant[q].second * 1e3 << "]";
    o << "],\"tuned\":[";
    for (size_t q = 0; q < plan->tuned.size(); q++)
      o << (q ? "," : "") << "[" << plan->tuned[q].first << "," << plan->tuned[q].second << "]";
    o << "]}";
    {   // the streaming path (stream.hpp)
      const StreamCfg &st = plan->stream;
      const SParams &k = st.kp;
      o << ",\"stream\":{\"on\":" << (st.on ? 1 : 0) << ",\"active\":" << (plan->stream_active ? 1 : 0)
        << ",\"why\":\"" << st.why << "\"";
      if (st.on) {
        o << ",\"mode\":\"" << (st.mode == SM_K ? "K" : st.mode == SM_M ? "M" : "T") << "\",\"X\":\"" << (st.X == 1 ? "A" : "B") << "\",\"tiles\":{";
        for (size_t i = 0; i < c.ix.size(); i++) o << (i ? "," : "") << "\"" << c.ix[i].name << "\":" << st.T[i];
        o << "},\"KB\":" << k.KB << ",\"nks\":" << k.nks << ",\"stages\":" << k.stages
          << ",\"stage_bytes\":" << k.stage_bytes << ",\"ntiles\":" << k.ntiles << ",\"units\":" << k.nunits
          << ",\"NB\":" << st.NB << ",\"AR\":" << st.AR << ",\"occ\":" << st.occ << ",\"nstg\":" << k.nstg << ",\"xswz\":" << st.xswz << ",\"smem\":" << st.smem
          << ",\"grid\":" << plan->stream_grid
          << ",\"t_pred_ms\":" << st.t_pred * 1e3 << ",\"bytes\":" << st.bytes
          << ",\"rank\":" << st.rank << ",\"nranks\":" << st.nranks;
      }
      o << "}";
    }
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
