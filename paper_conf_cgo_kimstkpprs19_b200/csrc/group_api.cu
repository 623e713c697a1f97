// group_api.cu — C ABI of the fused grouped contraction (include/libtc.h: tc_group_plan,
// tc_group_execute, tc_group_info, tc_group_destroy, R34).
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <sstream>
#include <string>
#include <vector>

#include "group.hpp"
#include "kernel_group.cuh"
#include "plan_internal.hpp"

namespace tc {
const void *group_kernel_ptr(int v, bool tma, int tma_stage, size_t *smem, int *threads);   // kernels_group.cu
}

struct tc_group_s {
  GroupTables gt;
  int n = 0;
  int device = -1;
  bool host_only = false;
  struct Launch {             // one kernel instance: [0] cp.async gathers, [1] TMA boxes
    const void *fn = nullptr;
    size_t smem = 0;
    int threads = 0, grid = 0;
  } launch[2];
  GParams kp{};               // device table pointers; per-call fields set in execute
  const int32_t *ctab[2] = {nullptr, nullptr};
  std::vector<int64_t> spanA, spanB;   // bytes of each member's A / B view (overlap checks)
  int64_t spanC = 0;
  void *dev = nullptr;
  ~tc_group_s() {
    if (dev) {
      int cur = -1;
      cudaGetDevice(&cur);
      if (cur != device) cudaSetDevice(device);
      cudaFree(dev);
      if (cur != device && cur >= 0) cudaSetDevice(cur);
    }
  }
};

namespace {

bool overlaps(const void *a, size_t na, const void *b, size_t nb) {
  const char *x = (const char *)a, *y = (const char *)b;
  return x < y + nb && y < x + na;
}

PFN_cuTensorMapEncodeTiled_v12000 encoder() {
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

// TMA descriptor of one member operand at this call's pointer: the operand's own dims
// (memory order), byte strides, the tile box (dim 0 split into boxes of ch), swizzle 64/128 B,
// out-of-range elements zero-filled
bool encode_operand(const GroupTables::TmaSpec &s, const double *base, TmaDesc &out) {
  auto enc = encoder();
  if (!enc) return false;
  const double *origin = base + s.base;
  if ((uintptr_t)origin % 16) return false;
  cuuint64_t dims[kGMaxTmaDims], strides[kGMaxTmaDims];
  cuuint32_t box[kGMaxTmaDims], es[kGMaxTmaDims];
  for (int j = 0; j < s.rank; j++) {
    dims[j] = s.dims[j];
    box[j] = s.box[j];
    es[j] = 1;
    if (j + 1 < s.rank) strides[j] = s.strides[j];
  }
  static_assert(sizeof(TmaDesc) == sizeof(CUtensorMap), "descriptor size");
  // (dims 1.. in a permuted order: the strides need not grow; no swizzle — the dim order and
  //  the padded k pitch make the fragment loads conflict-free, group.cpp)
  const CUresult e = enc(reinterpret_cast<CUtensorMap *>(&out), CU_TENSOR_MAP_DATA_TYPE_FLOAT64, (cuuint32_t)s.rank,
                         (void *)origin, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return e == CUDA_SUCCESS;
}

// One device buffer with every table of the group (as api.cu's upload for plans).
Status upload_group(tc_group_s *G, std::string &err) {
  const GroupTables &g = G->gt;
  struct Part { const void *src; size_t bytes; size_t off; };
  std::vector<Part> parts;
  size_t o = 0;
  auto add = [&](const void *src, size_t bytes) {
    parts.push_back({src, bytes, o});
    o = (o + bytes + 255) & ~(size_t)255;
    return parts.size() - 1;
  };
  const size_t iMem = add(g.mem.data(), sizeof(GMemberDev) * g.mem.size());
  const size_t iSt = add(g.steps.data(), sizeof(GStepDev) * g.steps.size());
  const size_t iRr = add(g.runRel.data(), 4 * g.runRel.size());
  const size_t iRs = add(g.runSoff.data(), 4 * g.runSoff.size());
  const size_t iRd = add(g.runDig.data(), 8 * g.runDig.size());
  const size_t iPd = add(g.pad.data(), 4 * g.pad.size());
  const size_t iT0 = add(g.ctab[0].data(), 4 * g.ctab[0].size());
  const size_t iT1 = add(g.ctab[1].data(), 4 * g.ctab[1].size());
  const size_t iUr = add(g.unitRel.data(), 8 * g.unitRel.size());
  const size_t iUd = add(g.unitDig.data(), 8 * g.unitDig.size());
  std::vector<char> h(o + 256, 0);
  for (auto &p : parts) if (p.bytes) std::memcpy(h.data() + p.off, p.src, p.bytes);
  cudaError_t e = cudaMalloc(&G->dev, h.size());
  if (e != cudaSuccess) { err = std::string("cudaMalloc: ") + cudaGetErrorString(e); return ST_ALLOC; }
  e = cudaMemcpy(G->dev, h.data(), h.size(), cudaMemcpyHostToDevice);
  if (e != cudaSuccess) { err = std::string("cudaMemcpy: ") + cudaGetErrorString(e); return ST_CUDA; }
  char *b = (char *)G->dev;
  GParams &kp = G->kp;
  kp.mem = (const GMemberDev *)(b + parts[iMem].off);
  kp.steps = (const GStepDev *)(b + parts[iSt].off);
  kp.runRel = (const int32_t *)(b + parts[iRr].off);
  kp.runSoff = (const uint32_t *)(b + parts[iRs].off);
  kp.runDig = (const uint64_t *)(b + parts[iRd].off);
  kp.pad = (const uint32_t *)(b + parts[iPd].off);
  G->ctab[0] = (const int32_t *)(b + parts[iT0].off);
  G->ctab[1] = (const int32_t *)(b + parts[iT1].off);
  kp.unitRel = (const int64_t *)(b + parts[iUr].off);
  kp.unitDig = (const uint64_t *)(b + parts[iUd].off);
  kp.nmem = G->n;
  kp.rank = g.rank;
  kp.ntiles = (int)g.ntiles;
  kp.nunits = (int)g.unitRel.size();
  kp.stage_bytes = g.tma_stage_bytes;
  kp.cbase = g.cbase;
  kp.Tpack = 0;
  for (int p = 0; p < kGMaxCdims; p++) {
    kp.ntl[p] = p < g.rank ? g.ntl[p] : 1;
    kp.T[p] = p < g.rank ? g.T[p] : 1;
    kp.N[p] = p < g.rank ? g.N[p] : 1;
    kp.cstep[p] = p < g.rank ? (int64_t)g.T[p] * g.cstride[p] : 0;
    if (p < g.rank) kp.Tpack |= (uint64_t)g.T[p] << (8 * p);
  }
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, G->device);
  for (int mode = 0; mode < 2; mode++) {
    if (mode == 1 && !g.tma) continue;
    tc_group_s::Launch &L = G->launch[mode];
    size_t base = 0;
    L.fn = group_kernel_ptr(g.variant, mode == 1, g.tma_stage_bytes, &base, &L.threads);
    if (!L.fn) { err = "no group kernel for this variant"; return ST_NO_CONFIG; }
    // cp.async: + the member records (copied to smem by every CTA); the attribute is the
    // kernel's, shared by every group: set the largest any group needs
    const size_t per_member = mode == 0 ? sizeof(GMemberDev) : 0;
    L.smem = base + per_member * (size_t)G->n;
    e = cudaFuncSetAttribute(L.fn, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)(base + per_member * kGMaxMembers));
    if (e != cudaSuccess) { err = std::string("cudaFuncSetAttribute: ") + cudaGetErrorString(e); return ST_CUDA; }
    int occ = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, L.fn, L.threads, L.smem);
    if (e != cudaSuccess || occ < 1) { err = "group kernel cannot be resident"; return ST_CUDA; }
    L.grid = (int)std::min<int64_t>(g.ntiles, (int64_t)sms * std::min(occ, 2));
  }
  return ST_OK;
}

}  // namespace

extern "C" {

tc_status_t tc_group_plan(tc_group_t *group, const tc_plan_t *plans, int n) {
  if (!group) return set_error(ST_INVALID_ARG, "group is NULL");
  *group = nullptr;
  if (!plans || n < 1) return set_error(ST_INVALID_ARG, "NULL plans or n < 1");
  if (n > kGMaxMembers) return set_error(ST_UNSUPPORTED, "more than 32 members");
  for (int i = 0; i < n; i++)
    if (!plans[i]) return set_error(ST_INVALID_ARG, "NULL plan in group");
  try {
    // the members must give C one layout (as tc_execute_group), be FP64 and on one device
    const Contraction &c0 = plans[0]->parsed;
    for (int i = 0; i < n; i++) {
      const Contraction &ci = plans[i]->parsed;
      if (plans[i]->dtype != TC_F64) return set_error(ST_UNSUPPORTED, "fused groups are FP64 (the paper's precision)");
      if (plans[i]->host_only != plans[0]->host_only || plans[i]->device != plans[0]->device)
        return set_error(ST_INVALID_ARG, "group member " + std::to_string(i) + " is on another device");
      bool same = ci.t[0].idx.size() == c0.t[0].idx.size() && ci.t[0].base == c0.t[0].base &&
                  ci.parent_numel[0] == c0.parent_numel[0];
      for (size_t k = 0; same && k < c0.t[0].idx.size(); k++)
        same = ci.ix[ci.t[0].idx[k]].n == c0.ix[c0.t[0].idx[k]].n && ci.t[0].stride[k] == c0.t[0].stride[k];
      if (!same) return set_error(ST_INVALID_ARG, "group member " + std::to_string(i) + " gives C another layout");
    }
    // host_only members (planning without a GPU): the group is planned, not uploaded, and
    // tc_group_execute refuses it
    const bool host_only = plans[0]->host_only;
    int cur = -1;
    if (!host_only && (cudaGetDevice(&cur) != cudaSuccess || cur != plans[0]->device))
      return set_error(ST_INVALID_ARG, "current device differs from the plans' device");
    tc_group_s *G = new tc_group_s();
    G->n = n;
    G->device = cur;
    G->host_only = host_only;
    std::vector<const Contraction *> mem;
    for (int i = 0; i < n; i++) {
      mem.push_back(&plans[i]->parsed);
      G->spanA.push_back(8 * plans[i]->parsed.span(1));
      G->spanB.push_back(8 * plans[i]->parsed.span(2));
    }
    G->spanC = 8 * c0.span(0);
    std::string err;
    Status s = plan_group(mem, G->gt, err);
    if (s == ST_OK && !host_only) s = upload_group(G, err);
    if (s != ST_OK) {
      delete G;
      return set_error(s, err);
    }
    *group = G;
    return TC_SUCCESS;
  } catch (...) {
    return set_error(ST_ALLOC, "exception in tc_group_plan");
  }
}

tc_status_t tc_group_execute(const tc_group_t group, const void *const *A, const void *const *B, void *C,
                             double alpha, double beta, tc_stream_t stream) {
  if (!group || !A || !B || !C) return set_error(ST_INVALID_ARG, "NULL group or tensor array");
  const tc_group_s *G = group;
  if (G->host_only || !G->dev) return set_error(ST_CUDA, "group was planned from host_only plans");
  int cur = -1;
  if (cudaGetDevice(&cur) != cudaSuccess || cur != G->device)
    return set_error(ST_INVALID_ARG, "current device differs from the group's device");
  GParams kp = G->kp;
  kp.vecmask = 0;
  bool tma = G->gt.tma;
  for (int o = 0; o < G->n; o++) {
    if (!A[o] || !B[o]) return set_error(ST_INVALID_ARG, "NULL tensor pointer in group");
    if (overlaps(C, G->spanC, A[o], G->spanA[o]) || overlaps(C, G->spanC, B[o], G->spanB[o]))
      return set_error(ST_INVALID_ARG, "C overlaps A or B of member " + std::to_string(o));
  }
  for (int i = 0; i < G->n; i++) {   // i: execution position; o: the caller's member
    const int o = G->gt.order[i];
    const bool xa = G->gt.mem[i].xIsA;
    kp.X[i] = static_cast<const double *>(xa ? A[o] : B[o]);
    kp.Y[i] = static_cast<const double *>(xa ? B[o] : A[o]);
    if ((uintptr_t)kp.X[i] % 16 == 0) kp.vecmask |= 1ull << (2 * i);
    if ((uintptr_t)kp.Y[i] % 16 == 0) kp.vecmask |= 1ull << (2 * i + 1);
    // TMA boxes when every operand's origin is 16-B aligned and its map encodes
    if (tma) tma = encode_operand(G->gt.tmaX[i], kp.X[i], kp.xmap[i]) && encode_operand(G->gt.tmaY[i], kp.Y[i], kp.ymap[i]);
  }
  const int mode = tma ? 1 : 0;
  const tc_group_s::Launch &L = G->launch[mode];
  kp.ctab = G->ctab[mode];
  kp.C = static_cast<double *>(C);
  kp.alpha = alpha;
  kp.beta = beta;
  // C copy-out units: the plan's (1 or 2 elements); 16-B stores only on a 16-B aligned C
  kp.uvec = G->gt.uvec;
  kp.cvec16 = G->gt.uvec == 2 && ((uintptr_t)(static_cast<double *>(C) + G->gt.cbase) % 16 == 0);
#ifdef TC_GROUP_TRACE
  // (trace side builds: the timeline buffer's device address comes from the environment)
  if (const char *tp = getenv("TC_GROUP_TRACE_PTR")) kp.trace = (unsigned long long *)strtoull(tp, nullptr, 0);
#endif
  void *args[] = {&kp};
  cudaError_t e = cudaLaunchKernel(L.fn, dim3(L.grid), dim3(L.threads), args, L.smem, (cudaStream_t)stream);
  if (e != cudaSuccess) return set_error(ST_CUDA, std::string("launch: ") + cudaGetErrorString(e));
  return TC_SUCCESS;
}

tc_status_t tc_group_info(const tc_group_t group, char *json, size_t cap, size_t *needed) {
  if (!group) return set_error(ST_INVALID_ARG, "group is NULL");
  try {
    const GroupTables &g = group->gt;
    std::ostringstream o;
    o << "{\"members\":" << group->n << ",\"rank\":" << g.rank << ",\"T\":[";
    for (int p = 0; p < g.rank; p++) o << (p ? "," : "") << g.T[p];
    o << "],\"ntiles\":" << g.ntiles << ",\"box\":" << g.box << ",\"BK\":" << g.BK << ",\"variant\":" << g.variant
      << ",\"tma\":" << (g.tma ? "true" : "false") << ",\"uvec\":" << g.uvec;
    for (int mode = 0; mode < 2; mode++)
      o << ",\"" << (mode ? "tma" : "cpasync") << "_launch\":{\"grid\":" << group->launch[mode].grid
        << ",\"threads\":" << group->launch[mode].threads << ",\"smem\":" << group->launch[mode].smem << "}";
    o << ",\"flops\":" << g.flops << ",\"padded_flops\":" << g.padded_flops << ",\"plan_ms\":" << g.plan_ms
      << ",\"order\":[";
    for (int i = 0; i < group->n; i++) o << (i ? "," : "") << g.order[i];
    o << "],\"per_member\":[";   // (in execution order)
    for (int i = 0; i < group->n; i++) {
      const GMemberDev &m = g.mem[i];
      o << (i ? "," : "") << "{\"Mt\":" << g.Mt[i] << ",\"Nt\":" << g.Nt[i] << ",\"Kt\":" << g.Kt[i]
        << ",\"nsteps\":" << m.nsteps << ",\"X\":\"" << (m.xIsA ? "A" : "B")
        << "\",\"vecX\":" << m.x.vec << ",\"vecY\":" << m.y.vec << ",\"runlenX\":" << m.x.runlen
        << ",\"runlenY\":" << m.y.runlen << ",\"tma_bytes\":[" << m.x.tma_tx << "," << m.y.tma_tx
        << "],\"flush_wf\":" << g.flushWf[i] << ",\"load_wf\":" << g.loadWf[i]
        << ",\"tma_frag_wf\":" << g.fragWf[i] << ",\"chain\":[" << (int)m.chain[0] << "," << (int)m.chain[1] << "]}";
    }
    o << "]}";
    const std::string s = o.str();
    if (needed) *needed = s.size() + 1;
    if (json && cap) {
      const size_t k = std::min(cap - 1, s.size());
      std::memcpy(json, s.data(), k);
      json[k] = 0;
    }
    return TC_SUCCESS;
  } catch (...) {
    return set_error(ST_ALLOC, "exception in tc_group_info");
  }
}

void tc_group_destroy(tc_group_t group) { delete group; }

}  // extern "C"
