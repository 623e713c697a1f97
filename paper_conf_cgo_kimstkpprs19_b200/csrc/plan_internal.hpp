// plan_internal.hpp — the plan object behind tc_plan_t (shared by api.cu and group_api.cu;
// not part of the C ABI).
#pragma once
#include <atomic>
#include <string>
#include <utility>
#include <vector>

#include <cuda_runtime.h>

#include "../../include/libtc.h"
#include "contraction.hpp"
#include "kparams.hpp"
#include "planner.hpp"
#include "stream.hpp"
#include "tiles.hpp"

using namespace tc;   // (internal header: the plan object is written in the library's namespace)

struct tc_plan_s {
  std::atomic<int> refs{1};   // tc_plan_destroy releases one; the plan cache holds one
  Contraction parsed;      // as parsed (before normalisation) — restriction starts here
  Contraction c;           // normalised (dropped extent-1 indices, fused runs)
  int dtype = 0;
  int device = -1;
  int sms = 148;
  bool host_only = false;
  Config cfg;
  PlanStats stats;
  tc_plan_opts opts{};
  std::string force_tiles;
  TileTables tt;
  SlotTable slotX1, slotY1, slotX2, slotY2;   // scalar and cfg.vecX / cfg.vecY wide slots
  int cvec = 1;            // c_vec_width of the plan (16-B C stores when > 1)
  int pf_step = 0;         // FP64: old-C L2 prefetch step in tile rows when beta != 0 (0: none)
  // tcgen05: operand tensor maps for the TMA producer (tiles.cpp umma_tma_spec); the pointers
  // come per call, so tc_execute encodes the maps from these shapes
  bool umma_tma = false;
  std::string expr;        // the expression as given (tc_plan / tc_plan_ex): resizable plans
  bool resized = false;    // the configuration came from a representative-size plan (NEXT-1)
  bool pair = false;
  bool out_f32 = false;    // BF16 operands, FP32 C (kernels_umma_f32out.cu)       // tcgen05: launch the CTA-pair instance (clusters of 2) with TMA operands
  OperandMap mapX, mapY;
  // the streaming path (stream.hpp): on when eligible unless opts / a forced variant say
  // otherwise; tc_execute takes it for beta == 0 when both tensor maps encode
  StreamCfg stream;
  bool stream_active = false;   // tc_execute takes the path (preferred, or opts.stream == 2)
  int stream_grid = 0;     // persistent CTAs (SMs x resident CTAs)
  // batch (Hadamard) indices (R31): extent and element strides in X, Y, C.  tc_execute
  // launches the kernel once per batch slab with the operands offset to it — the kernels
  // carry no batch code (the FP64 variants run at their 128-register cap).
  struct BatchDim { int64_t n, sX, sY, sC; };
  std::vector<BatchDim> batch;
  std::vector<std::pair<int, double>> tuned;   // tc_plan_tuned: (variant, measured ms) per candidate
  KParams kp{};            // device pointers filled in; X/Y/C/alpha/beta/slots set per call
  void *dev = nullptr;     // one device buffer with every table
  size_t dev_bytes = 0;
  const int32_t *d_relX1 = nullptr, *d_relY1 = nullptr, *d_relX2 = nullptr, *d_relY2 = nullptr;
  const uint32_t *d_packX1 = nullptr, *d_packY1 = nullptr, *d_packX2 = nullptr, *d_packY2 = nullptr;
  ~tc_plan_s() {
    if (dev) {
      int cur = -1;
      cudaGetDevice(&cur);
      if (cur != device) cudaSetDevice(device);
      cudaFree(dev);
      if (cur != device && cur >= 0) cudaSetDevice(cur);
    }
  }
};

namespace tc {
// thread-local detail string of the C ABI (tc_last_error) and the status it goes with
tc_status_t set_error(Status s, const std::string &msg);
std::string &last_error_string();
}  // namespace tc
