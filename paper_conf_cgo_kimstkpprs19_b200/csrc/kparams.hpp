// kparams.hpp — launch metadata passed by value to the libtc kernels.
//
// The contraction is executed as C(m, n) = sum_k X(m, k) * Y(k, n) over a grid of CTA
// tiles, where m runs over the externals of X (the input holding C's FVI),
// n over the externals of Y, k over the internal indices.  Each is a multi-index whose
// digits carry their own tile size T_i (a CTA owns a hyper-rectangle prod T_i of
// C; the grid has prod ceil(N_i / T_i) CTAs).  Addresses are separable:
//   addr_X(m, k) = baseX + rowX(m) + stepX(s) + relKX(k)
// so one compiled kernel serves every index permutation; only tile shapes are templates.
#pragma once
#include <cstdint>

namespace tc {

constexpr int kMaxDigits = 8;

struct SideDesc {           // the m side (X externals) or the n side (Y externals)
  int nd;                   // number of digits, compute order (C order; C's FVI first on m)
  int T[kMaxDigits];        // tile size per digit; prod T <= BM (or BN)
  int64_t N[kMaxDigits];    // extent per digit
  int64_t ntile[kMaxDigits];// ceil(N / T)
  int64_t sOp[kMaxDigits];  // element stride in the operand (X for m, Y for n)
  int64_t sC[kMaxDigits];   // element stride in C
  int64_t tiles;            // prod ntile
};

struct KParams {
  const void *X;            // M-side operand (A or B)
  const void *Y;            // N-side operand
  void *C;
  double alpha, beta;
  int64_t baseX, baseY, baseC;   // element offsets of the origins (restricted plans)
  SideDesc m, n;
  int64_t nctas;            // m.tiles * n.tiles
  int group_m;              // CTA rasterisation: m-tiles per group (L2 locality)
  // k side: host tables indexed by step s (mixed radix over the internal tile grid)
  int nsteps;
  const int64_t *stepX;     // [nsteps] element offset of step s's origin in X
  const int64_t *stepY;     // [nsteps]
  const uint64_t *kmask;    // [nsteps] bit k set <=> tile-local k is in range at step s
  int64_t relKX[64];        // tile-local k -> element offset in X (BK <= 64)
  int64_t relKY[64];
  // load slots: the X tile (Mt x Kt) and the Y tile (Kt x Nt) enumerated in each
  // operand's OWN memory order (threads along x walk the input's FVI);
  // entry = (m << 8) | k  (resp. (n << 8) | k), first element of a V-vector.
  const uint32_t *slotX;
  const uint32_t *slotY;
  int nslotX, nslotY;
  int vecX, vecY;           // 1 or 2 elements per slot (16-B cp.async when 2)
  int xKmajor, yKmajor;     // smem layout: 1 = k contiguous, 0 = m (n) contiguous
};

}  // namespace tc
