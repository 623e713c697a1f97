// kparams.hpp — launch metadata passed by value to the libtc kernels.
//
// The contraction is executed as C(m, n) = sum_k X(m, k) * Y(k, n) over a grid of CTA
// tiles, where m runs over the externals of X (the input holding C's FVI),
// n over the externals of Y, k over the internal indices.  Each is a multi-index whose
// digits carry their own tile size T_i (a CTA owns a hyper-rectangle prod T_i of
// C; the grid has prod ceil(N_i / T_i) tiles).  Addresses are separable:
//   addr_X(tile, step, m, k) = tileX[mt] + stepX[s] + rel_slot(m, k)
//   addr_C(tile, m, n)       = tileM[mt].c + tileN[nt].c + relCm[m] + relCn[n]
// so one compiled kernel serves every index permutation; only tile shapes are templates.
// Bounds ("correct for any problem size"): each tile carries its per-digit limits
// packed one byte per digit (lim-1, 7 bits) and every tile-local row / column its packed
// digits; "in range" is one SWAR compare.
#pragma once
#include <cstdint>

namespace tc {

constexpr int kMaxDigits = 8;

struct TileInfo {           // one m-tile (or n-tile)
  int64_t op;               // element offset of the tile origin in X (or Y), incl. base
  int64_t c;                // element offset of the tile origin in C (m: incl. C's base)
  uint64_t lim;             // byte d = min(T_d, N_d - origin_d) - 1
};

struct KParams {
  const void *X;            // M-side operand (A or B)
  const void *Y;            // N-side operand
  void *C;
  double alpha, beta;
  int mtiles, ntiles, ntotal;   // tiles per side, total tiles
  int group_m;              // CTA rasterisation: m-tiles per group (L2 locality)
  int Mt, Nt;               // tile extents (<= BM, BN)
  const TileInfo *tileM;    // [mtiles]
  const TileInfo *tileN;    // [ntiles]
  uint64_t fullM, fullN;    // lim of a full (interior) tile
  // tile-local row / column tables [BM] / [BN]
  const int64_t *relCm;     // offset in C of tile-local m
  const uint64_t *digM;     // packed digits of tile-local m
  const int64_t *relCn;
  const uint64_t *digN;
  // k side: steps in mixed radix over the internal tile grid
  int nsteps;
  const int64_t *stepX;     // [nsteps] element offset of step s's origin in X
  const int64_t *stepY;     // [nsteps]
  const uint64_t *kmask;    // [nsteps] bit k set <=> tile-local k is in range at step s
  // load slots: the X tile (Mt x Kt) and the Y tile (Kt x Nt) enumerated in each
  // operand's OWN memory order (threads along x walk the input's FVI)
  const int64_t *relX;      // [nslotX] element offset of the slot inside (tile, step)
  const uint32_t *packX;    // [nslotX] smem offset | k << 13 | m << 19
  const int64_t *relY;
  const uint32_t *packY;
  int nslotX, nslotY;
  int vecX, vecY;           // 1 or 2 elements per slot (16-B cp.async when 2)
  int xKmajor, yKmajor;     // smem layout: 1 = k contiguous, 0 = m (n) contiguous
};

#ifdef __CUDACC__
#define TC_HD __host__ __device__
#else
#define TC_HD
#endif

// byte-wise a_d <= b_d for 8 packed 7-bit values
TC_HD inline bool swar_le(uint64_t a, uint64_t b) {
  const uint64_t H = 0x8080808080808080ull;
  return (((b | H) - a) & H) == H;
}

}  // namespace tc
