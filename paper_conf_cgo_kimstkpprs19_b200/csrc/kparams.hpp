// kparams.hpp — launch metadata passed by value to the libtc kernels.
//
// The contraction is executed as C(m, n) = sum_k X(m, k) * Y(k, n) over a grid of CTA
// tiles, where m runs over the externals of X (the input holding C's FVI),
// n over the externals of Y, k over the internal indices.  Each is a multi-index whose
// digits carry their own tile size T_i (a CTA owns a hyper-rectangle prod T_i of
// C; the grid has prod ceil(N_i / T_i) tiles).  Addresses are separable:
//   addr_X(tile, step, slot) = tileM[mt].op + stepX[s] + relX[slot]
//   addr_C(tile, m, n)       = tileM[mt].c + tileN[nt].c + relCm[m] + relCn[n]
// so one compiled kernel serves every index permutation; only tile shapes are templates.
// Bounds ("correct for any problem size"): every tile carries a bitmask of its
// in-range tile-local rows (m) / columns (n); every k-step a bitmask of in-range k.
#pragma once
#include <cstdint>

namespace tc {

constexpr int kMaxDigits = 8;
constexpr int kMaskWords = 2;   // BM, BN <= 128 -> two 64-bit words per tile

constexpr int kMaxTmaDims = 5;

struct TileInfo {           // one m-tile (or n-tile)
  int64_t op;               // element offset of the tile origin in X (or Y), incl. base
  int64_t c;                // element offset of the tile origin in C (m side incl. C's base)
  uint64_t mask[kMaskWords];// bit r: tile-local row (column) r lies inside the tensor
  int32_t coord[kMaxTmaDims];// origin index per C dimension (this side's dims, 0 elsewhere)
  int32_t pad_;
};

struct KOuter {            // one combination of the outer moving k digits
  int64_t x, y;
  uint64_t mask;
};

// Opaque 128-B TMA descriptor (CUtensorMap); kept as bytes so host-only code needs no
// driver headers.
struct alignas(64) TmaDesc {
  unsigned char bytes[128];
};

// tcgen05 kernel, TMA operand loads (api.cu umma_tma_layout): one elected producer thread
// issues, per stage, the boxes of X and Y straight into the 128-B swizzled UMMA planes
struct TmaOperand {
  uint32_t pack;            // per map dim j < 5: 3 bits of source (0-4: C position -> tile
                            // origin coordinate; 7: the k index -> k-step origin), rank at bit 16
  int nsub;                 // boxes along map dim 0 (MN-major operands wider than one atom)
  int sub_bytes;            // smem stride between those boxes
  int sub_crd;              // coordinate step along dim 0 between them
  int tx;                   // bytes one box delivers
};

struct KParams {
  TmaDesc xmap, ymap;       // tcgen05 + TMA: the operands' tensor maps (per call: they hold the pointers)
  TmaOperand xt, yt;
  int kt;                   // tcgen05 + TMA: k-tile extent (coordinate step per k-step)
  TmaDesc cmap;             // TMA descriptor of C (tile box = the C tile), if use_tma
  int use_tma;              // 1: epilogue stages the C tile in smem and TMA-stores it
  int c_rank;               // dimensions of the C descriptor
  int Mt, Nt;               // tile extents (<= BM, BN)
  const void *X;            // M-side operand (A or B)
  const void *Y;            // N-side operand
  void *C;
  double alpha, beta;
  int mtiles, ntiles, ntotal;   // tiles per side, total tiles
  int group_m;              // CTA rasterisation: m-tiles per group (L2 locality)
  const TileInfo *tileM;    // [mtiles]
  const TileInfo *tileN;    // [ntiles]
  uint64_t fullM[kMaskWords], fullN[kMaskWords];  // masks of an interior tile
  uint64_t fullK;           // k mask of a step with every tile-local k in range
  const int64_t *relCm;     // [BM] offset in C of tile-local m
  const int64_t *relCn;     // [BN]
  const int32_t *boxM;      // [BM] offset of tile-local m in the smem C box (TMA epilogue)
  const int32_t *boxN;      // [BN]
  // k side: steps in mixed radix over the internal tile grid (kdig order, first digit
  // fastest).  Digits whose tile covers the extent never move (their mask is folded into
  // kbase); the first moving digit is stepped in registers, the others (rare carries) come
  // from a small table, prefetched one carry ahead (KStep, kernel_f64.cuh).
  int nsteps;
  int kcnt0;                // tiles of the inner moving digit (1: none)
  int64_t kdX0, kdY0;       // offset in X / Y of one inner tile step
  uint64_t ktail0;          // k-mask factor while the inner digit is at its last tile
  uint64_t kbase;           // k mask of the fixed digits (all in-range bits otherwise)
  int nouter;               // combinations of the outer moving digits
  const KOuter *kouter;     // [nouter] their X / Y offsets and k-mask factor
  // load slots: the X tile (Mt x Kt) and the Y tile (Kt x Nt) enumerated in each
  // operand's OWN memory order (threads along x walk the input's FVI)
  const int32_t *relX;      // [nslotX] element offset of the slot inside (tile, step)
  const uint32_t *packX;    // [nslotX] smem offset | k << 13 | m << 19
  const int32_t *relY;
  const uint32_t *packY;
  int nslotX, nslotY;
  int vecX, vecY;           // elements per slot (16-B cp.async at 2 FP64 / 8 BF16)
  int pf_mstep;             // FP64, beta != 0: producers prefetch the tile's old C into L2, one
                            // address per pf_mstep tile rows (0: off; C's FVI must lead m)
  int vecC;                 // C vector (elements): BF16 8 / FP64 STG 2 => tile rows come in aligned
                            // C-contiguous runs of vecC (16-B stores); 1 => per-element stores
  int nmma, kmma;           // UMMA: instruction N (<= BN) and K-instructions per stage (<= BK / KI)
  int cs0, ct0;             // UMMA: tile-row stride and tile of C's FVI among the m digits
                            // (cs0 == 1: C's FVI leads m; the runs are consecutive rows)
};

}  // namespace tc
