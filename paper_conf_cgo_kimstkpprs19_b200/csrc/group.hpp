// group.hpp — fused grouped contraction: several contractions that all
// write one output C, e.g. the 9 sd_t_d1 + 9 sd_t_d2 CCSD(T) triples accumulating into t3
// (P:L27, L330, L344), executed as ONE persistent kernel that keeps each C tile on chip
// across all members and writes it once:
//     C = alpha * sum_i sum_int A_i * B_i + beta * C.
// The C tile is a hyper-rectangle prod_p T_p over C's positions (the same for every member,
// P:L119); member i sees it as an Mt_i x Nt_i matrix (rows = the C positions of its operand
// X_i, columns = those of Y_i) and contracts over its own internal indices.  The
// member's DMMA register tile starts from the C tile's current values in an XOR-swizzled
// shared-memory box and is written back after the member's last k-step; the box is stored to
// C once per tile (kernel_group.cuh).
//
// Operand tiles reach shared memory either by TMA (one box per 16 / 8 elements of the
// operand's FVI, SWIZZLE_128B / 64B, every operand of every member eligible and 16-B aligned)
// or by cp.async gathers along the FVI into padded-pitch planes (any layout).
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "contraction.hpp"

#ifdef __CUDACC__
#define TC_HD __host__ __device__
#else
#define TC_HD
#endif

namespace tc {

constexpr int kGMaxMembers = 32;
constexpr int kGMaxCdims = 8;
constexpr int kGMaxOpDims = 8;
constexpr int kGMaxTmaDims = 5;
constexpr int kGBM = 64, kGBN = 64;   // member tile bounds (Mt_i <= 64, Nt_i <= 64)
constexpr int kGCtab = 4 * 64;        // consumer table entries per member: rowX, rowY, boxM, boxN

// Box swizzle (doubles): the low 4 bits (16 doubles = one 128-B bank row) are XORed with
// bits 4..7 ^ 8..11 of the box offset, which makes the member flushes (fragment layout ->
// box) conflict-free for the triples' digit orders (planner simulation, group.cpp).
inline TC_HD int gbox_sw(int o) { return o ^ (((o >> 4) ^ (o >> 8)) & 15); }

// Byte offset of a plane element under the plane's swizzle (TMA SWIZZLE_128B: mask 0x70,
// SWIZZLE_64B: 0x30 — byte bits [4,7) / [4,6) XORed with bits [7,10) / [7,9); pitched
// cp.async planes: 0).
inline TC_HD uint32_t gplane_sw(uint32_t b, uint32_t mask) { return b ^ ((b >> 3) & mask); }

// One operand tile of one member.
struct GOperandDev {
  int64_t tstep[kGMaxCdims];   // cp.async: element offset of one tile step along C position p
  int32_t run0, nrun;          // cp.async: slice of the run tables
  int32_t runlen;              // cp.async: elements per run (tile of the operand's dim 0, or 1)
  int32_t vec;                 // cp.async: elements per copy (2: 16 B, 1: 8 B) the plan allows
  int32_t ndim;
  int32_t cpos[kGMaxOpDims];   // C position of operand dim j, or -1 (internal)
  // consumer k addressing of the plane, k = 4 kk + t:
  //   byte(k) = (k >> kch_log2) * kchunk + (k & (2^kch_log2 - 1)) * kmul   (then swizzled)
  int32_t kch_log2[2], kchunk[2], kmul[2], swz[2];   // [0] cp.async planes, [1] TMA boxes
  // TMA: one box per (tile, k-step) over the operand's dims in a PERMUTED order (dim 0 = the
  // FVI; the others ordered so that the DMMA fragment loads of the dense box are
  // conflict-free, group.cpp); box = the tile (a k-FVI box padded to a pitch of 4 mod 8)
  int32_t tma_cpos[kGMaxTmaDims];   // C position of map dim j (-1: the k dim or unused)
  int32_t tma_kdim;                 // map dim of the internal index (-1: none)
  int32_t tma_tx;                   // bytes the box delivers (expect-tx)
  uint32_t tma_pack;                // the producer's copy: 4 bits of tma_cpos per map dim (15: none),
                                    // the map's rank at bit 20, tma_kdim at bit 24 (15: none)
};

struct GMemberDev {
  GOperandDev x, y;
  int32_t step0, nsteps;       // slice of the step table
  int32_t pad0, npad;          // cp.async: slice of the k-padding zero list (Kt < BK)
  int32_t xIsA;                // 1: X = A, Y = B; 0: X = B, Y = A
  int32_t kq;                  // k4 groups per step (ceil(Kt / 4))
  int32_t tma_yoff;            // TMA: byte offset of the Y box in the stage (after the X box)
  // per load mode: 1 when the next member (execution order) maps its register tile onto the
  // box exactly as this one — the tile then stays in registers across the two (no write-back
  // and reload in between: the d1 / d2 triples come in such pairs)
  uint8_t chain[2];
  uint8_t pad_[2];
};

struct GStepDev {
  int64_t kx, ky;              // offsets of the k tile in X / Y (elements)
  uint64_t klimX, klimY;       // per operand dim (bytes): k-tile limits (0 for C dims)
  int32_t kc;                  // TMA: origin of the k tile (one internal index)
  int32_t full;                // every k digit complete
};

struct GroupTables {
  int rank = 0;                // C positions
  int64_t N[kGMaxCdims] = {}, cstride[kGMaxCdims] = {}, cbase = 0;
  int32_t T[kGMaxCdims] = {}, ntl[kGMaxCdims] = {};
  int64_t ntiles = 0;
  int BK = 24, variant = 0;
  int box = 0;                 // prod T (elements of the C tile)
  int uvec = 1;                // copy-out elements per unit (2: 16-B stores allowed)
  bool tma = false;            // every operand has a TMA box layout
  std::vector<GMemberDev> mem;
  std::vector<GStepDev> steps;
  std::vector<int32_t> runRel;
  std::vector<uint32_t> runSoff;
  std::vector<uint64_t> runDig;
  std::vector<uint32_t> pad;   // byte offsets (from the stage base) to zero per k-padded step
  std::vector<int32_t> ctab[2];      // per mode, per member kGCtab entries (group.hpp layout)
  std::vector<int64_t> unitRel;      // copy-out: C offset of unit u relative to the tile origin
  std::vector<uint64_t> unitDig;     // its digits (bytes)
  // TMA tensor maps are encoded per call (they hold the operand pointers): per member and
  // side, the operand's dims, byte strides and box
  struct TmaSpec {
    int rank = 0;
    uint64_t dims[kGMaxTmaDims] = {}, strides[kGMaxTmaDims] = {};   // strides[j] of dim j+1, bytes
    uint32_t box[kGMaxTmaDims] = {};
    int64_t base = 0;          // element offset of the view's origin
  };
  int tma_stage_bytes = 0;     // largest X box + Y box of a member (<= the TMA stage)
  std::vector<TmaSpec> tmaX, tmaY;
  // execution order: position k runs member order[k] (members with one register-tile mapping
  // adjacent, group.cpp); every per-member vector here is in execution order
  std::vector<int> order;
  // planner statistics (tc_group_info)
  std::vector<int64_t> Mt, Nt, Kt;
  std::vector<double> flushWf, loadWf, fragWf;   // simulated smem wavefronts per member-tile
  double flops = 0, padded_flops = 0, plan_ms = 0;
};

// Plan the fused group of n member contractions (parsed, unnormalised).  Every member must
// give C the same layout (checked by the caller), hold no batch index, and fit the tile
// bounds; otherwise ST_UNSUPPORTED with a reason in err.
Status plan_group(const std::vector<const Contraction *> &members, GroupTables &out, std::string &err);

// Shared-memory stage geometry of the group kernel (must match kernel_group.cuh).
inline int gplane_doubles(int BMN, int BK) {   // cp.async plane: padded pitch
  const int a = BMN * (BK + 4), b = BK * (BMN + 4);
  return (a > b ? a : b) + 2;
}
// TMA stage: the X box and the Y box of one member (a k-FVI box carries a padded pitch)
inline int gtma_stage_bytes(int BK) { return 2 * kGBM * (BK + 4) * 8; }

}  // namespace tc
