// group.hpp — fused grouped contraction: several contractions that all
// write one output C, e.g. the 9 sd_t_d1 + 9 sd_t_d2 CCSD(T) triples accumulating into t3
// (P:L27, L330, L344), executed as ONE persistent kernel that keeps each C tile on chip
// across all members and writes it once:
//     C = alpha * sum_i sum_int A_i * B_i + beta * C.
// The C tile is a hyper-rectangle prod_p T_p over C's positions (the same for every member,
// P:L119); member i sees it as an Mt_i x Nt_i matrix (rows = the C positions of its operand
// X_i, columns = those of Y_i) and contracts over its own internal indices.  The
// member's accumulators (DMMA register tiles, as in the single-contraction kernel) are added
// into an XOR-swizzled shared-memory box of the C tile after the member's last k-step; the
// box is stored to C once per tile (kernel_group.cuh).
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
constexpr int kGBM = 64, kGBN = 64;   // member tile bounds (Mt_i <= 64, Nt_i <= 64)

// Box swizzle (doubles): the low 4 bits (16 doubles = one 128-B bank row) are XORed with
// bits 4..7 ^ 8..11 of the box offset, which makes the member flushes (fragment layout ->
// box) conflict-free for the triples' digit orders (planner simulation, group.cpp).
inline TC_HD int gbox_sw(int o) { return o ^ (((o >> 4) ^ (o >> 8)) & 15); }

// One operand tile of one member, gathered by runs along the operand's FVI (P:L138-145:
// consecutive threads walk the operand's memory order).
struct GOperandDev {
  int64_t tstep[kGMaxCdims];   // element offset of one tile step along C position p
  int32_t run0, nrun;          // slice of the run tables
  int32_t runlen;              // elements per run (tile of the operand's dim 0, or 1)
  int32_t vec;                 // elements per cp.async (2: 16 B, 1: 8 B) the plan allows
  int32_t ndim;
  int32_t cpos[kGMaxOpDims];   // C position of operand dim j, or -1 (internal)
};

struct GMemberDev {
  GOperandDev x, y;
  int32_t layout;              // bit 0: X plane k-major, bit 1: Y plane k-major
  int32_t step0, nsteps;       // slice of the step table
  int32_t pad0, npad;          // slice of the k-padding zero list (Kt < BK)
  int32_t xIsA;                // 1: X = A, Y = B; 0: X = B, Y = A
};

struct GStepDev {
  int64_t kx, ky;              // offsets of the k tile in X / Y
  uint64_t klimX, klimY;       // per operand dim (bytes): k-tile limits (0 for C dims)
  int32_t full;                // every k digit complete
  int32_t pad_;
};

struct GroupTables {
  int rank = 0;                // C positions
  int64_t N[kGMaxCdims] = {}, cstride[kGMaxCdims] = {}, cbase = 0;
  int32_t T[kGMaxCdims] = {}, ntl[kGMaxCdims] = {};
  int64_t ntiles = 0;
  int BK = 24, stages = 3, variant = 0;
  int box = 0;                 // prod T (elements of the C tile)
  int uvec = 1;                // copy-out elements per unit (2: 16-B stores allowed)
  std::vector<GMemberDev> mem;
  std::vector<GStepDev> steps;
  std::vector<int32_t> runRel;
  std::vector<uint32_t> runSoff;
  std::vector<uint64_t> runDig;
  std::vector<uint32_t> pad;   // byte offsets (from the stage base) to zero per k-padded step
  std::vector<int32_t> boxM, boxN;   // per member kGBM / kGBN entries (-1: row outside Mt)
  std::vector<int64_t> unitRel;      // copy-out: C offset of unit u relative to the tile origin
  std::vector<uint64_t> unitDig;     // its digits (bytes, position 0 excluded)
  // planner statistics (tc_group_info)
  std::vector<int64_t> Mt, Nt, Kt;
  std::vector<double> flushWf, loadWf;   // simulated smem wavefronts per member-tile
  double flops = 0, padded_flops = 0, plan_ms = 0;
};

// Plan the fused group of n member contractions (parsed, unnormalised).  Every member must
// give C the same layout (checked by the caller), hold no batch index, and fit the tile
// bounds; otherwise ST_UNSUPPORTED with a reason in err.
Status plan_group(const std::vector<const Contraction *> &members, GroupTables &out, std::string &err);

// Shared-memory stage geometry of the group kernel (must match kernel_group.cuh).
inline int gplane_doubles(int BMN, int BK) {
  const int a = BMN * (BK + 4), b = BK * (BMN + 4);
  return (a > b ? a : b) + 2;
}

}  // namespace tc
