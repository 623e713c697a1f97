// stream.hpp — the streaming path for low-intensity "tensor x matrix" contractions (the ML
// cases TCCG #1-8): the Y operand is a small matrix kept whole in
// shared memory, X streams through in TMA boxes cut in X's own index order (each
// input read along its FVI, whole boxes per request), and every C element leaves in a run of
// consecutive values of C's FVI straight from the MMA accumulators — whatever the permutation
// between X and C, with no on-chip transpose: a warp owns AR consecutive values a0 .. a0+AR-1
// of C's FVI `a` and runs one m16 MMA block per value, so the accumulator element (row, n) of
// its AR blocks is the run C[a0 .. a0+AR-1, row, n] (C stored along its FVI).
//
// Scope (stream_plan decides): BF16, TF32, FP32 (split TF32) and FP64 (DMMA m8n8k4), no batch
// index, exactly one internal index k and one Y-side external index n (after fusion) with n <= 32
// (n <= 72 on FP64: NB = 9, AR = 2) and Y small enough for shared memory, X of rank <= 5 with
// 16-B multiple strides (TMA), C's FVI on X (X = the input holding C's FVI; SM_M when it
// is also X's FVI, FP64 only).  beta != 0 runs the BETA instances (kernels_stream_beta.cu) on
// FP64 / FP32 C; on BF16 it runs the plan's tile configuration (which the planner always keeps):
// its epilogue rounds alpha * sum + beta * C to BF16 once.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

#include "contraction.hpp"
#include "kparams.hpp"

namespace tc {

constexpr int kSMaxMdims = 4;       // X externals (m dims)
constexpr int kSWarps = 8;          // compute warps (+ 1 TMA producer warp)
constexpr int kSThreads = (kSWarps + 1) * 32;
constexpr int kSRows = 16;          // rows of one MMA block (m16)

// resident CTAs per SM an instance is compiled for (__launch_bounds__): two while the
// accumulators (AR x NB blocks of 4 registers) leave room under the 2-CTA register cap
constexpr int stream_occ(int NB, int AR) { return AR * NB * 4 <= 48 ? 2 : 1; }

enum StreamMode { SM_T = 0, SM_M = 1, SM_K = 2 };
// SM_T: X's FVI is an external E != C's FVI a: a block's 16 rows are two octets of 8
//       consecutive E (ldmatrix.trans over k rows of the X box).
// SM_K: X's FVI is k: a block's 16 rows are any 16 m-rows at one a (ldmatrix, k-contiguous).
// SM_M (FP64): X's FVI is C's FVI a: a block's 8 rows are an octet of a, the warp's AR blocks
//       run over the next X external (C's runs come from the 8 lanes, not from the registers).

struct SParams {
  TmaDesc xmap;
  const void *Y;            // the whole Y operand (read once per CTA into smem)
  void *C;                  // C's origin
  const uint32_t *tab;      // per unit: [16] X box byte offsets of its rows (at a0, k = 0),
                            // [16] C box element offsets of its rows (at a0, n = 0); then per
                            // 16-B chunk of the C box its element offset in C from the tile origin
  int64_t ysk, ysn;         // element strides of k and n in Y
  int64_t csn;              // element stride of n in C
  int64_t mCs[kSMaxMdims];  // element strides of the m dims in C
  float alpha;
  double alpha64;           // (FP64 kernel)
  double beta;              // C = alpha * sum + beta * C (FP64 / FP32 C; BF16 plans run beta != 0 on the tile kernel)
  int xrank;
  int nmd;                  // m dims, raster order (C's FVI first)
  int mT[kSMaxMdims], mNt[kSMaxMdims], mX[kSMaxMdims], mN[kSMaxMdims];
  int kX;                   // X map dim of k
  int K, N, KP, YP;         // k extent, n extent, k padded to 16, Y smem pitch (elements)
  int ntiles;
  int KB, nks;              // k per stage (box extent along k), k-steps per tile
  int nunits;               // warp units per tile (<= kSWarps): (row set, a group)
  int ru;                   // rows per unit: 16 (BF16 m16n8k16) or 8 (FP64 DMMA m8n8k4)
  int stages, stage_bytes, stage_pitch;   // X ring: stages, box bytes, bytes between stages
  int xpitchk;              // SM_T: bytes between consecutive k in the X box
  int xpitcha;              // bytes between consecutive a in the X box
  int xswz;                 // the X box's swizzle mask over address bits 7.. (0, 1 = 32B, 3 = 64B, 7 = 128B)
  int off_y, off_tab, off_bar, off_stg;   // smem byte offsets from the 1 KB aligned base
  // the C box (C order; m dims T, n 8 NB): staged in smem, 16-B chunks XOR-swizzled (chunk ^=
  // fold(chunk >> 3) & 7, fold = x ^ x >> cs1 ^ x >> cs2: the planner's simulated choice),
  // stored by every compute thread as 16-B runs along C's FVI
  int crank, nchunk, cbsn;  // C box rank, 16-B chunks, box element stride of n
  int cbsj;                 // C box element stride of the run dim (1: the runs are along C's FVI)
  int nstg, stg_pitch;      // C boxes in smem (1 or 2: tile i+1 fills one while tile i's is stored)
  int cbox[kMaxTmaDims];    // C box extents (C order)
  int cmd[kMaxTmaDims];     // per C dim: its m dim (raster order), or -1 for n
  int cs1, cs2;             // staging swizzle fold shifts
};

struct StreamCfg {
  bool on = false;          // the contraction is a streaming shape (planned below)
  bool preferred = false;   // ... and the path beats the tile kernels by default: always for BF16;
                            // FP64 below 0.8 of the DMMA ridge (above it the DMMA tile kernel
                            // keeps the pipe busier; tuning still times both)
  int NB = 0, AR = 0;       // kernel instance: n8 blocks, C-FVI run length per warp
  int X = 1;                // 1: X = A, 2: X = B
  int mode = SM_T;
  int xrank = 0;
  int64_t xdims[kMaxTmaDims] = {}, xstr[kMaxTmaDims] = {};
  uint32_t xbox[kMaxTmaDims] = {};
  int64_t xbase = 0, cbase = 0, ybase = 0;
  int occ = 1;              // resident CTAs per SM the instance is built for
  int xswz = 0;             // CUtensorMapSwizzle of the X map (0 none, 1 32B, 2 64B, 3 128B)
  SParams kp{};             // host copy (pointers / maps filled per call)
  std::vector<uint32_t> tab;
  size_t smem = 0;
  double t_pred = 0;        // model time (s)
  double bytes = 0;         // algorithmic bytes (X + Y + C)
  int T[kMaxIdx] = {};      // per normalised index: tile (k: KB, n: N)
  std::string why;          // why the path is off (for tc_plan_info)
  int rank = 0, nranks = 0; // which of the model's best configurations this is, of how many
};

// Decide whether the streaming path applies to the normalised contraction and choose its
// tiles (dtype kind from tiles.hpp).  sms: SMs of the device; rank: the model's rank-th best
// configuration (0 = its first choice; tc_plan_tuned times the first kStreamRanks).
constexpr int kStreamRanks = 3;
bool stream_plan(const Contraction &c, int kind, int sms, StreamCfg &s, int rank = 0);

}  // namespace tc
