// tiles.hpp — digit orders, load-slot tables, shared-memory bank simulation and tile tables
// (SURVEY 8(a) rows a3/a4).  Shared by the planner (for the cost model) and the launcher
// (for the device tables), so the model scores exactly what the kernel will execute.
#pragma once
#include <cstdint>
#include <vector>

#include "contraction.hpp"
#include "kparams.hpp"

namespace tc {

// Compiled kernel shapes (kernel_f64.cuh template instances, api.cu kernel table).
// F64: DMMA register tiles (kernel_f64.cuh).  The others share the tcgen05 kernel
// (kernel_umma.cuh): BF16 = kind::f16, TF32 = kind::tf32 on FP32 storage, F32X3 = FP32 data
// as a 3-pass split TF32 product (hi*hi + hi*lo + lo*hi, near-FP32 accuracy).
enum Kind { KIND_F64_DMMA = 0, KIND_BF16_UMMA = 1, KIND_TF32_UMMA = 2, KIND_F32X3_UMMA = 3 };
inline bool is_umma(int kind) { return kind != KIND_F64_DMMA; }
inline int kind_esize(int kind) { return kind == KIND_F64_DMMA ? 8 : kind == KIND_BF16_UMMA ? 2 : 4; }

constexpr int kNumVariants = 27;   // ids 0..20, 25, 26 (variants.def + BF16 11, 12) + TF32 21, 22 + F32X3 23, 24

struct Variant {
  int BM = 0, BN = 0, BK = 0, WM = 0, WN = 0, stages = 0, pw = 0, occ = 0;   // pw = producer warps
  int kind = KIND_F64_DMMA;
  int stg = 0;                                // 1: staged epilogue drained by the producers
  double cal = 1.0;                           // B200 model calibration: measured / predicted time
                                              // (tiles.cpp, fitted on B200, tools/model_calib.py)
  int threads() const {
    return is_umma(kind) ? 17 * 32 : ((BM / WM) * (BN / WN) + pw) * 32;   // UMMA: 8 + 8 + 1 (split: 8 + 4 + 1 + 4)
  }
  int cwarps() const { return is_umma(kind) ? 8 : (BM / WM) * (BN / WN); }
  int esize() const { return kind_esize(kind); }
};
const std::vector<Variant> &variants();

// Smem offset (in elements) of element (row mn, k) of one operand stage.
//  FP64 (kernel_f64.cuh SmemLayout): pitch 4 (mod 16) doubles, k- or mn-contiguous.
//  UMMA kinds (kernel_umma.cuh): 128-B swizzled layouts (stage base 1 KB aligned); the 16-B
//  chunk index inside a 128-B row is XORed with the row's index inside its 8-row atom.  With
//  E = 128 / esize elements per 128-B row (BF16 64, TF32 32):
//  K-major (BK = E = one 128-B row): row mn at (mn/8) KB + (mn%8) 128 B, k along the row.
//  MN-major: atom (mn/E, k/8) at ((k/8) (BMN/E) + mn/E) KB, row k%8, mn%E along the row;
//  4-byte elements use 4-row atoms with 32-B granules instead (see below).
inline int smem_off(int kind, bool kmajor, int mn, int k, int BMN, int BK) {
  if (is_umma(kind)) {
    const int es = kind_esize(kind), E = 128 / es;
    int byte;
    if (kmajor) {
      const int r = mn % 8, kb = k * es;
      byte = (mn / 8) * 1024 + r * 128 + (((kb >> 4) ^ r) << 4) + (kb & 15);
    } else if (es == 4) {
      // FP32 / TF32 MN-major (SWIZZLE_128B_BASE32B): 4-k x 128-B atoms of 512 B, atom
      // (mn/32, k/4) at ((mn/32) (BK/4) + k/4) 512 B (the k groups of an MN atom adjacent: a
      // TMA box of 32 MN x BK k), row k%4, the 32-B granule XORed with it
      const int r = k % 4, eb = (mn % E) * es;
      byte = ((mn / E) * (BK / 4) + k / 4) * 512 + r * 128 + (((eb >> 5) ^ r) << 5) + (eb & 31);
    } else {
      const int r = k % 8, eb = (mn % E) * es;
      byte = ((mn / E) * (BK / 8) + k / 8) * 1024 + r * 128 + (((eb >> 4) ^ r) << 4) + (eb & 15);
    }
    (void)BMN;
    return byte / es;
  }
  return kmajor ? mn * (BK + 4) + k : k * (BMN + 4) + mn;
}

struct Config {
  int variant = -1;
  int kind = KIND_F64_DMMA;          // which kernel family (from the dtype)
  int X = 1, Y = 2;                  // tensor ids (1 = A, 2 = B) on the M / N side
  int morder = 0;                    // 0: m digits in C order (C's FVI first); 1: X order
  int korder = 0;                    // 0: k digits in X order; 1: in Y order
  std::vector<int> mdig, ndig, kdig; // index ids, compute order
  std::vector<int> T;                // tile per index id (size = nidx)
  bool xKmajor = false, yKmajor = false;
  int vecX = 1, vecY = 1;            // vector width the plan allows (aligned pointers)
  int64_t Mt = 1, Nt = 1, Kt = 1, mtiles = 1, ntiles = 1, nctas = 1, nsteps = 1;
  // model outputs
  double t_pred = 0, t_comp = 0, t_mem = 0, t_l2 = 0, dram_bytes = 0, flops_pad = 0;
  double wfX = 0, wfY = 0;           // LDGSTS smem wavefronts per stage (simulated)
  double secX = 0, secY = 0;         // global 32-B sectors per stage (simulated)
  double paper_cost = 0;             // Alg. 3 transactions (paper mode)
  std::string paper_mapping;         // Table II lists (paper mode)
};

// Digit lists for the given order options (X = input holding C's FVI).
void digit_orders(const Contraction &c, Config &cfg);
// Tile counts / extents from cfg.T.
void finish_counts(const Contraction &c, Config &cfg);
// Can operand t use 16-B vectors with this config?
bool vec_possible(const Contraction &c, const Config &cfg, int t);
// Largest elements-per-slot vector (<= maxv, power of two) the operand's layout allows.
int vec_width(const Contraction &c, const Config &cfg, int t, int maxv);
// Largest w <= maxv (power of two) such that tile rows come in runs of w consecutive,
// w-aligned C elements: C's FVI is the first m digit, its tile, its extent, C's base and
// every other C stride are multiples of w.
int c_vec_width(const Contraction &c, const Config &cfg, int maxv);
// UMMA instruction trimming for a plan: N = Nt rounded up to 16 (K-major Y) or to a whole
// 128-B swizzle atom (MN-major Y: 64 BF16 / 32 FP32 columns), capped at BN; K instructions
// per stage = ceil(Kt / KI), KI = 32 B of k (16 BF16 / 8 TF32).
inline void umma_trim(const Config &cfg, const Variant &v, int *nmma, int *kmma) {
  const int es = kind_esize(v.kind), ki = 32 / es, nq = cfg.yKmajor ? 16 : 128 / es;
  const int n = (int)((cfg.Nt + nq - 1) / nq * nq);
  *nmma = n < v.BN ? n : v.BN;
  const int k = (int)((cfg.Kt + ki - 1) / ki);
  *kmma = k < v.BK / ki ? k : v.BK / ki;
}

// UMMA staged epilogue (kernel_umma.cuh): C's FVI f may sit anywhere among the m digits.
// Returns w (or 1) such that every w consecutive values of f's tile digit (w-aligned) are w
// consecutive, w-aligned C elements; *s0 = tile-row stride of f (product of the tiles of
// the m digits before it), *t0 = f's tile.  Rows r = lo + s0 (w j + t0 hi) start the runs.
int c_run_rows(const Contraction &c, const Config &cfg, int w, int *s0, int *t0);

struct SlotTable {
  std::vector<int64_t> rel;    // element offset inside (tile, step)
  std::vector<uint32_t> pack;  // smem offset | k << 13 | mn << 19
};
// Slots of operand t (X or Y) in the operand's own memory order.
SlotTable build_slots(const Contraction &c, const Config &cfg, int t, int vec, bool kmajor,
                      int BMN, int BK);
// Shared-memory wavefronts of the cp.async writes of one stage (32 consecutive slots per
// warp instruction; a bank serves one 32-bit word per wavefront).
double slot_wavefronts(const SlotTable &s, int vec, int esize = 8, int kind = KIND_F64_DMMA);
// Global-memory 32-B sectors one stage of loads touches (sum over warp instructions of the
// distinct sectors of 32 consecutive slots; the tile origin is taken as sector-aligned).
double slot_sectors(const SlotTable &s, int vec, int esize = 8);
// Smem offset field of a packed slot (13 bits for FP64, 14 bits for the UMMA kinds).
inline uint32_t slot_off(uint32_t pack, int kind) { return is_umma(kind) ? (pack & 0x3FFF) : (pack & 8191); }

// Device-side tables for one configuration.
struct TileTables {
  std::vector<TileInfo> tileM, tileN;
  std::vector<int64_t> relCm, relCn;
  // TMA epilogue: the C tile is a box of C (dims in C order, box dim = tile size)
  bool tma_ok = false;                 // C rank <= 5, 16-B strides, even FVI tile
  std::vector<int32_t> boxM, boxN;     // offset of tile-local m / n inside the smem box
  // k walk (KParams::kcnt0 ...): inner moving digit, fixed-digit mask, outer table
  int kcnt0 = 1;
  int64_t kdX0 = 0, kdY0 = 0;
  uint64_t ktail0 = 0, kbase = 0;
  std::vector<KOuter> kouter;
};
TileTables build_tile_tables(const Contraction &c, const Config &cfg, const Variant &v);

// tcgen05 operand t loaded by TMA boxes (kernel_umma.cuh TMA producer): the tensor-map shape
// (the pointer comes per call) and the kernel's per-box record.  Returns false when the
// plan's tiles / layout do not fit a box (the operand then keeps the cp.async producers).
struct OperandMap {
  int rank = 0;
  int64_t dims[kMaxTmaDims] = {}, strides[kMaxTmaDims] = {};   // strides in bytes, dims 1..
  uint32_t box[kMaxTmaDims] = {};
  int64_t base = 0;                                            // element offset of the view
  bool swz32 = false;                                          // 4-byte MN-major: 32-B granules
};
bool umma_tma_spec(const Contraction &c, const Config &cfg, const Variant &v, int t,
                   OperandMap *map = nullptr, TmaOperand *op = nullptr);
// CTA pairs by default (planner's choice; cfg.mtiles / ntiles set): a BN = 128 BF16 / TF32
// variant (12 / 22) with TMA operands and at least two waves of 2 x 2 blocks on the 74 pairs
inline bool cta_pair_default(const Config &cfg) {
  return (cfg.variant == 12 || cfg.variant == 22) && ((cfg.mtiles + 1) / 2) * ((cfg.ntiles + 1) / 2) >= 148;
}

}  // namespace tc
