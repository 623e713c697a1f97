// kernel_f64.cuh — the FP64 direct-contraction kernel of libtc for sm_100a.
//
// The paper's four steps (Alg. 1) re-designed for B200:
//   (1) GMEM -> SMEM: PRODUCER warps gather the X tile (Mt x Kt) and Y tile (Kt x Nt) of
//       each k-step with cp.async (16 B when the operand's FVI allows; zero-fill outside the
//       tensor), walking each operand in its own memory order, into a
//       STAGES-deep ring; completion is signalled on a per-stage mbarrier
//       (cp.async.mbarrier.arrive), release by the consumers on a second mbarrier.  The
//       paper's kernel was single-buffered with two __syncthreads per step.
//   (2) SMEM -> REG: CONSUMER warps load DMMA fragments (mma.sync.m8n8k4.f64 -> SASS
//       DMMA.8x8x4; measured at 37.1 TFLOP/s = the FP64 pipe's peak, profiles/
//       r01_peaks.json).  The smem layout per operand (k- or m-contiguous) is a template
//       parameter, so fragment addresses are immediates; pitch = 4 (mod 16) doubles keeps
//       them bank-conflict-free.
//   (3) outer product: each consumer warp owns a WM x WN register tile of C (P:L117:
//       accumulate in registers); the paper's r_C[T_b][T_c] rank-1 updates become
//       (WM/8) x (WN/8) DMMA tiles per k4.
//   (4) REG -> GMEM: C = alpha * acc + beta * C through separable row / column offsets,
//       predicated by the tile's row / column bitmasks (correct for any size).
//       Direct variants store from the fragments.  DEFERRED variants (STG) park the raw
//       accumulators in a per-warp smem staging tile and go straight on with the next tile;
//       the same warp drains the parked tile a few columns per k4 step of the next tile's
//       mainloop (lane = tile row: coalesced along C's FVI, 16 B pairs when C allows), so
//       the C write of tile i is issued in the shadow of tile i+1's DMMAs and no register of
//       an in-flight store is overwritten by the next tile's accumulators (the near-ridge
//       K = 24 CCSD(T) and the memory-bound ML contractions, where the C write is most of the
//       traffic).  No barrier is involved: each warp owns its staging region.
// CTAs are persistent (grid = 148 x CTAs/SM, tiles round-robin): the producers run up to
// STAGES k-steps ahead ACROSS tile boundaries, so tile i's epilogue stores overlap tile
// i+1's loads — the overlap the K = 24 CCSD(T) contractions need (SURVEY 7.2 part 1).
#pragma once
#include <cstdint>
#include "kparams.hpp"

namespace tc {

__device__ __forceinline__ void cp_async8(uint32_t dst, const double *src, int srcbytes) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(dst), "l"(src), "r"(srcbytes));
}
__device__ __forceinline__ void cp_async16(uint32_t dst, const double *src, int srcbytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(dst), "l"(src), "r"(srcbytes));
}
__device__ __forceinline__ void mbar_init(uint32_t bar, int count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_arrive_cp_async(uint32_t bar) {
  asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];\n" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n}\n" ::"r"(bar), "r"(parity) : "memory");
}

// Wait with back-off: for warps that wait long (e.g. the epilogue during a long k loop), so
// that their polling does not steal issue slots and barrier-unit bandwidth from the warps
// on the critical path.
__device__ __forceinline__ void mbar_wait_sleep(uint32_t bar, uint32_t parity) {
  uint32_t done;
  for (;;) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done) : "r"(bar), "r"(parity) : "memory");
    if (done) return;
    __nanosleep(256);
  }
}

// TMA store of the smem box at `src` to the C tile at `crd` (cp.async.bulk.tensor, tile mode)
__device__ __forceinline__ void tma_store(const TmaDesc *map, int rank, const int32_t *crd, uint32_t src) {
  const uint64_t m = reinterpret_cast<uint64_t>(map);
  switch (rank) {
    case 1:
      asm volatile("cp.async.bulk.tensor.1d.global.shared::cta.bulk_group [%0, {%1}], [%2];\n"
                   ::"l"(m), "r"(crd[0]), "r"(src) : "memory");
      break;
    case 2:
      asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];\n"
                   ::"l"(m), "r"(crd[0]), "r"(crd[1]), "r"(src) : "memory");
      break;
    case 3:
      asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%1, %2, %3}], [%4];\n"
                   ::"l"(m), "r"(crd[0]), "r"(crd[1]), "r"(crd[2]), "r"(src) : "memory");
      break;
    case 4:
      asm volatile("cp.async.bulk.tensor.4d.global.shared::cta.bulk_group [%0, {%1, %2, %3, %4}], [%5];\n"
                   ::"l"(m), "r"(crd[0]), "r"(crd[1]), "r"(crd[2]), "r"(crd[3]), "r"(src) : "memory");
      break;
    default:
      asm volatile("cp.async.bulk.tensor.5d.global.shared::cta.bulk_group [%0, {%1, %2, %3, %4, %5}], [%6];\n"
                   ::"l"(m), "r"(crd[0]), "r"(crd[1]), "r"(crd[2]), "r"(crd[3]), "r"(crd[4]), "r"(src)
                   : "memory");
      break;
  }
  asm volatile("cp.async.bulk.commit_group;\n" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(bar), "r"(bytes) : "memory");
}

// TMA load of one box at (c0..c4) into smem dst, completing on mbarrier bar, with an L2 policy
// (the fused group kernel and the tcgen05 kernel's TMA producers)
__device__ __forceinline__ void tma_load(const TmaDesc *map, int rank, int32_t c0, int32_t c1, int32_t c2,
                                         int32_t c3, int32_t c4, uint32_t dst, uint32_t bar, uint64_t pol) {
  const uint64_t m = reinterpret_cast<uint64_t>(map);
  switch (rank) {
    case 1:
      asm volatile("cp.async.bulk.tensor.1d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint"
                   " [%0], [%1, {%2}], [%3], %4;\n" ::"r"(dst), "l"(m), "r"(c0), "r"(bar), "l"(pol) : "memory");
      break;
    case 2:
      asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint"
                   " [%0], [%1, {%2, %3}], [%4], %5;\n" ::"r"(dst), "l"(m), "r"(c0), "r"(c1), "r"(bar), "l"(pol)
                   : "memory");
      break;
    case 3:
      asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint"
                   " [%0], [%1, {%2, %3, %4}], [%5], %6;\n" ::"r"(dst), "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(bar),
                   "l"(pol) : "memory");
      break;
    case 4:
      asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint"
                   " [%0], [%1, {%2, %3, %4, %5}], [%6], %7;\n" ::"r"(dst), "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(c3),
                   "r"(bar), "l"(pol) : "memory");
      break;
    default:
      asm volatile("cp.async.bulk.tensor.5d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint"
                   " [%0], [%1, {%2, %3, %4, %5, %6}], [%7], %8;\n" ::"r"(dst), "l"(m), "r"(c0), "r"(c1), "r"(c2),
                   "r"(c3), "r"(c4), "r"(bar), "l"(pol) : "memory");
      break;
  }
}

__device__ __forceinline__ void tma_wait_read() { asm volatile("cp.async.bulk.wait_group.read 0;\n" ::: "memory"); }
__device__ __forceinline__ void tma_wait_all() { asm volatile("cp.async.bulk.wait_group 0;\n" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory"); }
__device__ __forceinline__ void consumer_sync(int nthreads) {
  asm volatile("bar.sync 1, %0;\n" ::"r"(nthreads) : "memory");
}

// st.global.f64 under a predicate (keeps the epilogue free of branches)
#ifndef TC_F64_ST_OP        // side builds (tools/f64_epi_ab.py): st.global.cs.f64 etc.
#define TC_F64_ST_OP "st.global.f64"
#endif
__device__ __forceinline__ void st_pred(double *ptr, double v, uint32_t ok) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %2, 0;\n\t@p " TC_F64_ST_OP " [%0], %1;\n}\n"
               ::"l"(ptr), "d"(v), "r"(ok) : "memory");
}

__device__ __forceinline__ void dmma884(double &c0, double &c1, double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
               : "+d"(c0), "+d"(c1) : "d"(a), "d"(b));
}

template <int BM, int BN, int BK>
struct SmemLayout {
  static constexpr int PM = BM + 4, PN = BN + 4, PK = BK + 4;  // pitches, 4 mod 16 doubles
  // + 2 doubles of scratch per stage: the landing spot of padding ("null") load slots
  static constexpr int XS = ((BM * PK > BK * PM) ? BM * PK : BK * PM) + 2;
  static constexpr int YS = ((BN * PK > BK * PN) ? BN * PK : BK * PN) + 2;
};

template <int BM, int BN, int BK, int WM, int WN, int STAGES, int PW, bool STG = false>
struct F64Kernel {
  static constexpr int WARPS_M = BM / WM, WARPS_N = BN / WN;
  static constexpr int CWARPS = WARPS_M * WARPS_N;            // consumer warps
  static constexpr int THREADS = (CWARPS + PW) * 32;
  static constexpr int MI = WM / 8, NJ = WN / 8;
  static constexpr int EX = (BM * BK + PW * 32 - 1) / (PW * 32);  // X slots per producer thread
  static constexpr int EY = (BN * BK + PW * 32 - 1) / (PW * 32);
  using L = SmemLayout<BM, BN, BK>;
  // deferred epilogue: per consumer warp a [WN][SP] staging tile (lane = row, SP = 36
  // doubles: the fragment writes take the 2-wavefront minimum, the row reads are contiguous)
  static constexpr int SP = 36;
  static constexpr size_t ring_bytes() {
    return sizeof(double) * (size_t)STAGES * (L::XS + L::YS) + 16 * (size_t)STAGES + 12 * (size_t)(BM + BN);
  }
  static constexpr size_t kStageOffset = (ring_bytes() + 127) / 128 * 128;   // bytes
  static constexpr size_t stg_bytes() { return STG ? 8 * (size_t)CWARPS * WN * SP : 0; }
  static constexpr size_t base_bytes() { return kStageOffset + stg_bytes(); }
  // ring + barriers + tables; the optional TMA staging box starts at the next 1 KB boundary
  static constexpr size_t kStagingOffset = (base_bytes() + 1023) / 1024 * 1024 / 8;   // in doubles
  static constexpr size_t smem_bytes(bool tma) {
    return tma ? kStagingOffset * 8 + 8 * (size_t)BM * BN : base_bytes();
  }
  static_assert(BK % 4 == 0 && BK <= 64, "BK");
  static_assert(WM % 8 == 0 && WN % 8 == 0, "warp tile");
  static_assert(BM % WM == 0 && BN % WN == 0, "warp grid");
  static_assert(BM <= 64 * kMaskWords && BN <= 64 * kMaskWords, "tile masks");
  static_assert(L::XS < 8192 && L::YS < 8192, "13-bit smem offsets");
  static_assert(!STG || WM == 32, "deferred epilogue: one lane per warp-tile row");
};

// (mt, nt) of tile t with grouped rasterisation (group_m m-tiles share a band of n-tiles).
__device__ __forceinline__ void tile_coords(const KParams &p, int t, int &mt, int &nt) {
  const int per_group = p.group_m * p.ntiles;
  const int g = t / per_group;
  const int first = g * p.group_m;
  const int gsz = min(p.group_m, p.mtiles - first);
  const int r = t - g * per_group;
  mt = first + r % gsz;
  nt = r / gsz;
}

__device__ __forceinline__ void prefetch_l1(const void *ptr) {
  asm volatile("prefetch.global.L1 [%0];\n" ::"l"(ptr));
}

// Walk over the k-tile grid (P:L126 mixed radix): origin offsets of the current step in X and
// Y and its k mask.  The inner moving digit steps in registers; a carry into the outer
// digits reads the next entry of p.kouter (prefetched into L1 at the previous carry).
struct KStep {
  int c0, o;
  int64_t s0x, s0y;          // inner digit's offsets
  KOuter cur;                // outer digits' current combination
  __device__ __forceinline__ void reset(const KParams &p) {
    c0 = 0;
    o = 0;
    s0x = s0y = 0;
    cur = p.kouter[0];
    if (p.nouter > 1) prefetch_l1(p.kouter + 1);
  }
  __device__ __forceinline__ int64_t sx() const { return cur.x + s0x; }
  __device__ __forceinline__ int64_t sy() const { return cur.y + s0y; }
  __device__ __forceinline__ uint64_t mask(const KParams &p) const {
    return (c0 == p.kcnt0 - 1 ? p.ktail0 : p.kbase) & cur.mask;
  }
  __device__ __forceinline__ void advance(const KParams &p) {
    if (++c0 < p.kcnt0) {
      s0x += p.kdX0;
      s0y += p.kdY0;
      return;
    }
    c0 = 0;
    s0x = s0y = 0;
    if (p.nouter > 1) {
      o = o + 1 == p.nouter ? 0 : o + 1;
      cur = p.kouter[o];
      prefetch_l1(p.kouter + (o + 1 == p.nouter ? 0 : o + 1));
    }
  }
};

// A producer's view of one CTA tile: operand origins and row masks.
struct ProdTile {
  int64_t ox, oy;
  uint64_t mm[kMaskWords], mn[kMaskWords];
  bool fm, fn;   // interior on the m / n side
  // pull tile t's two TileInfo records into L1 (read by fetch at the tile's first step)
  static __device__ __forceinline__ void prefetch(const KParams &p, int t) {
    int mt, nt;
    tile_coords(p, t, mt, nt);
    prefetch_l1(p.tileM + mt);
    prefetch_l1(p.tileN + nt);
  }
  __device__ __forceinline__ void fetch(const KParams &p, int t) {
    int mt, nt;
    tile_coords(p, t, mt, nt);
    const TileInfo &tm = p.tileM[mt];
    const TileInfo &tn = p.tileN[nt];
    ox = tm.op;
    oy = tn.op;
    fm = fn = true;
#pragma unroll
    for (int w = 0; w < kMaskWords; w++) {
      mm[w] = tm.mask[w];
      mn[w] = tn.mask[w];
      fm &= mm[w] == p.fullM[w];
      fn &= mn[w] == p.fullN[w];
    }
  }
};

// (select, not a dynamic array index: keeps the mask in registers, no local memory)
__device__ __forceinline__ bool bit_of(const uint64_t (&m)[kMaskWords], int r) {
  static_assert(kMaskWords == 2, "bit_of");
  return ((r < 64 ? m[0] : m[1]) >> (r & 63)) & 1;
}

__device__ __forceinline__ void cp_async16_full(uint32_t dst, const double *src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(dst), "l"(src));
}
__device__ __forceinline__ void cp_async8_full(uint32_t dst, const double *src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(dst), "l"(src));
}

// Producer: issue this thread's E register-cached slots of one operand for one
// (tile, step).  Interior tile and full k-step: no bounds work at all (every slot, padding
// ones included, copies from inside the tile to its smem spot / the stage's scratch).
// Otherwise each slot tests its k bit and its row bit and zero-fills when out of range.
template <int E, bool VEC>
__device__ __forceinline__ void issue_slots(const double *__restrict__ src, uint32_t sdst,
                                            const int32_t (&rel)[E], const uint32_t (&pack)[E],
                                            int64_t base, bool fast, uint64_t kmask,
                                            const uint64_t (&rmask)[kMaskWords]) {
  const double *b = src + base;
  if (fast) {
#pragma unroll
    for (int i = 0; i < E; i++) {
      const uint32_t dst = sdst + (pack[i] & 8191) * 8;
      if (VEC) cp_async16_full(dst, b + rel[i]);
      else cp_async8_full(dst, b + rel[i]);
    }
  } else {
#pragma unroll
    for (int i = 0; i < E; i++) {
      const uint32_t pk = pack[i];
      const int k = (pk >> 13) & 63, m = pk >> 19;
      const bool ok = ((kmask >> k) & 1) && bit_of(rmask, m);
      const uint32_t dst = sdst + (pk & 8191) * 8;
      if (VEC) cp_async16(dst, ok ? b + rel[i] : src, ok ? 16 : 0);
      else cp_async8(dst, ok ? b + rel[i] : src, ok ? 8 : 0);
    }
  }
}

template <int E>
__device__ __forceinline__ void load_slots(int32_t (&rel)[E], uint32_t (&pack)[E],
                                           const int32_t *__restrict__ r, const uint32_t *__restrict__ p,
                                           int n, int first, int stride, uint32_t scratch) {
#pragma unroll
  for (int i = 0; i < E; i++) {
    const int s = first + i * stride;
    // padding slot: copies the tile origin into the stage's scratch; never in range on the
    // checked path (k = 63 is never a valid tile-local k, BK <= 24)
    rel[i] = s < n ? __ldg(r + s) : 0;
    pack[i] = s < n ? __ldg(p + s) : (scratch | (63u << 13));
  }
}

// Deferred epilogue (STG variants): drain columns [c0, c0 + NC) of the warp's parked tile.
// Lane l owns tile row wm * 32 + l (its C offset Cr, validity rok); column c of the warp
// tile is tile column n0 + c (C offset relCn, validity bit of cmask).  VC: 16-B pairs (lane
// pairs share a column: lanes 0-15 take rows 2l, 2l + 1 of column c, lanes 16-31 of c + 1).
template <int WN, int SP, int NC, bool VC>
__device__ __forceinline__ void drain_cols(const double *__restrict__ st, int c0, int lane, double *Cr, bool rok,
                                           const int64_t *relCn, int n0, const uint64_t (&cmask)[kMaskWords],
                                           double alpha, double beta, bool plain) {
  if (VC) {
#pragma unroll
    for (int d = 0; d < NC; d += 2) {
      const int c = c0 + d + (lane >> 4);
      if (c < WN && rok && bit_of(cmask, n0 + c)) {
        double2 v = *reinterpret_cast<const double2 *>(st + c * SP + 2 * (lane & 15));
        double2 *dst = reinterpret_cast<double2 *>(Cr + relCn[n0 + c]);
        if (!plain) {
          if (beta != 0.0) {
            const double2 o = *dst;
            v.x = fma(beta, o.x, alpha * v.x);
            v.y = fma(beta, o.y, alpha * v.y);
          } else {
            v.x *= alpha;
            v.y *= alpha;
          }
        }
        *dst = v;
      }
    }
  } else {
#pragma unroll
    for (int d = 0; d < NC; d++) {
      const int c = c0 + d;
      if (c < WN && rok && bit_of(cmask, n0 + c)) {
        double v = st[c * SP + lane];
        double *dst = Cr + relCn[n0 + c];
        if (!plain) v = beta != 0.0 ? fma(beta, *dst, alpha * v) : alpha * v;
        *dst = v;
      }
    }
  }
}

template <int BM, int BN, int BK, int WM, int WN, int STAGES, int PW, int MINB, bool XK, bool YK, bool STG>
__global__ void __launch_bounds__(F64Kernel<BM, BN, BK, WM, WN, STAGES, PW, STG>::THREADS, MINB)
tc_f64_dmma_kernel(const __grid_constant__ KParams p) {
  using K = F64Kernel<BM, BN, BK, WM, WN, STAGES, PW, STG>;
  using L = typename K::L;
  constexpr int MI = K::MI, NJ = K::NJ, CW = K::CWARPS;
  extern __shared__ __align__(1024) double smem[];
  double *sX = smem;                              // the cp.async ring
  double *sY = smem + STAGES * L::XS;
  uint64_t *bars = reinterpret_cast<uint64_t *>(sY + STAGES * L::YS);  // full[S], empty[S]
  int64_t *relCm = reinterpret_cast<int64_t *>(bars + 2 * STAGES);
  int64_t *relCn = relCm + BM;
  int32_t *boxM = reinterpret_cast<int32_t *>(relCn + BN);
  int32_t *boxN = boxM + BM;
  // [BM * BN] C staging box of the TMA epilogue: present only when launched with it
  double *sC = smem + K::kStagingOffset;
  // [STG] this consumer warp's deferred-epilogue staging tile
  double *stg_base = reinterpret_cast<double *>(reinterpret_cast<char *>(smem) + K::kStageOffset);

  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int ntl = (p.ntotal - (int)blockIdx.x + (int)gridDim.x - 1) / (int)gridDim.x;
  if (ntl <= 0) return;
  const int total = ntl * p.nsteps;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(smem);
  const uint32_t bar0 = (uint32_t)__cvta_generic_to_shared(bars);

  // ---- once per CTA: zero the ring (positions no slot writes must read as 0), tables,
  //      barriers ------------------------------------------------------------------------
  for (int i = tid; i < STAGES * (L::XS + L::YS); i += K::THREADS) smem[i] = 0.0;
  for (int r = tid; r < BM; r += K::THREADS) { relCm[r] = p.relCm[r]; boxM[r] = p.boxM[r]; }
  for (int r = tid; r < BN; r += K::THREADS) { relCn[r] = p.relCn[r]; boxN[r] = p.boxN[r]; }
  if (tid == 0) {
    for (int s = 0; s < STAGES; s++) {
      mbar_init(bar0 + 8 * s, PW * 32);               // full: every producer thread
      mbar_init(bar0 + 8 * (STAGES + s), CW);         // empty: one arrive per consumer warp
    }

    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();

  if (warp >= CW) {
    // ======================= producer warps ===============================================
    const int ptid = tid - CW * 32;
    const double *__restrict__ X = static_cast<const double *>(p.X);
    const double *__restrict__ Y = static_cast<const double *>(p.Y);
    int32_t rx[K::EX], ry[K::EY];
    uint32_t px[K::EX], py[K::EY];
    load_slots(rx, px, p.relX, p.packX, p.nslotX, ptid, PW * 32, L::XS - 2);
    load_slots(ry, py, p.relY, p.packY, p.nslotY, ptid, PW * 32, L::YS - 2);
    const bool vx = p.vecX == 2, vy = p.vecY == 2;
    int step = 0, lt = 0;
    // the next tile's operand origins and masks are fetched while the current tile's last
    // stage is issued (their load latency hides behind it)
    ProdTile cur;
    cur.fetch(p, (int)blockIdx.x);
    KStep ks;
    ks.reset(p);
    for (int j = 0; j < total; j++) {
      const int s = j % STAGES;
      if (j >= STAGES) mbar_wait(bar0 + 8 * (STAGES + s), ((j / STAGES) & 1) ^ 1);
      if (step + 1 == p.nsteps && lt + 1 < ntl) ProdTile::prefetch(p, (int)blockIdx.x + (lt + 1) * (int)gridDim.x);
      const int64_t ox = cur.ox, oy = cur.oy;
      const bool fm = cur.fm, fn = cur.fn;
      const uint64_t(&mm)[kMaskWords] = cur.mm;
      const uint64_t(&mn)[kMaskWords] = cur.mn;
      const uint64_t km = ks.mask(p);
      const bool fk = km == p.fullK;
      const int64_t bx = ox + ks.sx(), by = oy + ks.sy();
      const uint32_t dx = sbase + 8u * (uint32_t)(s * L::XS);
      const uint32_t dy = sbase + 8u * (uint32_t)(STAGES * L::XS + s * L::YS);
      if (vx) issue_slots<K::EX, true>(X, dx, rx, px, bx, fm && fk, km, mm);
      else issue_slots<K::EX, false>(X, dx, rx, px, bx, fm && fk, km, mm);
      if (vy) issue_slots<K::EY, true>(Y, dy, ry, py, by, fn && fk, km, mn);
      else issue_slots<K::EY, false>(Y, dy, ry, py, by, fn && fk, km, mn);
      mbar_arrive_cp_async(bar0 + 8 * s);
      if (p.pf_mstep > 0 && step == 0) {
        // beta != 0: the epilogue reads this tile's old C; pull it into L2 now (the producers
        // run STAGES k-steps ahead of the consumers' epilogue), a line per pf_mstep rows
        int mt, nt;
        tile_coords(p, (int)blockIdx.x + lt * (int)gridDim.x, mt, nt);
        const double *Ct = static_cast<const double *>(p.C) + (p.tileM[mt].c + p.tileN[nt].c);
        const int nm = (p.Mt + p.pf_mstep - 1) / p.pf_mstep;
        for (int q = ptid; q < nm * p.Nt; q += PW * 32) {
          const int n = q / nm, mi = (q - n * nm) * p.pf_mstep;
          asm volatile("prefetch.global.L2 [%0];\n" ::"l"(Ct + relCm[mi] + relCn[n]));
        }
      }
      ks.advance(p);
      if (++step == p.nsteps) {
        step = 0;
        if (++lt < ntl) cur.fetch(p, (int)blockIdx.x + lt * (int)gridDim.x);
      }
    }
    return;
  }

  // ======================= consumer warps =================================================
  double *__restrict__ C = static_cast<double *>(p.C);
  const int wm = warp % K::WARPS_M, wn = warp / K::WARPS_M;
  const int g = lane >> 2, t = lane & 3;
  // fragment offsets (compile-time layouts): A(m, k) and B(k, n)
  const int aoff = XK ? (wm * WM + g) * L::PK + t : t * L::PM + wm * WM + g;
  const int boff = YK ? (wn * WN + g) * L::PK + t : t * L::PN + wn * WN + g;
  constexpr int AI = XK ? 8 * L::PK : 8, AK = XK ? 4 : 4 * L::PM;
  constexpr int BJ = YK ? 8 * L::PK : 8, BKs = YK ? 4 : 4 * L::PN;

  double acc[MI][NJ][2];
#pragma unroll
  for (int i = 0; i < MI; i++)
#pragma unroll
    for (int jj = 0; jj < NJ; jj++) acc[i][jj][0] = acc[i][jj][1] = 0.0;

  const double alpha = p.alpha, beta = p.beta;
  // this thread's C rows are the same in every tile: their offsets live in registers
  int64_t roff[MI];
#pragma unroll
  for (int i = 0; i < MI; i++) roff[i] = relCm[wm * WM + i * 8 + g];
  // [STG] deferred epilogue state: the parked tile's C row pointer (this lane's row),
  // row validity, column mask and the next column to drain
  double *const stg = stg_base + warp * WN * K::SP;
  const bool plain = alpha == 1.0 && beta == 0.0;
  const bool vc = STG && p.vecC == 2;
  const int drow = wm * WM + (vc ? 2 * (lane & 15) : lane);   // tile row this lane drains
  const int64_t droff = STG ? relCm[drow] : 0;
  double *dCr = C;
  bool drok = false, pend = false;
  uint64_t dmn[kMaskWords] = {0, 0};
  int dcol = 0;
  // columns per k4 step so that a parked tile is drained within one k-step of the next tile
  constexpr int KQ = BK / 4;
  constexpr int DQ = ((WN + KQ - 1) / KQ + 1) / 2 * 2;
  // [STG, beta != 0] the old C of the tile being computed is fetched by cp.async into the
  // warp's staging tile as soon as the previous parked tile has drained (lane l: row l of the
  // warp tile, all WN columns; zero-filled outside C), and combined at park time
  // (alpha * acc + beta * old, from smem): the drain then only stores, and the old C's
  // latency hides behind the rest of the tile's DMMAs instead of stalling each drain step
  const bool pfc = STG && beta != 0.0;
  bool pf_issued = false, combined = false;
  auto oldc_fetch = [&](int64_t coff, const uint64_t (&tm)[kMaskWords], const uint64_t (&tn)[kMaskWords]) {
    const int r = wm * WM + lane;
    const bool rok = bit_of(tm, r);
    const double *src = C + coff + relCm[r];
    const uint32_t d0 = (uint32_t)__cvta_generic_to_shared(stg) + 8u * (uint32_t)lane;
#pragma unroll 1
    for (int c = 0; c < WN; c++) {
      const int cidx = wn * WN + c;
      const bool ok = rok && bit_of(tn, cidx);
      cp_async8(d0 + 8u * (uint32_t)(c * K::SP), ok ? src + relCn[cidx] : C, ok ? 8 : 0);
    }
  };
  auto drain = [&](int c0) {
    const bool pl = plain || combined;
    if (vc) drain_cols<WN, K::SP, DQ, true>(stg, c0, lane, dCr, drok, relCn, wn * WN, dmn, alpha, beta, pl);
    else drain_cols<WN, K::SP, DQ, false>(stg, c0, lane, dCr, drok, relCn, wn * WN, dmn, alpha, beta, pl);
  };
  // TMA epilogue: box offsets of tile-local rows / columns come from smem tables
  const bool use_tma = p.use_tma && beta == 0.0;
  const uint32_t sCaddr = (uint32_t)__cvta_generic_to_shared(sC);
  int step = 0, lt = 0;
  int64_t cm = 0, cn = 0;                          // tile origin in C (m part, n part)
  uint64_t mm[kMaskWords], mn[kMaskWords];         // tile row / column masks
  int32_t crd[kMaxTmaDims];                        // tile origin coordinates (TMA)
  for (int j = 0; j < total; j++) {
    const int s = j % STAGES;
    if (step == 0) {
      // tile info for this tile's epilogue, loaded now and first USED in the epilogue, so
      // the load latency hides behind the mainloop
      int mt, nt;
      tile_coords(p, (int)blockIdx.x + lt * (int)gridDim.x, mt, nt);
      const TileInfo &tm = p.tileM[mt];
      const TileInfo &tn = p.tileN[nt];
      cm = tm.c;
      cn = tn.c;
#pragma unroll
      for (int w = 0; w < kMaskWords; w++) { mm[w] = tm.mask[w]; mn[w] = tn.mask[w]; }
#pragma unroll
      for (int d = 0; d < kMaxTmaDims; d++) crd[d] = tm.coord[d] + tn.coord[d];
    }
    mbar_wait(bar0 + 8 * s, (j / STAGES) & 1);
    const double *xs = sX + s * L::XS + aoff;
    const double *ys = sY + s * L::YS + boff;
#pragma unroll
    for (int kk = 0; kk < BK / 4; kk++) {
      double a[MI], b[NJ];
#pragma unroll
      for (int i = 0; i < MI; i++) a[i] = xs[i * AI + kk * AK];
#pragma unroll
      for (int jj = 0; jj < NJ; jj++) b[jj] = ys[jj * BJ + kk * BKs];
#pragma unroll
      for (int i = 0; i < MI; i++)
#pragma unroll
        for (int jj = 0; jj < NJ; jj++) dmma884(acc[i][jj][0], acc[i][jj][1], a[i], b[jj]);
      // [STG] a few columns of the parked tile per k4 step, in the shadow of the DMMAs
      // (twice as many with beta != 0, so the old-C fetch of this tile starts early)
      if (STG && pend && dcol < WN) {
        drain(dcol);
        dcol += DQ;
        if (pfc && dcol < WN) {
          drain(dcol);
          dcol += DQ;
        }
      }
      if (pfc && !pf_issued && (!pend || dcol >= WN)) {
        __syncwarp();   // every lane's drain reads of the staging tile are done
        oldc_fetch(cm + cn, mm, mn);
        pf_issued = true;
      }
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(bar0 + 8 * (STAGES + s));
    if (++step == p.nsteps) {
      // ---- epilogue of tile lt: C = alpha * acc + beta * C (beta == 0: C not read) --------
      uint32_t rbits = 0;
#pragma unroll
      for (int i = 0; i < MI; i++) rbits |= (uint32_t)bit_of(mm, wm * WM + i * 8 + g) << i;
      double *Ct = C + (cm + cn);
      if (STG) {
        // finish the previous parked tile, then park this one (raw accumulators; the drain
        // applies alpha / beta) and record where it goes
        if (pend) {
          for (; dcol < WN; dcol += DQ) drain(dcol);
        }
        if (pfc && !pf_issued) {   // (a tile too short to fetch its old C ahead)
          __syncwarp();
          oldc_fetch(cm + cn, mm, mn);
        }
        if (pfc) asm volatile("cp.async.wait_all;\n" ::: "memory");
        __syncwarp();
#pragma unroll
        for (int jj = 0; jj < NJ; jj++)
#pragma unroll
          for (int h = 0; h < 2; h++) {
            double *col = stg + (jj * 8 + 2 * t + h) * K::SP + g;
#pragma unroll
            for (int i = 0; i < MI; i++) col[i * 8] = pfc ? fma(beta, col[i * 8], alpha * acc[i][jj][h]) : acc[i][jj][h];
          }
        __syncwarp();
        combined = pfc;
        pf_issued = false;
        dCr = Ct + droff;
        drok = bit_of(mm, drow);
        dmn[0] = mn[0];
        dmn[1] = mn[1];
        pend = true;
        dcol = 0;
        (void)rbits;      } else if (use_tma) {
        // stage alpha * acc as the tile's box in smem, one elected thread TMA-stores it;
        // the hardware clips the box at the tensor bounds
        if (threadIdx.x == 0) tma_wait_read();     // previous tile's store has read sC
        consumer_sync(CW * 32);
#pragma unroll
        for (int jj = 0; jj < NJ; jj++)
#pragma unroll
          for (int h = 0; h < 2; h++) {
            const int cidx = wn * WN + jj * 8 + 2 * t + h;
            if (cidx < p.Nt) {
              double *col = sC + boxN[cidx];
#pragma unroll
              for (int i = 0; i < MI; i++) {
                const int r = wm * WM + i * 8 + g;
                if (r < p.Mt) col[boxM[r]] = alpha * acc[i][jj][h];
              }
            }
          }
        fence_proxy_async();
        consumer_sync(CW * 32);
        if (threadIdx.x == 0) tma_store(&p.cmap, p.c_rank, crd, sCaddr);
      } else if (beta == 0.0) {
        // predicated stores (no branches); alpha == 1 skips the FP64-pipe multiply
        if (alpha != 1.0) {
#pragma unroll
          for (int i = 0; i < MI; i++)
#pragma unroll
            for (int jj = 0; jj < NJ; jj++) {
              acc[i][jj][0] *= alpha;
              acc[i][jj][1] *= alpha;
            }
        }
#pragma unroll
        for (int jj = 0; jj < NJ; jj++)
#pragma unroll
          for (int h = 0; h < 2; h++) {
            const int cidx = wn * WN + jj * 8 + 2 * t + h;
            const uint32_t ok = bit_of(mn, cidx) ? rbits : 0u;
            double *col = Ct + relCn[cidx];
#pragma unroll
            for (int i = 0; i < MI; i++) st_pred(col + roff[i], acc[i][jj][h], (ok >> i) & 1);
          }
      } else {
#pragma unroll
        for (int jj = 0; jj < NJ; jj++)
#pragma unroll
          for (int h = 0; h < 2; h++) {
            const int cidx = wn * WN + jj * 8 + 2 * t + h;
            const uint32_t ok = bit_of(mn, cidx) ? rbits : 0u;
            double *col = Ct + relCn[cidx];
#pragma unroll
            for (int i = 0; i < MI; i++)
              if ((ok >> i) & 1) col[roff[i]] = fma(beta, col[roff[i]], alpha * acc[i][jj][h]);
          }
      }
#pragma unroll
      for (int i = 0; i < MI; i++)
#pragma unroll
        for (int jj = 0; jj < NJ; jj++) acc[i][jj][0] = acc[i][jj][1] = 0.0;
      step = 0;
      ++lt;
    }
  }
  if (STG && pend) {
    for (; dcol < WN; dcol += DQ) drain(dcol);
  }
  if (use_tma && threadIdx.x == 0) tma_wait_all();   // the last box must be read out
}

}  // namespace tc
