// kernel_bf16.cuh — the BF16 direct-contraction kernel of libtc on the 5th-generation tensor
// cores (tcgen05 + TMEM), sm_100a.
//
// Same four steps as the FP64 kernel, mapped onto Blackwell's async MMA:
//   (1) producer warps gather the X tile (128 x 64) and the Y tile (BN x 64) of each k-step
//       with cp.async in each operand's own memory order straight into the
//       UMMA canonical no-swizzle layout (8 x 16-B core matrices; K- or MN-major per operand,
//       chosen from the operand's FVI, so the smem write side stays coalesced);
//   (2)+(3) one elected thread of the MMA warp issues tcgen05.mma.kind::f16 (BF16 x BF16 ->
//       FP32, M = 128, N = BN, K = 16) from smem descriptors into a TMEM accumulator;
//       tcgen05.commit releases each smem stage and, per tile, hands the accumulator over;
//   (4) eight epilogue warps drain TMEM (tcgen05.ld 32x32b: warp w owns lanes
//       32(w%4)..+31 = tile rows, and column half w/4) and store C = alpha * acc + beta * C
//       in FP32, rounded to BF16 (RNE), through the separable row / column offsets,
//       predicated by the tile masks.
// The TMEM accumulator is double-buffered (2 x BN columns) so the epilogue of tile i
// overlaps the MMAs of tile i+1; CTAs are persistent like the FP64 kernel.
#pragma once
#include <cuda_bf16.h>
#include <cstdint>
#include <type_traits>

#include "kernel_f64.cuh"   // cp.async / mbarrier helpers, tile_coords, bit_of
#include "kparams.hpp"

namespace tc {

__device__ __forceinline__ void cp_async4(uint32_t dst, const void *src, int srcbytes) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;\n" ::"r"(dst), "l"(src), "r"(srcbytes));
}
__device__ __forceinline__ void cp_async8v(uint32_t dst, const void *src, int srcbytes) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(dst), "l"(src), "r"(srcbytes));
}
__device__ __forceinline__ void cp_async16v(uint32_t dst, const void *src, int srcbytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(dst), "l"(src), "r"(srcbytes));
}
__device__ __forceinline__ void tc05_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory"); }
__device__ __forceinline__ void tc05_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory"); }
__device__ __forceinline__ void tc05_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"r"(bar)
               : "memory");
}
template <bool TF32>
__device__ __forceinline__ void tc05_mma(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                         uint32_t accumulate) {
  if constexpr (TF32)
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate) : "memory");
  else
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate) : "memory");
}
// CTA pair (cta_group::2, cluster of 2 on one TPC): the leader (rank 0) issues M = 256 MMAs
// reading each CTA's half of A (its 128 rows) and of B (its N/2 columns) from the same smem
// offsets; D rows 128 r.. land in CTA r's TMEM.
template <bool TF32>
__device__ __forceinline__ void tc05_mma2(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                          uint32_t accumulate) {
  if constexpr (TF32)
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::tf32 [%0], %1, %2, %3, p;\n}\n" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate) : "memory");
  else
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate) : "memory");
}
// completion of the leader's MMAs arrives at the barrier at this offset in BOTH CTAs
__device__ __forceinline__ void tc05_commit2(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;\n"
               ::"r"(bar), "h"((uint16_t)3) : "memory");
}
__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;\n" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;\n" ::: "memory");
}
// arrive (release, cluster scope) on the barrier at this offset in CTA `cta` of the cluster
__device__ __forceinline__ void mbar_arrive_cta(uint32_t bar, uint32_t cta) {
  asm volatile(
      "{\n\t.reg .b32 ra;\n\tmapa.shared::cluster.u32 ra, %0, %1;\n\t"
      "mbarrier.arrive.release.cluster.shared::cluster.b64 _, [ra];\n}\n" ::"r"(bar), "r"(cta) : "memory");
}
__device__ __forceinline__ void mbar_wait_acq_cluster(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAITC_%=:\n\t"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAITC_%=;\n}\n" ::"r"(bar), "r"(parity) : "memory");
}
// TMA box of a CTA pair: lands in this CTA's smem, completes on the LEADER's barrier (the
// barrier offset with the peer bit cleared)
__device__ __forceinline__ void tma_load_pair(const TmaDesc *map, int rank, int32_t c0, int32_t c1, int32_t c2,
                                              int32_t c3, int32_t c4, uint32_t dst, uint32_t bar, uint64_t pol) {
  const uint64_t m = reinterpret_cast<uint64_t>(map);
  bar &= 0xFEFFFFFFu;
  switch (rank) {
    case 1:
      asm volatile("cp.async.bulk.tensor.1d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
                   " [%0], [%1, {%2}], [%3], %4;\n" ::"r"(dst), "l"(m), "r"(c0), "r"(bar), "l"(pol) : "memory");
      break;
    case 2:
      asm volatile("cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
                   " [%0], [%1, {%2, %3}], [%4], %5;\n" ::"r"(dst), "l"(m), "r"(c0), "r"(c1), "r"(bar), "l"(pol)
                   : "memory");
      break;
    case 3:
      asm volatile("cp.async.bulk.tensor.3d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
                   " [%0], [%1, {%2, %3, %4}], [%5], %6;\n" ::"r"(dst), "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(bar),
                   "l"(pol) : "memory");
      break;
    case 4:
      asm volatile("cp.async.bulk.tensor.4d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
                   " [%0], [%1, {%2, %3, %4, %5}], [%6], %7;\n" ::"r"(dst), "l"(m), "r"(c0), "r"(c1), "r"(c2), "r"(c3),
                   "r"(bar), "l"(pol) : "memory");
      break;
    default:
      asm volatile("cp.async.bulk.tensor.5d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
                   " [%0], [%1, {%2, %3, %4, %5, %6}], [%7], %8;\n" ::"r"(dst), "l"(m), "r"(c0), "r"(c1), "r"(c2),
                   "r"(c3), "r"(c4), "r"(bar), "l"(pol) : "memory");
      break;
  }
}
// pair unit u -> (pm, pn) over the grid of 2 x 2 tile blocks, rasterised like tile_coords
__device__ __forceinline__ void pair_coords(const KParams &p, int u, int &pm, int &pn) {
  const int pmt = (p.mtiles + 1) >> 1, pnt = (p.ntiles + 1) >> 1;
  const int gm = max(1, p.group_m >> 1);
  const int per_group = gm * pnt;
  const int g = u / per_group;
  const int first = g * gm;
  const int gsz = min(gm, pmt - first);
  const int r = u - g * per_group;
  pm = first + r % gsz;
  pn = r / gsz;
}

__device__ __forceinline__ void tc05_ld16(uint32_t taddr, uint32_t (&v)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];\n"
      "tcgen05.wait::ld.sync.aligned;\n"   // same statement: no use of v can move above it
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
        "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
      : "r"(taddr)
      : "memory");
}

__device__ __forceinline__ void cp_async16v_full(uint32_t dst, const void *src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(dst), "l"(src));
}
__device__ __forceinline__ void cp_async8v_full(uint32_t dst, const void *src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(dst), "l"(src));
}

// Register-cached slots (4- or 8-element vectors): this thread's slots first + i * 128 of
// one operand; `cnt` of the E entries are real.  Interior tile and full k-step: no bounds
// work; otherwise each slot tests its k bit and its row bit and zero-fills.
template <int E, int ES>
__device__ __forceinline__ void umma_load_slots(int32_t (&rel)[E], uint32_t (&soff)[E], const int32_t *__restrict__ r,
                                                const uint32_t *__restrict__ pk, int n, int first, int stride) {
#pragma unroll
  for (int i = 0; i < E; i++) {
    const int q = first + i * stride;
    rel[i] = q < n ? __ldg(r + q) : 0;
    soff[i] = q < n ? (uint32_t)ES * (__ldg(pk + q) & 0x3FFF) : 0u;   // smem byte offset in the stage
  }
}

// One operand, one (tile, step): this thread's `cnt` cached 16-B slots.  Interior tile and
// full k-step (fast): straight copies.  Otherwise each slot re-reads its packed (k, row) from
// the slot table, tests the step's k mask and the tile's row mask and zero-fills.
template <int E, typename T>
__device__ __forceinline__ void umma_issue(const T *__restrict__ src, uint32_t sdst,
                                           const int32_t (&rel)[E], const uint32_t (&soff)[E], int cnt,
                                           int64_t base, bool fast, uint64_t kmask, const uint64_t (&rmask)[kMaskWords],
                                           const uint32_t *__restrict__ pack, int first, int stride) {
  const T *b = src + base;
  if (fast) {
#pragma unroll
    for (int i = 0; i < E; i++)
      if (i < cnt) cp_async16v_full(sdst + soff[i], b + rel[i]);
  } else {
#pragma unroll
    for (int i = 0; i < E; i++) {
      if (i < cnt) {
        const uint32_t pk = __ldg(pack + first + i * stride);
        const int k = (pk >> 14) & 63, m = pk >> 20;
        const bool ok = ((kmask >> k) & 1) && bit_of(rmask, m);
        cp_async16v(sdst + soff[i], ok ? b + rel[i] : src, ok ? 16 : 0);
      }
    }
  }
}

// Generic producer path (any vector width, slot tables read from global memory): every slot
// tests its k bit and its row bit and zero-fills when out of range.
template <int PW, typename T>
__device__ __forceinline__ void umma_issue_generic_t(const KParams &p, const T *__restrict__ X,
                                                     const T *__restrict__ Y, int pt, uint32_t dx,
                                                     uint32_t dy, int64_t bx, int64_t by, uint64_t km,
                                                     const uint64_t (&mm)[kMaskWords],
                                                     const uint64_t (&mn)[kMaskWords]) {
  for (int side = 0; side < 2; side++) {
    const T *src = side ? Y : X;
    const int32_t *rel = side ? p.relY : p.relX;
    const uint32_t *pack = side ? p.packY : p.packX;
    const int n = side ? p.nslotY : p.nslotX, vec = side ? p.vecY : p.vecX;
    const int64_t base = side ? by : bx;
    const uint32_t dst0 = side ? dy : dx;
    const uint64_t *rm = side ? mn : mm;
    if (vec * (int)sizeof(T) == 2) {
      // single BF16 elements (cp.async has no 2-byte form): 8 independent loads in flight per
      // thread, then their stores — a load-store chain per element would serialise the
      // global latency (the TCCG #14 / #27 layouts: k digits in opposite orders in X and Y)
      constexpr int U = 8;
      for (int q0 = pt; q0 < n; q0 += U * PW * 32) {
        unsigned short v[U];
        uint32_t d[U];
#pragma unroll
        for (int i = 0; i < U; i++) {
          const int q = q0 + i * PW * 32;
          v[i] = 0;
          d[i] = 0xFFFFFFFFu;
          if (q < n) {
            const uint32_t pk = __ldg(pack + q);
            const int k = (pk >> 14) & 63, m = pk >> 20;
            const bool ok = ((km >> k) & 1) && ((((m < 64) ? rm[0] : rm[1]) >> (m & 63)) & 1);
            d[i] = dst0 + (uint32_t)sizeof(T) * (pk & 0x3FFF);
            if (ok) v[i] = __ldg(reinterpret_cast<const unsigned short *>(src + (base + __ldg(rel + q))));
          }
        }
#pragma unroll
        for (int i = 0; i < U; i++)
          if (d[i] != 0xFFFFFFFFu) asm volatile("st.shared.u16 [%0], %1;\n" ::"r"(d[i]), "h"(v[i]) : "memory");
      }
      continue;
    }
    for (int q = pt; q < n; q += PW * 32) {
      const uint32_t pk = __ldg(pack + q);
      const int k = (pk >> 14) & 63, m = pk >> 20;
      const bool ok = ((km >> k) & 1) && ((((m < 64) ? rm[0] : rm[1]) >> (m & 63)) & 1);
      const T *g = ok ? src + (base + __ldg(rel + q)) : src;
      const uint32_t d = dst0 + (uint32_t)sizeof(T) * (pk & 0x3FFF);
      const int bytes = vec * (int)sizeof(T);
      if (bytes == 16) cp_async16v(d, g, ok ? 16 : 0);
      else if (bytes == 8) cp_async8v(d, g, ok ? 8 : 0);
      else if (bytes == 4) cp_async4(d, g, ok ? 4 : 0);
      else {   // single elements: plain load / store (cp.async has no 2-byte form)
        const unsigned short v = ok ? *reinterpret_cast<const unsigned short *>(g) : (unsigned short)0;
        asm volatile("st.shared.u16 [%0], %1;\n" ::"r"(d), "h"(v) : "memory");
      }
    }
  }
}

// tcgen05.ld 32x32b: W consecutive accumulator columns of this thread's TMEM lane.
template <int W>
__device__ __forceinline__ void tc05_ld(uint32_t taddr, uint32_t (&v)[W]) {
  static_assert(W == 16 || W == 32, "tc05_ld width");
  if constexpr (W == 16) {
    tc05_ld16(taddr, v);
  } else {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];\n"
        "tcgen05.wait::ld.sync.aligned;\n"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),
          "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),
          "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
        : "r"(taddr)
        : "memory");
  }
}

// UMMA shared-memory descriptor, 128-B swizzle (SM100 layout: start>>4 [0,14), LBO>>4
// [16,30), SBO>>4 [32,46), version 1 [46,48), base offset 0 [49,52), layout type
// SWIZZLE_128B = 2 [61,64)).
// MN-major FP32 (TF32) operands use SWIZZLE_128B_BASE32B = 1 instead: 4-row x 128-B atoms
// whose 32-B granules are XORed with the row (CUTLASS Layout_MN_SW128_32B_Atom).
template <int LAYOUT = 2>
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
         ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46) | ((uint64_t)LAYOUT << 61);
}

// KIND (tiles.hpp): 1 = BF16 (kind::f16), 2 = TF32 on FP32 storage (kind::tf32),
// 3 = FP32 as split TF32: SW split warps rewrite each landed stage as hi = tf32 truncation
// (in place) and lo = x - hi (a second plane), and the MMA warp issues hi*hi + hi*lo + lo*hi.
// STAGED = false (CTA-pair instances): no per-epilogue-warp FP32 staging in smem — the
// epilogue stores straight from TMEM rows (C's FVI leads m), which buys a sixth stage.
template <int KIND, int BN, int STAGES, bool STAGED = true>
struct UmmaKernel {
  using T = typename std::conditional<KIND == 1, __nv_bfloat16, float>::type;
  static constexpr int ES = KIND == 1 ? 2 : 4;       // element bytes
  static constexpr bool SPLIT = KIND == 3;
  static constexpr int BM = 128, BK = 128 / ES;      // one UMMA M = 128; 128-B k rows
  static constexpr int KI = 32 / ES;                 // K per MMA instruction (f16: 16, tf32: 8)
  static constexpr int EW = 8;                       // epilogue warps
  // producer warps: their cp.async issue is the stage's critical path (tools/trace_umma.py);
  // 8 instead of 4 measured +43 % on BF16 ab-ac-cb and +15 % on the memory-bound BF16 suite
  // (12 spill in the epilogue)
  // (17 warps: 5 on one SM sub-partition cap the registers at 96; 16-warp splits with 7 or 3
  // producers measured worse for FP32)
  static constexpr int PW = SPLIT ? 4 : 8;
  static constexpr int SW = SPLIT ? 4 : 0;           // split warps (3 measured -10 %)
  static constexpr int THREADS = (EW + PW + 1 + SW) * 32; // + one MMA warp
  static constexpr int XS = BM * BK, YS = BN * BK;   // elements per stage plane (1 KB multiples)
  static constexpr int PLANES = SPLIT ? 2 : 1;       // hi (in place) + lo
  static constexpr int NBUF = 512 / BN;              // FP32 accumulators in flight (all of TMEM)
  static constexpr int TMEM_COLS = NBUF * BN;
  static constexpr size_t smem_bytes() {
    return 1024 + (size_t)ES * PLANES * STAGES * (XS + YS) + 8 * (3 * STAGES + 2 * NBUF) + 16 +
           8 * (size_t)(BM + BN) + 16 + (STAGED ? 4 * (size_t)EW * 32 * 32 : 0);   // + per-epilogue-warp FP32 staging (32 x 32)
  }
  // register-cached slots per producer thread (16-B vectors)
  static constexpr int EX = (BM * BK * ES / 16 + PW * 32 - 1) / (PW * 32);
  static constexpr int EY = (BN * BK * ES / 16 + PW * 32 - 1) / (PW * 32);
  static_assert(BN % 32 == 0 && BN <= 128, "BN");
  static_assert(TMEM_COLS >= 32 && (TMEM_COLS & (TMEM_COLS - 1)) == 0, "TMEM allocation");
  static_assert(smem_bytes() <= 232448, "smem");
};

// UMMA instruction descriptor: BF16 x BF16 or TF32 x TF32 -> F32 (c_format 1 at [4,6),
// a/b_format at [7,10) / [10,13): BF16 = 1, TF32 = 2), M = 128, N = BN, majors per operand.
__host__ __device__ constexpr uint32_t umma_idesc(int fmt, int n, bool a_mn, bool b_mn, int m = 128) {
  return (1u << 4) | ((uint32_t)fmt << 7) | ((uint32_t)fmt << 10) | ((uint32_t)a_mn << 15) |
         ((uint32_t)b_mn << 16) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(m >> 4) << 24);
}

__device__ __forceinline__ void st_out(__nv_bfloat16 *d, float v) { *d = __float2bfloat16_rn(v); }
__device__ __forceinline__ void st_out(float *d, float v) { *d = v; }
__device__ __forceinline__ float ld_out(const __nv_bfloat16 *d) { return __bfloat162float(*d); }
__device__ __forceinline__ float ld_out(const float *d) { return *d; }

// 8 consecutive C elements (16-B aligned): C = x + beta * C (x already scaled by alpha)
__device__ __forceinline__ void store_run8(float *dst, float (&x)[8], float beta) {
  float4 *d = reinterpret_cast<float4 *>(dst);
  if (beta != 0.0f) {
    const float4 o0 = d[0], o1 = d[1];
    x[0] = fmaf(beta, o0.x, x[0]); x[1] = fmaf(beta, o0.y, x[1]); x[2] = fmaf(beta, o0.z, x[2]);
    x[3] = fmaf(beta, o0.w, x[3]); x[4] = fmaf(beta, o1.x, x[4]); x[5] = fmaf(beta, o1.y, x[5]);
    x[6] = fmaf(beta, o1.z, x[6]); x[7] = fmaf(beta, o1.w, x[7]);
  }
  d[0] = make_float4(x[0], x[1], x[2], x[3]);
  d[1] = make_float4(x[4], x[5], x[6], x[7]);
}
__device__ __forceinline__ void store_run8(__nv_bfloat16 *dst, float (&x)[8], float beta) {
  uint4 *d = reinterpret_cast<uint4 *>(dst);
  if (beta != 0.0f) {
    const uint4 o = *d;
    const uint32_t ow[4] = {o.x, o.y, o.z, o.w};
#pragma unroll
    for (int j = 0; j < 4; j++) {
      x[2 * j] = fmaf(beta, __uint_as_float(ow[j] << 16), x[2 * j]);
      x[2 * j + 1] = fmaf(beta, __uint_as_float(ow[j] & 0xFFFF0000u), x[2 * j + 1]);
    }
  }
  uint32_t w[4];
#pragma unroll
  for (int j = 0; j < 4; j++) {
    const __nv_bfloat162 b2 = __floats2bfloat162_rn(x[2 * j], x[2 * j + 1]);
    w[j] = *reinterpret_cast<const uint32_t *>(&b2);
  }
  *d = make_uint4(w[0], w[1], w[2], w[3]);
}

// Development trace: CTA 0 records clock64() at the hand-off points of the first 1024 stages
// / tiles into the C buffer (which then holds no result): [0..) producer warp 0 after its
// EMPTY wait, [1024..) after its FULL arrive, [2048..) MMA after its FULL wait, [3072..) MMA
// after its commits, [4096..) epilogue warp 0 after TFULL, [5120..) after TEMPTY, [6144..)
// producer warp 0 at the loop top, [7168..) after its tile switch.  Compiled in only in a
// -DTC_TRACE side build (tools/trace_umma.py); the shipped library has no trace code.
#ifdef TC_TRACE
constexpr bool kTrace = true;
#else
constexpr bool kTrace = false;
#endif
__device__ __forceinline__ void trace_at(const KParams &p, int slot, int j) {
  if (kTrace && blockIdx.x == 0 && j < 1024)
    static_cast<unsigned long long *>(p.C)[slot * 1024 + j] = clock64();
}

// The boxes of one operand for (tile, k-step): coordinate per map dim = the tile origin along
// its C position (TileInfo::coord) or the k-step origin; nsub boxes along map dim 0.
// umma_box_origin resolves the per-dim sources once per tile (registers: a global read per
// k-step would put its latency on every stage); umma_tma_boxes issues one k-step.
struct UmmaBox {
  int32_t c[kMaxTmaDims];   // tile origin per map dim (0 at the k dim)
  uint32_t kmask;           // bit j: map dim j is the k index
};
__device__ __forceinline__ void umma_box_origin(const TmaOperand &o, const int32_t (&coord)[kMaxTmaDims], UmmaBox &b) {
  b.kmask = 0;
#pragma unroll
  for (int j = 0; j < kMaxTmaDims; j++) {
    const uint32_t src = (o.pack >> (3 * j)) & 7;
    int32_t v = 0;
#pragma unroll
    for (int q = 0; q < kMaxTmaDims; q++) v = src == (uint32_t)q ? coord[q] : v;   // (select: registers)
    b.c[j] = v;
    b.kmask |= (src == 7 ? 1u : 0u) << j;
  }
}
template <bool PAIR>
__device__ __forceinline__ void umma_tma_boxes(const TmaDesc *map, const TmaOperand &o, const UmmaBox &b, int rank,
                                               int32_t kc, uint32_t dst, uint32_t bar, uint64_t pol) {
  int32_t c[kMaxTmaDims];
#pragma unroll
  for (int j = 0; j < kMaxTmaDims; j++) c[j] = (b.kmask >> j) & 1 ? kc : b.c[j];
  for (int q = 0; q < o.nsub; q++) {
    if (PAIR) tma_load_pair(map, rank, c[0], c[1], c[2], c[3], c[4], dst + (uint32_t)(q * o.sub_bytes), bar, pol);
    else tma_load(map, rank, c[0], c[1], c[2], c[3], c[4], dst + (uint32_t)(q * o.sub_bytes), bar, pol);
    c[0] += o.sub_crd;
  }
}
__device__ __forceinline__ void load_coord(const TileInfo *t, int32_t (&c)[kMaxTmaDims]) {
#pragma unroll
  for (int q = 0; q < kMaxTmaDims; q++) c[q] = t->coord[q];
}

// PAIR (with TMA): a cluster of two CTAs computes a 2 x 2 block of the plan's tiles as one
// 256 x 2BN accumulator pair: CTA r loads the X box of m-tile 2 pm + r and the Y box of n-tile
// 2 pn + r, the leader's MMAs (M = 256, N = 2 BN) read both CTAs' planes, and CTA r's epilogue
// drains m-tile 2 pm + r against n-tiles 2 pn and 2 pn + 1 (TMEM columns 0 / BN of the
// buffer).  Per k-step each CTA then loads half the operand bytes per MMA of the single-CTA
// kernel (the L2 -> SM traffic that bounds BF16 GEMM-like plans).  A block past the tile grid
// reads the tables' padding entry (coordinates out of the tensor: TMA zero-fills; masks 0).
// OUTF32 (BF16 operands only): C is FP32 — the accumulator is stored without the BF16
// rounding (split-K partials that are summed before the final rounding, dist.py).
template <int KIND, int BN, int STAGES, bool XK, bool YK, bool TMA = false, bool PAIR = false, bool OUTF32 = false>
__global__ void __launch_bounds__(UmmaKernel<KIND, BN, STAGES, !PAIR>::THREADS, 1)
tc_umma_kernel(const __grid_constant__ KParams p) {
  using K = UmmaKernel<KIND, BN, STAGES, !PAIR>;
  using TC = typename std::conditional<OUTF32, float, typename K::T>::type;   // C's element type
  static_assert(!PAIR || (TMA && !K::SPLIT), "CTA pairs take TMA operands, BF16 / TF32");
  constexpr int ACCW = PAIR ? 2 * BN : BN;            // accumulator columns per tile (unit)
  constexpr int NBUF = 512 / ACCW;                    // accumulators in flight
  constexpr int NSUB = PAIR ? 2 : 1;                  // tiles per unit in this CTA's epilogue
  using T = typename K::T;
  constexpr int BM = K::BM, BK = K::BK, ES = K::ES;
  extern __shared__ __align__(1024) unsigned char smem_dyn[];
  // the 128-B swizzle atoms (8 rows x 128 B) must sit on 1 KB boundaries
  unsigned char *smem_raw =
      smem_dyn + ((1024u - ((uint32_t)__cvta_generic_to_shared(smem_dyn) & 1023u)) & 1023u);
  // stage planes: [X hi | Y hi] x STAGES, then (SPLIT) the lo planes at + LO bytes
  T *sX = reinterpret_cast<T *>(smem_raw);
  T *sY = sX + STAGES * K::XS;
  constexpr uint32_t LO = (uint32_t)ES * STAGES * (K::XS + K::YS);
  // full, empty, tfull[NBUF], tempty[NBUF], split[STAGES]
  // [EW][32 columns][32 rows] FP32 epilogue staging right after the planes (1 KB aligned),
  // then the barriers and tables
  float *stage = reinterpret_cast<float *>(smem_raw + (size_t)LO * K::PLANES);
  uint64_t *bars = reinterpret_cast<uint64_t *>(stage + (PAIR ? 0 : K::EW * 32 * 32));
  uint32_t *tmem_holder = reinterpret_cast<uint32_t *>(bars + 3 * STAGES + 2 * K::NBUF);
  int64_t *relCm = reinterpret_cast<int64_t *>(tmem_holder + 4);
  int64_t *relCn = relCm + BM;


  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  // work units: tiles, or (PAIR) 2 x 2 tile blocks per cluster
  const int crank = PAIR ? (int)cluster_rank() : 0;
  const int cid = PAIR ? (int)blockIdx.x >> 1 : (int)blockIdx.x;
  const int ncl = PAIR ? (int)gridDim.x >> 1 : (int)gridDim.x;
  const int nunits = PAIR ? ((p.mtiles + 1) >> 1) * ((p.ntiles + 1) >> 1) : p.ntotal;
  const int ntl = (nunits - cid + ncl - 1) / ncl;
  const int total = max(ntl, 0) * p.nsteps;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(smem_raw);
  const uint32_t bar0 = (uint32_t)__cvta_generic_to_shared(bars);
  const uint32_t FULL = bar0, EMPTY = bar0 + 8 * STAGES, TFULL = bar0 + 16 * STAGES,
                 TEMPTY = TFULL + 8 * NBUF, SPLITB = TEMPTY + 8 * NBUF;

  // ---- once per CTA ------------------------------------------------------------------------
  for (int i = tid; i < (int)(LO * K::PLANES / 16); i += K::THREADS)
    reinterpret_cast<uint4 *>(smem_raw)[i] = make_uint4(0, 0, 0, 0);
  for (int r = tid; r < BM; r += K::THREADS) relCm[r] = p.relCm[r];
  for (int r = tid; r < BN; r += K::THREADS) relCn[r] = p.relCn[r];
  if (tid == 0) {
    for (int s = 0; s < STAGES; s++) {
      mbar_init(FULL + 8 * s, TMA ? 1 : K::PW * 32);   // the TMA thread / every producer thread
      mbar_init(EMPTY + 8 * s, 1);           // tcgen05.commit of the MMA thread
    }
    for (int b = 0; b < NBUF; b++) {
      mbar_init(TFULL + 8 * b, 1);           // tcgen05.commit after a tile's last MMA
      mbar_init(TEMPTY + 8 * b, NSUB * K::EW);   // one arrive per epilogue warp (of both CTAs)
    }
    for (int s = 0; s < STAGES; s++) mbar_init(SPLITB + 8 * s, K::SW > 0 ? K::SW : 1);   // split warps
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  if (warp == K::EW + K::PW) {               // the MMA warp owns the TMEM allocation
    if (PAIR) {   // (both CTAs, same warp)
      asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(
                       (uint32_t)__cvta_generic_to_shared(tmem_holder)),
                   "r"(K::TMEM_COLS));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;\n" ::);
    } else {
      asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(
                       (uint32_t)__cvta_generic_to_shared(tmem_holder)),
                   "r"(K::TMEM_COLS));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n" ::);
    }
  }
  tc05_fence_before();
  if (PAIR) cluster_sync_all();   // the peer's boxes / arrivals target the leader's barriers
  else __syncthreads();
  tc05_fence_after();
  const uint32_t tmem = *tmem_holder;

  if (TMA && warp >= K::EW && warp < K::EW + K::PW) {
    // ======================= TMA producer: one elected thread =============================
    // per stage: the boxes of X and Y land straight in the 128-B swizzled UMMA planes
    // (K-major: rows of BK k; MN-major: 64-element atoms, the k groups adjacent), completing
    // the stage's FULL barrier by their byte count; the other producer threads idle
    if (tid == K::EW * 32) {
      uint64_t policy;
#if defined(TC_UMMA_TMA_POL) && TC_UMMA_TMA_POL == 0
      asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;\n" : "=l"(policy));
#elif defined(TC_UMMA_TMA_POL) && TC_UMMA_TMA_POL == 2
      asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;\n" : "=l"(policy));
#else
      asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;\n" : "=l"(policy));
#endif
      const uint32_t tx = (uint32_t)(p.xt.nsub * p.xt.tx + p.yt.nsub * p.yt.tx) * (PAIR ? 2u : 1u);
      const int rx = (int)((p.xt.pack >> 16) & 7), ry = (int)((p.yt.pack >> 16) & 7);
      int step = 0, lt = 0, mt = 0, nt = 0;
      UmmaBox bx, by;
      int32_t nxc[kMaxTmaDims], nyc[kMaxTmaDims];   // the next unit's origins, read one unit ahead
      auto unit = [&](int u) {
        if (PAIR) {
          int pm, pn;
          pair_coords(p, u, pm, pn);
          mt = 2 * pm + crank;
          nt = 2 * pn + crank;
        } else {
          tile_coords(p, u, mt, nt);
        }
        load_coord(&p.tileM[mt], nxc);
        load_coord(&p.tileN[nt], nyc);
      };
      if (ntl > 0) {
        unit(cid);
        umma_box_origin(p.xt, nxc, bx);
        umma_box_origin(p.yt, nyc, by);
        if (ntl > 1) unit(cid + ncl);
      }
      for (int j = 0; j < total; j++) {
        const int s = j % STAGES;
        if (j >= STAGES) mbar_wait(EMPTY + 8 * s, ((j / STAGES) & 1) ^ 1);
        if (!PAIR || crank == 0) mbar_expect_tx(FULL + 8 * s, tx);   // (pair: both CTAs' bytes)
        const uint32_t dx = sbase + (uint32_t)ES * (uint32_t)(s * K::XS);
        const uint32_t dy = sbase + (uint32_t)ES * (uint32_t)(STAGES * K::XS + s * K::YS);
        const int32_t kc = step * p.kt;
        umma_tma_boxes<PAIR>(&p.xmap, p.xt, bx, rx, kc, dx, FULL + 8 * s, policy);
        umma_tma_boxes<PAIR>(&p.ymap, p.yt, by, ry, kc, dy, FULL + 8 * s, policy);
        if (++step == p.nsteps) {
          step = 0;
          if (++lt < ntl) {
            umma_box_origin(p.xt, nxc, bx);
            umma_box_origin(p.yt, nyc, by);
            if (lt + 1 < ntl) unit(cid + (lt + 1) * ncl);
          }
        }
      }
    }
  } else if (warp >= K::EW && warp < K::EW + K::PW) {
    // ======================= producers ===================================================
    const int pt = tid - K::EW * 32;
    const T *__restrict__ X = static_cast<const T *>(p.X);
    const T *__restrict__ Y = static_cast<const T *>(p.Y);
    // fast path: both operands in 16-B vectors, slots cached in registers
    const bool cached = p.vecX == 16 / ES && p.vecY == 16 / ES && p.nslotX <= K::EX * K::PW * 32 &&
                        p.nslotY <= K::EY * K::PW * 32;
    int32_t rx[K::EX], ry[K::EY];
    uint32_t px[K::EX], py[K::EY];
    int cx = 0, cy = 0;
    if (cached) {
      umma_load_slots<K::EX, ES>(rx, px, p.relX, p.packX, p.nslotX, pt, K::PW * 32);
      umma_load_slots<K::EY, ES>(ry, py, p.relY, p.packY, p.nslotY, pt, K::PW * 32);
      cx = (p.nslotX - pt + K::PW * 32 - 1) / (K::PW * 32);
      cy = (p.nslotY - pt + K::PW * 32 - 1) / (K::PW * 32);
    }
    // next tile's origins / masks fetched during the current tile's last stage; k steps by
    // the register odometer
    ProdTile cur;
    if (ntl > 0) cur.fetch(p, (int)blockIdx.x);
    KStep ks;
    ks.reset(p);
    int step = 0, lt = 0;
    for (int j = 0; j < total; j++) {
      const int s = j % STAGES;
      if (pt == 0) trace_at(p, 6, j);
      if (j >= STAGES) mbar_wait(EMPTY + 8 * s, ((j / STAGES) & 1) ^ 1);
      if (pt == 0) trace_at(p, 0, j);
      // (no prefetch.global.L1 of the next tile's records here: measured slower)
      const uint64_t km = ks.mask(p);
      const bool fk = km == p.fullK;
      const bool fm = cur.fm, fn = cur.fn;
      const uint64_t(&mm)[kMaskWords] = cur.mm;
      const uint64_t(&mn)[kMaskWords] = cur.mn;
      const int64_t bx = cur.ox + ks.sx(), by = cur.oy + ks.sy();
      const uint32_t dx = sbase + (uint32_t)ES * (uint32_t)(s * K::XS);
      const uint32_t dy = sbase + (uint32_t)ES * (uint32_t)(STAGES * K::XS + s * K::YS);
#if defined(TC_UMMA_ABLATE) && TC_UMMA_ABLATE == 2
      if (true) {   // (ablation side build: the producers load nothing)
        mbar_arrive(FULL + 8 * s);
      } else
#endif
      if (cached) {
        umma_issue<K::EX>(X, dx, rx, px, cx, bx, fm && fk, km, mm, p.packX, pt, K::PW * 32);
        umma_issue<K::EY>(Y, dy, ry, py, cy, by, fn && fk, km, mn, p.packY, pt, K::PW * 32);
        mbar_arrive_cp_async(FULL + 8 * s);
      } else {
        umma_issue_generic_t<K::PW>(p, X, Y, pt, dx, dy, bx, by, km, mm, mn);
        if (ES == 2 && (p.vecX == 1 || p.vecY == 1)) {
          // plain stores are published by a release arrive once this thread's copies landed
          asm volatile("cp.async.wait_all;\n" ::: "memory");
          mbar_arrive(FULL + 8 * s);
        } else {
          mbar_arrive_cp_async(FULL + 8 * s);
        }
      }
      if (pt == 0) trace_at(p, 1, j);
      ks.advance(p);
      if (++step == p.nsteps) {
        step = 0;
        if (++lt < ntl) cur.fetch(p, (int)blockIdx.x + lt * (int)gridDim.x);
        if (pt == 0) trace_at(p, 7, j);
      }
    }
  } else if (warp == K::EW + K::PW && (!PAIR || crank == 0)) {
    // ======================= MMA issuer ===================================================
    // N and the number of K-instructions trimmed to the plan's tile (host: umma_trim): a
    // 24-column tile issues N = 32 (K-major Y) instead of BN, a 36-deep k step 3 of 4
    const uint32_t IDESC = PAIR ? umma_idesc(ES == 2 ? 1 : 2, 2 * BN, !XK, !YK, 256)
                                : umma_idesc(ES == 2 ? 1 : 2, p.nmma, !XK, !YK);
    const int kmma = p.kmma;
    // canonical no-swizzle layouts (bytes): K-major LBO = 128 (k groups), SBO = 1024 (8-row
    // groups); MN-major SBO = 128 (8-row groups), LBO = rows/8 * 128 (k groups)
    // 128-B swizzled layouts (tiles.hpp smem_off): K-major = 8-row x 128-B atoms stacked
    // along M/N (SBO = 1 KB; K = 16 advances the start by 32 B inside the atom); MN-major =
    // 64-element x 8-k atoms, the k groups of one MN atom adjacent (SBO = 1 KB) and the MN
    // atoms BK/8 KB apart (LBO) — the order a TMA box of (64 MN, BK k) lands in smem
    // (E = 128 / ES elements per 128-B row; one MMA consumes K = KI = 32 B of k.  BF16
    // MN-major: 8-k x 128-B atoms (1 KB), K = 16 = two k groups.  TF32 MN-major
    // (SWIZZLE_128B_BASE32B): 4-k x 128-B atoms (512 B), K = 8 = two k groups.)
    constexpr int E = 128 / ES;
    constexpr uint32_t ATOM = ES == 4 ? 512 : 1024, KG = ES == 4 ? 4 : 8;   // MN-major atom bytes, k rows
    constexpr int XL = XK || ES == 2 ? 2 : 1, YL = YK || ES == 2 ? 2 : 1;   // descriptor layout types
    constexpr uint32_t A_LBO = XK ? 16 : (BK / KG) * ATOM, A_SBO = XK ? 1024 : ATOM;
    constexpr uint32_t B_LBO = YK ? 16 : (BK / KG) * ATOM, B_SBO = YK ? 1024 : ATOM;
    constexpr uint32_t A_KSTEP = XK ? 32 : (K::KI / KG) * A_SBO, B_KSTEP = YK ? 32 : (K::KI / KG) * B_SBO;
    int step = 0, lt = 0;
    for (int j = 0; j < total; j++) {
      const int s = j % STAGES;
      const int buf = lt % NBUF;
      if (step == 0 && lt >= NBUF) {
        if (PAIR) mbar_wait_acq_cluster(TEMPTY + 8 * buf, ((lt / NBUF) & 1) ^ 1);   // both CTAs drained it
        else mbar_wait(TEMPTY + 8 * buf, ((lt / NBUF) & 1) ^ 1);
      }
      if (K::SPLIT) mbar_wait(SPLITB + 8 * s, (j / STAGES) & 1);
      else mbar_wait(FULL + 8 * s, (j / STAGES) & 1);
      if (lane == 0) trace_at(p, 2, j);
      // the stage was written through the generic proxy (cp.async / st.shared); the MMA
      // reads it through the async proxy
      asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
      tc05_fence_after();
      if (lane == 0) {
        const uint32_t ax = sbase + (uint32_t)ES * (uint32_t)(s * K::XS);
        const uint32_t by = sbase + (uint32_t)ES * (uint32_t)(STAGES * K::XS + s * K::YS);
        const uint32_t d = tmem + (uint32_t)(buf * ACCW);
#pragma unroll
        for (int kk = 0; kk < BK / K::KI; kk++) {
          if (kk >= kmma) break;
          const uint64_t ah = umma_desc<XL>(ax + kk * A_KSTEP, A_LBO, A_SBO);
          const uint64_t bh = umma_desc<YL>(by + kk * B_KSTEP, B_LBO, B_SBO);
          if (K::SPLIT) {   // small terms first: lo*hi, hi*lo, then hi*hi
            tc05_mma<true>(d, umma_desc<XL>(ax + LO + kk * A_KSTEP, A_LBO, A_SBO), bh, IDESC, (step > 0 || kk > 0) ? 1u : 0u);
            tc05_mma<true>(d, ah, umma_desc<YL>(by + LO + kk * B_KSTEP, B_LBO, B_SBO), IDESC, 1u);
            tc05_mma<true>(d, ah, bh, IDESC, 1u);
          } else if (PAIR) {
            tc05_mma2<ES == 4>(d, ah, bh, IDESC, (step > 0 || kk > 0) ? 1u : 0u);
          } else {
            tc05_mma<ES == 4>(d, ah, bh, IDESC, (step > 0 || kk > 0) ? 1u : 0u);
          }
        }
        if (PAIR) {   // both CTAs' stage / accumulator
          tc05_commit2(EMPTY + 8 * s);
          if (step + 1 == p.nsteps) tc05_commit2(TFULL + 8 * buf);
        } else {
          tc05_commit(EMPTY + 8 * s);                           // smem stage free once MMAs read it
          if (step + 1 == p.nsteps) tc05_commit(TFULL + 8 * buf);   // accumulator ready
        }
        trace_at(p, 3, j);
      }
      __syncwarp();
      if (++step == p.nsteps) { step = 0; ++lt; }
    }
  } else if (K::SPLIT && warp > K::EW + K::PW) {
    // ======================= split warps (F32X3) ==========================================
    // once a stage has landed: x -> hi = x with the low 13 mantissa bits cleared (exactly the
    // TF32 value the MMA reads) in place, lo = x - hi (exact in FP32) into the lo plane
    const int st = tid - (K::EW + K::PW + 1) * 32;
    constexpr int N4 = (K::XS + K::YS) / 4;          // float4 per stage plane
    for (int j = 0; j < total; j++) {
      const int s = j % STAGES;
      mbar_wait(FULL + 8 * s, (j / STAGES) & 1);
      float4 *hx = reinterpret_cast<float4 *>(smem_raw) + (size_t)s * (K::XS / 4);
      float4 *hy = reinterpret_cast<float4 *>(smem_raw) + (size_t)STAGES * (K::XS / 4) + (size_t)s * (K::YS / 4);
#pragma unroll 4
      for (int i = st; i < N4; i += K::SW * 32) {
        float4 *h = i < K::XS / 4 ? hx + i : hy + (i - K::XS / 4);
        float4 *l = reinterpret_cast<float4 *>(reinterpret_cast<unsigned char *>(h) + LO);
        const float4 x = *h;
        float4 hi, lo;
        hi.x = __uint_as_float(__float_as_uint(x.x) & 0xFFFFE000u); lo.x = x.x - hi.x;
        hi.y = __uint_as_float(__float_as_uint(x.y) & 0xFFFFE000u); lo.y = x.y - hi.y;
        hi.z = __uint_as_float(__float_as_uint(x.z) & 0xFFFFE000u); lo.z = x.z - hi.z;
        hi.w = __uint_as_float(__float_as_uint(x.w) & 0xFFFFE000u); lo.w = x.w - hi.w;
        *h = hi;
        *l = lo;
      }
      // generic-proxy writes -> visible to the MMA's async-proxy reads
      asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
      __syncwarp();
      if (lane == 0) mbar_arrive(SPLITB + 8 * s);
    }
  } else if (warp < K::EW) {
    // ======================= epilogue =====================================================
    // warp w drains TMEM lane quarter w % 4 (tile rows 32(w%4) .. +31; one row per thread)
    // and column half w / 4; FP32 arithmetic on the FP32 accumulator, stored as T (BF16: RNE)
    TC *__restrict__ C = static_cast<TC *>(p.C);
    const float alpha = (float)p.alpha, beta = (float)p.beta;
    const int quarter = warp & 3, half = warp >> 2;
    const int row = quarter * 32 + lane;               // TMEM lane = tile row m
    const int64_t roff = relCm[row];
    constexpr int HC = BN / 2;                          // columns per warp
    // staged path: lane drains row group g (8 C-contiguous rows) of columns lane/4 + 8i
    float *stg = stage + warp * 32 * 32;
    const int g = lane & 3;
    const int grow = quarter * 32 + g * 8;
    const int64_t goff = relCm[grow];
    // tile info is fetched one tile ahead: its load latency hides behind the current tile
    // (PAIR: this CTA's m-tile against the unit's two n-tiles)
    int64_t nmc = 0, nnc[NSUB];   // (raw records: summed at use, so the loads overlap a tile)
    uint64_t nrm0 = 0, nrm1 = 0, ncm0[NSUB], ncm1[NSUB];
    auto fetch = [&](int t) {
      int mt, nt;
      if (PAIR) {
        int pm, pn;
        pair_coords(p, cid + t * ncl, pm, pn);
        mt = 2 * pm + crank;
        nt = 2 * pn;
      } else {
        tile_coords(p, cid + t * ncl, mt, nt);
      }
      nrm0 = p.tileM[mt].mask[0];
      nrm1 = p.tileM[mt].mask[1];
      nmc = p.tileM[mt].c;
#pragma unroll
      for (int q = 0; q < NSUB; q++) {
        nnc[q] = p.tileN[nt + q].c;
        ncm0[q] = p.tileN[nt + q].mask[0];
        ncm1[q] = p.tileN[nt + q].mask[1];
      }
    };
    if (ntl > 0) fetch(0);
    // CTA-wide staged path (cs0 > 1): thread -> (run, first column, column step).  With
    // nruns | 256 (the host guarantees it for this path) every thread keeps one run: rows
    // rr + cs0 * i, i < 8, of columns rcol0, rcol0 + rcstep, ...
    int rr = 0, rcol0 = 0, rcstep = 1;
    int64_t rroff = 0;
    const int rs0 = p.cs0;
    if (p.vecC == 8 && p.cs0 > 1) {
      const int nruns = p.Mt >> 3, t8 = p.ct0 >> 3;
      const int etid = warp * 32 + lane;
      const int run = etid % nruns;
      const int lo = run % rs0, tq = run / rs0;
      rr = lo + rs0 * (8 * (tq % t8) + p.ct0 * (tq / t8));
      rcol0 = etid / nruns;
      rcstep = K::EW * 32 / nruns;
      rroff = relCm[rr];
    }
    for (int lt = 0; lt < ntl; lt++) {
      const int buf = lt % NBUF;
      int64_t coffs[NSUB];
      uint64_t cm0s[NSUB], cm1s[NSUB];
      const int64_t mc = nmc;
#pragma unroll
      for (int q = 0; q < NSUB; q++) {
        coffs[q] = nnc[q];
        cm0s[q] = ncm0[q];
        cm1s[q] = ncm1[q];
      }
      const uint64_t rm0 = nrm0, rm1 = nrm1;
      if (lt + 1 < ntl) fetch(lt + 1);
      const bool rok = ((row < 64 ? rm0 : rm1) >> (row & 63)) & 1;
      const bool gok = ((grow < 64 ? rm0 : rm1) >> (grow & 63)) & 1;
      mbar_wait_sleep(TFULL + 8 * buf, (lt / NBUF) & 1);
      tc05_fence_after();
#pragma unroll 1
      for (int q = 0; q < NSUB; q++) {
      const int64_t coff = mc + coffs[q];
      const uint64_t cm0 = cm0s[q], cm1 = cm1s[q];
      const uint32_t cb = (uint32_t)(buf * ACCW + q * BN);   // this tile's TMEM columns
      TC *Crow = C + (coff + roff);
      const bool cfull = cm0 == p.fullN[0] && cm1 == p.fullN[1];
      TC *Cg = C + (coff + goff);
#if defined(TC_UMMA_ABLATE) && TC_UMMA_ABLATE == 1
      if (true) {   // (ablation side build: the epilogue drains nothing)
#else
      if (kTrace) {
#endif
        if (warp == 0 && lane == 0) trace_at(p, 4, lt);
      } else if (!PAIR && p.vecC == 8 && p.cs0 > 1) {
        // CTA-wide staged epilogue: C's FVI is an inner m digit (tile-row stride cs0), so the
        // 8 C-contiguous elements of a run live in rows r, r + cs0, ..., r + 7 cs0 of
        // different warps.  Per 64-column pass all eight warps park their TMEM rows in smem
        // ([column][row] FP32), then each thread stores whole runs: 16-B (BF16) / 2 x 16-B
        // (FP32) stores along C's FVI, whatever the m digit order (the X loads keep theirs).
        const bool rrok = ((rr < 64 ? rm0 : rm1) >> (rr & 63)) & 1;
        TC *Cr = C + (coff + rroff);
        for (int pc = 0; pc < BN && pc < p.Nt; pc += 64) {
          uint32_t v[32];
          tc05_ld<32>(tmem + ((uint32_t)(quarter * 32) << 16) + cb + (uint32_t)(pc + half * 32), v);
#pragma unroll
          for (int q = 0; q < 32; q++) stage[(half * 32 + q) * 128 + row] = __uint_as_float(v[q]);
          asm volatile("bar.sync 1, %0;\n" ::"r"(K::EW * 32) : "memory");
          // this thread's run (fixed for the kernel when nruns divides the 256 threads)
          const int ncols = min(64, p.Nt - pc);
          if (rrok) {
            for (int col = rcol0; col < ncols; col += rcstep) {
              const int c = pc + col;
              if (!(((c < 64 ? cm0 : cm1) >> (c & 63)) & 1)) continue;
              float x[8];
#pragma unroll
              for (int i = 0; i < 8; i++) x[i] = alpha * stage[col * 128 + rr + rs0 * i];
              store_run8(Cr + relCn[c], x, beta);
            }
          }
          asm volatile("bar.sync 1, %0;\n" ::"r"(K::EW * 32) : "memory");
        }
      } else
#pragma unroll
      for (int c0 = 0; c0 < HC; c0 += 32 > HC ? HC : 32) {
        constexpr int W = 32 > HC ? HC : 32;
        if (half * HC + c0 >= p.Nt) break;             // columns past the tile's Nt: padding
        uint32_t v[W];
        tc05_ld<W>(tmem + ((uint32_t)(quarter * 32) << 16) + cb + (uint32_t)(half * HC + c0), v);
        if (!PAIR && p.vecC == 8) {
          // FP32 accumulators to smem as [column][row], then one 16-B store per 8 rows
          // (C's FVI leads m with an 8-multiple tile: 8 tile rows are 8 C-contiguous elements)
#pragma unroll
          for (int q = 0; q < W; q++) stg[q * 32 + lane] = __uint_as_float(v[q]);
          __syncwarp();
          // all smem reads first (independent), then the stores
          float4 d[W / 8][2];
          int64_t rc[W / 8];
          bool ok[W / 8];
#pragma unroll
          for (int i = 0; i < W / 8; i++) {
            const int cc = (lane >> 2) + 8 * i;
            const int c = half * HC + c0 + cc;
            ok[i] = gok && c < p.Nt && (((c < 64 ? cm0 : cm1) >> (c & 63)) & 1);
            rc[i] = relCn[c];
            d[i][0] = *reinterpret_cast<const float4 *>(stg + cc * 32 + g * 8);
            d[i][1] = *reinterpret_cast<const float4 *>(stg + cc * 32 + g * 8 + 4);
          }
#pragma unroll
          for (int i = 0; i < W / 8; i++) {
            if (ok[i]) {
              float r[8] = {alpha * d[i][0].x, alpha * d[i][0].y, alpha * d[i][0].z, alpha * d[i][0].w,
                            alpha * d[i][1].x, alpha * d[i][1].y, alpha * d[i][1].z, alpha * d[i][1].w};
              if constexpr (sizeof(TC) == 4) {
                float4 *dst = reinterpret_cast<float4 *>(Cg + rc[i]);
                if (beta != 0.0f) {
                  const float4 o0 = dst[0], o1 = dst[1];
                  r[0] = fmaf(beta, o0.x, r[0]); r[1] = fmaf(beta, o0.y, r[1]);
                  r[2] = fmaf(beta, o0.z, r[2]); r[3] = fmaf(beta, o0.w, r[3]);
                  r[4] = fmaf(beta, o1.x, r[4]); r[5] = fmaf(beta, o1.y, r[5]);
                  r[6] = fmaf(beta, o1.z, r[6]); r[7] = fmaf(beta, o1.w, r[7]);
                }
                dst[0] = make_float4(r[0], r[1], r[2], r[3]);
                dst[1] = make_float4(r[4], r[5], r[6], r[7]);
                continue;
              }
              uint4 *dst = reinterpret_cast<uint4 *>(Cg + rc[i]);
              if (beta != 0.0f) {
                const uint4 o = *dst;
                const uint32_t ow[4] = {o.x, o.y, o.z, o.w};
#pragma unroll
                for (int j = 0; j < 4; j++) {
                  r[2 * j] = fmaf(beta, __uint_as_float(ow[j] << 16), r[2 * j]);
                  r[2 * j + 1] = fmaf(beta, __uint_as_float(ow[j] & 0xFFFF0000u), r[2 * j + 1]);
                }
              }
              uint32_t w[4];
#pragma unroll
              for (int j = 0; j < 4; j++) {
                const __nv_bfloat162 b2 = __floats2bfloat162_rn(r[2 * j], r[2 * j + 1]);
                w[j] = *reinterpret_cast<const uint32_t *>(&b2);
              }
              *dst = make_uint4(w[0], w[1], w[2], w[3]);
            }
          }
          __syncwarp();
        } else if (rok) {
          if (cfull && beta == 0.0f) {
#pragma unroll
            for (int q = 0; q < W; q++)
              if (half * HC + c0 + q < p.Nt)               // (the full mask covers Nt columns)
                st_out(Crow + relCn[half * HC + c0 + q], alpha * __uint_as_float(v[q]));
          } else {
#pragma unroll
            for (int q = 0; q < W; q++) {
              const int c = half * HC + c0 + q;
              if (((c < 64 ? cm0 : cm1) >> (c & 63)) & 1) {
                TC *dst = Crow + relCn[c];
                float r = alpha * __uint_as_float(v[q]);
                if (beta != 0.0f) r = fmaf(beta, ld_out(dst), r);
                st_out(dst, r);
              }
            }
          }
        }
      }
      }   // tiles of the unit
      tc05_fence_before();
      __syncwarp();
      if (lane == 0) {
        if (PAIR) mbar_arrive_cta(TEMPTY + 8 * buf, 0);   // the leader's MMAs reuse the buffer
        else mbar_arrive(TEMPTY + 8 * buf);
      }
      if (warp == 0 && lane == 0) trace_at(p, 5, lt);
    }
  }
  if (PAIR) cluster_sync_all();   // no CTA leaves while its peer may still signal it
  else __syncthreads();
  if (warp == K::EW + K::PW) {
    tc05_fence_after();
    if (PAIR) asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "r"(K::TMEM_COLS));
    else asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "r"(K::TMEM_COLS));
  }
}

}  // namespace tc
