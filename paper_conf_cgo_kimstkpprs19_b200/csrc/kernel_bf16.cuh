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
__device__ __forceinline__ void tc05_mma_bf16(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                              uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate) : "memory");
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
template <int E>
__device__ __forceinline__ void bf16_load_slots(int32_t (&rel)[E], uint32_t (&pack)[E], const int32_t *__restrict__ r,
                                                const uint32_t *__restrict__ pk, int n, int first, int stride) {
#pragma unroll
  for (int i = 0; i < E; i++) {
    const int q = first + i * stride;
    rel[i] = q < n ? __ldg(r + q) : 0;
    pack[i] = q < n ? __ldg(pk + q) : 0u;
  }
}

template <int E, int VB>
__device__ __forceinline__ void bf16_issue(const __nv_bfloat16 *__restrict__ src, uint32_t sdst,
                                           const int32_t (&rel)[E], const uint32_t (&pack)[E], int cnt,
                                           int64_t base, bool fast, uint64_t kmask, const uint64_t (&rmask)[kMaskWords]) {
  const __nv_bfloat16 *b = src + base;
  if (fast) {
#pragma unroll
    for (int i = 0; i < E; i++) {
      if (i < cnt) {
        const uint32_t d = sdst + 2u * (pack[i] & 0x3FFF);
        if (VB == 16) cp_async16v_full(d, b + rel[i]);
        else cp_async8v_full(d, b + rel[i]);
      }
    }
  } else {
#pragma unroll
    for (int i = 0; i < E; i++) {
      if (i < cnt) {
        const uint32_t pk = pack[i];
        const int k = (pk >> 14) & 63, m = pk >> 20;
        const bool ok = ((kmask >> k) & 1) && bit_of(rmask, m);
        const uint32_t d = sdst + 2u * (pk & 0x3FFF);
        if (VB == 16) cp_async16v(d, ok ? b + rel[i] : src, ok ? 16 : 0);
        else cp_async8v(d, ok ? b + rel[i] : src, ok ? 8 : 0);
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

// UMMA shared-memory descriptor, no swizzle (SM100 layout: start>>4 [0,14), LBO>>4
// [16,30), SBO>>4 [32,46), version 1 [46,48), layout type 0 [61,64)).
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
         ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46);
}

template <int BN, int STAGES>
struct Bf16Kernel {
  static constexpr int BM = 128, BK = 64;            // one UMMA M = 128, four K = 16 per stage
  static constexpr int EW = 8, PW = 4;               // epilogue warps, producer warps
  static constexpr int THREADS = (EW + PW + 1) * 32; // + one MMA warp
  static constexpr int XS = BM * BK + 8, YS = BN * BK + 8;   // elements per stage (+16-B scratch)
  static constexpr int TMEM_COLS = 2 * BN;           // double-buffered FP32 accumulator
  static constexpr size_t smem_bytes() {
    return 2 * (size_t)STAGES * (XS + YS) + 8 * (2 * STAGES + 4) + 16 + 8 * (size_t)(BM + BN);
  }
  // register-cached slots per producer thread (16-B vectors)
  static constexpr int EX = BM * BK / 8 / (PW * 32), EY = BN * BK / 8 / (PW * 32);
  static_assert(BN % 16 == 0 && BN <= 128, "BN");
  static_assert(TMEM_COLS >= 32 && (TMEM_COLS & (TMEM_COLS - 1)) == 0, "TMEM allocation");
};

// UMMA instruction descriptor: BF16 x BF16 -> F32, M = 128, N = BN, majors per operand.
__host__ __device__ constexpr uint32_t umma_idesc_bf16(int n, bool a_mn, bool b_mn) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)a_mn << 15) | ((uint32_t)b_mn << 16) |
         ((uint32_t)(n >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
}

template <int BN, int STAGES, bool XK, bool YK>
__global__ void __launch_bounds__(Bf16Kernel<BN, STAGES>::THREADS, 1)
tc_bf16_umma_kernel(const __grid_constant__ KParams p) {
  using K = Bf16Kernel<BN, STAGES>;
  constexpr int BM = K::BM, BK = K::BK;
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  __nv_bfloat16 *sX = reinterpret_cast<__nv_bfloat16 *>(smem_raw);
  __nv_bfloat16 *sY = sX + STAGES * K::XS;
  uint64_t *bars = reinterpret_cast<uint64_t *>(sY + STAGES * K::YS);  // full, empty, tfull[2], tempty[2]
  uint32_t *tmem_holder = reinterpret_cast<uint32_t *>(bars + 2 * STAGES + 4);
  int64_t *relCm = reinterpret_cast<int64_t *>(tmem_holder + 4);
  int64_t *relCn = relCm + BM;

  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int ntl = (p.ntotal - (int)blockIdx.x + (int)gridDim.x - 1) / (int)gridDim.x;
  const int total = max(ntl, 0) * p.nsteps;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(smem_raw);
  const uint32_t bar0 = (uint32_t)__cvta_generic_to_shared(bars);
  const uint32_t FULL = bar0, EMPTY = bar0 + 8 * STAGES, TFULL = bar0 + 16 * STAGES, TEMPTY = TFULL + 16;

  // ---- once per CTA ------------------------------------------------------------------------
  for (int i = tid; i < STAGES * (K::XS + K::YS) / 8; i += K::THREADS)
    reinterpret_cast<uint4 *>(smem_raw)[i] = make_uint4(0, 0, 0, 0);
  for (int r = tid; r < BM; r += K::THREADS) relCm[r] = p.relCm[r];
  for (int r = tid; r < BN; r += K::THREADS) relCn[r] = p.relCn[r];
  if (tid == 0) {
    for (int s = 0; s < STAGES; s++) {
      mbar_init(FULL + 8 * s, K::PW * 32);   // producer threads (cp.async arrivals)
      mbar_init(EMPTY + 8 * s, 1);           // tcgen05.commit of the MMA thread
    }
    for (int b = 0; b < 2; b++) {
      mbar_init(TFULL + 8 * b, 1);           // tcgen05.commit after a tile's last MMA
      mbar_init(TEMPTY + 8 * b, K::EW);      // one arrive per epilogue warp
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  if (warp == K::EW + K::PW) {               // the MMA warp owns the TMEM allocation
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(
                     (uint32_t)__cvta_generic_to_shared(tmem_holder)),
                 "r"(K::TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n" ::);
  }
  tc05_fence_before();
  __syncthreads();
  tc05_fence_after();
  const uint32_t tmem = *tmem_holder;

  if (warp >= K::EW && warp < K::EW + K::PW) {
    // ======================= producers ===================================================
    const int pt = tid - K::EW * 32;
    const __nv_bfloat16 *__restrict__ X = static_cast<const __nv_bfloat16 *>(p.X);
    const __nv_bfloat16 *__restrict__ Y = static_cast<const __nv_bfloat16 *>(p.Y);
    int step = 0, lt = 0;
    int64_t ox = 0, oy = 0;
    uint64_t mm[kMaskWords], mn[kMaskWords];
    bool fm = true, fn = true;
    // fast path: both operands in 16-B vectors, slots cached in registers
    const bool cached = p.vecX == 8 && p.vecY == 8 && p.nslotX <= K::EX * K::PW * 32 &&
                        p.nslotY <= K::EY * K::PW * 32;
    int32_t rx[K::EX], ry[K::EY];
    uint32_t px[K::EX], py[K::EY];
    int cx = 0, cy = 0;
    if (cached) {
      bf16_load_slots(rx, px, p.relX, p.packX, p.nslotX, pt, K::PW * 32);
      bf16_load_slots(ry, py, p.relY, p.packY, p.nslotY, pt, K::PW * 32);
      cx = (p.nslotX - pt + K::PW * 32 - 1) / (K::PW * 32);
      cy = (p.nslotY - pt + K::PW * 32 - 1) / (K::PW * 32);
    }
    for (int j = 0; j < total; j++) {
      const int s = j % STAGES;
      if (j >= STAGES) mbar_wait(EMPTY + 8 * s, ((j / STAGES) & 1) ^ 1);
      if (step == 0) {
        int mt, nt;
        tile_coords(p, (int)blockIdx.x + lt * (int)gridDim.x, mt, nt);
        ox = p.tileM[mt].op;
        oy = p.tileN[nt].op;
#pragma unroll
        for (int w = 0; w < kMaskWords; w++) { mm[w] = p.tileM[mt].mask[w]; mn[w] = p.tileN[nt].mask[w]; }
        fm = fn = true;
#pragma unroll
        for (int w = 0; w < kMaskWords; w++) { fm &= mm[w] == p.fullM[w]; fn &= mn[w] == p.fullN[w]; }
      }
      const uint64_t km = __ldg(p.kmask + step);
      const bool fk = km == p.fullK;
      const int64_t bx = ox + __ldg(p.stepX + step), by = oy + __ldg(p.stepY + step);
      const uint32_t dx = sbase + 2u * (uint32_t)(s * K::XS);
      const uint32_t dy = sbase + 2u * (uint32_t)(STAGES * K::XS + s * K::YS);
      if (cached) {
        bf16_issue<K::EX, 16>(X, dx, rx, px, cx, bx, fm && fk, km, mm);
        bf16_issue<K::EY, 16>(Y, dy, ry, py, cy, by, fn && fk, km, mn);
        mbar_arrive_cp_async(FULL + 8 * s);
        if (++step == p.nsteps) { step = 0; ++lt; }
        continue;
      }
      for (int side = 0; side < 2; side++) {
        const __nv_bfloat16 *src = side ? Y : X;
        const int32_t *rel = side ? p.relY : p.relX;
        const uint32_t *pack = side ? p.packY : p.packX;
        const int n = side ? p.nslotY : p.nslotX, vec = side ? p.vecY : p.vecX;
        const int64_t base = side ? by : bx;
        const uint32_t dst0 = side ? dy : dx;
        const uint64_t *rm = side ? mn : mm;
        for (int q = pt; q < n; q += K::PW * 32) {
          const uint32_t pk = __ldg(pack + q);
          const int k = (pk >> 14) & 63, m = pk >> 20;
          const bool ok = ((km >> k) & 1) && ((((m < 64) ? rm[0] : rm[1]) >> (m & 63)) & 1);
          const __nv_bfloat16 *g = ok ? src + (base + __ldg(rel + q)) : src;
          const uint32_t d = dst0 + 2u * (pk & 0x3FFF);
          if (vec == 8) cp_async16v(d, g, ok ? 16 : 0);
          else if (vec == 4) cp_async8v(d, g, ok ? 8 : 0);
          else if (vec == 2) cp_async4(d, g, ok ? 4 : 0);
          else {   // single elements: plain load / store (cp.async has no 2-byte form)
            const unsigned short v = ok ? *reinterpret_cast<const unsigned short *>(g) : (unsigned short)0;
            asm volatile("st.shared.u16 [%0], %1;\n" ::"r"(d), "h"(v) : "memory");
          }
        }
      }
      if (p.vecX == 1 || p.vecY == 1) {
        // plain stores are published by a release arrive once this thread's copies landed
        asm volatile("cp.async.wait_all;\n" ::: "memory");
        mbar_arrive(FULL + 8 * s);
      } else {
        mbar_arrive_cp_async(FULL + 8 * s);
      }
      if (++step == p.nsteps) { step = 0; ++lt; }
    }
  } else if (warp == K::EW + K::PW) {
    // ======================= MMA issuer ===================================================
    constexpr uint32_t IDESC = umma_idesc_bf16(BN, !XK, !YK);
    // canonical no-swizzle layouts (bytes): K-major LBO = 128 (k groups), SBO = 1024 (8-row
    // groups); MN-major SBO = 128 (8-row groups), LBO = rows/8 * 128 (k groups)
    constexpr uint32_t A_LBO = XK ? 128 : (BM / 8) * 128, A_SBO = XK ? (BK / 8) * 128 : 128;
    constexpr uint32_t B_LBO = YK ? 128 : (BN / 8) * 128, B_SBO = YK ? (BK / 8) * 128 : 128;
    constexpr uint32_t A_KSTEP = XK ? 256 : 2 * A_LBO, B_KSTEP = YK ? 256 : 2 * B_LBO;  // per K = 16
    int step = 0, lt = 0;
    for (int j = 0; j < total; j++) {
      const int s = j % STAGES;
      const int buf = lt & 1;
      if (step == 0 && lt >= 2) mbar_wait(TEMPTY + 8 * buf, ((lt >> 1) & 1) ^ 1);
      mbar_wait(FULL + 8 * s, (j / STAGES) & 1);
      // the stage was written through the generic proxy (cp.async / st.shared); the MMA
      // reads it through the async proxy
      asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
      tc05_fence_after();
      if (lane == 0) {
        const uint32_t ax = sbase + 2u * (uint32_t)(s * K::XS);
        const uint32_t by = sbase + 2u * (uint32_t)(STAGES * K::XS + s * K::YS);
#pragma unroll
        for (int kk = 0; kk < BK / 16; kk++)
          tc05_mma_bf16(tmem + (uint32_t)(buf * BN), umma_desc(ax + kk * A_KSTEP, A_LBO, A_SBO),
                        umma_desc(by + kk * B_KSTEP, B_LBO, B_SBO), IDESC, (step > 0 || kk > 0) ? 1u : 0u);
        tc05_commit(EMPTY + 8 * s);                      // smem stage free once MMAs read it
        if (step + 1 == p.nsteps) tc05_commit(TFULL + 8 * buf);   // accumulator ready
      }
      __syncwarp();
      if (++step == p.nsteps) { step = 0; ++lt; }
    }
  } else if (warp < K::EW) {
    // ======================= epilogue =====================================================
    // warp w drains TMEM lane quarter w % 4 (tile rows 32(w%4) .. +31; one row per thread)
    // and column half w / 4; FP32 arithmetic on the FP32 accumulator, RNE to BF16
    __nv_bfloat16 *__restrict__ C = static_cast<__nv_bfloat16 *>(p.C);
    const float alpha = (float)p.alpha, beta = (float)p.beta;
    const int quarter = warp & 3, half = warp >> 2;
    const int row = quarter * 32 + lane;               // TMEM lane = tile row m
    const int64_t roff = relCm[row];
    constexpr int HC = BN / 2;                          // columns per warp
    for (int lt = 0; lt < ntl; lt++) {
      const int buf = lt & 1;
      int mt, nt;
      tile_coords(p, (int)blockIdx.x + lt * (int)gridDim.x, mt, nt);
      const TileInfo &tm = p.tileM[mt];
      const TileInfo &tn = p.tileN[nt];
      const bool rok = ((row < 64 ? tm.mask[0] : tm.mask[1]) >> (row & 63)) & 1;
      __nv_bfloat16 *Crow = C + (tm.c + tn.c + roff);
      const uint64_t cm0 = tn.mask[0], cm1 = tn.mask[1];
      const bool cfull = cm0 == p.fullN[0] && cm1 == p.fullN[1];
      mbar_wait(TFULL + 8 * buf, (lt >> 1) & 1);
      tc05_fence_after();
#pragma unroll
      for (int c0 = 0; c0 < HC; c0 += 32 > HC ? HC : 32) {
        constexpr int W = 32 > HC ? HC : 32;
        if (half * HC + c0 >= p.Nt) break;             // columns past the tile's Nt: padding
        uint32_t v[W];
        tc05_ld<W>(tmem + ((uint32_t)(quarter * 32) << 16) + (uint32_t)(buf * BN + half * HC + c0), v);
        if (rok) {
          if (cfull && beta == 0.0f) {
#pragma unroll
            for (int q = 0; q < W; q++)
              if (half * HC + c0 + q < p.Nt)               // (the full mask covers Nt columns)
                Crow[relCn[half * HC + c0 + q]] = __float2bfloat16_rn(alpha * __uint_as_float(v[q]));
          } else {
#pragma unroll
            for (int q = 0; q < W; q++) {
              const int c = half * HC + c0 + q;
              if (((c < 64 ? cm0 : cm1) >> (c & 63)) & 1) {
                __nv_bfloat16 *dst = Crow + relCn[c];
                float r = alpha * __uint_as_float(v[q]);
                if (beta != 0.0f) r = fmaf(beta, __bfloat162float(*dst), r);
                *dst = __float2bfloat16_rn(r);
              }
            }
          }
        }
      }
      tc05_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(TEMPTY + 8 * buf);
    }
  }
  __syncthreads();
  if (warp == K::EW + K::PW) {
    tc05_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tmem), "r"(K::TMEM_COLS));
  }
}

}  // namespace tc
