// kernel_stream.cuh — the streaming BF16 contraction kernel (stream.hpp) for low-intensity
// tensor x matrix contractions (TCCG #1-8), sm_100a.
//
// The paper's four steps:
//   (1) one producer thread streams X boxes (X's own index order; one box per
//       (tile, k-step), zero-filled outside the tensor) into a STAGES-deep ring;
//   (2)+(3) each compute warp owns one unit of the tile — AR consecutive values a0.. of C's FVI
//       times 16 rows — and runs, per k16 step, AR mma.sync m16n8k16 BF16 -> FP32 blocks (one
//       per a value) with A fragments from the ring (ldmatrix; .trans when X's FVI is an m
//       index) and B fragments from Y, which stays whole in shared memory;
//   (4) accumulator element (row, n) of the AR blocks is the run C[a0 .. a0+AR-1, row, n]:
//       alpha, RNE to BF16 and one 8- or 16-B streaming store per run straight from registers
//        — no transpose, no staging, no block-wide barrier.
// Persistent CTAs walk the tiles with C's FVI tile fastest, so neighbouring CTAs complete the
// same C lines at the same time.
#pragma once
#include <cuda_bf16.h>
#include <cstdint>

#include "kernel_f64.cuh"   // mbarrier / TMA helpers
#include "stream.hpp"

namespace tc {

__device__ __forceinline__ void ldsm_x4(uint32_t addr, uint32_t (&r)[4]) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];\n"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "r"(addr) : "memory");
}
__device__ __forceinline__ void ldsm_x4_t(uint32_t addr, uint32_t (&r)[4]) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];\n"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "r"(addr) : "memory");
}
__device__ __forceinline__ void ldsm_x2(uint32_t addr, uint32_t &r0, uint32_t &r1) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x2.shared.b16 {%0,%1}, [%2];\n" : "=r"(r0), "=r"(r1) : "r"(addr) : "memory");
}
__device__ __forceinline__ void mma_bf16_16816(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
  asm("mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};\n"
      : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
__device__ __forceinline__ uint32_t pack_bf16(float lo, float hi) {
  const __nv_bfloat162 v = __floats2bfloat162_rn(lo, hi);
  return *reinterpret_cast<const uint32_t *>(&v);
}

// a TMA box's swizzle: 16-B chunks XOR address bits 7.. under mask m (0 none, 1 32B, 3 64B, 7 128B)
__device__ __forceinline__ uint32_t s_swz(uint32_t off, int m) { return off ^ (((off >> 7) & (uint32_t)m) << 4); }

// tile t -> origin per m dim (raster order, C's FVI fastest)
__device__ __forceinline__ void s_tile(const SParams &p, int t, int32_t (&o)[kSMaxMdims]) {
#pragma unroll
  for (int d = 0; d < kSMaxMdims; d++) {
    o[d] = 0;
    if (d < p.nmd) {
      const int n = p.mNt[d];
      const int q = t / n;
      o[d] = (t - q * n) * p.mT[d];
      t = q;
    }
  }
}

// Ablation side builds only (tools/stream_ablation.py compiles libtc with -DTC_STREAM_ABLATE=k;
// the shipped library has kSAbl = 0): 1 = no MMAs, 2 = no C stores, 3 = neither (the X stream alone).
#ifdef TC_STREAM_ABLATE
constexpr int kSAbl = TC_STREAM_ABLATE;
#else
constexpr int kSAbl = 0;
#endif

// The TMA producer (one thread): for every tile of this CTA and every k-step, one X box into the
// next ring stage once the compute warps have released it
__device__ __forceinline__ void s_produce(const SParams &p, int ntl, uint32_t sbase, uint32_t FULL, uint32_t EMPTY) {
  uint64_t policy;   // X is read once: keep it from displacing C lines being completed in L2
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;\n" : "=l"(policy));
  int s = 0;
  uint32_t ph = 0;
  for (int lt = 0; lt < ntl; lt++) {
    int32_t o[kSMaxMdims];
    s_tile(p, (int)blockIdx.x + lt * (int)gridDim.x, o);
    int32_t c[kMaxTmaDims];
#pragma unroll
    for (int j = 0; j < kMaxTmaDims; j++) {
      int32_t v = 0;
#pragma unroll
      for (int d = 0; d < kSMaxMdims; d++) v = (d < p.nmd && p.mX[d] == j) ? o[d] : v;
      c[j] = v;
    }
    for (int ks = 0; ks < p.nks; ks++) {
      mbar_wait(EMPTY + 8 * s, ph ^ 1);   // (passes at once on the ring's first lap)
      mbar_expect_tx(FULL + 8 * s, (uint32_t)p.stage_bytes);
#pragma unroll
      for (int j = 0; j < kMaxTmaDims; j++)
        if (j == p.kX) c[j] = ks * p.KB;
      tma_load(&p.xmap, p.xrank, c[0], c[1], c[2], c[3], c[4], sbase + (uint32_t)(s * p.stage_pitch),
               FULL + 8 * s, policy);
      if (++s == p.stages) { s = 0; ph ^= 1; }
    }
  }
}

// byte address in the C box of byte offset b: its 16-B chunk ch moved to ch ^ (fold(ch >> 3) & 7),
// fold(x) = x ^ x >> s1 ^ x >> s2 (stream.cpp picks s1, s2 by simulating the writes)
__device__ __forceinline__ uint32_t s_cswzb(uint32_t b, int s1, int s2) {
  const uint32_t ch = b >> 4, x = ch >> 3;
  return ((ch ^ ((x ^ (x >> s1) ^ (x >> s2)) & 7u)) << 4) | (b & 15u);
}

// beta != 0 (FP64 / FP32 C): the staged alpha * sum plus beta * the old C, one fma per element
// (the tile kernels' order); beta == 0 never reads C (R26)
// (register arithmetic on the words: no address of a chunk is taken, which would move it to
//  local memory)
__device__ __forceinline__ uint4 s_beta(uint4 v, uint4 o, double beta, const double *) {
  const double a0 = fma(beta, __hiloint2double((int)o.y, (int)o.x), __hiloint2double((int)v.y, (int)v.x));
  const double a1 = fma(beta, __hiloint2double((int)o.w, (int)o.z), __hiloint2double((int)v.w, (int)v.z));
  return make_uint4((uint32_t)__double2loint(a0), (uint32_t)__double2hiint(a0), (uint32_t)__double2loint(a1),
                    (uint32_t)__double2hiint(a1));
}
__device__ __forceinline__ uint4 s_beta(uint4 v, uint4 o, double beta, const float *) {
  const float bt = (float)beta;
  return make_uint4(__float_as_uint(fmaf(bt, __uint_as_float(o.x), __uint_as_float(v.x))),
                    __float_as_uint(fmaf(bt, __uint_as_float(o.y), __uint_as_float(v.y))),
                    __float_as_uint(fmaf(bt, __uint_as_float(o.z), __uint_as_float(v.z))),
                    __float_as_uint(fmaf(bt, __uint_as_float(o.w), __uint_as_float(v.w))));
}
__device__ __forceinline__ uint4 s_beta(uint4 v, uint4, double, const __nv_bfloat16 *) { return v; }

// beta != 0, interior tile: four chunks' old C in flight per thread before their stores
template <typename TE>
__device__ __forceinline__ void s_store_box_beta(const SParams &p, TE *Ct, const unsigned char *sb, const uint32_t *ctab,
                                              int tid, int nthr) {
  for (int c0 = tid; c0 < p.nchunk; c0 += 4 * nthr) {
    uint4 o[4];
    TE *d[4];
#pragma unroll
    for (int i = 0; i < 4; i++) {
      const int ch = c0 + i * nthr;
      d[i] = Ct + (int32_t)ctab[ch < p.nchunk ? ch : 0];
      if (ch < p.nchunk) o[i] = __ldcs(reinterpret_cast<const uint4 *>(d[i]));
    }
#pragma unroll
    for (int i = 0; i < 4; i++) {
      const int ch = c0 + i * nthr;
      if (ch < p.nchunk) {
        const uint4 v = *reinterpret_cast<const uint4 *>(sb + s_cswzb((uint32_t)ch * 16u, p.cs1, p.cs2));
        __stcs(reinterpret_cast<uint4 *>(d[i]), s_beta(v, o[i], p.beta, (const TE *)nullptr));
      }
    }
  }
}

// The C box (smem, C order) leaves as 16-B runs along C's FVI: chunk c at ctab[c] elements from
// the tile origin.  Interior tiles store every chunk; tiles on the tensor's edge store what lies
// inside (every coordinate below its limit).
template <typename TE, bool BETA>
__device__ __forceinline__ void s_store_box(const SParams &p, TE *C, const unsigned char *sm, uint32_t stg_off,
                                            const uint32_t *ctab, int t, int tid, int nthr, int NB) {
  constexpr int EPC = 16 / (int)sizeof(TE);   // elements per chunk
  int64_t corg = 0;
  uint32_t lims = 0;
  bool interior = p.N == 8 * NB;
#pragma unroll
  for (int d = 0; d < kSMaxMdims; d++) {
    if (d < p.nmd) {
      const int n = p.mNt[d];
      const int qd = t / n;
      const int od = (t - qd * n) * p.mT[d];
      t = qd;
      const int l = min(p.mT[d], p.mN[d] - od);
      interior &= l == p.mT[d];
      lims |= (uint32_t)l << (8 * d);
      corg += (int64_t)od * p.mCs[d];
    }
  }
  TE *Ct = C + corg;
  const unsigned char *sb = sm + stg_off;
  if (BETA && interior) {
    s_store_box_beta<TE>(p, Ct, sb, ctab, tid, nthr);
    return;
  }
  for (int ch = tid; ch < p.nchunk; ch += nthr) {
    const uint4 v = *reinterpret_cast<const uint4 *>(sb + s_cswzb((uint32_t)ch * 16u, p.cs1, p.cs2));
    TE *dst = Ct + (int32_t)ctab[ch];
    if (interior) {
      __stcs(reinterpret_cast<uint4 *>(dst), v);
      continue;
    }
    int rem = ch, c0 = 0;
    bool ok = true;
#pragma unroll
    for (int j2 = 0; j2 < kMaxTmaDims; j2++) {
      if (j2 < p.crank) {
        const int ext = j2 == 0 ? p.cbox[0] / EPC : p.cbox[j2];
        const int cj = rem % ext;
        rem /= ext;
        const int lim = p.cmd[j2] < 0 ? p.N : (int)((lims >> (8 * p.cmd[j2])) & 0xFF);
        if (j2 == 0) c0 = EPC * cj;
        else ok &= cj < lim;
      }
    }
    const int lim0 = p.cmd[0] < 0 ? p.N : (int)((lims >> (8 * p.cmd[0])) & 0xFF);
    const int ne = ok ? max(0, min(EPC, lim0 - c0)) : 0;
    if (ne == EPC) {
      __stcs(reinterpret_cast<uint4 *>(dst),
             BETA ? s_beta(v, __ldcs(reinterpret_cast<const uint4 *>(dst)), p.beta, (const TE *)nullptr) : v);
    } else {
      // (elements picked out of the registers: taking v's address would put every chunk of
      //  every tile through local memory)
#pragma unroll
      for (int q2 = 0; q2 < EPC; q2++) {
        if (q2 < ne) {
          const uint32_t w = q2 * (int)sizeof(TE) / 4 == 0 ? v.x : q2 * (int)sizeof(TE) / 4 == 1 ? v.y
                           : q2 * (int)sizeof(TE) / 4 == 2 ? v.z : v.w;
          if constexpr (sizeof(TE) == 2) {
            const unsigned short h = (unsigned short)(q2 & 1 ? w >> 16 : w & 0xFFFFu);
            reinterpret_cast<unsigned short *>(dst)[q2] = h;
          } else if constexpr (sizeof(TE) == 4) {
            const float e = __uint_as_float(w);
            dst[q2] = BETA ? fmaf((float)p.beta, dst[q2], e) : e;
          } else {
            const uint32_t w2 = q2 == 0 ? v.y : v.w;   // (high words of the two doubles)
            const double e = __hiloint2double((int)w2, (int)w);
            dst[q2] = BETA ? fma(p.beta, dst[q2], e) : e;
          }
        }
      }
    }
  }
}

template <int NB, int AR, bool TRANS>
__global__ void __launch_bounds__(kSThreads, stream_occ(NB, AR)) tc_stream_bf16_kernel(const __grid_constant__ SParams p) {
  extern __shared__ __align__(1024) unsigned char smem_dyn[];
  unsigned char *sm = smem_dyn + ((1024u - ((uint32_t)__cvta_generic_to_shared(smem_dyn) & 1023u)) & 1023u);
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(sm);
  const uint32_t FULL = sbase + p.off_bar, EMPTY = FULL + 8 * p.stages;
  const uint32_t YS = sbase + p.off_y;
  uint32_t *tab = reinterpret_cast<uint32_t *>(sm + p.off_tab);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int ntl = (p.ntiles - (int)blockIdx.x + (int)gridDim.x - 1) / (int)gridDim.x;

  // ---- once per CTA: Y as [n][k] (k contiguous, pitch YP; zero past N and K), the tables
  {
    const __nv_bfloat16 *Y = static_cast<const __nv_bfloat16 *>(p.Y);
    __nv_bfloat16 *ys = reinterpret_cast<__nv_bfloat16 *>(sm + p.off_y);
    const int tot = 8 * NB * p.YP;
    for (int i = tid; i < tot; i += kSThreads) {
      const int n = i / p.YP, k = i - n * p.YP;
      ys[i] = (n < p.N && k < p.K) ? Y[(int64_t)k * p.ysk + (int64_t)n * p.ysn] : __float2bfloat16_rn(0.f);
    }
    for (int i = tid; i < p.nunits * 2 * p.ru + p.nchunk; i += kSThreads) tab[i] = __ldg(p.tab + i);
  }
  if (tid == 0) {
    for (int s = 0; s < p.stages; s++) {
      mbar_init(FULL + 8 * s, 1);          // the TMA thread (+ the box bytes)
      mbar_init(EMPTY + 8 * s, p.nunits);  // one arrive per working compute warp
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();

  if (warp == kSWarps) {
    // ======================= TMA producer ===================================================
    if (lane == 0) s_produce(p, ntl, sbase, FULL, EMPTY);
    return;
  }
  if (warp >= p.nunits) return;

  // ======================= compute warps: unit `warp` of every tile =========================
  const uint32_t *ut = tab + warp * 2 * kSRows;
  const int q = lane >> 3, r = lane & 7, g = lane >> 2, t4 = lane & 3;
  // ldmatrix row address in a stage (a0, k = 0): .trans rows are k (16 B of 8 consecutive E of
  // the row octet q & 1); plain rows are the unit's rows (16 B of 8 consecutive k)
  const uint32_t xr = TRANS ? ut[8 * (q & 1)] + (uint32_t)((r + 8 * (q >> 1)) * p.xpitchk)
                            : ut[r + 8 * (q & 1)] + (uint32_t)(16 * (q >> 1));
  const int xsw = p.xswz;   // the X box's TMA swizzle (conflict-free ldmatrix rows)
  const uint32_t kstep16 = TRANS ? (uint32_t)(16 * p.xpitchk) : 32u;
  const uint32_t xpa = (uint32_t)p.xpitcha;
  // this thread's two accumulator rows g and g + 8: C offsets (tile origin, a0) and coordinates
  const uint32_t bo0 = ut[kSRows + g], bo1 = ut[kSRows + 8 + g];   // C box offsets of rows g, g + 8
  const uint32_t *ctab = tab + p.nunits * 2 * kSRows;
  const uint32_t STG = sbase + p.off_stg;
  const int nthr = p.nunits * 32;   // the working compute threads
  // B fragments: ldmatrix rows n, 8 k per row
  const uint32_t ybq = YS + (uint32_t)(((q >> 1) * 8 + r) * p.YP * 2 + 16 * (q & 1));
  const float alpha = p.alpha;
  __nv_bfloat16 *C = static_cast<__nv_bfloat16 *>(p.C);
  int s = 0;
  uint32_t ph = 0;
  for (int lt = 0; lt < ntl; lt++) {
    float acc[AR][NB][4];
#pragma unroll
    for (int j = 0; j < AR; j++)
#pragma unroll
      for (int n = 0; n < NB; n++)
#pragma unroll
        for (int e = 0; e < 4; e++) acc[j][n][e] = 0.f;
    for (int ks = 0; ks < p.nks; ks++) {
      mbar_wait(FULL + 8 * s, ph);
      const uint32_t xs = sbase + (uint32_t)(s * p.stage_pitch);
      const int k0 = ks * p.KB;
      const int nk16 = min(p.KB, p.KP - k0) >> 4;
      for (int kk = 0; kk < ((kSAbl & 1) ? 0 : nk16); kk++) {
        uint32_t bf[NB][2];
        const uint32_t yb = ybq + (uint32_t)(2 * (k0 + 16 * kk));
#pragma unroll
        for (int n = 0; n + 1 < NB; n += 2) {
          uint32_t v[4];
          ldsm_x4(yb + (uint32_t)(n * 8 * p.YP * 2), v);
          bf[n][0] = v[0]; bf[n][1] = v[1]; bf[n + 1][0] = v[2]; bf[n + 1][1] = v[3];
        }
        if (NB & 1) ldsm_x2(yb + (uint32_t)((NB - 1) * 8 * p.YP * 2), bf[NB - 1][0], bf[NB - 1][1]);
        const uint32_t xa = xr + (uint32_t)kk * kstep16;
#pragma unroll
        for (int j = 0; j < AR; j++) {
          uint32_t af[4];
          const uint32_t ad = xs + s_swz(xa + (uint32_t)j * xpa, xsw);
          if (TRANS) ldsm_x4_t(ad, af);
          else ldsm_x4(ad, af);
#pragma unroll
          for (int n = 0; n < NB; n++) mma_bf16_16816(acc[j][n], af, bf[n][0], bf[n][1]);
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(EMPTY + 8 * s);
      if (++s == p.stages) { s = 0; ph ^= 1; }
    }
    // ---- epilogue: runs of AR values of C's FVI straight from the accumulators into the C box
    // (smem, C order, swizzled 16-B chunks), then the whole box out as 16-B runs along C's FVI
    const int t = (int)blockIdx.x + lt * (int)gridDim.x;
    // one C box: wait until the previous tile's box has been stored; two boxes: this tile's box
    // was last read by tile lt - 2's stores, which every warp finished before the barrier below
    // of tile lt - 1
    const uint32_t STGb = STG + (p.nstg == 2 ? (uint32_t)((lt & 1) * p.stg_pitch) : 0u);
    if (p.nstg == 1) consumer_sync(nthr);
    if (!(kSAbl & 2)) {
#pragma unroll
      for (int h = 0; h < 2; h++)
#pragma unroll
        for (int n = 0; n < NB; n++)
#pragma unroll
          for (int c2 = 0; c2 < 2; c2++) {
            const uint32_t boh = h ? bo1 : bo0;
            if (boh == 0xFFFFFFFFu) continue;   // a padding row
            const uint32_t el = boh + (uint32_t)((8 * n + 2 * t4 + c2) * p.cbsn);
            const uint32_t ad = STGb + s_cswzb(2u * el, p.cs1, p.cs2);
            if constexpr (AR == 8) {
              asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};\n" ::"r"(ad),
                           "r"(pack_bf16(alpha * acc[0][n][2 * h + c2], alpha * acc[1][n][2 * h + c2])),
                           "r"(pack_bf16(alpha * acc[2][n][2 * h + c2], alpha * acc[3][n][2 * h + c2])),
                           "r"(pack_bf16(alpha * acc[4][n][2 * h + c2], alpha * acc[5][n][2 * h + c2])),
                           "r"(pack_bf16(alpha * acc[6][n][2 * h + c2], alpha * acc[7][n][2 * h + c2]))
                           : "memory");
            } else {
              asm volatile("st.shared.v2.b32 [%0], {%1,%2};\n" ::"r"(ad),
                           "r"(pack_bf16(alpha * acc[0][n][2 * h + c2], alpha * acc[1][n][2 * h + c2])),
                           "r"(pack_bf16(alpha * acc[2][n][2 * h + c2], alpha * acc[3][n][2 * h + c2]))
                           : "memory");
            }
          }
    }
    consumer_sync(nthr);   // the box is complete
    if (!(kSAbl & 2)) s_store_box<__nv_bfloat16, false>(p, C, sm, STGb - sbase, ctab, t, tid, nthr, NB);
  }
}


// ============================================================================================
// FP64 (the paper's precision): the same streaming structure with DMMA m8n8k4 register blocks.
// A unit is AR consecutive values of C's FVI times 8 rows (SM_T: one octet of X's FVI; SM_K:
// 8 rows of the other m dims); thread (g, t) loads A(row g, k t) and B(k t, n g) as doubles
// straight from the (swizzled) stage and from Y, and holds C(row g, n 2t / 2t+1) of each of its
// AR blocks: the run C[a0 .. a0+AR-1, row g, n].
template <int NB, int AR, bool TRANS, bool BETA>
__global__ void __launch_bounds__(kSThreads, stream_occ(NB, AR)) tc_stream_f64_kernel(const __grid_constant__ SParams p) {
  extern __shared__ __align__(1024) unsigned char smem_dyn[];
  unsigned char *sm = smem_dyn + ((1024u - ((uint32_t)__cvta_generic_to_shared(smem_dyn) & 1023u)) & 1023u);
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(sm);
  const uint32_t FULL = sbase + p.off_bar, EMPTY = FULL + 8 * p.stages;
  uint32_t *tab = reinterpret_cast<uint32_t *>(sm + p.off_tab);
  double *ys = reinterpret_cast<double *>(sm + p.off_y);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int ntl = (p.ntiles - (int)blockIdx.x + (int)gridDim.x - 1) / (int)gridDim.x;
  {
    const double *Y = static_cast<const double *>(p.Y);
    const int tot = 8 * NB * p.YP;
    for (int i = tid; i < tot; i += kSThreads) {
      const int n = i / p.YP, k = i - n * p.YP;
      ys[i] = (n < p.N && k < p.K) ? Y[(int64_t)k * p.ysk + (int64_t)n * p.ysn] : 0.0;
    }
    for (int i = tid; i < p.nunits * 2 * p.ru + p.nchunk; i += kSThreads) tab[i] = __ldg(p.tab + i);
  }
  if (tid == 0) {
    for (int s = 0; s < p.stages; s++) {
      mbar_init(FULL + 8 * s, 1);
      mbar_init(EMPTY + 8 * s, p.nunits);
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();
  if (warp == kSWarps) {
    if (lane == 0) s_produce(p, ntl, sbase, FULL, EMPTY);
    return;
  }
  if (warp >= p.nunits) return;
  const uint32_t *ut = tab + warp * 2 * 8;
  const int g = lane >> 2, t4 = lane & 3;
  // A(row g, k t4) in a stage (a0, k-step origin): SM_T rows are 8 consecutive E (8 B apart)
  // of the unit's octet, k rows xpitchk apart; SM_K rows are the unit's rows, k contiguous
  // k of thread t in DMMA step kk: SM_T takes k = 8 (kk / 2) + kk % 2 + 2 t (every other k row,
  // so the four k rows of one step fall in different swizzle phases of the 128-B box rows: no
  // bank conflicts); SM_K the plain k = 4 kk + t (rows are m rows there)
  const uint32_t xks = TRANS ? (uint32_t)p.xpitchk : 8u;   // bytes per k in the stage
  const int lk = TRANS ? 2 * t4 : t4;
  const uint32_t xr = ut[g] + (uint32_t)lk * xks;
  const uint32_t xpa = (uint32_t)p.xpitcha;
  const int xsw = p.xswz;
  const uint32_t bo = ut[8 + g];
  const uint32_t *ctab = tab + p.nunits * 2 * 8;
  const uint32_t STG = sbase + p.off_stg;
  const int nthr = p.nunits * 32;
  const double *yb0 = ys + g * p.YP + lk;
  const double alpha = p.alpha64;
  double *C = static_cast<double *>(p.C);
  int s = 0;
  uint32_t ph = 0;
  for (int lt = 0; lt < ntl; lt++) {
    double acc[AR][NB][2];
#pragma unroll
    for (int j = 0; j < AR; j++)
#pragma unroll
      for (int n = 0; n < NB; n++) acc[j][n][0] = acc[j][n][1] = 0.0;
    for (int ks = 0; ks < p.nks; ks++) {
      mbar_wait(FULL + 8 * s, ph);
      const unsigned char *xs = sm + (uint32_t)(s * p.stage_pitch);
      const int k0 = ks * p.KB;
      const int nk4 = min(p.KB, p.KP - k0) >> 2;
      for (int kk = 0; kk < ((kSAbl & 1) ? 0 : nk4); kk++) {
        const int kofs = TRANS ? 8 * (kk >> 1) + (kk & 1) : 4 * kk;
        double bf[NB];
#pragma unroll
        for (int n = 0; n < NB; n++) bf[n] = yb0[n * 8 * p.YP + k0 + kofs];
        const uint32_t xa = xr + (uint32_t)kofs * xks;
#pragma unroll
        for (int j = 0; j < AR; j++) {
          const double av = *reinterpret_cast<const double *>(xs + s_swz(xa + (uint32_t)j * xpa, xsw));
#pragma unroll
          for (int n = 0; n < NB; n++) dmma884(acc[j][n][0], acc[j][n][1], av, bf[n]);
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(EMPTY + 8 * s);
      if (++s == p.stages) { s = 0; ph ^= 1; }
    }
    const int t = (int)blockIdx.x + lt * (int)gridDim.x;
    const uint32_t STGb = STG + (p.nstg == 2 ? (uint32_t)((lt & 1) * p.stg_pitch) : 0u);
    if (p.nstg == 1) consumer_sync(nthr);
    if (!(kSAbl & 2) && bo != 0xFFFFFFFFu) {
#pragma unroll
      for (int n = 0; n < NB; n++)
#pragma unroll
        for (int c2 = 0; c2 < 2; c2++) {
          const uint32_t b = 8u * (bo + (uint32_t)((8 * n + 2 * t4 + c2) * p.cbsn));
          if (p.cbsj == 1) {   // the AR values are consecutive along C's FVI: 16-B pairs
#pragma unroll
            for (int j = 0; j < AR; j += 2)
              asm volatile("st.shared.v2.f64 [%0], {%1,%2};\n" ::"r"(STGb + s_cswzb(b + 8u * j, p.cs1, p.cs2)),
                           "d"(alpha * acc[j][n][c2]), "d"(alpha * acc[j + 1][n][c2]) : "memory");
          } else {             // SM_M: runs along the 8 lanes of a row octet; the AR values apart
#pragma unroll
            for (int j = 0; j < AR; j++)
              asm volatile("st.shared.f64 [%0], %1;\n" ::"r"(STGb + s_cswzb(b + 8u * (uint32_t)(j * p.cbsj), p.cs1, p.cs2)),
                           "d"(alpha * acc[j][n][c2]) : "memory");
          }
        }
    }
    consumer_sync(nthr);
    if (!(kSAbl & 2)) s_store_box<double, BETA>(p, C, sm, STGb - sbase, ctab, t, tid, nthr, NB);
  }
}


// ============================================================================================
// FP32 storage: TF32 products (mma.sync m16n8k8 .tf32, the tensor core reads the FP32 bits,
// DESIGN R30) or FP32 as three TF32 products (SPLIT: hi = x & 0xFFFFE000, lo = x - hi;
// lo*hi + hi*lo + hi*hi, R32).  Same units, C runs and store phase as the BF16 kernel; the
// fragments are single 32-bit elements, loaded with plain shared loads (ldmatrix cannot
// transpose 32-bit elements).
__device__ __forceinline__ void mma_tf32_1688(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
  asm("mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};\n"
      : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
__device__ __forceinline__ uint32_t tf32_hi(uint32_t x) { return x & 0xFFFFE000u; }
__device__ __forceinline__ uint32_t tf32_lo(uint32_t x) {
  return __float_as_uint(__uint_as_float(x) - __uint_as_float(x & 0xFFFFE000u));
}

template <int NB, int AR, bool TRANS, bool SPLIT, bool BETA>
__global__ void __launch_bounds__(kSThreads, stream_occ(NB, AR)) tc_stream_tf32_kernel(const __grid_constant__ SParams p) {
  extern __shared__ __align__(1024) unsigned char smem_dyn[];
  unsigned char *sm = smem_dyn + ((1024u - ((uint32_t)__cvta_generic_to_shared(smem_dyn) & 1023u)) & 1023u);
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(sm);
  const uint32_t FULL = sbase + p.off_bar, EMPTY = FULL + 8 * p.stages;
  uint32_t *tab = reinterpret_cast<uint32_t *>(sm + p.off_tab);
  float *ys = reinterpret_cast<float *>(sm + p.off_y);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int ntl = (p.ntiles - (int)blockIdx.x + (int)gridDim.x - 1) / (int)gridDim.x;
  {
    const float *Y = static_cast<const float *>(p.Y);
    const int tot = 8 * NB * p.YP;
    for (int i = tid; i < tot; i += kSThreads) {
      const int n = i / p.YP, k = i - n * p.YP;
      ys[i] = (n < p.N && k < p.K) ? Y[(int64_t)k * p.ysk + (int64_t)n * p.ysn] : 0.f;
    }
    for (int i = tid; i < p.nunits * 2 * p.ru + p.nchunk; i += kSThreads) tab[i] = __ldg(p.tab + i);
  }
  if (tid == 0) {
    for (int s = 0; s < p.stages; s++) {
      mbar_init(FULL + 8 * s, 1);
      mbar_init(EMPTY + 8 * s, p.nunits);
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();
  if (warp == kSWarps) {
    if (lane == 0) s_produce(p, ntl, sbase, FULL, EMPTY);
    return;
  }
  if (warp >= p.nunits) return;
  const uint32_t *ut = tab + warp * 2 * kSRows;
  const int g = lane >> 2, t4 = lane & 3;
  const uint32_t xks = TRANS ? (uint32_t)p.xpitchk : 4u;   // bytes per k in the stage
  // A(row g | g + 8, k t4 | t4 + 4): the unit's rows g and g + 8
  const uint32_t xr0 = ut[g] + (uint32_t)t4 * xks, xr1 = ut[8 + g] + (uint32_t)t4 * xks;
  const uint32_t xpa = (uint32_t)p.xpitcha;
  const int xsw = p.xswz;
  const uint32_t bo0 = ut[kSRows + g], bo1 = ut[kSRows + 8 + g];
  const uint32_t *ctab = tab + p.nunits * 2 * kSRows;
  const uint32_t STG = sbase + p.off_stg;
  const int nthr = p.nunits * 32;
  const float *yb0 = ys + g * p.YP + t4;
  const float alpha = p.alpha;
  float *C = static_cast<float *>(p.C);
  int s = 0;
  uint32_t ph = 0;
  for (int lt = 0; lt < ntl; lt++) {
    float acc[AR][NB][4];
#pragma unroll
    for (int j = 0; j < AR; j++)
#pragma unroll
      for (int n = 0; n < NB; n++)
#pragma unroll
        for (int e = 0; e < 4; e++) acc[j][n][e] = 0.f;
    for (int ks = 0; ks < p.nks; ks++) {
      mbar_wait(FULL + 8 * s, ph);
      const unsigned char *xs = sm + (uint32_t)(s * p.stage_pitch);
      const int k0 = ks * p.KB;
      const int nk8 = min(p.KB, p.KP - k0) >> 3;
      for (int kk = 0; kk < ((kSAbl & 1) ? 0 : nk8); kk++) {
        uint32_t bh[NB][2], bl[NB][2];
#pragma unroll
        for (int n = 0; n < NB; n++) {
          const float *yb = yb0 + n * 8 * p.YP + k0 + 8 * kk;
          const uint32_t v0 = __float_as_uint(yb[0]), v1 = __float_as_uint(yb[4]);
          bh[n][0] = SPLIT ? tf32_hi(v0) : v0;
          bh[n][1] = SPLIT ? tf32_hi(v1) : v1;
          if (SPLIT) { bl[n][0] = tf32_lo(v0); bl[n][1] = tf32_lo(v1); }
        }
        const uint32_t ko = (uint32_t)(8 * kk) * xks, ko4 = ko + 4u * xks;
#pragma unroll
        for (int j = 0; j < AR; j++) {
          const uint32_t jo = (uint32_t)j * xpa;
          uint32_t a[4] = {*reinterpret_cast<const uint32_t *>(xs + s_swz(xr0 + jo + ko, xsw)),
                           *reinterpret_cast<const uint32_t *>(xs + s_swz(xr1 + jo + ko, xsw)),
                           *reinterpret_cast<const uint32_t *>(xs + s_swz(xr0 + jo + ko4, xsw)),
                           *reinterpret_cast<const uint32_t *>(xs + s_swz(xr1 + jo + ko4, xsw))};
          if (SPLIT) {
            uint32_t ah[4], al[4];
#pragma unroll
            for (int e = 0; e < 4; e++) { ah[e] = tf32_hi(a[e]); al[e] = tf32_lo(a[e]); }
#pragma unroll
            for (int n = 0; n < NB; n++) {   // small terms first: lo*hi, hi*lo, then hi*hi
              mma_tf32_1688(acc[j][n], al, bh[n][0], bh[n][1]);
              mma_tf32_1688(acc[j][n], ah, bl[n][0], bl[n][1]);
              mma_tf32_1688(acc[j][n], ah, bh[n][0], bh[n][1]);
            }
          } else {
#pragma unroll
            for (int n = 0; n < NB; n++) mma_tf32_1688(acc[j][n], a, bh[n][0], bh[n][1]);
          }
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(EMPTY + 8 * s);
      if (++s == p.stages) { s = 0; ph ^= 1; }
    }
    const int t = (int)blockIdx.x + lt * (int)gridDim.x;
    const uint32_t STGb = STG + (p.nstg == 2 ? (uint32_t)((lt & 1) * p.stg_pitch) : 0u);
    if (p.nstg == 1) consumer_sync(nthr);
    if (!(kSAbl & 2)) {
#pragma unroll
      for (int h = 0; h < 2; h++)
#pragma unroll
        for (int n = 0; n < NB; n++)
#pragma unroll
          for (int c2 = 0; c2 < 2; c2++) {
            const uint32_t boh = h ? bo1 : bo0;
            if (boh == 0xFFFFFFFFu) continue;   // a padding row
            const uint32_t b = 4u * (boh + (uint32_t)((8 * n + 2 * t4 + c2) * p.cbsn));
#pragma unroll
            for (int j = 0; j < AR; j += 4)
              asm volatile("st.shared.v4.f32 [%0], {%1,%2,%3,%4};\n" ::"r"(STGb + s_cswzb(b + 4u * j, p.cs1, p.cs2)),
                           "f"(alpha * acc[j][n][2 * h + c2]), "f"(alpha * acc[j + 1][n][2 * h + c2]),
                           "f"(alpha * acc[j + 2][n][2 * h + c2]), "f"(alpha * acc[j + 3][n][2 * h + c2])
                           : "memory");
          }
    }
    consumer_sync(nthr);
    if (!(kSAbl & 2)) s_store_box<float, BETA>(p, C, sm, STGb - sbase, ctab, t, tid, nthr, NB);
  }
}

}  // namespace tc
