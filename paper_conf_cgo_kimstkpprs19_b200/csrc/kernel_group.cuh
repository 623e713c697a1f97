// kernel_group.cuh — the fused grouped FP64 contraction kernel (group.hpp).
//
// The CCSD(T) triples (9 sd_t_d1 + 9 sd_t_d2 contractions, all adding into
// one t3) run as one persistent kernel.  Per C tile (a hyper-rectangle prod_p T_p of t3,
// P:L119), for every member i in turn:
//   (1) PRODUCER warps gather member i's X_i tile (Mt_i x Kt_i) and Y_i tile (Kt_i x Nt_i)
//       of each k-step with cp.async into a STAGES-deep ring (the paper's step 1),
//       walking each operand in its own memory order by runs along its FVI;
//       zero-fill outside the tensors;
//   (2)+(3) CONSUMER warps multiply with DMMA m8n8k4 register tiles (steps 2-3)
//       exactly as the single-contraction kernel (kernel_f64.cuh), the smem layout (k- or
//       mn-major per operand) chosen per member at run time;
//   then the member's accumulators are added into the C tile's XOR-swizzled smem box (the
//   digit orders of the member's rows / columns make this conflict-free, group.cpp).
// After the last member the box leaves for C once: C = alpha * box + beta * C (step 4,
// P:L84) — t3 is written once instead of 18 times, and read once when beta != 0.
#pragma once
#include <cstdint>

#include "group.hpp"
#include "kernel_f64.cuh"

namespace tc {

struct GParams {
  const double *X[kGMaxMembers];   // per member: its X / Y operand (A or B, group.hpp)
  const double *Y[kGMaxMembers];
  uint64_t vecmask;                // bit 2i: X_i may use 16-B vectors; bit 2i+1: Y_i
  double *C;
  double alpha, beta;
  int nmem, rank, ntiles, nunits;
  int uvec;                        // C elements per copy-out unit (1 or 2, group.cpp)
  int cvec16;                      // 1: units of 2 are stored as one 16-B vector (C aligned)
  int32_t ntl[kGMaxCdims];
  int64_t cstep[kGMaxCdims];       // T_p * C stride of position p
  int64_t N[kGMaxCdims];
  int32_t T[kGMaxCdims];
  int64_t cbase;
  uint64_t Tpack;                  // T_p as bytes: the limits of an interior tile
  const GMemberDev *mem;
  const GStepDev *steps;
  const int32_t *runRel;
  const uint32_t *runSoff;
  const uint64_t *runDig;
  const uint32_t *pad;
  const int32_t *boxM, *boxN;
  const int64_t *unitRel;
  const uint64_t *unitDig;
};

template <int BK, int STAGES>
struct GroupCfg {
  static constexpr int BM = kGBM, BN = kGBN, WM = 32, WN = 32;
  static constexpr int CW = 4, PW = 4;                      // consumer / producer warps
  static constexpr int THREADS = (CW + PW) * 32;
  static constexpr int PM = BM + 4, PN = BN + 4, PK = BK + 4;
  static constexpr int XS = (BM * PK > BK * PM ? BM * PK : BK * PM) + 2;   // = gplane_doubles
  static constexpr int YS = (BN * PK > BK * PN ? BN * PK : BK * PN) + 2;
  static constexpr int BOX = BM * BN;
  static constexpr size_t smem_bytes() { return 8 * ((size_t)STAGES * (XS + YS) + BOX) + 16 * STAGES; }
  static_assert(BK % 4 == 0 && BK <= 32, "BK");
};

// SWAR: every byte selected by maskH (0x80 per used byte) has dig < lim (bytes < 128)
__device__ __forceinline__ bool g_all_lt(uint64_t dig, uint64_t lim, uint64_t maskH) {
  const uint64_t H = 0x8080808080808080ull, L1 = 0x0101010101010101ull;
  return ((((lim | H) - dig - L1) & maskH) == maskH);
}

// this operand's per-dim limits for the tile: byte j = limit of the C position of dim j
__device__ __forceinline__ uint64_t g_op_lims(const GOperandDev &op, uint64_t Lc) {
  uint64_t L = 0;
#pragma unroll
  for (int j = 0; j < kGMaxOpDims; j++) {
    const int cp = op.cpos[j];
    if (j < op.ndim && cp >= 0) L |= ((Lc >> (8 * cp)) & 0xFF) << (8 * j);
  }
  return L;
}

// Gather one operand tile (one k-step) into a stage plane: vector w = pt + 128 i is vector v
// of run q; runs lie along the operand's FVI, consecutive threads take consecutive vectors.
__device__ __forceinline__ void g_gather(const GParams &p, const double *__restrict__ base, uint32_t sdst,
                                         const GOperandDev &op, int vec, int pt, bool fast, uint64_t L) {
  const int vpr = op.runlen / vec;
  const int nvec = op.nrun * vpr;
  const int32_t *__restrict__ rr = p.runRel + op.run0;
  const uint32_t *__restrict__ rs = p.runSoff + op.run0;
  const uint64_t *__restrict__ rd = p.runDig + op.run0;
  int q = pt / vpr, v = pt - (pt / vpr) * vpr;
  const int dq = 128 / vpr, dv = 128 - (128 / vpr) * vpr;
  // bytes checked by SWAR: dims 1.. when runs cover dim 0, else every dim
  const int jfirst = op.runlen > 1 ? 1 : 0;
  uint64_t maskH = 0;
  for (int j = jfirst; j < op.ndim; j++) maskH |= 0x80ull << (8 * j);
  const int lim0 = (int)(L & 0xFF);
  for (int w = pt; w < nvec; w += 128) {
    const int rel = __ldg(rr + q) + v * vec;
    const uint32_t dst = sdst + 8u * (__ldg(rs + q) + (uint32_t)(v * vec));
    const double *src = base + rel;
    if (fast) {
      if (vec == 2) cp_async16_full(dst, src);
      else cp_async8_full(dst, src);
    } else {
      int nval = g_all_lt(__ldg(rd + q), L, maskH) ? vec : 0;
      if (op.runlen > 1) nval = min(nval, max(0, lim0 - v * vec));
      if (vec == 2) cp_async16(dst, nval ? src : base, 8 * nval);
      else cp_async8(dst, nval ? src : base, 8 * nval);
    }
    q += dq;
    v += dv;
    if (v >= vpr) { v -= vpr; q++; }
  }
}

// One k-step of one member on the consumer warps: DMMA over the stage (compile-time layouts).
template <int BK, bool XK, bool YK>
__device__ __forceinline__ void g_mma_step(double (&acc)[4][4][2], const double *__restrict__ xs,
                                           const double *__restrict__ ys, int wm, int wn, int g, int t) {
  constexpr int PK = BK + 4, PM = kGBM + 4, PN = kGBN + 4;
  const int aoff = XK ? (wm * 32 + g) * PK + t : t * PM + wm * 32 + g;
  const int boff = YK ? (wn * 32 + g) * PK + t : t * PN + wn * 32 + g;
  constexpr int AI = XK ? 8 * PK : 8, AK = XK ? 4 : 4 * PM;
  constexpr int BJ = YK ? 8 * PK : 8, BKs = YK ? 4 : 4 * PN;
#pragma unroll
  for (int kk = 0; kk < BK / 4; kk++) {
    double a[4], b[4];
#pragma unroll
    for (int i = 0; i < 4; i++) a[i] = xs[aoff + i * AI + kk * AK];
#pragma unroll
    for (int j = 0; j < 4; j++) b[j] = ys[boff + j * BJ + kk * BKs];
#pragma unroll
    for (int i = 0; i < 4; i++)
#pragma unroll
      for (int j = 0; j < 4; j++) dmma884(acc[i][j][0], acc[i][j][1], a[i], b[j]);
  }
}

// tile t -> C coordinates (position 0 fastest), packed limits, interior flag, C origin
struct GTile {
  int32_t c[kGMaxCdims];
  uint64_t Lc;
  bool interior;
  __device__ __forceinline__ void decode(const GParams &p, int t) {
    Lc = 0;
#pragma unroll
    for (int q = 0; q < kGMaxCdims; q++) {
      c[q] = 0;
      if (q < p.rank) {
        const int n = p.ntl[q];
        const int d = t / n;
        c[q] = t - d * n;
        t = d;
        const int64_t lim = min((int64_t)p.T[q], p.N[q] - (int64_t)c[q] * p.T[q]);
        Lc |= (uint64_t)lim << (8 * q);
      }
    }
    interior = Lc == p.Tpack;
  }
  __device__ __forceinline__ int64_t off(const int64_t *step, int rank) const {
    int64_t o = 0;
#pragma unroll
    for (int q = 0; q < kGMaxCdims; q++)
      if (q < rank) o += (int64_t)c[q] * step[q];
    return o;
  }
};

template <int BK, int STAGES>
__global__ void __launch_bounds__(GroupCfg<BK, STAGES>::THREADS, 2)
tc_f64_group_kernel(const __grid_constant__ GParams p) {
  using K = GroupCfg<BK, STAGES>;
  extern __shared__ __align__(1024) double smem[];
  // smem: [STAGES][X plane XS | Y plane YS], then the C box, then the barriers
  double *box = smem + STAGES * (K::XS + K::YS);
  uint64_t *bars = reinterpret_cast<uint64_t *>(box + K::BOX);   // full[S], empty[S]
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int ntl = (p.ntiles - (int)blockIdx.x + (int)gridDim.x - 1) / (int)gridDim.x;
  if (ntl <= 0) return;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(smem);
  const uint32_t bar0 = (uint32_t)__cvta_generic_to_shared(bars);
  constexpr uint32_t STAGE_BYTES = 8u * (K::XS + K::YS);

  // zero the ring once (rows / k positions a member does not write are never flushed, but
  // must not hold NaN patterns that reach a valid accumulator: k padding is re-zeroed per step)
  for (int i = tid; i < STAGES * (K::XS + K::YS); i += K::THREADS) smem[i] = 0.0;
  if (tid == 0) {
    for (int s = 0; s < STAGES; s++) {
      mbar_init(bar0 + 8 * s, K::PW * 32);
      mbar_init(bar0 + 8 * (STAGES + s), K::CW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();

  if (warp >= K::CW) {
    // ======================= producers ====================================================
    const int pt = tid - K::CW * 32;
    int j = 0;
    for (int lt = 0; lt < ntl; lt++) {
      GTile tile;
      tile.decode(p, (int)blockIdx.x + lt * (int)gridDim.x);
      for (int i = 0; i < p.nmem; i++) {
        const GMemberDev &M = p.mem[i];
        const double *__restrict__ Xb = p.X[i] + tile.off(M.x.tstep, p.rank);
        const double *__restrict__ Yb = p.Y[i] + tile.off(M.y.tstep, p.rank);
        const int vx = ((p.vecmask >> (2 * i)) & 1) ? M.x.vec : 1;
        const int vy = ((p.vecmask >> (2 * i + 1)) & 1) ? M.y.vec : 1;
        // (needed by partial k-steps of interior tiles too)
        const uint64_t Lx = g_op_lims(M.x, tile.Lc);
        const uint64_t Ly = g_op_lims(M.y, tile.Lc);
        for (int s = 0; s < M.nsteps; s++, j++) {
          const int st = j % STAGES;
          if (j >= STAGES) mbar_wait(bar0 + 8 * (STAGES + st), ((j / STAGES) & 1) ^ 1);
          const GStepDev &S = p.steps[M.step0 + s];
          const bool fast = tile.interior && S.full;
          const uint32_t dst = sbase + st * STAGE_BYTES;
          g_gather(p, Xb + S.kx, dst, M.x, vx, pt, fast, Lx | S.klimX);
          g_gather(p, Yb + S.ky, dst + 8u * K::XS, M.y, vy, pt, fast, Ly | S.klimY);
          for (int w = pt; w < M.npad; w += K::PW * 32) cp_async8(dst + __ldg(p.pad + M.pad0 + w), Xb, 0);
          mbar_arrive_cp_async(bar0 + 8 * st);
        }
      }
    }
    return;
  }

  // ======================= consumers ======================================================
  const int wm = warp & 1, wn = warp >> 1;
  const int g = lane >> 2, t = lane & 3;
  double acc[4][4][2];
#pragma unroll
  for (int i = 0; i < 4; i++)
#pragma unroll
    for (int jj = 0; jj < 4; jj++) acc[i][jj][0] = acc[i][jj][1] = 0.0;
  double *__restrict__ C = p.C;
  const double alpha = p.alpha, beta = p.beta;
  int j = 0;
  for (int lt = 0; lt < ntl; lt++) {
    for (int i = 0; i < p.nmem; i++) {
      const int layout = p.mem[i].layout, nsteps = p.mem[i].nsteps;
      for (int s = 0; s < nsteps; s++, j++) {
        const int st = j % STAGES;
        mbar_wait(bar0 + 8 * st, (j / STAGES) & 1);
        const double *xs = smem + st * (K::XS + K::YS);
        const double *ys = xs + K::XS;
        switch (layout) {
          case 0: g_mma_step<BK, false, false>(acc, xs, ys, wm, wn, g, t); break;
          case 1: g_mma_step<BK, true, false>(acc, xs, ys, wm, wn, g, t); break;
          case 2: g_mma_step<BK, false, true>(acc, xs, ys, wm, wn, g, t); break;
          default: g_mma_step<BK, true, true>(acc, xs, ys, wm, wn, g, t); break;
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(bar0 + 8 * (STAGES + st));
      }
      // ---- flush member i into the box (after every consumer finished the previous flush
      //      or the previous tile's copy-out: the box entries of two members differ per thread)
      const int32_t *bm = p.boxM + i * kGBM, *bn = p.boxN + i * kGBN;
      int rb[4], cb[4][2];
#pragma unroll
      for (int q = 0; q < 4; q++) rb[q] = __ldg(bm + wm * 32 + q * 8 + g);
#pragma unroll
      for (int q = 0; q < 4; q++) {
        cb[q][0] = __ldg(bn + wn * 32 + q * 8 + 2 * t);
        cb[q][1] = __ldg(bn + wn * 32 + q * 8 + 2 * t + 1);
      }
      consumer_sync(K::CW * 32);
#pragma unroll
      for (int a = 0; a < 4; a++)
#pragma unroll
        for (int b = 0; b < 4; b++)
#pragma unroll
          for (int h = 0; h < 2; h++) {
            if (rb[a] >= 0 && cb[b][h] >= 0) {
              const int o = gbox_sw(rb[a] + cb[b][h]);
              box[o] = i == 0 ? acc[a][b][h] : box[o] + acc[a][b][h];
            }
            acc[a][b][h] = 0.0;
          }
    }
    // ---- the tile leaves for C once: C = alpha * box + beta * C (beta == 0: C not read)
    consumer_sync(K::CW * 32);
    GTile tile;
    tile.decode(p, (int)blockIdx.x + lt * (int)gridDim.x);
    double *Ct = C + p.cbase + tile.off(p.cstep, p.rank);
    const uint64_t mH = (0x8080808080808080ull >> (8 * (8 - p.rank))) & ~0x80ull;   // positions 1..rank-1
    const int lim0 = (int)(tile.Lc & 0xFF);
    for (int u = tid; u < p.nunits; u += K::CW * 32) {
      const int o = u * p.uvec;
      double *dst = Ct + __ldg(p.unitRel + u);
      if (tile.interior && p.cvec16) {
        double2 v = make_double2(alpha * box[gbox_sw(o)], alpha * box[gbox_sw(o + 1)]);
        double2 *d2 = reinterpret_cast<double2 *>(dst);
        if (beta != 0.0) {
          const double2 old = *d2;
          v.x = fma(beta, old.x, v.x);
          v.y = fma(beta, old.y, v.y);
        }
        *d2 = v;
      } else {
        const uint64_t dg = __ldg(p.unitDig + u);
        const bool ok = tile.interior || g_all_lt(dg, tile.Lc, mH);
        const int d0 = (int)(dg & 0xFF);
        for (int e = 0; e < p.uvec; e++) {
          if (ok && (tile.interior || d0 + e < lim0)) {
            double v = alpha * box[gbox_sw(o + e)];
            if (beta != 0.0) v = fma(beta, dst[e], v);
            dst[e] = v;
          }
        }
      }
    }
  }
}

}  // namespace tc
