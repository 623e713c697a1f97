// kernel_f64.cuh — the FP64 direct-contraction kernel of libtc for sm_100a.
//
// The paper's four steps (Alg. 1) re-designed for B200:
//   (1) GMEM -> SMEM: the X tile (Mt x Kt) and Y tile (Kt x Nt) of one k-step are gathered
//       with cp.async (16-B when the operand's FVI allows, zero-fill outside the tensor),
//       walking each operand in its own memory order, into a STAGES-deep ring
//       (the paper's kernel was single-buffered with two syncs per step).
//   (2) SMEM -> REG: DMMA fragments (mma.sync.m8n8k4.f64 -> SASS DMMA.8x8x4; measured on
//       B200 at 37.1 TFLOP/s = the FP64 pipe's peak, profiles/r01_peaks.json).  The smem
//       pitch is 4 (mod 16) doubles so fragment loads are conflict-free in both layouts.
//   (3) outer product: each warp owns a WM x WN register tile of C (accumulate in
//       registers, not smem); the paper's r_C[T_b][T_c] of rank-1 updates becomes
//       (WM/8) x (WN/8) DMMA tiles per k4.
//   (4) REG -> GMEM: C = alpha * acc + beta * C through separable row / column offset
//       tables, predicated on the tensor bounds (correct for any size).
#pragma once
#include <cstdint>
#include "kparams.hpp"

namespace tc {

__device__ __forceinline__ void cp_async8(double *dst, const double *src, int srcbytes) {
  unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(d), "l"(src), "r"(srcbytes));
}
__device__ __forceinline__ void cp_async16(double *dst, const double *src, int srcbytes) {
  unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(d), "l"(src), "r"(srcbytes));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N)); }

__device__ __forceinline__ void dmma884(double &c0, double &c1, double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
               : "+d"(c0), "+d"(c1) : "d"(a), "d"(b));
}

template <int BM, int BN, int BK>
struct SmemLayout {
  static constexpr int PM = BM + 4, PN = BN + 4, PK = BK + 4;  // pitches, 4 mod 16 doubles
  static constexpr int XS = (BM * PK > BK * PM) ? BM * PK : BK * PM;
  static constexpr int YS = (BN * PK > BK * PN) ? BN * PK : BK * PN;
};

template <int BM, int BN, int BK, int WM, int WN, int STAGES>
struct F64Kernel {
  static constexpr int WARPS_M = BM / WM, WARPS_N = BN / WN;
  static constexpr int THREADS = WARPS_M * WARPS_N * 32;
  static constexpr int MI = WM / 8, NJ = WN / 8;
  static constexpr int EX = (BM * BK + THREADS - 1) / THREADS;
  static constexpr int EY = (BN * BK + THREADS - 1) / THREADS;
  using L = SmemLayout<BM, BN, BK>;
  static constexpr size_t smem_bytes() {
    return sizeof(double) * (size_t)STAGES * (L::XS + L::YS) + sizeof(int64_t) * 2 * (BM + BN);
  }
  static_assert(BK % 4 == 0 && BK <= 64, "BK");
  static_assert(WM % 8 == 0 && WN % 8 == 0, "warp tile");
  static_assert(BM <= 256 && BN <= 256, "slot packing");
};

template <int BM, int BN, int BK, int WM, int WN, int STAGES>
__global__ void __launch_bounds__(F64Kernel<BM, BN, BK, WM, WN, STAGES>::THREADS, 1)
tc_f64_dmma_kernel(const KParams p) {
  using K = F64Kernel<BM, BN, BK, WM, WN, STAGES>;
  using L = typename K::L;
  constexpr int THREADS = K::THREADS, MI = K::MI, NJ = K::NJ, EX = K::EX, EY = K::EY;
  extern __shared__ __align__(16) double smem[];
  double *sX = smem;
  double *sY = smem + STAGES * L::XS;
  int64_t *rowX = reinterpret_cast<int64_t *>(sY + STAGES * L::YS);
  int64_t *rowC = rowX + BM;
  int64_t *colY = rowC + BM;
  int64_t *colC = colY + BN;

  const int tid = threadIdx.x;
  const double *__restrict__ X = static_cast<const double *>(p.X);
  const double *__restrict__ Y = static_cast<const double *>(p.Y);
  double *__restrict__ C = static_cast<double *>(p.C);

  // ---- CTA -> (m-tile, n-tile), grouped rasterisation for L2 reuse --------------------
  int64_t mt, nt;
  {
    const int64_t id = blockIdx.x;
    const int64_t per_group = (int64_t)p.group_m * p.n.tiles;
    const int64_t g = id / per_group;
    const int64_t first_m = g * p.group_m;
    const int64_t gsz = min((int64_t)p.group_m, p.m.tiles - first_m);
    const int64_t r = id - g * per_group;
    mt = first_m + r % gsz;
    nt = r / gsz;
  }

  // ---- row / column offset tables (separable addresses; -1 = outside the tensor) ------
  {
    int lim[kMaxDigits];
    int64_t bOp = 0, bC = 0;
    int64_t q = mt;
    for (int d = 0; d < p.m.nd; d++) {
      const int64_t c = q % p.m.ntile[d];
      q /= p.m.ntile[d];
      const int64_t t0 = c * p.m.T[d];
      lim[d] = (int)min((int64_t)p.m.T[d], p.m.N[d] - t0);
      bOp += t0 * p.m.sOp[d];
      bC += t0 * p.m.sC[d];
    }
    for (int r = tid; r < BM; r += THREADS) {
      int rr = r;
      bool ok = true;
      int64_t ox = bOp, oc = bC;
      for (int d = 0; d < p.m.nd; d++) {
        const int dd = rr % p.m.T[d];
        rr /= p.m.T[d];
        ok &= dd < lim[d];
        ox += dd * p.m.sOp[d];
        oc += dd * p.m.sC[d];
      }
      ok &= rr == 0;
      rowX[r] = ok ? p.baseX + ox : -1;
      rowC[r] = ok ? p.baseC + oc : -1;
    }
    bOp = 0; bC = 0; q = nt;
    for (int d = 0; d < p.n.nd; d++) {
      const int64_t c = q % p.n.ntile[d];
      q /= p.n.ntile[d];
      const int64_t t0 = c * p.n.T[d];
      lim[d] = (int)min((int64_t)p.n.T[d], p.n.N[d] - t0);
      bOp += t0 * p.n.sOp[d];
      bC += t0 * p.n.sC[d];
    }
    for (int r = tid; r < BN; r += THREADS) {
      int rr = r;
      bool ok = true;
      int64_t oy = bOp, oc = bC;
      for (int d = 0; d < p.n.nd; d++) {
        const int dd = rr % p.n.T[d];
        rr /= p.n.T[d];
        ok &= dd < lim[d];
        oy += dd * p.n.sOp[d];
        oc += dd * p.n.sC[d];
      }
      ok &= rr == 0;
      colY[r] = ok ? p.baseY + oy : -1;
      colC[r] = ok ? oc : -1;
    }
  }
  // zero the ring once: positions no slot ever writes (m >= Mt, k >= Kt) must read as 0
  for (int i = tid; i < STAGES * (L::XS + L::YS); i += THREADS) smem[i] = 0.0;
  __syncthreads();

  // ---- per-thread load slots (fixed across k-steps) ---------------------------------
  const int xpm = p.xKmajor ? L::PK : 1, xpk = p.xKmajor ? 1 : L::PM;
  const int ypn = p.yKmajor ? L::PK : 1, ypk = p.yKmajor ? 1 : L::PN;
  int64_t gx[EX], gy[EY];
  uint32_t sx[EX], sy[EY];
#pragma unroll
  for (int i = 0; i < EX; i++) {
    const int s = tid + i * THREADS;
    gx[i] = -2;
    sx[i] = 0;
    if (s < p.nslotX) {
      const uint32_t e = p.slotX[s];
      const int m = e >> 8, k = e & 255;
      const int64_t r = rowX[m];
      gx[i] = r < 0 ? -1 : r + p.relKX[k];
      sx[i] = (uint32_t)(m * xpm + k * xpk) | ((uint32_t)k << 20);
    }
  }
#pragma unroll
  for (int i = 0; i < EY; i++) {
    const int s = tid + i * THREADS;
    gy[i] = -2;
    sy[i] = 0;
    if (s < p.nslotY) {
      const uint32_t e = p.slotY[s];
      const int n = e >> 8, k = e & 255;
      const int64_t r = colY[n];
      gy[i] = r < 0 ? -1 : r + p.relKY[k];
      sy[i] = (uint32_t)(n * ypn + k * ypk) | ((uint32_t)k << 20);
    }
  }
  const bool vx = p.vecX == 2, vy = p.vecY == 2;

  auto load_stage = [&](int step, int stage) {
    const int64_t bx = p.stepX[step], by = p.stepY[step];
    const uint64_t mask = p.kmask[step];
    double *dX = sX + stage * L::XS;
    double *dY = sY + stage * L::YS;
#pragma unroll
    for (int i = 0; i < EX; i++) {
      if (gx[i] != -2) {
        const int k = sx[i] >> 20;
        const bool ok = gx[i] >= 0 && ((mask >> k) & 1);
        const double *src = ok ? X + (gx[i] + bx) : X;
        double *dst = dX + (sx[i] & 0xFFFFF);
        if (vx) cp_async16(dst, src, ok ? 16 : 0);
        else cp_async8(dst, src, ok ? 8 : 0);
      }
    }
#pragma unroll
    for (int i = 0; i < EY; i++) {
      if (gy[i] != -2) {
        const int k = sy[i] >> 20;
        const bool ok = gy[i] >= 0 && ((mask >> k) & 1);
        const double *src = ok ? Y + (gy[i] + by) : Y;
        double *dst = dY + (sy[i] & 0xFFFFF);
        if (vy) cp_async16(dst, src, ok ? 16 : 0);
        else cp_async8(dst, src, ok ? 8 : 0);
      }
    }
  };

  // ---- warp tile ----------------------------------------------------------------------
  const int warp = tid >> 5, lane = tid & 31;
  const int wm = warp % K::WARPS_M, wn = warp / K::WARPS_M;
  const int g = lane >> 2, t = lane & 3;
  const int aoff = (wm * WM + g) * xpm + t * xpk;
  const int boff = (wn * WN + g) * ypn + t * ypk;
  const int astep_i = 8 * xpm, astep_k = 4 * xpk;
  const int bstep_j = 8 * ypn, bstep_k = 4 * ypk;

  double acc[MI][NJ][2];
#pragma unroll
  for (int i = 0; i < MI; i++)
#pragma unroll
    for (int j = 0; j < NJ; j++) acc[i][j][0] = acc[i][j][1] = 0.0;

  const int nsteps = p.nsteps;
#pragma unroll
  for (int s = 0; s < STAGES - 1; s++) {
    if (s < nsteps) load_stage(s, s);
    cp_async_commit();
  }
  for (int step = 0; step < nsteps; step++) {
    cp_async_wait<STAGES - 2>();
    __syncthreads();
    {
      const int nxt = step + STAGES - 1;
      if (nxt < nsteps) load_stage(nxt, nxt % STAGES);
      cp_async_commit();
    }
    const double *xs = sX + (step % STAGES) * L::XS + aoff;
    const double *ys = sY + (step % STAGES) * L::YS + boff;
#pragma unroll
    for (int kk = 0; kk < BK / 4; kk++) {
      double a[MI], b[NJ];
#pragma unroll
      for (int i = 0; i < MI; i++) a[i] = xs[i * astep_i + kk * astep_k];
#pragma unroll
      for (int j = 0; j < NJ; j++) b[j] = ys[j * bstep_j + kk * bstep_k];
#pragma unroll
      for (int i = 0; i < MI; i++)
#pragma unroll
        for (int j = 0; j < NJ; j++) dmma884(acc[i][j][0], acc[i][j][1], a[i], b[j]);
    }
  }
  cp_async_wait<0>();

  // ---- epilogue: C = alpha * acc + beta * C (beta == 0: C not read) --------------------
  const double alpha = p.alpha, beta = p.beta;
#pragma unroll
  for (int i = 0; i < MI; i++) {
    const int64_t rc = rowC[wm * WM + i * 8 + g];
    if (rc < 0) continue;
#pragma unroll
    for (int j = 0; j < NJ; j++) {
#pragma unroll
      for (int h = 0; h < 2; h++) {
        const int64_t cc = colC[wn * WN + j * 8 + 2 * t + h];
        if (cc < 0) continue;
        double *dst = C + (rc + cc);
        const double v = alpha * acc[i][j][h];
        *dst = beta != 0.0 ? fma(beta, *dst, v) : v;
      }
    }
  }
}

}  // namespace tc
