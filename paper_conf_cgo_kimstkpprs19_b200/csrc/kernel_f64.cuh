// kernel_f64.cuh — the FP64 direct-contraction kernel of libtc for sm_100a.
//
// The paper's four steps (Alg. 1) re-designed for B200:
//   (1) GMEM -> SMEM: the X tile (Mt x Kt) and Y tile (Kt x Nt) of one k-step are gathered
//       with cp.async (16 B when the operand's FVI allows, zero-fill outside the tensor),
//       walking each operand in its own memory order, into a STAGES-deep ring
//       (the paper's kernel was single-buffered with two syncs per step).
//   (2) SMEM -> REG: DMMA fragments (mma.sync.m8n8k4.f64 -> SASS DMMA.8x8x4; measured on
//       B200 at 37.1 TFLOP/s = the FP64 pipe's peak, profiles/r01_peaks.json).  The smem
//       pitch is 4 (mod 16) doubles so fragment loads are conflict-free in both layouts.
//   (3) outer product: each warp owns a WM x WN register tile of C (accumulate in
//       registers, not smem); the paper's r_C[T_b][T_c] of rank-1 updates becomes
//       (WM/8) x (WN/8) DMMA tiles per k4.
//   (4) REG -> GMEM: C = alpha * acc + beta * C through separable row / column offsets,
//       predicated on the tensor bounds (correct for any size).
// The CTAs are persistent (grid = 148 x CTAs/SM) and the cp.async ring runs ACROSS tile
// boundaries: the loads of tile i+1 are in flight while tile i's epilogue stores drain —
// the overlap the K = 24 CCSD(T) contractions need (SURVEY 7.2 hard part 1).
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
    return sizeof(double) * (size_t)STAGES * (L::XS + L::YS) + 16 * (size_t)(BM + BN);
  }
  static_assert(BK % 4 == 0 && BK <= 64, "BK");
  static_assert(WM % 8 == 0 && WN % 8 == 0, "warp tile");
  static_assert(BM <= 256 && BN <= 256, "slot packing");
  static_assert(L::XS < 8192 && L::YS < 8192, "13-bit smem offsets");
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

template <int BM, int BN, int BK, int WM, int WN, int STAGES, int MINB>
__global__ void __launch_bounds__(F64Kernel<BM, BN, BK, WM, WN, STAGES>::THREADS, MINB)
tc_f64_dmma_kernel(const KParams p) {
  using K = F64Kernel<BM, BN, BK, WM, WN, STAGES>;
  using L = typename K::L;
  constexpr int THREADS = K::THREADS, MI = K::MI, NJ = K::NJ, EX = K::EX, EY = K::EY;
  extern __shared__ __align__(16) double smem[];
  double *sX = smem;
  double *sY = smem + STAGES * L::XS;
  int64_t *relCm = reinterpret_cast<int64_t *>(sY + STAGES * L::YS);
  int64_t *relCn = relCm + BM;
  uint64_t *digM = reinterpret_cast<uint64_t *>(relCn + BN);
  uint64_t *digN = digM + BM;

  const int tid = threadIdx.x;
  const double *__restrict__ X = static_cast<const double *>(p.X);
  const double *__restrict__ Y = static_cast<const double *>(p.Y);
  double *__restrict__ C = static_cast<double *>(p.C);

  // tiles of this CTA: blockIdx.x, blockIdx.x + gridDim.x, ...
  const int ntl = (p.ntotal - (int)blockIdx.x + (int)gridDim.x - 1) / (int)gridDim.x;
  if (ntl <= 0) return;
  const int total = ntl * p.nsteps;

  // ---- once per CTA: tile-local tables, zeroed ring, per-thread load slots ------------
  for (int r = tid; r < BM; r += THREADS) { relCm[r] = p.relCm[r]; digM[r] = p.digM[r]; }
  for (int r = tid; r < BN; r += THREADS) { relCn[r] = p.relCn[r]; digN[r] = p.digN[r]; }
  // positions no slot writes (m >= Mt, k >= Kt) must read as 0 forever
  for (int i = tid; i < STAGES * (L::XS + L::YS); i += THREADS) smem[i] = 0.0;
  int64_t gx[EX], gy[EY];
  uint32_t sx[EX], sy[EY];
#pragma unroll
  for (int i = 0; i < EX; i++) {
    const int s = tid + i * THREADS;
    const bool in = s < p.nslotX;
    gx[i] = in ? p.relX[s] : 0;
    sx[i] = in ? p.packX[s] : 0xFFFFFFFFu;
  }
#pragma unroll
  for (int i = 0; i < EY; i++) {
    const int s = tid + i * THREADS;
    const bool in = s < p.nslotY;
    gy[i] = in ? p.relY[s] : 0;
    sy[i] = in ? p.packY[s] : 0xFFFFFFFFu;
  }
  __syncthreads();
  const bool vx = p.vecX == 2, vy = p.vecY == 2;

  // ---- producer state (which job is loaded next) ----------------------------------------
  int is_ = 0, it_ = 0;                 // step / local tile index of the next job to issue
  int64_t ibx = 0, iby = 0;             // tile origins in X / Y of the issue tile
  uint64_t ilm = 0, iln = 0;            // tile limits
  bool ipm = false, ipn = false;        // issue tile is partial (needs the bounds test)
  auto issue_tile = [&]() {
    int mt, nt;
    tile_coords(p, (int)blockIdx.x + it_ * (int)gridDim.x, mt, nt);
    const TileInfo tm = p.tileM[mt], tn = p.tileN[nt];
    ibx = tm.op; iby = tn.op; ilm = tm.lim; iln = tn.lim;
    ipm = ilm != p.fullM; ipn = iln != p.fullN;
  };
  auto issue = [&](int stage) {
    if (is_ == 0) issue_tile();
    const int64_t bx = ibx + p.stepX[is_], by = iby + p.stepY[is_];
    const uint64_t mask = p.kmask[is_];
    double *dX = sX + stage * L::XS;
    double *dY = sY + stage * L::YS;
#pragma unroll
    for (int i = 0; i < EX; i++) {
      const uint32_t pk = sx[i];
      if (pk != 0xFFFFFFFFu) {
        const int k = (pk >> 13) & 63, m = pk >> 19;
        bool ok = (mask >> k) & 1;
        if (ipm) ok = ok && swar_le(digM[m], ilm);
        const double *src = ok ? X + (bx + gx[i]) : X;
        double *dst = dX + (pk & 8191);
        if (vx) cp_async16(dst, src, ok ? 16 : 0);
        else cp_async8(dst, src, ok ? 8 : 0);
      }
    }
#pragma unroll
    for (int i = 0; i < EY; i++) {
      const uint32_t pk = sy[i];
      if (pk != 0xFFFFFFFFu) {
        const int k = (pk >> 13) & 63, n = pk >> 19;
        bool ok = (mask >> k) & 1;
        if (ipn) ok = ok && swar_le(digN[n], iln);
        const double *src = ok ? Y + (by + gy[i]) : Y;
        double *dst = dY + (pk & 8191);
        if (vy) cp_async16(dst, src, ok ? 16 : 0);
        else cp_async8(dst, src, ok ? 8 : 0);
      }
    }
    if (++is_ == p.nsteps) { is_ = 0; ++it_; }
  };

  // ---- warp tile ----------------------------------------------------------------------
  const int warp = tid >> 5, lane = tid & 31;
  const int wm = warp % K::WARPS_M, wn = warp / K::WARPS_M;
  const int g = lane >> 2, t = lane & 3;
  const int xpm = p.xKmajor ? L::PK : 1, xpk = p.xKmajor ? 1 : L::PM;
  const int ypn = p.yKmajor ? L::PK : 1, ypk = p.yKmajor ? 1 : L::PN;
  const int aoff = (wm * WM + g) * xpm + t * xpk;
  const int boff = (wn * WN + g) * ypn + t * ypk;
  const int astep_i = 8 * xpm, astep_k = 4 * xpk;
  const int bstep_j = 8 * ypn, bstep_k = 4 * ypk;

  double acc[MI][NJ][2];
#pragma unroll
  for (int i = 0; i < MI; i++)
#pragma unroll
    for (int j = 0; j < NJ; j++) acc[i][j][0] = acc[i][j][1] = 0.0;

#pragma unroll
  for (int s = 0; s < STAGES - 1; s++) {
    if (s < total) issue(s);
    cp_async_commit();
  }
  int cs = 0, ct = 0;   // consumer step / local tile
  const double alpha = p.alpha, beta = p.beta;
  for (int j = 0; j < total; j++) {
    cp_async_wait<STAGES - 2>();
    __syncthreads();
    if (j + STAGES - 1 < total) issue((j + STAGES - 1) % STAGES);
    cp_async_commit();
    const double *xs = sX + (j % STAGES) * L::XS + aoff;
    const double *ys = sY + (j % STAGES) * L::YS + boff;
#pragma unroll
    for (int kk = 0; kk < BK / 4; kk++) {
      double a[MI], b[NJ];
#pragma unroll
      for (int i = 0; i < MI; i++) a[i] = xs[i * astep_i + kk * astep_k];
#pragma unroll
      for (int jj = 0; jj < NJ; jj++) b[jj] = ys[jj * bstep_j + kk * bstep_k];
#pragma unroll
      for (int i = 0; i < MI; i++)
#pragma unroll
        for (int jj = 0; jj < NJ; jj++) dmma884(acc[i][jj][0], acc[i][jj][1], a[i], b[jj]);
    }
    if (++cs == p.nsteps) {
      // ---- epilogue of tile ct: C = alpha * acc + beta * C (beta == 0: C not read) -------
      int mt, nt;
      tile_coords(p, (int)blockIdx.x + ct * (int)gridDim.x, mt, nt);
      const TileInfo tm = p.tileM[mt], tn = p.tileN[nt];
      const int64_t cb = tm.c + tn.c;
      const bool pm = tm.lim != p.fullM, pn = tn.lim != p.fullN;
#pragma unroll
      for (int i = 0; i < MI; i++) {
        const int r = wm * WM + i * 8 + g;
        const bool rok = r < p.Mt && (!pm || swar_le(digM[r], tm.lim));
        const int64_t rc = cb + relCm[r];
#pragma unroll
        for (int jj = 0; jj < NJ; jj++) {
#pragma unroll
          for (int h = 0; h < 2; h++) {
            const int cidx = wn * WN + jj * 8 + 2 * t + h;
            const bool ok = rok && cidx < p.Nt && (!pn || swar_le(digN[cidx], tn.lim));
            if (ok) {
              double *dst = C + (rc + relCn[cidx]);
              const double v = alpha * acc[i][jj][h];
              *dst = beta != 0.0 ? fma(beta, *dst, v) : v;
            }
            acc[i][jj][h] = 0.0;
          }
        }
      }
      cs = 0;
      ++ct;
    }
  }
  cp_async_wait<0>();
}

}  // namespace tc
