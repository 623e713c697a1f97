// kernel_group.cuh — the fused grouped FP64 contraction kernel (group.hpp).
//
// The CCSD(T) triples (9 sd_t_d1 + 9 sd_t_d2 contractions, all adding into
// one t3) run as one persistent kernel.  Per C tile (a hyper-rectangle prod_p T_p of t3,
// P:L119), for every member i in turn:
//   (1) the member's X_i tile (Mt_i x Kt_i) and Y_i tile (Kt_i x Nt_i) of each k-step reach a
//       STAGES-deep shared-memory ring (the paper's step 1): by TMA — one elected
//       thread issues cp.async.bulk.tensor boxes over each operand's own index order
//       (P:L138-145), SWIZZLE_128B / 64B, out-of-range elements zero-filled by the hardware
//        — or, when some operand cannot be a TMA box, by producer warps gathering runs
//       along each operand's FVI with cp.async into padded-pitch planes;
//   (2)+(3) CONSUMER warps run DMMA m8n8k4 register tiles over the stage (steps 2-3,
//       P:L82-83); fragment addresses come from per-member row / k tables (swizzled for the
//       TMA planes), so one code path serves every member's layout;
//   the member's register tile STARTS from the C tile's current values in an XOR-swizzled smem
//   box and is written back after its last k-step (the DMMAs do the accumulation: no separate
//   adds on the FP64 pipe).  After the last member the box leaves for C once:
//   C = alpha * box + beta * C (step 4) — t3 is written once instead of 18 times.
#pragma once
#include <cstdint>

#include "group.hpp"
#include "kernel_f64.cuh"

namespace tc {

// Ablation side builds only (tools/group_ablation.py compiles libtc with -DTC_GROUP_ABLATE=k;
// the shipped library has kGAbl = 0): 1 = producers skip the loads, 2 = consumers skip the
// DMMAs, 3 = consumers skip the box load / store.
#ifdef TC_GROUP_ABLATE
constexpr int kGAbl = TC_GROUP_ABLATE;
#else
constexpr int kGAbl = 0;
#endif
// Hand-off timeline (-DTC_GROUP_TRACE side builds only, tools/group_trace.py): CTA 0, consumer
// warp 0 / producer warp 0, lane 0, clock64 at slot * 1024 + step of p.trace.
#ifdef TC_GROUP_TRACE
#define GTRACE(slot, step)                                                                   \
  do {                                                                                       \
    if (blockIdx.x == 0 && (threadIdx.x & 127) == 0 && (step) >= 0 && (step) < 1024)         \
      p.trace[(slot) * 1024 + (step)] = clock64();                                           \
  } while (0)
#else
#define GTRACE(slot, step) do { } while (0)
#endif

struct GParams {
  TmaDesc xmap[kGMaxMembers];      // TMA mode: per member the tensor maps of X_i and Y_i
  TmaDesc ymap[kGMaxMembers];
  const double *X[kGMaxMembers];   // per member: its X / Y operand (A or B, group.hpp)
  const double *Y[kGMaxMembers];
  uint64_t vecmask;                // cp.async: bit 2i: X_i may use 16-B vectors; bit 2i+1: Y_i
  double *C;
  double alpha, beta;
  int nmem, rank, ntiles, nunits;
  int uvec;                        // C elements per copy-out unit (1 or 2, group.cpp)
  int cvec16;                      // 1: units of 2 are stored as one 16-B vector (C aligned)
  int stage_bytes;                 // TMA: bytes per ring stage (group.hpp tma_stage_bytes)
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
  const int32_t *ctab;             // this launch mode's consumer tables (group.hpp)
  const int64_t *unitRel;
  const uint64_t *unitDig;
  unsigned long long *trace;       // (-DTC_GROUP_TRACE side builds only)
};

template <int BK, int STAGES, bool TMA>
struct GroupCfg {
  static constexpr int BM = kGBM, BN = kGBN;
  static constexpr int CW = 4, PW = 4;                      // consumer / producer warps
  static constexpr int THREADS = (CW + PW) * 32;
  static constexpr int PM = BM + 4, PN = BN + 4, PK = BK + 4;
  static constexpr int XS = (BM * PK > BK * PM ? BM * PK : BK * PM) + 2;   // = gplane_doubles
  // plane bytes: TMA boxes (1 KB aligned, group.hpp gtma_plane_bytes) or padded-pitch planes
  // cp.async: padded-pitch planes; TMA: the stage size comes from the plan (p.stage_bytes:
  // the largest X box + Y box of a member), the Y box right after the member's X box
  static constexpr int PLANE = 8 * XS;
  static constexpr int STAGE = 2 * PLANE;
  static constexpr int BOX = BM * BN;
  // + 128 B: the ring is aligned to 128 B inside the dynamic smem (TMA destinations)
  static constexpr size_t smem_bytes(int tma_stage) {
    return 128 + (size_t)STAGES * (TMA ? tma_stage : STAGE) + 8 * BOX + 16 * STAGES;
  }
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

// ---------------------------------------------------------------- cp.async producer path
// Gather of one operand tile (one k-step) into a padded-pitch plane, in two phases so that the
// run-table latency hides behind the stage wait: vector w = pt + 128 e (e < 8 per chunk) is
// vector v of run q; runs lie along the operand's FVI, consecutive threads take consecutive
// vectors.
struct GFetch {
  int32_t rel[8];     // element offset of the vector in the operand tile
  uint32_t so[8];     // smem element offset in the plane
};

__device__ __forceinline__ void g_qv(int w0, int vpr, int &q, int &v, int &dq, int &dv) {
  q = w0 / vpr;
  v = w0 - q * vpr;
  dq = 128 / vpr;
  dv = 128 - dq * vpr;
}

__device__ __forceinline__ void g_fetch(const GParams &p, const GOperandDev &op, int vec, int nvec, int pt,
                                        int chunk, GFetch &f) {
  const int vpr = op.runlen / vec;
  const int32_t *__restrict__ rr = p.runRel + op.run0;
  const uint32_t *__restrict__ rs = p.runSoff + op.run0;
  const int w0 = pt + 1024 * chunk;
  int q, v, dq, dv;
  g_qv(w0, vpr, q, v, dq, dv);
#pragma unroll
  for (int e = 0; e < 8; e++) {
    if (w0 + 128 * e < nvec) {
      f.rel[e] = __ldg(rr + q) + v * vec;
      f.so[e] = __ldg(rs + q) + (uint32_t)(v * vec);
    }
    q += dq;
    v += dv;
    if (v >= vpr) { v -= vpr; q++; }
  }
}

__device__ __forceinline__ void g_issue(const GParams &p, const double *__restrict__ base, uint32_t sdst,
                                        const GOperandDev &op, int vec, int nvec, int pt, int chunk,
                                        const GFetch &f, bool fast, uint64_t L) {
  const int w0 = pt + 1024 * chunk;
  if (fast) {
#pragma unroll
    for (int e = 0; e < 8; e++) {
      if (w0 + 128 * e < nvec) {
        if (vec == 2) cp_async16_full(sdst + 8u * f.so[e], base + f.rel[e]);
        else cp_async8_full(sdst + 8u * f.so[e], base + f.rel[e]);
      }
    }
    return;
  }
  // bytes checked by SWAR: dims 1.. when runs cover dim 0, else every dim
  const int jfirst = op.runlen > 1 ? 1 : 0;
  uint64_t maskH = 0;
  for (int j = jfirst; j < op.ndim; j++) maskH |= 0x80ull << (8 * j);
  const int lim0 = (int)(L & 0xFF);
  const uint64_t *__restrict__ rd = p.runDig + op.run0;
  const int vpr = op.runlen / vec;
  int q, v, dq, dv;
  g_qv(w0, vpr, q, v, dq, dv);
  for (int e = 0; e < 8; e++) {
    if (w0 + 128 * e < nvec) {
      int nval = g_all_lt(__ldg(rd + q), L, maskH) ? vec : 0;
      if (op.runlen > 1) nval = min(nval, max(0, lim0 - v * vec));
      const uint32_t dst = sdst + 8u * f.so[e];
      if (vec == 2) cp_async16(dst, nval ? base + f.rel[e] : base, 8 * nval);
      else cp_async8(dst, nval ? base + f.rel[e] : base, 8 * nval);
    }
    q += dq;
    v += dv;
    if (v >= vpr) { v -= vpr; q++; }
  }
}

// ---------------------------------------------------------------- TMA producer path
// The TMA producer's per-member recipe (group.hpp GOperandDev::tma_pack: 4 bits of C position
// per map dim, 15 = the k dim / unused; rank at bit 20; k dim at bit 24).
struct GTmaRec {
  uint32_t tx, yoff, xpack, ypack;
  int32_t nsteps, step0;
  __device__ __forceinline__ void load(const GMemberDev &m) {
    tx = (uint32_t)(m.x.tma_tx + m.y.tma_tx);
    yoff = (uint32_t)m.tma_yoff;
    xpack = m.x.tma_pack;
    ypack = m.y.tma_pack;
    nsteps = m.nsteps;
    step0 = m.step0;
  }
};

// the box of one operand for (tile, k-step): coordinate per map dim = the tile origin of its
// C position (tcT) or the k-tile origin (the internal dim); all in registers
__device__ __forceinline__ void g_tma_operand(const TmaDesc *map, uint32_t pack, const int32_t (&tcT)[kGMaxCdims],
                                              int32_t kc, uint32_t dst, uint32_t bar, uint64_t pol) {
  int32_t c[kGMaxTmaDims];
  const int kd = (int)((pack >> 24) & 15);
#pragma unroll
  for (int j = 0; j < kGMaxTmaDims; j++) {
    const int cp = (int)((pack >> (4 * j)) & 15);
    int32_t v = 0;
#pragma unroll
    for (int q = 0; q < kGMaxCdims; q++) v = cp == q ? tcT[q] : v;   // (select: no local memory)
    c[j] = j == kd ? kc : v;
  }
  tma_load(map, (int)((pack >> 20) & 15), c[0], c[1], c[2], c[3], c[4], dst, bar, pol);
}

// ---------------------------------------------------------------- consumers
// Per member, per consumer thread (loaded one member ahead): the plane byte offsets of its
// fragment rows, the byte step of k in each plane (k is linear in both the padded-pitch
// planes and the TMA boxes), the box offsets of its accumulators (group.hpp consumer table),
// the Y plane's offset, the member's k-steps and k4 groups.
struct GRows {
  uint32_t rx[4], ry[4];
  int32_t bm[4], bn[4][2];
  uint32_t kmx, kmy;          // bytes per k
  int32_t yoff, nsteps, kq;
  bool chain;                 // the next member continues this register tile
  __device__ __forceinline__ void load(const int32_t *__restrict__ tb, const GMemberDev &m, int mode, int plane,
                                       int wm, int wn, int g, int t) {
#pragma unroll
    for (int a = 0; a < 4; a++) {
      rx[a] = (uint32_t)__ldg(tb + wm * 32 + a * 8 + g);
      ry[a] = (uint32_t)__ldg(tb + 64 + wn * 32 + a * 8 + g);
      bm[a] = __ldg(tb + 128 + wm * 32 + a * 8 + g);
      bn[a][0] = __ldg(tb + 192 + wn * 32 + a * 8 + 2 * t);
      bn[a][1] = __ldg(tb + 192 + wn * 32 + a * 8 + 2 * t + 1);
    }
    kmx = (uint32_t)m.x.kmul[mode];
    kmy = (uint32_t)m.y.kmul[mode];
    yoff = plane >= 0 ? plane : m.tma_yoff;
    nsteps = m.nsteps;
    kq = m.kq;
    chain = m.chain[mode] != 0;
  }
};

// One k-step of one member: DMMA over the stage; thread (g, t) loads A(row, 4 kk + t) and
// B(4 kk + t, col) from the member's row offsets and k steps.
template <int BK>
__device__ __forceinline__ void g_mma_step(double (&acc)[4][4][2], const char *__restrict__ xs,
                                           const char *__restrict__ ys, const GRows &r, int t, int kq) {
  const char *xt = xs + t * r.kmx, *yt = ys + t * r.kmy;
  const uint32_t sx = 4 * r.kmx, sy = 4 * r.kmy;
#pragma unroll
  for (int kk = 0; kk < BK / 4; kk++) {
    if (kk < kq) {
      double a[4], b[4];
#pragma unroll
      for (int i = 0; i < 4; i++) a[i] = *reinterpret_cast<const double *>(xt + r.rx[i] + kk * sx);
#pragma unroll
      for (int j = 0; j < 4; j++) b[j] = *reinterpret_cast<const double *>(yt + r.ry[j] + kk * sy);
#pragma unroll
      for (int i = 0; i < 4; i++)
#pragma unroll
        for (int j = 0; j < 4; j++) dmma884(acc[i][j][0], acc[i][j][1], a[i], b[j]);
    }
  }
}

// tile t -> C coordinates (position 0 fastest), packed limits, interior flag
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

template <int BK, int STAGES, bool TMA>
__global__ void __launch_bounds__(GroupCfg<BK, STAGES, TMA>::THREADS, 2)
tc_f64_group_kernel(const __grid_constant__ GParams p) {
  using K = GroupCfg<BK, STAGES, TMA>;
  constexpr int MODE = TMA ? 1 : 0;
  extern __shared__ __align__(128) unsigned char smem_dyn[];
  // smem: [STAGES][X | Y] (128-B aligned), the C box, the barriers, then (cp.async) the member
  // records (group_api.cu sizes it)
  unsigned char *ring = smem_dyn + ((128u - ((uint32_t)__cvta_generic_to_shared(smem_dyn) & 127u)) & 127u);
  const int SB = TMA ? p.stage_bytes : K::STAGE;   // bytes per stage
  double *box = reinterpret_cast<double *>(ring + STAGES * SB);
  uint64_t *bars = reinterpret_cast<uint64_t *>(box + K::BOX);   // full[S], empty[S]
  GMemberDev *smem_mem = reinterpret_cast<GMemberDev *>(bars + 2 * STAGES);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int ntl = (p.ntiles - (int)blockIdx.x + (int)gridDim.x - 1) / (int)gridDim.x;
  if (ntl <= 0) return;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(ring);
  const uint32_t bar0 = (uint32_t)__cvta_generic_to_shared(bars);

  // zero the ring once (cp.async: rows / k positions a member does not write are never
  // flushed, but must not hold NaN patterns that reach a valid accumulator)
  for (int i = tid; i < STAGES * SB / 16; i += K::THREADS)
    reinterpret_cast<uint4 *>(ring)[i] = make_uint4(0, 0, 0, 0);
  if (!TMA) {   // (the cp.async producers read their member records often: keep them in smem)
    const int nw = p.nmem * (int)(sizeof(GMemberDev) / 4);
    const uint32_t *src = reinterpret_cast<const uint32_t *>(p.mem);
    for (int i = tid; i < nw; i += K::THREADS) reinterpret_cast<uint32_t *>(smem_mem)[i] = src[i];
  }
  const GMemberDev *mems = TMA ? p.mem : smem_mem;
  if (tid == 0) {
    for (int s = 0; s < STAGES; s++) {
      mbar_init(bar0 + 8 * s, TMA ? 1 : K::PW * 32);   // full: the TMA thread / every producer
      mbar_init(bar0 + 8 * (STAGES + s), K::CW);       // empty: one arrive per consumer warp
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  // (generic-proxy zeroing of the ring before the TMA's async-proxy writes)
  asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
  __syncthreads();

  if (warp >= K::CW) {
    // ======================= producers ====================================================
    asm volatile("setmaxnreg.dec.sync.aligned.u32 88;\n" ::: "memory");   // registers to the consumers
    if (TMA) {
      if (warp != K::CW || lane != 0) return;
      // inputs are re-read by many tiles: keep them in L2 against the streaming C stores
      uint64_t policy;
      asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;\n" : "=l"(policy));
      int j = 0;
      GTmaRec nxt;
      nxt.load(p.mem[0]);
      for (int lt = 0; lt < ntl; lt++) {
        GTile tile;
        tile.decode(p, (int)blockIdx.x + lt * (int)gridDim.x);
        int32_t tcT[kGMaxCdims];   // tile origin per C position
#pragma unroll
        for (int q = 0; q < kGMaxCdims; q++) tcT[q] = tile.c[q] * p.T[q];
        for (int i = 0; i < p.nmem; i++) {
          // this member's recipe was loaded one member ahead (its latency hides behind the
          // previous member's stage wait)
          const GTmaRec M = nxt;
          nxt.load(p.mem[i + 1 < p.nmem ? i + 1 : 0]);
          for (int s = 0; s < M.nsteps; s++, j++) {
            const int st = j % STAGES;
            const int32_t kc = s == 0 ? 0 : p.steps[M.step0 + s].kc;   // (step 0 starts at k = 0)
            GTRACE(3, j);
            if (j >= STAGES) mbar_wait(bar0 + 8 * (STAGES + st), ((j / STAGES) & 1) ^ 1);
            GTRACE(4, j);
            const uint32_t full = bar0 + 8 * st;
            if (kGAbl == 1) { mbar_arrive(full); continue; }
            mbar_expect_tx(full, M.tx);
            const uint32_t dst = sbase + st * SB;
            g_tma_operand(&p.xmap[i], M.xpack, tcT, kc, dst, full, policy);
            g_tma_operand(&p.ymap[i], M.ypack, tcT, kc, dst + M.yoff, full, policy);
            GTRACE(5, j);
          }
        }
      }
      return;
    }
    const int pt = tid - K::CW * 32;
    int j = 0;
    for (int lt = 0; lt < ntl; lt++) {
      GTile tile;
      tile.decode(p, (int)blockIdx.x + lt * (int)gridDim.x);
      for (int i = 0; i < p.nmem; i++) {
        const GMemberDev &M = mems[i];
        const double *__restrict__ Xb = p.X[i] + tile.off(M.x.tstep, p.rank);
        const double *__restrict__ Yb = p.Y[i] + tile.off(M.y.tstep, p.rank);
        const int vx = ((p.vecmask >> (2 * i)) & 1) ? M.x.vec : 1;
        const int vy = ((p.vecmask >> (2 * i + 1)) & 1) ? M.y.vec : 1;
        // (needed by partial k-steps of interior tiles too)
        const uint64_t Lx = g_op_lims(M.x, tile.Lc);
        const uint64_t Ly = g_op_lims(M.y, tile.Lc);
        const int nvx = M.x.nrun * (M.x.runlen / vx), nvy = M.y.nrun * (M.y.runlen / vy);
        for (int s = 0; s < M.nsteps; s++, j++) {
          const int st = j % STAGES;
          // this thread's run-table entries (and the step record) are fetched BEFORE waiting
          // for the stage: their latency hides behind the consumers' work
          GTRACE(3, j);
          const GStepDev S = p.steps[M.step0 + s];
          GFetch fx, fy;
          if (kGAbl != 1) {
            g_fetch(p, M.x, vx, nvx, pt, 0, fx);
            g_fetch(p, M.y, vy, nvy, pt, 0, fy);
          }
          if (j >= STAGES) mbar_wait(bar0 + 8 * (STAGES + st), ((j / STAGES) & 1) ^ 1);
          GTRACE(4, j);
          if (kGAbl == 1) { mbar_arrive_cp_async(bar0 + 8 * st); continue; }
          const bool fast = tile.interior && S.full;
          const uint32_t dst = sbase + st * K::STAGE;
          g_issue(p, Xb + S.kx, dst, M.x, vx, nvx, pt, 0, fx, fast, Lx | S.klimX);
          g_issue(p, Yb + S.ky, dst + K::PLANE, M.y, vy, nvy, pt, 0, fy, fast, Ly | S.klimY);
          for (int c = 1; c * 8 * 128 < nvx; c++) {      // (operand tiles of more than 1024 vectors)
            g_fetch(p, M.x, vx, nvx, pt, c, fx);
            g_issue(p, Xb + S.kx, dst, M.x, vx, nvx, pt, c, fx, fast, Lx | S.klimX);
          }
          for (int c = 1; c * 8 * 128 < nvy; c++) {
            g_fetch(p, M.y, vy, nvy, pt, c, fy);
            g_issue(p, Yb + S.ky, dst + K::PLANE, M.y, vy, nvy, pt, c, fy, fast, Ly | S.klimY);
          }
          for (int w = pt; w < M.npad; w += K::PW * 32) cp_async8(dst + __ldg(p.pad + M.pad0 + w), Xb, 0);
          mbar_arrive_cp_async(bar0 + 8 * st);
          GTRACE(5, j);
        }
      }
    }
    return;
  }

  // ======================= consumers ======================================================
  asm volatile("setmaxnreg.inc.sync.aligned.u32 168;\n" ::: "memory");   // accumulators + tables
  const int wm = warp & 1, wn = warp >> 1;
  const int g = lane >> 2, t = lane & 3;
  double acc[4][4][2];
  double *__restrict__ C = p.C;
  const double alpha = p.alpha, beta = p.beta;
  // this thread's recipe of member 0; each member loads the next one's while it runs
  GRows cur;
  cur.load(p.ctab, mems[0], MODE, TMA ? -1 : K::PLANE, wm, wn, g, t);
  int j = 0;
  bool chained = false;   // the previous member left its register tile for this one
  for (int lt = 0; lt < ntl; lt++) {
    for (int i = 0; i < p.nmem; i++) {
      const int nsteps = cur.nsteps, kq = cur.kq;
      const int yoff = cur.yoff;
      GRows nxt;
      const int in = i + 1 < p.nmem ? i + 1 : 0;
      nxt.load(p.ctab + in * kGCtab, mems[in], MODE, TMA ? -1 : K::PLANE, wm, wn, g, t);
      // ---- the member's register tile starts from the box (every consumer finished the
      //      previous member's write-back — or the previous tile's copy-out — first), or
      //      simply continues when the previous member mapped it onto the box the same way
      if (!chained) {
        consumer_sync(K::CW * 32);
#pragma unroll
        for (int a = 0; a < 4; a++)
#pragma unroll
          for (int b = 0; b < 4; b++)
#pragma unroll
            for (int h = 0; h < 2; h++) {
              const bool ok = i > 0 && kGAbl != 3 && cur.bm[a] >= 0 && cur.bn[b][h] >= 0;
              acc[a][b][h] = ok ? box[gbox_sw(cur.bm[a] + cur.bn[b][h])] : 0.0;
            }
      }
      for (int s = 0; s < nsteps; s++, j++) {
        const int st = j % STAGES;
        mbar_wait(bar0 + 8 * st, (j / STAGES) & 1);
        GTRACE(0, j);
        const char *xs = reinterpret_cast<const char *>(ring) + st * SB;
        if (kGAbl != 2) g_mma_step<BK>(acc, xs, xs + yoff, cur, t, kq);
        __syncwarp();
        if (lane == 0) mbar_arrive(bar0 + 8 * (STAGES + st));
        GTRACE(1, j);
      }
      // ---- write the member's tile back into the box (unless the next member continues it)
      chained = cur.chain;
      if (kGAbl != 3 && !chained) {
#pragma unroll
        for (int a = 0; a < 4; a++)
#pragma unroll
          for (int b = 0; b < 4; b++)
#pragma unroll
            for (int h = 0; h < 2; h++)
              if (cur.bm[a] >= 0 && cur.bn[b][h] >= 0) box[gbox_sw(cur.bm[a] + cur.bn[b][h])] = acc[a][b][h];
      }
      GTRACE(2, j - 1);
      cur = nxt;
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
        // (C streams through L2 once: evict-first loads and stores keep the inputs there)
        if (beta != 0.0) {
          const double2 old = __ldcs(d2);
          v.x = fma(beta, old.x, v.x);
          v.y = fma(beta, old.y, v.y);
        }
        __stcs(d2, v);
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
