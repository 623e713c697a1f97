// kernel_table.cuh — the compiled FP64 kernel instances, one row per tiles.cpp variant.
// Each kernels_<XK><YK>.cu instantiates the table for one pair of smem layouts, so the
// 4 x |variants| instances compile in parallel translation units.
// Consumer warps own 32 x 32 warp tiles (64 accumulator registers); a 4-warp producer
// group keeps its load slots in registers.  Warps per SM stay <= 16 so that no instance
// has fewer than 128 registers per thread (the register file is 16 K per sub-partition).
// Shared memory = BM x BN C staging box (TMA epilogue) + STAGES ring stages; the stage
// counts keep MINB CTAs resident within 227 KB.
#pragma once
#include "kernel_f64.cuh"

namespace tc {

template <bool XK, bool YK>
const void *kernel_ptr(int v) {
  switch (v) {
    //                                           BM   BN  BK  WM  WN  ST PW MINB
    case 0: return (const void *)&tc_f64_dmma_kernel<128, 64, 16, 32, 32, 3, 4, 1, XK, YK>;
    case 1: return (const void *)&tc_f64_dmma_kernel<64, 128, 16, 32, 32, 3, 4, 1, XK, YK>;
    case 2: return (const void *)&tc_f64_dmma_kernel<64, 64, 16, 32, 32, 4, 4, 2, XK, YK>;
    case 3: return (const void *)&tc_f64_dmma_kernel<64, 64, 24, 32, 32, 3, 4, 2, XK, YK>;
    case 4: return (const void *)&tc_f64_dmma_kernel<128, 64, 24, 32, 32, 3, 4, 1, XK, YK>;
    case 5: return (const void *)&tc_f64_dmma_kernel<64, 128, 24, 32, 32, 3, 4, 1, XK, YK>;
    case 6: return (const void *)&tc_f64_dmma_kernel<128, 32, 16, 32, 32, 4, 4, 2, XK, YK>;
    case 7: return (const void *)&tc_f64_dmma_kernel<32, 128, 16, 32, 32, 4, 4, 2, XK, YK>;
    case 8: return (const void *)&tc_f64_dmma_kernel<128, 32, 24, 32, 32, 3, 4, 1, XK, YK>;
    case 9: return (const void *)&tc_f64_dmma_kernel<32, 128, 24, 32, 32, 3, 4, 1, XK, YK>;
    case 10: return (const void *)&tc_f64_dmma_kernel<64, 64, 8, 32, 32, 4, 4, 2, XK, YK>;
  }
  return nullptr;
}

// defined in kernels_00.cu / _01 / _10 / _11
const void *kernel_ptr_00(int v);
const void *kernel_ptr_01(int v);
const void *kernel_ptr_10(int v);
const void *kernel_ptr_11(int v);
// defined in kernels_bf16.cu (BF16 tcgen05 variants; smem bytes and block size out)
const void *kernel_ptr_bf16(int v, bool xk, bool yk, size_t *smem, int *threads);

}  // namespace tc
