// kernel_table.cuh — the compiled FP64 kernel instances, one row of variants.def each.
// Each kernels_<XK><YK>.cu instantiates the table for one pair of smem layouts, so the
// 4 x |variants| instances compile in parallel translation units.
// Consumer warps own WM x WN warp tiles (at most 64 accumulator registers); a 4-warp producer
// group keeps its load slots in registers.  Warps per SM stay <= 16 so that no instance has
// fewer than 128 registers per thread (the register file is 16 K per sub-partition).
// Shared memory = STAGES ring stages (+ the staged-epilogue tile for STG variants, + the
// BM x BN TMA box when the optional TMA epilogue is on); the stage counts keep OCC CTAs
// resident within 227 KB.
#pragma once
#include "kernel_f64.cuh"

namespace tc {

struct F64Instance {
  const void *fn;
  int threads;
  size_t smem;       // without the TMA staging box
  size_t smem_tma;   // with it
};

template <bool XK, bool YK>
F64Instance f64_instance(int v) {
  switch (v) {
#define TC_F64_VARIANT(id, BM, BN, BK, WM, WN, ST, PW, OCC, STG)                                   \
  case id: {                                                                                       \
    using K = F64Kernel<BM, BN, BK, WM, WN, ST, PW, STG>;                                         \
    static_assert(K::smem_bytes(false) <= 227 * 1024, "variant exceeds shared memory");           \
    return {(const void *)&tc_f64_dmma_kernel<BM, BN, BK, WM, WN, ST, PW, OCC, XK, YK, STG>,      \
            K::THREADS, K::smem_bytes(false), K::smem_bytes(true)};                               \
  }
#include "variants.def"
#undef TC_F64_VARIANT
  }
  return {nullptr, 0, 0, 0};
}

// defined in kernels_00.cu / _01 / _10 / _11
F64Instance f64_instance_00(int v);
F64Instance f64_instance_01(int v);
F64Instance f64_instance_10(int v);
F64Instance f64_instance_11(int v);
// defined in kernels_umma.cu (BF16 / TF32 / F32X3 tcgen05 variants; smem bytes and block size out)
const void *kernel_ptr_umma(int v, bool xk, bool yk, bool tma, size_t *smem, int *threads);   // tma: TMA producer
// CTA-pair instances (BN = 128 BF16 / TF32 variants 12 / 22; nullptr otherwise)
const void *kernel_ptr_umma_pair(int v, bool xk, bool yk, size_t *smem, int *threads);
// the streaming kernels (kernels_stream.cu): FP64 or BF16, n8 blocks NB, C-FVI runs AR, .trans A loads
const void *stream_kernel_ptr(int kind, int NB, int AR, bool trans, bool beta);
// BF16 operands, FP32 C (variants 11 / 12; cp.async producers; nullptr otherwise)
const void *kernel_ptr_umma_f32out(int v, bool xk, bool yk, size_t *smem, int *threads);

}  // namespace tc
