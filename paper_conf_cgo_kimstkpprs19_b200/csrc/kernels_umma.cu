// kernels_umma.cu — tcgen05 kernel instances (kernel_umma.cuh) with cp.async producers, one per
// tiles.cpp UMMA variant and smem-layout pair; the TMA-producer instances are in
// kernels_umma_tma.cu (a second translation unit: the two compile in parallel).
#include "kernel_umma.cuh"

namespace tc {

const void *kernel_ptr_umma_tma(int v, bool xk, bool yk, size_t *smem, int *threads);   // kernels_umma_tma.cu

template <int KIND, int BN, int ST>
static const void *pick(bool xk, bool yk, size_t *smem, int *threads) {
  *smem = UmmaKernel<KIND, BN, ST>::smem_bytes();
  *threads = UmmaKernel<KIND, BN, ST>::THREADS;
  return xk ? (yk ? (const void *)&tc_umma_kernel<KIND, BN, ST, true, true>
                  : (const void *)&tc_umma_kernel<KIND, BN, ST, true, false>)
            : (yk ? (const void *)&tc_umma_kernel<KIND, BN, ST, false, true>
                  : (const void *)&tc_umma_kernel<KIND, BN, ST, false, false>);
}

// Variant ids as in tiles.cpp: BF16 11 = 128 x 64 x 64 (6 stages), 12 = 128 x 128 x 64 (5);
// TF32 21 = 128 x 64 x 32 (6), 22 = 128 x 128 x 32 (5); F32X3 23 = 128 x 64 x 32 (3),
// 24 = 128 x 128 x 32 (2).
const void *kernel_ptr_umma(int v, bool xk, bool yk, bool tma, size_t *smem, int *threads) {
  if (tma) return kernel_ptr_umma_tma(v, xk, yk, smem, threads);
  switch (v) {
    case 11: return pick<1, 64, 6>(xk, yk, smem, threads);
    case 12: return pick<1, 128, 5>(xk, yk, smem, threads);
    case 21: return pick<2, 64, 6>(xk, yk, smem, threads);
    case 22: return pick<2, 128, 5>(xk, yk, smem, threads);
    case 23: return pick<3, 64, 3>(xk, yk, smem, threads);
    case 24: return pick<3, 128, 2>(xk, yk, smem, threads);
  }
  *smem = 0;
  *threads = 0;
  return nullptr;
}

}  // namespace tc
