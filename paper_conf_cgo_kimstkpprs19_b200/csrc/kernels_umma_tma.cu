// kernels_umma_tma.cu — tcgen05 kernel instances whose operands arrive by TMA (one elected
// producer thread, kernel_umma.cuh), one per BF16 / TF32 variant and smem-layout pair (the split
// FP32 kind converts its operands in smem and keeps the cp.async producers).
#include "kernel_umma.cuh"

namespace tc {

template <int KIND, int BN, int ST>
static const void *pick_tma(bool xk, bool yk, size_t *smem, int *threads) {
  *smem = UmmaKernel<KIND, BN, ST>::smem_bytes();
  *threads = UmmaKernel<KIND, BN, ST>::THREADS;
  return xk ? (yk ? (const void *)&tc_umma_kernel<KIND, BN, ST, true, true, true>
                  : (const void *)&tc_umma_kernel<KIND, BN, ST, true, false, true>)
            : (yk ? (const void *)&tc_umma_kernel<KIND, BN, ST, false, true, true>
                  : (const void *)&tc_umma_kernel<KIND, BN, ST, false, false, true>);
}

const void *kernel_ptr_umma_tma(int v, bool xk, bool yk, size_t *smem, int *threads) {
  switch (v) {
    case 11: return pick_tma<1, 64, 6>(xk, yk, smem, threads);
    case 12: return pick_tma<1, 128, 5>(xk, yk, smem, threads);
    case 21: return pick_tma<2, 64, 6>(xk, yk, smem, threads);
    case 22: return pick_tma<2, 128, 5>(xk, yk, smem, threads);
  }
  *smem = 0;
  *threads = 0;
  return nullptr;
}

}  // namespace tc
