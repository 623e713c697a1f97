// kernels_umma_pair.cu — tcgen05 kernel instances for CTA pairs (kernel_umma.cuh PAIR: a
// cluster of two CTAs, M = 256 MMAs over a 2 x 2 block of BN = 128 tiles, TMA operands), one
// per BF16 / TF32 BN = 128 variant and smem-layout pair.
#include "kernel_umma.cuh"

namespace tc {

template <int KIND, int BN, int ST>
static const void *pick_pair(bool xk, bool yk, size_t *smem, int *threads) {
  *smem = UmmaKernel<KIND, BN, ST, false>::smem_bytes();
  *threads = UmmaKernel<KIND, BN, ST, false>::THREADS;
  return xk ? (yk ? (const void *)&tc_umma_kernel<KIND, BN, ST, true, true, true, true>
                  : (const void *)&tc_umma_kernel<KIND, BN, ST, true, false, true, true>)
            : (yk ? (const void *)&tc_umma_kernel<KIND, BN, ST, false, true, true, true>
                  : (const void *)&tc_umma_kernel<KIND, BN, ST, false, false, true, true>);
}

const void *kernel_ptr_umma_pair(int v, bool xk, bool yk, size_t *smem, int *threads) {
  switch (v) {
    case 12: return pick_pair<1, 128, 6>(xk, yk, smem, threads);   // (no epilogue staging: 6 stages)
    case 22: return pick_pair<2, 128, 6>(xk, yk, smem, threads);
  }
  *smem = 0;
  *threads = 0;
  return nullptr;
}

}  // namespace tc
