// kernels_umma_f32out.cu — BF16 tcgen05 instances with an FP32 C (kernel_umma.cuh OUTF32;
// cp.async producers): split-K partial sums keep FP32 until the reduction (dist.py), one per
// BF16 variant and smem-layout pair.
#include "kernel_umma.cuh"

namespace tc {

template <int BN, int ST>
static const void *pick_f32out(bool xk, bool yk, size_t *smem, int *threads) {
  *smem = UmmaKernel<1, BN, ST>::smem_bytes();
  *threads = UmmaKernel<1, BN, ST>::THREADS;
  return xk ? (yk ? (const void *)&tc_umma_kernel<1, BN, ST, true, true, false, false, true>
                  : (const void *)&tc_umma_kernel<1, BN, ST, true, false, false, false, true>)
            : (yk ? (const void *)&tc_umma_kernel<1, BN, ST, false, true, false, false, true>
                  : (const void *)&tc_umma_kernel<1, BN, ST, false, false, false, false, true>);
}

const void *kernel_ptr_umma_f32out(int v, bool xk, bool yk, size_t *smem, int *threads) {
  switch (v) {
    case 11: return pick_f32out<64, 6>(xk, yk, smem, threads);
    case 12: return pick_f32out<128, 5>(xk, yk, smem, threads);
  }
  *smem = 0;
  *threads = 0;
  return nullptr;
}

}  // namespace tc
