// kernels_bf16.cu — BF16 tcgen05 kernel instances (kernel_bf16.cuh), one per tiles.cpp BF16
// variant and smem-layout pair.
#include "kernel_bf16.cuh"

namespace tc {

template <int BN, int ST>
static const void *pick(bool xk, bool yk, size_t *smem) {
  *smem = Bf16Kernel<BN, ST>::smem_bytes();
  return xk ? (yk ? (const void *)&tc_bf16_umma_kernel<BN, ST, true, true>
                  : (const void *)&tc_bf16_umma_kernel<BN, ST, true, false>)
            : (yk ? (const void *)&tc_bf16_umma_kernel<BN, ST, false, true>
                  : (const void *)&tc_bf16_umma_kernel<BN, ST, false, false>);
}

// Variant ids as in tiles.cpp: 11 = 128 x 64 x 64 (6 stages), 12 = 128 x 128 x 64 (5 stages).
const void *kernel_ptr_bf16(int v, bool xk, bool yk, size_t *smem, int *threads) {
  *threads = Bf16Kernel<64, 6>::THREADS;
  switch (v) {
    case 11: return pick<64, 6>(xk, yk, smem);
    case 12: return pick<128, 5>(xk, yk, smem);
  }
  *smem = 0;
  return nullptr;
}

}  // namespace tc
