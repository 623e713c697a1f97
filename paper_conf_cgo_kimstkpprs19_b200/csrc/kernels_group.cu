// kernels_group.cu — instances of the fused grouped FP64 kernel (kernel_group.cuh), 2 CTAs per
// SM each: variant 0 = BK 16, variant 1 = BK 24 (group.cpp picks the BK with the fewest
// padded k-steps); cp.async gathers into padded-pitch planes (3 / 2 stages) or TMA boxes
// (4 / 3 stages).
#include "kernel_group.cuh"

namespace tc {

template <int BK, int ST, bool TMA>
static const void *gpick(int tma_stage, size_t *smem, int *threads) {
  *smem = GroupCfg<BK, ST, TMA>::smem_bytes(tma_stage);
  *threads = GroupCfg<BK, ST, TMA>::THREADS;
  return (const void *)&tc_f64_group_kernel<BK, ST, TMA>;
}

const void *group_kernel_ptr(int v, bool tma, int tma_stage, size_t *smem, int *threads) {
  switch (v * 2 + (tma ? 1 : 0)) {
    case 0: return gpick<16, 3, false>(tma_stage, smem, threads);
    case 1: return gpick<16, 4, true>(tma_stage, smem, threads);
    case 2: return gpick<24, 2, false>(tma_stage, smem, threads);
    case 3: return gpick<24, 3, true>(tma_stage, smem, threads);
  }
  *smem = 0;
  *threads = 0;
  return nullptr;
}

}  // namespace tc
