// kernels_group.cu — instances of the fused grouped FP64 kernel (kernel_group.cuh): variant 0 =
// BK 16 with 3 stages, variant 1 = BK 24 with 2 stages (both 2 CTAs per SM; group.cpp picks
// the BK with the fewest padded k-steps).
#include "kernel_group.cuh"

namespace tc {

const void *group_kernel_ptr(int v, size_t *smem, int *threads) {
  switch (v) {
    case 0:
      *smem = GroupCfg<16, 3>::smem_bytes();
      *threads = GroupCfg<16, 3>::THREADS;
      return (const void *)&tc_f64_group_kernel<16, 3>;
    case 1:
      *smem = GroupCfg<24, 2>::smem_bytes();
      *threads = GroupCfg<24, 2>::THREADS;
      return (const void *)&tc_f64_group_kernel<24, 2>;
  }
  *smem = 0;
  *threads = 0;
  return nullptr;
}

}  // namespace tc
