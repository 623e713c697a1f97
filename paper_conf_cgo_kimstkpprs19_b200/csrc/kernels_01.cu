// kernels_01.cu — FP64 kernel instances with smem layouts XK=false, YK=true (kernel_table.cuh).
#include "kernel_table.cuh"

namespace tc {
const void *kernel_ptr_01(int v) { return kernel_ptr<false, true>(v); }
}  // namespace tc
