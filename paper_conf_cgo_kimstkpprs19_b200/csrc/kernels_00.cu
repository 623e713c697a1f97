// kernels_00.cu — FP64 kernel instances with smem layouts XK=false, YK=false (kernel_table.cuh).
#include "kernel_table.cuh"

namespace tc {
const void *kernel_ptr_00(int v) { return kernel_ptr<false, false>(v); }
}  // namespace tc
