// kernels_10.cu — FP64 kernel instances with smem layouts XK=true, YK=false (kernel_table.cuh).
#include "kernel_table.cuh"

namespace tc {
const void *kernel_ptr_10(int v) { return kernel_ptr<true, false>(v); }
}  // namespace tc
