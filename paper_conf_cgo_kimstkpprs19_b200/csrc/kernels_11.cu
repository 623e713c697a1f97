// kernels_11.cu — FP64 kernel instances with smem layouts XK=true, YK=true (kernel_table.cuh).
#include "kernel_table.cuh"

namespace tc {
const void *kernel_ptr_11(int v) { return kernel_ptr<true, true>(v); }
}  // namespace tc
