// kernels_11.cu — FP64 kernel instances with smem layouts XK=true, YK=true (kernel_table.cuh).
#include "kernel_table.cuh"

namespace tc {
F64Instance f64_instance_11(int v) { return f64_instance<true, true>(v); }
}  // namespace tc
