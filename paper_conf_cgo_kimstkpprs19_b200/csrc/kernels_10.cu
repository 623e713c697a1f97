// kernels_10.cu — FP64 kernel instances with smem layouts XK=true, YK=false (kernel_table.cuh).
#include "kernel_table.cuh"

namespace tc {
F64Instance f64_instance_10(int v) { return f64_instance<true, false>(v); }
}  // namespace tc
