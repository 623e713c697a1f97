// kernels_01.cu — FP64 kernel instances with smem layouts XK=false, YK=true (kernel_table.cuh).
#include "kernel_table.cuh"

namespace tc {
F64Instance f64_instance_01(int v) { return f64_instance<false, true>(v); }
}  // namespace tc
