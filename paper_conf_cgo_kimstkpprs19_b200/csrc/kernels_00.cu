// kernels_00.cu — FP64 kernel instances with smem layouts XK=false, YK=false (kernel_table.cuh).
#include "kernel_table.cuh"

namespace tc {
F64Instance f64_instance_00(int v) { return f64_instance<false, false>(v); }
}  // namespace tc
