// kernels_stream_beta.cu — the streaming kernels' beta != 0 instances (FP64 / TF32 / FP32-split C:
// the store phase reads the old C; BF16 runs beta != 0 on the tile kernels).  See
// kernels_stream.cu.
#include "kernel_stream.cuh"
#include "tiles.hpp"

namespace tc {

template <int NB, int AR>
static const void *spickb(int kind, bool trans) {
  switch (kind) {
    case KIND_F64_DMMA:
      return trans ? (const void *)&tc_stream_f64_kernel<NB, AR, true, true>
                   : (const void *)&tc_stream_f64_kernel<NB, AR, false, true>;
    case KIND_TF32_UMMA:
      return trans ? (const void *)&tc_stream_tf32_kernel<NB, AR, true, false, true>
                   : (const void *)&tc_stream_tf32_kernel<NB, AR, false, false, true>;
    case KIND_F32X3_UMMA:
      return trans ? (const void *)&tc_stream_tf32_kernel<NB, AR, true, true, true>
                   : (const void *)&tc_stream_tf32_kernel<NB, AR, false, true, true>;
  }
  return nullptr;
}

const void *stream_kernel_ptr_beta(int kind, int NB, int AR, bool trans) {
  switch (NB * 16 + AR) {
    case 1 * 16 + 4: return spickb<1, 4>(kind, trans);
    case 1 * 16 + 8: return spickb<1, 8>(kind, trans);
    case 2 * 16 + 4: return spickb<2, 4>(kind, trans);
    case 2 * 16 + 8: return spickb<2, 8>(kind, trans);
    case 3 * 16 + 4: return spickb<3, 4>(kind, trans);
    case 3 * 16 + 8: return spickb<3, 8>(kind, trans);
    case 4 * 16 + 4: return spickb<4, 4>(kind, trans);
    case 9 * 16 + 2:
      if (kind != KIND_F64_DMMA) return nullptr;
      return trans ? (const void *)&tc_stream_f64_kernel<9, 2, true, true>
                   : (const void *)&tc_stream_f64_kernel<9, 2, false, true>;
  }
  return nullptr;
}

}  // namespace tc
