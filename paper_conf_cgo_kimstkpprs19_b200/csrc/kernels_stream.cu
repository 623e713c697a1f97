// kernels_stream.cu — instances of the streaming kernels (kernel_stream.cuh): FP64 (DMMA) or BF16
// (mma.sync) x NB n8 blocks (n <= 8 NB) x AR-long runs of C's FVI per warp x .trans or plain A
// loads (stream.cpp instance_exists / instance_exists_f64 keep the lists in step).
#include "kernel_stream.cuh"

namespace tc {

template <int NB, int AR>
static const void *spick(bool f64, bool trans) {
  if (f64)
    return trans ? (const void *)&tc_stream_f64_kernel<NB, AR, true> : (const void *)&tc_stream_f64_kernel<NB, AR, false>;
  return trans ? (const void *)&tc_stream_bf16_kernel<NB, AR, true> : (const void *)&tc_stream_bf16_kernel<NB, AR, false>;
}

const void *stream_kernel_ptr(bool f64, int NB, int AR, bool trans) {
  switch (NB * 16 + AR) {
    case 1 * 16 + 4: return spick<1, 4>(f64, trans);
    case 1 * 16 + 8: return spick<1, 8>(f64, trans);
    case 2 * 16 + 4: return spick<2, 4>(f64, trans);
    case 2 * 16 + 8: return spick<2, 8>(f64, trans);
    case 3 * 16 + 4: return spick<3, 4>(f64, trans);
    case 3 * 16 + 8: return spick<3, 8>(f64, trans);
    case 4 * 16 + 4: return spick<4, 4>(f64, trans);
  }
  return nullptr;
}

}  // namespace tc
