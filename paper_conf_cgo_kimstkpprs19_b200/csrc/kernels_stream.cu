// kernels_stream.cu — instances of the streaming BF16 kernel (kernel_stream.cuh): NB n8 blocks
// (n <= 8 NB) x AR-long runs of C's FVI per warp x ldmatrix.trans or plain A fragments
// (stream.cpp instance_exists keeps the two in step).
#include "kernel_stream.cuh"

namespace tc {

template <int NB, int AR>
static const void *spick(bool trans) {
  return trans ? (const void *)&tc_stream_bf16_kernel<NB, AR, true> : (const void *)&tc_stream_bf16_kernel<NB, AR, false>;
}

const void *stream_kernel_ptr(int NB, int AR, bool trans) {
  switch (NB * 16 + AR) {
    case 1 * 16 + 4: return spick<1, 4>(trans);
    case 1 * 16 + 8: return spick<1, 8>(trans);
    case 2 * 16 + 4: return spick<2, 4>(trans);
    case 2 * 16 + 8: return spick<2, 8>(trans);
    case 3 * 16 + 4: return spick<3, 4>(trans);
    case 3 * 16 + 8: return spick<3, 8>(trans);
    case 4 * 16 + 4: return spick<4, 4>(trans);
  }
  return nullptr;
}

}  // namespace tc
