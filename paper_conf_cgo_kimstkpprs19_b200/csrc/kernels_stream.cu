// kernels_stream.cu — instances of the streaming kernels (kernel_stream.cuh) for beta == 0: FP64
// (DMMA), BF16 (mma.sync m16n8k16), TF32 / FP32-split (mma.sync m16n8k8) x NB n8 blocks (n <= 8 NB)
// x AR-long runs of C's FVI per warp x .trans / plain A loads (stream.cpp instance_exists keeps
// the lists in step).  The beta != 0 instances (FP64 / FP32 C) are in kernels_stream_beta.cu:
// a separate instance keeps the old-C reads out of the beta = 0 kernels' register allocation.
#include "kernel_stream.cuh"
#include "tiles.hpp"

namespace tc {

const void *stream_kernel_ptr_beta(int kind, int NB, int AR, bool trans);   // kernels_stream_beta.cu

template <int NB, int AR>
static const void *spick(int kind, bool trans) {
  switch (kind) {
    case KIND_F64_DMMA:
      return trans ? (const void *)&tc_stream_f64_kernel<NB, AR, true, false>
                   : (const void *)&tc_stream_f64_kernel<NB, AR, false, false>;
    case KIND_BF16_UMMA:
      return trans ? (const void *)&tc_stream_bf16_kernel<NB, AR, true> : (const void *)&tc_stream_bf16_kernel<NB, AR, false>;
    case KIND_TF32_UMMA:
      return trans ? (const void *)&tc_stream_tf32_kernel<NB, AR, true, false, false>
                   : (const void *)&tc_stream_tf32_kernel<NB, AR, false, false, false>;
    default:
      return trans ? (const void *)&tc_stream_tf32_kernel<NB, AR, true, true, false>
                   : (const void *)&tc_stream_tf32_kernel<NB, AR, false, true, false>;
  }
}

const void *stream_kernel_ptr(int kind, int NB, int AR, bool trans, bool beta) {
  if (beta) return kind == KIND_BF16_UMMA ? nullptr : stream_kernel_ptr_beta(kind, NB, AR, trans);
  switch (NB * 16 + AR) {
    case 1 * 16 + 4: return spick<1, 4>(kind, trans);
    case 1 * 16 + 8: return spick<1, 8>(kind, trans);
    case 2 * 16 + 4: return spick<2, 4>(kind, trans);
    case 2 * 16 + 8: return spick<2, 8>(kind, trans);
    case 3 * 16 + 4: return spick<3, 4>(kind, trans);
    case 3 * 16 + 8: return spick<3, 8>(kind, trans);
    case 4 * 16 + 4: return spick<4, 4>(kind, trans);
    // FP64 only: n up to 72 (9 n8 blocks)
    case 9 * 16 + 2:
      if (kind != KIND_F64_DMMA) return nullptr;
      return trans ? (const void *)&tc_stream_f64_kernel<9, 2, true, false>
                   : (const void *)&tc_stream_f64_kernel<9, 2, false, false>;
  }
  return nullptr;
}

}  // namespace tc
