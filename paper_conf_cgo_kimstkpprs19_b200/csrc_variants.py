"""Compiled kernel variants (tiles.cpp variants(), kernel_table.cuh, kernels_bf16.cu)."""
NUM_VARIANTS = 11                 # FP64 DMMA variants: ids 0 .. NUM_VARIANTS-1
BF16_VARIANTS = (11, 12)          # BF16 tcgen05 variants (BM = 128, BK = 64; BN = 64 / 128)
