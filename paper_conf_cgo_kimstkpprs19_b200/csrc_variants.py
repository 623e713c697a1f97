"""Number of compiled FP64 kernel variants (tiles.cpp variants(), api.cu kernels())."""
NUM_VARIANTS = 11
