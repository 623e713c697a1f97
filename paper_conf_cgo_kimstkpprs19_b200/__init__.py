"""libtc — direct (transpose-free) tensor contraction on B200 (sm_100a).

After Kim et al., "A Code Generator for High-Performance Tensor Contractions on GPUs"
(CGO 2019).  The product is the C-ABI library ``libtc.so`` (include/libtc.h); this package
is its thin Python binding (``libtc``) plus the multi-GPU driver (``dist``).
"""
from .binding import (Plan, TcError, check, plan, shape_of, version, SLAB_A, SLAB_B,  # noqa: F401
                    SLAB_C)
