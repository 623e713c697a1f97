"""Compiled kernel variants, read from csrc/variants.def (the list tiles.cpp and
kernel_table.cuh are generated from) so the tests cannot drift from the library."""
import os
import re

_DEF = os.path.join(os.path.dirname(os.path.abspath(__file__)), "csrc", "variants.def")
_ROW = re.compile(r"^TC_F64_VARIANT\(\s*(\d+)((?:\s*,\s*\d+){9})\s*\)", re.M)

F64_SHAPES = {}
for _m in _ROW.finditer(open(_DEF).read()):
    _v = [int(x) for x in _m.group(2).split(",")[1:]]
    F64_SHAPES[int(_m.group(1))] = dict(zip(("BM", "BN", "BK", "WM", "WN", "stages", "pw", "occ", "stg"), _v))

F64_VARIANTS = tuple(sorted(F64_SHAPES))            # FP64 DMMA variants (direct + staged)
STG_VARIANTS = tuple(v for v in F64_VARIANTS if F64_SHAPES[v]["stg"])
BF16_VARIANTS = (11, 12)          # BF16 tcgen05 variants (BM = 128, BK = 64; BN = 64 / 128)
TF32_VARIANTS = (21, 22)          # TF32 tcgen05 (FP32 storage; BK = 32; BN = 64 / 128)
F32_VARIANTS = (23, 24)           # FP32 as split TF32 (hi*hi + hi*lo + lo*hi; BN = 64 / 128)
