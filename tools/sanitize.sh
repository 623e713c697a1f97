#!/bin/bash
# compute-sanitizer (memcheck, racecheck, synccheck) over the small parity set: every kernel
# family once — FP64 DMMA (direct, staged, TMA epilogue, beta), BF16/TF32 tcgen05 (cp.async,
# TMA operands, CTA pairs), the fused triples group.  Logs: gpurun_out/${TAG}_sanitize_*.log
TAG=${1:-r02}
mkdir -p gpurun_out
SEL_F64='tests/test_gpu_parity.py::test_eq1_worked_example tests/test_gpu_parity.py::test_alpha_beta_and_nan_c tests/test_gpu_parity.py::test_unaligned_pointers_use_scalar_loads'
SEL_UMMA='tests/test_gpu_umma_tma.py::test_bf16_tma_operands[0] tests/test_gpu_umma_tma.py::test_tf32_tma_operands[2] tests/test_gpu_umma_tma.py::test_cta_pair[bf16-0] tests/test_gpu_bf16.py::test_bf16_unaligned_pointers_and_tails'
SEL_GROUP='tests/test_gpu_group_fused.py::test_triples_fused_ragged'
for tool in memcheck racecheck synccheck; do
  for sel in F64 UMMA GROUP; do
    eval tests=\$SEL_$sel
    timeout 1500 compute-sanitizer --tool $tool --error-exitcode 99 --target-processes all \
      python -m pytest $tests -x -q -p no:cacheprovider > gpurun_out/${TAG}_sanitize_${tool}_${sel}.log 2>&1
    echo "$tool $sel rc=$?" >> gpurun_out/${TAG}_sanitize_summary.txt
  done
done
cat gpurun_out/${TAG}_sanitize_summary.txt
