#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_f32.py tests/test_gpu_bf16.py -q -x > gpurun_out/pytest_f32.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_f32.log
timeout 900 python bench.py --no-e2e --no-cpu --suites membound --cases 1 > gpurun_out/bench_suites.json 2> gpurun_out/bench_suites.err
