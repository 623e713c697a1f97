mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py --no-e2e --no-cpu --suites "" > gpurun_out/bench_q.json 2> gpurun_out/bench_q.err
DBGS=14,16398,0 timeout 200 python tools/dbg_umma.py 1:bf16 18:bf16 > gpurun_out/dbg_umma.log 2>&1
