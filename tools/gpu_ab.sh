mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/ab_pytest.log 2>&1; echo rc=$? >> gpurun_out/ab_pytest.log
DBGS=14,0 timeout 300 python tools/dbg_umma.py 1:bf16 8:tf32 18:bf16 >> gpurun_out/ab.log 2>&1
timeout 600 python bench.py --no-e2e --no-cpu --suites "" --steps 5 --cases 1,3,6,9,12,13,16,19,30,31,33,40,46 >> gpurun_out/ab.log 2>&1
