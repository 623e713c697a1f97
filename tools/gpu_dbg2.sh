mkdir -p gpurun_out
DBGS=14,16398,0 timeout 200 python tools/dbg_umma.py 1:bf16 18:bf16 > gpurun_out/dbg_umma.log 2>&1
