mkdir -p gpurun_out
timeout 300 python tools/_dbg_f32.py > gpurun_out/dbg.log 2>&1
timeout 600 compute-sanitizer --tool memcheck --print-limit 5 python tools/_dbg_f32.py > gpurun_out/dbg_san.log 2>&1
