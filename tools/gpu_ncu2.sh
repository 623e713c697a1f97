mkdir -p gpurun_out
timeout 600 ncu --set full --import-source on --clock-control none -k regex:tc_ -s 1 -c 1 -o gpurun_out/d14 -f python tools/dbg_one.py 8 tf32 14 > gpurun_out/ncu_d14.log 2>&1
python tools/ncu_top.py gpurun_out/d14.ncu-rep 40 > gpurun_out/d14_top.txt 2>&1
ncu -i gpurun_out/d14.ncu-rep --page source --csv --print-source cuda > gpurun_out/d14_src.csv 2>&1
