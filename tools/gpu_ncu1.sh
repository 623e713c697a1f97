mkdir -p gpurun_out
for dt in tf32 bf16; do
TC_DTYPE=$dt timeout 600 ncu --set full --import-source on --clock-control none -k regex:tc_ -s 2 -c 1 -o gpurun_out/mb_$dt -f python tools/run_case.py 1 3 > gpurun_out/ncu_mb_$dt.log 2>&1
python tools/ncu_top.py gpurun_out/mb_$dt.ncu-rep 40 > gpurun_out/mb_${dt}_top.txt 2>&1
done
