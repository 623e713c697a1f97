mkdir -p gpurun_out
rm -f gpurun_out/ab4.log
for so in libtc.so build/sw3/libtc.so; do
echo "== $so" >> gpurun_out/ab4.log
LIBTC_SO=$PWD/paper_conf_cgo_kimstkpprs19_b200/$so DBGS=0 timeout 300 python tools/dbg_umma.py 18:f32 1:f32 6:f32 8:f32 >> gpurun_out/ab4.log 2>&1
LIBTC_SO=$PWD/paper_conf_cgo_kimstkpprs19_b200/$so timeout 300 python -m pytest tests/test_gpu_f32.py -q -x -k "f32 and not tf32" 2>&1 | tail -1 >> gpurun_out/ab4.log
done
