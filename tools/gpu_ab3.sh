mkdir -p gpurun_out
rm -f gpurun_out/ab3.log
for so in build/base/libtc.so libtc.so; do
echo "== $so" >> gpurun_out/ab3.log
LIBTC_SO=$PWD/paper_conf_cgo_kimstkpprs19_b200/$so DBGS=0 timeout 300 python tools/dbg_umma.py 18:bf16 18:tf32 1:bf16 1:tf32 6:bf16 8:tf32 >> gpurun_out/ab3.log 2>&1
LIBTC_SO=$PWD/paper_conf_cgo_kimstkpprs19_b200/$so timeout 600 python bench.py --no-e2e --no-cpu --suites membound --cases 1 --steps 3 >> gpurun_out/ab3.log 2>&1
done
