mkdir -p gpurun_out
rm -f gpurun_out/ab2.log
for so in libtc.so build/pf2/libtc.so libtc.so build/pf2/libtc.so; do
echo "== $so" >> gpurun_out/ab2.log
LIBTC_SO=$PWD/paper_conf_cgo_kimstkpprs19_b200/$so timeout 600 python bench.py --no-e2e --no-cpu --suites "" --steps 5 --cases 1,3,6,8,13,16,31,33,35,40,44,46 >> gpurun_out/ab2.log 2>&1
done
