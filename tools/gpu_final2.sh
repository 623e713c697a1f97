#!/bin/bash
# One GPU call for the round's evidence (streaming build): GPU tests, smoke, the default bench
# line, the ncu launch list of the bench step, the ncu --set full traffic capture (one launch
# per case), and --set full captures of the streaming kernels (FP64 / BF16 / TF32 on TCCG #1)
# and of the dominant tile kernel.  usage: tools/gpu_final2.sh TAG
TAG=${1:-r02f}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q --durations=10 > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
start=$(date +%s); timeout 1500 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench wall s: $(( $(date +%s) - start ))" >> gpurun_out/${TAG}_bench.err
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
   python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu --suites "" --no-scale6d --no-splitk > gpurun_out/${TAG}_bench_ncu_launch.log 2>&1
timeout 1500 ncu --set full --clock-control none --profile-from-start off -k regex:tc_ \
   -o gpurun_out/${TAG}_traffic -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu --suites "" --no-scale6d --no-splitk --profile > gpurun_out/${TAG}_bench_ncu_full.log 2>&1
python tools/ncu_traffic.py gpurun_out/${TAG}_traffic.ncu-rep gpurun_out/profile_cases.json gpurun_out/${TAG}_ncu_traffic.json >> gpurun_out/${TAG}_bench_ncu_full.log 2>&1
python tools/ncu_top.py gpurun_out/${TAG}_traffic.ncu-rep 10 > gpurun_out/${TAG}_traffic_top.txt 2>&1
sz=$(stat -c %s gpurun_out/${TAG}_traffic.ncu-rep); [ "$sz" -gt 40000000 ] && rm gpurun_out/${TAG}_traffic.ncu-rep
for dt in f64 bf16 tf32; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:tc_stream -s 2 -c 1 -o gpurun_out/${TAG}_stream_${dt}_c1 -f \
     python tools/run_one.py abcde-efbad-cf "a:48;b:36;c:24;d:36;e:48;f:36" $dt > /dev/null 2>&1
done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:tc_stream -s 2 -c 1 -o gpurun_out/${TAG}_stream_f64_c7 -f \
   python tools/run_one.py abcd-ebad-ce "a:72;b:72;c:24;d:72;e:72" f64 > /dev/null 2>&1
for v in 10 0; do   # TCCG #33: the model's pick (v10) runs 2x the tuned one (v0)
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:tc_f64 -s 2 -c 1 -o gpurun_out/${TAG}_c33_v${v} -f \
     python tools/run_case.py 33 3 b200 $v > /dev/null 2>&1
done
ls -la gpurun_out | tail -30
