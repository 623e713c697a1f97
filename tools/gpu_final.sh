#!/bin/bash
# One GPU call for the round's evidence: GPU tests, smoke, the default bench line, the ncu
# launch list of the bench step, the ncu --set full traffic capture (one launch per case), and
# --set full captures of the kernels the DESIGN discusses.  usage: tools/gpu_final.sh TAG
TAG=${1:-r02z}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -x -q --durations=15 > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
start=$(date +%s); timeout 1500 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench wall s: $(( $(date +%s) - start ))" >> gpurun_out/${TAG}_bench.err
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
   python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu --suites "" --no-scale6d --no-splitk > gpurun_out/${TAG}_bench_ncu_launch.log 2>&1
timeout 1500 ncu --set full --clock-control none --profile-from-start off -k regex:tc_ \
   -o gpurun_out/${TAG}_traffic -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu --suites "" --no-scale6d --no-splitk --profile > gpurun_out/${TAG}_bench_ncu_full.log 2>&1
python tools/ncu_traffic.py gpurun_out/${TAG}_traffic.ncu-rep gpurun_out/profile_cases.json gpurun_out/${TAG}_ncu_traffic.json >> gpurun_out/${TAG}_bench_ncu_full.log 2>&1
python tools/ncu_top.py gpurun_out/${TAG}_traffic.ncu-rep 10 > gpurun_out/${TAG}_traffic_top.txt 2>&1
sz=$(stat -c %s gpurun_out/${TAG}_traffic.ncu-rep); [ "$sz" -gt 40000000 ] && rm gpurun_out/${TAG}_traffic.ncu-rep
# kernels discussed in DESIGN.md: BF16 ab-ac-cb (CTA pairs, TMA), FP64 #31 (near ridge), FP64 #1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:tc_umma -s 2 -c 1 -o gpurun_out/${TAG}_pair -f \
   python tools/run_one.py ab-ac-cb "a:5136;b:5120;c:5136" bf16 > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:tc_f64 -s 2 -c 1 -o gpurun_out/${TAG}_c31 -f \
   python tools/run_one.py abcdef-dega-gfbc "a:24;b:16;c:16;d:24;e:16;f:16;g:24" f64 - 10 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_f64_group -s 1 -c 1 -o gpurun_out/${TAG}_fused -f \
   python tools/bench_fused.py "a:24;b:24;c:24;d:24;e:24;f:24;g:24" > /dev/null 2>&1
ls -la gpurun_out | tail -30
