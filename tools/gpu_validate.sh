#!/bin/bash
# One GPU call: tests, smoke, bench, launch list, ncu --set full traffic capture.
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
start=$(date +%s); timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench wall s: $(( $(date +%s) - start ))" > gpurun_out/bench_wall.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
   python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu > gpurun_out/bench_ncu_launch.log 2>&1
timeout 1500 ncu --set full --clock-control none --profile-from-start off -k regex:tc_ \
   -o gpurun_out/traffic -f python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu --profile > gpurun_out/bench_ncu_full.log 2>&1
python tools/ncu_traffic.py gpurun_out/traffic.ncu-rep gpurun_out/profile_cases.json gpurun_out/ncu_traffic.json >> gpurun_out/bench_ncu_full.log 2>&1
python tools/ncu_top.py gpurun_out/traffic.ncu-rep 10 > gpurun_out/traffic_top.txt 2>&1
sz=$(stat -c %s gpurun_out/traffic.ncu-rep); [ "$sz" -gt 40000000 ] && rm gpurun_out/traffic.ncu-rep
ls -la gpurun_out
