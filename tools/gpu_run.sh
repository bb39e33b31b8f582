#!/bin/bash
# One gpurun session: parity tests, bench, ncu launch list and a full ncu capture of the MSV kernel.
# Usage (from the repo root, under gpurun): bash tools/gpu_run.sh [tag] [tests|notests]
set -u
TAG=${1:-r01}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks_event_reasons.active --format=csv > gpurun_out/nvsmi_$TAG.txt 2>&1
python __graft_entry__.py smoke > gpurun_out/smoke_$TAG.log 2>&1
if [ "${2:-tests}" = "tests" ]; then
  timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/gpu_tests_$TAG.log 2>&1
fi
timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch_bench_$TAG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:msv_fast -s 3 -c 1 \
  -o gpurun_out/msv_$TAG -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_msv_$TAG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:vit_reg -s 3 -c 1 \
  -o gpurun_out/vit_$TAG -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_vit_$TAG.log 2>&1
echo "done $TAG"
