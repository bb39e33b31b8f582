#!/bin/bash
# One gpurun session collecting the round's evidence: parity tests, smoke, bench (both arms),
# ncu launch list, ncu --set full captures of every kernel of the path, all-config table.
# Usage (repo root, under gpurun): bash tools/gpu_run.sh <tag> [notests]
set -u
TAG=${1:-r01}
O=gpurun_out
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks_event_reasons.active --format=csv > $O/nvsmi_$TAG.txt 2>&1
timeout 300 python __graft_entry__.py smoke > $O/smoke_$TAG.log 2>&1
if [ "${2:-tests}" = "tests" ]; then
  timeout 1200 python -m pytest tests -q -m gpu -p no:randomly > $O/gpu_tests_$TAG.log 2>&1
fi
timeout 900 python bench.py > $O/bench_$TAG.json 2> $O/bench_$TAG.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > $O/bench_ref_$TAG.json 2> $O/bench_ref_$TAG.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $O/ncu_launch_bench_$TAG.log 2>&1
for K in msv_fast vit_reg pipe_long_msv pipe_long_vit; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 3 -c 1 \
    -o $O/${K}_$TAG -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > $O/ncu_full_${K}_$TAG.log 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:vit_cta -c 1 \
  -o $O/vit_cta_$TAG -f python tools/vit_one.py 2048 20000 > $O/ncu_full_vit_cta_$TAG.log 2>&1
timeout 900 python tools/configs_bench.py 1,2,3,4,5 > $O/configs_$TAG.jsonl 2> $O/configs_$TAG.err
echo "done $TAG"
