#!/bin/bash
# One gpurun session collecting the round's evidence: parity tests, smoke, bench (both arms),
# ncu launch list, ncu --set full captures of every kernel of the path (+ Forward and batch
# kernels), all-config table, Forward and batch throughput tables.
# Usage (repo root, under gpurun): bash tools/gpu_run.sh <tag> [notests]
set -u
TAG=${1:-r01}
O=gpurun_out
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks_event_reasons.active --format=csv > $O/nvsmi_$TAG.txt 2>&1
timeout 300 python __graft_entry__.py smoke > $O/smoke_$TAG.log 2>&1
if [ "${2:-tests}" = "tests" ]; then
  timeout 1500 python -m pytest tests -q -m gpu -p no:randomly > $O/gpu_tests_$TAG.log 2>&1
fi
timeout 900 python bench.py > $O/bench_$TAG.json 2> $O/bench_$TAG.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > $O/bench_ref_$TAG.json 2> $O/bench_ref_$TAG.err
B="python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-graph"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-graph --batch 0 --no-forward \
  > $O/ncu_launch_bench_$TAG.log 2>&1
for K in msv_fast vit_pair pipe_long_msv pipe_long_vp; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 3 -c 1 \
    -o $O/${K}_$TAG -f $B --batch 0 --no-forward > $O/ncu_full_${K}_$TAG.log 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fwd_kernel -c 1 \
  -o $O/fwd_kernel_$TAG -f python tools/fwd_bench.py 400 100000 1 > $O/ncu_full_fwd_$TAG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:msv_multi -c 1 \
  -o $O/msv_multi_$TAG -f $B --batch 64 --no-forward > $O/ncu_full_msv_multi_$TAG.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:vit_c -c 1 \
  -o $O/vit_cpair_$TAG -f python tools/vit_one.py 2048 20000 > $O/ncu_full_vit_cpair_$TAG.log 2>&1
timeout 900 python tools/configs_bench.py 1,2,3,4,5 > $O/configs_$TAG.jsonl 2> $O/configs_$TAG.err
timeout 300 python tools/fwd_bench.py > $O/fwd_bench_$TAG.jsonl 2>&1
timeout 600 python tools/batch_bench.py 64 > $O/batch_bench_$TAG.jsonl 2>&1
# summaries on the box (gpurun copies back at most 64 MiB): keep only the MSV report
python tools/ncu_summary.py $O/*_$TAG.ncu-rep > $O/ncu_full_$TAG.md 2>&1
python tools/launch_summary.py $O/launches_$TAG.csv "bench launch list ($TAG)" > $O/launches_$TAG.md 2>&1
mkdir -p /tmp/ncu_reps_$TAG
for f in $O/*_$TAG.ncu-rep; do case "$f" in *msv_fast_*) ;; *) mv "$f" /tmp/ncu_reps_$TAG/ ;; esac; done
echo "done $TAG"
