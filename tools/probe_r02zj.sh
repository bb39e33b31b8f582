#!/bin/bash
# Evidence for the branch-free MSV row loop (693fd01): ncu --set full + source counters of the
# config-3 MSV kernel, the bench-step launch list, the bench line with its configs leg.
set -u
TAG=${1:-r02zj}
O=gpurun_out
mkdir -p $O
B="python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-graph --no-configs --no-forward --batch 0"
timeout 900 python bench.py --no-cpu-baseline > $O/bench_$TAG.json 2> $O/bench_$TAG.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-graph --batch 0 --no-forward --no-configs \
  > $O/ncu_launch_bench_$TAG.log 2>&1
python tools/launch_summary.py $O/launches_$TAG.csv "bench config 3 step ($TAG)" > $O/launches_$TAG.md 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:msv_fast -s 3 -c 1 \
  -o $O/msv_fast_$TAG -f $B > $O/ncu_full_msv_fast_$TAG.log 2>&1
python tools/ncu_summary.py $O/msv_fast_$TAG.ncu-rep > $O/ncu_full_$TAG.md 2>&1
ncu -i $O/msv_fast_$TAG.ncu-rep --page source --csv --print-source sass > $O/src_msv_fast_$TAG.csv 2>/dev/null
mkdir -p /tmp/ncu_reps_$TAG
mv $O/*_$TAG.ncu-rep /tmp/ncu_reps_$TAG/ 2>/dev/null
echo "done $TAG"
